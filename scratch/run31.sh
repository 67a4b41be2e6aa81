mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1250 python -m pytest tests -q -m gpu -x 2>&1 | tail -6) > gpurun_out/t31.log
(timeout 60 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t31.log
