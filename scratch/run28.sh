mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -6) > gpurun_out/t28.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t28.log
(timeout 400 python bench.py) > gpurun_out/bench28_c2.log 2>&1
(timeout 300 python bench.py --config C5 --no-cpu-baseline) > gpurun_out/bench28_c5.log 2>&1
(timeout 400 python bench.py --config C3 --no-cpu-baseline) > gpurun_out/bench28_c3.log 2>&1
(timeout 400 python bench.py --config C4 --no-cpu-baseline) > gpurun_out/bench28_c4.log 2>&1
