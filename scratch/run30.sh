mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "split_cone or one_adam or final_loss or search_group or deterministic" 2>&1 | tail -4) > gpurun_out/t30.log
(timeout 120 python tools/dag_timing.py C2) > gpurun_out/dag30.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench30_c2.log 2>&1
