mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1200 python -m pytest tests/test_gpu_parity.py -q -k "split_cone or one_adam or final_loss or search_group or multitask or scoring or deterministic" 2>&1 | tail -6) > gpurun_out/t24.log
for sc in 0 1; do (FELIX_SC=$sc timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag24.log 2>&1; done
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench24_c2.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench24_c5.log 2>&1
