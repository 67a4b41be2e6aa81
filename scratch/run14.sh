mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -s -k "split_cone or one_adam or final_loss or deterministic or edge or full_size_c2 or device_init or search_group" 2>&1 | grep -v "^$" | tail -25) > gpurun_out/t14.log
for sc in 0 1; do (FELIX_SC=$sc timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag14.log 2>&1; done
(FELIX_SCW=2 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag14.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench14_c2.log 2>&1
(FELIX_SC=1 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench14_c5p1.log 2>&1
(FELIX_SC=1 FELIX_P=2 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench14_c5p2.log 2>&1
(FELIX_SC=1 timeout 400 python bench.py --steps 5 --config C3 --no-cpu-baseline --no-e2e) > gpurun_out/bench14_c3.log 2>&1
(FELIX_SC=1 timeout 400 python bench.py --steps 5 --config C4 --no-cpu-baseline --no-e2e) > gpurun_out/bench14_c4.log 2>&1
