mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests/test_gpu_parity.py -q -s -k "split_cone or one_adam or final_loss or deterministic or edge or full_size or device_init or search_group or multitask or modes or scoring" 2>&1 | grep -v "^$" | tail -30) > gpurun_out/t18.log
for sc in 0 1; do (FELIX_SC=$sc timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag18.log 2>&1; done
(FELIX_R=2 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag18.log 2>&1
(FELIX_SCW=2 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag18.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench18_c2.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench18_c5p1.log 2>&1
(FELIX_P=2 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench18_c5p2.log 2>&1
(FELIX_SC=1 timeout 400 python bench.py --steps 5 --config C3 --no-cpu-baseline --no-e2e) > gpurun_out/bench18_c3.log 2>&1
(FELIX_SC=1 timeout 400 python bench.py --steps 5 --config C4 --no-cpu-baseline --no-e2e) > gpurun_out/bench18_c4.log 2>&1
