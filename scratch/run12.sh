mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -s -k "split_cone or one_adam or final_loss or deterministic or edge or full_size_c2 or device_init or search_group or multitask or subgraph" 2>&1 | grep -v "^$" | tail -25) > gpurun_out/t12.log
for sc in 0 1; do for p in 4 8; do (FELIX_SC=$sc FELIX_P=$p timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag12.log 2>&1; done; done
for w in 2 3 8; do (FELIX_SC=1 FELIX_SCW=$w timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag12.log 2>&1; done
(FELIX_SC=0 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench12_sc0.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench12_sc1.log 2>&1
(FELIX_P=8 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench12_sc1p8.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench12_c5.log 2>&1
(FELIX_SC=1 FELIX_P=2 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench12_c5sc.log 2>&1
