mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -s -k "split_cone" 2>&1 | grep -v "^$" | tail -25) > gpurun_out/t15.log
for p in 4 8; do for w in 2 4; do (FELIX_SCF=1 FELIX_P=$p FELIX_SCW=$w timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag15.log 2>&1; done; done
(FELIX_SCF=1 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench15_c2.log 2>&1
(FELIX_SCF=1 FELIX_SC=1 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench15_c5p1.log 2>&1
(FELIX_SCF=1 FELIX_SC=1 FELIX_P=2 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench15_c5p2.log 2>&1
