mkdir -p gpurun_out
python __graft_entry__.py
(python tools/dag_timing.py C2; FELIX_CPB=0 python tools/dag_timing.py C2; FELIX_P=4 python tools/dag_timing.py C2; python tools/dag_timing.py C2 32768; FELIX_P=8 python tools/dag_timing.py C2 32768; FELIX_CPB=0 python tools/dag_timing.py C2 32768) > gpurun_out/cpb7.log 2>&1
(timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or full_size or history or multitask or edge or deterministic or every_c3" 2>&1 | tail -5) > gpurun_out/t7.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench7.log 2>&1
