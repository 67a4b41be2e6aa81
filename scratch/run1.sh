mkdir -p gpurun_out
python __graft_entry__.py
(./scratch/chain_trace 4096 128 64 1; ./scratch/chain_trace 4096 128 64 4) > gpurun_out/chain_trace.log 2>&1
(python tools/dag_timing.py C2; FELIX_NEWTON=1 python tools/dag_timing.py C2) > gpurun_out/dag_newton.log 2>&1
(FELIX_NEWTON=1 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or every_c3" 2>&1 | tail -5) > gpurun_out/newton_tests.log
(FELIX_NEWTON=1 python bench.py --steps 10 --no-cpu-baseline --no-e2e; python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench_newton.log 2>&1
