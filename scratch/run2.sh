mkdir -p gpurun_out
python __graft_entry__.py
(timeout 60 ./scratch/chain_trace 4096 128 64 1 0; timeout 60 ./scratch/chain_trace 4096 128 64 1 1; timeout 60 ./scratch/chain_trace 8192 128 64 1 1) > gpurun_out/chain_trace2.log 2>&1
(FELIX_CHAIN_CS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or deterministic or subgraph or full_size or multitask or history" 2>&1 | tail -5) > gpurun_out/flags_tests.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e; FELIX_CHAIN_CS=1 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e; FELIX_CHAIN_CS=1 FELIX_CHAIN_FLAGS=0 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e; timeout 300 python bench.py --steps 5 --seeds 8192 --no-cpu-baseline --no-e2e; FELIX_CHAIN_FLAGS=0 timeout 300 python bench.py --steps 5 --seeds 8192 --no-cpu-baseline --no-e2e) > gpurun_out/bench_flags.log 2>&1
