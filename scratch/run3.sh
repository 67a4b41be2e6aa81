mkdir -p gpurun_out
python __graft_entry__.py
(timeout 60 ./scratch/chain_trace 4096 128 64 4 0; timeout 60 ./scratch/chain_trace 4096 128 64 1 1) > gpurun_out/chain_trace3.log 2>&1
(timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or tile or deterministic or full_size" 2>&1 | tail -5) > gpurun_out/t3.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e; timeout 300 python bench.py --config C5 --steps 3 --no-cpu-baseline --no-e2e) > gpurun_out/bench3.log 2>&1
