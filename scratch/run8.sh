mkdir -p gpurun_out
python __graft_entry__.py
(timeout 60 ./scratch/chain_trace 4096 128 64 1 1 0; timeout 60 ./scratch/chain_trace 4096 128 64 1 1 1) > gpurun_out/chain_trace8.log 2>&1
(python tools/dag_timing.py C2; FELIX_CHAIN_REUSE=0 python tools/dag_timing.py C2; python tools/dag_timing.py C2 8192; FELIX_CHAIN_REUSE=0 python tools/dag_timing.py C2 8192) > gpurun_out/reuse8.log 2>&1
(timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or full_size or history or multitask or deterministic or subgraph or edge" 2>&1 | tail -5) > gpurun_out/t8.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench8.log 2>&1
