mkdir -p gpurun_out
python __graft_entry__.py
(timeout 60 ./scratch/chain_trace 4096 128 64 1 1 1) > gpurun_out/chain_trace10.log 2>&1
(timeout 1500 python -m pytest tests/test_gpu_parity.py -x -q -k "eval_parity or one_adam or modes or score or topk or history or full_size or multitask or deterministic or subgraph or edge or tile" 2>&1 | tail -5) > gpurun_out/t10.log
(python tools/dag_timing.py C2; python tools/dag_timing.py C2 8192) > gpurun_out/dag10.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench10.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"score_layer" -c 8 --csv --log-file gpurun_out/finish10.csv python tools/profile_search.py --steps 2 > /dev/null 2>&1
