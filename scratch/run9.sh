mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -5) > gpurun_out/t9.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t9.log
(python tools/dag_timing.py C2) > gpurun_out/dag9.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench9.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"felix_init|score_layer|topk|round_|felix_hard" -c 40 --csv --log-file gpurun_out/finish9.csv python tools/profile_search.py --steps 2 > /dev/null 2>&1
