mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "scoring or score_fp64 or round_topk or history_topk or multitask" 2>&1 | tail -4) > gpurun_out/t26.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench26_c2.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench26_c5.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"score" -c 12 --csv --log-file gpurun_out/score26.csv python tools/profile_search.py --steps 2 > /dev/null 2>&1
