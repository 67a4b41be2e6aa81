mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "scoring or score_fp64 or round_topk or history_topk" 2>&1 | tail -6) > gpurun_out/t23.log
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench23_c2.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench23_c5.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:score_layer_v2 -s 1 -c 1 -o gpurun_out/prof_score_v2b_c2 python tools/profile_search.py --steps 2 > gpurun_out/ncu23.log 2>&1
