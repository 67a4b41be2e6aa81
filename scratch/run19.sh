mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -8) > gpurun_out/t19.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t19.log
(timeout 400 python bench.py) > gpurun_out/bench19_c2.log 2>&1
(timeout 300 python bench.py --config C5 --no-cpu-baseline) > gpurun_out/bench19_c5.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches19.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/launches19_bench.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:felix_rev_sc -s 3 -c 1 -o gpurun_out/prof_rev_sc_c2 python tools/profile_search.py --steps 4 > gpurun_out/ncu19a.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:felix_fwd_adam -s 3 -c 1 -o gpurun_out/prof_fwd_adam_c2 python tools/profile_search.py --steps 4 > gpurun_out/ncu19b.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:score_layer_v2 -s 1 -c 1 -o gpurun_out/prof_score_v2_c2 python tools/profile_search.py --steps 2 > gpurun_out/ncu19c.log 2>&1
