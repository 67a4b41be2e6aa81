mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -6) > gpurun_out/t22.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t22.log
(timeout 400 python bench.py) > gpurun_out/bench22_c2.log 2>&1
(timeout 400 python bench.py --impl reference --steps 3 --warmup 3) > gpurun_out/bench22_ref.log 2>&1
(timeout 300 python bench.py --config C5 --no-cpu-baseline) > gpurun_out/bench22_c5.log 2>&1
(timeout 400 python bench.py --config C3 --no-cpu-baseline) > gpurun_out/bench22_c3.log 2>&1
(timeout 400 python bench.py --config C4 --no-cpu-baseline) > gpurun_out/bench22_c4.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches22.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/launches22_bench.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:mlp_chain -s 5 -c 1 -o gpurun_out/prof_chain_c2_v14 python tools/profile_search.py --steps 4 > gpurun_out/ncu22a.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:mlp_tile -s 1 -c 1 -o gpurun_out/prof_tile_c5_v14 python tools/profile_search.py --config C5 --n 131072 --steps 2 > gpurun_out/ncu22b.log 2>&1
