mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -5) > gpurun_out/t6.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t6.log
timeout 400 python bench.py > gpurun_out/bench_c2_v9.json 2> gpurun_out/bench_c2_v9.err
timeout 300 python bench.py --config C5 --steps 5 > gpurun_out/bench_c5_v9.json 2> gpurun_out/bench_c5_v9.err
