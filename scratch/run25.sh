mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -6) > gpurun_out/t25.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t25.log
(timeout 400 python bench.py) > gpurun_out/bench25_c2.log 2>&1
(timeout 400 python bench.py --impl reference --steps 3 --warmup 3) > gpurun_out/bench25_ref.log 2>&1
(timeout 300 python bench.py --config C5 --no-cpu-baseline) > gpurun_out/bench25_c5.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches25.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/launches25_bench.log 2>&1
