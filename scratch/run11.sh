mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1800 python -m pytest tests -x -q -m gpu 2>&1 | tail -8) > gpurun_out/t11.log
(timeout 120 python __graft_entry__.py smoke 2>&1 | tail -2) >> gpurun_out/t11.log
(timeout 400 python bench.py) > gpurun_out/bench11.log 2>&1
(timeout 400 python bench.py --impl reference --steps 3 --warmup 3) > gpurun_out/bench11_ref.log 2>&1
(timeout 400 python bench.py --config C5 --no-cpu-baseline) > gpurun_out/bench11_c5.log 2>&1
(timeout 400 python bench.py --config C3 --no-cpu-baseline) > gpurun_out/bench11_c3.log 2>&1
(timeout 400 python bench.py --config C4 --no-cpu-baseline) > gpurun_out/bench11_c4.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches11.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/launches11_bench.log 2>&1
