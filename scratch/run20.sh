mkdir -p gpurun_out
python __graft_entry__.py
(timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "modes or tile_mlp or search_group or full_size_c5" 2>&1 | tail -6) > gpurun_out/t20.log
(FELIX_MASK_EXACT=0 timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench20_c5_ex0.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench20_c5_ex1.log 2>&1
(FELIX_MASK_EXACT=0 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench20_c2_ex0.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench20_c2_ex1.log 2>&1
