mkdir -p gpurun_out
python __graft_entry__.py
(timeout 1200 python -m pytest tests/test_gpu_parity.py -q -s -k "modes or scoring or eval_parity or score_fp64 or round_topk or tile_mlp or split_cone" 2>&1 | grep -v "^$" | tail -30) > gpurun_out/t17.log
for ex in 0 1; do (FELIX_CHAIN_EXACT=$ex timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag17.log 2>&1; done
(FELIX_R=2 timeout 120 python tools/dag_timing.py C2) >> gpurun_out/dag17.log 2>&1
(FELIX_SCORE=1 timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench17_c2_score1.log 2>&1
(timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e) > gpurun_out/bench17_c2.log 2>&1
(timeout 300 python bench.py --steps 5 --config C5 --no-cpu-baseline --no-e2e) > gpurun_out/bench17_c5.log 2>&1
