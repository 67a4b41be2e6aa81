"""C2 subgraph with its three symbolic programs (Eq. 3): concurrent (one stream per program) vs
sequential search + top-k, CUDA-event timed, warm.  Prints one JSON line (experiment, not the headline)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import felix_inputs as fi  # noqa: E402
import paper_conf_asplos_zhaosam24_b200 as fx  # noqa: E402
from paper_conf_asplos_zhaosam24_b200.subgraph import SubgraphSearch  # noqa: E402

n, T, k, reps = 4096, 200, 16, 5
cm = fx.CostModel.from_weights(fi.make_mlp(fi.DEFAULT_MLP))
drv = SubgraphSearch(fi.c2_sketches(), cm)
out = {}
for conc in (True, False):
    for _ in range(2):
        drv.run(n, T, k, rng_seed=5, concurrent=conc)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        best = drv.run(n, T, k, rng_seed=5, concurrent=conc)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    out["concurrent" if conc else "sequential"] = {"ms_per_subgraph": ms, "cand_steps_per_s": 3 * n * T / (ms * 1e-3)}
out["best"] = {"sketch": best[0].sketch, "idx": best[0].idx, "score": best[0].score}
out["workload"] = "C2 subgraph, 3 symbolic programs x 4096 seeds x 200 steps + per-program round/top-k + merge"
print(json.dumps(out))
