"""Short C2 search for ncu captures: W warm-up searches then one search of S Adam steps + round/top-k."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import felix_inputs as fi  # noqa: E402
import paper_conf_asplos_zhaosam24_b200 as fx  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--steps", type=int, default=4)
ap.add_argument("--warmup", type=int, default=1)
ap.add_argument("--n", type=int, default=0)
a = ap.parse_args()
cfg = fi.config(a.config)
sp = cfg.spaces[0]
n = a.n or cfg.n_seeds
space = fx.Space(sp)
cm = fx.CostModel.from_weights(fi.make_mlp(cfg.mlp_dims))
y = torch.empty((sp.n_vars, n), device="cuda")
for _ in range(a.warmup + 1):
    space.search(cm, y, a.steps, rng_seed=cfg.rng_seed, init_from_y=False)
    space.round_topk(cm, y, cfg.topk)
torch.cuda.synchronize()
print("done", space.info)
