"""Per-kernel-class device time of a short search (profiling events); env P = cone width (felix_tune)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import felix_inputs as fi
import paper_conf_asplos_zhaosam24_b200 as fx
if os.environ.get("P"):
    fx.tune(cone_width=int(os.environ["P"]))
cfg = fi.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
n = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.n_seeds
sp = cfg.spaces[0]
space = fx.Space(sp)
cm = fx.CostModel.from_weights(fi.make_mlp(cfg.mlp_dims))
y = torch.empty((sp.n_vars, n), device="cuda")
space.search(cm, y, 20, rng_seed=cfg.rng_seed, init_from_y=False)
torch.cuda.synchronize()
space.profile_reset(); space.profile(True)
space.search(cm, y, 50, rng_seed=cfg.rng_seed, init_from_y=False)
torch.cuda.synchronize()
space.profile(False)
pr = space.profile_read()
print(json.dumps({"P": os.environ.get("P", "auto"), "n": n, "regs": [space.info.regs_fwd, space.info.regs_rev],
                  **{k: round(v[0] / max(v[1], 1) * 1e3, 2) for k, v in pr.items()}}))
