"""Phase timing of the generated DAG kernels inside the graph-replayed search (felix_tune trace=1):
per-block %globaltimer stamps of the last Adam step's felix_fwd_adam (start, after griddepcontrol.wait,
after the Adam prologue, after the cone compute, end) and felix_rev_sc (start, after wait, after
compute, end), relative to the first forward block's start.  Usage: python tools/dag_trace.py [C2|C5] [n]"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import felix_inputs as fi
import paper_conf_asplos_zhaosam24_b200 as fx

fx.tune(trace=1)
cfg = fi.config(sys.argv[1] if len(sys.argv) > 1 else "C2")
n = int(sys.argv[2]) if len(sys.argv) > 2 else cfg.n_seeds
sp = cfg.spaces[0]
space = fx.Space(sp)
cm = fx.CostModel.from_weights(fi.make_mlp(cfg.mlp_dims))
y = torch.empty((sp.n_vars, n), device="cuda")
for _ in range(3):
    space.search(cm, y, 20, rng_seed=cfg.rng_seed, init_from_y=False)
torch.cuda.synchronize()
tr, wt = space.debug_trace(warps=True)
tr, wt = tr.astype(np.int64), wt.astype(np.int64)
f = tr[0][tr[0, :, 0] > 0]
r = tr[1][tr[1, :, 0] > 0]
t0 = f[:, 0].min()
q = lambda a: [round(float(np.min(a)) / 1e3, 2), round(float(np.median(a)) / 1e3, 2), round(float(np.max(a)) / 1e3, 2)]
out = {"config": cfg.name, "n": n, "fwd_blocks": len(f), "rev_blocks": len(r),
       "fwd_us_rel_min_med_max": {"start": q(f[:, 0] - t0), "after_wait": q(f[:, 1] - t0), "after_adam": q(f[:, 2] - t0),
                                  "after_compute": q(f[:, 3] - t0), "end": q(f[:, 4] - t0)},
       "fwd_adam_parts_us_med": {"loads_to_sync1": q(f[:, 5] - f[:, 1])[1], "loss_ballot_sync2": q(f[:, 6] - f[:, 5])[1],
                                 "adam_exp": q(f[:, 7] - f[:, 6])[1], "zero_phi_sync3": q(f[:, 2] - f[:, 7])[1]},
       "fwd_phase_us_med": {"wait": q(f[:, 1] - f[:, 0])[1], "adam_prologue": q(f[:, 2] - f[:, 1])[1],
                            "cones": q(f[:, 3] - f[:, 2])[1], "phi_store": q(f[:, 4] - f[:, 3])[1]},
       "rev_us_rel_min_med_max": {"start": q(r[:, 0] - t0), "after_wait": q(r[:, 1] - t0), "after_compute": q(r[:, 2] - t0),
                                  "end": q(r[:, 3] - t0)},
       "rev_phase_us_med": {"wait": q(r[:, 1] - r[:, 0])[1], "cone": q(r[:, 2] - r[:, 1])[1], "store": q(r[:, 3] - r[:, 2])[1]},
       "span_us": round((max(f[:, 4].max(), r[:, 3].max()) - t0) / 1e3, 2)}
# cone imbalance of the forward: per warp (cone q = warp % P of its replica), cone end - after-Adam stamp
nb = len(f)
w = wt[:nb]
rel = np.where(w > 0, w - tr[0, :nb, 2][:, None], 0)
nw = int((w[0] > 0).sum())
out["fwd_cone_end_us_med_per_warp"] = [round(float(np.median(rel[:, k])) / 1e3, 2) for k in range(nw)]
# reverse: per cone q (block % P, P = argv[3], default 4), median of (after compute - after wait)
P = int(sys.argv[3]) if len(sys.argv) > 3 else 4
rb = np.nonzero(tr[1, :, 0] > 0)[0]
out["rev_cone_us_med_per_q"] = [round(float(np.median((tr[1, rb[rb % P == q], 2] - tr[1, rb[rb % P == q], 1]))) / 1e3, 2)
                                for q in range(P)]
print(json.dumps(out))
