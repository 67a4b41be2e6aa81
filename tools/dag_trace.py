"""Phase timing of the generated DAG kernels (felix_tune trace): one graph-replayed Adam step's fwd/rev blocks."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import felix_inputs as fi
import paper_conf_asplos_zhaosam24_b200 as fx
fx.tune(trace=1)
cfg = fi.config("C2")
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
sp = cfg.spaces[0]
space = fx.Space(sp)
cm = fx.CostModel.from_weights(fi.make_mlp(cfg.mlp_dims))
y = torch.empty((sp.n_vars, n), device="cuda")
space.search(cm, y, 10, rng_seed=cfg.rng_seed, init_from_y=False)
torch.cuda.synchronize()
tr = space.debug_trace().astype(np.int64)
nb = (n + 31) // 32
T0 = tr[0, :nb, 1].min()          # common origin: the forward kernel's first block past griddepcontrol.wait
for k, name in enumerate(["fwd", "rev"]):
    t = tr[k, :nb]
    t0 = T0
    rel = (t - t0) / 1e3
    print(f"{name} P={os.environ.get('P','auto')} n={n}: start {rel[:,0].min():.2f}..{rel[:,0].max():.2f} | after-wait {rel[:,1].min():.2f}..{rel[:,1].max():.2f} | "
          f"after-compute {rel[:,2].min():.2f}/{np.median(rel[:,2]):.2f}/{rel[:,2].max():.2f} | end {rel[:,3].min():.2f}/{np.median(rel[:,3]):.2f}/{rel[:,3].max():.2f} us")
