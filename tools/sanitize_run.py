"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck): search + eval + search-path eval +
round/top-k on a config at n candidates with a forced MLP mode.  Usage:
python tools/sanitize_run.py <C1|C2|composite8> <n> <auto|chain|tile> [tile_cta_group]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import felix_inputs as fi  # noqa: E402
import paper_conf_asplos_zhaosam24_b200 as fx  # noqa: E402

name, n, mode = sys.argv[1], int(sys.argv[2]), sys.argv[3]
cg = int(sys.argv[4]) if len(sys.argv) > 4 else 1
knobs = {"mlp": {"auto": -1, "chain": 1, "tile": 0}[mode], "tile_cta_group": cg}
fx.tune(**knobs)
if name == "composite8":
    sp, mlp = fi.composite_space(8), fi.make_mlp(fi.DEFAULT_MLP)
else:
    cfg = fi.config(name)
    sp, mlp = cfg.spaces[0], fi.make_mlp(cfg.mlp_dims)
space = fx.Space(sp)
cm = fx.CostModel.from_weights(mlp)
y = torch.from_numpy(fi.make_y0(sp, n, seed=3)).cuda()
if name != "composite8":
    space.eval(cm, y)
    space.eval_search_path(cm, y)
    space.search(cm, y, 3, init_from_y=True)
idx, sc, sched = space.round_topk(cm, y, 16)
torch.cuda.synchronize()
print("ok", sys.argv[1:], len(idx))
