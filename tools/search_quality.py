"""Search-quality diagnostic (a Felix-only analogue of Fig. 8):
best and 64th-best predicted score of the distinct valid schedules visited vs. schedules searched.

Felix: a search of s Adam steps is exactly the first s steps of a longer search (deterministic, Adam
state starts fresh each call), so history_topk(64) after s steps gives the curves at s * n_seeds
schedules searched (Alg. 1's varValuesHistory, l.13/17/20).  Reference: the same number of random
valid starting points (the rejection sampler), rounded and scored the same way
(P:L1141's random-sampling comparison).  Ansor's evolutionary search is out of scope.

    python tools/search_quality.py [--config C2] [--out profiles/r01/search_quality_c2.json]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import felix_inputs as fi  # noqa: E402
import paper_conf_asplos_zhaosam24_b200 as fx  # noqa: E402


def curves(space, cm, n, steps, rng_seed, lr, lam, kq=64):
    y = torch.empty((space.n_vars, n), device="cuda")
    out = []
    for s in steps:
        space.search(cm, y, s, lr=lr, lam=lam, rng_seed=rng_seed, init_from_y=False, history=True)
        _, st, sc, _, nu = space.history_topk(cm, kq)
        out.append({"steps": s, "searched": s * n, "distinct": nu, "best": float(sc[0]) if len(sc) else None,
                    f"top{kq}": float(sc[kq - 1]) if len(sc) >= kq else None,
                    "best_first_step": int(st[0]) if len(st) else None})
    return out


def random_curves(space, cm, n, steps, rng_seed, kq=64):
    out = []
    for s in steps:
        m = s * n
        yr = space.init_sample(m, rng_seed + 1)
        _, sc, _ = space.round_topk(cm, yr, kq)
        out.append({"searched": m, "best": float(sc[0]) if len(sc) else None,
                    f"top{kq}": float(sc[kq - 1]) if len(sc) >= kq else None})
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    cfg = fi.config(a.config)
    sp = cfg.spaces[0]
    space = fx.Space(sp)
    cm = fx.CostModel.from_weights(fi.make_mlp(cfg.mlp_dims))
    steps = [s for s in (1, 2, 5, 10, 20, 50, 100, 200) if s <= cfg.n_steps]
    res = {"workload": f"{cfg.name}: {sp.name}, {cfg.n_seeds} seeds, MLP {list(cfg.mlp_dims)} (random-init weights)",
           "felix": curves(space, cm, cfg.n_seeds, steps, cfg.rng_seed, cfg.lr, cfg.lam),
           "random": random_curves(space, cm, cfg.n_seeds, [s for s in steps if s <= 50], cfg.rng_seed)}
    line = json.dumps(res)
    if a.out:
        with open(a.out, "w") as f:
            f.write(line + "\n")
    print(line)


if __name__ == "__main__":
    main()
