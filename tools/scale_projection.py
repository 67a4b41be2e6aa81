"""Projected multi-GPU scaling from one GPU: for N = 1, 2, 4, 8 build the shard plan every rank of an
N-GPU run would get (paper_conf_asplos_zhaosam24_b200/tasks.py), time the heaviest rank's
shards on this GPU exactly as that rank would run them (one felix_search_group over its shards, then
round / top-k per shard), and report

    value(N) = (candidate-steps of the whole job) / (max over ranks of the rank's time)

with the all-gather of the top-k records (a few KB) neglected.  The candidates / tasks are independent
(Eq. 4 is a sum of per-candidate terms; subgraphs are tuned independently), so a
rank's time does not depend on the other ranks: this is the curve an 8-GPU box would measure, minus
NVLink all-gather latency.

    python tools/scale_projection.py C4 [--steps 50] [--reps 3]      -> one JSON object
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import felix_inputs as fi  # noqa: E402
import paper_conf_asplos_zhaosam24_b200 as fx  # noqa: E402
from paper_conf_asplos_zhaosam24_b200 import tasks  # noqa: E402


def time_rank(cfg, shards, cm, T, k, reps):
    runner = tasks.TaskRunner(cfg.spaces, shards, cm)
    runner.run(T, k, rng_seed=cfg.rng_seed, lr=cfg.lr, lam=cfg.lam)          # warm-up (plans, graphs)
    torch.cuda.synchronize()
    best = float("inf")
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        runner.run(T, k, rng_seed=cfg.rng_seed, lr=cfg.lr, lam=cfg.lam)
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) * 1e-3)
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", choices=["C3", "C4"])
    ap.add_argument("--steps", type=int, default=0, help="Adam steps per search (default: the config's)")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--gpus", default="1,2,4,8")
    args = ap.parse_args()
    cfg = fi.config(args.config)
    T = args.steps or cfg.n_steps
    mlp = fi.make_mlp(cfg.mlp_dims)
    cm = fx.CostModel.from_weights(mlp)
    mode = tasks.config_mode(cfg.name)
    flops = cm.mlp_flops_per_candidate_step()
    costs = [tasks.est_cost(cfg.n_seeds, T, flops, sp.nodes.shape[0]) for sp in cfg.spaces]
    total = len(cfg.spaces) * cfg.n_seeds * T
    out = {"config": cfg.name, "mode": mode, "n_tasks": len(cfg.spaces), "n_seeds_per_task": cfg.n_seeds,
           "n_steps": T, "gpu": torch.cuda.get_device_name(), "points": []}
    v1 = None
    for N in [int(x) for x in args.gpus.split(",")]:
        plan = tasks.plan(len(cfg.spaces), cfg.n_seeds, N, mode, costs)
        # the heaviest rank by the planner's estimate (seed mode: all ranks alike, the first is the largest)
        est = [sum(costs[s.task] * s.n / cfg.n_seeds for s in sh) for sh in plan]
        r = max(range(N), key=lambda q: (est[q], -q))
        t0 = time.perf_counter()
        t = time_rank(cfg, plan[r], cm, T, cfg.topk, args.reps)
        value = total / t
        if v1 is None:
            v1 = value
        out["points"].append({"n_gpus": N, "heaviest_rank": r, "rank_shards": len(plan[r]),
                              "rank_rows": sum(s.n for s in plan[r]), "rank_time_s": t,
                              "value_cand_steps_per_s": value, "efficiency_vs_1": value / (N * v1),
                              "planner_makespan_eff": (sum(costs) / N) / max(est), "wall_s": time.perf_counter() - t0})
        print(json.dumps(out["points"][-1]), file=sys.stderr, flush=True)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
