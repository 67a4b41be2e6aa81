"""Multi-task workloads across ranks (BASELINE configs C3 and C4).

A DNN is partitioned into subgraphs (tasks) that are tuned independently (PAPER.md L391-394,
L513-515), and inside one task Eq. 4 is a sum of per-seed terms with an elementwise Adam update
(P:L842-857, L884-885), so work shards two ways with no per-step communication:

* ``"task"`` (C3, full ResNet-50): whole tasks go to ranks by LPT (longest processing time first)
  on the estimated cost ``n_seeds * n_steps * (mlp_flops + DAG_WEIGHT * n_nodes)``: tasks in
  decreasing cost (ties: lower task index first) each go to the rank with the least assigned cost
  (ties: lower rank).
* ``"hybrid"`` (C3 default): LPT alone caps the efficiency when tasks are few per rank (21 nearly
  equal ResNet-50 tasks on 8 ranks: makespan 3 tasks against a mean of 2.625, 0.875).  Every task is
  cut into ``ceil(cost / target)`` equal seed chunks (target = total / (world * CHUNKS_PER_RANK)), the
  chunks go to ranks by LPT, and the chunks of one task a rank received become ONE contiguous seed
  range of that task (ranges allotted in rank order), so every rank holds at most one shard per task
  and global seed indices still partition ``[0, n_seeds)``.
* ``"seeds"`` (C4, BERT-base): every task's seeds are cut into ``world`` contiguous ranges,
  rank r searching ``[r*n/world, (r+1)*n/world)`` with ``index_base`` = the range start, so global
  candidate indices (and therefore the top-k tie-breaks) do not depend on the rank count.

On a rank, all its shards are searched as one group (``felix_search_group``): every Adam step runs each
task's DAG kernels on its own stream and ONE tensor-core MLP pass over the candidates of all tasks (the
tasks share the cost model), so the small per-task populations fill the GPU like one large population.

The only exchange is at the end: one all-gather of every task's local top-k records, merged per
task exactly as ``dist.merge_records`` does for one task (dedup by schedule keeping the smallest
global index, order by (score desc, index asc)).  The merged per-task lists equal the single-process
top-k of every task for any world size.

The planner is plain host logic (no libfelix needed) so it is unit-tested on CPU; the runner calls
the C ABI only (``search_group`` / ``Space.search`` / ``Space.round_topk``).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Dict, List, Sequence, Tuple

import numpy as np

# DAG nodes are a few FP64 ops each, forward + reverse: ~10 FLOP-equivalents per node
# and candidate-step, against 4 * sum d_l d_{l+1} MLP FLOPs.  Only the ranking of tasks matters.
DAG_WEIGHT = 10.0


@dataclass(frozen=True)
class Shard:
    task: int            # index into the config's task list
    seed_lo: int         # first global seed index of this shard (= index_base)
    n: int               # seeds in this shard


def est_cost(n_seeds: int, n_steps: int, mlp_flops: int, n_nodes: int) -> float:
    """Estimated cost of one task's search (n_seeds * (4*MACs + c*n_nodes) per step)."""
    return float(n_seeds) * n_steps * (mlp_flops + DAG_WEIGHT * n_nodes)


def lpt_assign(costs: Sequence[float], world: int) -> List[List[int]]:
    """Longest-processing-time-first: deterministic, every task exactly once, makespan <= 4/3 OPT."""
    if world < 1:
        raise ValueError("world must be >= 1")
    order = sorted(range(len(costs)), key=lambda t: (-costs[t], t))
    load = [0.0] * world
    out: List[List[int]] = [[] for _ in range(world)]
    for t in order:
        r = min(range(world), key=lambda i: (load[i], i))
        out[r].append(t)
        load[r] += costs[t]
    for r in range(world):
        out[r].sort()
    return out


CHUNKS_PER_RANK = 8


def hybrid_assign(costs: Sequence[float], n_seeds: int, world: int,
                  chunks_per_rank: int = CHUNKS_PER_RANK) -> List[List[Shard]]:
    """Seed-split LPT (mode "hybrid"): returns per-rank shard lists, at most one shard per (rank, task)."""
    if world < 1:
        raise ValueError("world must be >= 1")
    total = float(sum(costs))
    target = total / (world * chunks_per_rank) if total > 0 else 1.0
    n_chunks = [max(1, min(n_seeds, int(np.ceil(c / target - 1e-9)))) for c in costs]
    # chunk (t, i) covers seed_range(n_seeds, i, n_chunks[t]); cost proportional to its seeds
    chunks = [(t, i) for t in range(len(costs)) for i in range(n_chunks[t])]
    ccost = {(t, i): costs[t] * (seed_range(n_seeds, i, n_chunks[t])[1] - seed_range(n_seeds, i, n_chunks[t])[0]) / n_seeds
             for (t, i) in chunks}
    order = sorted(chunks, key=lambda ti: (-ccost[ti], ti))
    load = [0.0] * world
    cnt = [[0] * world for _ in costs]          # chunks of task t on rank r
    for ti in order:
        r = min(range(world), key=lambda q: (load[q], q))
        load[r] += ccost[ti]
        cnt[ti[0]][r] += 1
    out: List[List[Shard]] = [[] for _ in range(world)]
    for t in range(len(costs)):
        first = 0                               # next unassigned chunk of task t, ranks in order
        for r in range(world):
            if cnt[t][r] == 0:
                continue
            lo = seed_range(n_seeds, first, n_chunks[t])[0]
            hi = seed_range(n_seeds, first + cnt[t][r] - 1, n_chunks[t])[1]
            out[r].append(Shard(t, lo, hi - lo))
            first += cnt[t][r]
    return out


def makespan(shards: List[List[Shard]], costs: Sequence[float], n_seeds: int) -> float:
    """Largest per-rank estimated cost of a plan (cost of a shard = task cost x its share of the seeds)."""
    return max((sum(costs[s.task] * s.n / n_seeds for s in sh) for sh in shards), default=0.0)


def seed_range(n: int, rank: int, world: int) -> Tuple[int, int]:
    """Contiguous [lo, hi) seed range of `rank` (sizes differ by at most one)."""
    return rank * n // world, (rank + 1) * n // world


def plan(n_tasks: int, n_seeds: int, world: int, mode: str, costs: Sequence[float] = ()) -> List[List[Shard]]:
    """Per-rank shard lists for `n_tasks` tasks of `n_seeds` seeds each."""
    if mode == "task":
        if len(costs) != n_tasks:
            raise ValueError("task mode needs one cost per task")
        return [[Shard(t, 0, n_seeds) for t in ts] for ts in lpt_assign(costs, world)]
    if mode == "hybrid":
        if len(costs) != n_tasks:
            raise ValueError("hybrid mode needs one cost per task")
        return hybrid_assign(costs, n_seeds, world)
    if mode == "seeds":
        out = []
        for r in range(world):
            lo, hi = seed_range(n_seeds, r, world)
            out.append([Shard(t, lo, hi - lo) for t in range(n_tasks) if hi > lo])
        return out
    raise ValueError(f"unknown shard mode {mode!r}")


def config_mode(name: str) -> str:
    """C3 shards by subgraph with seed-split LPT (hybrid), C4 shards every task's seeds."""
    return {"C3": "hybrid", "MBV2": "hybrid", "C4": "seeds"}.get(name, "seeds")


# ----------------------------------------------------------------------------- top-k records
def pack_task_records(per_task: Dict[int, Tuple[np.ndarray, np.ndarray, np.ndarray]], n_tasks: int, k: int,
                      max_vars: int) -> np.ndarray:
    """[n_tasks * k, 2 + max_vars] float64 rows (idx, score, sched...); rows of tasks this rank did not
    run, and missing rows, have idx = -1.  Indices, scores (FP64) and factors are exact in float64."""
    out = np.zeros((n_tasks * k, 2 + max_vars), dtype=np.float64)
    out[:, 0] = -1
    for t, (idx, sc, sched) in per_task.items():
        m = len(idx)
        rows = out[t * k:t * k + m]
        rows[:, 0] = idx
        rows[:, 1] = sc
        rows[:, 2:2 + sched.shape[1]] = sched
    return out


def merge_task_records(gathered: np.ndarray, n_tasks: int, k: int, n_vars: Sequence[int]):
    """gathered: [world * n_tasks * k, 2 + max_vars] (rank-major).  Per task: dedup + order as
    dist.merge_records; returns {task: (idx, score, sched[:, :n_vars[task]])}."""
    world = gathered.shape[0] // (n_tasks * k)
    g = gathered.reshape(world, n_tasks, k, -1)
    out = {}
    from . import merge_topk
    for t in range(n_tasks):
        rows = g[:, t].reshape(world * k, -1)
        out[t] = merge_topk(rows[:, 0].astype(np.int64), rows[:, 1], rows[:, 2:2 + n_vars[t]].astype(np.int32), k)
    return out


def allgather_task_topk(per_task, n_tasks: int, k: int, n_vars: Sequence[int], group=None, device=None):
    """All-gather every rank's per-task top-k records (NCCL on GPUs, gloo on CPU) and merge per task."""
    import torch
    import torch.distributed as dist
    rec = torch.from_numpy(pack_task_records(per_task, n_tasks, k, max(n_vars)))
    if device is not None:
        rec = rec.to(device)
    world = dist.get_world_size(group)
    out = torch.empty((world * rec.shape[0], rec.shape[1]), dtype=torch.float64, device=rec.device)
    dist.all_gather_into_tensor(out, rec, group=group)
    return merge_task_records(out.cpu().numpy(), n_tasks, k, n_vars)


# ----------------------------------------------------------------------------- runner (C ABI only)
class TaskRunner:
    """One rank's shards of a multi-task workload: felix_search_group over all shards (or felix_search of
    every shard on its own CUDA stream), then felix_round_topk per shard."""

    def __init__(self, spaces, shards: Sequence[Shard], cm, device: int = 0):
        from . import Space
        self.shards = list(shards)
        self.cm = cm
        self.device = device
        self.spaces = {s.task: Space(spaces[s.task], device=device) for s in self.shards}

    def run(self, n_steps: int, k: int, *, rng_seed: int, lr: float = 0.05, lam: float = 1.0,
            y0: Dict[int, object] = None, loss_out: Dict[int, object] = None, concurrent: bool = True,
            batched: bool = True):
        """Search every shard (device init, or from y0[task] if given: a device [n_vars, n] tensor
        that is overwritten), then round / top-k.  Returns {task: (idx, score, sched)}.
        batched: one felix_search_group over all shards (each Adam step: every task's DAG kernels on
        its own stream, ONE tensor-core MLP pass over the candidates of all tasks, since they share the
        cost model); else one felix_search per shard, on its own stream if `concurrent`."""
        import torch
        from . import search_group
        dev = torch.device("cuda", self.device)
        main = torch.cuda.current_stream(dev)
        if not hasattr(self, "_streams"):
            self._streams = [torch.cuda.Stream(device=dev) for _ in self.shards]
            self._y = {s.task: torch.empty((self.spaces[s.task].n_vars, s.n), dtype=torch.float32, device=dev)
                       for s in self.shards}
        if batched and len(self.shards) > 0:
            ys = [self._y[s.task] if y0 is None else y0[s.task] for s in self.shards]
            search_group([self.spaces[s.task] for s in self.shards], self.cm, ys, n_steps, lr=lr, lam=lam,
                         rng_seeds=[rng_seed + s.task for s in self.shards], index_bases=[s.seed_lo for s in self.shards],
                         init_from_y=y0 is not None,
                         final_losses=None if loss_out is None else [loss_out[s.task] for s in self.shards], stream=main)
            return {s.task: self.spaces[s.task].round_topk(self.cm, y, k, index_base=s.seed_lo, stream=main)
                    for s, y in zip(self.shards, ys)}
        streams = self._streams if concurrent else [main] * len(self.shards)
        for s, st in zip(self.shards, streams):
            st.wait_stream(main)
            y = self._y[s.task] if y0 is None else y0[s.task]
            lo = None if loss_out is None else loss_out[s.task]
            self.spaces[s.task].search(self.cm, y, n_steps, lr=lr, lam=lam, rng_seed=rng_seed + s.task,
                                       init_from_y=y0 is not None, index_base=s.seed_lo, final_loss=lo, stream=st)
        out = {}
        for s, st in zip(self.shards, streams):
            y = self._y[s.task] if y0 is None else y0[s.task]
            out[s.task] = self.spaces[s.task].round_topk(self.cm, y, k, index_base=s.seed_lo, stream=st)
        for st in streams:
            main.wait_stream(st)
        return out

    def cand_steps(self, n_steps: int) -> int:
        return sum(s.n for s in self.shards) * n_steps
