"""Multi-GPU top-k exchange.

Candidates shard naturally: Eq. 4 is a sum of per-seed terms and Adam is elementwise (PAPER.md
L884-885, L926-927), so every rank searches its own contiguous seed range (index_base = rank * n)
with no per-step communication.  The only exchange is at the end: each rank's local top-k records
(global index, FP64 score, schedule) are all-gathered over NCCL (NVLink / NVSwitch) and every rank
merges them identically: dedup by schedule keeping the smallest global index, then order by
(score desc, global index asc).  Because indices are global and the per-rank top-k already keeps
each schedule's smallest index, the merged list equals the single-GPU top-k of the union.
"""
from __future__ import annotations

from typing import Tuple

import numpy as np


def pack_records(idx: np.ndarray, score: np.ndarray, sched: np.ndarray, k: int, n_vars: int) -> np.ndarray:
    """[k, 2 + n_vars] float64 rows (idx, score, sched...); missing rows have idx = -1."""
    out = np.zeros((k, 2 + n_vars), dtype=np.float64)
    out[:, 0] = -1
    m = len(idx)
    out[:m, 0] = idx
    out[:m, 1] = score
    out[:m, 2:] = sched
    return out


def merge_records(rows: np.ndarray, k: int) -> Tuple[np.ndarray, np.ndarray, np.ndarray]:
    """Deterministic merge of gathered records [R, 2 + n_vars] through the C ABI (felix_merge_topk):
    dedup by schedule, order (score desc, global index asc), best k."""
    from . import merge_topk
    return merge_topk(rows[:, 0].astype(np.int64), rows[:, 1], rows[:, 2:].astype(np.int32), k)


def allgather_topk(idx, score, sched, k: int, n_vars: int, group=None, device=None):
    """All-gather local top-k records across the process group (NCCL on GPUs, gloo on CPU) and
    merge them.  Scores travel as float64 (bit-exact), indices and factors are exact in float64."""
    import torch
    import torch.distributed as dist
    rec = torch.from_numpy(pack_records(idx, score, sched, k, n_vars))
    if device is not None:
        rec = rec.to(device)
    world = dist.get_world_size(group)
    out = torch.empty((world * k, 2 + n_vars), dtype=torch.float64, device=rec.device)
    dist.all_gather_into_tensor(out, rec, group=group)
    return merge_records(out.cpu().numpy(), k)
