"""Several symbolic programs of one subgraph (Eq. 3):

    max_{p*_i} max_{x_i} C(Feat_{p*_i}(x_i))  s.t.  g_ir(x_i) <= 0.

Each program p*_i has its own variables x_i and Eq. 4 sums the per-program terms, so the
programs are searched independently.  Here every program's search runs on its own CUDA stream, so the
small, latency-bound searches of a subgraph overlap on the GPU, and the best schedules of the subgraph
are the per-program top-k lists merged by (score desc, program index asc, global index asc): schedules
of different programs are different programs (no cross-program dedup), and the merged top-k is always
contained in the union of the per-program top-k lists.

Host orchestration only: every step of the path runs in libfelix's kernels (felix_search,
felix_round_topk / felix_history_topk).  The concurrent launches are safe with the MLP kernels this
library selects: the cluster chain and the tile kernel need only one cluster / CTA co-scheduled at a
time, and the grid-barrier chain is launched cooperatively.
"""
from dataclasses import dataclass
from typing import List, Optional, Sequence

import numpy as np

from . import CostModel, Space


@dataclass
class SubgraphRecord:
    sketch: int          # index of the symbolic program p*_i
    idx: int             # global candidate index within that program's search
    score: float         # FP64 predicted performance C(slog(Feat_hard(x)))
    sched: np.ndarray    # int32 [n_vars of that program]
    step: int = -1       # first visit (history mode), else -1


class SubgraphSearch:
    """felix_search + top-k over the symbolic programs `spaces` of one subgraph."""

    def __init__(self, spaces: Sequence, cm: CostModel, device: int = 0):
        self.spaces = [Space(sp, device=device) for sp in spaces]
        self.cm = cm
        self.device = device

    def run(self, n_seeds: int, n_steps: int, k: int, *, rng_seed: int = 0, index_base: int = 0, lr: float = 0.05,
            lam: float = 1.0, history: bool = False, concurrent: bool = True) -> List[SubgraphRecord]:
        import torch
        dev = torch.device("cuda", self.device)
        main = torch.cuda.current_stream(dev)
        streams = [torch.cuda.Stream(device=dev) if concurrent else main for _ in self.spaces]
        ys = []
        for sp, st in zip(self.spaces, streams):
            st.wait_stream(main)
            with torch.cuda.stream(st):
                y = torch.empty((sp.n_vars, n_seeds), dtype=torch.float32, device=dev)
            # each program draws its own starting points (the sampler is per space)
            sp.search(self.cm, y, n_steps, lr=lr, lam=lam, rng_seed=rng_seed, init_from_y=False,
                      index_base=index_base, history=history, stream=st)
            ys.append(y)
        recs: List[SubgraphRecord] = []
        for i, (sp, st, y) in enumerate(zip(self.spaces, streams, ys)):
            if history:
                idx, step, sc, sched, _ = sp.history_topk(self.cm, k, stream=st)
            else:
                idx, sc, sched = sp.round_topk(self.cm, y, k, index_base=index_base, stream=st)
                step = np.full(len(idx), -1, dtype=np.int32)
            recs += [SubgraphRecord(i, int(idx[r]), float(sc[r]), sched[r].copy(), int(step[r])) for r in range(len(idx))]
        for st in streams:
            main.wait_stream(st)
        recs.sort(key=lambda r: (-r.score, r.sketch, r.step, r.idx))
        return recs[:k]
