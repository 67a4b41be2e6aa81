"""Multi-rank top-k exchange on CPU (gloo, world_size 2): the only collective of the path
(SURVEY §8(e)).  Each rank holds the oracle's local top-k of its own seed shard (global indices via
index_base); after the all-gather + host merge every rank must hold exactly the single-process top-k
of the union (shard invariance)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import felix_inputs as fi
from oracle import felix_oracle as fo


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _load_dist_module():
    """paper_conf_asplos_zhaosam24_b200.dist (the merge runs in libfelix's host code: felix_merge_topk)."""
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_zhaosam24_b200 import dist
    return dist


def _worker(rank, world, port, y_all, k, out):
    import torch.distributed as dist
    fdist = _load_dist_module()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    c = fi.config("C1")
    sp = c.spaces[0]
    mlp = fi.make_mlp(c.mlp_dims)
    n = y_all.shape[1] // world
    base = rank * n
    idx, sc, sched = fo.round_topk(sp, mlp.W, mlp.b, np.ascontiguousarray(y_all[:, base:base + n]), k, index_base=base)
    gidx, gsc, gsched = fdist.allgather_topk(idx, sc, sched, k, sp.n_vars)
    out[rank] = (gidx.tolist(), gsc.tolist(), gsched.tolist())
    dist.destroy_process_group()


@pytest.fixture(scope="module")
def fdist():
    pytest.importorskip("torch.distributed")
    return _load_dist_module()


def test_merge_records_dedup_and_order(fdist):
    # identical schedules carry identical scores (deterministic FP64 scoring)
    rows = fdist.pack_records(np.array([5, 2]), np.array([1.0, 2.0]),
                              np.array([[1, 2], [3, 4]], dtype=np.int32), 4, 2)
    rows2 = fdist.pack_records(np.array([1, 3, 7]), np.array([2.0, 1.0, 0.5]),
                               np.array([[3, 4], [1, 2], [5, 6]], dtype=np.int32), 4, 2)
    idx, sc, sched = fdist.merge_records(np.concatenate([rows, rows2]), 3)
    # (score desc, global index asc); each schedule once, with its smallest global index
    assert list(idx) == [1, 3, 7] and list(sc) == [2.0, 1.0, 0.5]
    assert sched.tolist() == [[3, 4], [1, 2], [5, 6]]


@pytest.mark.timeout(300)
def test_gloo_world2_topk_equals_single_process():
    c = fi.config("C1")
    sp = c.spaces[0]
    mlp = fi.make_mlp(c.mlp_dims)
    y_all = fi.make_y0(sp, 512, seed=21)
    y_all[:, 300:340] = y_all[:, 10:50]                 # cross-shard duplicates
    k = 16
    ridx, rsc, rsched = fo.round_topk(sp, mlp.W, mlp.b, y_all, k)
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_worker, args=(r, 2, port, y_all, k, out)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(240)
        assert p.exitcode == 0
    for r in range(2):
        gidx, gsc, gsched = out[r]
        assert gidx == list(ridx)
        assert np.allclose(gsc, rsc, rtol=0, atol=0)
        assert gsched == rsched.tolist()
