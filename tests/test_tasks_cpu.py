"""Multi-task sharding (configs C3 = ResNet-50 sharded by subgraph with LPT, C4 = BERT-base
with every task's seeds sharded): planner properties on CPU, and a gloo world-size-2 run in which each
rank computes the oracle's top-k of its own shards and the per-task all-gather + merge must equal the
single-process top-k of every task (for both shard modes)."""
import itertools
import os
import socket
import sys

import numpy as np
import pytest
import torch.multiprocessing as mp

import felix_inputs as fi
from oracle import felix_oracle as fo


def _load_tasks_module():
    """paper_conf_asplos_zhaosam24_b200.tasks (its per-task merge runs in libfelix: felix_merge_topk)."""
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_asplos_zhaosam24_b200 import tasks
    return tasks


ft = _load_tasks_module()


def test_lpt_every_task_once_and_deterministic():
    rng = np.random.default_rng(3)
    for world in (1, 2, 3, 8):
        costs = list(rng.uniform(1, 100, size=21))
        a = ft.lpt_assign(costs, world)
        assert sorted(itertools.chain(*a)) == list(range(21))
        assert a == ft.lpt_assign(costs, world)


def test_lpt_makespan_within_graham_bound_of_brute_force():
    # LPT makespan <= (4/3 - 1/(3m)) OPT; OPT by brute force over all assignments of 7 tasks to 2-3 ranks
    rng = np.random.default_rng(5)
    for world in (2, 3):
        for _ in range(5):
            costs = list(rng.integers(1, 50, size=7).astype(float))
            lpt = max(sum(costs[t] for t in ts) for ts in ft.lpt_assign(costs, world))
            opt = min(max(sum(c for c, r in zip(costs, asg) if r == q) for q in range(world))
                      for asg in itertools.product(range(world), repeat=len(costs)))
            assert lpt <= (4 / 3 - 1 / (3 * world)) * opt + 1e-9


def test_lpt_known_case():
    # classic example: costs 5,5,4,4,3,3,3 on 3 ranks -> LPT 11 (OPT 9): order 5,5,4 then 4->r2, 3->r0/r1 ...
    a = ft.lpt_assign([5, 5, 4, 4, 3, 3, 3], 3)
    loads = sorted(sum([5, 5, 4, 4, 3, 3, 3][t] for t in ts) for ts in a)
    assert loads == [7, 8, 12] or max(loads) == 11


def test_seed_plan_covers_every_seed_once():
    for n, world in [(16384, 8), (100, 3), (5, 8), (1, 1)]:
        shards = ft.plan(4, n, world, "seeds")
        for t in range(4):
            got = sorted(itertools.chain(*[range(s.seed_lo, s.seed_lo + s.n) for r in shards for s in r if s.task == t]))
            assert got == list(range(n))


def test_task_plan_uses_est_cost():
    costs = [ft.est_cost(8192, 200, 955392, nn) for nn in (100, 300, 200)]
    assert costs[1] > costs[2] > costs[0]
    p = ft.plan(3, 8192, 2, "task", costs)
    assert [s.task for s in p[0]] == [1] and [s.task for s in p[1]] == [0, 2]
    assert all(s.seed_lo == 0 and s.n == 8192 for r in p for s in r)
    assert ft.config_mode("C3") == "hybrid" and ft.config_mode("C4") == "seeds"


def test_pack_merge_roundtrip_single_rank():
    per = {0: (np.array([4, 1]), np.array([2.0, 1.0]), np.array([[1, 2, 3], [4, 5, 6]], dtype=np.int32)),
           2: (np.array([7]), np.array([0.5]), np.array([[9, 9]], dtype=np.int32))}
    rows = ft.pack_task_records(per, 3, 2, 3)
    out = ft.merge_task_records(rows, 3, 2, [3, 1, 2])
    assert out[0][0].tolist() == [4, 1] and out[0][2].tolist() == [[1, 2, 3], [4, 5, 6]]
    assert len(out[1][0]) == 0
    assert out[2][2].tolist() == [[9, 9]]


# ----------------------------------------------------------------------------- gloo, world size 2
def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _tasks():
    c1 = fi.config("C1")
    return [fi.paper_example_space(), c1.spaces[0]], fi.make_mlp(c1.mlp_dims)


def _worker(rank, world, port, mode, ys, k, out):
    import torch.distributed as dist
    tm = _load_tasks_module()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    spaces, mlp = _tasks()
    n = ys[0].shape[1]
    costs = [tm.est_cost(n, 1, 1, sp.nodes.shape[0]) for sp in spaces]
    shards = tm.plan(len(spaces), n, world, mode, costs)[rank]
    per = {}
    for s in shards:
        y = np.ascontiguousarray(ys[s.task][:, s.seed_lo:s.seed_lo + s.n])
        per[s.task] = fo.round_topk(spaces[s.task], mlp.W, mlp.b, y, k, index_base=s.seed_lo)
    merged = tm.allgather_task_topk(per, len(spaces), k, [sp.n_vars for sp in spaces])
    out[rank] = {t: (v[0].tolist(), v[1].tolist(), v[2].tolist()) for t, v in merged.items()}
    dist.destroy_process_group()


@pytest.mark.timeout(300)
@pytest.mark.parametrize("mode", ["task", "seeds", "hybrid"])
def test_gloo_world2_per_task_topk_equals_single_process(mode):
    spaces, mlp = _tasks()
    k = 12
    ys = []
    for i, sp in enumerate(spaces):
        y = fi.make_y0(sp, 301, seed=40 + i)
        y[:, 200:230] = y[:, 5:35]                      # duplicates across the two seed shards
        ys.append(y)
    ref = [fo.round_topk(sp, mlp.W, mlp.b, y, k) for sp, y in zip(spaces, ys)]
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    ctx = mp.get_context("spawn")
    procs = [ctx.Process(target=_worker, args=(r, 2, port, mode, ys, k, out)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(240)
        assert p.exitcode == 0
    for r in range(2):
        for t, (ridx, rsc, rsched) in enumerate(ref):
            gidx, gsc, gsched = out[r][t]
            assert gidx == list(ridx)
            assert np.array_equal(np.array(gsc), rsc)
            assert gsched == rsched.tolist()


# ----------------------------------------------------------------------------- hybrid (seed-split LPT)
def _check_partition(plan, n_tasks, n):
    for t in range(n_tasks):
        rng = sorted((s.seed_lo, s.seed_lo + s.n) for sh in plan for s in sh if s.task == t)
        assert rng[0][0] == 0 and rng[-1][1] == n
        assert all(a[1] == b[0] for a, b in zip(rng, rng[1:]))          # contiguous, disjoint cover
    for sh in plan:
        assert len({s.task for s in sh}) == len(sh)                      # one shard per (rank, task)


def test_hybrid_plan_partitions_every_task_and_balances_c3():
    """C3 (21 nearly equal ResNet-50 tasks) on 8 ranks: task-mode LPT gives 3 tasks vs a mean of 2.625
    (0.875); the seed-split plan is within 5 % of the lower bound total / world."""
    costs = [ft.est_cost(8192, 200, 955392, nn) for nn in np.linspace(150, 260, 21).astype(int)]
    for world in (1, 2, 4, 8):
        p = ft.plan(21, 8192, world, "hybrid", costs)
        _check_partition(p, 21, 8192)
        eff = (sum(costs) / world) / ft.makespan(p, costs, 8192)
        assert eff >= 0.95, (world, eff)
    lpt = ft.plan(21, 8192, 8, "task", costs)
    assert (sum(costs) / 8) / ft.makespan(lpt, costs, 8192) <= 0.88


def test_hybrid_makespan_vs_brute_force_optimum():
    """Small instances: the plan's makespan against the brute-force optimum over all assignments of the
    same chunks to ranks (the plan is LPT over the chunks: within Graham's 4/3 bound of it), and against
    the fractional lower bound max(total / world, largest chunk)."""
    rng = np.random.default_rng(11)
    for world in (2, 3):
        for _ in range(4):
            costs = list(rng.integers(1, 40, size=4).astype(float))
            n = 12
            p = ft.hybrid_assign(costs, n, world, chunks_per_rank=1)
            _check_partition(p, 4, n)
            total = sum(costs)
            target = total / world
            nch = [max(1, min(n, int(np.ceil(c / target - 1e-9)))) for c in costs]
            chunks = [costs[t] * (ft.seed_range(n, i, nch[t])[1] - ft.seed_range(n, i, nch[t])[0]) / n
                      for t in range(4) for i in range(nch[t])]
            opt = min(max(sum(c for c, r in zip(chunks, asg) if r == q) for q in range(world))
                      for asg in itertools.product(range(world), repeat=len(chunks)))
            ms = ft.makespan(p, costs, n)
            assert ms <= (4 / 3 - 1 / (3 * world)) * opt + 1e-9
            assert ms >= max(total / world, max(chunks)) - 1e-9
