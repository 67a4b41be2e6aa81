"""GPU parity of the branch-and-bound divisor rounding (aux_kernels.cuh round_bnb_kernel; SURVEY §7c
hard part 7) against the float64 oracle's exhaustive scan (oracle/felix_oracle.py
round_schedules: the divisor-respecting tuple minimising sum_j (y_j - ln f_j)^2, ties -> the
lexicographically smallest).  Bit-exact, as every integer decision.

* highly composite extent 720720 split four ways (6.6e5 tuples: no table, branch and bound by default),
  with adversarial points: ties between permutations (equal y), y exactly at ln d, log-midpoints,
  far outside the box, non-finite;
* felix_tune(round_bnb=1) on the workload spaces: branch and bound everywhere equals the table scan
  and the oracle;
* eight ways (1.5e8 tuples, beyond any table): the result is feasible and no single-variable change
  or prime move between two variables lowers the cost (necessary conditions of the argmin, computed
  in numpy float64 the oracle's way).
"""
import math

import numpy as np
import pytest
import torch

import felix_inputs as fi
from oracle import felix_oracle as fo

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def fx():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_asplos_zhaosam24_b200 as m
    assert torch.cuda.is_available()
    yield m
    m.tune(round_bnb=0)


def _oracle_round(sp, y, chunk=32):
    return np.concatenate([fo.round_schedules(sp, y[:, i:i + chunk]) for i in range(0, y.shape[1], chunk)])


def _adversarial_y(sp, n, seed):
    """make_y0 points plus ties, exact ln d, log-midpoints and out-of-box / non-finite values on the
    first split component (vars 0..3 of composite_space)."""
    y = fi.make_y0(sp, n, seed=seed, margin=0.5).astype(np.float32)
    rng = np.random.default_rng(seed)
    divs = [d for d in range(1, 720721) if 720720 % d == 0]
    for i in range(0, n, 7):              # all four tile variables equal: permutations tie exactly
        y[0:4, i] = y[0, i]
    for i in range(1, n, 7):              # exactly at ln d (as float32)
        y[0:4, i] = np.log(rng.choice(divs, 4)).astype(np.float32)
    for i in range(2, n, 7):              # log-midpoints between consecutive divisors
        k = rng.integers(0, len(divs) - 1, 4)
        y[0:4, i] = (0.5 * (np.log(np.array(divs)[k]) + np.log(np.array(divs)[k + 1]))).astype(np.float32)
    for i in range(3, n, 7):              # far outside the box
        y[0:4, i] = rng.choice([-20.0, 30.0], 4).astype(np.float32)
    y[1, 4] = np.nan
    y[2, 5] = np.inf
    y[0, 6] = -np.inf
    y[5, 11] = np.nan                     # non-finite in the second component only
    return np.ascontiguousarray(y)


def test_composite_extent_default_bnb_matches_oracle(fx):
    sp = fi.composite_space(4)
    space = fx.Space(sp)
    assert space.info.n_tuples_total == 14000       # the 720720 component has no table
    y = _adversarial_y(sp, 97, seed=61)
    ref = _oracle_round(sp, y)
    sched, valid = space.round(torch.from_numpy(y).cuda())
    assert np.array_equal(sched.cpu().numpy(), ref)
    fx.tune(round_bnb=1)                             # second component by branch and bound too
    try:
        sched2, _ = space.round(torch.from_numpy(y).cuda())
    finally:
        fx.tune(round_bnb=0)
    assert np.array_equal(sched2.cpu().numpy(), ref)
    # the rest of the finish runs on these schedules: validity and top-k against the oracle
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    yf = np.ascontiguousarray(np.nan_to_num(y, nan=0.0, posinf=5.0, neginf=-5.0)[:, :32])
    idx, sc, sch = space.round_topk(cm, torch.from_numpy(yf).cuda(), 8)
    ridx, rsc, rsch = fo.round_topk(sp, mlp.W, mlp.b, yf, 8)
    assert np.array_equal(idx, ridx) and np.array_equal(sch, rsch)
    assert np.allclose(sc, rsc, rtol=1e-12, atol=0)


@pytest.mark.parametrize("name", ["C1", "C2", "allops", "r50_conv1", "bert_ln"])
def test_forced_bnb_equals_table_scan_and_oracle(fx, name):
    if name == "allops":
        sp = fi.allops_space()
    elif name == "r50_conv1":
        sp = fi.resnet50_spaces()[0]
    elif name == "bert_ln":
        sp = [s for s in fi.bert_spaces() if "layernorm" in s.name][0]
    else:
        sp = fi.config(name).spaces[0]
    space = fx.Space(sp)
    y = fi.make_y0(sp, 1000, seed=77, margin=0.6)
    y[:, ::5] = y[0:1, ::5]                          # equal coordinates: exact ties between permutations
    yt = torch.from_numpy(np.ascontiguousarray(y)).cuda()
    table, _ = space.round(yt)
    fx.tune(round_bnb=1)
    try:
        bnb, _ = space.round(yt)
    finally:
        fx.tune(round_bnb=0)
    assert torch.equal(table, bnb)
    assert np.array_equal(bnb.cpu().numpy(), fo.round_schedules(sp, y))


def _cost(yc, f):
    acc = 0.0
    for a, b in zip(yc, f):
        d = a - math.log(b)
        acc = acc + d * d
    return acc


def test_eight_way_split_feasible_and_locally_optimal(fx):
    sp = fi.composite_space(8)
    space = fx.Space(sp)                             # 1.5e8 tuples: unsupported before branch and bound
    y = fi.make_y0(sp, 64, seed=83, margin=0.3)
    sched = space.round(torch.from_numpy(y).cuda())[0].cpu().numpy()
    primes = [2, 3, 5, 7, 11, 13]
    divs = [d for d in range(1, 720721) if 720720 % d == 0]
    y64 = y.astype(np.float64)
    for i in range(sched.shape[0]):
        f = [int(v) for v in sched[i, :8]]
        assert 720720 % math.prod(f) == 0
        yc = y64[:8, i]
        c0 = _cost(yc, f)
        room = 720720 // math.prod(f)
        for j in range(8):                           # one variable to any divisor that keeps feasibility
            for d in divs:
                if (room * f[j]) % d == 0 and d != f[j]:
                    g = list(f); g[j] = d
                    assert _cost(yc, g) >= c0
        for a in range(8):                           # move a prime factor from one variable to another
            for b in range(8):
                for p in primes:
                    if a != b and f[a] % p == 0:
                        g = list(f); g[a] //= p; g[b] *= p
                        assert _cost(yc, g) >= c0
