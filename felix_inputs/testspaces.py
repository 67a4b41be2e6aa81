"""Hand-built test spaces that exercise the whole operator set and the non-finite rule (input
generation only: DAG construction, no evaluation arithmetic).

* allops_space(): 82 feature roots over three variables that use every one of the 25 opcodes of the
  input format ("+, -, *, /, pow, min, max, select, etc."), several times each and in
  different combinations, plus a user constraint; a SPLIT pair sharing one split so that rounding
  has a two-variable component.
* rnan_space(): features whose smooth or hard value is non-finite on part of the domain — LOG of a
  negative number (x_a < 3) and DIV by zero at the integer point x_a = 2 — for the R-NaN reading (a
  candidate with a non-finite loss or gradient is frozen; a rounded schedule with a non-finite
  feature is invalid).
"""
from __future__ import annotations

import math

import numpy as np

from .dag import (DagBuilder, Space, Split, Var, VAR_INT, VAR_SPLIT, OP_EQ, OP_GE, OP_LT, OP_NE)


def allops_space() -> Space:
    B = DagBuilder()
    x0, x1, x2, x3 = B.var(0), B.var(1), B.var(2), B.var(3)
    xs = [x0, x1, x2, x3]
    f = []
    # the 27-node core of tests/test_oracle.py test_reverse_mode_all_ops_vs_fd
    f += [B.add(x0, x1), B.sub(x0, x2), B.mul(x1, x2), B.div(x0, x2), B.neg(x1), B.pow(x0, 1.7),
          B.exp(B.div(x1, B.const(10.0))), B.log(x2), B.sqrt(x0), B.min(x0, x1), B.max(x1, x2)]
    c1, c2, c3 = B.gt(x0, x1), B.cmp(OP_GE, x1, x2), B.cmp(OP_LT, x0, x2)
    c4, c5, c6 = B.le(x1, x0), B.cmp(OP_EQ, x0, x1), B.cmp(OP_NE, x1, x2)
    f += [B.select(c, x0, x2) for c in (c1, c2, c3, c4, c5, c6)]
    f += [B.select(B.land(c1, c3), x1, x2), B.select(B.lor(c2, c4), x0, x1), B.select(B.lnot(c6), x2, x0),
          B.floordiv(x0, x1), B.ceildiv(x2, x1)]
    # more combinations until 82 roots: every binary / unary op on every ordered variable pair,
    # nested so that adjoints flow through chains of different ops
    pairs = [(a, b) for a in range(4) for b in range(4) if a != b]
    k = 0
    while len(f) < 82 and k < 10000:
        a, b = pairs[(k // 12 + 5 * k) % len(pairs)]
        xa, xb = xs[a], xs[b]
        t = k % 12
        if t == 0:
            e = B.mul(B.max(xa, B.const(4.0)), B.min(xb, B.const(8.0)))
        elif t == 1:
            e = B.select(B.cmp(OP_EQ, B.floordiv(xa, xb), B.const(1.0)), B.sqrt(B.mul(xa, xb)), B.pow(xb, -0.5))
        elif t == 2:
            e = B.log(B.add(B.ceildiv(xa, xb), B.const(1.0)))
        elif t == 3:
            e = B.select(B.lor(B.gt(xa, B.const(6.0)), B.cmp(OP_NE, xb, B.const(2.0))), B.exp(B.div(xa, B.const(16.0))), B.neg(xb))
        elif t == 4:
            e = B.div(B.pow(xa, 2.0), B.add(xb, B.const(1.0)))
        elif t == 5:
            e = B.max(B.sub(xa, xb), B.const(0.0))
        elif t == 6:
            e = B.mul(B.select(B.land(B.cmp(OP_GE, xa, xb), B.lnot(B.gt(xb, B.const(9.0)))), xa, xb), B.const(3.0))
        elif t == 7:
            e = B.sqrt(B.add(B.pow(xa, 3.0), B.mul(xb, xb)))
        elif t == 8:
            e = B.min(B.floordiv(B.mul(xa, B.const(64.0)), xb), B.const(100.0))
        elif t == 9:
            e = B.select(B.cmp(OP_LT, xa, xb), B.log(B.add(xa, xb)), B.exp(B.neg(B.div(xb, B.const(8.0)))))
        elif t == 10:
            e = B.sub(B.select(B.cmp(OP_NE, xa, xb), xa, B.const(0.0)), B.select(B.cmp(OP_EQ, xa, B.const(4.0)), xb, B.const(1.0)))
        else:
            e = B.add(B.ceildiv(B.const(56.0), xa), B.floordiv(B.const(64.0), B.max(xb, B.const(1.0))))
        if e not in f:
            f.append(e)
        k += 1
    con = B.sub(B.log(B.mul(x0, x1)), B.const(math.log(256.0)))
    nodes = B.nodes()
    vars_ = [Var("a", VAR_SPLIT, 1, 64), Var("b", VAR_SPLIT, 1, 64), Var("c", VAR_INT, 1, 64),
             Var("d", VAR_SPLIT, 1, 48)]
    return Space("allops", vars_, [Split(64, [0]), Split(64, [1]), Split(48, [3, 0])], nodes,
                 np.array(f[:82], dtype=np.int32), np.array([con], dtype=np.int32),
                 feature_names=[f"f{i}" for i in range(82)], constraint_names=["log_ab"])


def rnan_space() -> Space:
    """C1's dense 64x64x64 space (6 variables, its 58 features) with two reserved feature slots replaced by
    LOG(x_0 - 3) and x_1 / (x_0 - 2): a real, well-conditioned feature set in which candidates with
    x_0 < 3 have a non-finite smooth feature and schedules with x_0 in {1, 2} a non-finite hard one."""
    from .configs import c1_space
    base = c1_space()
    nodes = list(base.nodes.tolist())
    def add(op, a=-1, b=-1, c=-1, imm=0.0):
        nodes.append((op, a, b, c, imm))
        return len(nodes) - 1
    from .dag import OP_CONST, OP_VAR, OP_SUB, OP_LOG, OP_DIV
    x0, x1 = add(OP_VAR, imm=0.0), add(OP_VAR, imm=1.0)
    f_log = add(OP_LOG, add(OP_SUB, x0, add(OP_CONST, imm=3.0)))
    f_div = add(OP_DIV, x1, add(OP_SUB, x0, add(OP_CONST, imm=2.0)))
    arr = np.zeros(len(nodes), dtype=base.nodes.dtype)
    for i, r in enumerate(nodes):
        arr[i] = r
    froots = base.feature_roots.copy()
    names = list(base.feature_names)
    free = [k for k, nm in enumerate(names) if nm.startswith("reserved")]
    froots[free[0]], froots[free[1]] = f_log, f_div
    names[free[0]], names[free[1]] = "log(x0-3)", "x1/(x0-2)"
    return Space("rnan", base.vars, base.splits, arr, froots, base.constraint_roots.copy(), names,
                 list(base.constraint_names), None)


def composite_space(n_tile_vars: int = 4, extent: int = 720720) -> Space:
    """Highly composite split extents for the rounding search (SURVEY §7c hard part 7; "N is
    ... typically smaller than 10^6"): `extent` = 720720 = 2^4 3^2 5 7 11 13 (240 divisors) tiled by
    `n_tile_vars` variables (4: 6.6e5 divisor tuples; 8: 1.5e8), a second component in which one
    variable sits in two splits (5040 and 2520), and an INT variable; 82 feature roots over all of them
    (products, ratios, logs) so a cost model of the default dims scores the schedules."""
    B = DagBuilder()
    nt = n_tile_vars
    xs = [B.var(j) for j in range(nt + 4)]
    f = []
    for a in range(len(xs)):
        f += [xs[a], B.log(B.add(xs[a], B.const(1.0)))]
    for a in range(len(xs)):
        for b in range(a + 1, len(xs)):
            f += [B.mul(xs[a], xs[b]), B.div(xs[a], B.add(xs[b], B.const(1.0)))]
            if len(f) >= 82:
                break
        if len(f) >= 82:
            break
    while len(f) < 82:
        f.append(B.add(f[len(f) % 7], B.const(float(len(f)))))
    con = B.sub(B.mul(xs[0], xs[1]), B.const(4096.0))
    nodes = B.nodes()
    vars_ = [Var(f"t{j}", VAR_SPLIT, 1, extent) for j in range(nt)]
    vars_ += [Var("s0", VAR_SPLIT, 1, 2520), Var("s1", VAR_SPLIT, 1, 5040), Var("s2", VAR_SPLIT, 1, 2520),
              Var("u", VAR_INT, 1, 100)]
    splits = [Split(extent, list(range(nt))), Split(5040, [nt, nt + 1]), Split(2520, [nt, nt + 2])]
    return Space(f"composite{nt}", vars_, splits, nodes, np.array(f[:82], dtype=np.int32),
                 np.array([con], dtype=np.int32), feature_names=[f"f{i}" for i in range(82)],
                 constraint_names=["t0t1"])
