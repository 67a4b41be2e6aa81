"""Pins for the float64 oracle against things other than itself (CPU; -m "not gpu").

Each test names what fixes the expected value: the paper's printed formulas / examples, a closed
form, brute-force enumeration, finite differences, or a library routine (torch float64).
"""
import json
import math
import os

import numpy as np
import pytest
import torch

import felix_inputs as fi
from felix_inputs.programs import build_space, conv2d_spec, dense_spec, depthwise_conv2d_spec, layernorm_spec, softmax_spec
from oracle import felix_oracle as fo
from tests.sim.loopnest import enumerate_valid, simulate, simulate_epilogue

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_dense_add_s1.json")))

TINY_SPECS = [
    dense_spec("tiny_dense", 8, 4, 8, i_levels="vti", j_levels="ti", k_vars=2, bias=True),
    dense_spec("tiny_bmm", 4, 4, 4, batch=2, i_levels="ti", j_levels="vti", k_vars=1, bias=False),
    conv2d_spec("tiny_conv3x3", 2, 4, 4, 2, 3, 3, 1, rc_vars=1),
    conv2d_spec("tiny_conv1x1_s2", 2, 3, 3, 2, 1, 1, 2, rc_vars=2),
    conv2d_spec("tiny_conv3x3_s2", 2, 3, 3, 2, 3, 3, 2, rc_vars=1),
    softmax_spec("tiny_softmax", 2, 4, 8, j_vars=1),
    layernorm_spec("tiny_layernorm", 4, 8, j_vars=2),
    depthwise_conv2d_spec("tiny_dwconv3x3_s2", 4, 3, 3, 3, 3, 2),
]


# ----------------------------------------------------------------------------- O-pin-1
@pytest.mark.parametrize("spec", TINY_SPECS, ids=lambda s: s.name)
def test_two_statement_features_equal_bruteforce(spec):
    """Per-statement features (statements=2, TenSet segment-sum layout): the main statement equals the
    brute-force count without the epilogue ops, the epilogue statement equals its own enumeration."""
    sp = build_space(spec, statements=2)
    assert len(sp.feature_roots) == 2 * 82
    pts = enumerate_valid(sp)
    rng = np.random.default_rng(11)
    for i in rng.choice(len(pts), min(40, len(pts)), replace=False):
        p = dict(pts[i])
        if spec.unroll:
            p["UNROLL"] = int(rng.choice([1, 2, 4, 16, 1024]))
        x = np.array([[p[v.name]] for v in sp.vars], dtype=float)
        F = fo.eval_dag(sp, x, smooth=False).F[:, 0]
        main, epi = simulate(spec, p), simulate_epilogue(spec, p)
        for k, nm in enumerate(sp.feature_names):
            st, base = nm.split(".", 1)
            if base.startswith("reserved"):
                assert F[k] == 0.0
                continue
            if st == "S0":
                # the main statement without the epilogue's ops (the epilogue statement counts them)
                exp = main[base] - epi[base] if base in ("float_addsub", "float_cmp", "float_math") else main[base]
            else:
                exp = epi[base]
            assert abs(F[k] - exp) <= 1e-12 * max(1.0, abs(exp)), (spec.name, nm, p, F[k], exp)


@pytest.mark.parametrize("spec", TINY_SPECS, ids=lambda s: s.name)
def test_hard_features_equal_bruteforce_loop_nest(spec):
    """Hard-semantics DAG at every sampled valid integer point == brute-force enumeration of the
    concrete tiled loop nest (exact counts; ratios to 1e-12)."""
    sp = build_space(spec)
    pts = enumerate_valid(sp)
    rng = np.random.default_rng(7)
    sel = [pts[i] for i in rng.choice(len(pts), min(80, len(pts)), replace=False)]
    for p in sel:
        p = dict(p)
        if spec.unroll:
            p["UNROLL"] = int(rng.choice([1, 2, 3, 4, 8, 16, 64, 1024]))
        x = np.array([[p[v.name]] for v in sp.vars], dtype=float)
        ev = fo.eval_dag(sp, x, smooth=False)
        sim = simulate(spec, p)
        for k, nm in enumerate(sp.feature_names):
            got = ev.F[k, 0]
            if nm.startswith("reserved"):
                assert got == 0.0
                continue
            exp = sim[nm]
            assert abs(got - exp) <= 1e-12 * max(1.0, abs(exp)), (spec.name, nm, p, got, exp)
        # constraints: log-form limits on the simulated quantities
        lim = {"threads<=limit": (sim["_threads"], spec.thread_limit),
               "smem<=limit": (sim["_smem"], spec.smem_limit),
               "local<=limit": (sim["_local"], spec.local_limit * 4),
               "vthreads<=limit": (sim["_vthreads"], spec.vthread_limit)}
        for r, nm in enumerate(sp.constraint_names):
            q, L = lim[nm]
            assert abs(ev.g_user[r, 0] - (math.log(q) - math.log(L))) < 1e-12


def test_paper_dense_add_example_formulas():
    """P:L668-671 literally, at TILE0 in {1,2,8,64}: hard values, smooth values, slog values."""
    sp = fi.paper_example_space()
    for row in GOLD["rows"]:
        x = np.array([[row["TILE0"]], [16.0]])
        hard = fo.eval_dag(sp, x, smooth=False).F[:, 0]
        smooth = fo.eval_dag(sp, x, smooth=True).F[:, 0]
        assert hard[0] == row["float_add"] and hard[1] == row["blockIdx_len"] and hard[2] == row["int_add_hard"]
        assert smooth[0] == row["float_add"] and smooth[1] == row["blockIdx_len"]
        assert abs(smooth[2] - row["int_add_smooth"]) < 1e-6
        ph = fo.slog(smooth)
        assert abs(ph[0] - row["slog_float_add"]) < 1e-8
        assert abs(ph[1] - row["slog_blockIdx_len"]) < 1e-8
        assert abs(ph[2] - row["slog_int_add_smooth"]) < 1e-8
        assert np.all(hard[3:] == 0)


def test_paper_constraint_example_and_penalty_scale():
    """g11 = 1 - TILE0, g12 = TILE0 - K; W2 penalty scale x-space vs log-space."""
    sp = fi.paper_example_space()
    w = GOLD["penalty_W2"]
    ev = fo.eval_dag(sp, np.array([[w["TILE0"]], [1.0]]), smooth=True)
    assert ev.g_user[0, 0] == 1 - w["TILE0"] and ev.g_user[1, 0] == w["TILE0"] - w["K"]
    assert max(ev.g_user[1, 0], 0) ** 2 * w["lambda"] == w["xspace_penalty"]
    g = math.log(w["TILE0"]) - math.log(w["K"])
    assert abs(g - w["logspace_root"]) < 1e-6 and abs(g * g - w["logspace_penalty"]) < 1e-6


# ----------------------------------------------------------------------------- smoothing closed forms
def test_smooth_ops_closed_forms():
    t = np.linspace(-50, 50, 20001)
    S, R, dS = fo.smooth_S(t), fo.smooth_R(t), fo.smooth_dS(t)
    assert fo.smooth_S(np.array([0.0]))[0] == 0.5 and fo.smooth_R(np.array([0.0]))[0] == 0.5
    # R is a smooth upper bound of relu with gap <= 1/(4|t|); S within 1/(4 t^2) of the step
    big = np.abs(t) > 1
    assert np.all(R - np.maximum(t, 0) > 0)
    assert np.all((R - np.maximum(t, 0))[big] <= 1 / (4 * np.abs(t[big])) + 1e-15)
    assert np.all(np.abs(S - (t > 0))[big] <= 1 / (4 * t[big] ** 2) + 1e-15)
    # R' = S and S' = dS (central differences)
    h = 1e-5
    assert np.allclose((fo.smooth_R(t + h) - fo.smooth_R(t - h)) / (2 * h), S, atol=1e-8)
    assert np.allclose((fo.smooth_S(t + h) - fo.smooth_S(t - h)) / (2 * h), dS, atol=1e-8)
    # S is the CDF of the kernel: integral of dS over R is 1
    assert abs(np.trapezoid(fo.smooth_dS(np.linspace(-1e4, 1e4, 2_000_001)), dx=1e-2) - 1.0) < 1e-4
    # naive forms agree where they do not cancel
    mid = np.abs(t) < 5
    assert np.allclose(S[mid], 0.5 * (1 + t[mid] / np.sqrt(1 + t[mid] ** 2)), atol=1e-15)
    assert np.allclose(R[mid], 0.5 * (t[mid] + np.sqrt(1 + t[mid] ** 2)), atol=1e-14)
    # stable at huge magnitudes (features reach 1e9)
    assert fo.smooth_R(np.array([-1e12]))[0] > 0 and fo.smooth_S(np.array([1e12]))[0] == 1.0
    for v in (1e30, 1e200):
        assert np.isfinite(fo.smooth_R(np.array([v])))[0] and fo.smooth_S(np.array([-v]))[0] >= 0


def test_smooth_eq_ne_value_pins():
    """EQ(a,b) = S(a-b+1/2) S(b-a+1/2), NE = 1 - EQ (reading O3): values at d = a - b typed in from the
    closed form S(t) = (1 + t/sqrt(1+t^2))/2: EQ(0) = S(1/2)^2 = (3 + sqrt 5)/10 = 0.52360680,
    EQ(+-1) = S(3/2) S(-1/2) = 0.25318312; symmetric in d, maximal at d = 0, -> 0 as |d| grows."""
    B = fi.DagBuilder()
    a, b = B.var(0), B.var(1)
    eq, ne = B.cmp(fi.OP_EQ, a, b), B.cmp(fi.OP_NE, a, b)
    nodes = B.nodes()
    sp = fi.Space("eqne", [fi.Var("a", fi.VAR_SPLIT, 1, 64), fi.Var("b", fi.VAR_SPLIT, 1, 64)],
                  [fi.Split(64, [0]), fi.Split(64, [1])], nodes, np.array([a], np.int32), np.array([], np.int32))
    x = np.array([[5.0, 6.0, 4.0, 2.5, 40.0, 7.0], [5.0, 5.0, 5.0, 2.0, 7.0, 7.0 + 1e-9]])
    ev = fo.eval_dag(sp, x, smooth=True)
    E, N = ev.vals[eq], ev.vals[ne]
    assert abs(E[0] - 0.52360680) < 1e-8 and abs(E[0] - (3 + math.sqrt(5)) / 10) < 1e-15
    assert abs(E[1] - 0.25318312) < 1e-8 and abs(E[2] - 0.25318312) < 1e-8
    assert np.allclose(N, 1.0 - E, atol=0, rtol=0)
    assert E[3] < E[0] and E[3] > E[1] and E[4] < 1e-3 and abs(E[5] - E[0]) < 1e-9
    hard = fo.eval_dag(sp, np.array([[5.0, 6.0], [5.0, 5.0]]), smooth=False)
    assert list(hard.vals[eq]) == [1.0, 0.0] and list(hard.vals[ne]) == [0.0, 1.0]


def test_rnan_freeze_rule_first_step_closed_form():
    """Reading R-NaN: a candidate whose loss or gradient is non-finite is not updated (y, m, v stay);
    every other candidate takes the closed-form first Adam step y - lr g/(|g| + eps)."""
    sp = fi.rnan_space()
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    y0 = fi.make_y0(sp, 200, seed=9).astype(np.float64)
    ob = fo.objective(sp, mlp.W, mlp.b, y0, 1.0)
    ok = np.isfinite(ob.loss) & np.all(np.isfinite(ob.grad), axis=0)
    assert 0.2 < ok.mean() < 0.95
    # the non-finite ones are exactly those with x_0 < 3 (LOG of a negative number)
    assert np.array_equal(~ok, np.exp(y0[0]) < 3.0)
    y1, m1, v1, _ = fo.search(sp, mlp.W, mlp.b, y0, 1, lr=0.05, lam=1.0)
    assert np.array_equal(y1[:, ~ok], y0[:, ~ok]) and np.all(m1[:, ~ok] == 0) and np.all(v1[:, ~ok] == 0)
    g = ob.grad[:, ok]
    assert np.allclose(y1[:, ok], y0[:, ok] - 0.05 * g / (np.abs(g) + 1e-8), rtol=0, atol=1e-12)
    # rounding: schedules with a non-finite hard feature (x_0 in {1, 2}) are invalid
    rs = fo.round_schedules(sp, y0.astype(np.float32))
    v = fo.validate(sp, rs)
    assert not np.any(v & (rs[:, 0] <= 2)) and np.any(v)


def test_fig4_shapes():
    """Fig. 4: smoothed select(x>0,5,2) stays in (2,5); smoothed max(x,0) > 0 -> x."""
    g4 = GOLD["fig4_select_smooth"]
    x = np.array(g4["x"], dtype=float)
    sel = 2 + 3 * fo.smooth_S(x)
    assert np.allclose(sel, g4["value"], atol=5e-4)
    r = fo.smooth_R(np.array(GOLD["fig4_relu_smooth"]["x"], dtype=float))
    assert np.allclose(r, GOLD["fig4_relu_smooth"]["value"], atol=5e-4)


# ----------------------------------------------------------------------------- gradients
def _fd_grad(sp, W, b, y, lam, h=1e-6):
    g = np.zeros_like(y)
    for j in range(y.shape[0]):
        hj = h * np.maximum(1.0, np.abs(y[j]))
        yp, ym = y.copy(), y.copy()
        yp[j] += hj
        ym[j] -= hj
        g[j] = (fo.objective(sp, W, b, yp, lam, with_grad=False).loss
                - fo.objective(sp, W, b, ym, lam, with_grad=False).loss) / (2 * hj)
    return g


@pytest.mark.parametrize("which", ["C1", "C2", "paper"])
def test_reverse_mode_equals_finite_differences(which):
    if which == "paper":
        sp, dims = fi.paper_example_space(), (82, 64, 1)
    else:
        c = fi.config(which)
        sp, dims = c.spaces[0], (82, 64, 32, 1)
    mlp = fi.make_mlp(dims)
    y = fi.make_y0(sp, 24, seed=3).astype(np.float64)
    ob = fo.objective(sp, mlp.W, mlp.b, y, 1.0)
    fd = _fd_grad(sp, mlp.W, mlp.b, y, 1.0)
    # skip candidates sitting on a ReLU kink (FD across a kink is not a derivative)
    for i in range(y.shape[1]):
        margin = min(np.min(np.abs(z[:, i])) / (np.sqrt(np.mean(z[:, i] ** 2)) + 1e-300) for z in ob.zs)
        if margin < 1e-4:
            continue
        num = np.linalg.norm(ob.grad[:, i] - fd[:, i])
        den = max(np.linalg.norm(fd[:, i]), 1e-8)
        assert num / den < 1e-5, (which, i, ob.grad[:, i], fd[:, i])


def test_reverse_mode_all_ops_vs_fd():
    """Every opcode's adjoint rule, on a hand-built DAG touching all 25 ops."""
    B = fi.DagBuilder()
    x0, x1, x2 = B.var(0), B.var(1), B.var(2)
    ops = []
    ops.append(B.add(x0, x1)); ops.append(B.sub(x0, x2)); ops.append(B.mul(x1, x2)); ops.append(B.div(x0, x2))
    ops.append(B.neg(x1)); ops.append(B.pow(x0, 1.7)); ops.append(B.exp(B.div(x1, B.const(10.0))))
    ops.append(B.log(x2)); ops.append(B.sqrt(x0)); ops.append(B.min(x0, x1)); ops.append(B.max(x1, x2))
    c1, c2, c3 = B.gt(x0, x1), B.cmp(fi.OP_GE, x1, x2), B.cmp(fi.OP_LT, x0, x2)
    c4, c5, c6 = B.le(x1, x0), B.cmp(fi.OP_EQ, x0, x1), B.cmp(fi.OP_NE, x1, x2)
    ops += [B.select(c, x0, x2) for c in (c1, c2, c3, c4, c5, c6)]
    ops.append(B.select(B.land(c1, c3), x1, x2)); ops.append(B.select(B.lor(c2, c4), x0, x1))
    ops.append(B.select(B.lnot(c6), x2, x0))
    ops.append(B.floordiv(x0, x1)); ops.append(B.ceildiv(x2, x1))
    feats = ops + [B.const(0.0)] * (82 - len(ops))
    con = B.sub(B.log(B.mul(x0, x1)), B.const(math.log(100.0)))
    nodes = B.nodes()
    sp = fi.Space("allops", [fi.Var("a", fi.VAR_SPLIT, 1, 64), fi.Var("b", fi.VAR_SPLIT, 1, 64),
                             fi.Var("c", fi.VAR_INT, 1, 64)],
                  [fi.Split(64, [0]), fi.Split(64, [1])], nodes, np.array(feats, dtype=np.int32),
                  np.array([con], dtype=np.int32))
    mlp = fi.make_mlp((82, 32, 1))
    rng = np.random.default_rng(0)
    y = rng.uniform(0.1, 3.0, size=(3, 32))
    ob = fo.objective(sp, mlp.W, mlp.b, y, 0.5)
    fd = _fd_grad(sp, mlp.W, mlp.b, y, 0.5)
    for i in range(y.shape[1]):
        margin = min(np.min(np.abs(z[:, i])) / np.sqrt(np.mean(z[:, i] ** 2)) for z in ob.zs)
        if margin < 1e-4:
            continue
        assert np.linalg.norm(ob.grad[:, i] - fd[:, i]) / np.linalg.norm(fd[:, i]) < 1e-5


def test_mlp_forward_and_input_grad_vs_torch_float64():
    """C(phi) and dC/dphi against torch.nn.Linear + ReLU in float64 with autograd."""
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    rng = np.random.default_rng(1)
    phi = rng.uniform(0, 30, size=(82, 257))
    c, zs = fo.mlp_forward(mlp.W, mlp.b, phi)
    dphi = fo.mlp_input_grad(mlp.W, zs, -np.ones(257))
    layers = []
    for l, (w, bb) in enumerate(zip(mlp.W, mlp.b)):
        lin = torch.nn.Linear(w.shape[1], w.shape[0]).double()
        with torch.no_grad():
            lin.weight.copy_(torch.from_numpy(w.astype(np.float64)))
            lin.bias.copy_(torch.from_numpy(bb.astype(np.float64)))
        layers.append(lin)
        if l < len(mlp.W) - 1:
            layers.append(torch.nn.ReLU())
    net = torch.nn.Sequential(*layers)
    t = torch.from_numpy(phi.T.copy()).requires_grad_(True)
    out = net(t)[:, 0]
    (-out.sum()).backward()
    assert np.allclose(c, out.detach().numpy(), rtol=1e-13, atol=1e-13)
    assert np.allclose(dphi, t.grad.numpy().T, rtol=1e-12, atol=1e-13)


def test_adam_vs_torch_optim_adam_float64():
    rng = np.random.default_rng(2)
    y = rng.normal(size=(5, 7))
    grads = [rng.normal(size=(5, 7)) * 10 ** rng.uniform(-9, 2) for _ in range(6)]
    p = torch.nn.Parameter(torch.from_numpy(y.copy()))
    opt = torch.optim.Adam([p], lr=0.05, betas=(0.9, 0.999), eps=1e-8)
    m = np.zeros_like(y)
    v = np.zeros_like(y)
    for t, g in enumerate(grads, 1):
        p.grad = torch.from_numpy(g.copy())
        opt.step()
        y, m, v = fo.adam_step(y, m, v, g, t, 0.05)
        assert np.allclose(y, p.detach().numpy(), rtol=0, atol=1e-14)


def test_adam_first_step_closed_form():
    g = np.array([1e-3, -2.0, 5e-9, 0.0])
    y1, _, _ = fo.adam_step(np.zeros(4), np.zeros(4), np.zeros(4), g, 1, 0.05)
    assert np.allclose(y1, -0.05 * g / (np.abs(g) + 1e-8), rtol=1e-12, atol=1e-18)


# ----------------------------------------------------------------------------- rounding
def _exhaustive_round(sp, y):
    """Enumerate every divisor-respecting assignment of all SPLIT vars jointly; pick the minimum of
    sum_j (y_j - ln x_j)^2 (ties: lexicographically smallest over the var order)."""
    pts = enumerate_valid(sp)
    names = [v.name for v in sp.vars]
    split_j = [j for j, v in enumerate(sp.vars) if v.kind == fi.VAR_SPLIT]
    cand = sorted(tuple(p[names[j]] for j in split_j) for p in pts)
    best, bd = None, None
    for t in cand:
        d = 0.0
        for k, j in enumerate(split_j):
            e = float(np.float32(y[j])) - math.log(t[k])
            d = d + e * e
        if bd is None or d < bd:
            best, bd = t, d
    return best


@pytest.mark.parametrize("spec", TINY_SPECS[:3], ids=lambda s: s.name)
def test_rounding_equals_exhaustive_enumeration(spec):
    sp = build_space(spec)
    rng = np.random.default_rng(11)
    ub = np.log(fi.var_upper_bounds(sp))
    y = rng.uniform(-0.5, ub[:, None] + 0.5, size=(sp.n_vars, 40)).astype(np.float32)
    # adversarial: exact log-midpoints between consecutive divisors and out-of-range values
    for i in range(10):
        j = i % sp.n_vars
        if sp.vars[j].kind == fi.VAR_SPLIT:
            e = int(fi.var_upper_bounds(sp)[j])
            ds = [d for d in range(1, e + 1) if e % d == 0]
            if len(ds) > 1:
                y[j, i] = np.float32(0.5 * (math.log(ds[0]) + math.log(ds[1])))
    sched = fo.round_schedules(sp, y)
    split_j = [j for j, v in enumerate(sp.vars) if v.kind == fi.VAR_SPLIT]
    for i in range(y.shape[1]):
        assert tuple(sched[i, split_j]) == _exhaustive_round(sp, y[:, i])


def test_rounding_paper_examples():
    """W3 single-var geometric-mean threshold (TILE0 in splits {64, 64}), W4 joint split of 56,
    INT var nearest-integer rounding."""
    sp = fi.paper_example_space()
    for xv, exp in GOLD["rounding_W3"]["cases"]:
        y = np.array([[math.log(xv)], [0.0]], dtype=np.float32)
        assert fo.round_schedules(sp, y)[0, 0] == exp
    # single-var closed form: round up iff x >= sqrt(d_i d_{i+1})
    divs = [1, 2, 4, 8, 16, 32, 64]
    xs = np.exp(np.linspace(-1, 5, 997))
    y = np.stack([np.log(xs), np.zeros_like(xs)]).astype(np.float32)
    got = fo.round_schedules(sp, y)[:, 0]
    for x, gv in zip(np.exp(y[0].astype(np.float64)), got):
        exp = divs[0]
        for a, bnext in zip(divs[:-1], divs[1:]):
            if math.log(x) > 0.5 * (math.log(a) + math.log(bnext)):
                exp = bnext
        assert gv == exp
    w4 = GOLD["rounding_W4"]
    sp4 = fi.Space("w4", [fi.Var("f1", fi.VAR_SPLIT, 1, 56), fi.Var("f2", fi.VAR_SPLIT, 1, 56)],
                   [fi.Split(56, [0, 1])], np.zeros(0, dtype=fi.NODE_DTYPE), np.zeros(0, np.int32), np.zeros(0, np.int32))
    assert len(fo.component_tuples(sp4, [0, 1])) == w4["n_tuples"]
    y = np.log(np.array([[w4["x"][0]], [w4["x"][1]]])).astype(np.float32)
    assert list(fo.round_schedules(sp4, y)[0]) == w4["joint"]
    for xv, exp in GOLD["rounding_int"]["cases"]:
        y = np.array([[0.0], [math.log(xv)]], dtype=np.float32)
        assert fo.round_schedules(sp, y)[0, 1] == exp


def test_components_and_tuple_counts():
    """Known counts of ordered factor tuples: 3 factors of 64 -> C(9,3)=84; of 56 = 2^3*7 -> 20*4=80."""
    sp = fi.c2_space()
    comps = fo.components(sp)
    assert [len(c) for c in comps] == [3, 3, 3, 2]
    counts = [len(fo.component_tuples(sp, c)) for c in comps]
    assert counts == [84, 80, 80, 28]


# ----------------------------------------------------------------------------- sampler / top-k / search
def test_init_sampler_feasible_and_deterministic():
    sp = fi.c2_space()
    y = fo.init_sample(sp, 512, 0x5EED0002)
    g = np.concatenate([fo.eval_dag(sp, np.exp(y.astype(np.float64)), True).g_user,
                        fo.auto_roots(sp, y.astype(np.float64))])
    assert np.all(g <= 1e-6)
    assert np.array_equal(y, fo.init_sample(sp, 512, 0x5EED0002))
    # candidates are independent of the batch they are drawn in (counter-based)
    assert np.array_equal(y[:, 100:110], fo.init_sample(sp, 10, 0x5EED0002, index_base=100))
    # not degenerate: most candidates leave the all-ones fallback
    assert np.mean(np.all(y == 0, axis=0)) < 0.05


def test_counter_uniform_distribution():
    u = fo.counter_uniform(1234, np.arange(200000), 3, 5)
    assert 0 <= u.min() and u.max() < 1
    hist, _ = np.histogram(u, bins=20, range=(0, 1))
    assert np.all(np.abs(hist - 10000) < 600)


def test_topk_dedup_and_order_vs_stable_sort():
    c = fi.config("C1")
    sp = c.spaces[0]
    mlp = fi.make_mlp(c.mlp_dims)
    y = fi.make_y0(sp, 300, seed=5)
    y[:, 150:] = y[:, :150]          # duplicates -> dedup keeps the smaller index
    idx, sc, sched = fo.round_topk(sp, mlp.W, mlp.b, y, 16, index_base=1000)
    assert len(idx) == 16 and np.all(idx < 1150)
    full = fo.round_schedules(sp, y)
    valid = fo.validate(sp, full)
    scores = fo.score(sp, mlp.W, mlp.b, full)
    seen, ref = set(), []
    for i in sorted(range(300), key=lambda i: (-scores[i], i)):      # library stable sort
        if valid[i] and tuple(full[i]) not in seen:
            seen.add(tuple(full[i]))
            ref.append(1000 + i)
    assert list(idx) == ref[:16]


def test_search_decreases_loss_and_beats_random():
    """Sanity only (parity unpinned vs the paper's numbers): Alg. 1 on C1 lowers the mean loss and
    its best predicted score beats the best of 1600 random valid samples."""
    c = fi.config("C1")
    sp = c.spaces[0]
    mlp = fi.make_mlp(c.mlp_dims)
    y0 = fo.init_sample(sp, 64, c.rng_seed)
    l0 = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), c.lam, with_grad=False).loss
    y, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 60, c.lr, c.lam)
    l1 = fo.objective(sp, mlp.W, mlp.b, y, c.lam, with_grad=False).loss
    assert np.mean(l1) < np.mean(l0)
    _, sc, _ = fo.round_topk(sp, mlp.W, mlp.b, y.astype(np.float32), 16)
    yr = fo.init_sample(sp, 1600, 99)
    _, scr, _ = fo.round_topk(sp, mlp.W, mlp.b, yr, 1)
    assert sc[0] >= scr[0] - 1e-9


def _history_setup(n=60, steps=6):
    c = fi.config("C1")
    sp = c.spaces[0]
    mlp = fi.make_mlp(c.mlp_dims)
    y0 = fo.init_sample(sp, n, c.rng_seed)
    _, _, _, hist = fo.search(sp, mlp.W, mlp.b, y0, steps, c.lr, c.lam, history=True)
    return sp, mlp, [h[0].astype(np.float32) for h in hist]


def test_history_topk_single_step_is_round_topk():
    """Alg. 1 l.20-21 over a one-entry history = final-point rounding of that entry (round_topk)."""
    sp, mlp, ys = _history_setup()
    idx, step, sc, sched, _ = fo.round_topk_history(sp, mlp.W, mlp.b, ys[:1], 16, index_base=500)
    ridx, rsc, rsched = fo.round_topk(sp, mlp.W, mlp.b, ys[0], 16, index_base=500)
    assert np.all(step == 0)
    assert np.array_equal(idx, ridx) and np.array_equal(sc, rsc) and np.array_equal(sched, rsched)


def test_history_topk_equals_round_topk_of_concatenated_points():
    """The history as one population: point (step i, seed s) -> column i*n + s.  Ordering by
    (step, seed) is ordering by that column index, so dedup (first visit) and the (score, index)
    order coincide with round_topk on the concatenation."""
    sp, mlp, ys = _history_setup()
    n = ys[0].shape[1]
    idx, step, sc, sched, n_unique = fo.round_topk_history(sp, mlp.W, mlp.b, ys, 32)
    cat = np.concatenate(ys, axis=1)
    cidx, csc, csched = fo.round_topk(sp, mlp.W, mlp.b, cat, 32)
    assert np.array_equal(idx, cidx % n) and np.array_equal(step, cidx // n)
    assert np.array_equal(sc, csc) and np.array_equal(sched, csched)
    assert n_unique == len({r.tobytes() for r in fo.round_schedules(sp, cat)})


def test_history_topk_monotone_and_revisits_add_nothing():
    sp, mlp, ys = _history_setup()
    best = [fo.round_topk_history(sp, mlp.W, mlp.b, ys[:t], 1)[2][0] for t in range(1, len(ys) + 1)]
    assert all(b1 >= b0 for b0, b1 in zip(best, best[1:]))              # more history never hurts
    perm = ys[0][:, ::-1].copy()                                        # same points, other seeds, later step
    a = fo.round_topk_history(sp, mlp.W, mlp.b, ys[:1], 16)
    b = fo.round_topk_history(sp, mlp.W, mlp.b, ys[:1] + [perm], 16)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) and a[4] == b[4]


def test_subgraph_topk_equals_bruteforce_over_all_sketches():
    """Eq. 3's max over programs: merging the per-sketch top-k lists equals ranking every valid
    rounded point of every sketch (dedup within a sketch only) in one sort."""
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    sks = fi.c2_sketches()
    ys = [fi.make_y0(sp, 120, seed=40 + i) for i, sp in enumerate(sks)]
    per = [fo.round_topk(sp, mlp.W, mlp.b, y, 8) for sp, y in zip(sks, ys)]
    got = fo.subgraph_topk(per, 8)
    allrec = []
    for i, (sp, y) in enumerate(zip(sks, ys)):
        sched = fo.round_schedules(sp, y)
        ok = fo.validate(sp, sched)
        sc = fo.score(sp, mlp.W, mlp.b, sched)
        seen = set()
        for s in range(y.shape[1]):
            if ok[s] and np.isfinite(sc[s]) and sched[s].tobytes() not in seen:
                seen.add(sched[s].tobytes())
                allrec.append((i, s, sc[s]))
    allrec.sort(key=lambda r: (-r[2], r[0], r[1]))
    assert [(r[0], r[1]) for r in got] == [(r[0], r[1]) for r in allrec[:8]]
    assert [r[2] for r in got] == [r[2] for r in allrec[:8]]


def test_segment_sum_cost_and_gradient():
    """Two-statement C2 space: C = MLP(phi_S0) + MLP(phi_S1) checked against the plain MLP on each
    block and against the torch float64 MLP on the summed outputs; the search gradient of the
    two-statement objective against central finite differences."""
    sp = build_space(conv2d_spec("c2_two_stmt", 64, 56, 56, 64, 3, 3, 1), statements=2)
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    y = fi.make_y0(sp, 6, seed=3).astype(np.float64)
    ob = fo.objective(sp, mlp.W, mlp.b, y, 1.0)
    c0, _ = fo.mlp_forward(mlp.W, mlp.b, ob.phi[:82])
    c1, _ = fo.mlp_forward(mlp.W, mlp.b, ob.phi[82:])
    assert np.allclose(ob.c, c0 + c1, rtol=0, atol=1e-12)
    net = torch.nn.Sequential(*[m for l in range(len(mlp.W)) for m in
                                ([torch.nn.Linear(mlp.W[l].shape[1], mlp.W[l].shape[0]).double()] +
                                 ([torch.nn.ReLU()] if l < len(mlp.W) - 1 else []))])
    with torch.no_grad():
        for l, lin in enumerate([m for m in net if isinstance(m, torch.nn.Linear)]):
            lin.weight.copy_(torch.from_numpy(mlp.W[l].astype(np.float64)))
            lin.bias.copy_(torch.from_numpy(mlp.b[l].astype(np.float64)))
        ref = (net(torch.from_numpy(ob.phi[:82].T.copy())) + net(torch.from_numpy(ob.phi[82:].T.copy()))).numpy()[:, 0]
    assert np.allclose(ob.c, ref, rtol=1e-12, atol=1e-12)
    h = 1e-6
    for j in range(sp.n_vars):
        yp, ym = y.copy(), y.copy()
        yp[j] += h
        ym[j] -= h
        fd = (fo.objective(sp, mlp.W, mlp.b, yp, 1.0, with_grad=False).loss
              - fo.objective(sp, mlp.W, mlp.b, ym, 1.0, with_grad=False).loss) / (2 * h)
        assert np.allclose(ob.grad[j], fd, rtol=1e-4, atol=1e-6 * np.max(np.abs(fd)) + 1e-8), (j, ob.grad[j], fd)
