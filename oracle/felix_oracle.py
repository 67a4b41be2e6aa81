"""Felix hot-path ORACLE — plain, slow, obviously-correct float64 CPU implementation.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` leg may import this module.  It shares no code with the CUDA path
(paper_conf_asplos_zhaosam24_b200/); both consume the same input arrays from felix_inputs/.

Every function cites the PAPER.md passage it follows ("P:Lnnn").  Where the paper is silent or
garbled, the reading taken is the one of SURVEY.md §8(c), listed in DESIGN.md "Readings".

Pins (tests/test_oracle_*.py, run with -m "not gpu"):
  * hard features at integer points == brute-force loop-nest enumeration (tests/sim/loopnest.py)
  * paper's Dense-Add s*1 formulas and golden values (tests/golden/paper_dense_add.json)
  * smooth-op closed forms (R(0)=S(0)=1/2, R'=S, tail bounds, Fig. 4 ranges)
  * reverse-mode gradient == central finite differences (fp64)
  * MLP forward / input-gradient == torch.nn.Linear/ReLU float64 autograd (library routine)
  * Adam == torch.optim.Adam float64 (library routine)
  * rounding == exhaustive enumeration of all valid configurations (tiny spaces) and the
    single-variable geometric-mean closed form
  * top-k == stable sort (library routine)
parity unpinned: the whole-search trajectory against the paper's own numbers (needs TVM, trained
weights and the paper's GPUs) — only sanity properties are checked (loss decreases, etc.).
"""
from __future__ import annotations

import math
from dataclasses import dataclass
from itertools import product as _iproduct
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

# opcodes of the input format (include/felix.h felix_op; felix_inputs/dag.py)
OP_CONST, OP_VAR, OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_NEG, OP_POW = 0, 1, 2, 3, 4, 5, 6, 7
OP_EXP, OP_LOG, OP_SQRT, OP_MIN, OP_MAX, OP_SELECT = 8, 9, 10, 11, 12, 13
OP_GT, OP_GE, OP_LT, OP_LE, OP_EQ, OP_NE, OP_AND, OP_OR, OP_NOT = 14, 15, 16, 17, 18, 19, 20, 21, 22
OP_FLOORDIV, OP_CEILDIV = 23, 24
VAR_SPLIT, VAR_INT = 0, 1

LN2 = math.log(2.0)
VALID_TOL = 1e-9   # reading R-valid: a hard constraint holds iff g <= 1e-9 (absorbs 1-ulp libm noise)


# =============================================================================== O3 smoothing
# f_smooth(x) := integral f(x - t) phi(t) dt with a heavy-tailed kernel "more numerically
# stable compared to ... Gaussian or bump".  The printed kernel 1/sqrt(1+t^2) is not integrable
# (garbled); reading: phi(t) = 1/2 (1+t^2)^(-3/2), which gives
#   S(t) = (H * phi)(t)    = 1/2 (1 + t / sqrt(1+t^2))      smooth step
#   R(t) = (relu * phi)(t) = 1/2 (t + sqrt(1+t^2))          smooth ReLU,   R' = S,  S' = phi.
# Evaluated in cancellation-free forms (reading R-stable).

def _hyp(t: np.ndarray) -> np.ndarray:
    """sqrt(1 + t^2) without overflow for large |t|."""
    a = np.abs(t)
    with np.errstate(over="ignore", invalid="ignore", divide="ignore"):
        big = a > 1.0
        safe = np.where(big, a, 1.0)
        return np.where(big, a * np.sqrt(1.0 + (1.0 / safe) ** 2), np.sqrt(1.0 + t * t))


def smooth_S(t: np.ndarray) -> np.ndarray:
    t = np.asarray(t, dtype=np.float64)
    h = _hyp(t)
    a = np.abs(t)
    with np.errstate(over="ignore"):
        tail = 1.0 / (2.0 * h * (h + a))      # = 1/2 (1 - |t|/h), no cancellation
    return np.where(t >= 0.0, 1.0 - tail, tail)


def smooth_dS(t: np.ndarray) -> np.ndarray:
    t = np.asarray(t, dtype=np.float64)
    h = _hyp(t)
    with np.errstate(over="ignore"):
        return 0.5 / (h * h * h)


def smooth_R(t: np.ndarray) -> np.ndarray:
    t = np.asarray(t, dtype=np.float64)
    return np.where(t >= 0.0, t, 0.0) + smooth_Rgap(t)


def smooth_Rgap(t: np.ndarray) -> np.ndarray:
    """R(t) - relu(t) = 1/2 (sqrt(1+t^2) - |t|) = 1 / (2 (sqrt(1+t^2) + |t|))  (> 0, <= 1/2)."""
    t = np.asarray(t, dtype=np.float64)
    h = _hyp(t)
    return 1.0 / (2.0 * (h + np.abs(t)))


def smooth_min(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    """min(a,b) smoothed = a - R(a-b) (rule table O3), evaluated without the cancellation of
    a - (a - b): for t = a - b >= 0 it is b - gap(t), else a - gap(t) (reading R-stable)."""
    t = a - b
    return np.where(t >= 0.0, b, a) - smooth_Rgap(t)


def smooth_max(a: np.ndarray, b: np.ndarray) -> np.ndarray:
    """max(a,b) smoothed = b + R(a-b) = (t >= 0 ? a : b) + gap(t)."""
    t = a - b
    return np.where(t >= 0.0, a, b) + smooth_Rgap(t)


# =============================================================================== forward evaluation
@dataclass
class Eval:
    vals: List[np.ndarray]        # node values, each float64 [B]
    F: np.ndarray                 # [K, B] feature formulas Feat_k(x)
    g_user: np.ndarray            # [R_user, B] user constraint functions


def _args(nd) -> Tuple[int, int, int, int, float]:
    return int(nd["op"]), int(nd["a"]), int(nd["b"]), int(nd["c"]), float(nd["imm"])


def eval_dag(space, x: np.ndarray, smooth: bool) -> Eval:
    """Evaluate the feature DAG at x [M, B] (float64).
    smooth=True : the rewritten differentiable formulas (rule table SURVEY §8(c) O3).
    smooth=False: hard semantics (exact comparisons, SELECT picks a branch, floor/ceil divisions) —
                  what TVM's extractor would report for the concrete program."""
    x = np.asarray(x, dtype=np.float64)
    B = x.shape[1]
    vals: List[np.ndarray] = []
    with np.errstate(all="ignore"):
        for nd in space.nodes:
            op, a, b, c, imm = _args(nd)
            if op == OP_CONST:
                v = np.full(B, imm)
            elif op == OP_VAR:
                v = x[int(imm)].copy()
            elif op == OP_ADD:
                v = vals[a] + vals[b]
            elif op == OP_SUB:
                v = vals[a] - vals[b]
            elif op == OP_MUL:
                v = vals[a] * vals[b]
            elif op == OP_DIV:
                v = vals[a] / vals[b]
            elif op == OP_NEG:
                v = -vals[a]
            elif op == OP_POW:
                v = np.power(vals[a], imm)
            elif op == OP_EXP:
                v = np.exp(vals[a])
            elif op == OP_LOG:
                v = np.log(vals[a])
            elif op == OP_SQRT:
                v = np.sqrt(vals[a])
            elif op == OP_MIN:
                v = smooth_min(vals[a], vals[b]) if smooth else np.minimum(vals[a], vals[b])
            elif op == OP_MAX:
                v = smooth_max(vals[a], vals[b]) if smooth else np.maximum(vals[a], vals[b])
            elif op in (OP_GT, OP_GE):
                if smooth:
                    v = smooth_S(vals[a] - vals[b])
                else:
                    v = (vals[a] > vals[b]) if op == OP_GT else (vals[a] >= vals[b])
                    v = v.astype(np.float64)
            elif op in (OP_LT, OP_LE):
                if smooth:
                    v = smooth_S(vals[b] - vals[a])
                else:
                    v = (vals[a] < vals[b]) if op == OP_LT else (vals[a] <= vals[b])
                    v = v.astype(np.float64)
            elif op in (OP_EQ, OP_NE):
                if smooth:
                    d = vals[a] - vals[b]
                    eq = smooth_S(d + 0.5) * smooth_S(0.5 - d)
                else:
                    eq = (vals[a] == vals[b]).astype(np.float64)
                v = eq if op == OP_EQ else 1.0 - eq
            elif op == OP_AND:
                v = vals[a] * vals[b]
            elif op == OP_OR:
                v = vals[a] + vals[b] - vals[a] * vals[b]
            elif op == OP_NOT:
                v = 1.0 - vals[a]
            elif op == OP_SELECT:
                cond = vals[a] if smooth else (vals[a] != 0.0).astype(np.float64)
                v = vals[c] + (vals[b] - vals[c]) * cond
                if not smooth:
                    v = np.where(vals[a] != 0.0, vals[b], vals[c])
            elif op == OP_FLOORDIV:
                v = vals[a] / vals[b] if smooth else np.floor(vals[a] / vals[b])
            elif op == OP_CEILDIV:
                v = vals[a] / vals[b] if smooth else np.ceil(vals[a] / vals[b])
            else:
                raise ValueError(f"bad opcode {op}")
            vals.append(np.asarray(v, dtype=np.float64))
    F = np.stack([vals[int(r)] for r in space.feature_roots]) if len(space.feature_roots) else np.zeros((0, B))
    G = np.stack([vals[int(r)] for r in space.constraint_roots]) if len(space.constraint_roots) else np.zeros((0, B))
    return Eval(vals, F, G)


# =============================================================================== O2 validity roots
def auto_roots(space, y: np.ndarray) -> np.ndarray:
    """Automatic penalty functions in log space (reading O2):
       SPLIT var j:   -y_j <= 0                    (x >= 1, "value 1 = no-op" L1009-1010)
       split s:        sum_{j in s} y_j - ln(extent_s) <= 0     (N mod x = 0  ->  y <= ln N, L791-797)
       INT var j:      ln(lo_j) - y_j <= 0,  y_j - ln(hi_j) <= 0
    Order: SPLIT vars (var order), splits (split order), INT vars (lo, hi per var)."""
    y = np.asarray(y, dtype=np.float64)
    rows = []
    for j, v in enumerate(space.vars):
        if v.kind == VAR_SPLIT:
            rows.append(-y[j])
    for s in space.splits:
        acc = np.zeros(y.shape[1])
        for j in s.vars:
            acc = acc + y[j]
        rows.append(acc - math.log(s.extent))
    for j, v in enumerate(space.vars):
        if v.kind == VAR_INT:
            rows.append(math.log(v.lo) - y[j])
            rows.append(y[j] - math.log(v.hi))
    return np.stack(rows) if rows else np.zeros((0, y.shape[1]))


def n_constraints(space) -> int:
    n_split = sum(1 for v in space.vars if v.kind == VAR_SPLIT)
    n_int = sum(1 for v in space.vars if v.kind == VAR_INT)
    return len(space.constraint_roots) + n_split + len(space.splits) + 2 * n_int


# =============================================================================== O4 slog features
def slog(F: np.ndarray) -> np.ndarray:
    """Log of the smooth features ("Felix takes logarithm of the smooth program
    features"); reading O4: sign(F) log2(1 + |F|) (defined at F = 0, C^1)."""
    return np.sign(F) * np.log2(1.0 + np.abs(F))


def slog_prime(F: np.ndarray) -> np.ndarray:
    return 1.0 / ((1.0 + np.abs(F)) * LN2)


# =============================================================================== O5 cost model
def mlp_forward(W: Sequence[np.ndarray], b: Sequence[np.ndarray], phi: np.ndarray):
    """C(phi): h0 = phi, z_l = W_l h_{l-1} + b_l, h_l = relu(z_l) (l < L), c = z_L  (TenSet MLP,
    P:L1056-1059).  phi: [K, B].  Returns c [B] and the pre-activations z_l [d_l, B] (l < L)."""
    h = np.asarray(phi, dtype=np.float64)
    zs = []
    L = len(W)
    for l in range(L):
        z = np.asarray(W[l], dtype=np.float64) @ h + np.asarray(b[l], dtype=np.float64)[:, None]
        if l < L - 1:
            zs.append(z)
            h = np.maximum(z, 0.0)
        else:
            h = z
    return h[0], zs


def mlp_input_grad(W: Sequence[np.ndarray], zs: Sequence[np.ndarray], dc: np.ndarray) -> np.ndarray:
    """Back-propagation to the input only (the weights are fixed during the search):
    delta_L = dc;  delta_{l-1} = W_l^T delta_l (.) [z_{l-1} > 0];  dphi = W_1^T delta_1.
    relu'(0) = 0 as in PyTorch."""
    L = len(W)
    delta = np.asarray(dc, dtype=np.float64)[None, :]
    for l in range(L - 1, -1, -1):
        delta = np.asarray(W[l], dtype=np.float64).T @ delta
        if l > 0:
            delta = delta * (zs[l - 1] > 0.0)
    return delta


def segment_sum_forward(W: Sequence[np.ndarray], b: Sequence[np.ndarray], phi: np.ndarray):
    """TenSet-style cost over per-statement feature vectors (per-statement feature
    examples P:L668-671): phi [S*K0, B] statement-major, C = sum_s MLP(phi_s).  S = 1 is mlp_forward.
    Returns c [B] and the per-statement pre-activation lists."""
    K0 = np.asarray(W[0]).shape[1]
    S = phi.shape[0] // K0
    assert S * K0 == phi.shape[0]
    c, zs_all = None, []
    for s in range(S):
        cs, zs = mlp_forward(W, b, phi[s * K0:(s + 1) * K0])
        c = cs if c is None else c + cs
        zs_all.append(zs)
    return c, zs_all


def segment_sum_input_grad(W: Sequence[np.ndarray], zs_all, dc: np.ndarray) -> np.ndarray:
    """dC/dphi of segment_sum_forward: each statement's MLP input gradient (dC/dc_s = dC/dc)."""
    return np.concatenate([mlp_input_grad(W, zs, dc) for zs in zs_all], axis=0)


# =============================================================================== O6/O7 objective + grad
@dataclass
class Objective:
    x: np.ndarray          # [M, B]
    F: np.ndarray          # [K, B]
    phi: np.ndarray        # [K, B]
    g: np.ndarray          # [R, B]  user roots then auto roots
    c: np.ndarray          # [B]     predicted performance (higher = better)
    loss: np.ndarray       # [B]
    grad: np.ndarray       # [M, B]  dLoss/dy
    zs: list               # MLP pre-activations
    dphi: np.ndarray       # [K, B]


def objective(space, W, b, y: np.ndarray, lam: float, with_grad: bool = True) -> Objective:
    """Per-candidate Eq. 4:  L = -C(Feat(x)) + lambda * sum_r max(g_r(x), 0)^2,
    with x = e^y.  The sum over seeds decouples (one term per candidate).
    Gradient by reverse mode (Alg. 1 line 18 AutoDiff):
      adj(F_k) = dphi_k * slog'(F_k),  adj(g_r) = 2 lambda max(g_r, 0),  dL/dy_j = x_j adj(x_j)."""
    y = np.asarray(y, dtype=np.float64)
    with np.errstate(all="ignore"):
        x = np.exp(y)
    ev = eval_dag(space, x, smooth=True)
    g = np.concatenate([ev.g_user, auto_roots(space, y)], axis=0)
    phi = slog(ev.F)
    c, zs_all = segment_sum_forward(W, b, phi)                # one statement unless the space has S of them
    zs = [z for zst in zs_all for z in zst]
    with np.errstate(all="ignore"):
        pen = np.maximum(g, 0.0)
        loss = -c + lam * np.sum(pen * pen, axis=0)
    if not with_grad:
        return Objective(x, ev.F, phi, g, c, loss, None, zs, None)
    dphi = segment_sum_input_grad(W, zs_all, -np.ones_like(c))   # dL/dc = -1
    with np.errstate(all="ignore"):
        seedF = dphi * slog_prime(ev.F)
        seedG = 2.0 * lam * pen
    grad_x = reverse_sweep(space, ev.vals, seedF, seedG[: len(space.constraint_roots)])
    with np.errstate(all="ignore"):
        grad = x * grad_x
    # auto roots are functions of y directly
    gy = _auto_roots_grad(space, seedG[len(space.constraint_roots):], y.shape[1])
    grad = grad + gy
    return Objective(x, ev.F, phi, g, c, loss, grad, zs, dphi)


def _auto_roots_grad(space, seed: np.ndarray, B: int) -> np.ndarray:
    gy = np.zeros((space.n_vars, B))
    r = 0
    for j, v in enumerate(space.vars):
        if v.kind == VAR_SPLIT:
            gy[j] -= seed[r]
            r += 1
    for s in space.splits:
        for j in s.vars:
            gy[j] += seed[r]
        r += 1
    for j, v in enumerate(space.vars):
        if v.kind == VAR_INT:
            gy[j] -= seed[r]
            gy[j] += seed[r + 1]
            r += 2
    return gy


def reverse_sweep(space, vals: List[np.ndarray], seedF: np.ndarray, seedG: np.ndarray) -> np.ndarray:
    """Reverse-mode adjoints of the smoothed DAG in reverse topological order; returns adj(x_j) [M, B]."""
    n = len(space.nodes)
    B = vals[0].shape[0] if n else seedF.shape[1]
    adj = [np.zeros(B) for _ in range(n)]
    for k, r in enumerate(space.feature_roots):
        adj[int(r)] = adj[int(r)] + seedF[k]
    for k, r in enumerate(space.constraint_roots):
        adj[int(r)] = adj[int(r)] + seedG[k]
    gx = np.zeros((space.n_vars, B))
    with np.errstate(all="ignore"):
        for i in range(n - 1, -1, -1):
            op, a, b, c, imm = _args(space.nodes[i])
            g = adj[i]
            if op == OP_CONST:
                continue
            if op == OP_VAR:
                gx[int(imm)] += g
                continue
            if not np.any(g != 0.0):
                continue
            if op == OP_ADD:
                adj[a] = adj[a] + g; adj[b] = adj[b] + g
            elif op == OP_SUB:
                adj[a] = adj[a] + g; adj[b] = adj[b] - g
            elif op == OP_MUL:
                adj[a] = adj[a] + g * vals[b]; adj[b] = adj[b] + g * vals[a]
            elif op == OP_DIV:
                adj[a] = adj[a] + g / vals[b]
                adj[b] = adj[b] - g * vals[a] / (vals[b] * vals[b])
            elif op == OP_NEG:
                adj[a] = adj[a] - g
            elif op == OP_POW:
                adj[a] = adj[a] + g * imm * np.power(vals[a], imm - 1.0)
            elif op == OP_EXP:
                adj[a] = adj[a] + g * vals[i]
            elif op == OP_LOG:
                adj[a] = adj[a] + g / vals[a]
            elif op == OP_SQRT:
                adj[a] = adj[a] + g * 0.5 / vals[i]
            elif op == OP_MAX:      # b + R(a - b)
                s = smooth_S(vals[a] - vals[b])
                adj[a] = adj[a] + g * s; adj[b] = adj[b] + g * (1.0 - s)
            elif op == OP_MIN:      # a - R(a - b)
                s = smooth_S(vals[a] - vals[b])
                adj[a] = adj[a] + g * (1.0 - s); adj[b] = adj[b] + g * s
            elif op in (OP_GT, OP_GE):   # S(a - b)
                d = g * smooth_dS(vals[a] - vals[b])
                adj[a] = adj[a] + d; adj[b] = adj[b] - d
            elif op in (OP_LT, OP_LE):   # S(b - a)
                d = g * smooth_dS(vals[b] - vals[a])
                adj[a] = adj[a] - d; adj[b] = adj[b] + d
            elif op in (OP_EQ, OP_NE):   # S(d + 1/2) S(1/2 - d), d = a - b ; NE = 1 - EQ
                dd = vals[a] - vals[b]
                p, q = smooth_S(dd + 0.5), smooth_S(0.5 - dd)
                deq = smooth_dS(dd + 0.5) * q - p * smooth_dS(0.5 - dd)
                gg = g * deq if op == OP_EQ else -g * deq
                adj[a] = adj[a] + gg; adj[b] = adj[b] - gg
            elif op == OP_AND:
                adj[a] = adj[a] + g * vals[b]; adj[b] = adj[b] + g * vals[a]
            elif op == OP_OR:
                adj[a] = adj[a] + g * (1.0 - vals[b]); adj[b] = adj[b] + g * (1.0 - vals[a])
            elif op == OP_NOT:
                adj[a] = adj[a] - g
            elif op == OP_SELECT:   # c + (b' - c') * cond  with (cond, then, else) = (a, b, c)
                adj[a] = adj[a] + g * (vals[b] - vals[c])
                adj[b] = adj[b] + g * vals[a]
                adj[c] = adj[c] + g * (1.0 - vals[a])
            elif op in (OP_FLOORDIV, OP_CEILDIV):   # smoothed to a / b
                adj[a] = adj[a] + g / vals[b]
                adj[b] = adj[b] - g * vals[a] / (vals[b] * vals[b])
            else:
                raise ValueError(op)
    return gx


# =============================================================================== O8 Adam
def adam_step(y, m, v, grad, t: int, lr: float, beta1=0.9, beta2=0.999, eps=1e-8):
    """One Adam update (Kingma & Ba [17]; torch.optim.Adam defaults):
       m <- b1 m + (1-b1) g ;  v <- b2 v + (1-b2) g^2
       y <- y - (lr / (1 - b1^t)) * m / (sqrt(v) / sqrt(1 - b2^t) + eps)."""
    m = beta1 * m + (1.0 - beta1) * grad
    v = beta2 * v + (1.0 - beta2) * grad * grad
    bc1 = 1.0 - beta1 ** t
    bc2 = 1.0 - beta2 ** t
    y = y - (lr / bc1) * m / (np.sqrt(v) / math.sqrt(bc2) + eps)
    return y, m, v


def search(space, W, b, y0: np.ndarray, n_steps: int, lr: float = 0.05, lam: float = 1.0,
           beta1=0.9, beta2=0.999, eps=1e-8, history: bool = False):
    """Algorithm 1 lines 13-19: Adam on all nSeeds candidates for nSteps.
    Reading R-NaN: a candidate whose loss or gradient is non-finite is not updated that step."""
    y = np.asarray(y0, dtype=np.float64).copy()
    m = np.zeros_like(y)
    v = np.zeros_like(y)
    hist = []
    ob = None
    for t in range(1, n_steps + 1):
        ob = objective(space, W, b, y, lam)
        if history:
            hist.append((y.copy(), ob.loss.copy()))
        ok = np.isfinite(ob.loss) & np.all(np.isfinite(ob.grad), axis=0)
        g = np.where(ok[None, :], ob.grad, 0.0)
        y1, m1, v1 = adam_step(y, m, v, g, t, lr, beta1, beta2, eps)
        y = np.where(ok[None, :], y1, y)
        m = np.where(ok[None, :], m1, m)
        v = np.where(ok[None, :], v1, v)
    return y, m, v, hist


# =============================================================================== O9 init sampler
_GOLD = 0x9E3779B97F4A7C15
_M64 = (1 << 64) - 1


def _mix64(z):
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def counter_uniform(seed: int, cand: np.ndarray, attempt: int, var: int) -> np.ndarray:
    """Counter-based uniform in [0,1) (53 bits): splitmix64 finaliser chained over
    (seed, candidate, attempt, var).  Specified in include/felix.h; both sides implement it."""
    with np.errstate(over="ignore"):
        g = np.uint64(_GOLD)
        h = np.uint64(seed & _M64)
        h = _mix64(h + g * (np.asarray(cand, dtype=np.uint64) + np.uint64(1)))
        h = _mix64(h + g * np.uint64(attempt + 1))
        h = _mix64(h + g * np.uint64(var + 1))
    return (h >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)


def components(space) -> List[List[int]]:
    """Connected components of the var-split incidence graph (SPLIT vars only), var order."""
    parent = list(range(space.n_vars))

    def find(i):
        while parent[i] != i:
            parent[i] = parent[parent[i]]
            i = parent[i]
        return i
    for s in space.splits:
        for j in s.vars[1:]:
            parent[find(j)] = find(s.vars[0])
    comps: Dict[int, List[int]] = {}
    for j, v in enumerate(space.vars):
        if v.kind == VAR_SPLIT:
            comps.setdefault(find(j), []).append(j)
    return sorted(comps.values(), key=lambda c: c[0])


def init_sample(space, n: int, rng_seed: int, index_base: int = 0, max_attempts: int = 64) -> np.ndarray:
    """RandomInitSchedVars (Alg. 1 line 12): rejection sampling of starting points that
    satisfy every constraint.  Reading O9 (two-level rejection):
      for outer attempt a2 < 64:
        for each split component c: for a1 < 64: draw y_j = u * ln(ub_j) for j in c with
            u = counter_uniform(seed, cand, 64*a2 + a1, j); accept the first draw whose split roots
            are all <= 0 (else y_c = 0);
        INT vars: y_j = ln lo + u (ln hi - ln lo), u = counter_uniform(seed, cand, 64*a2, j)
        accept y if all user roots (smooth semantics) are <= 0
      fallback y = ln lo (every factor 1).   Returns float32 SoA [M][n]."""
    M = space.n_vars
    cand = np.arange(index_base, index_base + n, dtype=np.uint64)
    ub = np.zeros(M)
    for j, v in enumerate(space.vars):
        ub[j] = v.hi if v.kind == VAR_INT else min(s.extent for s in space.splits if j in s.vars)
    comps = components(space)
    comp_splits = [[s for s in space.splits if s.vars[0] in comp] for comp in comps]
    out = np.zeros((M, n))
    for j, v in enumerate(space.vars):
        out[j] = math.log(v.lo) if v.kind == VAR_INT else 0.0
    done = np.zeros(n, dtype=bool)
    for a2 in range(max_attempts):
        y = np.zeros((M, n))
        for comp, splits in zip(comps, comp_splits):
            acc = np.zeros(n, dtype=bool)
            for a1 in range(max_attempts):
                att = a2 * max_attempts + a1
                ys = {j: counter_uniform(rng_seed, cand, att, j) * math.log(ub[j]) for j in comp}
                ok = np.ones(n, dtype=bool)
                for s in splits:
                    tot = np.zeros(n)
                    for j in s.vars:
                        tot = tot + ys[j]
                    ok &= (tot - math.log(s.extent)) <= 0.0
                take = ok & ~acc
                for j in comp:
                    y[j] = np.where(take, ys[j], y[j])
                acc |= ok
                if acc.all():
                    break
        for j, v in enumerate(space.vars):
            if v.kind == VAR_INT:
                u = counter_uniform(rng_seed, cand, a2 * max_attempts, j)
                y[j] = math.log(v.lo) + u * (math.log(v.hi) - math.log(v.lo))
        with np.errstate(all="ignore"):
            ev = eval_dag(space, np.exp(y), smooth=True)
            ok = np.all(ev.g_user <= 0.0, axis=0) if ev.g_user.shape[0] else np.ones(n, dtype=bool)
        take = ok & ~done
        out[:, take] = y[:, take]
        done |= ok
        if done.all():
            break
    return out.astype(np.float32)


# =============================================================================== O10 rounding
def _divisors(n: int) -> List[int]:
    return [d for d in range(1, n + 1) if n % d == 0]


def component_tuples(space, comp: Sequence[int]) -> List[Tuple[int, ...]]:
    """All integer tuples (x_j, j in comp ascending) with every split's product dividing its
    extent, in lexicographic order."""
    splits = [s for s in space.splits if s.vars[0] in comp or any(j in comp for j in s.vars)]
    out: List[Tuple[int, ...]] = []

    def rec(k: int, rem: Dict[int, int], cur: List[int]):
        if k == len(comp):
            out.append(tuple(cur))
            return
        j = comp[k]
        mine = [si for si, s in enumerate(splits) if j in s.vars]
        g = 0
        for si in mine:
            g = math.gcd(g, rem[si])
        for d in _divisors(g):
            nrem = dict(rem)
            for si in mine:
                nrem[si] = rem[si] // d
            rec(k + 1, nrem, cur + [d])
    rec(0, {si: s.extent for si, s in enumerate(splits)}, [])
    return out


def round_schedules(space, y: np.ndarray) -> np.ndarray:
    """GetValidSchedules' rounding (Alg. 1 line 20): "Felix rounds y to the
    closest ln N_i where N_i is an integer factor of N".  Reading O10: per split component, the
    divisor-respecting tuple f minimising sum_j (y_j - ln f_j)^2 (float64, var order, no FMA; ties
    -> lexicographically smallest); INT var: x = lo + #{k in [lo, hi-1] : ln(k + 1/2) <= y}
    (nearest-integer rounding).  Returns int32 [B, M]."""
    y64 = np.asarray(y, dtype=np.float32).astype(np.float64)
    M, B = y64.shape
    sched = np.zeros((B, M), dtype=np.int32)
    for comp in components(space):
        tup = np.array(component_tuples(space, comp), dtype=np.int64)           # [T, |c|]
        lnf = np.array([[math.log(int(f)) for f in row] for row in tup])        # same libm as host
        acc = np.zeros((B, tup.shape[0]))
        for k, j in enumerate(comp):
            d = y64[j][:, None] - lnf[None, :, k]
            acc = acc + d * d
        best = np.argmin(acc, axis=1)         # first minimum == lexicographically smallest
        sched[:, comp] = tup[best]
    for j, v in enumerate(space.vars):
        if v.kind == VAR_INT:
            thr = np.array([math.log(k + 0.5) for k in range(v.lo, v.hi)])
            sched[:, j] = v.lo + np.sum(thr[None, :] <= y64[j][:, None], axis=1)
    return sched


def validate(space, sched: np.ndarray) -> np.ndarray:
    """Remove invalid rounded schedules (Alg. 1 line 20; "valid iff all g <= 0"):
    hard semantics at the integer point, float64; reading R-valid (g <= 1e-9) and finiteness."""
    x = sched.T.astype(np.float64)
    ev = eval_dag(space, x, smooth=False)
    with np.errstate(invalid="ignore"):
        ok = np.all(np.isfinite(ev.F), axis=0)
        if ev.g_user.shape[0]:
            ok &= np.all(np.isfinite(ev.g_user), axis=0) & np.all(ev.g_user <= VALID_TOL, axis=0)
    return ok


def score(space, W, b, sched: np.ndarray) -> np.ndarray:
    """Predicted performance of a concrete schedule: C(slog(Feat_hard(x_int))) in float64
    (TopNSchedulesByPredPerf, Alg. 1 line 21)."""
    x = sched.T.astype(np.float64)
    ev = eval_dag(space, x, smooth=False)
    phi = slog(ev.F)
    # A score is a function of its schedule alone (the top-k order and its shard invariance,
    # SURVEY §8(e), depend on that): the MLP runs on one candidate column at a time, because a
    # batched BLAS matmul may sum in a different order for different batch shapes.
    c = np.empty(phi.shape[1], dtype=np.float64)
    for i in range(phi.shape[1]):
        c[i] = segment_sum_forward(W, b, phi[:, i:i + 1])[0][0]
    return c


def round_topk(space, W, b, y: np.ndarray, k: int, index_base: int = 0):
    """Rounding -> validity -> dedup -> top-k by (score desc, global index asc) (P:L919-920,
    P:L928-935).  Returns (idx int64 [n], score f64 [n], sched int32 [n, M])."""
    sched = round_schedules(space, y)
    valid = validate(space, sched)
    sc = score(space, W, b, sched)
    B = sched.shape[0]
    gidx = index_base + np.arange(B, dtype=np.int64)
    keep = valid & np.isfinite(sc)
    seen = {}
    for i in np.nonzero(keep)[0]:
        key = sched[i].tobytes()
        if key not in seen:
            seen[key] = i                     # smallest global index (ascending scan)
    uniq = np.array(sorted(seen.values()), dtype=np.int64)
    if len(uniq) == 0:
        return np.zeros(0, np.int64), np.zeros(0), np.zeros((0, space.n_vars), np.int32)
    order = sorted(uniq.tolist(), key=lambda i: (-sc[i], gidx[i]))
    sel = np.array(order[:k], dtype=np.int64)
    return gidx[sel], sc[sel], sched[sel]


def subgraph_topk(per_sketch, k: int):
    """Eq. 3: the best schedules of a subgraph are the best over all its symbolic programs
    p*_i.  per_sketch[i] = (idx, score, sched) = round_topk of sketch i (distinct schedules of one
    program).  Schedules of different programs are different programs, so there is no cross-sketch
    dedup, and the global top-k lies in the union of the per-sketch top-k lists.  Order: (score desc,
    sketch asc, global index asc).  Returns a list of (sketch, idx, score, sched)."""
    recs = []
    for i, (idx, sc, sched) in enumerate(per_sketch):
        recs += [(i, int(idx[r]), float(sc[r]), np.asarray(sched[r])) for r in range(len(idx))]
    recs.sort(key=lambda r: (-r[2], r[0], r[1]))
    return recs[:k]


def round_topk_history(space, W, b, ys: Sequence[np.ndarray], k: int, index_base: int = 0):
    """Algorithm 1 lines 20-21 over varValuesHistory (lines 13, 17; "takes all
    the variable values traversed in the optimization process, rounds them to integers ... removes
    invalid rounded schedules ... takes the best nMeasure schedules").  ys[i] is sigma_x at which step
    i's objective was evaluated.  Every point is rounded, validated and scored exactly as round_topk;
    a schedule visited several times counts once, with its first (step, global index); the best k are
    returned by (score desc, step asc, global index asc).
    Returns (idx int64 [m], step int32 [m], score f64 [m], sched int32 [m, M], n_unique)."""
    first = {}                                   # schedule bytes -> (step, seed, score, valid, sched)
    for i, y in enumerate(ys):
        sched = round_schedules(space, y)
        valid = validate(space, sched)
        sc = score(space, W, b, sched)
        for s in range(sched.shape[0]):          # ascending (step, seed): the first visit is kept
            key = sched[s].tobytes()
            if key not in first:
                first[key] = (i, s, sc[s], bool(valid[s]) and bool(np.isfinite(sc[s])), sched[s].copy())
    n_unique = len(first)
    recs = [r for r in first.values() if r[3]]
    recs.sort(key=lambda r: (-r[2], r[0], r[1]))
    recs = recs[:k]
    M = space.n_vars
    idx = np.array([index_base + r[1] for r in recs], dtype=np.int64)
    step = np.array([r[0] for r in recs], dtype=np.int32)
    scr = np.array([r[2] for r in recs], dtype=np.float64)
    sch = np.array([r[4] for r in recs], dtype=np.int32).reshape(len(recs), M)
    return idx, step, scr, sch, n_unique
