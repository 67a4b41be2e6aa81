"""Feature-expression DAG format + a hash-consing builder.

This module defines the *input format* of a Felix search space — the thing the paper's analysis
pass hands to the optimizer: schedule variables x_j, the feature formulas Feat_k(x) over a fixed
operator set "+, -, *, /, pow, min, max, select, etc." (§3.3), and the
constraint functions g_r(x) <= 0 (L782-789).  It holds NO evaluation arithmetic (no smoothing, no
derivatives): both the oracle (oracle/) and the CUDA path (paper_conf_asplos_zhaosam24_b200) consume
the same node arrays.  Opcode values mirror `felix_op` in include/felix.h (a test checks this).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

# ---- opcodes (include/felix.h: felix_op) -------------------------------------------------------
OP_CONST, OP_VAR, OP_ADD, OP_SUB, OP_MUL, OP_DIV, OP_NEG, OP_POW = 0, 1, 2, 3, 4, 5, 6, 7
OP_EXP, OP_LOG, OP_SQRT, OP_MIN, OP_MAX, OP_SELECT = 8, 9, 10, 11, 12, 13
OP_GT, OP_GE, OP_LT, OP_LE, OP_EQ, OP_NE, OP_AND, OP_OR, OP_NOT = 14, 15, 16, 17, 18, 19, 20, 21, 22
OP_FLOORDIV, OP_CEILDIV = 23, 24
N_OPS = 25

OP_NAMES = {
    OP_CONST: "CONST", OP_VAR: "VAR", OP_ADD: "ADD", OP_SUB: "SUB", OP_MUL: "MUL", OP_DIV: "DIV",
    OP_NEG: "NEG", OP_POW: "POW", OP_EXP: "EXP", OP_LOG: "LOG", OP_SQRT: "SQRT", OP_MIN: "MIN",
    OP_MAX: "MAX", OP_SELECT: "SELECT", OP_GT: "GT", OP_GE: "GE", OP_LT: "LT", OP_LE: "LE",
    OP_EQ: "EQ", OP_NE: "NE", OP_AND: "AND", OP_OR: "OR", OP_NOT: "NOT", OP_FLOORDIV: "FLOORDIV",
    OP_CEILDIV: "CEILDIV",
}
ARITY = {OP_CONST: 0, OP_VAR: 0, OP_NEG: 1, OP_EXP: 1, OP_LOG: 1, OP_SQRT: 1, OP_NOT: 1, OP_POW: 1,
         OP_SELECT: 3}
BOOL_RESULT = {OP_GT, OP_GE, OP_LT, OP_LE, OP_EQ, OP_NE, OP_AND, OP_OR, OP_NOT}

VAR_SPLIT, VAR_INT = 0, 1

# numpy mirror of `felix_node` {int32 op, a, b, c; double imm}
NODE_DTYPE = np.dtype([("op", "<i4"), ("a", "<i4"), ("b", "<i4"), ("c", "<i4"), ("imm", "<f8")], align=True)


@dataclass
class Var:
    name: str
    kind: int            # VAR_SPLIT or VAR_INT
    lo: int = 1
    hi: int = 1


@dataclass
class Split:
    extent: int
    vars: List[int]      # product of x[vars] must divide extent


@dataclass
class Space:
    """One symbolic schedule s*_i of a subgraph: its variables, divisibility
    splits, feature DAG, K feature roots and user constraint roots g_r(x) <= 0."""
    name: str
    vars: List[Var]
    splits: List[Split]
    nodes: np.ndarray                # NODE_DTYPE[n]
    feature_roots: np.ndarray        # int32[K]
    constraint_roots: np.ndarray     # int32[R_user]
    feature_names: List[str] = field(default_factory=list)
    constraint_names: List[str] = field(default_factory=list)
    program: Optional[object] = None  # ProgramSpec for the brute-force simulator (tests)
    n_statements: int = 1            # feature_roots = n_statements per-statement vectors (statement-major)

    @property
    def n_vars(self) -> int:
        return len(self.vars)

    @property
    def n_features(self) -> int:
        return int(self.feature_roots.shape[0])


class DagBuilder:
    """Hash-consing builder: structurally identical sub-expressions share one node (CSE) and
    constant sub-expressions of + - * / are folded.  Nodes are appended in topological order."""

    def __init__(self) -> None:
        self.rows: List[Tuple[int, int, int, int, float]] = []
        self.memo: Dict[Tuple, int] = {}
        self.is_bool: List[bool] = []

    def _emit(self, op: int, a: int = -1, b: int = -1, c: int = -1, imm: float = 0.0) -> int:
        key = (op, a, b, c, float(imm))
        if op in (OP_ADD, OP_MUL, OP_MIN, OP_MAX, OP_EQ, OP_NE, OP_AND, OP_OR) and a > b >= 0:
            key = (op, b, a, c, float(imm))
            a, b = b, a
        hit = self.memo.get(key)
        if hit is not None:
            return hit
        idx = len(self.rows)
        self.rows.append((op, a, b, c, float(imm)))
        self.is_bool.append(op in BOOL_RESULT)
        self.memo[key] = idx
        return idx

    def const_value(self, i: int) -> Optional[float]:
        op, _, _, _, imm = self.rows[i]
        return imm if op == OP_CONST else None

    # ---- leaves
    def const(self, v: float) -> int:
        return self._emit(OP_CONST, imm=float(v))

    def var(self, j: int) -> int:
        return self._emit(OP_VAR, imm=float(j))

    # ---- arithmetic with constant folding of exact integer-valued constants
    def add(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(ca + cb)
        if ca == 0.0:
            return b
        if cb == 0.0:
            return a
        return self._emit(OP_ADD, a, b)

    def sub(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(ca - cb)
        if cb == 0.0:
            return a
        return self._emit(OP_SUB, a, b)

    def mul(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(ca * cb)
        if ca == 1.0:
            return b
        if cb == 1.0:
            return a
        if ca == 0.0 or cb == 0.0:
            return self.const(0.0)
        return self._emit(OP_MUL, a, b)

    def div(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None and cb != 0.0:
            return self.const(ca / cb)
        if cb == 1.0:
            return a
        return self._emit(OP_DIV, a, b)

    def prod(self, xs: Sequence[int]) -> int:
        out = self.const(1.0)
        for x in xs:
            out = self.mul(out, x)
        return out

    def sum(self, xs: Sequence[int]) -> int:
        out = self.const(0.0)
        for x in xs:
            out = self.add(out, x)
        return out

    def neg(self, a: int) -> int:
        return self._emit(OP_NEG, a)

    def pow(self, a: int, e: float) -> int:
        return self._emit(OP_POW, a, imm=float(e))

    def exp(self, a: int) -> int:
        return self._emit(OP_EXP, a)

    def log(self, a: int) -> int:
        return self._emit(OP_LOG, a)

    def sqrt(self, a: int) -> int:
        return self._emit(OP_SQRT, a)

    def min(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(min(ca, cb))
        return self._emit(OP_MIN, a, b)

    def max(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(max(ca, cb))
        return self._emit(OP_MAX, a, b)

    def select(self, c: int, a: int, b: int) -> int:
        if a == b:
            return a
        cc = self.const_value(c)
        if cc is not None:
            return a if cc != 0.0 else b
        return self._emit(OP_SELECT, c, a, b)

    def cmp(self, op: int, a: int, b: int) -> int:
        assert op in (OP_GT, OP_GE, OP_LT, OP_LE, OP_EQ, OP_NE)
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:   # fold: a constant condition is not a feature
            r = {OP_GT: ca > cb, OP_GE: ca >= cb, OP_LT: ca < cb, OP_LE: ca <= cb,
                 OP_EQ: ca == cb, OP_NE: ca != cb}[op]
            return self.const(1.0 if r else 0.0)
        return self._emit(op, a, b)

    def gt(self, a: int, b: int) -> int:
        return self.cmp(OP_GT, a, b)

    def le(self, a: int, b: int) -> int:
        return self.cmp(OP_LE, a, b)

    def land(self, a: int, b: int) -> int:
        return self._emit(OP_AND, a, b)

    def lor(self, a: int, b: int) -> int:
        return self._emit(OP_OR, a, b)

    def lnot(self, a: int) -> int:
        return self._emit(OP_NOT, a)

    def floordiv(self, a: int, b: int) -> int:
        return self._emit(OP_FLOORDIV, a, b)

    def ceildiv(self, a: int, b: int) -> int:
        ca, cb = self.const_value(a), self.const_value(b)
        if ca is not None and cb is not None:
            return self.const(float(math.ceil(ca / cb)))
        return self._emit(OP_CEILDIV, a, b)

    def nodes(self) -> np.ndarray:
        arr = np.zeros(len(self.rows), dtype=NODE_DTYPE)
        for i, (op, a, b, c, imm) in enumerate(self.rows):
            arr[i] = (op, a, b, c, imm)
        return arr


def prune(nodes: np.ndarray, roots: Sequence[np.ndarray]) -> Tuple[np.ndarray, List[np.ndarray]]:
    """Drop nodes unreachable from the roots; renumber (keeps topological order)."""
    live = np.zeros(len(nodes), dtype=bool)
    stack = [int(r) for rs in roots for r in rs]
    while stack:
        i = stack.pop()
        if live[i]:
            continue
        live[i] = True
        op = int(nodes[i]["op"])
        if op in (OP_CONST, OP_VAR):
            continue
        ar = ARITY.get(op, 2)
        for f in ("a", "b", "c")[:ar]:
            stack.append(int(nodes[i][f]))
    new_idx = -np.ones(len(nodes), dtype=np.int64)
    new_idx[live] = np.arange(int(live.sum()))
    out = nodes[live].copy()
    for i in range(len(out)):
        op = int(out[i]["op"])
        if op in (OP_CONST, OP_VAR):
            continue
        ar = ARITY.get(op, 2)
        for f in ("a", "b", "c")[:ar]:
            out[i][f] = new_idx[int(out[i][f])]
    return out, [new_idx[np.asarray(r, dtype=np.int64)].astype(np.int32) for r in roots]
