"""Synthetic symbolic programs: an Ansor-like GPU multi-level-tiling sketch of a tensor contraction
and the closed-form feature formulas of the tiled program (SUPPORT for the hot path).

PAPER.md §3.2-3.3 (L522-679): Felix applies a symbolic schedule s* (Tile / Annotation(blockIdx,
vthread, threadIdx) / CacheRead / Unroll with variable parameters, Fig. 3) to the subgraph
and extracts 82 feature formulas Feat_k(x) from the symbolic program.  Felix's real extractor needs
TVM (out of scope); this module builds the same *kind* of formulas for a fixed
sketch whose concrete loop nest is simple enough that every feature has an independent brute-force
definition (tests/sim/loopnest.py enumerates the concrete nest and must reproduce each formula
exactly at every valid integer point — the O-pin-1 check).

Sketch (per spatial axis i with extent E_i, per reduction axis j with extent K_j):
    blockIdx  b_i in [0, E_i / (V_i T_i I_i))          (fused over i)
      vthread   v_i in [0, V_i)
      threadIdx t_i in [0, T_i)
        for ro_j in [0, K_j / Rt_j)                      # outer reduction, CacheRead tiles per ro
          for rm_j in [0, RI1_j)          (2-var reduction axes only)
            for v_i ...                                  # vthread loop (virtual threads)
              for ri_j in [0, RI2_j | RI_j | K_j)
                for in_i in [0, I_i)
                  O[s] += A[...] * B[...]
    s_i = b_i*(V_i T_i I_i) + v_i*(T_i I_i) + t_i*I_i + in_i
    r_j = ro_j*Rt_j + rm_j*RI2_j + ri_j            (Rt_j = product of the axis' tile vars, or K_j)
Per-thread loop list L (outer -> inner): ro_*, rm_*, v_*, ri_*, in_*.

With statements=2 (TenSet-style per-statement features; the paper's feature
examples count one statement), the fused bias / activation epilogue is a statement of its
own, run by the same threads after the reduction:
            for v_i in [0, V_i):
              for in_i in [0, I_i):
                O[s] = act(O[s] + Bias[s_c])           (s_c = the spatial axis `bias_axis`)
Its epilogue loop list L_E is v_*, in_*; its read buffers are [Bias] (if any).  Both statements use
the same 82 feature definitions; the main statement then carries no epilogue op counts.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

from .dag import (DagBuilder, Space, Split, Var, VAR_INT, VAR_SPLIT, OP_EQ, prune)

N_FEATURES = 82          # "a total of 82 distinct features"
# Arithmetic of one reduction-statement instance (op-count features and flop counts):
#   "mad"      O[s] += A * B                    contraction (dense, bmm, conv)
#   "exp_sum"  O[s] += exp(A)                   softmax's exp-sum stage (Fig. 9 operator mix)
#   "sum_sq"   O1[s] += A; O2[s] += A * A       layernorm's mean / variance statistics
STMT_OPS = {"mad": {"mad": 1, "addsub": 0, "math": 0},
            "exp_sum": {"mad": 0, "addsub": 1, "math": 1},
            "sum_sq": {"mad": 1, "addsub": 1, "math": 0}}
STMT_FLOPS = {"mad": 2.0, "exp_sum": 2.0, "sum_sq": 3.0}
UNROLL_MAX = 1024        # Unroll(max_step=UNROLL0), Fig. 3 L584 / L599; search range [1, 1024]


@dataclass
class SAxis:
    name: str
    extent: int
    levels: str = "vti"      # which of vthread / thread / inner are schedule variables


@dataclass
class RAxis:
    name: str
    extent: int
    n_vars: int = 1          # 0: fully inner, 1: (outer, RI), 2: (outer, RI1, RI2)


@dataclass
class Buffer:
    name: str
    dims: List[List[Tuple[str, int]]]   # each dim: sum of coeff * axis_index


@dataclass
class ProgramSpec:
    name: str
    spatial: List[SAxis]
    reduction: List[RAxis]
    inputs: List[Buffer]
    bias: bool = False
    relu: bool = False
    gelu: bool = False
    unroll: bool = True
    bias_axis: str = ""        # spatial axis indexing the bias vector (epilogue statement's read buffer)
    smem_limit: int = 48 * 1024
    thread_limit: int = 1024
    local_limit: int = 256
    vthread_limit: int = 64
    stmt: str = "mad"          # reduction statement kind (STMT_OPS)

    def axis_extent(self, name: str) -> int:
        for a in self.spatial:
            if a.name == name:
                return a.extent
        for a in self.reduction:
            if a.name == name:
                return a.extent
        raise KeyError(name)

    def is_spatial(self, name: str) -> bool:
        return any(a.name == name for a in self.spatial)

    def buffer_shape(self, buf: Buffer) -> List[int]:
        shape = []
        for dim in buf.dims:
            shape.append(sum(c * (self.axis_extent(a) - 1) for a, c in dim) + 1 if dim else 1)
        return shape


# ------------------------------------------------------------------------------ variable layout
def var_layout(spec: ProgramSpec) -> Tuple[List[Var], List[Split], Dict[str, int]]:
    """Variables in a fixed order: per spatial axis V,T,I (as present), per reduction axis RI1,RI2
    (or RI), then UNROLL.  Each axis' vars form one divisibility split of its extent (L791-797)."""
    vars_: List[Var] = []
    splits: List[Split] = []
    index: Dict[str, int] = {}
    for ax in spec.spatial:
        ids = []
        for lv, tag in (("v", "V"), ("t", "T"), ("i", "I")):
            if lv in ax.levels:
                index[f"{tag}_{ax.name}"] = len(vars_)
                ids.append(len(vars_))
                vars_.append(Var(f"{tag}_{ax.name}", VAR_SPLIT, 1, ax.extent))
        if ids:
            splits.append(Split(ax.extent, ids))
    for ax in spec.reduction:
        ids = []
        names = [] if ax.n_vars == 0 else ([f"RI_{ax.name}"] if ax.n_vars == 1 else [f"RI1_{ax.name}", f"RI2_{ax.name}"])
        for nm in names:
            index[nm] = len(vars_)
            ids.append(len(vars_))
            vars_.append(Var(nm, VAR_SPLIT, 1, ax.extent))
        if ids:
            splits.append(Split(ax.extent, ids))
    if spec.unroll:
        index["UNROLL"] = len(vars_)
        vars_.append(Var("UNROLL", VAR_INT, 1, UNROLL_MAX))
    return vars_, splits, index


# ------------------------------------------------------------------------------ feature formulas
class _Ctx:
    def __init__(self, spec: ProgramSpec, b: DagBuilder, index: Dict[str, int]):
        self.spec, self.b, self.index = spec, b, index

    def v(self, name: str) -> int:
        """Node for var `name`, or constant 1 if the level is not a schedule variable."""
        j = self.index.get(name)
        return self.b.var(j) if j is not None else self.b.const(1.0)

    # spatial axis quantities
    def V(self, ax: SAxis) -> int: return self.v(f"V_{ax.name}")
    def T(self, ax: SAxis) -> int: return self.v(f"T_{ax.name}")
    def I(self, ax: SAxis) -> int: return self.v(f"I_{ax.name}")

    def Tb(self, ax: SAxis) -> int:
        return self.b.prod([self.V(ax), self.T(ax), self.I(ax)])

    def Nb(self, ax: SAxis) -> int:
        return self.b.div(self.b.const(ax.extent), self.Tb(ax))

    # reduction axis quantities
    def red_levels(self, ax: RAxis) -> Tuple[Optional[int], int]:
        """(rm extent node or None, ri extent node)."""
        if ax.n_vars == 0:
            return None, self.b.const(ax.extent)
        if ax.n_vars == 1:
            return None, self.v(f"RI_{ax.name}")
        return self.v(f"RI1_{ax.name}"), self.v(f"RI2_{ax.name}")

    def Rt(self, ax: RAxis) -> int:
        rm, ri = self.red_levels(ax)
        return ri if rm is None else self.b.mul(rm, ri)

    def Ro(self, ax: RAxis) -> int:
        return self.b.div(self.b.const(ax.extent), self.Rt(ax))

    def loops(self) -> List[Tuple[str, int, str, int]]:
        """Per-thread loop list L (outer -> inner): (kind, extent node, axis name, step node)."""
        b, out = self.b, []
        for ax in self.spec.reduction:
            out.append(("ro", self.Ro(ax), ax.name, self.Rt(ax)))
        for ax in self.spec.reduction:
            rm, ri = self.red_levels(ax)
            if rm is not None:
                out.append(("rm", rm, ax.name, ri))
        for ax in self.spec.spatial:
            out.append(("v", self.V(ax), ax.name, b.mul(self.T(ax), self.I(ax))))
        for ax in self.spec.reduction:
            _, ri = self.red_levels(ax)
            out.append(("ri", ri, ax.name, b.const(1.0)))
        for ax in self.spec.spatial:
            out.append(("in", self.I(ax), ax.name, b.const(1.0)))
        return out


def _dim_footprint(ctx: _Ctx, dim: List[Tuple[str, int]], scope: str) -> int:
    """Distinct values of one buffer index dim  sum(coeff * axis)  touched by block 0 / thread 0
    during the first outer-reduction iteration (ro = 0 for every reduction axis)."""
    b, spec = ctx.b, ctx.spec
    if not dim:
        return b.const(1.0)
    sp = [(a, c) for a, c in dim if spec.is_spatial(a)]
    rd = [(a, c) for a, c in dim if not spec.is_spatial(a)]
    assert len(sp) <= 1 and len(rd) <= 1, "index dims combine at most one spatial + one reduction axis"
    if not sp:
        (a, c), = rd
        assert c == 1
        ax = next(x for x in spec.reduction if x.name == a)
        return ctx.Rt(ax)
    (sa, c), = sp
    ax = next(x for x in spec.spatial if x.name == sa)
    if not rd:
        # spatial only: block covers a contiguous run of Tb; thread covers V runs of I (stride T*I)
        return ctx.Tb(ax) if scope == "block" else b.mul(ctx.V(ax), ctx.I(ax))
    (ra, rc), = rd
    rax = next(x for x in spec.reduction if x.name == ra)
    assert rax.n_vars == 0 and rc == 1, "halo dims use an unsplit reduction axis"
    R = rax.extent
    run = ctx.Tb(ax) if scope == "block" else ctx.I(ax)
    if c > R:   # index c*s + r with r < R < c: all (s, r) pairs distinct, runs never overlap
        n = run if scope == "block" else b.mul(ctx.V(ax), run)
        return b.mul(n, b.const(R))
    # one run of s of length n gives the interval [c*s0, c*(s0+n-1)+R): length c*(n-1)+R
    L = b.add(b.mul(b.const(c), b.sub(run, b.const(1.0))), b.const(R))
    if scope == "block":
        return L
    # thread: V intervals of length L with stride S = c*T*I; union = V*L - (V-1)*max(0, L-S)
    S = b.mul(b.const(c), b.mul(ctx.T(ax), ctx.I(ax)))
    V = ctx.V(ax)
    overlap = b.max(b.const(0.0), b.sub(L, S))
    return b.sub(b.mul(V, L), b.mul(b.sub(V, b.const(1.0)), overlap))


def _dim_bbox(ctx: _Ctx, dim: List[Tuple[str, int]]) -> int:
    """Bounding-box extent (max - min + 1) of one index dim over block 0's first outer-reduction tile:
    the shared-memory tile a block allocates for it (row-major over the dims' boxes)."""
    b, spec = ctx.b, ctx.spec
    if not dim:
        return b.const(1.0)
    sp = [(a, c) for a, c in dim if spec.is_spatial(a)]
    rd = [(a, c) for a, c in dim if not spec.is_spatial(a)]
    if not sp:
        (a, _), = rd
        return ctx.Rt(next(x for x in spec.reduction if x.name == a))
    (sa, c), = sp
    ax = next(x for x in spec.spatial if x.name == sa)
    if not rd:
        return ctx.Tb(ax)
    (ra, _), = rd
    R = next(x for x in spec.reduction if x.name == ra).extent
    return b.add(b.mul(b.const(c), b.sub(ctx.Tb(ax), b.const(1.0))), b.const(R))


def _smem_stride(ctx: _Ctx, buf: Buffer, loops) -> int:
    """Shared-memory address delta (elements, row-major over the dims' bounding boxes) along the innermost
    non-trivial loop of L; 0 when that loop is an outer-reduction loop (each ro tile reuses the buffer)."""
    b = ctx.b
    boxes = [_dim_bbox(ctx, d) for d in buf.dims]
    pitch = []
    for d in range(len(buf.dims)):
        pitch.append(b.prod(boxes[d + 1:]))
    stride = b.const(0.0)
    for kind, ext, axn, step in loops:
        coef = [c for d, dim in enumerate(buf.dims) for a, c in dim if a == axn]
        dpos = [d for d, dim in enumerate(buf.dims) for a, c in dim if a == axn]
        if kind == "ro" or not coef:
            delta = b.const(0.0)
        else:
            delta = b.sum([b.mul(b.mul(step, b.const(float(c))), pitch[d]) for c, d in zip(coef, dpos)])
        stride = b.select(b.gt(ext, b.const(1.0)), delta, stride)
    return stride, b.prod(boxes)


def _out_stride(spec: ProgramSpec, loops) -> float:
    """(per loop) output linear-index delta: spatial axes row-major in spec.spatial order."""
    E = [ax.extent for ax in spec.spatial]
    pitch = {ax.name: float(np.prod(E[i + 1:])) for i, ax in enumerate(spec.spatial)}
    return pitch


def _loop_shape_feats(ctx: _Ctx, loops, NB, NT) -> List[Tuple[str, int]]:
    """GPU-mapping / loop-structure features shared by both statements."""
    b = ctx.b
    inner_len, outer_len = b.const(1.0), b.const(1.0)
    for _, ext, _, _ in loops:                   # outer -> inner: the innermost non-trivial loop wins
        inner_len = b.select(b.gt(ext, b.const(1.0)), ext, inner_len)
    for _, ext, _, _ in reversed(loops):         # inner -> outer: the outermost non-trivial loop wins
        outer_len = b.select(b.gt(ext, b.const(1.0)), ext, outer_len)
    mx = b.const(1.0)
    for _, ext, _, _ in loops:
        mx = b.max(mx, ext)
    return [("total_threads", b.mul(NB, NT)), ("innermost_len", inner_len), ("outermost_len", outer_len),
            ("max_loop_extent", mx)]


def _out_feats(ctx: _Ctx, loops) -> List[Tuple[str, int]]:
    """Output-buffer slot: store stride along the innermost non-trivial loop (reduction loops do not
    move the output), its vectorizability, and the outputs a block writes."""
    b, spec = ctx.b, ctx.spec
    pitch = _out_stride(spec, loops)
    stride = b.const(0.0)
    for kind, ext, axn, step in loops:
        d = b.mul(step, b.const(pitch[axn])) if axn in pitch else b.const(0.0)
        stride = b.select(b.gt(ext, b.const(1.0)), d, stride)
    vec = b.select(b.cmp(OP_EQ, stride, b.const(1.0)), b.const(1.0), b.const(0.0))
    return [("out.innermost_stride", stride), ("out.vectorizable", vec),
            ("out.block_footprint", b.prod([ctx.Tb(ax) for ax in spec.spatial]))]


def _linear_stride(spec: ProgramSpec, buf: Buffer, axis: str) -> int:
    """Address delta (elements, row-major buffer) when `axis` index increases by 1."""
    shape = spec.buffer_shape(buf)
    pitch = [int(np.prod(shape[d + 1:])) for d in range(len(shape))]
    return sum(pitch[d] * c for d, dim in enumerate(buf.dims) for a, c in dim if a == axis)


def _epilogue_feats(spec: ProgramSpec, ctx: "_Ctx") -> List[Tuple[str, int]]:
    """Feature formulas of the epilogue statement (module docstring), same names / order / definitions
    as the main statement's."""
    b = ctx.b
    E = float(np.prod([ax.extent for ax in spec.spatial]))
    NB = b.prod([ctx.Nb(ax) for ax in spec.spatial])
    NT = b.prod([ctx.T(ax) for ax in spec.spatial])
    NV = b.prod([ctx.V(ax) for ax in spec.spatial])
    opt = b.prod([b.mul(ctx.V(ax), ctx.I(ax)) for ax in spec.spatial])      # instances = outputs per thread
    loops = [("v", ctx.V(ax), ax.name, b.mul(ctx.T(ax), ctx.I(ax))) for ax in spec.spatial] + \
            [("in", ctx.I(ax), ax.name, b.const(1.0)) for ax in spec.spatial]
    nontriv = b.sum([b.select(b.gt(ext, b.const(1.0)), b.const(1.0), b.const(0.0)) for _, ext, _, _ in loops])
    n_ops = float(spec.bias) + float(spec.relu) + float(spec.gelu)
    f: List[Tuple[str, int]] = []
    f.append(("float_mad", b.const(0.0)))
    f.append(("float_addsub", b.const(E if spec.bias else 0.0)))
    f.append(("float_cmp", b.const(E if spec.relu else 0.0)))
    f.append(("float_math", b.const(E if spec.gelu else 0.0)))
    f.append(("blockIdx_len", NB))
    f.append(("vthread_len", NV))
    f.append(("threadIdx_len", NT))
    f.append(("outputs_per_thread", opt))
    f.append(("stmts_per_thread", opt))
    f.append(("n_nontrivial_loops", nontriv))
    f.append(("int_addsub", b.mul(b.const(E), b.add(b.const(2.0), nontriv))))
    n_block_axes = b.sum([b.select(b.gt(ctx.Nb(ax), b.const(1.0)), b.const(1.0), b.const(0.0)) for ax in spec.spatial])
    f.append(("int_mul", b.mul(b.const(E), n_block_axes)))
    f.append(("reduction_outer_iters", b.const(1.0)))
    if spec.unroll:
        U = ctx.v("UNROLL")
        f.append(("unroll_len", b.min(U, opt)))
        cum, cnt = b.const(1.0), []
        for _, ext, _, _ in reversed(loops):
            cum = b.mul(cum, ext)
            cnt.append(b.select(b.le(cum, U), b.const(1.0), b.const(0.0)))
        f.append(("unrolled_loops", b.sum(cnt)))
    else:
        f.append(("unroll_len", b.const(0.0)))
        f.append(("unrolled_loops", b.const(0.0)))
    gbytes, smem = [], []
    bufs = [Buffer("Bias", [[(spec.bias_axis, 1)]])] if spec.bias else []
    for slot in range(len(spec.inputs)):
        if slot < len(bufs):
            buf = bufs[slot]
            blk = _dim_footprint(ctx, buf.dims[0], "block")
            thr = _dim_footprint(ctx, buf.dims[0], "thread")
            gl = b.mul(NB, blk)
            gb = b.mul(b.const(4.0), gl)
            gbytes.append(gb)
            smem.append(blk)
            stride = b.const(0.0)
            for kind, ext, axn, step in loops:
                d = b.mul(step, b.const(float(_linear_stride(spec, buf, axn))))
                stride = b.select(b.gt(ext, b.const(1.0)), d, stride)
            sstride, bbox = _smem_stride(ctx, buf, loops)
            vals = [blk, gl, gb, b.ceildiv(blk, NT), thr, b.div(opt, thr), b.div(b.mul(opt, NT), blk),
                    b.div(b.const(E), gl), stride, b.mul(b.const(4.0), blk),
                    b.select(b.cmp(OP_EQ, stride, b.const(1.0)), b.const(1.0), b.const(0.0)),
                    b.div(gl, b.const(float(np.prod(spec.buffer_shape(buf))))), sstride, bbox, b.div(blk, bbox)]
        else:
            vals = [b.const(0.0)] * 15
        names = ["block_footprint", "global_load_elems", "global_bytes", "coop_loads_per_thread", "thread_footprint",
                 "thread_reuse", "block_reuse", "global_reuse", "innermost_stride", "shared_bytes",
                 "vectorizable", "load_ratio", "smem_inner_stride", "smem_tile_elems", "smem_tile_util"]
        f += [(f"in{slot}.{nm}", v) for nm, v in zip(names, vals)]
    gsum = b.sum(gbytes) if gbytes else b.const(0.0)
    f += [
        ("out.stores", b.const(E)),
        ("shared_bytes_total", b.mul(b.const(4.0), b.sum(smem)) if smem else b.const(0.0)),
        ("local_bytes", b.mul(b.const(4.0), opt)),
        ("flops_per_global_byte", b.div(b.const(n_ops * E), b.add(gsum, b.const(4.0 * E)))),
        ("flops_per_thread", b.mul(b.const(n_ops), opt)),
        ("global_bytes_per_block", b.div(gsum, NB)),
    ]
    f += _out_feats(ctx, loops)
    f += _loop_shape_feats(ctx, loops, NB, NT)
    return f


def build_space(spec: ProgramSpec, statements: int = 1) -> Space:
    """statements=1: one feature vector (the main statement, epilogue ops folded in); statements=2:
    [main statement | epilogue statement], 82 features each, statement-major (TenSet segment sum)."""
    assert statements in (1, 2)
    vars_, splits, index = var_layout(spec)
    b = DagBuilder()
    ctx = _Ctx(spec, b, index)
    feats: List[Tuple[str, int]] = []

    E = [ax.extent for ax in spec.spatial]
    Kx = [ax.extent for ax in spec.reduction]
    prodE = float(np.prod(E))
    nmac = float(np.prod(E) * np.prod(Kx))
    NB = b.prod([ctx.Nb(ax) for ax in spec.spatial])
    NT = b.prod([ctx.T(ax) for ax in spec.spatial])
    NV = b.prod([ctx.V(ax) for ax in spec.spatial])
    out_per_thread = b.prod([b.mul(ctx.V(ax), ctx.I(ax)) for ax in spec.spatial])
    stmts_per_thread = b.div(b.const(nmac), b.mul(NB, NT))
    ro_iters = b.prod([ctx.Ro(ax) for ax in spec.reduction])
    loops = ctx.loops()
    nontriv = [b.select(b.gt(ext, b.const(1.0)), b.const(1.0), b.const(0.0)) for _, ext, _, _ in loops]
    n_nontriv = b.sum(nontriv)

    # -- op counts / GPU mapping / loop structure
    epi_in_main = statements == 1
    ops = STMT_OPS[spec.stmt]
    fpi = STMT_FLOPS[spec.stmt]
    feats.append(("float_mad", b.const(nmac * ops["mad"])))
    feats.append(("float_addsub", b.const((prodE if spec.bias and epi_in_main else 0.0) + nmac * ops["addsub"])))
    feats.append(("float_cmp", b.const(prodE if spec.relu and epi_in_main else 0.0)))
    feats.append(("float_math", b.const((prodE if spec.gelu and epi_in_main else 0.0) + nmac * ops["math"])))
    feats.append(("blockIdx_len", NB))
    feats.append(("vthread_len", NV))
    feats.append(("threadIdx_len", NT))
    feats.append(("outputs_per_thread", out_per_thread))
    feats.append(("stmts_per_thread", stmts_per_thread))
    feats.append(("n_nontrivial_loops", n_nontriv))
    # paper's example shape: int_add = NMK * select(TILE0 > 1, 5, 2)  (L668-671)
    feats.append(("int_addsub", b.mul(b.const(nmac), b.add(b.const(2.0), n_nontriv))))
    n_block_axes = b.sum([b.select(b.gt(ctx.Nb(ax), b.const(1.0)), b.const(1.0), b.const(0.0)) for ax in spec.spatial])
    feats.append(("int_mul", b.mul(b.const(nmac), n_block_axes)))
    feats.append(("reduction_outer_iters", ro_iters))
    per_ro = b.div(stmts_per_thread, ro_iters)
    if spec.unroll:
        U = ctx.v("UNROLL")
        feats.append(("unroll_len", b.min(U, per_ro)))
        cum, cnt = b.const(1.0), []
        for _, ext, _, _ in reversed(loops):
            cum = b.mul(cum, ext)
            cnt.append(b.select(b.le(cum, U), b.const(1.0), b.const(0.0)))
        feats.append(("unrolled_loops", b.sum(cnt)))
    else:
        feats.append(("unroll_len", b.const(0.0)))
        feats.append(("unrolled_loops", b.const(0.0)))

    # -- per-input-buffer memory features
    gbytes = []
    smem_elems = []
    stmts_per_block_ro = b.div(b.mul(stmts_per_thread, NT), ro_iters)
    for buf in spec.inputs:
        blk = b.prod([_dim_footprint(ctx, d, "block") for d in buf.dims])
        thr = b.prod([_dim_footprint(ctx, d, "thread") for d in buf.dims])
        gl = b.mul(b.mul(NB, ro_iters), blk)
        gb = b.mul(b.const(4.0), gl)
        gbytes.append(gb)
        smem_elems.append(blk)
        # stride along the innermost non-trivial loop of L (0 if every loop is trivial)
        stride = b.const(0.0)
        for kind, ext, axn, step in loops:     # outer -> inner: the innermost wins
            s = _linear_stride(spec, buf, axn)
            d = b.mul(step, b.const(float(s)))
            stride = b.select(b.gt(ext, b.const(1.0)), d, stride)
        sstride, bbox = _smem_stride(ctx, buf, loops)
        feats += [
            (f"{buf.name}.block_footprint", blk),
            (f"{buf.name}.global_load_elems", gl),
            (f"{buf.name}.global_bytes", gb),
            (f"{buf.name}.coop_loads_per_thread", b.ceildiv(blk, NT)),
            (f"{buf.name}.thread_footprint", thr),
            (f"{buf.name}.thread_reuse", b.div(per_ro, thr)),
            (f"{buf.name}.block_reuse", b.div(stmts_per_block_ro, blk)),
            (f"{buf.name}.global_reuse", b.div(b.const(nmac), gl)),
            (f"{buf.name}.innermost_stride", stride),
            (f"{buf.name}.shared_bytes", b.mul(b.const(4.0), blk)),
            # global-side vectorizability and re-fetch ratio, shared-memory tile (bounding box) layout
            (f"{buf.name}.vectorizable", b.select(b.cmp(OP_EQ, stride, b.const(1.0)), b.const(1.0), b.const(0.0))),
            (f"{buf.name}.load_ratio", b.div(gl, b.const(float(np.prod(spec.buffer_shape(buf)))))),
            (f"{buf.name}.smem_inner_stride", sstride),
            (f"{buf.name}.smem_tile_elems", bbox),
            (f"{buf.name}.smem_tile_util", b.div(blk, bbox)),
        ]
    smem_bytes = b.mul(b.const(4.0), b.sum(smem_elems))
    feats += [
        ("out.stores", b.const(prodE)),
        ("shared_bytes_total", smem_bytes),
        ("local_bytes", b.mul(b.const(4.0), out_per_thread)),
        ("flops_per_global_byte", b.div(b.const(fpi * nmac), b.add(b.sum(gbytes), b.const(4.0 * prodE)))),
        ("flops_per_thread", b.mul(b.const(fpi), stmts_per_thread)),
        ("global_bytes_per_block", b.div(b.sum(gbytes), NB)),
    ]
    feats += _out_feats(ctx, loops)
    feats += _loop_shape_feats(ctx, loops, NB, NT)
    assert len(feats) <= N_FEATURES
    n_used = len(feats)
    zero = b.const(0.0)
    for k in range(N_FEATURES - n_used):   # annotation slots this sketch never produces
        feats.append((f"reserved_{k}", zero))
    if statements == 2:
        ef = _epilogue_feats(spec, ctx)
        assert len(ef) == n_used
        feats = [(f"S0.{nm}", v) for nm, v in feats] + [(f"S1.{nm}", v) for nm, v in ef] + \
                [(f"S1.reserved_{k}", zero) for k in range(N_FEATURES - n_used)]

    # -- user constraints g(x) <= 0, in log form so lambda has a uniform scale (SURVEY O2 reading)
    cons: List[Tuple[str, int]] = []
    cons.append(("threads<=limit", b.sub(b.log(NT), b.const(math.log(spec.thread_limit)))))
    cons.append(("smem<=limit", b.sub(b.log(smem_bytes), b.const(math.log(spec.smem_limit)))))
    cons.append(("local<=limit", b.sub(b.log(b.mul(b.const(4.0), out_per_thread)), b.const(math.log(spec.local_limit * 4)))))
    if any("v" in ax.levels for ax in spec.spatial):
        cons.append(("vthreads<=limit", b.sub(b.log(NV), b.const(math.log(spec.vthread_limit)))))

    nodes = b.nodes()
    nodes, (froots, croots) = prune(nodes, [np.array([f for _, f in feats], dtype=np.int32),
                                             np.array([c for _, c in cons], dtype=np.int32)])
    return Space(spec.name, vars_, splits, nodes, froots, croots,
                 [n for n, _ in feats], [n for n, _ in cons], spec, n_statements=statements)


# ------------------------------------------------------------------------------ concrete workloads
def dense_spec(name: str, N: int, M: int, K: int, *, i_levels="ti", j_levels="ti", k_vars=1,
               bias=True, relu=False, gelu=False, batch: int = 0) -> ProgramSpec:
    """O[i, j] += A[i, k] * B[k, j]  (Dense / Dense-Add, Fig. 3).  batch > 0 adds a leading
    spatial axis b (bmm): A[b, i, k], B[b, k, j]."""
    spatial = [SAxis("i", N, i_levels), SAxis("j", M, j_levels)]
    a_dims = [[("i", 1)], [("k", 1)]]
    b_dims = [[("k", 1)], [("j", 1)]]
    if batch:
        spatial = [SAxis("b", batch, "t")] + spatial
        a_dims = [[("b", 1)]] + a_dims
        b_dims = [[("b", 1)]] + b_dims
    return ProgramSpec(name, spatial, [RAxis("k", K, k_vars)],
                       [Buffer("A", a_dims), Buffer("B", b_dims)], bias=bias, relu=relu, gelu=gelu, bias_axis="j")


def conv2d_spec(name: str, C: int, H: int, W: int, K: int, R: int, S: int, stride: int = 1, *,
                co_levels="vti", h_levels="vti", w_levels="vti", rc_vars=2, bias=True, relu=True) -> ProgramSpec:
    """O[co, h, w] += In[rc, stride*h + rh, stride*w + rw] * Wt[co, rc, rh, rw] (batch 1, input
    pre-padded), H, W = output sizes."""
    spatial = [SAxis("co", K, co_levels), SAxis("h", H, h_levels), SAxis("w", W, w_levels)]
    red = [RAxis("rc", C, rc_vars), RAxis("rh", R, 0), RAxis("rw", S, 0)]
    inp = Buffer("In", [[("rc", 1)], [("h", stride), ("rh", 1)], [("w", stride), ("rw", 1)]])
    wt = Buffer("Wt", [[("co", 1)], [("rc", 1)], [("rh", 1)], [("rw", 1)]])
    return ProgramSpec(name, spatial, red, [inp, wt], bias=bias, relu=relu, bias_axis="co")


def depthwise_conv2d_spec(name: str, C: int, H: int, W: int, R: int, S: int, stride: int = 1, *,
                          c_levels="vti", h_levels="vti", w_levels="vti", bias=True, relu=True) -> ProgramSpec:
    """Depthwise conv (MobileNet-v2): O[c, h, w] += In[c, stride*h + rh, stride*w + rw] * Wt[c, rh, rw]
    (batch 1, pre-padded input; no reduction over channels, so the only reduction axes are the unsplit
    kernel window rh, rw)."""
    spatial = [SAxis("c", C, c_levels), SAxis("h", H, h_levels), SAxis("w", W, w_levels)]
    red = [RAxis("rh", R, 0), RAxis("rw", S, 0)]
    inp = Buffer("In", [[("c", 1)], [("h", stride), ("rh", 1)], [("w", stride), ("rw", 1)]])
    wt = Buffer("Wt", [[("c", 1)], [("rh", 1)], [("rw", 1)]])
    return ProgramSpec(name, spatial, red, [inp, wt], bias=bias, relu=relu, bias_axis="c")


def softmax_spec(name: str, B: int, N: int, M: int, *, i_levels="vti", j_vars=1) -> ProgramSpec:
    """Softmax's reduction stage over the last axis, O[b, i] += exp(A[b, i, j]) (BERT attention scores,
    batch x heads folded into b; the operator mix of Fig. 9).  The normalisation stage is an
    elementwise pass without schedule variables of its own."""
    spatial = [SAxis("b", B, "t"), SAxis("i", N, i_levels)]
    return ProgramSpec(name, spatial, [RAxis("j", M, j_vars)], [Buffer("A", [[("b", 1)], [("i", 1)], [("j", 1)]])],
                       bias=False, stmt="exp_sum")


def layernorm_spec(name: str, N: int, D: int, *, i_levels="vti", j_vars=2) -> ProgramSpec:
    """LayerNorm's statistics stage, O1[i] += A[i, j], O2[i] += A[i, j]^2 (BERT hidden states)."""
    return ProgramSpec(name, [SAxis("i", N, i_levels)], [RAxis("j", D, j_vars)], [Buffer("A", [[("i", 1)], [("j", 1)]])],
                       bias=False, stmt="sum_sq")


def paper_dense_add_s1(N: int = 64, M: int = 64, K: int = 64) -> Space:
    """The paper's worked example, symbolic schedule s*_1 of Dense-Add (Fig. 3) with
    variables TILE0 (tiles both M and K, L579-581) and UNROLL0, and exactly the three feature
    formulas printed at L668-671:  float_add = N*M*K,  blockIdx_len = N*M/TILE0,
    int_add = NMK * select(TILE0 > 1, 5, 2);  constraint c11 = (1 <= TILE0 <= K) as the penalty
    functions g11 = 1 - TILE0, g12 = TILE0 - K (L786-788).  Remaining feature slots are zero."""
    b = DagBuilder()
    t = b.var(0)
    nmk = b.const(float(N * M * K))
    f_add = nmk
    f_blk = b.div(b.const(float(N * M)), t)
    f_int = b.mul(nmk, b.select(b.gt(t, b.const(1.0)), b.const(5.0), b.const(2.0)))
    zero = b.const(0.0)
    feats = [f_add, f_blk, f_int] + [zero] * (N_FEATURES - 3)
    g11 = b.sub(b.const(1.0), t)
    g12 = b.sub(t, b.const(float(K)))
    nodes = b.nodes()
    nodes, (fr, cr) = prune(nodes, [np.array(feats, dtype=np.int32), np.array([g11, g12], dtype=np.int32)])
    vars_ = [Var("TILE0", VAR_SPLIT, 1, min(M, K)), Var("UNROLL0", VAR_INT, 1, UNROLL_MAX)]
    splits = [Split(M, [0]), Split(K, [0])]
    names = ["float_add", "blockIdx_len", "int_add"] + [f"reserved_{k}" for k in range(N_FEATURES - 3)]
    return Space("paper_dense_add_s1", vars_, splits, nodes, fr, cr, names, ["g11", "g12"], None)
