"""Brute-force simulator of the concrete tiled loop nest (test-only pin for the oracle's hard
feature evaluation).

Given a ProgramSpec (felix_inputs/programs.py: the sketch in its module docstring) and an INTEGER
assignment of the schedule variables, this module materialises every statement instance of the
concrete program — (block, thread, per-thread loop indices) -> axis indices -> buffer element
indices — and COUNTS each feature from its definition (distinct elements, executions, loop
extents, address deltas).  It never looks at the feature DAG or its formulas.
"""
from __future__ import annotations

import itertools
from typing import Dict, List, Tuple

import numpy as np


def _levels(spec, x: Dict[str, int]):
    sp = []
    for ax in spec.spatial:
        V = x.get(f"V_{ax.name}", 1) if "v" in ax.levels else 1
        T = x.get(f"T_{ax.name}", 1) if "t" in ax.levels else 1
        I = x.get(f"I_{ax.name}", 1) if "i" in ax.levels else 1
        assert ax.extent % (V * T * I) == 0
        sp.append(dict(name=ax.name, E=ax.extent, V=V, T=T, I=I, Nb=ax.extent // (V * T * I)))
    rd = []
    for ax in spec.reduction:
        if ax.n_vars == 0:
            rm, ri = 1, ax.extent
        elif ax.n_vars == 1:
            rm, ri = 1, x[f"RI_{ax.name}"]
        else:
            rm, ri = x[f"RI1_{ax.name}"], x[f"RI2_{ax.name}"]
        assert ax.extent % (rm * ri) == 0
        rd.append(dict(name=ax.name, K=ax.extent, rm=rm, ri=ri, Ro=ax.extent // (rm * ri), nv=ax.n_vars))
    return sp, rd


def _loop_list(sp, rd):
    """Per-thread loops outer -> inner: ro_*, rm_* (2-var axes), v_*, ri_*, in_*."""
    L = []
    for r in rd:
        L.append(("ro", r["name"], r["Ro"]))
    for r in rd:
        if r["nv"] == 2:
            L.append(("rm", r["name"], r["rm"]))
    for s in sp:
        L.append(("v", s["name"], s["V"]))
    for r in rd:
        L.append(("ri", r["name"], r["ri"]))
    for s in sp:
        L.append(("in", s["name"], s["I"]))
    return L


def _instances(spec, sp, rd):
    """All statement instances as integer arrays: block id, thread id, ro tuple id, axis indices,
    per-thread loop indices."""
    L = _loop_list(sp, rd)
    blk_ranges = [range(s["Nb"]) for s in sp]
    thr_ranges = [range(s["T"]) for s in sp]
    loop_ranges = [range(e) for _, _, e in L]
    rows = []
    for bi, bt in enumerate(itertools.product(*blk_ranges)):
        for ti, tt in enumerate(itertools.product(*thr_ranges)):
            for li in itertools.product(*loop_ranges):
                rows.append((bi, ti) + tuple(bt) + tuple(tt) + tuple(li))
    arr = np.array(rows, dtype=np.int64)
    ns = len(sp)
    blk = arr[:, 0]
    thr = arr[:, 1]
    bvec = arr[:, 2:2 + ns]
    tvec = arr[:, 2 + ns:2 + 2 * ns]
    lvec = arr[:, 2 + 2 * ns:]
    # decode axis indices
    idx = {}
    li = {(k, a): lvec[:, n] for n, (k, a, _) in enumerate(L)}
    for i, s in enumerate(sp):
        idx[s["name"]] = (bvec[:, i] * (s["V"] * s["T"] * s["I"]) + li[("v", s["name"])] * (s["T"] * s["I"])
                          + tvec[:, i] * s["I"] + li[("in", s["name"])])
    ro_cols = []
    for r in rd:
        rm = li.get(("rm", r["name"]), np.zeros(len(arr), dtype=np.int64))
        idx[r["name"]] = li[("ro", r["name"])] * (r["rm"] * r["ri"]) + rm * r["ri"] + li[("ri", r["name"])]
        ro_cols.append(li[("ro", r["name"])])
    ro = np.zeros(len(arr), dtype=np.int64)
    for r, col in zip(rd, ro_cols):
        ro = ro * r["Ro"] + col
    return L, blk, thr, ro, idx, lvec


def _buffer_index(spec, buf, idx) -> np.ndarray:
    """Linear (row-major) element index of `buf` for every instance."""
    shape = spec.buffer_shape(buf)
    lin = np.zeros_like(next(iter(idx.values())))
    for d, dim in enumerate(buf.dims):
        v = sum(c * idx[a] for a, c in dim) if dim else 0
        lin = lin * shape[d] + v
    return lin


def _dim_values(spec, buf, idx):
    """Per index dim of `buf`: its value for every instance."""
    n = len(next(iter(idx.values())))
    return [sum(c * idx[a] for a, c in dim) if dim else np.zeros(n, dtype=np.int64) for dim in buf.dims]


def _smem_layout(dims, sel):
    """Bounding box (max - min + 1 per dim) of the instances `sel` and the row-major local index of every
    instance inside it (the block's shared-memory tile)."""
    lo = [int(d[sel].min()) for d in dims]
    box = [int(d[sel].max()) - l + 1 for d, l in zip(dims, lo)]
    local = np.zeros_like(dims[0])
    for d, l, e in zip(dims, lo, box):
        local = local * e + (d - l)
    return box, local


def _shape_feats(L, NB, NT):
    ext = [e for _, _, e in L]
    nontriv = [e for e in ext if e > 1]
    return {"total_threads": NB * NT, "innermost_len": nontriv[-1] if nontriv else 1,
            "outermost_len": nontriv[0] if nontriv else 1, "max_loop_extent": max([1] + ext)}


def simulate(spec, x: Dict[str, int]) -> Dict[str, float]:
    sp, rd = _levels(spec, x)
    L, blk, thr, ro, idx, lvec = _instances(spec, sp, rd)
    n = len(blk)
    f: Dict[str, float] = {}
    E = int(np.prod([s["E"] for s in sp]))
    # outputs
    out_lin = np.zeros(n, dtype=np.int64)
    for s in sp:
        out_lin = out_lin * s["E"] + idx[s["name"]]
    assert len(np.unique(out_lin)) == E
    # one reduction-statement instance does: "mad" 1 multiply-add; "exp_sum" 1 exp + 1 add;
    # "sum_sq" 1 add + 1 multiply-add (written out here independently of the feature DAG)
    k_mad, k_add, k_math, k_flops = {"mad": (1, 0, 0, 2), "exp_sum": (0, 1, 1, 2), "sum_sq": (1, 1, 0, 3)}[spec.stmt]
    f["float_mad"] = n * k_mad
    f["float_addsub"] = (E if spec.bias else 0) + n * k_add
    f["float_cmp"] = E if spec.relu else 0
    f["float_math"] = (E if spec.gelu else 0) + n * k_math
    NB = len(np.unique(blk))
    NT = len(np.unique(thr))
    f["blockIdx_len"] = NB
    f["vthread_len"] = int(np.prod([s["V"] for s in sp]))
    f["threadIdx_len"] = NT
    t0 = (blk == 0) & (thr == 0)
    f["outputs_per_thread"] = len(np.unique(out_lin[t0]))
    f["stmts_per_thread"] = int(t0.sum())
    nontriv = sum(1 for _, _, e in L if e > 1)
    f["n_nontrivial_loops"] = nontriv
    f["int_addsub"] = float(sum(2 + nontriv for _ in range(1))) * n   # every instance sits in all of L
    f["int_mul"] = n * sum(1 for s in sp if s["Nb"] > 1)
    f["reduction_outer_iters"] = len(np.unique(ro))
    per_ro = int((t0 & (ro == 0)).sum())
    if spec.unroll:
        U = x["UNROLL"]
        f["unroll_len"] = min(U, per_ro)
        cum, cnt = 1, 0
        for _, _, e in reversed(L):
            cum *= e
            if cum <= U:
                cnt += 1
        f["unrolled_loops"] = cnt
    else:
        f["unroll_len"] = 0
        f["unrolled_loops"] = 0
    gbytes_total = 0
    smem_total = 0
    b0r0 = (blk == 0) & (ro == 0)
    t0r0 = t0 & (ro == 0)
    # innermost non-trivial loop of L (for the stride feature)
    inner = None
    for pos in range(len(L) - 1, -1, -1):
        if L[pos][2] > 1:
            inner = pos
            break
    if inner is None:
        sel0 = sel1 = None
    else:
        sel0 = t0 & np.all(lvec == 0, axis=1)
        one = np.zeros(len(L), dtype=np.int64)
        one[inner] = 1
        sel1 = t0 & np.all(lvec == one[None, :], axis=1)
    for buf in spec.inputs:
        lin = _buffer_index(spec, buf, idx)
        blk_fp = len(np.unique(lin[b0r0]))
        box, local = _smem_layout(_dim_values(spec, buf, idx), b0r0)
        if inner is None or L[inner][0] == "ro":
            sstride = 0                                # no loop, or a new tile per outer-reduction step
        else:
            sstride = int(local[sel1][0] - local[sel0][0])
        # per (block, ro) distinct counts
        key = blk * (ro.max() + 1) + ro
        order = np.lexsort((lin, key))
        k_s, l_s = key[order], lin[order]
        first = np.ones(n, dtype=bool)
        first[1:] = (k_s[1:] != k_s[:-1]) | (l_s[1:] != l_s[:-1])
        gl = int(first.sum())
        thr_fp = len(np.unique(lin[t0r0]))
        # cooperative load: footprint elements dealt round-robin to NT threads
        per_thread = np.bincount(np.arange(blk_fp) % NT, minlength=NT)
        if inner is None:
            stride = 0
        else:
            sel0 = t0 & np.all(lvec == 0, axis=1)
            one = np.zeros(len(L), dtype=np.int64)
            one[inner] = 1
            sel1 = t0 & np.all(lvec == one[None, :], axis=1)
            stride = int(lin[sel1][0] - lin[sel0][0])
        f[f"{buf.name}.block_footprint"] = blk_fp
        f[f"{buf.name}.global_load_elems"] = gl
        f[f"{buf.name}.global_bytes"] = 4 * gl
        f[f"{buf.name}.coop_loads_per_thread"] = int(per_thread.max())
        f[f"{buf.name}.thread_footprint"] = thr_fp
        f[f"{buf.name}.thread_reuse"] = per_ro / thr_fp
        f[f"{buf.name}.block_reuse"] = int(b0r0.sum()) / blk_fp
        f[f"{buf.name}.global_reuse"] = n / gl
        f[f"{buf.name}.innermost_stride"] = stride
        f[f"{buf.name}.shared_bytes"] = 4 * blk_fp
        f[f"{buf.name}.vectorizable"] = 1 if stride == 1 else 0
        f[f"{buf.name}.load_ratio"] = gl / int(np.prod(spec.buffer_shape(buf)))
        f[f"{buf.name}.smem_inner_stride"] = sstride
        f[f"{buf.name}.smem_tile_elems"] = int(np.prod(box))
        f[f"{buf.name}.smem_tile_util"] = blk_fp / int(np.prod(box))
        gbytes_total += 4 * gl
        smem_total += 4 * blk_fp
    f["out.stores"] = E
    f["shared_bytes_total"] = smem_total
    f["local_bytes"] = 4 * f["outputs_per_thread"]
    f["flops_per_global_byte"] = k_flops * n / (gbytes_total + 4 * E)
    f["flops_per_thread"] = k_flops * f["stmts_per_thread"]
    f["global_bytes_per_block"] = gbytes_total / NB
    ostride = 0 if inner is None else int(out_lin[sel1][0] - out_lin[sel0][0])
    f["out.innermost_stride"] = ostride
    f["out.vectorizable"] = 1 if ostride == 1 else 0
    f["out.block_footprint"] = len(np.unique(out_lin[blk == 0]))
    f.update(_shape_feats(L, NB, NT))
    # constraint quantities
    f["_threads"] = NT
    f["_smem"] = smem_total
    f["_local"] = 4 * f["outputs_per_thread"]
    f["_vthreads"] = f["vthread_len"]
    return f


def enumerate_valid(space) -> List[Dict[str, int]]:
    """All divisor-respecting integer assignments of the SPLIT vars (INT vars excluded)."""
    names = [v.name for v in space.vars]
    split_vars = [j for j, v in enumerate(space.vars) if v.kind == 0]
    out = []

    def rec(k, cur):
        if k == len(split_vars):
            ok = all(s.extent % int(np.prod([cur[j] for j in s.vars])) == 0 for s in space.splits)
            if ok:
                out.append(dict(cur))
            return
        j = split_vars[k]
        ub = min(s.extent for s in space.splits if j in s.vars)
        for d in range(1, ub + 1):
            if all(s.extent % d == 0 for s in space.splits if j in s.vars):
                cur[j] = d
                # prune: partial products must divide
                if all(s.extent % int(np.prod([cur.get(i, 1) for i in s.vars])) == 0 for s in space.splits):
                    rec(k + 1, cur)
                del cur[j]
    rec(0, {})
    return [{names[j]: v for j, v in a.items()} for a in out]


def simulate_epilogue(spec, x: Dict[str, int]) -> Dict[str, float]:
    """The fused bias / activation epilogue statement (felix_inputs/programs.py docstring), counted from
    its enumerated instances (block, thread, v_*, in_*): one instance per output element."""
    sp, _ = _levels(spec, x)
    L = [("v", s["name"], s["V"]) for s in sp] + [("in", s["name"], s["I"]) for s in sp]
    blk_ranges = [range(s["Nb"]) for s in sp]
    thr_ranges = [range(s["T"]) for s in sp]
    rows = []
    for bi, bt in enumerate(itertools.product(*blk_ranges)):
        for ti, tt in enumerate(itertools.product(*thr_ranges)):
            for li in itertools.product(*[range(e) for _, _, e in L]):
                rows.append((bi, ti) + tuple(bt) + tuple(tt) + tuple(li))
    arr = np.array(rows, dtype=np.int64)
    ns = len(sp)
    blk, thr = arr[:, 0], arr[:, 1]
    bvec, tvec, lvec = arr[:, 2:2 + ns], arr[:, 2 + ns:2 + 2 * ns], arr[:, 2 + 2 * ns:]
    li = {(k, a): lvec[:, n] for n, (k, a, _) in enumerate(L)}
    idx = {}
    for i, s in enumerate(sp):
        idx[s["name"]] = (bvec[:, i] * (s["V"] * s["T"] * s["I"]) + li[("v", s["name"])] * (s["T"] * s["I"])
                          + tvec[:, i] * s["I"] + li[("in", s["name"])])
    n = len(blk)
    E = int(np.prod([s["E"] for s in sp]))
    assert n == E
    f: Dict[str, float] = {}
    f["float_mad"] = 0
    f["float_addsub"] = E if spec.bias else 0
    f["float_cmp"] = E if spec.relu else 0
    f["float_math"] = E if spec.gelu else 0
    NB, NT = len(np.unique(blk)), len(np.unique(thr))
    f["blockIdx_len"] = NB
    f["vthread_len"] = int(np.prod([s["V"] for s in sp]))
    f["threadIdx_len"] = NT
    t0 = (blk == 0) & (thr == 0)
    f["outputs_per_thread"] = int(t0.sum())
    f["stmts_per_thread"] = int(t0.sum())
    nontriv = sum(1 for _, _, e in L if e > 1)
    f["n_nontrivial_loops"] = nontriv
    f["int_addsub"] = n * (2 + nontriv)
    f["int_mul"] = n * sum(1 for s in sp if s["Nb"] > 1)
    f["reduction_outer_iters"] = 1
    per_thread = int(t0.sum())
    if spec.unroll:
        U = x["UNROLL"]
        f["unroll_len"] = min(U, per_thread)
        cum, cnt = 1, 0
        for _, _, e in reversed(L):
            cum *= e
            if cum <= U:
                cnt += 1
        f["unrolled_loops"] = cnt
    else:
        f["unroll_len"] = 0
        f["unrolled_loops"] = 0
    inner = None
    for pos in range(len(L) - 1, -1, -1):
        if L[pos][2] > 1:
            inner = pos
            break
    names = ["block_footprint", "global_load_elems", "global_bytes", "coop_loads_per_thread", "thread_footprint",
             "thread_reuse", "block_reuse", "global_reuse", "innermost_stride", "shared_bytes",
             "vectorizable", "load_ratio", "smem_inner_stride", "smem_tile_elems", "smem_tile_util"]
    if inner is None:
        sel0 = sel1 = None
    else:
        sel0 = t0 & np.all(lvec == 0, axis=1)
        one = np.zeros(len(L), dtype=np.int64)
        one[inner] = 1
        sel1 = t0 & np.all(lvec == one[None, :], axis=1)
    out_lin = np.zeros(n, dtype=np.int64)
    for s in sp:
        out_lin = out_lin * s["E"] + idx[s["name"]]
    gsum = smem = 0
    for slot in range(len(spec.inputs)):
        if slot == 0 and spec.bias:
            lin = idx[spec.bias_axis]                       # Bias[s_c], a vector
            b0 = blk == 0
            blk_fp = len(np.unique(lin[b0]))
            gl = int(sum(len(np.unique(lin[blk == bb])) for bb in range(NB)))
            thr_fp = len(np.unique(lin[t0]))
            pt = np.bincount(np.arange(blk_fp) % NT, minlength=NT)
            stride = 0 if inner is None else int(lin[sel1][0] - lin[sel0][0])
            box, local = _smem_layout([lin], b0)
            sstride = 0 if inner is None else int(local[sel1][0] - local[sel0][0])
            size = spec.axis_extent(spec.bias_axis)
            vals = [blk_fp, gl, 4 * gl, int(pt.max()), thr_fp, per_thread / thr_fp, int(b0.sum()) / blk_fp, n / gl,
                    stride, 4 * blk_fp, 1 if stride == 1 else 0, gl / size, sstride, box[0], blk_fp / box[0]]
            gsum += 4 * gl
            smem += 4 * blk_fp
        else:
            vals = [0] * 15
        for nm, v in zip(names, vals):
            f[f"in{slot}.{nm}"] = v
    n_ops = int(spec.bias) + int(spec.relu) + int(spec.gelu)
    f["out.stores"] = E
    f["shared_bytes_total"] = smem
    f["local_bytes"] = 4 * f["outputs_per_thread"]
    f["flops_per_global_byte"] = n_ops * E / (gsum + 4 * E)
    f["flops_per_thread"] = n_ops * per_thread
    f["global_bytes_per_block"] = gsum / NB
    ostride = 0 if inner is None else int(out_lin[sel1][0] - out_lin[sel0][0])
    f["out.innermost_stride"] = ostride
    f["out.vectorizable"] = 1 if ostride == 1 else 0
    f["out.block_footprint"] = len(np.unique(out_lin[blk == 0]))
    f.update(_shape_feats(L, NB, NT))
    return f
