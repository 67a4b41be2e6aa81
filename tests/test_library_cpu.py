"""Host-side checks of the C-ABI library that need no GPU (-m "not gpu"): the .so loads, exports every
symbol include/felix.h declares, its opcode/struct layout matches the input format, the space
validator rejects malformed input, and the generated expression kernels compile for sm_100a (NVRTC)."""
import ctypes
import os
import re

import numpy as np
import pytest

import felix_inputs as fi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = open(os.path.join(ROOT, "include", "felix.h")).read()


@pytest.fixture(scope="module")
def fx():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_asplos_zhaosam24_b200 as m
    return m


def test_library_exports_every_header_symbol(fx):
    declared = set(re.findall(r"FELIX_EXPORT\s+[\w\s\*]+?\b(felix_\w+)\s*\(", HEADER))
    assert len(declared) >= 16
    lib = ctypes.CDLL(fx.LIB_PATH)
    for name in declared:
        assert hasattr(lib, name), name
    assert declared == set(fx.EXPORTED)
    assert fx.abi_version() == int(re.search(r"#define FELIX_ABI_VERSION (\d+)", HEADER).group(1))


def test_library_does_not_link_libcuda(fx):
    import subprocess
    out = subprocess.run(["ldd", fx.LIB_PATH], capture_output=True, text=True).stdout
    assert "libcuda.so" not in out   # driver reached through cudaGetDriverEntryPoint at run time


def test_opcodes_match_header():
    for name, val in re.findall(r"FELIX_OP_(\w+) = (\d+)", HEADER):
        assert getattr(fi, "OP_" + name) == int(val), name
    assert fi.NODE_DTYPE.itemsize == 24


def _space(nodes, froots, croots=(), vars_=None, splits=None):
    vars_ = vars_ or [fi.Var("a", fi.VAR_SPLIT, 1, 64)]
    splits = splits if splits is not None else [fi.Split(64, [0])]
    arr = np.zeros(len(nodes), dtype=fi.NODE_DTYPE)
    for i, r in enumerate(nodes):
        arr[i] = r
    return fi.Space("t", vars_, splits, arr, np.array(froots, np.int32), np.array(croots, np.int32))


@pytest.mark.parametrize("case,status", [
    ("forward_ref", 2), ("bool_root", 2), ("type_error", 2), ("var_range", 2),
    ("int_in_split", 1), ("split_var_no_split", 1), ("bad_opcode", 2),
])
def test_validator_rejects(fx, case, status):
    V = (fi.OP_VAR, -1, -1, -1, 0.0)
    C1 = (fi.OP_CONST, -1, -1, -1, 1.0)
    if case == "forward_ref":
        sp = _space([V, (fi.OP_ADD, 0, 2, -1, 0.0), C1], [1])
    elif case == "bool_root":
        sp = _space([V, C1, (fi.OP_GT, 0, 1, -1, 0.0)], [2])
    elif case == "type_error":
        sp = _space([V, C1, (fi.OP_AND, 0, 1, -1, 0.0)], [0])
    elif case == "var_range":
        sp = _space([(fi.OP_VAR, -1, -1, -1, 3.0)], [0])
    elif case == "int_in_split":
        sp = _space([V], [0], vars_=[fi.Var("u", fi.VAR_INT, 1, 8)], splits=[fi.Split(8, [0])])
    elif case == "split_var_no_split":
        sp = _space([V], [0], splits=[])
    else:
        sp = _space([(99, -1, -1, -1, 0.0)], [0])
    with pytest.raises(fx.FelixError) as e:
        fx.codegen(sp)
    assert e.value.status == status


@pytest.mark.parametrize("which", ["paper", "C1", "C2", "allops", "rnan"])
def test_generated_kernels_compile_for_sm100a(fx, which):
    sp = {"paper": fi.paper_example_space, "C1": fi.c1_space, "C2": fi.c2_space, "allops": fi.allops_space,
          "rnan": fi.rnan_space}[which]()
    src = fx.codegen(sp, compile=True)
    for k in ("felix_fwd", "felix_rev_adam", "felix_rev_eval", "felix_hard", "felix_init", "felix_fwd_adam", "felix_rev_sc",
              "felix_adam_sc"):
        assert re.search(r"__global__ void __launch_bounds__\([^)]*\) " + k + r"\(", src), k


def test_device_calls_fail_loudly_without_gpu(fx):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(fx.FelixError) as e:
        fx.Space(fi.c1_space())
    assert e.value.status == 5


def _kernel_body(src, name):
    i = src.index(" " + name + "(")
    j = src.find('extern "C" __global__', i + 1)
    return src[i:j if j > 0 else len(src)]


@pytest.mark.parametrize("P", ["1", "2", "4", "8"])
def test_split_cone_codegen_partitions_every_seed_once(fx, P):
    """The generated split-cone reverse kernel has one branch per cone, seeds every variable-dependent
    feature's adjoint from dL/dphi exactly once across the cones (the cone partition covers the roots
    without overlap), and each cone writes a partial adjoint for every variable; the cone-group reverse
    kernel (felix_rev_adam's body) seeds the same features once.  felix_fwd_adam applies step
    *step_ctr - 1 (the reverse kernel advances the counter)."""
    sp = fi.c2_space()
    with fx.tuned(codegen_cone_width=int(P), codegen_replicas=1):
        src = fx.codegen(sp)
    rev = _kernel_body(src, "felix_rev_sc")
    assert len(re.findall(r"if \(cq_ == \d+\)", rev)) == int(P)
    seeds = re.findall(r"dphi\[\(size_t\)(\d+) \* ld_dphi", rev)
    n_dep = sum(1 for r in sp.feature_roots if _depends_on_var(sp, r))
    assert sorted(int(k) for k in seeds) == sorted(set(int(k) for k in seeds)) and len(seeds) == n_dep
    for q in range(int(P)):
        for j in range(sp.n_vars):
            assert f"part[((size_t){q} * NV + {j}) * n + c]" in rev
    body = src[src.index("void rev_body("):src.index('extern "C" __global__ void __launch_bounds__(PG * 32 * NREP) felix_rev_adam')]
    assert sorted(re.findall(r"dphi\[\(size_t\)(\d+) \* ld_dphi", body)) == sorted(seeds)
    assert "*step_ctr - 1" in src and "*step_ctr += 1" in rev


def _depends_on_var(sp, root):
    seen, stack = set(), [root]
    while stack:
        i = stack.pop()
        if i in seen:
            continue
        seen.add(i)
        op, a, b, c, _ = sp.nodes[i]
        if op == fi.OP_VAR:
            return True
        stack.extend(x for x in (a, b, c) if x >= 0)
    return False


def test_tune_knobs_validated(fx):
    """felix_tune: the only way to change execution knobs (the library reads no environment variables)."""
    with pytest.raises(fx.FelixError) as e:
        fx.tune(no_such_knob=1)
    assert e.value.status == 1
    with pytest.raises(fx.FelixError):
        fx.tune(cone_width=3)
    with fx.tuned(mlp="chain", cone_width=8, split_cone=0):
        pass
    csrc = os.path.join(ROOT, "paper_conf_asplos_zhaosam24_b200", "csrc")
    for f in os.listdir(csrc):
        assert "getenv" not in open(os.path.join(csrc, f)).read(), f


def test_split_cone_reverse_is_fp32_and_forward_keeps_fp64_values(fx):
    """Precision plan of the expression kernels: the split-cone reverse kernel is FP32
    throughout (no double arithmetic besides the penalty it stores; comparison / logic nodes carry their
    complements c = 1 - v), the search forward evaluates node
    values in FP64 with FP32 tails of the smooth step (sm_Sf), min / max gaps in FP64."""
    src = fx.codegen(fi.c2_space())
    rev = _kernel_body(src, "felix_rev_sc")
    assert "const double" not in rev and "sf_tail(" in rev and "sf_dSh(" in rev and "const float c" in rev
    fwd = src[src.index("void fwd_body("):src.index('extern "C" __global__ void __launch_bounds__(PG * 32 * NREP) felix_fwd(')]
    assert "sm_Sf(" in fwd and "const double v" in fwd


def test_merge_topk_host_call_against_brute_force(fx):
    """felix_merge_topk (the multi-GPU exchange's merge, host code in libfelix) against a brute-force
    reference: rank every row by (score desc, key asc; NaN last), keep the first row of each schedule."""
    rng = np.random.default_rng(5)
    for trial in range(20):
        R, nv, k = int(rng.integers(0, 40)), int(rng.integers(1, 5)), int(rng.integers(0, 12))
        key = rng.permutation(1000)[:R].astype(np.int64)
        key[rng.random(R) < 0.15] = -1                                   # empty rows
        sched = rng.integers(1, 3, size=(R, nv)).astype(np.int32)        # many duplicate schedules
        score = np.round(rng.normal(size=R), 1)                          # many equal scores
        score[rng.random(R) < 0.1] = np.nan
        rows = [r for r in range(R) if key[r] >= 0]
        rows.sort(key=lambda r: (np.isnan(score[r]), -score[r] if not np.isnan(score[r]) else 0.0, key[r]))
        seen, ref = set(), []
        for r in rows:
            t = tuple(sched[r])
            if t in seen:
                continue
            seen.add(t)
            ref.append(r)
        ref = ref[:k]
        ko, so, xo = fx.merge_topk(key, score, sched.reshape(R, nv), k)
        assert list(ko) == [key[r] for r in ref]
        assert np.array_equal(so, score[ref], equal_nan=True)
        assert np.array_equal(xo, sched[ref].reshape(len(ref), nv))
