"""GPU parity, part 2: the whole operator set, raw features, the search path's own gradient, the
tile kernel at full size, and the non-finite rule — all through the C ABI against the float64 oracle.

Tolerances as tests/test_gpu_parity.py (BASELINE.json north_star):
  raw features F, phi, g      rel <= 1e-4, floor 1
  cost c, loss L              <= 1e-4 of the batch RMS
  dL/dy                       normwise per candidate <= 1e-3, R-kink exemption (< 1 %)
  rounding, validity, top-k   bit-exact (scores rel <= 1e-12)
R-NaN (DESIGN.md readings): a candidate whose loss or gradient is non-finite is not updated; a rounded
schedule with a non-finite hard feature is invalid.
"""
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
    return m


_cache = {}


def _setup(fx, key, make, dims=fi.DEFAULT_MLP):
    if key not in _cache:
        sp = make()
        mlp = fi.make_mlp(dims)
        _cache[key] = (sp, mlp, fx.Space(sp), fx.CostModel.from_weights(mlp))
    return _cache[key]


def kink_margin(zs):
    m = np.full(zs[0].shape[1], np.inf)
    for z in zs:
        rms = np.sqrt(np.mean(z * z, axis=0)) + 1e-300
        m = np.minimum(m, np.min(np.abs(z), axis=0) / rms)
    return m


def rel_floor1(a, b):
    return np.abs(a - b) / np.maximum(np.abs(b), 1.0)


def check_grad(got, gref, zs, tol=1e-3):
    err = np.linalg.norm(got - gref, axis=0) / np.maximum(np.linalg.norm(gref, axis=0), 1e-12)
    bad = err > tol
    exempt = bad & (kink_margin(zs) < 1e-4)
    assert not np.any(bad & ~exempt), (np.nonzero(bad & ~exempt)[0][:10], err[bad & ~exempt][:10])
    assert exempt.mean() < 0.01
    return err


def check_eval(out, ref, cols=None):
    sel = (lambda a: a) if cols is None else (lambda a: a[..., cols])
    assert np.max(rel_floor1(sel(out["F"]), ref.F)) <= 1e-4, "raw features"
    assert np.max(rel_floor1(sel(out["phi"]), ref.phi)) <= 1e-4, "phi"
    assert np.max(rel_floor1(sel(out["g"]), ref.g)) <= 1e-4, "g"
    for key, r in (("cost", ref.c), ("loss", ref.loss)):
        assert np.max(np.abs(sel(out[key]) - r)) / np.sqrt(np.mean(r ** 2)) <= 1e-4, key
    check_grad(sel(out["grad"]), ref.grad, ref.zs)


# ------------------------------------------------------------------------------------ all 25 opcodes
def test_allops_space_uses_every_opcode():
    sp = fi.allops_space()
    assert set(int(o) for o in sp.nodes["op"]) == set(range(fi.N_OPS))
    assert len(set(sp.feature_roots.tolist())) == 82


@pytest.mark.parametrize("n", [600, 4096])
def test_allops_eval_parity(fx, n):
    """Every opcode's smooth forward, slog, MLP, penalty and adjoint rule on the GPU against the oracle:
    raw F, phi, g, cost, loss, dL/dy (eval kernels) and loss / dL/dy of the search path."""
    sp, mlp, space, cm = _setup(fx, "allops", fi.allops_space)
    y0 = fi.make_y0(sp, n, seed=41)
    yt = torch.from_numpy(y0).cuda()
    out = {k: v.cpu().numpy() for k, v in space.eval(cm, yt, lam=0.7, features=True).items()}
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 0.7)
    assert np.all(np.isfinite(ref.loss))
    check_eval(out, ref)
    sp_out = {k: v.cpu().numpy() for k, v in space.eval_search_path(cm, yt, lam=0.7).items()}
    assert np.max(np.abs(sp_out["loss"] - ref.loss)) / np.sqrt(np.mean(ref.loss ** 2)) <= 1e-4
    check_grad(sp_out["grad"], ref.grad, ref.zs)
    assert torch.equal(yt, torch.from_numpy(y0).cuda())            # the hook does not move y


def test_allops_rounding_validity_topk_score(fx):
    sp, mlp, space, cm = _setup(fx, "allops", fi.allops_space)
    y0 = fi.make_y0(sp, 700, seed=42, margin=1.0)
    y0[:, 350:370] = y0[:, :20]
    yt = torch.from_numpy(y0).cuda()
    sched, valid = space.round(yt)
    rs = fo.round_schedules(sp, y0)
    assert np.array_equal(sched.cpu().numpy(), rs)
    rv = fo.validate(sp, rs)
    assert np.array_equal(valid.cpu().numpy().astype(bool), rv)
    assert 0.05 < rv.mean() < 1.0                                   # both outcomes occur
    got = space.score(cm, sched).cpu().numpy()
    ref = fo.score(sp, mlp.W, mlp.b, rs)
    ok = np.isfinite(ref)
    assert np.all(np.abs(got[ok] - ref[ok]) <= 1e-12 * np.maximum(np.abs(ref[ok]), 1e-3))
    idx, sc, sch = space.round_topk(cm, yt, 16, index_base=5)
    ridx, rsc, rsch = fo.round_topk(sp, mlp.W, mlp.b, y0, 16, index_base=5)
    assert np.array_equal(idx, ridx) and np.array_equal(sch, rsch)
    assert np.all(np.abs(sc - rsc) <= 1e-12 * np.maximum(np.abs(rsc), 1e-3))


def test_allops_one_adam_step(fx):
    sp, mlp, space, cm = _setup(fx, "allops", fi.allops_space)
    y0 = fi.make_y0(sp, 500, seed=43)
    y = torch.from_numpy(y0).cuda()
    loss = torch.empty(500, device="cuda")
    space.search(cm, y, 1, lr=0.05, lam=1.0, init_from_y=True, final_loss=loss)
    ob = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    ry, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 1, lr=0.05, lam=1.0)
    exempt = (np.abs(ob.grad) < 1e-6) | (kink_margin(ob.zs) < 1e-4)[None, :]
    assert not np.any((np.abs(y.cpu().numpy() - ry) > 1e-4 * (1 + np.abs(ry))) & ~exempt)
    assert np.max(np.abs(loss.cpu().numpy() - ob.loss)) / np.sqrt(np.mean(ob.loss ** 2)) <= 1e-4


# ------------------------------------------------------------------------------------ search path, full size
def test_search_path_gradient_c2_full_population(fx):
    """BASELINE configs[1] (C2, 4096 seeds) in the launch configuration felix_search uses: the dL/dy
    its Adam step consumes (split-cone partial adjoints, summed in fixed order) and its loss, for
    EVERY candidate, against the oracle; raw features / phi / g / cost from the eval kernels too."""
    sp, mlp, space, cm = _setup(fx, "C2", fi.c2_space)
    y0 = fo.init_sample(sp, 4096, 0x5EED0002)
    yt = torch.from_numpy(y0).cuda()
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    out = {k: v.cpu().numpy() for k, v in space.eval_search_path(cm, yt).items()}
    assert np.max(np.abs(out["loss"] - ref.loss)) / np.sqrt(np.mean(ref.loss ** 2)) <= 1e-4
    check_grad(out["grad"], ref.grad, ref.zs)
    ev = {k: v.cpu().numpy() for k, v in space.eval(cm, yt, features=True).items()}
    check_eval(ev, ref)


def test_search_path_gradient_c2_made_starts(fx):
    """Same on starting points that violate the validity bounds (penalty terms active)."""
    sp, mlp, space, cm = _setup(fx, "C2", fi.c2_space)
    y0 = fi.make_y0(sp, 4096, seed=44)
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    out = {k: v.cpu().numpy() for k, v in space.eval_search_path(cm, torch.from_numpy(y0).cuda()).items()}
    assert np.max(np.abs(out["loss"] - ref.loss)) / np.sqrt(np.mean(ref.loss ** 2)) <= 1e-4
    check_grad(out["grad"], ref.grad, ref.zs)


@pytest.mark.timeout(900)
def test_tile_kernel_full_size_c5_shard(fx):
    """C5's per-GPU shard (131072 candidates): the MLP runs in the persistent multi-tile-per-CTA tile
    kernel (one full wave of 128-row tiles and more).  Raw F, phi, g, cost, loss and dL/dy from the
    eval kernels, and loss / dL/dy of the search path, on 256 sampled candidates."""
    sp, mlp, space, cm = _setup(fx, "C5", fi.c5_space)
    n = 131072
    y0 = fo.init_sample(sp, n, 0x5EED0005)
    y0[:, ::7] = fi.make_y0(sp, n, seed=45)[:, ::7]            # some starts with active penalties
    yt = torch.from_numpy(np.ascontiguousarray(y0)).cuda()
    pick = np.sort(np.random.default_rng(3).choice(n, 256, replace=False))
    pick[-1] = n - 1                                            # the ragged last tile
    ref = fo.objective(sp, mlp.W, mlp.b, y0[:, pick].astype(np.float64), 1.0)
    ev = {k: v.cpu().numpy() for k, v in space.eval(cm, yt, features=True).items()}
    check_eval(ev, ref, cols=pick)
    sp_out = {k: v.cpu().numpy()[..., pick] for k, v in space.eval_search_path(cm, yt).items()}
    assert np.max(np.abs(sp_out["loss"] - ref.loss)) / np.sqrt(np.mean(ref.loss ** 2)) <= 1e-4
    check_grad(sp_out["grad"], ref.grad, ref.zs)


# ------------------------------------------------------------------------------------ R-NaN
def _rnan_y0(sp, n, seed):
    y0 = fi.make_y0(sp, n, seed=seed)
    # keep x_a away from the LOG / DIV singularities at 3 and 2 (a 1-ulp exp difference must not
    # decide which side of them a candidate is on)
    xa = np.exp(y0[0].astype(np.float64))
    for s in (2.0, 3.0):
        near = np.abs(xa - s) < 1e-3
        y0[0, near] = np.float32(np.log(s + 0.01))
    return y0


def _ok(loss, grad):
    return np.isfinite(loss) & np.all(np.isfinite(grad), axis=0)


def test_rnan_eval_and_freeze(fx):
    sp, mlp, space, cm = _setup(fx, "rnan", fi.rnan_space)
    n = 640
    y0 = _rnan_y0(sp, n, 46)
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    rok = _ok(ref.loss, ref.grad)
    assert 0.2 < rok.mean() < 0.95
    yt = torch.from_numpy(y0).cuda()
    ev = {k: v.cpu().numpy() for k, v in space.eval(cm, yt).items()}
    assert np.array_equal(_ok(ev["loss"], ev["grad"]), rok)
    spo = {k: v.cpu().numpy() for k, v in space.eval_search_path(cm, yt).items()}
    assert np.array_equal(_ok(spo["loss"], spo["grad"]), rok)
    # finite candidates: the usual tolerances
    s = np.sqrt(np.mean(ref.loss[rok] ** 2))
    assert np.max(np.abs(ev["loss"][rok] - ref.loss[rok])) / s <= 1e-4
    assert np.max(np.abs(spo["loss"][rok] - ref.loss[rok])) / s <= 1e-4
    zs = [z[:, rok] for z in ref.zs]
    check_grad(ev["grad"][:, rok], ref.grad[:, rok], zs)
    check_grad(spo["grad"][:, rok], ref.grad[:, rok], zs)
    # one Adam step: non-finite candidates are not moved (bit for bit), the rest as the oracle
    y = torch.from_numpy(y0).cuda()
    space.search(cm, y, 1, init_from_y=True)
    got = y.cpu().numpy()
    ry, rm, rv, _ = fo.search(sp, mlp.W, mlp.b, y0, 1)
    assert np.array_equal(got[:, ~rok], y0[:, ~rok]) and np.array_equal(ry[:, ~rok], y0[:, ~rok].astype(np.float64))
    exempt = (np.abs(ref.grad) < 1e-6) | (kink_margin(ref.zs) < 1e-4)[None, :]
    bad = (np.abs(got - ry) > 1e-4 * (1 + np.abs(ry))) & ~exempt & rok[None, :]
    assert not np.any(bad)
    # several steps: the frozen set is the same on both sides
    y = torch.from_numpy(y0).cuda()
    space.search(cm, y, 6, init_from_y=True)
    ry6, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 6)
    frozen_gpu = np.all(y.cpu().numpy() == y0, axis=0)
    frozen_ref = np.all(ry6 == y0.astype(np.float64), axis=0)
    assert np.array_equal(frozen_gpu, frozen_ref) and np.array_equal(frozen_ref, ~rok)


def test_rnan_rounding_validity_topk(fx):
    """Hard semantics at integer points: LOG(x_0 - 3) is NaN / -inf for x_0 in {1, 2}, x_1 / (x_0 - 2)
    divides by zero at x_0 = 2; those schedules are invalid on both sides and never in the top-k."""
    sp, mlp, space, cm = _setup(fx, "rnan", fi.rnan_space)
    y0 = fi.make_y0(sp, 500, seed=47, margin=0.5)
    yt = torch.from_numpy(y0).cuda()
    sched, valid = space.round(yt)
    rs = fo.round_schedules(sp, y0)
    assert np.array_equal(sched.cpu().numpy(), rs)
    rv = fo.validate(sp, rs)
    assert np.array_equal(valid.cpu().numpy().astype(bool), rv)
    assert not np.any(rv & (rs[:, 0] <= 2)) and np.any(rv)
    idx, sc, sch = space.round_topk(cm, yt, 16)
    ridx, rsc, rsch = fo.round_topk(sp, mlp.W, mlp.b, y0, 16)
    assert np.array_equal(idx, ridx) and np.array_equal(sch, rsch) and np.all(sch[:, 0] >= 4)


def test_module_cache_reuses_compiled_kernels(fx):
    """A second space with the same DAG loads the process-wide cubin cache (felix_api.cu
    compile_module_parts) instead of recompiling, and its kernels give bit-identical results."""
    sp, mlp, space, cm = _setup(fx, "C1", lambda: fi.config("C1").spaces[0])
    again = fx.Space(sp)
    assert again.info.nvrtc_ms < 1000.0
    y0 = torch.from_numpy(fi.make_y0(sp, 300, seed=5)).cuda()
    a, b = space.eval(cm, y0, lam=1.0), again.eval(cm, y0, lam=1.0)
    for key in ("phi", "cost", "loss", "grad"):
        assert torch.equal(a[key], b[key]), key
