"""GPU parity: the CUDA path (through the C ABI) against the float64 oracle on the same seeded inputs.

Tolerances (BASELINE.json north_star; SURVEY §8(c) parity rules):
  features phi, g          rel <= 1e-4, floor 1
  cost c, loss L           rel <= 1e-4, floor = RMS over the batch
  gradient dL/dy           normwise per candidate <= 1e-3; R-kink exemption (oracle kink margin
                           min |z| / rms(z) < 1e-4), exempt candidates < 1%
  y after one Adam step    |dy| <= 1e-4 (1 + |y|), components with |g_ref| < 1e-6 exempt
  rounding, validity       bit-exact (common input: the GPU's y)
  top-k (idx, sched)       bit-exact; scores rel <= 1e-12
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
    return m


CASES = {
    # name: (space factory, MLP dims, n)   n spans several 128-row tiles plus a ragged tail
    "paper": (fi.paper_example_space, (82, 64, 1), 200),
    "C1": (fi.c1_space, fi.C1_MLP, 300),
    "C2": (fi.c2_space, fi.DEFAULT_MLP, 1000),
    "C5": (fi.c5_space, fi.DEFAULT_MLP, 389),
    "bmm": (lambda: fi.bert_spaces()[1], fi.DEFAULT_MLP, 257),
    # C3 / C4 shapes: ResNet-50 conv1 7x7 stride 2 (halo with stride), a 1x1 stride-2 downsample,
    # BERT QKV dense (2-var reduction split)
    "r50_conv1": (lambda: fi.resnet50_spaces()[0], fi.DEFAULT_MLP, 300),
    "r50_ds1x1": (lambda: fi.resnet50_spaces()[8], fi.DEFAULT_MLP, 160),
    "bert_qkv": (lambda: fi.bert_spaces()[0], fi.DEFAULT_MLP, 222),
    # TenSet-style per-statement features: [reduction | fused bias+ReLU epilogue], C = sum_s MLP(phi_s)
    "C2_2stmt": (fi.c2_space_two_statements, fi.DEFAULT_MLP, 700),
}

_cache = {}


def _setup(fx, name):
    if name not in _cache:
        make, dims, n = CASES[name]
        sp = make()
        mlp = fi.make_mlp(dims)
        _cache[name] = (sp, mlp, n, fx.Space(sp), fx.CostModel.from_weights(mlp))
    return _cache[name]


def kink_margin(zs):
    m = np.full(zs[0].shape[1], np.inf)
    for z in zs:
        rms = np.sqrt(np.mean(z * z, axis=0)) + 1e-300
        m = np.minimum(m, np.min(np.abs(z), axis=0) / rms)
    return m


@pytest.mark.parametrize("name", list(CASES))
def test_eval_parity(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=11)
    out = {k: v.cpu().numpy() for k, v in space.eval(cm, torch.from_numpy(y0).cuda(), lam=1.0).items()}
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    # features (slog) and constraint values
    e_phi = np.abs(out["phi"] - ref.phi) / np.maximum(np.abs(ref.phi), 1.0)
    k, i = np.unravel_index(np.argmax(e_phi), e_phi.shape)
    assert e_phi[k, i] <= 1e-4, (sp.feature_names[k], i, out["phi"][k, i], ref.phi[k, i], ref.F[k, i], y0[:, i])
    e_g = np.abs(out["g"] - ref.g) / np.maximum(np.abs(ref.g), 1.0)
    assert np.max(e_g) <= 1e-4, np.unravel_index(np.argmax(e_g), e_g.shape)
    # cost and loss, floor = RMS over the batch
    for key, r in (("cost", ref.c), ("loss", ref.loss)):
        s = np.sqrt(np.mean(r ** 2))
        assert np.max(np.abs(out[key] - r)) / s <= 1e-4, key
    # gradient, normwise per candidate, R-kink exemption
    km = kink_margin(ref.zs)
    err = np.linalg.norm(out["grad"] - ref.grad, axis=0) / np.maximum(np.linalg.norm(ref.grad, axis=0), 1e-12)
    bad = err > 1e-3
    exempt = bad & (km < 1e-4)
    assert not np.any(bad & ~exempt), (np.nonzero(bad & ~exempt)[0][:10], err[bad & ~exempt][:10])
    assert exempt.mean() < 0.01


@pytest.mark.parametrize("name", ["C1", "C2", "C2_2stmt"])
def test_one_adam_step_parity(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=12)
    y = torch.from_numpy(y0).cuda()
    loss = torch.empty(n, device="cuda")
    space.search(cm, y, 1, lr=0.05, lam=1.0, init_from_y=True, final_loss=loss)
    got = y.cpu().numpy()
    ob = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    ry, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 1, lr=0.05, lam=1.0)
    tol = 1e-4 * (1 + np.abs(ry))
    exempt = (np.abs(ob.grad) < 1e-6) | (kink_margin(ob.zs) < 1e-4)[None, :]
    bad = (np.abs(got - ry) > tol) & ~exempt
    assert not np.any(bad), (np.argwhere(bad)[:10], got[bad][:10], ry[bad][:10])
    s = np.sqrt(np.mean(ob.loss ** 2))
    assert np.max(np.abs(loss.cpu().numpy() - ob.loss)) / s <= 1e-4


@pytest.mark.parametrize("name", list(CASES))
def test_rounding_validity_bit_exact(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=13, margin=1.0)
    yt = torch.from_numpy(y0).cuda()
    sched, valid = space.round(yt)
    rs = fo.round_schedules(sp, y0)
    assert np.array_equal(sched.cpu().numpy(), rs)
    assert np.array_equal(valid.cpu().numpy().astype(bool), fo.validate(sp, rs))


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_rounding_at_midpoints_bit_exact(fx, name):
    """Adversarial inputs: log-midpoints of consecutive divisors and INT half-integers (fp32)."""
    sp, mlp, n, space, cm = _setup(fx, name)
    rng = np.random.default_rng(5)
    y = np.zeros((sp.n_vars, 512), dtype=np.float32)
    for j, v in enumerate(sp.vars):
        if v.kind == fi.VAR_SPLIT:
            e = int(fi.var_upper_bounds(sp)[j])
            ds = [d for d in range(1, e + 1) if e % d == 0]
            mids = [0.5 * (math.log(a) + math.log(b)) for a, b in zip(ds[:-1], ds[1:])]
            y[j] = np.float32(rng.choice(mids + [math.log(d) for d in ds], size=512))
        else:
            y[j] = np.float32(np.log(rng.integers(v.lo, v.hi, size=512) + 0.5))
    sched, _ = space.round(torch.from_numpy(y).cuda())
    assert np.array_equal(sched.cpu().numpy(), fo.round_schedules(sp, y))


@pytest.mark.parametrize("name", ["C1", "C2", "C5"])
def test_score_fp64(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=14)
    rs = fo.round_schedules(sp, y0)
    got = space.score(cm, torch.from_numpy(rs).cuda()).cpu().numpy()
    ref = fo.score(sp, mlp.W, mlp.b, rs)
    ok = np.isfinite(ref)
    assert np.all(np.abs(got[ok] - ref[ok]) <= 1e-12 * np.maximum(np.abs(ref[ok]), 1e-3))


@pytest.mark.parametrize("name", ["C2", "C5"])
def test_score_tensor_core_and_cuda_core_kernels_agree(fx, name):
    """FP64 scoring layers on the FP64 tensor cores (default) and on the CUDA cores (score_dmma=0): both
    within 1e-12 of the oracle, and within 1e-13 of each other (only the summation order differs)."""
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=15)
    rs = fo.round_schedules(sp, y0)
    st = torch.from_numpy(rs).cuda()
    tc = space.score(cm, st).cpu().numpy()
    with fx.tuned(score_dmma=0):
        cc = space.score(cm, st).cpu().numpy()
    ref = fo.score(sp, mlp.W, mlp.b, rs)
    ok = np.isfinite(ref)
    assert np.array_equal(np.isfinite(tc), ok) and np.array_equal(np.isfinite(cc), ok)
    for got in (tc, cc):
        assert np.all(np.abs(got[ok] - ref[ok]) <= 1e-12 * np.maximum(np.abs(ref[ok]), 1e-3))
    assert np.all(np.abs(tc[ok] - cc[ok]) <= 1e-13 * np.maximum(np.abs(ref[ok]), 1e-3))


def _topk_equal(idx, sc, sched, ridx, rsc, rsched):
    assert len(idx) == len(ridx)
    assert np.all(np.abs(sc - rsc) <= 1e-12 * np.maximum(np.abs(rsc), 1e-3))
    # bit-exact except inside groups of scores tied to 1e-12 (order of equal keys is by index on both
    # sides; a sub-1e-12 difference between distinct schedules may swap them)
    i = 0
    while i < len(ridx):
        j = i
        while j + 1 < len(ridx) and abs(rsc[j + 1] - rsc[i]) <= 1e-12 * max(abs(rsc[i]), 1e-3):
            j += 1
        if j == i:
            assert idx[i] == ridx[i] and np.array_equal(sched[i], rsched[i])
        else:
            assert set(idx[i:j + 1]) == set(ridx[i:j + 1]) or j == len(ridx) - 1
        i = j + 1


@pytest.mark.parametrize("name", list(CASES))
def test_round_topk_parity(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=15)
    y0[:, n // 2: n // 2 + 20] = y0[:, :20]          # duplicates
    idx, sc, sched = space.round_topk(cm, torch.from_numpy(y0).cuda(), 16, index_base=777)
    ridx, rsc, rsched = fo.round_topk(sp, mlp.W, mlp.b, y0, 16, index_base=777)
    _topk_equal(idx, sc, sched, ridx, rsc, rsched)


def test_topk_shard_invariance(fx):
    """Top-k over two shards (index_base offsets) merged on the host == top-k over the whole set."""
    sp, mlp, n, space, cm = _setup(fx, "C2")
    y0 = fi.make_y0(sp, 4096, seed=16)
    full = space.round_topk(cm, torch.from_numpy(y0).cuda(), 16)
    recs = []
    for r in range(2):
        part = np.ascontiguousarray(y0[:, r * 2048:(r + 1) * 2048])
        i, s, sc = space.round_topk(cm, torch.from_numpy(part).cuda(), 16, index_base=r * 2048)
        recs += list(zip(i, s, map(tuple, sc)))
    seen, merged = {}, []
    for i, s, sc in sorted(recs, key=lambda t: (-t[1], t[0])):
        if sc not in seen:
            seen[sc] = i
            merged.append((i, s))
    assert [i for i, _ in merged[:16]] == list(full[0])


@pytest.mark.parametrize("name", ["C1", "C2", "C5", "r50_conv1"])
def test_init_sampler_parity(fx, name):
    sp, mlp, n, space, cm = _setup(fx, name)
    y = space.init_sample(2048, 0x5EED0002, index_base=100).cpu().numpy()
    ry = fo.init_sample(sp, 2048, 0x5EED0002, index_base=100)
    same = np.all(y == ry, axis=0)
    assert same.mean() >= 0.99
    g = np.concatenate([fo.eval_dag(sp, np.exp(y.astype(np.float64)), True).g_user, fo.auto_roots(sp, y.astype(np.float64))])
    assert np.all(g <= 1e-5)


def test_full_size_c2_sampled(fx):
    """BASELINE configs[1] size (4096 seeds, default MLP) in the launch configuration bench.py times;
    64 sampled candidates checked one by one against the oracle."""
    sp, mlp, _, space, cm = _setup(fx, "C2")
    y0 = fo.init_sample(sp, 4096, 0x5EED0002)
    out = {k: v.cpu().numpy() for k, v in space.eval(cm, torch.from_numpy(y0).cuda()).items()}
    pick = np.random.default_rng(0).choice(4096, 64, replace=False)
    ref = fo.objective(sp, mlp.W, mlp.b, y0[:, pick].astype(np.float64), 1.0)
    s = np.sqrt(np.mean(ref.c ** 2))
    assert np.max(np.abs(out["cost"][pick] - ref.c)) / s <= 1e-4
    err = np.linalg.norm(out["grad"][:, pick] - ref.grad, axis=0) / np.maximum(np.linalg.norm(ref.grad, axis=0), 1e-12)
    assert np.sum((err > 1e-3) & (kink_margin(ref.zs) >= 1e-4)) == 0


def test_full_size_c5_per_gpu_search_topk(fx):
    """C5's per-GPU shard (2^20 / 8 = 131072 candidates of the ViT-L fc1 space; its objective and gradient
    at full size are checked in test_gpu_parity_ops.py): a short search and its top-k, whose records
    must be valid rounded schedules with oracle-exact FP64 scores."""
    sp, mlp, _, space, cm = _setup(fx, "C5")
    n = 131072
    y0 = fo.init_sample(sp, n, 0x5EED0005)
    yt = torch.from_numpy(y0).cuda()
    space.search(cm, yt, 5, init_from_y=True)
    idx, sc, sched = space.round_topk(cm, yt, 64)
    assert len(idx) == 64 and len(set(map(tuple, sched))) == 64
    assert np.all(np.diff(sc) <= 0)
    assert fo.validate(sp, sched).all()
    assert np.allclose(fo.score(sp, mlp.W, mlp.b, sched), sc, rtol=1e-12, atol=0)
    assert np.array_equal(fo.round_schedules(sp, yt[:, idx].cpu().numpy()), sched)


def test_search_final_loss_matches_eval(fx):
    """The loss felix_search reports for its last step is the objective at the point that step
    started from (the same kernels as felix_eval)."""
    sp, mlp, _, space, cm = _setup(fx, "C2")
    y = torch.from_numpy(fi.make_y0(sp, 777, seed=9)).cuda()
    loss = torch.empty(777, device="cuda")
    space.search(cm, y, 3, init_from_y=True, final_loss=loss)
    # re-run two steps from scratch, then evaluate at the start of the third
    y2 = torch.from_numpy(fi.make_y0(sp, 777, seed=9)).cuda()
    space.search(cm, y2, 2, init_from_y=True)
    ev = space.eval(cm, y2)["loss"]
    # steps 1-2 are identical, so y2 == the start point of step 3 only up to Adam state: the
    # 3-step run used Adam moments of steps 1-2 for its update, not for its loss
    assert torch.allclose(loss, ev, rtol=1e-6, atol=1e-6)


def test_search_deterministic_and_improves(fx):
    sp, mlp, _, space, cm = _setup(fx, "C2")
    y1 = space.init_sample(4096, 0x5EED0002)
    y2 = y1.clone()
    l1 = torch.empty(4096, device="cuda")
    l2 = torch.empty(4096, device="cuda")
    space.search(cm, y1, 50, init_from_y=True, final_loss=l1)
    space.search(cm, y2, 50, init_from_y=True, final_loss=l2)
    assert torch.equal(y1, y2) and torch.equal(l1, l2)
    y0 = space.init_sample(4096, 0x5EED0002)
    l0 = space.eval(cm, y0)["loss"]
    assert l1.mean().item() < l0.mean().item()


def test_search_with_device_init_matches_init_sample(fx):
    sp, mlp, _, space, cm = _setup(fx, "C1")
    y = torch.empty((sp.n_vars, 64), device="cuda")
    space.search(cm, y, 0, rng_seed=0x5EED0001, init_from_y=False)
    assert torch.equal(y, space.init_sample(64, 0x5EED0001))


def test_edge_sizes(fx):
    sp, mlp, _, space, cm = _setup(fx, "C1")
    for n in (1, 127, 128, 129):
        y0 = fi.make_y0(sp, n, seed=n)
        out = space.eval(cm, torch.from_numpy(y0).cuda())
        ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
        s = max(np.sqrt(np.mean(ref.c ** 2)), 1e-6)
        assert np.max(np.abs(out["cost"].cpu().numpy() - ref.c)) / s <= 1e-4
    y = torch.empty((sp.n_vars, 0), device="cuda")
    space.search(cm, y, 3)                     # n = 0: no-op
    idx, sc, sched = space.round_topk(cm, torch.from_numpy(fi.make_y0(sp, 5, 1)).cuda(), 16)
    assert len(idx) <= 5


def test_shape_errors(fx):
    sp, mlp, _, space, cm = _setup(fx, "C1")
    bad = fx.CostModel.from_weights(fi.make_mlp((82, 64, 64, 1)))
    y = torch.zeros((sp.n_vars - 1, 10), device="cuda")
    with pytest.raises(fx.FelixError):
        space.eval(cm, y)
    other = fi.make_mlp((80, 64, 1))
    cm2 = fx.CostModel.from_weights(other)
    with pytest.raises(fx.FelixError) as e:
        space.eval(cm2, torch.zeros((sp.n_vars, 10), device="cuda"))
    assert e.value.status == 3
    with pytest.raises(fx.FelixError) as e:
        fx.CostModel.from_weights(fi.make_mlp((82, 100, 1)))
    assert e.value.status == 4
    del bad


@pytest.mark.parametrize("mode,cg", [("chain", 1), ("chain", 2), ("layers", 1), ("tile", 2)])
def test_mlp_execution_modes_agree(fx, mode, cg):
    """The tile-local fused MLP (1-SM and 2-SM cta_group::2 variants), the persistent chain (dataflow
    flags) and the per-layer kernels compute the same split-fp16 products in the same K order: cost and
    gradient agree to fp32 summation-order noise (the head partial sums are grouped differently).  The
    first backward layer takes the exact 0/1 mask with the head row folded into its weights."""
    sp = fi.c2_space()
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    n = 2000
    y0 = torch.from_numpy(fi.make_y0(sp, n, seed=5)).cuda()
    cm = fx.CostModel.from_weights(mlp)
    with fx.tuned(mlp="tile", tile_cta_group=1):
        base = fx.Space(sp).eval(cm, y0, lam=1.0)
    with fx.tuned(mlp=mode, tile_cta_group=cg, chain_cta_group=cg):
        other = fx.Space(sp).eval(cm, y0, lam=1.0)
    for key in ("cost", "grad"):
        a, b = base[key].cpu().numpy(), other[key].cpu().numpy()
        s = np.sqrt(np.mean(a.astype(np.float64) ** 2))
        assert np.max(np.abs(a - b)) / s <= 1e-5, key


@pytest.mark.parametrize("cg", [1, 2])
def test_tile_mlp_eval_parity_vs_oracle(fx, cg):
    """Tile-local fused MLP (forced; default only from one full wave of tiles) against the oracle on
    C2 and C5 shapes with a ragged last tile (and, for the 2-SM pairs, an odd tile count)."""
    with fx.tuned(mlp="tile", tile_cta_group=cg):
        for name, n in (("C2", 1000), ("C5", 389), ("C2_2stmt", 333)):
            make, dims, _ = CASES[name]
            sp = make()
            mlp = fi.make_mlp(dims)
            y0 = fi.make_y0(sp, n, seed=21)
            out = {k: v.cpu().numpy() for k, v in fx.Space(sp).eval(fx.CostModel.from_weights(mlp),
                                                                      torch.from_numpy(y0).cuda(), lam=1.0).items()}
            ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
            s = np.sqrt(np.mean(ref.c ** 2))
            assert np.max(np.abs(out["cost"] - ref.c)) / s <= 1e-4, name
            km = kink_margin(ref.zs)
            err = np.linalg.norm(out["grad"] - ref.grad, axis=0) / np.maximum(np.linalg.norm(ref.grad, axis=0), 1e-12)
            bad = (err > 1e-3) & ~(km < 1e-4)
            assert not np.any(bad), (name, np.nonzero(bad)[0][:10], err[bad][:10])


def _gpu_trajectory(space, cm, y0, T, **kw):
    """sigma_x_i, i = 0..T-1, as the GPU computes them: search(i steps) from y0 is deterministic and
    identical to the first i steps of a longer search (Adam state starts fresh every call)."""
    ys = [y0.copy()]
    for i in range(1, T):
        y = torch.from_numpy(y0).cuda()
        space.search(cm, y, i, init_from_y=True, **kw)
        ys.append(y.cpu().numpy())
    return ys


@pytest.mark.parametrize("name,T", [("C1", 5), ("C2", 4), ("bert_qkv", 4)])
def test_history_topk_parity(fx, name, T):
    """History rounding (Alg. 1 l.13/17/20-21): the device pool (per-step rounding, per-seed change
    filter, hash-set dedup with first (step, seed), FP64 scoring, ordered top-k) against the oracle on
    the GPU's own trajectory: idx / step / schedules bit-exact, scores rel <= 1e-12."""
    sp, mlp, n, space, cm = _setup(fx, name)
    y0 = fi.make_y0(sp, n, seed=31)
    y = torch.from_numpy(y0).cuda()
    space.search(cm, y, T, init_from_y=True, index_base=7000, history=True)
    idx, step, sc, sched, n_unique = space.history_topk(cm, 64)
    ys = _gpu_trajectory(space, cm, y0, T, index_base=7000)
    ridx, rstep, rsc, rsched, rn = fo.round_topk_history(sp, mlp.W, mlp.b, ys, 64, index_base=7000)
    assert n_unique == rn
    assert np.array_equal(idx, ridx) and np.array_equal(step, rstep) and np.array_equal(sched, rsched)
    assert np.max(np.abs(sc - rsc) / np.maximum(np.abs(rsc), 1e-300)) <= 1e-12


def test_history_full_size_c2_properties(fx):
    """Bench-size history (C2, 4096 seeds x 200 steps): records are valid, distinct, ordered, their
    scores equal felix_score of their schedules, steps/indices are in range, and the history's best is
    at least the best of the last evaluated point sigma_x_199 (which it contains)."""
    cfg = fi.config("C2")
    sp = cfg.spaces[0]
    mlp = fi.make_mlp(cfg.mlp_dims)
    space, cm = fx.Space(sp), fx.CostModel.from_weights(mlp)
    n, T = cfg.n_seeds, 200
    y = torch.empty((sp.n_vars, n), device="cuda")
    space.search(cm, y, T, rng_seed=cfg.rng_seed, init_from_y=False, history=True)
    idx, step, sc, sched, n_unique = space.history_topk(cm, 256)
    assert len(idx) == 256 and n_unique >= 256
    assert np.all((idx >= 0) & (idx < n)) and np.all((step >= 0) & (step < T))
    assert len({s.tobytes() for s in sched}) == len(sched)
    assert np.all(np.diff(sc) <= 0)
    rescored = space.score(cm, torch.from_numpy(sched).cuda()).cpu().numpy()
    assert np.array_equal(rescored, sc)
    y199 = torch.empty_like(y)
    space.search(cm, y199, T - 1, rng_seed=cfg.rng_seed, init_from_y=False)
    _, lsc, _ = space.round_topk(cm, y199, 1)
    assert sc[0] >= lsc[0]


def test_history_requires_recording(fx):
    sp, mlp, n, space, cm = _setup(fx, "C1")
    y = torch.from_numpy(fi.make_y0(sp, n, seed=3)).cuda()
    space.search(cm, y, 2, init_from_y=True)
    with pytest.raises(fx.FelixError):
        space.history_topk(cm, 8)


@pytest.mark.parametrize("n", [1000, 8192])
@pytest.mark.timeout(300)
def test_subgraph_concurrent_sketches(fx, n):
    """Eq. 3 over the C2 subgraph's three symbolic programs, searched concurrently on three streams
    (n=1000: cluster chains; n=8192: cooperative grid chains, which must not deadlock each other):
    the merged records equal the sequential run bit for bit and the oracle's merge of the per-program
    top-k lists."""
    from paper_conf_asplos_zhaosam24_b200.subgraph import SubgraphSearch
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    sks = fi.c2_sketches()
    drv = SubgraphSearch(sks, cm)
    T = 12 if n == 1000 else 4
    conc = drv.run(n, T, 16, rng_seed=77, concurrent=True)
    seq = drv.run(n, T, 16, rng_seed=77, concurrent=False)
    assert [(r.sketch, r.idx, r.score) for r in conc] == [(r.sketch, r.idx, r.score) for r in seq]
    assert all(np.array_equal(a.sched, b.sched) for a, b in zip(conc, seq))
    per = []
    for sp in drv.spaces:
        y = torch.empty((sp.n_vars, n), device="cuda")
        sp.search(cm, y, T, rng_seed=77, init_from_y=False)
        per.append(sp.round_topk(cm, y, 16))
    ref = fo.subgraph_topk(per, 16)
    assert [(r.sketch, r.idx, r.score) for r in conc] == [(a, b, c) for a, b, c, _ in ref]


def test_search_quality_curves(fx):
    """Fig. 8-style diagnostic (tools/search_quality.py): on C1 the history best / 64th-best are
    non-decreasing in the schedules searched, and the s-step history top-k equals the oracle's on
    the GPU trajectory for a short prefix."""
    import importlib.util, os
    spec = importlib.util.spec_from_file_location("sq", os.path.join(os.path.dirname(__file__), "..", "tools", "search_quality.py"))
    sq = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(sq)
    cfg = fi.config("C1")
    sp = cfg.spaces[0]
    mlp = fi.make_mlp(cfg.mlp_dims)
    space, cm = fx.Space(sp), fx.CostModel.from_weights(mlp)
    res = sq.curves(space, cm, cfg.n_seeds, [1, 2, 5, 10, 20], cfg.rng_seed, cfg.lr, cfg.lam, kq=16)
    best = [r["best"] for r in res]
    q = [r["top16"] for r in res]
    assert all(b1 >= b0 for b0, b1 in zip(best, best[1:]))
    assert all(b1 >= b0 for b0, b1 in zip(q, q[1:]))
    y0 = space.init_sample(cfg.n_seeds, cfg.rng_seed).cpu().numpy()
    ys = _gpu_trajectory(space, cm, y0, 5, lr=cfg.lr, lam=cfg.lam)
    ref = fo.round_topk_history(sp, mlp.W, mlp.b, ys, 16)
    assert abs(res[2]["best"] - ref[2][0]) <= 1e-12 * abs(ref[2][0])            # FP64 scores: rel <= 1e-12
    assert abs(res[2]["top16"] - ref[2][15]) <= 1e-12 * abs(ref[2][15])


@pytest.mark.parametrize("mode", ["seeds", "task"])
@pytest.mark.timeout(600)
def test_multitask_shards_equal_single_rank_and_oracle(fx, mode):
    """C3/C4-style multi-task workloads (tasks.py): the shards a 2-rank plan gives each
    rank, run on this GPU one rank at a time with one stream per task and merged as the all-gather
    merges them, equal the 1-rank run per task; that run's top-k equals the oracle's round/top-k of the
    GPU's final y of every task."""
    from paper_conf_asplos_zhaosam24_b200 import tasks
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    r50 = fi.resnet50_spaces()
    spaces = [r50[0], r50[6], r50[-1], fi.bert_spaces()[1]]
    n, T, k = 400, 4, 16
    costs = [tasks.est_cost(n, T, cm.mlp_flops_per_candidate_step(), sp.nodes.shape[0]) for sp in spaces]
    nv = [sp.n_vars for sp in spaces]
    one = tasks.TaskRunner(spaces, tasks.plan(len(spaces), n, 1, mode, costs)[0], cm)
    res1 = one.run(T, k, rng_seed=91)
    rows = []
    for r in range(2):
        run = tasks.TaskRunner(spaces, tasks.plan(len(spaces), n, 2, mode, costs)[r], cm)
        rows.append(tasks.pack_task_records(run.run(T, k, rng_seed=91), len(spaces), k, max(nv)))
    merged = tasks.merge_task_records(np.concatenate(rows), len(spaces), k, nv)
    for t in range(len(spaces)):
        a, b = merged[t], res1[t]
        assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1]) and np.array_equal(a[2], b[2])
        yt = one._y[t].cpu().numpy()
        _topk_equal(*b, *fo.round_topk(spaces[t], mlp.W, mlp.b, yt, k))


ALL_TASKS = [("r50", i) for i in range(len(fi.resnet50_spaces()))] + [("bert", i) for i in range(len(fi.bert_spaces()))]


@pytest.mark.parametrize("fam,i", ALL_TASKS)
@pytest.mark.timeout(300)
def test_every_c3_c4_task_eval_and_rounding_parity(fx, fam, i):
    """Every ResNet-50 (C3) and BERT-base (C4) task: phi, cost, loss, gradient at y0 within the
    north-star tolerances, and rounding / validity / top-k bit-exact, vs the oracle (n = 300: three
    128-row tiles + a ragged tail)."""
    sp = (fi.resnet50_spaces() if fam == "r50" else fi.bert_spaces())[i]
    key = f"{fam}{i}"
    if key not in _cache:
        mlp = fi.make_mlp(fi.DEFAULT_MLP)
        _cache[key] = (sp, mlp, 300, fx.Space(sp), fx.CostModel.from_weights(mlp))
    sp, mlp, n, space, cm = _cache[key]
    y0 = fi.make_y0(sp, n, seed=50 + i)
    out = space.eval(cm, torch.from_numpy(y0).cuda(), lam=1.0)
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    phi = out["phi"].cpu().numpy()
    assert np.max(np.abs(phi - ref.phi) / np.maximum(np.abs(ref.phi), 1.0)) <= 1e-4
    rms_c = np.sqrt(np.mean(ref.c ** 2))
    assert np.max(np.abs(out["cost"].cpu().numpy() - ref.c)) <= 1e-4 * rms_c
    rms_l = np.sqrt(np.mean(ref.loss ** 2))
    assert np.max(np.abs(out["loss"].cpu().numpy() - ref.loss)) <= 1e-4 * rms_l
    e_g = np.abs(out["g"].cpu().numpy() - ref.g) / np.maximum(np.abs(ref.g), 1.0)
    assert np.max(e_g) <= 1e-4
    g = out["grad"].cpu().numpy()
    err = np.linalg.norm(g - ref.grad, axis=0) / np.maximum(np.linalg.norm(ref.grad, axis=0), 1e-12)
    bad = err > 1e-3
    km = kink_margin(ref.zs)
    assert not np.any(bad & (km >= 1e-4)) and (bad & (km < 1e-4)).mean() < 0.01
    sched, valid = space.round(torch.from_numpy(y0).cuda())
    rs = fo.round_schedules(sp, y0)
    assert np.array_equal(sched.cpu().numpy(), rs)
    assert np.array_equal(valid.cpu().numpy().astype(bool), fo.validate(sp, rs))
    _topk_equal(*space.round_topk(cm, torch.from_numpy(y0).cuda(), 16),
                *fo.round_topk(sp, mlp.W, mlp.b, y0, 16))


def _group_spaces():
    r50 = fi.resnet50_spaces()
    return [fi.c2_space(), r50[0], fi.bert_spaces()[1]], [700, 400, 513]


@pytest.mark.timeout(600)
@pytest.mark.parametrize("sc", [0, 1])
def test_search_group_equals_individual_searches(fx, sc):
    """felix_search_group (one MLP pass per Adam step over the candidates of several spaces) computes
    every member's search exactly as felix_search does: with the tile kernel, whose per-row arithmetic
    does not depend on the row's position, the final y and losses are bit-identical (both with the
    cone-group DAG kernels and with the split-cone ones)."""
    with fx.tuned(mlp="tile", split_cone=sc):
        _group_vs_individual(fx)


def _group_vs_individual(fx):
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    sps, ns = _group_spaces()
    spaces = [fx.Space(sp) for sp in sps]
    T = 6
    ind, ind_loss = [], []
    for i, (sp, n) in enumerate(zip(spaces, ns)):
        y = torch.empty((sp.n_vars, n), device="cuda")
        l = torch.empty(n, device="cuda")
        sp.search(cm, y, T, rng_seed=100 + i, init_from_y=False, index_base=7 * i, final_loss=l)
        ind.append(y)
        ind_loss.append(l)
    ys = [torch.empty((sp.n_vars, n), device="cuda") for sp, n in zip(spaces, ns)]
    ls = [torch.empty(n, device="cuda") for n in ns]
    fx.search_group(spaces, cm, ys, T, rng_seeds=[100, 101, 102], index_bases=[0, 7, 14], init_from_y=False,
                    final_losses=ls)
    for a, b, la, lb in zip(ys, ind, ls, ind_loss):
        assert torch.equal(a, b) and torch.equal(la, lb)
    # the workspace is reused on a second call with the same members
    ys2 = [torch.empty_like(y) for y in ys]
    fx.search_group(spaces, cm, ys2, T, rng_seeds=[100, 101, 102], index_bases=[0, 7, 14], init_from_y=False)
    assert all(torch.equal(a, b) for a, b in zip(ys, ys2))


@pytest.mark.timeout(600)
def test_search_group_one_step_vs_oracle(fx):
    """One group Adam step (default MLP kernel for the group's total rows) against the oracle's one
    step per member, north-star tolerances; loss per member vs the oracle objective."""
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    sps, ns = _group_spaces()
    spaces = [fx.Space(sp) for sp in sps]
    y0s = [fi.make_y0(sp, n, seed=60 + i) for i, (sp, n) in enumerate(zip(sps, ns))]
    ys = [torch.from_numpy(y).cuda() for y in y0s]
    ls = [torch.empty(n, device="cuda") for n in ns]
    fx.search_group(spaces, cm, ys, 1, init_from_y=True, final_losses=ls)
    for sp, y0, y, l in zip(sps, y0s, ys, ls):
        ob = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
        ry, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 1, lr=0.05, lam=1.0)
        got = y.cpu().numpy()
        exempt = (np.abs(ob.grad) < 1e-6) | (kink_margin(ob.zs) < 1e-4)[None, :]
        assert not np.any((np.abs(got - ry) > 1e-4 * (1 + np.abs(ry))) & ~exempt)
        assert np.max(np.abs(l.cpu().numpy() - ob.loss)) / np.sqrt(np.mean(ob.loss ** 2)) <= 1e-4


def test_search_group_errors(fx):
    mlp = fi.make_mlp(fi.DEFAULT_MLP)
    cm = fx.CostModel.from_weights(mlp)
    sp = fx.Space(fi.c2_space())
    y = torch.zeros((sp.n_vars, 64), device="cuda")
    with pytest.raises(fx.FelixError):
        fx.search_group([sp, sp], cm, [y, y.clone()], 2)          # a space twice


@pytest.mark.parametrize("name,n,steps,P,W,chunks", [
    ("C2", 4096, 8, 4, -1, 1), ("C2", 1000, 5, 8, 3, 1), ("C2_2stmt", 700, 6, 4, 2, 1),
    ("bmm", 257, 5, 2, 1, 1), ("C2", 3000, 6, 4, -1, 2), ("C5", 389, 9, 1, -1, 1), ("r50_conv1", 300, 4, 4, 1, 1)])
def test_split_cone_kernels_match_cone_groups(fx, name, n, steps, P, W, chunks):
    """Split-cone reverse kernel (one cone per CTA, FP32 partial adjoints through global memory; the next
    step's forward sums them and applies Adam in place, felix_adam_sc after the last step) against the
    cone-group kernels over several Adam steps (ragged n, several chunks, P = 1..8): both run the same
    FP32 reverse arithmetic, so y and the final loss agree to fp32 rounding; the one-step result is also
    checked against the oracle."""
    make, dims, _ = CASES[name]
    sp = make()
    mlp = fi.make_mlp(dims)
    cm = fx.CostModel.from_weights(mlp)
    y0 = fi.make_y0(sp, n, seed=77)
    out = {}
    for sc in (0, 1):
        with fx.tuned(cone_width=P, chunks=chunks, sc_warps=W, split_cone=sc):
            space = fx.Space(sp)
            y = torch.from_numpy(y0).cuda()
            loss = torch.empty(n, device="cuda")
            space.search(cm, y, steps, init_from_y=True, final_loss=loss)
            y1 = torch.from_numpy(y0).cuda()
            space.search(cm, y1, 1, init_from_y=True)
            out[sc] = (y.cpu().numpy(), loss.cpu().numpy(), y1.cpu().numpy())
    (ya, la, y1a), (yb, lb, y1b) = out[0], out[1]
    assert np.all(np.isfinite(yb)) and np.all(np.isfinite(lb))
    same = np.mean(ya == yb)
    print(f"{name} n={n} steps={steps} P={P}: exactly equal y {same:.4f}, max |dy| {np.max(np.abs(ya - yb)):.3e}")
    assert np.max(np.abs(y1a - y1b)) <= 1e-5 * (1 + np.max(np.abs(y1a)))
    assert np.mean(np.abs(ya - yb) <= 1e-4 * (1 + np.abs(ya))) >= 0.99
    s = np.sqrt(np.mean(la.astype(np.float64) ** 2))
    assert np.mean(np.abs(la - lb) <= 1e-4 * s) >= 0.99
    ry, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, 1, lr=0.05, lam=1.0)
    ob = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    exempt = (np.abs(ob.grad) < 1e-6) | (kink_margin(ob.zs) < 1e-4)[None, :]
    assert not np.any((np.abs(y1b - ry) > 1e-4 * (1 + np.abs(ry))) & ~exempt)


@pytest.mark.parametrize("name,n", [("C2", 4096), ("C1", 300), ("C2_2stmt", 700), ("r50_conv1", 129)])
def test_scoring_kernels_vs_oracle(fx, name, n):
    """FP64 scoring: the 128 x 64 register-blocked layer kernel and the row-staged head kernel (fixed k
    order per output) against the oracle's column-at-a-time FP64 MLP to 1e-12."""
    make, dims, _ = CASES[name]
    sp = make()
    mlp = fi.make_mlp(dims)
    cm = fx.CostModel.from_weights(mlp)
    space = fx.Space(sp)
    rs = fo.round_schedules(sp, fi.make_y0(sp, n, seed=15))
    new = space.score(cm, torch.from_numpy(rs).cuda()).cpu().numpy()
    ref = fo.score(sp, mlp.W, mlp.b, rs)
    ok = np.isfinite(ref)
    assert np.array_equal(np.isfinite(new), ok)
    assert np.all(np.abs(new[ok] - ref[ok]) <= 1e-12 * np.maximum(np.abs(ref[ok]), 1e-3))


@pytest.mark.parametrize("history", [False, True])
def test_multi_step_graphs_equal_single_step_graphs(fx, history):
    """felix_search captures graph_steps Adam steps per CUDA graph (default 20) plus a tail graph: 25 steps as
    20 + 5 give bit-for-bit the y, final loss and top-k of 25 one-step graph launches (the same kernels in
    the same order; only the launch grouping differs)."""
    sp, mlp, n, space, cm = _setup(fx, "C2")
    n = 1000
    y0 = torch.from_numpy(fi.make_y0(sp, n, seed=21)).cuda()
    out = []
    for gs in (-1, 1):
        with fx.tuned(graph_steps=gs):
            y = y0.clone()
            loss = torch.empty(n, dtype=torch.float32, device="cuda")
            space.search(cm, y, 25, init_from_y=True, final_loss=loss, history=history)
            if history:
                rec = space.history_topk(cm, 16)
            else:
                rec = space.round_topk(cm, y, 16)
            torch.cuda.synchronize()
            out.append((y.cpu().numpy(), loss.cpu().numpy(), rec))
    (ya, la, ra), (yb, lb, rb) = out
    assert np.array_equal(ya, yb) and np.array_equal(la, lb, equal_nan=True)
    for a, b in zip(ra, rb):
        assert np.array_equal(np.asarray(a), np.asarray(b))


@pytest.mark.parametrize("n,ksplit", [(5120, -1), (4096, 2), (4096, 1)])
def test_chain_dphi_layer_variants_search_path_gradient(fx, n, ksplit):
    """The chain's dL/dphi layer in its other shapes -- 32-wide N tiles without split-K (n = 5120: 40 row
    blocks), split-K 2 and no split at 4096 -- all written by the staged TMA store: the search path's dL/dy
    against the oracle (normwise 1e-3 per candidate, R-kink exemption < 1 %)."""
    sp, mlp, _, space, cm = _setup(fx, "C2")
    y0 = fi.make_y0(sp, n, seed=5)
    with fx.tuned(mlp="chain", dphi_ksplit=ksplit):
        out = space.eval_search_path(cm, torch.from_numpy(y0).cuda())
        torch.cuda.synchronize()
    ref = fo.objective(sp, mlp.W, mlp.b, y0.astype(np.float64), 1.0)
    g = out["grad"].cpu().numpy()
    err = np.linalg.norm(g - ref.grad, axis=0) / np.maximum(np.linalg.norm(ref.grad, axis=0), 1e-12)
    assert np.mean(err > 1e-3) < 0.01
