#!/usr/bin/env python
"""Benchmark of the Felix hot path on B200 (BASELINE.json metric: candidate gradient-steps/s).

One bench "step" = one complete Algorithm-1 search of the workload (PAPER.md L899-924 lines 12-21):
the rejection-sampled init (a0), n_steps Adam steps of the fused objective/gradient (a1-a8), then
rounding, validity, FP64 scoring and top-k (a9-a12).  At N=1 the workload is BASELINE configs[1]
(C2: ResNet-50 conv2d 3x3 56x56x64, 12 vars, 4096 seeds x 200 steps, TenSet MLP [82,512,256,256,1]).
value = seeds x steps x ranks / max-over-ranks device time of the timed steps (weak scaling: every
rank searches its own 4096 seeds, index_base = rank * 4096; the only exchange is the final top-k
all-gather over NCCL).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl {felix,reference}] [--config C2]

`--config C3` (ResNet-50: 21 tasks x 8192 seeds, subgraphs sharded by LPT) and `--config C4` (BERT-base:
6 tasks x 16384 seeds x 500 steps, every task's seeds sharded) run the multi-task workloads
(paper_conf_asplos_zhaosam24_b200/tasks.py): strong scaling, one CUDA stream per task.

`--impl reference` times the float64 oracle (oracle/, numpy) on the host cores for the same
workload on a bounded sample per step (this tier's reference arm: there is no reference code).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "candidate gradient-steps/sec (whole box)"
UNIT = "cand-steps/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="felix", choices=["felix", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="target CPU time of the oracle sample")
    ap.add_argument("--ref-seconds", type=float, default=90.0, help="target wall time of the whole --impl reference run")
    ap.add_argument("--seeds", type=int, default=0, help="override seeds per GPU (experiments; not the headline)")
    ap.add_argument("--search-steps", type=int, default=0, help="override Adam steps per search (experiments)")
    ap.add_argument("--two-statements", action="store_true",
                    help="C2 with TenSet-style per-statement features [reduction | epilogue], C = sum_s MLP "
                         "(SURVEY 8(f) row 3; not the headline)")
    ap.add_argument("--unbatched", action="store_true",
                    help="C3/C4: one felix_search per task on its own stream instead of felix_search_group")
    ap.add_argument("--tune", action="append", default=[],
                    help="experiments: felix_tune knob key=value (repeatable; the headline uses the defaults)")
    ap.add_argument("--history", action="store_true",
                    help="paper-faithful Alg. 1: round every visited point (varValuesHistory, l.13/17/20) "
                         "instead of the final point only (SURVEY 8(f) row 1; not the headline)")
    return ap.parse_args()


# ------------------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 50 ms during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except FileNotFoundError:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                self.rows.append(parts)

    def stop(self):
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        if self.thread is not None:
            self.thread.join(timeout=2)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4) if r[5 + i].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------------------------- helpers
def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        with open(path) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback (B200_PROFILING.md)"


def apply_tune(fx, args):
    for kv in args.tune:
        k, v = kv.split("=")
        fx.tune(**{k: (v if k == "mlp" and not v.lstrip("-").isdigit() else int(v))})


def sp_info_flops(space):
    """(forward, reverse-sweep) FP64 ops per candidate of a space's DAG (felix_space_info)."""
    return int(space.info.dag_flops_fwd), int(space.info.dag_flops_rev)


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def oracle_baseline(cfg, seconds: float, history: bool = False):
    """The float64 oracle as it stands, timed on this host's cores on a bounded sample of the same
    workload: the first min(n_seeds, 4096) seeds of the same space/model/starting points, as many Adam
    steps as fit in ~`seconds`, then its rounding + top-k.  Returns (cand-steps/s, threads, sample)."""
    from oracle import felix_oracle as fo
    import felix_inputs as fi
    try:
        import threadpoolctl
        threads = max(i.get("num_threads", 1) for i in threadpoolctl.threadpool_info()) or os.cpu_count()
    except Exception:
        threads = os.cpu_count()
    sp = cfg.spaces[0]
    mlp = fi.make_mlp(cfg.mlp_dims)
    n = min(cfg.n_seeds, 4096)
    y0 = fo.init_sample(sp, n, cfg.rng_seed)
    # probe one step to size the sample
    t0 = time.perf_counter()
    fo.search(sp, mlp.W, mlp.b, y0, 1, cfg.lr, cfg.lam)
    one = time.perf_counter() - t0
    steps = int(max(2, min(cfg.n_steps, seconds / max(one, 1e-6))))
    if history:
        steps = max(2, steps // 3)
    t0 = time.perf_counter()
    y, _, _, hist = fo.search(sp, mlp.W, mlp.b, y0, steps, cfg.lr, cfg.lam, history=history)
    t_search = time.perf_counter() - t0
    t0 = time.perf_counter()
    if history:
        fo.round_topk_history(sp, mlp.W, mlp.b, [h[0].astype(np.float32) for h in hist], cfg.topk)
    else:
        fo.round_topk(sp, mlp.W, mlp.b, y.astype(np.float32), cfg.topk)
    t_fin = time.perf_counter() - t0
    # whole-job rate: the full search is n_steps steps + one finish; scale the measured parts (the history
    # finish grows with the steps recorded, so it is scaled with them)
    per_step = t_search / steps
    t_job = per_step * cfg.n_steps + (t_fin * cfg.n_steps / steps if history else t_fin)
    rate = n * cfg.n_steps / t_job
    what = "history round/validate/score/top-k of every visited point" if history else "round/top-k"
    sample = (f"{n} seeds x {steps} Adam steps of {sp.name} (of {cfg.n_steps}) + {what}, "
              f"extrapolated linearly to {cfg.n_steps} steps; numpy float64")
    return rate, threads, sample, t_search + t_fin


def workload_config(cfg, sp, n, T, k, world, hist=False):
    """The `config` object of the bench line — identical for the felix arm and the reference arm."""
    return {"workload": f"{cfg.name}: {sp.name}, {sp.n_vars} vars, {n} seeds x {T} steps per GPU, "
                        f"MLP {list(cfg.mlp_dims)}, top-{k}" + (f", {sp.n_statements} statements (segment sum)"
                                                               if sp.n_statements > 1 else "")
                        + (", history rounding (Alg. 1 l.20 over all visited points)" if hist else ""),
            "n_seeds_per_gpu": n, "n_steps": T, "topk": k, "parallelism": f"dp{world} (seed shards)",
            "l2": "flushed (256 MB write) between timed iterations"}


def felix_workload(args):
    """(cfg, space, n seeds per GPU, n_steps) of the felix arm for these arguments (shared by both arms)."""
    import felix_inputs as fi
    cfg = fi.config(args.config)
    if args.seeds:
        cfg.n_seeds = args.seeds
    elif args.config == "C5":
        cfg.n_seeds = (1 << 20) // 8          # C5 is 2^20 candidates over 8 GPUs: one GPU's shard
    if args.search_steps:
        cfg.n_steps = args.search_steps
    if args.two_statements:
        assert args.config == "C2", "--two-statements is defined for C2"
        cfg.spaces = [fi.c2_space_two_statements()]
    return cfg, cfg.spaces[0], cfg.n_seeds, cfg.n_steps


# ------------------------------------------------------------------------------------- reference arm
def oracle_sample(cfg, sp, mlp, y0, steps, history):
    """One bounded sample of the workload on the oracle: `steps` Adam steps of the given seeds, then the
    finish (round / validate / score / top-k).  Returns (t_search, t_finish) in seconds."""
    from oracle import felix_oracle as fo
    t0 = time.perf_counter()
    y, _, _, hist = fo.search(sp, mlp.W, mlp.b, y0, steps, cfg.lr, cfg.lam, history=history)
    t1 = time.perf_counter()
    if history:
        fo.round_topk_history(sp, mlp.W, mlp.b, [h[0].astype(np.float32) for h in hist], cfg.topk)
    else:
        fo.round_topk(sp, mlp.W, mlp.b, y.astype(np.float32), cfg.topk)
    return t1 - t0, time.perf_counter() - t1


def run_reference(args):
    """The reference arm (this tier: the float64 oracle, as it stands, on the host cores).  Each bench
    step is ONE bounded sample of the felix arm's workload — the first m seeds of the same space, model
    and starting points, s Adam steps, then round / top-k of those m — timed on the wall clock; value is
    the whole-job rate that sample measures (per candidate-step of the search, per candidate of the
    finish), ms_per_step the wall time a step actually took."""
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    import felix_inputs as fi
    from oracle import felix_oracle as fo
    cfg, sp, n, T = felix_workload(args)
    mlp = fi.make_mlp(cfg.mlp_dims)
    k = cfg.topk
    try:
        import threadpoolctl
        threads = max(i.get("num_threads", 1) for i in threadpoolctl.threadpool_info()) or os.cpu_count()
    except Exception:
        threads = os.cpu_count()
    W = max(args.warmup, 0)
    K = max(args.steps, 1)
    m = min(n, 1024)
    y0 = fo.init_sample(sp, m, cfg.rng_seed)
    # size s so that the whole run (W + K samples) takes about args.ref_seconds
    t0 = time.perf_counter()
    oracle_sample(cfg, sp, mlp, y0, 1, args.history)
    probe = time.perf_counter() - t0
    per_sample = max(0.5, args.ref_seconds / (W + K))
    s_steps = int(max(1, min(T, per_sample / max(probe, 1e-6))))
    rates, walls = [], []
    for it in range(W + K):
        t0 = time.perf_counter()
        ts, tf = oracle_sample(cfg, sp, mlp, y0, s_steps, args.history)
        wall = time.perf_counter() - t0
        if it >= W:
            per_cs = ts / (m * s_steps)                      # s per candidate-step of the search
            per_fin = tf / m if not args.history else tf / (m * s_steps) * T
            rates.append(n * T / (per_cs * n * T + per_fin * n))
            walls.append(wall)
    value = statistics.median(rates)
    sample = (f"per step: {m} of the {n} seeds x {s_steps} of {T} Adam steps of {sp.name} + round/top-k of those {m}, "
              f"numpy float64; value = whole-job rate from the per-candidate-step search time and per-candidate finish time")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": W, "ms_per_step": statistics.mean(walls) * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(cfg, sp, n, T, k, world, args.history),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------------------------- felix arm
def run_felix(args):
    import torch
    rank, world, local = dist_env()
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.cuda.current_device()
    import felix_inputs as fi
    import paper_conf_asplos_zhaosam24_b200 as fx
    from paper_conf_asplos_zhaosam24_b200 import dist as fdist
    apply_tune(fx, args)

    cfg, sp, _, _ = felix_workload(args)
    mlp = fi.make_mlp(cfg.mlp_dims)
    space = fx.Space(sp, device=dev)
    cm = fx.CostModel.from_weights(mlp, device=dev)
    n, T, k = cfg.n_seeds, cfg.n_steps, cfg.topk
    base = rank * n
    stream = torch.cuda.current_stream()
    y = torch.empty((sp.n_vars, n), dtype=torch.float32, device=dev)
    loss = torch.empty(n, dtype=torch.float32, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # > 126 MB L2

    hist = args.history

    def finish(yv):
        if not hist:
            return space.round_topk(cm, yv, k, index_base=base, stream=stream)
        idx, step, sc, sched, _ = space.history_topk(cm, k, stream=stream)
        # merge key for the multi-GPU top-k: (step, global index) packed so that its order is the
        # history order (score desc, step asc, global index asc)
        return (step.astype(np.int64) << 40) | idx, sc, sched

    def bench_step():
        # Algorithm 1: init (device sampler) -> T Adam steps -> round / validate / score / top-k
        space.search(cm, y, T, lr=cfg.lr, lam=cfg.lam, rng_seed=cfg.rng_seed, init_from_y=False,
                     index_base=base, final_loss=loss, history=hist, stream=stream)
        return finish(y)

    def barrier():
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        bench_step()
    barrier()

    K = args.steps
    clocks = ClockSampler(dev if "CUDA_VISIBLE_DEVICES" not in os.environ else
                          int(os.environ["CUDA_VISIBLE_DEVICES"].split(",")[dev]))
    clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    barrier()
    last = None
    for i in range(K):
        flush.zero_()                                    # L2 flush between timed iterations (untimed)
        ev[i][0].record(stream)
        last = bench_step()
        ev[i][1].record(stream)
    barrier()
    clocks.stop()
    t_ms = sum(a.elapsed_time(b) for a, b in ev)
    # max over ranks
    t_max = t_ms
    if world > 1:
        tt = torch.tensor([t_ms], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        t_max = float(tt.item())
    value = world * n * T * K / (t_max * 1e-3)

    # global top-k (the only exchange): NCCL all-gather of the local top-k records
    if world > 1:
        gidx, gsc, gsched = fdist.allgather_topk(*last, k, sp.n_vars, device=dev)
    else:
        gidx, gsc, gsched = last

    # ---- search-only timing and per-kernel-class device time (second timed pass, profiling events)
    space.profile_reset()
    space.profile(True)
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(K):
        space.search(cm, y, T, lr=cfg.lr, lam=cfg.lam, rng_seed=cfg.rng_seed, init_from_y=False, index_base=base,
                     final_loss=loss, history=hist, stream=stream)
    e1.record(stream)
    barrier()
    space.profile(False)
    prof = space.profile_read()
    prof_total_ms = e0.elapsed_time(e1)
    # finish (round/top-k) alone
    f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    f0.record(stream)
    finish(y)
    f1.record(stream)
    barrier()
    finish_ms = f0.elapsed_time(f1)

    # ---- roofline of the dominant kernel: the tcgen05 MLP (tensor-bound contraction).  Which MLP kernel
    # runs follows felix_api.cu mlp_mode(): the tile-local fused kernel from one full wave of 128-row
    # tiles (TenSet widths), the persistent layer chain below that.
    peaks, peak_src = measured_peaks()
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    tile_fits = tuple(cfg.mlp_dims[1:]) == (512, 256, 256, 1)
    n_rows = n * sp.n_statements
    mlp_kernel = "mlp_tile_kernel" if tile_fits and -(-n_rows // 128) >= sms else "mlp_chain_kernel"
    traffic = None
    tname = {"mlp_chain_kernel": "roofline_traffic.json", "mlp_tile_kernel": "roofline_traffic_tile.json"}.get(mlp_kernel, "")
    tpath = os.path.join(ROOT, "profiles", "r02", tname) if tname else ""
    if tname and os.path.exists(tpath):
        with open(tpath) as f:
            tj = json.load(f)
        traffic = tj["dram_bytes_read_per_launch"] + tj["dram_bytes_write_per_launch"]
    gemm_ms, gemm_launches = prof["mlp_gemm"]
    mlp_flops_step = cm.mlp_flops_per_candidate_step() * n * sp.n_statements   # algorithmic (1-pass) FLOPs / Adam step
    gemm_per_step_ms = gemm_ms / (K * T)         # one chain launch (or 2(L-1) layer launches) per Adam step
    achieved_tflops = mlp_flops_step / (gemm_per_step_ms * 1e-3) / 1e12
    clk = clocks.summary()
    capped = "sw_power_cap" in clk.get("reasons", [])
    # the MLP kernel is timed inside a ~12 ms search at the clocks above: the burst peak applies unless
    # the power cap engaged (then the sustained one); both fractions are reported
    peak_burst = float(peaks.get("bf16_tflops", 1590.0))
    peak_sust = float(peaks.get("bf16_tflops_sustained", peak_burst))
    peak = peak_sust if capped else peak_burst
    dag_fwd_ms, _ = prof["dag_fwd"]
    dag_rev_ms, _ = prof["dag_rev_adam"]
    # expression kernels (FP64 straight-line DAG code): algorithmic FP64 ops and HBM bytes per
    # candidate-step, against the FP64 ALU peak derived from unit counts (148 SMs x 64
    # FP64 FMA/clk x 2 x max SM clock) and the measured HBM bandwidth
    M, K0p = sp.n_vars, 96 if cfg.mlp_dims[0] <= 96 else 128
    P = 4 if n <= 8192 else 2
    ns = sp.n_statements
    sm_max = float(clk.get("sm_max_mhz") or peaks.get("sm_max_mhz", 1965.0))
    fp64_peak = sms * 64 * 2 * sm_max * 1e6 / 1e12
    hbm_peak = float(peaks.get("hbm_gbs", 6550.0))
    nht = 4   # head partials read by the Adam prologue (chain: two column halves of the 256-wide head layer x 2)
    fwd_bytes = 24 * M + 8 * P * M + 8 * P + 4 * nht + ns * 2 * 2 * K0p
    rev_bytes = 4 * M + 4 * ns * cfg.mlp_dims[0] + 8 * P * M + 8 * P
    fwd_ops = sp_info_flops(space)[0] + 15 * M
    rev_ops = sum(sp_info_flops(space))             # forward recompute + reverse sweep

    def kroof(ms_total, ops, nbytes):
        per_step_s = ms_total / (K * T) * 1e-3
        f = ops * n / per_step_s / 1e12
        b = nbytes * n / per_step_s / 1e9
        return {"us_per_adam_step": per_step_s * 1e6, "fp64_tflops": f, "fp64_peak_tflops": fp64_peak,
                "fp64_frac": f / fp64_peak, "hbm_gbs": b, "hbm_peak_gbs": hbm_peak, "hbm_frac": b / hbm_peak,
                "ops_per_candidate_step": ops, "bytes_per_candidate_step": nbytes,
                "bound": "latency (neither FP64 nor HBM: both fractions are small; DESIGN.md §6)"}

    # ---- end to end through the public API with host buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        import felix_inputs as fi2
        y0_host = torch.from_numpy(fi2.make_y0(sp, n, seed=1234 + rank)).pin_memory()
        loss_host = torch.empty(n, dtype=torch.float32).pin_memory()
        y_dev = torch.empty_like(y)

        def e2e_step():
            # the same work as a timed device step (L2 flush, search, finish) through the public API, with
            # the step's starting points coming from pinned host memory (H2D) instead of the device
            # rejection sampler, and the losses + top-k records read back (D2H)
            flush.zero_()
            y_dev.copy_(y0_host, non_blocking=True)                          # H2D: starting points
            space.search(cm, y_dev, T, lr=cfg.lr, lam=cfg.lam, init_from_y=True, index_base=base,
                         final_loss=loss, history=hist, stream=stream)
            loss_host.copy_(loss, non_blocking=True)                         # D2H: final losses
            return finish(y_dev)                                             # D2H: top-k records (synchronises)
        for _ in range(2):
            e2e_step()
        barrier()
        t0 = time.perf_counter()
        for _ in range(K):
            e2e_step()
        barrier()
        t_e2e = time.perf_counter() - t0
        if world > 1:
            tt = torch.tensor([t_e2e], device=dev, dtype=torch.float64)
            torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
            t_e2e = float(tt.item())
        h2d = sp.n_vars * n * 4
        d2h = n * 4 + k * (8 + 8 + 4 * sp.n_vars) + 4
        e2e = {"value": world * n * T * K / t_e2e, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "timing": "host wall clock over K steps (max over ranks); each step: L2 flush, pinned H2D of the "
                         "starting points, felix_search, felix_round_topk, D2H of losses + top-k",
               "work_vs_value": "value's work with a0 (device rejection sampler, ~0.5 % of a step) replaced by the "
                                "H2D of host starting points, and the L2 flush inside the timed region"}

    if rank != 0:
        if world > 1:
            torch.distributed.destroy_process_group()
        return 0

    cpu = None
    if not args.no_cpu_baseline and world == 1:
        rate, threads, sample, _ = oracle_baseline(cfg, args.cpu_seconds, hist)
        cpu = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample}

    n_gemm = len(cfg.mlp_dims) * 2 - 4          # (L-1) forward + (L-1) backward GEMM layers
    kernels = {"felix_fwd_adam": kroof(dag_fwd_ms, fwd_ops, fwd_bytes),
               "felix_rev_sc": kroof(dag_rev_ms, rev_ops, rev_bytes)}
    mlp_launches = 1
    # init + steps + finish; the reverse class counts the split-cone kernels' final Adam launch too
    rev_launches = int(round(prof["dag_rev_adam"][1] / K))
    init_launches = max(1, int(round(prof["init"][1] / K)))   # sampler (+ the split-cone counter reset)
    launches_per_step = init_launches + T * (1 + mlp_launches) + rev_launches + (6 + len(cfg.mlp_dims) - 1)
    ms_per_step = t_max / K
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "fp16 hi/lo split (fp32-accurate) MLP, f64 DAG forward, f32 DAG reverse, f32 Adam, f64 scoring", "data": "synthetic",
        "config": workload_config(cfg, sp, n, T, k, world, hist),
        "roofline": {"bound": "tensor", "achieved": achieved_tflops, "peak": peak, "unit": "TFLOP/s",
                     "frac": achieved_tflops / peak, "traffic": traffic,
                     "kernel": f"{mlp_kernel} (all {n_gemm} MLP layers of one Adam step, tcgen05 kind::f16, 3-pass hi/lo split)",
                     "traffic_source": (f"profiles/r02/{tname} (ncu --set full, DRAM bytes per launch)"
                                        if traffic is not None else None),
                     "algorithmic_flops_per_adam_step": mlp_flops_step,
                     "executed_tflops": 3 * achieved_tflops,
                     "peak_source": (f"{peak_src} bf16_tflops (burst; fp16 = bf16 rate)" if not capped else
                                     f"{peak_src} bf16_tflops_sustained (sw_power_cap seen; fp16 = bf16 rate)"),
                     "frac_vs_burst": achieved_tflops / peak_burst, "frac_vs_sustained": achieved_tflops / peak_sust},
        "kernel_rooflines": kernels,
        "breakdown_ms_per_adam_step": {"dag_fwd": dag_fwd_ms / (K * T), "mlp_gemms": gemm_per_step_ms,
                                       "dag_rev_adam": dag_rev_ms / (K * T),
                                       "search_total": prof_total_ms / (K * T)},
        "finish_ms": finish_ms,
        "gpu_launches": launches_per_step * K,
        "clocks": clk,
        "top1": ({"global_idx": int(gidx[0]) & ((1 << 40) - 1), "step": int(gidx[0]) >> 40, "score": float(gsc[0])}
                 if hist and len(gidx) else
                 {"global_idx": int(gidx[0]) if len(gidx) else None, "score": float(gsc[0]) if len(gsc) else None}),
    }
    if e2e is not None:
        line["e2e"] = e2e
    if cpu is not None:
        line["cpu_baseline"] = cpu
    if args.tune:
        line["tune"] = args.tune
    print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()
    return 0


# ------------------------------------------------------------------------------------- multi-task configs
def _tasks_module():
    from paper_conf_asplos_zhaosam24_b200 import tasks
    return tasks


def oracle_baseline_tasks(cfg, seconds: float):
    """The oracle on a bounded sample of a multi-task workload: the first m seeds of EVERY task (same
    device-independent starting points), as many Adam steps as fit in ~`seconds` overall, then its
    round/top-k; extrapolated linearly per task to n_seeds x n_steps + the finish at n_seeds."""
    from oracle import felix_oracle as fo
    import felix_inputs as fi
    try:
        import threadpoolctl
        threads = max(i.get("num_threads", 1) for i in threadpoolctl.threadpool_info()) or os.cpu_count()
    except Exception:
        threads = os.cpu_count()
    mlp = fi.make_mlp(cfg.mlp_dims)
    m = min(cfg.n_seeds, 1024)
    y0s = [fo.init_sample(sp, m, cfg.rng_seed + t) for t, sp in enumerate(cfg.spaces)]
    t0 = time.perf_counter()
    for sp, y0 in zip(cfg.spaces, y0s):
        fo.search(sp, mlp.W, mlp.b, y0, 1, cfg.lr, cfg.lam)
    one = time.perf_counter() - t0
    steps = int(max(2, min(cfg.n_steps, seconds / max(one, 1e-6))))
    t_job = 0.0
    t_meas = 0.0
    for sp, y0 in zip(cfg.spaces, y0s):
        t0 = time.perf_counter()
        y, _, _, _ = fo.search(sp, mlp.W, mlp.b, y0, steps, cfg.lr, cfg.lam)
        t1 = time.perf_counter()
        fo.round_topk(sp, mlp.W, mlp.b, y.astype(np.float32), cfg.topk)
        t2 = time.perf_counter()
        t_meas += t2 - t0
        t_job += (t1 - t0) * (cfg.n_seeds * cfg.n_steps) / (m * steps) + (t2 - t1) * cfg.n_seeds / m
    rate = len(cfg.spaces) * cfg.n_seeds * cfg.n_steps / t_job
    sample = (f"{m} seeds x {steps} Adam steps of each of the {len(cfg.spaces)} tasks (of {cfg.n_seeds} x "
              f"{cfg.n_steps}) + round/top-k, extrapolated linearly per task; numpy float64")
    return rate, threads, sample, t_meas


def run_felix_tasks(args):
    """C3 (ResNet-50, 21 tasks sharded by subgraph with LPT) / C4 (BERT-base, every task's seeds
    sharded): every rank runs its shards concurrently (one stream per task); one bench step = every
    task's full search + round/top-k; the per-task top-k lists are all-gathered once at the end."""
    import torch
    rank, world, local = dist_env()
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.cuda.current_device()
    import felix_inputs as fi
    import paper_conf_asplos_zhaosam24_b200 as fx
    apply_tune(fx, args)
    tasks = _tasks_module()

    cfg = fi.config(args.config)
    if args.seeds:
        cfg.n_seeds = args.seeds
    if args.search_steps:
        cfg.n_steps = args.search_steps
    mlp = fi.make_mlp(cfg.mlp_dims)
    cm = fx.CostModel.from_weights(mlp, device=dev)
    mode = tasks.config_mode(cfg.name)
    mlp_flops = cm.mlp_flops_per_candidate_step()
    costs = [tasks.est_cost(cfg.n_seeds, cfg.n_steps, mlp_flops, sp.nodes.shape[0]) for sp in cfg.spaces]
    shards = tasks.plan(len(cfg.spaces), cfg.n_seeds, world, mode, costs)[rank]
    runner = tasks.TaskRunner(cfg.spaces, shards, cm, device=dev)
    T, k = cfg.n_steps, cfg.topk
    stream = torch.cuda.current_stream()
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)

    batched = not args.unbatched

    def bench_step():
        return runner.run(T, k, rng_seed=cfg.rng_seed, lr=cfg.lr, lam=cfg.lam, batched=batched)

    def barrier():
        if world > 1:
            torch.distributed.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        bench_step()
    barrier()
    K = args.steps
    clocks = ClockSampler(dev if "CUDA_VISIBLE_DEVICES" not in os.environ else
                          int(os.environ["CUDA_VISIBLE_DEVICES"].split(",")[dev]))
    clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    barrier()
    last = None
    for i in range(K):
        flush.zero_()
        ev[i][0].record(stream)
        last = bench_step()
        ev[i][1].record(stream)
    barrier()
    clocks.stop()
    t_ms = sum(a.elapsed_time(b) for a, b in ev)
    t_max = t_ms
    if world > 1:
        tt = torch.tensor([t_ms], device=dev, dtype=torch.float64)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        t_max = float(tt.item())
    total = len(cfg.spaces) * cfg.n_seeds * T                 # candidate-steps of the whole job per bench step
    value = total * K / (t_max * 1e-3)
    local_cs = runner.cand_steps(T)
    n_vars = [sp.n_vars for sp in cfg.spaces]
    if world > 1:
        merged = tasks.allgather_task_topk(last, len(cfg.spaces), k, n_vars, device=dev)
    else:
        merged = tasks.merge_task_records(tasks.pack_task_records(last, len(cfg.spaces), k, max(n_vars)),
                                          len(cfg.spaces), k, n_vars)

    # ---- roofline of the MLP kernel: one profiled bench step (direct launches, CUDA events around every
    # MLP launch: batched = the one group MLP pass per Adam step over all tasks' rows; unbatched = the
    # shards searched one after another so the events time the kernels alone), algorithmic FLOPs / MLP time
    for sp in runner.spaces.values():
        sp.profile_reset()
        sp.profile(True)
    barrier()
    if batched:
        bench_step()
    else:
        runner.run(T, k, rng_seed=cfg.rng_seed, lr=cfg.lr, lam=cfg.lam, batched=False, concurrent=False)
    barrier()
    gemm_ms = 0.0
    dag_ms = 0.0
    for sp in runner.spaces.values():
        sp.profile(False)
        pr = sp.profile_read()
        gemm_ms += pr["mlp_gemm"][0]
        dag_ms += pr["dag_fwd"][0] + pr["dag_rev_adam"][0]
    mlp_flops_all = sum(mlp_flops * s.n * runner.spaces[s.task].n_statements * T for s in shards)
    achieved = mlp_flops_all / (gemm_ms * 1e-3) / 1e12
    peaks, peak_src = measured_peaks()
    peak = float(peaks.get("bf16_tflops_sustained", peaks.get("bf16_tflops")))

    # ---- end to end through the public API: pinned host starting points in, losses + top-k out
    e2e = None
    if not args.no_e2e:
        y_host = {s.task: torch.from_numpy(fi.make_y0(cfg.spaces[s.task], s.n, seed=1234 + s.task)).pin_memory()
                  for s in shards}
        y_dev = {s.task: torch.empty(tuple(y_host[s.task].shape), dtype=torch.float32, device=dev) for s in shards}
        l_dev = {s.task: torch.empty(s.n, dtype=torch.float32, device=dev) for s in shards}
        l_host = {s.task: torch.empty(s.n, dtype=torch.float32).pin_memory() for s in shards}

        def e2e_step():
            for s in shards:
                y_dev[s.task].copy_(y_host[s.task], non_blocking=True)
            out = runner.run(T, k, rng_seed=cfg.rng_seed, lr=cfg.lr, lam=cfg.lam, y0=y_dev, loss_out=l_dev, batched=batched)
            for s in shards:
                l_host[s.task].copy_(l_dev[s.task], non_blocking=True)
            torch.cuda.current_stream().synchronize()
            return out
        e2e_step()
        barrier()
        t0 = time.perf_counter()
        for _ in range(K):
            e2e_step()
        barrier()
        t_e2e = time.perf_counter() - t0
        if world > 1:
            tt = torch.tensor([t_e2e], device=dev, dtype=torch.float64)
            torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
            t_e2e = float(tt.item())
        h2d = sum(cfg.spaces[s.task].n_vars * s.n * 4 for s in shards)
        d2h = sum(s.n * 4 + k * (8 + 8 + 4 * cfg.spaces[s.task].n_vars) + 4 for s in shards)
        e2e = {"value": total * K / t_e2e, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "timing": "host wall clock incl. pinned H2D of every shard's y0 and D2H of losses + top-k (rank 0's bytes)"}

    if rank != 0:
        if world > 1:
            torch.distributed.destroy_process_group()
        return 0
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        rate, threads, sample, _ = oracle_baseline_tasks(cfg, args.cpu_seconds)
        cpu = {"value": rate, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample}
    # split-cone kernels (default for these population sizes) add one final Adam launch per task
    sc_final = 0                                                    # groups use the cone-group kernels
    launches = sum(1 + T * 3 + sc_final + (6 + len(cfg.mlp_dims) - 1) for _ in shards)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": t_max / K, "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
        "dtype": "fp16 hi/lo split (fp32-accurate) MLP, f64 DAG forward, f32 DAG reverse, f32 Adam, f64 scoring", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {len(cfg.spaces)} tasks x {cfg.n_seeds} seeds x {T} steps, "
                               f"MLP {list(cfg.mlp_dims)}, top-{k} per task",
                   "tasks": [sp.name for sp in cfg.spaces], "n_seeds_per_task": cfg.n_seeds, "n_steps": T,
                   "parallelism": {"task": f"dp{world}: subgraphs by LPT",
                                   "hybrid": f"dp{world}: seed-split LPT over task chunks (tasks.hybrid_assign)"}.get(
                                       mode, f"dp{world}: seed shards of every task"),
                   "rank0_tasks": [s.task for s in shards], "rank0_cand_steps_per_bench_step": local_cs,
                   "batching": ("felix_search_group: per Adam step every task's DAG kernels on its own stream, one "
                                "tensor-core MLP pass over all tasks' candidates" if batched else
                                "one felix_search per task, one CUDA stream per task"),
                   "l2": "flushed (256 MB write) between timed iterations"},
        "roofline": {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                     "traffic": None, "kernel": ("group MLP pass over all tasks' rows" if batched else
                                                 "MLP kernels of every task (searched one after another for this "
                                                 "measurement)") + ", tcgen05 kind::f16 3-pass split",
                     "executed_tflops": 3 * achieved,
                     "peak_source": f"{peak_src} bf16_tflops_sustained (fp16 = bf16 rate)"},
        "profiled_mlp_ms_per_bench_step": gemm_ms,
        "gpu_launches": launches * K,
        "clocks": clocks.summary(),
        "top1_per_task": {cfg.spaces[t].name: (float(v[1][0]) if len(v[1]) else None) for t, v in merged.items()},
    }
    if e2e is not None:
        line["e2e"] = e2e
    if cpu is not None:
        line["cpu_baseline"] = cpu
    print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()
    return 0


def run_reference_tasks(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return 0
    import felix_inputs as fi
    cfg = fi.config(args.config)
    if args.seeds:
        cfg.n_seeds = args.seeds
    if args.search_steps:
        cfg.n_steps = args.search_steps
    W = max(args.warmup, 0)
    K = max(args.steps, 1)
    rates = []
    for it in range(W + K):
        secs = max(2.0, args.cpu_seconds / max(1, (W + K)))
        rate, threads, sample, _ = oracle_baseline_tasks(cfg, secs)
        if it >= W:
            rates.append(rate)
    value = statistics.median(rates)
    total = len(cfg.spaces) * cfg.n_seeds * cfg.n_steps
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus, "steps": K,
        "warmup": W, "ms_per_step": total / value * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {len(cfg.spaces)} tasks x {cfg.n_seeds} seeds x {cfg.n_steps} steps, "
                               f"MLP {list(cfg.mlp_dims)}, top-{cfg.topk} per task"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def spawn_ranks(args) -> int:
    """`python bench.py --gpus N` without a torchrun environment: start N ranks (one per GPU) through
    torch.distributed.run on 127.0.0.1 and pass their output through.  NCCL init logging is on so the
    communicator size is visible in the log."""
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return spawn_ranks(args)
    multi = args.config in ("C3", "C4", "MBV2")
    if args.impl == "reference":
        return run_reference_tasks(args) if multi else run_reference(args)
    return run_felix_tasks(args) if multi else run_felix(args)


if __name__ == "__main__":
    sys.exit(main())
