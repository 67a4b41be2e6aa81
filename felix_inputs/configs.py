"""Seeded synthetic workloads: the BASELINE.json configs C1..C5 as search spaces, random-init cost
model weights, and parity-test starting points.  Input generation only — no method arithmetic.

* Spaces: layer shapes of the paper's workloads (ResNet-50 / ViT / BERT) in the
  sketch of felix_inputs/programs.py.
* Cost model: TenSet MLP architecture, 4 linear layers ~250K params (L1056-1059) -> dims
  [82, 512, 256, 256, 1]; trained weights are unavailable, so weights/biases are U(+-1/sqrt(fan_in))
  drawn from splitmix64 streams seeded 0xC0FFEE00 + layer.
* y0 for parity tests: numpy Generator, uniform in [-0.3, ln(ub) + 0.3] per variable so that some
  points violate the validity bounds (exercising the penalty, Eq. 4).
"""
from __future__ import annotations

import math
from dataclasses import dataclass
from typing import Dict, List, Sequence, Tuple

import numpy as np

from .dag import Space, VAR_INT, VAR_SPLIT
from .programs import (build_space, conv2d_spec, dense_spec, depthwise_conv2d_spec, layernorm_spec, paper_dense_add_s1,
                       softmax_spec)

MASK64 = (1 << 64) - 1
DEFAULT_MLP = (82, 512, 256, 256, 1)
C1_MLP = (82, 256, 1)


def splitmix64_stream(seed: int, n: int) -> np.ndarray:
    """n successive splitmix64 outputs (uint64) from state `seed` (used only to draw weights)."""
    out = np.empty(n, dtype=np.uint64)
    s = seed & MASK64
    for i in range(n):
        s = (s + 0x9E3779B97F4A7C15) & MASK64
        z = s
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
        out[i] = z ^ (z >> 31)
    return out


def _uniform_pm(seed: int, n: int, bound: float) -> np.ndarray:
    # vectorised splitmix64 (same recurrence as splitmix64_stream, unrolled over the counter)
    i = np.arange(1, n + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & MASK64) + i * np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    u = (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)   # [0, 1), 53 bits
    return ((2.0 * u - 1.0) * bound).astype(np.float32)


@dataclass
class MLPWeights:
    dims: Tuple[int, ...]
    W: List[np.ndarray]     # float32 [dims[l+1], dims[l]]
    b: List[np.ndarray]     # float32 [dims[l+1]]


def make_mlp(dims: Sequence[int] = DEFAULT_MLP, seed_base: int = 0xC0FFEE00) -> MLPWeights:
    W, B = [], []
    for l in range(len(dims) - 1):
        fan_in, fan_out = dims[l], dims[l + 1]
        bound = 1.0 / math.sqrt(fan_in)
        w = _uniform_pm(seed_base + 2 * l, fan_in * fan_out, bound).reshape(fan_out, fan_in)
        bb = _uniform_pm(seed_base + 2 * l + 1, fan_out, bound)
        W.append(np.ascontiguousarray(w))
        B.append(np.ascontiguousarray(bb))
    return MLPWeights(tuple(dims), W, B)


def var_upper_bounds(space: Space) -> np.ndarray:
    """ub_j: smallest extent among the var's splits (SPLIT) or hi (INT)."""
    ub = np.zeros(space.n_vars)
    for j, v in enumerate(space.vars):
        if v.kind == VAR_INT:
            ub[j] = v.hi
        else:
            ub[j] = min(s.extent for s in space.splits if j in s.vars)
    return ub


def make_y0(space: Space, n: int, seed: int, margin: float = 0.3) -> np.ndarray:
    """Parity-test starting points, float32 SoA [n_vars][n]."""
    rng = np.random.default_rng(seed)
    ub = np.log(var_upper_bounds(space))
    lo = np.array([math.log(v.lo) if v.kind == VAR_INT else 0.0 for v in space.vars])
    y = rng.uniform(lo[:, None] - margin, ub[:, None] + margin, size=(space.n_vars, n))
    return np.ascontiguousarray(y.astype(np.float32))


# ---------------------------------------------------------------------------- BASELINE.json configs
@dataclass
class Config:
    name: str
    spaces: List[Space]
    mlp_dims: Tuple[int, ...]
    n_seeds: int
    n_steps: int
    rng_seed: int
    lr: float = 0.05
    lam: float = 1.0
    topk: int = 16


def c1_space() -> Space:
    return build_space(dense_spec("dense_64x64x64", 64, 64, 64, i_levels="ti", j_levels="ti", k_vars=1, bias=True))


def c2_space() -> Space:
    return build_space(conv2d_spec("resnet50_conv3x3_56x56x64", 64, 56, 56, 64, 3, 3, 1))


def c2_space_two_statements() -> Space:
    """C2 with TenSet-style per-statement features: [reduction statement | fused bias+ReLU epilogue],
    82 features each."""
    return build_space(conv2d_spec("resnet50_conv3x3_56x56x64_2stmt", 64, 56, 56, 64, 3, 3, 1), statements=2)


def c2_sketches() -> List[Space]:
    """Several symbolic programs p*_i of the C2 subgraph (Eq. 3): the multi-level-tiling
    sketch with 3-level spatial tiling and a 2-way reduction split (= c2_space), with a 1-way
    reduction split, and with 2-level spatial tiling (no virtual threads)."""
    C, H, W, K, R, S = 64, 56, 56, 64, 3, 3
    return [
        build_space(conv2d_spec("resnet50_conv3x3_56x56x64", C, H, W, K, R, S, 1)),
        build_space(conv2d_spec("resnet50_conv3x3_56x56x64_rc1", C, H, W, K, R, S, 1, rc_vars=1)),
        build_space(conv2d_spec("resnet50_conv3x3_56x56x64_ti", C, H, W, K, R, S, 1,
                                co_levels="ti", h_levels="ti", w_levels="ti", rc_vars=2)),
    ]


def c5_space() -> Space:
    return build_space(dense_spec("vitl16_fc1_197x4096x1024", 197, 4096, 1024, i_levels="vti", j_levels="vti",
                                  k_vars=2, bias=True, gelu=True))


def bert_spaces() -> List[Space]:
    """BERT-base seq 128 subgraphs (C4, BASELINE.json configs[3] "batched matmul/softmax"): QKV / output /
    FFN dense layers, the two attention bmms, the attention softmax (12 heads x 128 x 128) and a layernorm
    (128 x 768)."""
    return [
        build_space(dense_spec("bert_qkv_128x2304x768", 128, 2304, 768, i_levels="vti", j_levels="vti", k_vars=2)),
        build_space(dense_spec("bert_bmm_qk_12x128x128x64", 128, 128, 64, batch=12, i_levels="ti", j_levels="vti", k_vars=1, bias=False)),
        build_space(dense_spec("bert_bmm_av_12x128x64x128", 128, 64, 128, batch=12, i_levels="ti", j_levels="vti", k_vars=1, bias=False)),
        build_space(dense_spec("bert_proj_128x768x768", 128, 768, 768, i_levels="vti", j_levels="vti", k_vars=2)),
        build_space(dense_spec("bert_ffn1_128x3072x768", 128, 3072, 768, i_levels="vti", j_levels="vti", k_vars=2, gelu=True)),
        build_space(dense_spec("bert_ffn2_128x768x3072", 128, 768, 3072, i_levels="vti", j_levels="vti", k_vars=2)),
        build_space(softmax_spec("bert_softmax_12x128x128", 12, 128, 128, i_levels="vti", j_vars=1)),
        build_space(layernorm_spec("bert_layernorm_128x768", 128, 768, i_levels="vti", j_vars=2)),
    ]


def resnet50_spaces() -> List[Space]:
    """Unique conv/dense layer shapes of ResNet-50 @224 (C3), batch 1."""
    S = []
    convs = [  # (C, H_out, W_out, K, R, S, stride)
        (3, 112, 112, 64, 7, 7, 2),
        (64, 56, 56, 64, 1, 1, 1), (64, 56, 56, 64, 3, 3, 1), (64, 56, 56, 256, 1, 1, 1), (256, 56, 56, 64, 1, 1, 1),
        (256, 28, 28, 128, 1, 1, 2), (128, 28, 28, 128, 3, 3, 1), (128, 28, 28, 512, 1, 1, 1), (256, 28, 28, 512, 1, 1, 2),
        (512, 28, 28, 128, 1, 1, 1),
        (512, 14, 14, 256, 1, 1, 2), (256, 14, 14, 256, 3, 3, 1), (256, 14, 14, 1024, 1, 1, 1), (512, 14, 14, 1024, 1, 1, 2),
        (1024, 14, 14, 256, 1, 1, 1),
        (1024, 7, 7, 512, 1, 1, 2), (512, 7, 7, 512, 3, 3, 1), (512, 7, 7, 2048, 1, 1, 1), (1024, 7, 7, 2048, 1, 1, 2),
        (2048, 7, 7, 512, 1, 1, 1),
    ]
    for (C, H, W, K, R, Ss, st) in convs:
        S.append(build_space(conv2d_spec(f"r50_conv_c{C}_h{H}_k{K}_r{R}_s{st}", C, H, W, K, R, Ss, st)))
    S.append(build_space(dense_spec("r50_fc_1x1000x2048", 1, 1000, 2048, i_levels="t", j_levels="vti", k_vars=2)))
    return S


def mobilenet_v2_spaces() -> List[Space]:
    """MobileNet-v2 @224 (the north star's "ResNet/MobileNet convs"): its depthwise 3x3 convs
    (stride 1 and 2) and representative pointwise 1x1 expansion / projection convs, batch 1."""
    dws = [(32, 112, 112, 1), (96, 56, 56, 2), (144, 56, 56, 1), (144, 28, 28, 2), (192, 28, 28, 1),
           (384, 14, 14, 1), (576, 7, 7, 2), (960, 7, 7, 1)]          # (C, H_out, W_out, stride)
    out = [build_space(depthwise_conv2d_spec(f"mbv2_dw_c{C}_h{H}_s{st}", C, H, W, 3, 3, st)) for C, H, W, st in dws]
    pws = [(16, 112, 112, 96), (24, 56, 56, 144), (144, 28, 28, 32), (384, 14, 14, 96), (960, 7, 7, 320)]
    out += [build_space(conv2d_spec(f"mbv2_pw_c{C}_h{H}_k{K}", C, H, W, K, 1, 1, 1)) for C, H, W, K in pws]
    return out


def config(name: str) -> Config:
    if name == "C1":
        return Config("C1", [c1_space()], C1_MLP, 64, 20, 0x5EED0001)
    if name == "C2":
        return Config("C2", [c2_space()], DEFAULT_MLP, 4096, 200, 0x5EED0002)
    if name == "C3":
        return Config("C3", resnet50_spaces(), DEFAULT_MLP, 8192, 200, 0x5EED0003)
    if name == "C4":
        return Config("C4", bert_spaces(), DEFAULT_MLP, 16384, 500, 0x5EED0004)
    if name == "MBV2":      # not a BASELINE config: MobileNet-v2 task set, searched like C3
        return Config("MBV2", mobilenet_v2_spaces(), DEFAULT_MLP, 8192, 200, 0x5EED0006)
    if name == "C5":
        return Config("C5", [c5_space()], DEFAULT_MLP, 1 << 20, 200, 0x5EED0005, topk=64)
    raise KeyError(name)


def paper_example_space() -> Space:
    return paper_dense_add_s1()
