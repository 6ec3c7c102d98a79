"""Parameter layout, deterministic initialisation and the weights file.

Layout (SURVEY §8(b) "Weights file"; shapes from P141-P149 read as in
DESIGN.md R1-R6): for each ANEE layer i = 1..L
    W_u[d][d_in]  W_e[d][d_e_in]  W_m[d][d]  a_s[d]  a_d[d]
with d_in = F_n, d_e_in = F_e for i = 1 and d otherwise; then per Graphormer layer j
(graphormer > 0) G{j}_ ln1_g ln1_b Wq bq Wk bk Wv bv Wo bo ln2_g ln2_b
F_W1 F_b1 F_W2 F_b2; with the Set-Transformer
decoder readout (readout = 1, R30-R34) the decoder's
parameters follow (seeds S[k][d]; the pre-pooling FFN P_*; the two MABs M1_*, M2_* each
Wq bq Wk bk Wv bv Wo bo ln1_g ln1_b F_W1 F_b1 F_W2 F_b2 ln2_g ln2_b; the final FFN D_*);
then the MLP head (P125)  W_1[d_h][k·d or d]  b_1[d_h]  w_2[d_h]  b_2[1].

Initialisation: element j of the flat parameter vector (file order) is
float32((2*u_j - 1) * bound(tensor)), u_j = splitmix64 uniform #j for the
seed, bound = 1/sqrt(fan_in) (PyTorch-Linear-like); LayerNorm gains are 1 and
biases 0 (PyTorch's LayerNorm init).  The C library's ``occu_init_weights`` implements the
same rule independently.

File: b"OCCUW001", u32[8] = (version, L, F_n, F_e, d, d_h, aggr, msg), f32 slope,
[version 2: u32[3] = (readout, k, heads); version 3: u32[4] = (readout, k, heads,
graphormer)], f32 payload (flat, file order), u64 FNV-1a of the payload bytes.  Version 1 =
mean readout, version 2 = decoder readout, version 3 = Graphormer layers (any readout).
No method arithmetic lives here.
"""
from __future__ import annotations

import math
import struct
from dataclasses import dataclass

import numpy as np

from .prng import uniform01

MAGIC = b"OCCUW001"
VERSION = 1
AGGR_SUM, AGGR_MEAN = 0, 1
MSG_CHANNEL_SOFTMAX, MSG_NEIGHBOR_SOFTMAX = 0, 1


@dataclass(frozen=True)
class ModelConfig:
    L: int = 3
    F_n: int = 80
    F_e: int = 4
    d: int = 128
    d_h: int = 128
    aggr: int = AGGR_SUM
    msg: int = MSG_CHANNEL_SOFTMAX
    slope: float = 0.01
    readout: int = 0        # 0: segmented mean (a7), 1: Set-Transformer decoder (NEXT-2)
    k: int = 4              # decoder seeds
    heads: int = 4          # decoder / Graphormer attention heads
    graphormer: int = 0     # Graphormer layers after the ANEE rounds (NEXT-3)


def param_specs(cfg: ModelConfig):
    """[(name, shape, fan_in)] in file order."""
    specs = []
    for i in range(cfg.L):
        d_in = cfg.F_n if i == 0 else cfg.d
        de_in = cfg.F_e if i == 0 else cfg.d
        specs += [
            (f"W_u{i}", (cfg.d, d_in), d_in),
            (f"W_e{i}", (cfg.d, de_in), de_in),
            (f"W_m{i}", (cfg.d, cfg.d), cfg.d),
            (f"a_s{i}", (cfg.d,), 2 * cfg.d),
            (f"a_d{i}", (cfg.d,), 2 * cfg.d),
        ]
    d = cfg.d
    hin = d
    # fan_in -1: constant 1 (LayerNorm gain), 0: constant 0 (LayerNorm bias)
    lin = lambda p: [(f"{p}W1", (d, d), d), (f"{p}b1", (d,), d), (f"{p}W2", (d, d), d), (f"{p}b2", (d,), d)]
    for j in range(cfg.graphormer):          # Graphormer layers (NEXT-3)
        g = f"G{j}_"
        specs += [(f"{g}ln1_g", (d,), -1), (f"{g}ln1_b", (d,), 0)]
        for w in ("q", "k", "v", "o"):
            specs += [(f"{g}W{w}", (d, d), d), (f"{g}b{w}", (d,), d)]
        specs += [(f"{g}ln2_g", (d,), -1), (f"{g}ln2_b", (d,), 0)] + lin(f"{g}F_")
    if cfg.readout == 1:
        specs += [("S", (cfg.k, d), d)] + lin("P_")
        for m in ("M1_", "M2_"):
            for w in ("q", "k", "v", "o"):
                specs += [(f"{m}W{w}", (d, d), d), (f"{m}b{w}", (d,), d)]
            specs += [(f"{m}ln1_g", (d,), -1), (f"{m}ln1_b", (d,), 0)] + lin(f"{m}F_")
            specs += [(f"{m}ln2_g", (d,), -1), (f"{m}ln2_b", (d,), 0)]
        specs += lin("D_")
        hin = cfg.k * d
    specs += [
        ("W_1", (cfg.d_h, hin), hin),
        ("b_1", (cfg.d_h,), hin),
        ("w_2", (cfg.d_h,), cfg.d_h),
        ("b_2", (1,), cfg.d_h),
    ]
    return specs


def num_params(cfg: ModelConfig) -> int:
    return sum(int(np.prod(s)) for _, s, _ in param_specs(cfg))


def init_flat(cfg: ModelConfig, seed: int) -> np.ndarray:
    """Flat float32 parameter vector, deterministic in ``seed``."""
    specs = param_specs(cfg)
    out = np.empty(num_params(cfg), dtype=np.float32)
    off = 0
    for _, shape, fan_in in specs:
        n = int(np.prod(shape))
        if fan_in <= 0:
            out[off:off + n] = 1.0 if fan_in < 0 else 0.0
        else:
            u = uniform01(seed, n, off)
            bound = 1.0 / math.sqrt(float(fan_in))
            out[off:off + n] = ((2.0 * u - 1.0) * bound).astype(np.float32)
        off += n
    return out


def unflatten(cfg: ModelConfig, flat: np.ndarray) -> dict:
    out, off = {}, 0
    for name, shape, _ in param_specs(cfg):
        n = int(np.prod(shape))
        out[name] = flat[off:off + n].reshape(shape)
        off += n
    assert off == flat.size
    return out


def flatten(cfg: ModelConfig, params: dict) -> np.ndarray:
    return np.concatenate([np.asarray(params[n], dtype=np.float32).ravel()
                           for n, _, _ in param_specs(cfg)])


def fnv1a64(data: bytes) -> int:
    h = 0xCBF29CE484222325
    arr = np.frombuffer(data, dtype=np.uint8)
    # chunked pure-python loop is slow for 0.5 MB; vectorise per byte sequentially
    for b in arr.tobytes():
        h ^= b
        h = (h * 0x100000001B3) & 0xFFFFFFFFFFFFFFFF
    return h


def write_weights(path: str, cfg: ModelConfig, flat: np.ndarray) -> None:
    flat = np.ascontiguousarray(flat, dtype="<f4")
    assert flat.size == num_params(cfg)
    payload = flat.tobytes()
    with open(path, "wb") as f:
        f.write(MAGIC)
        version = 3 if cfg.graphormer else (2 if cfg.readout else VERSION)
        f.write(struct.pack("<8I", version, cfg.L, cfg.F_n, cfg.F_e, cfg.d,
                            cfg.d_h, cfg.aggr, cfg.msg))
        f.write(struct.pack("<f", cfg.slope))
        if version == 2:
            f.write(struct.pack("<3I", cfg.readout, cfg.k, cfg.heads))
        elif version == 3:
            f.write(struct.pack("<4I", cfg.readout, cfg.k, cfg.heads, cfg.graphormer))
        f.write(payload)
        f.write(struct.pack("<Q", fnv1a64(payload)))


def unit_scale(cfg: ModelConfig, flat: np.ndarray) -> np.ndarray:
    """parity weights with W_u multiplied by d so activations keep
    their scale through the channel softmax (reading A)."""
    p = unflatten(cfg, flat.copy())
    for i in range(cfg.L):
        p[f"W_u{i}"] = (p[f"W_u{i}"].astype(np.float64) * cfg.d).astype(np.float32)
    return flatten(cfg, p)
