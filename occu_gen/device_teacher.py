"""Synthetic labels for batches whose features were synthesized on the GPU (CFG4 epoch).

Input generation only, like ``configs.teacher_targets`` (same formula, same constants):
y_b = σ(2·(u_b − μ)/σ_u), u_b = mean over graph b's nodes of X_u·w.  The per-node dot product
and the segment mean run as torch ops on the synthesized device features — this is the
workload generator standing in for profiled labels, not the method (every GNN step runs in the
library).  Agrees with the host teacher up to float rounding (tests/test_gpu_synth.py).
"""
from __future__ import annotations

import numpy as np

from . import configs
from .features import F_N
from .prng import uniform01

_W = {}


def targets(node_feat, node_off, seed: int):
    """node_feat: CUDA float32 [N, 80]; node_off: CUDA int32 [B + 1]; returns CUDA float32 [B]."""
    import torch
    if seed not in _W:
        w = 2.0 * uniform01(seed, F_N) - 1.0
        mu, sd = configs._teacher_norm(seed, w)
        _W[seed] = (torch.from_numpy(w), mu, sd)
    w, mu, sd = _W[seed]
    w = w.to(node_feat.device)
    un = node_feat.double() @ w
    off = node_off.long()
    cs = torch.cat([torch.zeros(1, dtype=torch.float64, device=un.device), torch.cumsum(un, 0)])
    cnt = (off[1:] - off[:-1]).double()
    u = (cs[off[1:]] - cs[off[:-1]]) / cnt
    return torch.sigmoid(2.0 * (u - mu) / sd).float()


def host_reference(batch, seed: int) -> np.ndarray:
    """The host teacher of the same graphs (for the GPU test)."""
    return configs.teacher_targets(
        [batch.node_feat[o0:o1] for o0, o1 in zip(*_offsets(batch))], seed)


def _offsets(batch):
    off = np.concatenate([[0], np.cumsum([g[0] for g in batch.graphs])])
    return off[:-1], off[1:]
