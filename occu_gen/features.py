"""Table I node and edge features (P97-P123, P129-P133) for synthetic graphs.

Node row (F_n = 80 floats, 320 B):
  [0:40]   operator type, one-hot (P129 "categorical -> one-hot")
  [40:42]  role bits: fwd 00, bwd 10, update 01, loss 11
  [42:58]  operator hyperparameters (kernel, stride, pad, dilation, groups, C, K ...)
  [58:66]  model configuration (batch, input channels, seq, H/W, ...)
  [66:74]  input/output tensor sizes: numel of up to 3 inputs + output, then bytes
  [74]     operator FLOPs (Conv: P131 closed form; GEMM: 2MNK, P133)
  [75]     temporary tensor size
  [76:79]  runtime config: GPU peak GFLOPS, GPU memory MB, #SMs (P110-P115)
  [79]     zero pad (keeps rows 16-byte aligned)
Edge row (F_e = 4): [is_fwd, is_bwd, log2(1+bytes)/40, log2(1+bw_GBps)/16].
Numeric values are encoded as log2(1+x)/40 so they fall in [0, 1].
"""
from __future__ import annotations

import numpy as np

from .dags import ROLE_BWD, ROLE_LOSS, ROLE_UPDATE, TrainGraph, numel

F_N = 80
F_E = 4

# Table III systems (+ B200 for context): peak fp32 FLOPS, memory bytes, SMs, HBM GB/s
GPUS = {
    "A100": (19.5e12, 80e9, 108, 2039.0),
    "RTX2080Ti": (13.4e12, 11e9, 68, 616.0),
    "P40": (11.8e12, 22.5e9, 30, 346.0),
    "B200": (80e12, 180e9, 148, 8000.0),
}


def _enc(x):
    return (np.log2(1.0 + np.asarray(x, dtype=np.float64)) / 40.0)


def node_edge_quantities(g: TrainGraph, hp: dict, gpu: str = "A100"):
    """The raw (unencoded) per-node / per-edge quantities of Table I for graph g at hp:
    dict(X = node rows with the hp-independent columns and the configuration columns already
    encoded, hpn [n,16] operator hyperparameters, sizes [n,4] tensor sizes, f [n] FLOPs,
    t [n] temporary size, E = edge rows with the constant columns, nbytes [m]).
    g.fwd must be the forward builder for the same hp (shapes depend on hp)."""
    ops = g.fwd.ops
    nf = len(ops)
    n = g.num_nodes
    peak, mem, sms, bw = GPUS[gpu]
    # per forward op descriptors
    out_numel = np.array([numel(o.out_shape) for o in ops], np.float64)
    in_numel = np.zeros((nf, 3), np.float64)
    for i, o in enumerate(ops):
        for j, u in enumerate(o.inputs[:3]):
            in_numel[i, j] = out_numel[u]
    flops = np.array([o.flops for o in ops], np.float64)
    temp = np.array([o.temp for o in ops], np.float64)
    ophp = np.zeros((nf, 16), np.float64)
    for i, o in enumerate(ops):
        h = list(o.hp)[:16]
        ophp[i, :len(h)] = h
    cfg = np.zeros(8, np.float64)
    keys = ("batch", "cin", "seq", "hw")
    for j, k in enumerate(keys):
        cfg[j] = float(hp.get(k, 0))
    param_numel = np.array([numel(s) for s in g.param_shapes] or [0], np.float64)

    X = np.zeros((n, F_N), np.float64)
    X[np.arange(n), g.node_op] = 1.0
    role = g.node_role
    X[:, 40] = ((role == ROLE_BWD) | (role == ROLE_LOSS)).astype(np.float64)
    X[:, 41] = ((role == ROLE_UPDATE) | (role == ROLE_LOSS)).astype(np.float64)
    fi = g.node_fwd
    X[:, 58:66] = _enc(cfg)[None, :]
    X[:, 76] = _enc(peak / 1e9)          # GFLOPS
    X[:, 77] = _enc(mem / 1e6)           # MB
    X[:, 78] = _enc(sms)

    sizes = np.zeros((n, 4), np.float64)
    f = np.zeros(n, np.float64)
    t = np.zeros(n, np.float64)
    hpn = np.zeros((n, 16), np.float64)
    fw = role == 0
    sizes[fw, :3] = in_numel[fi[fw]]
    sizes[fw, 3] = out_numel[fi[fw]]
    f[fw] = flops[fi[fw]]
    t[fw] = temp[fi[fw]]
    hpn[fw] = ophp[fi[fw]]
    bw_ = role == ROLE_BWD
    sizes[bw_, 0] = out_numel[fi[bw_]]          # incoming gradient
    sizes[bw_, 1] = in_numel[fi[bw_], 0]        # saved activation
    sizes[bw_, 3] = in_numel[fi[bw_], 0]        # gradient w.r.t. the input
    f[bw_] = 2.0 * flops[fi[bw_]]
    t[bw_] = temp[fi[bw_]]
    hpn[bw_] = ophp[fi[bw_]]
    up = role == ROLE_UPDATE
    pn = param_numel[np.maximum(g.node_param[up], 0)]
    sizes[up, 0] = pn
    sizes[up, 3] = pn
    f[up] = 4.0 * pn
    t[up] = 2.0 * pn
    ls = role == ROLE_LOSS
    sizes[ls, 0] = out_numel[nf - 1]
    sizes[ls, 3] = 1.0
    f[ls] = 3.0 * out_numel[nf - 1]
    m = g.num_edges
    E = np.zeros((m, F_E), np.float64)
    E[:, 0] = 1.0 - g.edge_bwd
    E[:, 1] = g.edge_bwd
    nbytes = 4.0 * out_numel[g.edge_fwd_src]
    upd_edge = g.node_role[g.dst] == ROLE_UPDATE
    if upd_edge.any():
        nbytes[upd_edge] = 4.0 * param_numel[g.node_param[g.dst[upd_edge]]]
    E[:, 3] = np.log2(1.0 + bw) / 16.0
    return dict(X=X, hpn=hpn, sizes=sizes, f=f, t=t, E=E, nbytes=nbytes)


def encode_features(q):
    """Table I encoding of node_edge_quantities' output -> (node_feat f32, edge_feat f32)."""
    X, E = q["X"].copy(), q["E"].copy()
    X[:, 42:58] = _enc(q["hpn"])
    X[:, 66:70] = _enc(q["sizes"])
    X[:, 70:74] = _enc(4.0 * q["sizes"])
    X[:, 74] = _enc(q["f"])
    X[:, 75] = _enc(q["t"])
    E[:, 2] = _enc(q["nbytes"])
    return X.astype(np.float32), E.astype(np.float32)


def node_edge_features(g: TrainGraph, hp: dict, gpu: str = "A100"):
    """Return (node_feat [n,80] f32, edge_feat [m,4] f32) for graph g at hp.

    g.fwd must be the forward builder for the same hp (shapes depend on hp).
    """
    return encode_features(node_edge_quantities(g, hp, gpu))
