"""Per-family feature templates for on-device feature synthesis.

Input generation only (no GNN arithmetic): a DL-model family's training DAG has one topology
for all of its hyperparameter variants (P237: batch, input channels, sequence length change
shapes, not operators), so a batch of variants can be built on the GPU from a per-family
template plus four numbers per graph.  Every hyperparameter-dependent Table I quantity of a
node (16 operator hyperparameters, 4 tensor sizes, FLOPs, temporary size: 22 per node) and of
an edge (bytes carried) is a polynomial of degree <= 1 in batch, <= 1 in cin and <= 2 in seq
(shapes are products of these; attention scores carry seq^2).  It is stored in tensor-product
Newton form on the nodes

    BATCH_NODES = (4, 8), CIN_NODES = (1, 2), SEQ_NODES = (16, 32, 48):
    q(b, c, s) = sum_{i<2, j<2, k<3} C[i, j, k] * Nb_i(b) * Nc_j(c) * Ns_k(s),
    Nb = (1, b - 4), Nc = (1, c - 1), Ns = (1, s - 16, (s - 16)(s - 32)),

coefficient index m = 6 i + 3 j + k.  The coefficients are divided differences with dyadic node
spacings, so for integer quantities below 2^53 they, the basis products and every partial sum
are exact in float64: the form reproduces the generator's float64 quantities exactly, which
``verify`` checks at held-out hyperparameters.  The library (occu_synthesize) evaluates the
same form in float64 on the device and applies the Table I encoding log2(1 + x) / 40.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import dags
from .features import node_edge_quantities

BATCH_NODES = (4, 8)
CIN_NODES = (1, 2)
SEQ_NODES = (16, 32, 48)
NODE_Q = 22          # hpn[16], sizes[4], f, t
NCOEF = 12
HP_KEYS = ("batch", "cin", "seq", "hw")


@dataclass
class Template:
    family: str
    num_nodes: int
    src: np.ndarray          # int32 [m] local ids (the family's training DAG)
    dst: np.ndarray
    node_static: np.ndarray  # float32 [n, 80]: hp-independent columns, zeros elsewhere
    node_coef: np.ndarray    # float64 [n, 22, 12]
    edge_static: np.ndarray  # float32 [m, 4]: hp-independent columns, zeros in column 2
    edge_coef: np.ndarray    # float64 [m, 12]


def hp_vector(family: str, hp: dict) -> np.ndarray:
    """The four per-graph numbers (batch, cin, seq, hw) exactly as the feature generator sees
    them (family defaults filled in, absent keys 0)."""
    full = dict(dags.default_hp(family), **hp)
    return np.array([float(full.get(k, 0)) for k in HP_KEYS], np.float64)


def _node_q(q):
    return np.concatenate([q["hpn"], q["sizes"], q["f"][:, None], q["t"][:, None]], axis=1)


def _divdiff(a, axis, nodes):
    """Newton divided differences of the samples along ``axis`` (nodes ascending)."""
    a = np.moveaxis(a, axis, 0).copy()
    x = np.asarray(nodes, np.float64)
    for lev in range(1, len(x)):
        for i in range(len(x) - 1, lev - 1, -1):
            a[i] = (a[i] - a[i - 1]) / (x[i] - x[i - lev])
    return np.moveaxis(a, 0, axis)


def build_template(family: str, gpu: str = "A100") -> Template:
    qn = np.empty((2, 2, 3), dtype=object)
    g0 = q0 = None
    for i, b in enumerate(BATCH_NODES):
        for j, c in enumerate(CIN_NODES):
            for k, s in enumerate(SEQ_NODES):
                hp = dict(dags.default_hp(family), batch=b, cin=c, seq=s)
                g = dags.training_graph(family, hp)
                q = node_edge_quantities(g, hp, gpu)
                if g0 is None:
                    g0, q0 = g, q
                qn[i, j, k] = (_node_q(q), q["nbytes"])
    n, m = g0.num_nodes, g0.num_edges
    N = np.stack([np.stack([np.stack([qn[i, j, k][0] for k in range(3)]) for j in range(2)])
                  for i in range(2)])                     # [2, 2, 3, n, 22]
    E = np.stack([np.stack([np.stack([qn[i, j, k][1] for k in range(3)]) for j in range(2)])
                  for i in range(2)])                     # [2, 2, 3, m]
    for ax, nodes in ((0, BATCH_NODES), (1, CIN_NODES), (2, SEQ_NODES)):
        N = _divdiff(N, ax, nodes)
        E = _divdiff(E, ax, nodes)
    node_coef = np.ascontiguousarray(N.reshape(NCOEF, n, NODE_Q).transpose(1, 2, 0))
    edge_coef = np.ascontiguousarray(E.reshape(NCOEF, m).T)
    X = q0["X"].copy()
    X[:, 42:76] = 0.0            # operator hp, configuration, sizes, FLOPs, temp: per graph
    Es = q0["E"].copy()
    Es[:, 2] = 0.0
    return Template(family, n, g0.src.astype(np.int32), g0.dst.astype(np.int32),
                    X.astype(np.float32), node_coef, Es.astype(np.float32), edge_coef)


def basis(hpv) -> np.ndarray:
    """The 12 Newton basis values at (batch, cin, seq) in coefficient order m = 6 i + 3 j + k."""
    b, c, s = float(hpv[0]), float(hpv[1]), float(hpv[2])
    nb = (1.0, b - BATCH_NODES[0])
    nc = (1.0, c - CIN_NODES[0])
    ns = (1.0, s - SEQ_NODES[0], (s - SEQ_NODES[0]) * (s - SEQ_NODES[1]))
    return np.array([nb[i] * nc[j] * ns[k] for i in range(2) for j in range(2) for k in range(3)])


def evaluate(t: Template, hpv):
    """Host evaluation of the template at one graph's (batch, cin, seq, hw): the node quantities
    [n, 22] and edge bytes [m], summed in coefficient order like the device."""
    bv = basis(hpv)
    nq = np.zeros((t.num_nodes, NODE_Q))
    eq = np.zeros(len(t.src))
    for mi in range(NCOEF):
        nq += t.node_coef[:, :, mi] * bv[mi]
        eq += t.edge_coef[:, mi] * bv[mi]
    return nq, eq


def verify(t: Template, hps, gpu: str = "A100") -> None:
    """Raise unless the template reproduces the generator's raw quantities exactly at ``hps``."""
    for hp in hps:
        full = dict(dags.default_hp(t.family), **hp)
        g = dags.training_graph(t.family, full)
        q = node_edge_quantities(g, full, gpu)
        nq, eq = evaluate(t, hp_vector(t.family, hp))
        if not (np.array_equal(nq, _node_q(q)) and np.array_equal(eq, q["nbytes"])):
            bad = np.argwhere(nq != _node_q(q))
            raise ValueError(f"{t.family}: template not exact at {hp} (first node/quantity {bad[:1]})")
