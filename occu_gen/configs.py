"""Seeded synthetic workloads for the BASELINE.json configs.

Every batch is (graphs, node_feat, edge_feat, targets):
  graphs     list of (num_nodes, src int32[m], dst int32[m]) with local ids
  node_feat  float32 [N, F_n]   graphs concatenated in caller order
  edge_feat  float32 [E, F_e]   graphs concatenated, INPUT edge order
  targets    float32 [B]        synthetic teacher labels in (0, 1)
Seeds: generator seed 1000 + config index.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import dags
from .features import F_E, F_N, node_edge_features
from .prng import Rng, uniform01


@dataclass
class Batch:
    graphs: list
    node_feat: np.ndarray
    edge_feat: np.ndarray
    targets: np.ndarray
    families: list

    @property
    def num_graphs(self):
        return len(self.graphs)

    @property
    def num_nodes(self):
        return int(sum(g[0] for g in self.graphs))

    @property
    def num_edges(self):
        return int(sum(len(g[1]) for g in self.graphs))

    def subset(self, idx):
        """Batch of graphs ``idx`` (in that order), features sliced accordingly."""
        noff = np.concatenate([[0], np.cumsum([g[0] for g in self.graphs])])
        eoff = np.concatenate([[0], np.cumsum([len(g[1]) for g in self.graphs])])
        nf = [self.node_feat[noff[i]:noff[i + 1]] for i in idx]
        ef = [self.edge_feat[eoff[i]:eoff[i + 1]] for i in idx]
        return Batch([self.graphs[i] for i in idx],
                     np.concatenate(nf) if nf else np.zeros((0, self.node_feat.shape[1]), np.float32),
                     np.concatenate(ef) if ef else np.zeros((0, self.edge_feat.shape[1]), np.float32),
                     self.targets[list(idx)].copy(), [self.families[i] for i in idx])


_TEACHER_NORM = {}


def _teacher_norm(seed: int, w: np.ndarray):
    """(mean, std) of the teacher's linear score u = mean(X)·w over a fixed reference set:
    the 21 families at their default hyperparameters (A100).  Fixed constants per seed, so a
    graph's label never depends on the batch it is drawn in."""
    if seed not in _TEACHER_NORM:
        us = []
        for fam in dags.FAMILIES:
            hp = dags.default_hp(fam)
            g = dags.training_graph(fam, hp)
            X, _ = node_edge_features(g, hp, "A100")
            us.append(float(X.astype(np.float64).mean(axis=0) @ w))
        _TEACHER_NORM[seed] = (float(np.mean(us)), float(np.std(us)) or 1.0)
    return _TEACHER_NORM[seed]


def teacher_targets(node_feat_list, seed: int) -> np.ndarray:
    """Synthetic labels: sigmoid of a seeded, standardised linear function of mean node
    features, y = σ(2·(u − μ)/σ_u) with u = mean(X)·w (μ, σ_u fixed per seed, see
    ``_teacher_norm``), so labels spread over (0, 1) across families and variants.

    Stands in for profiled occupancy (P85-P95), which needs the paper's GPUs.
    """
    w = 2.0 * uniform01(seed, F_N) - 1.0
    mu, sd = _teacher_norm(seed, w)
    ys = []
    for X in node_feat_list:
        u = float(X.astype(np.float64).mean(axis=0) @ w)
        z = 2.0 * (u - mu) / sd
        ys.append(1.0 / (1.0 + np.exp(-z)))
    return np.asarray(ys, np.float32)


def _make(families_hp, gpu="A100", seed=0):
    graphs, nfs, efs, fams = [], [], [], []
    for fam, hp in families_hp:
        g = dags.training_graph(fam, hp)
        X, E = node_edge_features(g, dict(dags.default_hp(fam), **hp), gpu)
        graphs.append((g.num_nodes, g.src, g.dst))
        nfs.append(X)
        efs.append(E)
        fams.append(fam)
    y = teacher_targets(nfs, seed + 7)
    return Batch(graphs, np.concatenate(nfs), np.concatenate(efs), y, fams)


def cnn_grid():
    """CNN variants: batch in {16,20..128} x C_in in 1..10, lexicographic (P237)."""
    return [{"batch": b, "cin": c} for b in range(16, 129, 4) for c in range(1, 11)]


def cfg1():
    """CFG1: one LeNet-5 training graph (~40 nodes); L=2, d=64, FP32 forward."""
    return _make([("lenet5", {"batch": 16, "cin": 1})], seed=1001)


def cfg2(num_graphs: int = 256):
    """CFG2: ResNet-50 training graphs, first 256 variants of the batch x C_in grid."""
    grid = cnn_grid()
    hps = [grid[i % len(grid)] for i in range(num_graphs)]
    return _make([("resnet50", hp) for hp in hps], seed=1002)


def transformer_variants(n: int, seed: int):
    r = Rng(seed)
    out = []
    for _ in range(n):
        out.append({"batch": int(4 * r.randint(4, 32)[0]), "cin": int(r.randint(1, 10)[0]),
                    "seq": int(r.choice([20, 512]))})
    return out


def cfg3(num_graphs: int = 512):
    """CFG3: BERT-base / GPT-2 training graphs (~5k nodes), half each."""
    hps = transformer_variants(num_graphs, 1003)
    fams = ["bert_base" if i < num_graphs // 2 else "gpt2" for i in range(num_graphs)]
    return _make(list(zip(fams, hps)), seed=1003)


def mixture_variant(family: str, r: Rng) -> dict:
    if family in dags.RNN:
        return {"batch": int(8 * r.randint(16, 64)[0]), "seq": int(8 * r.randint(2, 16)[0])}
    if family in dags.TRANSFORMER:
        return {"batch": int(4 * r.randint(4, 32)[0]), "cin": int(r.randint(1, 10)[0]),
                "seq": int(r.choice([20, 512]))}
    return {"batch": int(4 * r.randint(4, 32)[0]), "cin": int(r.randint(1, 10)[0])}


MIXTURE = [f for f in dags.FAMILIES if f != "bert_base"]   # the 20 Table II models


def mixture_specs(num_graphs: int, seed: int, start: int = 0):
    """(family, hp) of graphs ``start .. start+num_graphs-1`` of the 20-family mixture."""
    out = []
    for k in range(start, start + num_graphs):
        r = Rng((seed << 32) + k)
        fam = MIXTURE[int(r.randint(0, len(MIXTURE) - 1)[0])]
        out.append((fam, mixture_variant(fam, r)))
    return out


def mixture(num_graphs: int, seed: int, start: int = 0):
    """Graphs ``start .. start+num_graphs-1`` of the 20-family mixture (CFG4/CFG5)."""
    return _make(mixture_specs(num_graphs, seed, start), seed=seed)


def random_dag_batch(num_graphs: int, seed: int, max_nodes: int = 12, hub: bool = False,
                     f_n: int = F_N, f_e: int = F_E, allow_empty_edges: bool = True):
    """Small random DAGs (edges u<v, multi-edges allowed) with uniform features.

    Used for fuzzing the packer and for oracle / parity tests at tiny sizes.
    """
    r = Rng(seed)
    graphs, nfs, efs = [], [], []
    for _ in range(num_graphs):
        n = int(r.randint(1, max_nodes)[0])
        if n == 1:
            m = 0
        else:
            lo = 0 if allow_empty_edges else 1
            m = int(r.randint(lo, 2 * n)[0])
        s = r.randint(0, max(n - 2, 0), m) if m else np.zeros(0, np.int64)
        span = (n - 1 - s)
        t = s + 1 + np.floor(r.uniform(m) * span).astype(np.int64) if m else np.zeros(0, np.int64)
        if hub and n > 2 and m:
            h = n - 1
            extra = int(r.randint(1, 3 * n)[0])
            s = np.concatenate([s, r.randint(0, h - 1, extra)])
            t = np.concatenate([t, np.full(extra, h)])
        graphs.append((n, s.astype(np.int32), t.astype(np.int32)))
        nfs.append(r.uniform(n * f_n).reshape(n, f_n).astype(np.float32))
        efs.append(r.uniform(len(s) * f_e).reshape(len(s), f_e).astype(np.float32))
    y = r.uniform(num_graphs).astype(np.float32) * 0.8 + 0.1
    return Batch(graphs, np.concatenate(nfs), np.concatenate(efs).reshape(-1, f_e), y,
                 ["random"] * num_graphs)


def make(specs, seed: int):
    """Batch of the graphs described by ``specs`` [(family, hp)] (e.g. one rank's shard of
    ``mixture_specs``); labels from the teacher of ``seed`` as in ``mixture``."""
    return _make(list(specs), seed=seed)


def spec_work(specs) -> np.ndarray:
    """Work w = N_g + E_g of each (family, hp) spec without building its features (a
    family's topology does not depend on its hyperparameters, R39)."""
    out = []
    for fam, hp in specs:
        g = dags.training_graph(fam, hp)
        out.append(g.num_nodes + g.num_edges)
    return np.asarray(out, np.int64)


def mixture_arrays(num_graphs: int, seed: int, start: int = 0):
    """Vectorised ``mixture_specs``: (family index into MIXTURE [num], hp [num, 4]) with hp the
    ``templates.hp_vector`` row (batch, cin, seq, hw) of graph start .. start+num-1.  Same
    counter-based draws as ``mixture_specs`` (stream (seed << 32) + k, outputs 1..4), for the
    1M-graph CFG5 sweep and the 50k-graph CFG4 epoch (tests/test_gen.py checks the match)."""
    from .prng import _GOLDEN, _M1, _M2
    k = np.arange(start, start + num_graphs, dtype=np.uint64)
    base = (np.uint64(seed) << np.uint64(32)) + k

    def u(j):
        with np.errstate(over="ignore"):
            z = base + np.uint64(j) * _GOLDEN
            z = (z ^ (z >> np.uint64(30))) * _M1
            z = (z ^ (z >> np.uint64(27))) * _M2
            z = z ^ (z >> np.uint64(31))
        return (z >> np.uint64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)

    def ri(uu, lo, hi):
        return lo + np.floor(uu * (hi - lo + 1))

    u1, u2, u3, u4 = u(1), u(2), u(3), u(4)
    fam = ri(u1, 0, len(MIXTURE) - 1).astype(np.int64)
    kind = np.array([2 if f in dags.RNN else (1 if f in dags.TRANSFORMER else 0) for f in MIXTURE])[fam]
    hp = np.zeros((num_graphs, 4), np.float64)
    rnn, tr, cnn = kind == 2, kind == 1, kind == 0
    hp[rnn, 0] = 8 * ri(u2[rnn], 16, 64)
    hp[rnn, 1] = 1
    hp[rnn, 2] = 8 * ri(u3[rnn], 2, 16)
    hp[tr, 0] = 4 * ri(u2[tr], 4, 32)
    hp[tr, 1] = ri(u3[tr], 1, 10)
    hp[tr, 2] = np.where(ri(u4[tr], 0, 1) > 0, 512, 20)
    hp[cnn, 0] = 4 * ri(u2[cnn], 4, 32)
    hp[cnn, 1] = ri(u3[cnn], 1, 10)
    return fam, hp


def family_work() -> np.ndarray:
    """N_g + E_g of each MIXTURE family's training DAG (topology is hp-independent)."""
    out = []
    for f in MIXTURE:
        g = dags.training_graph(f, dags.default_hp(f))
        out.append(g.num_nodes + g.num_edges)
    return np.asarray(out, np.int64)
