"""Input transforms for SURVEY §8(d)'s supplementary micro-benchmarks (seeded, synthetic).

* ``skew``: 1 % of each graph's nodes become hubs of in-degree ``deg`` (default 1,024); the
  extra in-edges come from earlier nodes of the same graph (drawn with replacement, so the
  graph stays a DAG and multi-edges appear, R17), their features copied from random existing
  edges of the graph.
* ``shuffle``: a random node permutation within each graph (worst-case gather locality);
  node feature rows move with their nodes, edge order is unchanged.

No GNN arithmetic here: these only rearrange / extend inputs.
"""
from __future__ import annotations

import numpy as np

from .configs import Batch
from .prng import Rng


def _offsets(batch):
    noff = np.concatenate([[0], np.cumsum([g[0] for g in batch.graphs])])
    eoff = np.concatenate([[0], np.cumsum([len(g[1]) for g in batch.graphs])])
    return noff, eoff


def skew(batch: Batch, seed: int, frac: float = 0.01, deg: int = 1024) -> Batch:
    r = Rng(seed)
    noff, eoff = _offsets(batch)
    graphs, efs = [], []
    for b, (n, s, t) in enumerate(batch.graphs):
        ef = batch.edge_feat[eoff[b]:eoff[b + 1]]
        k = max(1, int(round(frac * n))) if n > 2 else 0
        hubs = (np.sort(r.randint(n // 2, n - 1, k)) if k else np.zeros(0, np.int64))
        ns, nt, nef = [s], [t], [ef]
        for h in hubs:
            src = r.randint(0, int(h) - 1, deg)
            ns.append(src.astype(np.int32))
            nt.append(np.full(deg, h, np.int32))
            pick = r.randint(0, max(len(s) - 1, 0), deg) if len(s) else np.zeros(deg, np.int64)
            nef.append(ef[pick] if len(s) else np.zeros((deg, batch.edge_feat.shape[1]), np.float32))
        graphs.append((n, np.concatenate(ns).astype(np.int32), np.concatenate(nt).astype(np.int32)))
        efs.append(np.concatenate(nef))
    return Batch(graphs, batch.node_feat.copy(), np.concatenate(efs).astype(np.float32),
                 batch.targets.copy(), list(batch.families))


def shuffle(batch: Batch, seed: int) -> Batch:
    r = Rng(seed)
    noff, _ = _offsets(batch)
    graphs, nfs = [], []
    for b, (n, s, t) in enumerate(batch.graphs):
        perm = np.argsort(r.uniform(n), kind="stable")       # new id of old node u = inv[u]
        inv = np.empty(n, np.int64)
        inv[perm] = np.arange(n)
        graphs.append((n, inv[s].astype(np.int32), inv[t].astype(np.int32)))
        nfs.append(batch.node_feat[noff[b]:noff[b + 1]][perm])
    return Batch(graphs, np.concatenate(nfs), batch.edge_feat.copy(), batch.targets.copy(),
                 list(batch.families))
