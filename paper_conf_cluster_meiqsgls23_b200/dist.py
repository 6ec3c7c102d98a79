"""Data-parallel plumbing around the C-ABI (north_star: "graph batches shard
data-parallel across the GPUs of one box, with an NCCL gradient allreduce";
"inference batches shard by graph with no collective").

* ``lpt_shard``: deterministic longest-processing-time assignment of graphs to
  ranks by work w_g = N_g + E_g, ties broken by graph index then
  rank; each shard keeps the caller's graph order.
* ``contiguous_shard``: work-balanced contiguous ranges (inference, CFG5).
* ``gather_and_pack``: graph-sharded inference's optional collection step (SURVEY §8(e),
  NEXT-4): every rank holds the predictions of its contiguous range; they are all-gathered in
  rank order (= global graph order) and rank 0 runs the occu-packing consumer on them.
* ``DataParallel``: one process per GPU; rank 0 asks the library for an NCCL
  unique id, torch.distributed broadcasts it, every rank calls occu_dist_init;
  ``train_step`` packs the local shard and calls occu_train_step with the
  GLOBAL batch size (loss scale 1/B_glob, R15) so the in-library
  allreduce(sum) yields the global gradient.  Only host-side orchestration
  lives here; every FLOP runs in the library.
"""
from __future__ import annotations

import heapq

import numpy as np


def graph_work(graphs) -> np.ndarray:
    return np.array([int(n) + len(s) for n, s, _ in graphs], dtype=np.int64)


def lpt_shard(work, world: int):
    """Return per-rank sorted index lists.  LPT: heaviest graph first onto the
    currently lightest rank (ties: lower graph index first, lower rank first)."""
    work = np.asarray(work, dtype=np.int64)
    order = sorted(range(len(work)), key=lambda i: (-int(work[i]), i))
    heap = [(0, r) for r in range(world)]
    heapq.heapify(heap)
    shards = [[] for _ in range(world)]
    for i in order:
        load, r = heapq.heappop(heap)
        shards[r].append(i)
        heapq.heappush(heap, (load + int(work[i]), r))
    return [sorted(s) for s in shards]


def contiguous_shard(work, world: int):
    """Contiguous ranges [start, end) with balanced prefix work (inference)."""
    work = np.asarray(work, dtype=np.int64)
    csum = np.concatenate([[0], np.cumsum(work)])
    total = csum[-1]
    bounds = [0]
    for r in range(1, world):
        bounds.append(int(np.searchsorted(csum, total * r / world, side="left")))
    bounds.append(len(work))
    bounds = np.maximum.accumulate(bounds)
    return [(int(bounds[r]), int(bounds[r + 1])) for r in range(world)]


def shard_batch(batch, idx):
    """Sub-batch (graphs, node_feat, edge_feat, targets) of a configs.Batch-like object."""
    return batch.subset(list(idx))


class DataParallel:
    """One rank of DP training over torch.distributed (NCCL inside the library)."""

    def __init__(self, model, rank: int, world: int, pg=None):
        self.model = model
        self.rank = rank
        self.world = world
        if world > 1:
            import torch.distributed as dist
            pg = pg or dist
            uid = [model.nccl_unique_id() if rank == 0 else None]
            pg.broadcast_object_list(uid, src=0)
            model.dist_init(rank, world, uid[0])

    def local_indices(self, graphs):
        return lpt_shard(graph_work(graphs), self.world)[self.rank]

    def train_step(self, batch, lr: float):
        """batch: global configs.Batch; returns the global mean loss."""
        from . import occu
        idx = self.local_indices(batch.graphs)
        local = shard_batch(batch, idx)
        csr = occu.pack(local.graphs)
        return self.model.train_step(csr, local.node_feat, local.edge_feat, local.targets, lr,
                                     global_num_graphs=batch.num_graphs)


def gather_and_pack(local_pred, rank: int, world: int, pg=None, capacity: float = 1.0):
    """All-gather every rank's predictions (contiguous shards, rank order = graph order) and
    run occu-packing (occu_pack_jobs, P390-P392) on rank 0.  Returns (all predictions, slot of
    each job, slot loads) on rank 0 and (all predictions, None, None) elsewhere."""
    import torch
    from . import occu
    local = torch.as_tensor(np.ascontiguousarray(local_pred, dtype=np.float32))
    if world > 1:
        import torch.distributed as dist
        pg = pg or dist
        sizes = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
        pg.all_gather(sizes, torch.tensor([local.numel()], dtype=torch.int64))
        mx = int(max(int(x.item()) for x in sizes))
        buf = torch.zeros(mx, dtype=torch.float32)
        buf[:local.numel()] = local
        parts = [torch.zeros(mx, dtype=torch.float32) for _ in range(world)]
        pg.all_gather(parts, buf)
        allp = np.concatenate([parts[r][:int(sizes[r].item())].numpy() for r in range(world)])
    else:
        allp = local.numpy()
    if rank != 0:
        return allp, None, None
    slots, loads = occu.pack_jobs(allp, capacity)
    return allp, slots, loads
