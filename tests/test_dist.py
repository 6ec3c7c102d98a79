"""Data-parallel host logic on CPU: LPT sharding, contiguous inference ranges,
and a world_size-2 gloo run checking that per-rank gradients of the LPT shards
(loss scaled by the GLOBAL batch, R15), summed by a real allreduce, equal the
full-batch gradient.  (The GPU path uses the same shards with NCCL inside the
library.)"""
import os

import numpy as np
import pytest

from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import dist


def test_lpt_shard_covers_and_balances():
    b = configs.mixture(60, 1004)
    w = dist.graph_work(b.graphs)
    for world in (1, 2, 3, 8):
        sh = dist.lpt_shard(w, world)
        flat = sorted(i for s in sh for i in s)
        assert flat == list(range(len(w)))
        loads = [int(w[s].sum()) for s in sh]
        assert max(loads) - min(loads) <= int(w.max())          # LPT bound
        assert sh == dist.lpt_shard(w, world)                   # deterministic
        assert all(s == sorted(s) for s in sh)


def test_contiguous_shard():
    w = np.array([5, 1, 1, 1, 8, 2, 2, 3, 9, 1])
    for world in (1, 2, 4):
        rg = dist.contiguous_shard(w, world)
        assert rg[0][0] == 0 and rg[-1][1] == len(w)
        assert all(rg[r][1] == rg[r + 1][0] for r in range(world - 1))


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    b = configs.random_dag_batch(12, 77, max_nodes=15, hub=True)
    cfg = dict(L=2, F_n=80, F_e=4, d=8, d_h=8, aggr=0, msg=0, slope=0.01)
    from occu_gen import weights
    params = oracle.unflatten(cfg, weights.init_flat(weights.ModelConfig(L=2, d=8, d_h=8), 3).astype(np.float64))
    idx = dist.lpt_shard(dist.graph_work(b.graphs), world)[rank]
    loc = b.subset(idx)
    loss, g = oracle.loss_and_grads(params, cfg, loc.graphs, loc.node_feat, loc.edge_feat,
                                    loc.targets, global_batch=b.num_graphs)
    flat = torch.tensor(np.concatenate([np.ravel(g[k]) for k, _ in oracle.param_shapes(cfg)] + [[loss]]))
    tdist.all_reduce(flat)
    if rank == 0:
        lf, gf = oracle.loss_and_grads(params, cfg, b.graphs, b.node_feat, b.edge_feat, b.targets)
        ref = np.concatenate([np.ravel(gf[k]) for k, _ in oracle.param_shapes(cfg)] + [[lf]])
        q.put(float(np.max(np.abs(flat.numpy() - ref)) / np.max(np.abs(ref))))
    tdist.barrier()
    tdist.destroy_process_group()


def test_dp_gloo_world2_matches_full_batch():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() % 1000)
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs)
    err = q.get(timeout=5)
    assert err < 1e-12, err


def _infer_worker(rank, world, port, q):
    import torch.distributed as tdist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    tdist.init_process_group("gloo", rank=rank, world_size=world)
    rng = np.random.default_rng(11)
    work = rng.integers(10, 500, size=37)
    preds = rng.random(37).astype(np.float32)          # stand-in for each graph's prediction
    lo, hi = dist.contiguous_shard(work, world)[rank]
    allp, slots, loads = dist.gather_and_pack(preds[lo:hi], rank, world)
    if rank == 0:
        ref_slots, ref_loads = dist.gather_and_pack(preds, 0, 1)[1:]
        q.put((bool(np.array_equal(allp, preds)), bool(np.array_equal(slots, ref_slots)),
               bool(np.array_equal(loads, ref_loads))))
    tdist.barrier()
    tdist.destroy_process_group()


def test_sharded_inference_gather_and_pack_gloo_world2():
    """Graph-sharded inference (contiguous work-balanced ranges, no collective on the data
    path) plus the optional rank-0 collection: the all-gathered predictions are the global
    vector in graph order and rank 0's occu-packing equals single-process packing."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 30500 + (os.getpid() % 1000)
    procs = [ctx.Process(target=_infer_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
    assert all(p.exitcode == 0 for p in procs)
    assert q.get(timeout=5) == (True, True, True)


def test_dataparallel_host_sharding_uses_global_batch():
    """DataParallel packs only its LPT shard and scales by the GLOBAL batch size."""
    b = configs.mixture(24, 1004)
    seen = {}

    class Fake:
        def nccl_unique_id(self):
            return b"u" * 128

        def dist_init(self, rank, world, uid):
            seen["init"] = (rank, world, uid)

        def train_step(self, csr, nf, ef, y, lr, global_num_graphs=None):
            seen["B"] = csr.num_graphs
            seen["G"] = global_num_graphs
            return 0.0

    class FakePG:                     # rank 0's id reaches every rank through the broadcast
        @staticmethod
        def broadcast_object_list(lst, src=0):
            lst[0] = b"u" * 128

    dp = dist.DataParallel(Fake(), 1, 3, pg=FakePG)
    dp.train_step(b, 1e-3)
    idx = dist.lpt_shard(dist.graph_work(b.graphs), 3)[1]
    assert seen == {"B": len(idx), "G": 24, "init": (1, 3, b"u" * 128)}
