"""The library's NCCL data plane on the GPU.

* world = 1: occu_dist_init + the in-library ncclAllReduce run on one GPU and leave the
  training trajectory bitwise equal to the communicator-free path (sum over one rank).
* world = 2 (skipped with fewer than 2 GPUs): two ranks train LPT shards of one global batch;
  the replicas stay bitwise equal and the global loss equals the single-process loss of the
  union batch.
* watchdog: a world-2 communicator with a missing peer fails with OCCU_ENCCL after the
  timeout (ncclCommAbort) instead of hanging; the ctx then refuses collectives until re-init.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import dist as odist
from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_cluster_meiqsgls23_b200 import build
    build.build()


def _flat(L=2, d=64, seed=5):
    wc = weights.ModelConfig(L=L, F_n=80, F_e=4, d=d, d_h=d)
    return weights.unit_scale(wc, weights.init_flat(wc, seed))


def test_world1_allreduce_is_bitwise_neutral():
    b = configs.random_dag_batch(30, 811, max_nodes=40, hub=True)
    flat = _flat()
    c = occu.config(L=2, F_n=80, F_e=4, d=64)
    ma, mb = occu.Model(c), occu.Model(c)
    ma.set_params(flat)
    mb.set_params(flat)
    ma.dist_init(0, 1, occu.Model.nccl_unique_id())
    csr = occu.pack(b.graphs)
    for _ in range(4):
        la = ma.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-3)
        lb = mb.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-3)
        assert la == lb
    assert np.array_equal(ma.get_params(), mb.get_params())
    ma.dist_sync()


_WORKER = r"""
import os, sys, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, {root!r})
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu, dist as odist
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(rank)
dist.init_process_group("gloo")
b = configs.random_dag_batch(48, 812, max_nodes=60, hub=True)
wc = weights.ModelConfig(L=2, F_n=80, F_e=4, d=64, d_h=64)
flat = weights.unit_scale(wc, weights.init_flat(wc, 6))
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64), device=rank)
m.set_params(flat)
dp = odist.DataParallel(m, rank, world)
losses = [dp.train_step(b, 1e-3) for _ in range(3)]
p = torch.from_numpy(m.get_params())
allp = [torch.zeros_like(p) for _ in range(world)]
dist.all_gather(allp, p)
if rank == 0:
    assert all(torch.equal(allp[0], x) for x in allp), "replicas diverged"
    ref = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64), device=0)
    ref.set_params(flat)
    l0 = ref.train_step(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets, 1e-3)
    assert abs(l0 - losses[0]) <= 1e-5 * abs(l0), (l0, losses[0])
    print("DIST_OK", losses)
dist.barrier()
"""


def test_world2_replicas_bitwise_and_global_loss(tmp_path):
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs")
    script = tmp_path / "w.py"
    script.write_text(_WORKER.format(root=ROOT))
    out = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
                          "--nproc-per-node=2", "--master-addr", "127.0.0.1", "--master-port=29613",
                          str(script)], capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    assert "DIST_OK" in out.stdout


_HANG = r"""
import sys, time
sys.path.insert(0, {root!r})
from paper_conf_cluster_meiqsgls23_b200 import occu
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64))
m.init_weights(1)
m.dist_set_timeout(3.0)
t0 = time.time()
try:
    m.dist_init(0, 2, occu.Model.nccl_unique_id())      # rank 1 never joins
    print("NO_ERROR")
except occu.OccuError as ex:
    print("ENCCL" if ex.status == occu.OCCU_ENCCL else "OTHER", round(time.time() - t0, 1))
"""


def test_watchdog_aborts_a_missing_peer(tmp_path):
    script = tmp_path / "h.py"
    script.write_text(_HANG.format(root=ROOT))
    out = subprocess.run([sys.executable, str(script)], capture_output=True, text=True, timeout=240)
    assert "ENCCL" in out.stdout, (out.stdout, out.stderr[-2000:])
    secs = float(out.stdout.split()[-1])
    assert 2.5 <= secs <= 60.0, secs
