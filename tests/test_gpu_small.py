"""GPU parity of the single-CTA small-batch forward (CFG1-sized batches: <= 64 nodes, <= 128
edges; kernels_small.cu) against the float64 oracle and against the regular multi-kernel path
(forced by keep_intermediates).  FP32 tolerance 1e-4."""
import numpy as np
import pytest

import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu
TOL = 1e-4


def ocfg(c):
    return dict(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg,
                slope=float(np.float32(c.slope)))


def wcfg(c):
    return weights.ModelConfig(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr)


@pytest.mark.parametrize("L,d,aggr,ng,seed", [(2, 64, 0, 1, 1), (3, 128, 0, 1, 2), (2, 64, 1, 4, 3),
                                              (3, 64, 0, 3, 5), (1, 128, 1, 2, 4)])
def test_small_forward_matches_oracle_and_regular_path(L, d, aggr, ng, seed):
    c = occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr)
    if ng == 1:
        b = configs.cfg1()
    else:
        b = configs.random_dag_batch(ng, 40 + seed, max_nodes=48 // ng, hub=False)
    assert b.num_nodes <= 64 and b.num_edges <= 128
    flat = weights.unit_scale(wcfg(c), weights.init_flat(wcfg(c), seed))
    m = occu.Model(c)
    m.set_params(flat)
    m.set_small_batch_kernel(True)
    csr = occu.pack(b.graphs)
    y_small = m.predict(csr, b.node_feat, b.edge_feat)
    if m.last_launch_count() > 1:                   # too big for one CTA's shared memory: the
        assert d == 128                             # regular path ran (CFG1 at d = 64 always fits)
        return
    assert m.last_launch_count() == 1               # the whole forward in one launch
    with pytest.raises(occu.OccuError):            # no per-layer tensors on the small path
        m.get_tensor(occu.T_HBAR, 0, (b.num_nodes, d))
    r_small = m.get_tensor(occu.T_R, 0, (b.num_graphs, d))
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    ref = oracle.forward(params, ocfg(c), oracle.pack(b.graphs), b.node_feat, b.edge_feat)
    yr = ref["yhat"]
    assert np.all(np.abs(y_small - yr) <= TOL * np.maximum(np.abs(yr), 1e-2)), np.abs(y_small - yr).max()
    assert np.linalg.norm(r_small - ref["r"]) <= TOL * np.linalg.norm(ref["r"])
    m.keep_intermediates(True)                     # the regular multi-kernel path
    y_reg = m.predict(csr, b.node_feat, b.edge_feat)
    assert np.allclose(y_small, y_reg, rtol=1e-5, atol=1e-7)
    m.keep_intermediates(False)
    assert np.array_equal(m.predict(csr, b.node_feat, b.edge_feat), y_small)    # deterministic


def test_small_forward_repeatable_under_repetition():
    """Race probe for the single-CTA kernel (named-barrier row exchange between the 4 warps of
    an m-tile, cp.async staging groups, two-level readout): 300 launches on the same inputs
    must give bitwise the same outputs (compute-sanitizer is not available on this pool)."""
    import torch
    c = occu.config(L=2, F_n=80, F_e=4, d=64)
    b = configs.cfg1()
    m = occu.Model(c)
    m.init_weights(7)
    m.set_small_batch_kernel(True)
    dev = torch.device("cuda", 0)
    csr = m.to_device(occu.pack(b.graphs))
    nf = torch.from_numpy(b.node_feat).to(dev)
    ef = torch.from_numpy(b.edge_feat).to(dev)
    outs = torch.empty(300, dtype=torch.float32, device=dev)
    for i in range(300):
        m.predict(csr, nf, ef, outs[i:i + 1])
    assert m.last_launch_count() == 1
    o = outs.cpu().numpy()
    assert np.all(o == o[0]), np.unique(o)
