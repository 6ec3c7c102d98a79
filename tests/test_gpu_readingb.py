"""GPU parity of ANEE reading B (OCCU_MSG_NEIGHBOR_SOFTMAX; R4):
the P149 softmax taken per channel over the in-edges of the destination instead of over the
channels.  The CUDA path (logits W_m e' on tensor cores, then one segmented online-softmax
aggregation pass; training keeps the weights and uses the closed-form segmented softmax
backward) against the float64 oracle's reading-B forward / backward (oracle.anee_layer /
oracle.backward with msg = 1, pinned by finite differences and the chain closed form in
tests/test_oracle.py).  FP32 tolerances as the reading-A path (R23)."""
import numpy as np
import pytest

import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu
TOL = 1e-4
GRAD_TOL = 1e-4
MSGB = occu.MSG_NEIGHBOR_SOFTMAX


def mk(L, d, aggr=0, F_n=80, F_e=4):
    return occu.config(L=L, F_n=F_n, F_e=F_e, d=d, aggr=aggr, msg=MSGB)


def ocfg(c):
    return dict(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg,
                slope=float(np.float32(c.slope)))


def wcfg(c):
    return weights.ModelConfig(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg)


def rel(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 0 else 1.0)


def wset(c, seed, kind):
    flat = weights.init_flat(wcfg(c), seed)
    if kind == "wide":      # larger logits: the in-edge softmax is far from uniform
        flat = flat.copy()
        L = oracle.param_shapes(ocfg(c))
        off = 0
        for name, shape in L:
            n = int(np.prod(shape))
            if name.startswith("W_m") or name.startswith("a_"):
                flat[off:off + n] *= 8.0
            off += n
    return flat


@pytest.mark.parametrize("kind", ["default", "wide"])
@pytest.mark.parametrize("L,d,aggr,seed", [(2, 64, 0, 1), (3, 128, 0, 2), (3, 128, 1, 3), (1, 64, 1, 4)])
def test_readingb_all_intermediates(L, d, aggr, seed, kind):
    c = mk(L, d, aggr)
    b = configs.random_dag_batch(40, 900 + seed, max_nodes=60, hub=True)
    flat = wset(c, seed, kind)
    m = occu.Model(c)
    m.set_params(flat)
    m.keep_intermediates(True)
    y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    ref = oracle.forward(params, ocfg(c), pk, b.node_feat, b.edge_feat)
    N, E, B = pk["num_nodes"], pk["num_edges"], pk["num_graphs"]
    for i in range(L):
        lay = ref["layers"][i]
        for t, k, shp in ((occu.T_HBAR, "hbar", (N, d)), (occu.T_P, "p", (N,)), (occu.T_Q, "q", (N,)),
                          (occu.T_E, "e", (E, d)), (occu.T_H, "h", (N, d))):
            assert rel(m.get_tensor(t, i, shp), lay[k]) <= TOL, (k, i, rel(m.get_tensor(t, i, shp), lay[k]))
    assert rel(m.get_tensor(occu.T_R, 0, (B, d)), ref["r"]) <= TOL
    yr = ref["yhat"]
    assert np.all(np.abs(y - yr) <= TOL * np.maximum(np.abs(yr), 1e-2)), np.abs(y - yr).max()


def test_readingb_single_in_edge_closed_form():
    """A node with one in-edge has w ≡ 1, so h_t = LReLU(h̄_src) exactly (bitwise against the
    path's own h̄); sources give 0 (SURVEY §8(f) NEXT-1 pin)."""
    c = mk(2, 64)
    chain = [(6, np.array([0, 1, 2, 3, 4], np.int32), np.array([1, 2, 3, 4, 5], np.int32))]
    rng = np.random.default_rng(5)
    nf = rng.normal(size=(6, 80)).astype(np.float32)
    ef = rng.uniform(size=(5, 4)).astype(np.float32)
    m = occu.Model(c)
    m.set_params(wset(c, 3, "wide"))
    m.keep_intermediates(True)
    m.predict(occu.pack(chain), nf, ef)
    for i in range(2):
        hb = m.get_tensor(occu.T_HBAR, i, (6, 64))
        h = m.get_tensor(occu.T_H, i, (6, 64))
        want = np.where(hb[:-1] > 0, hb[:-1], np.float32(0.01) * hb[:-1]).astype(np.float32)
        assert np.array_equal(h[1:], want), i
        assert np.array_equal(h[0], np.zeros(64, np.float32))


@pytest.mark.parametrize("L,d,aggr", [(2, 64, 0), (3, 128, 0), (3, 128, 1)])
def test_readingb_gradients_match_oracle(L, d, aggr):
    c = mk(L, d, aggr)
    b = configs.random_dag_batch(24, 950 + L + aggr, max_nodes=50, hub=True)
    flat = wset(c, 11, "wide")
    m = occu.Model(c)
    m.set_params(flat)
    loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets)
    g = weights.unflatten(wcfg(c), m.get_grads())
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    lref, gref = oracle.loss_and_grads(params, ocfg(c), b.graphs, b.node_feat, b.edge_feat, b.targets)
    assert abs(loss - lref) <= TOL * abs(lref)
    for k in gref:
        assert rel(g[k], gref[k]) <= GRAD_TOL, (k, rel(g[k], gref[k]))


def test_readingb_cfg2_full_size_sampled_and_deterministic():
    """CFG2 at full size (256 ResNet-50 graphs) under reading B: sampled graphs vs the oracle
    one by one (batching invariance at the same time) and bitwise-identical reruns."""
    c = mk(3, 128)
    b = configs.cfg2(256)
    flat = wset(c, 42, "default")
    m = occu.Model(c)
    m.set_params(flat)
    csr = occu.pack(b.graphs)
    y1 = m.predict(csr, b.node_feat, b.edge_feat)
    y2 = m.predict(csr, b.node_feat, b.edge_feat)
    assert np.array_equal(y1, y2)
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    for gi in (0, 77, 255):
        s = b.subset([gi])
        yr = oracle.predict(params, ocfg(c), s.graphs, s.node_feat, s.edge_feat)
        assert abs(y1[gi] - yr[0]) <= TOL * max(abs(yr[0]), 1e-2), gi


def test_readingb_training_trajectory():
    c = mk(2, 64)
    b = configs.random_dag_batch(16, 990, max_nodes=40, hub=True)
    flat = wset(c, 12, "wide")
    m = occu.Model(c)
    m.set_params(flat)
    csr = occu.pack(b.graphs)
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    st, lr = {}, 1e-3
    for step in range(10):
        loss = m.train_step(csr, b.node_feat, b.edge_feat, b.targets, lr)
        lref, gref = oracle.loss_and_grads(params, ocfg(c), b.graphs, b.node_feat, b.edge_feat, b.targets)
        params, st = oracle.adam_step(params, gref, st, lr)
        assert abs(loss - lref) <= TOL * abs(lref) + 1e-7, (step, loss, lref)


def test_readingb_errors():
    occu.Model(occu.config(L=2, d=64, msg=MSGB, prec=occu.BF16))      # valid since R40 (inference)
    with pytest.raises(occu.OccuError):
        occu.Model(occu.config(L=2, F_n=200, d=64, msg=MSGB))
    m = occu.Model(mk(2, 64))
    with pytest.raises(occu.OccuError):
        m.set_kernel_path(1)


# ------------------------------------------ reading B in OCCU_BF16 (R40), inference
def _mkb(L, d, aggr=0):
    return occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, prec=occu.BF16,
                       msg=occu.MSG_NEIGHBOR_SOFTMAX)


def _ocfgb(c):
    return dict(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg,
                slope=float(np.float32(c.slope)))


def _wcfgb(c):
    return weights.ModelConfig(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg)


def _relb(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 0 else 1.0)


@pytest.mark.parametrize("L,d,aggr,seed", [(2, 64, 0, 1), (3, 128, 0, 2), (3, 128, 1, 3)])
def test_readingb_bf16_intermediates_and_predictions(L, d, aggr, seed):
    """Every intermediate vs oracle.forward_bf16 (the mode's roundings in float64) at 3e-3,
    ŷ vs the float64 oracle at the BF16 criterion (rel-L2 <= 1e-2, per graph
    1e-2·max(|ŷ|, 0.1), R25)."""
    c = _mkb(L, d, aggr)
    b = configs.random_dag_batch(40, 700 + seed, max_nodes=60, hub=True)
    flat = weights.init_flat(_wcfgb(c), seed)
    m = occu.Model(c)
    m.set_params(flat)
    m.keep_intermediates(True)
    y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
    params = oracle.unflatten(_ocfgb(c), flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    emu = oracle.forward_bf16(params, _ocfgb(c), pk, b.node_feat, b.edge_feat)
    ref = oracle.forward(params, _ocfgb(c), pk, b.node_feat, b.edge_feat)
    N, E, B = pk["num_nodes"], pk["num_edges"], pk["num_graphs"]
    for i in range(L):
        lay = emu["layers"][i]
        assert _relb(m.get_tensor(occu.T_HBAR, i, (N, d)), lay["hbar"]) <= 3e-3, ("hbar", i)
        assert _relb(m.get_tensor(occu.T_E, i, (E, d)), lay["e"]) <= 3e-3, ("e", i)
        assert _relb(m.get_tensor(occu.T_H, i, (N, d)), lay["h"]) <= 3e-3, ("h", i)
    assert _relb(m.get_tensor(occu.T_R, 0, (B, d)), emu["r"]) <= 3e-3
    yr = ref["yhat"]
    assert _relb(y, yr) <= 1e-2
    assert np.all(np.abs(y - yr) <= 1e-2 * np.maximum(np.abs(yr), 0.1)), np.abs(y - yr).max()


def test_readingb_bf16_cfg2_sampled_and_training_rejected():
    c = _mkb(3, 128)
    b = configs.cfg2(256)
    flat = weights.init_flat(_wcfgb(c), 42)
    m = occu.Model(c)
    m.set_params(flat)
    csr = occu.pack(b.graphs)
    y1 = m.predict(csr, b.node_feat, b.edge_feat)
    assert np.array_equal(y1, m.predict(csr, b.node_feat, b.edge_feat))
    params = oracle.unflatten(_ocfgb(c), flat.astype(np.float64))
    for gi in (0, 131, 255):
        s = b.subset([gi])
        yr = oracle.predict(params, _ocfgb(c), s.graphs, s.node_feat, s.edge_feat)
        assert abs(y1[gi] - yr[0]) <= 1e-2 * max(abs(yr[0]), 0.1), gi
    with pytest.raises(occu.OccuError):
        m.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-4)
