"""GPU parity of the Set-Transformer decoder readout (OCCU_READOUT_SET_DECODER, SURVEY §8(f)
NEXT-2, P159-P205; R30-R34) against the float64 oracle (oracle.set_decoder, pinned
against torch's nn.MultiheadAttention / nn.LayerNorm in tests/test_oracle.py).  FP32 path:
predictions and the flattened decoder output within 1e-4."""
import numpy as np
import pytest

import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu
TOL = 1e-4


def mk(L, d, k, heads, aggr=0, msg=0):
    return occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, msg=msg,
                       readout=occu.READOUT_SET_DECODER, k=k, heads=heads)


def ocfg(c):
    return dict(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr, msg=c.msg,
                slope=float(np.float32(c.slope)), readout=1, k=c.k, heads=c.heads)


def wcfg(c):
    return weights.ModelConfig(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr,
                               msg=c.msg, readout=1, k=c.k, heads=c.heads)


def rel(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    nb = np.linalg.norm(b)
    return np.linalg.norm(a - b) / (nb if nb > 0 else 1.0)


def params_for(c, seed, spread=True, wu=4.0):
    """Default init; with spread, W_u x wu (node states O(1) under reading A) and non-trivial
    LayerNorm affine parameters."""
    flat = weights.init_flat(wcfg(c), seed).copy()
    p = weights.unflatten(wcfg(c), flat)
    if spread:
        rng = np.random.default_rng(seed)
        for i in range(c.L):
            p[f"W_u{i}"] *= wu
        for m in ("M1_", "M2_"):
            for ln in ("ln1", "ln2"):
                p[m + ln + "_g"][:] = (1.0 + 0.3 * rng.standard_normal(c.d)).astype(np.float32)
                p[m + ln + "_b"][:] = (0.2 * rng.standard_normal(c.d)).astype(np.float32)
    return weights.flatten(wcfg(c), p)


@pytest.mark.parametrize("L,d,k,heads,aggr,msg", [(2, 64, 4, 4, 0, 0), (3, 128, 4, 4, 0, 0),
                                                  (3, 128, 1, 1, 1, 0), (2, 128, 2, 8, 0, 1),
                                                  (1, 64, 8, 2, 1, 0)])
def test_decoder_readout_matches_oracle(L, d, k, heads, aggr, msg):
    c = mk(L, d, k, heads, aggr, msg)
    b = configs.random_dag_batch(30, 1300 + k + heads + L, max_nodes=90, hub=True)
    b.graphs.append((1, np.zeros(0, np.int32), np.zeros(0, np.int32)))    # single-node graph
    b = configs.Batch(b.graphs, np.concatenate([b.node_feat, np.ones((1, 80), np.float32)]),
                      b.edge_feat, np.concatenate([b.targets, [0.5]]).astype(np.float32),
                      b.families + ["single"])
    flat = params_for(c, 7 + k)
    m = occu.Model(c)
    m.set_params(flat)
    m.keep_intermediates(True)
    y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    ref = oracle.forward(params, ocfg(c), oracle.pack(b.graphs), b.node_feat, b.edge_feat)
    B = b.num_graphs
    assert rel(m.get_tensor(occu.T_R, 0, (B, k * d)), ref["r"]) <= TOL
    yr = ref["yhat"]
    assert np.all(np.abs(y - yr) <= TOL * np.maximum(np.abs(yr), 1e-2)), np.abs(y - yr).max()


def test_decoder_cfg2_full_size_sampled_and_deterministic():
    c = mk(3, 128, 4, 4)
    b = configs.cfg2(256)
    flat = params_for(c, 42, spread=False)
    m = occu.Model(c)
    m.set_params(flat)
    csr = occu.pack(b.graphs)
    y1 = m.predict(csr, b.node_feat, b.edge_feat)
    y2 = m.predict(csr, b.node_feat, b.edge_feat)
    assert np.array_equal(y1, y2)
    params = oracle.unflatten(ocfg(c), flat.astype(np.float64))
    for gi in (0, 100, 255):
        s = b.subset([gi])
        yr = oracle.predict(params, ocfg(c), s.graphs, s.node_feat, s.edge_feat)
        assert abs(y1[gi] - yr[0]) <= TOL * max(abs(yr[0]), 1e-2), gi


def test_decoder_init_and_weights_file_v2(tmp_path):
    """occu_init_weights == the Python generator (LayerNorm gains 1, biases 0), and the v2
    weights file round-trips through the library and the oracle's reader."""
    c = mk(2, 64, 3, 2)
    m = occu.Model(c)
    m.init_weights(13)
    flat = weights.init_flat(wcfg(c), 13)
    assert np.array_equal(m.get_params(), flat)
    p = weights.unflatten(wcfg(c), flat)
    assert np.all(p["M1_ln1_g"] == 1.0) and np.all(p["M2_ln2_b"] == 0.0)
    path = str(tmp_path / "dec.occw")
    m.save_weights(path)
    cfg2, params = oracle.read_weights(path)
    assert cfg2["readout"] == 1 and cfg2["k"] == 3 and cfg2["heads"] == 2
    assert np.array_equal(oracle.flatten(cfg2, params), flat.astype(np.float64))
    m2 = occu.Model(c)
    m2.load_weights(path)
    assert np.array_equal(m2.get_params(), flat)


def test_decoder_errors():
    for bad in (dict(k=0, heads=4), dict(k=4, heads=3), dict(k=8, heads=4)):
        with pytest.raises(occu.OccuError):
            occu.Model(mk(2, 64, **bad))
    occu.Model(occu.config(L=2, d=64, prec=occu.BF16, readout=occu.READOUT_SET_DECODER))   # R41
    c = mk(2, 64, 2, 2)
    m = occu.Model(c)
    m.init_weights(1)
    with pytest.raises(occu.OccuError):
        m.set_kernel_path(1)
    b = configs.random_dag_batch(3, 5, max_nodes=10)
    mb = occu.Model(occu.config(L=2, d=64, prec=occu.BF16, readout=occu.READOUT_SET_DECODER))
    mb.init_weights(1)
    with pytest.raises(occu.OccuError):          # training through the stack: OCCU_FP32 only
        mb.train_step(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets, 1e-4)


# ---------------------------------------------------------------- training (NEXT-2)
def _train_cfg(L, d, k, heads, aggr, G):
    return occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, readout=occu.READOUT_SET_DECODER, k=k,
                       heads=heads, graphormer=G)


def _ocfg_g(c):
    o = ocfg(c)
    o["graphormer"] = c.graphormer
    return o


def _wcfg_g(c):
    return weights.ModelConfig(L=c.L, F_n=c.F_n, F_e=c.F_e, d=c.d, d_h=c.d_h, aggr=c.aggr,
                               readout=1, k=c.k, heads=c.heads, graphormer=c.graphormer)


@pytest.mark.parametrize("L,d,k,heads,aggr,G", [(2, 64, 4, 4, 0, 0), (3, 128, 4, 4, 0, 0),
                                                (2, 128, 2, 8, 1, 0), (1, 64, 1, 1, 0, 0),
                                                (2, 128, 4, 4, 0, 2)])
def test_decoder_training_gradients_match_oracle(L, d, k, heads, aggr, G):
    """Training through the Set-Transformer decoder readout (P159-P205, P273's Adam) and, in the
    last case, the paper's full stack ANEE -> Graphormer x2 -> decoder -> head: the loss and every
    per-tensor gradient against the float64 oracle's hand-derived backward, rel-L2 <= 1e-4, at a
    well-conditioned weight scale (W_u x 32, R45)."""
    c = _train_cfg(L, d, k, heads, aggr, G)
    b = configs.random_dag_batch(24, 1500 + k + heads + L + G, max_nodes=90, hub=True)
    b.graphs.append((1, np.zeros(0, np.int32), np.zeros(0, np.int32)))    # single-node graph
    b = configs.Batch(b.graphs, np.concatenate([b.node_feat, np.ones((1, 80), np.float32)]),
                      b.edge_feat, np.concatenate([b.targets, [0.5]]).astype(np.float32),
                      b.families + ["single"])
    wc = _wcfg_g(c)
    p = weights.unflatten(wc, weights.init_flat(wc, 60 + k).copy())
    rng = np.random.default_rng(60 + k)
    for i in range(L):
        p[f"W_u{i}"] *= 32.0
    for m in ["M1_", "M2_"] + [f"G{j}_" for j in range(G)]:
        for ln in ("ln1", "ln2"):
            p[m + ln + "_g"][:] = (1.0 + 0.3 * rng.standard_normal(d)).astype(np.float32)
            p[m + ln + "_b"][:] = (0.2 * rng.standard_normal(d)).astype(np.float32)
    flat = weights.flatten(wc, p)
    m = occu.Model(c)
    m.set_params(flat)
    loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets,
                           global_num_graphs=40)
    g = weights.unflatten(wc, m.get_grads())
    params = oracle.unflatten(_ocfg_g(c), flat.astype(np.float64))
    lref, gref = oracle.loss_and_grads(params, _ocfg_g(c), b.graphs, b.node_feat, b.edge_feat,
                                       b.targets, global_batch=40)
    assert abs(loss - lref) <= TOL * abs(lref)
    # key biases get exactly zero gradient (softmax shift invariance): noise on both sides
    zero = {kk for kk in gref if kk.endswith("_bk")}
    for kk in zero:
        scale = max(np.linalg.norm(gref[kk[:-2] + w]) for w in ("Wq", "Wk", "Wv", "Wo"))
        assert np.linalg.norm(g[kk]) <= TOL * scale, kk
    bad = {kk: rel(g[kk], gref[kk]) for kk in gref if kk not in zero and rel(g[kk], gref[kk]) > TOL}
    assert not bad, bad


def test_decoder_training_trajectory():
    """Ten Adam steps through the decoder readout track the oracle's loss trajectory."""
    c = _train_cfg(2, 64, 4, 4, 0, 0)
    b = configs.random_dag_batch(12, 1600, max_nodes=40, hub=True)
    flat = params_for(c, 61, wu=32.0)
    m = occu.Model(c)
    m.set_params(flat)
    csr = occu.pack(b.graphs)
    params = oracle.unflatten(_ocfg_g(c), flat.astype(np.float64))
    st = {}
    for step in range(10):
        loss = m.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-3)
        lref, gref = oracle.loss_and_grads(params, _ocfg_g(c), b.graphs, b.node_feat, b.edge_feat, b.targets)
        params, st = oracle.adam_step(params, gref, st, 1e-3)
        assert abs(loss - lref) <= TOL * abs(lref) + 1e-7, (step, loss, lref)
