"""Pins for the CPU oracle (oracle/occu_oracle.py) — things fixed by the paper's
equations and by mathematics, not by the oracle itself.

* T1/T2/T3: toy DAGs worked out by hand from P141-P149 (derivations inline,
  expected decimals also in tests/golden/toy_examples.json).
* closed forms: a = 0 => e ≡ σ(0) = 1/2; W_m = 0 => g ≡ 1/d; path counts
  H^i = (A^T)^i X / d^i; d = 1 => ŷ independent of edge data; sources => 0;
  W_u = 0 => head closed form; reading B on chains => LReLU(h̄_src).
* invariances: node relabelling, batching, DP sharding of gradients.
* backward: central finite differences (float64) and an independent torch
  autograd implementation of the same forward.
* Adam: first-step closed form and torch.optim.Adam trajectory.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from occu_gen import configs, dags, weights

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "toy_examples.json")


def cfg_dict(L=1, F_n=2, F_e=2, d=2, d_h=2, aggr=0, msg=0, slope=0.01):
    return dict(L=L, F_n=F_n, F_e=F_e, d=d, d_h=d_h, aggr=aggr, msg=msg, slope=slope)


def toy_params(cfg, **over):
    p = {}
    for name, shape in oracle.param_shapes(cfg):
        p[name] = np.zeros(shape)
    p.update(over)
    return p


def sig(x):
    return 1.0 / (1.0 + math.exp(-x))


CHAIN = [(3, np.array([0, 1], np.int32), np.array([1, 2], np.int32))]
X_T1 = np.array([[1, 2], [3, 4], [5, 6]], np.float64)
EF_T1 = np.array([[0.1, 0.2], [0.3, 0.4]], np.float64)


def t1_params(cfg):
    return toy_params(cfg, W_u0=np.eye(2), W_e0=np.eye(2), W_m0=np.array([[1., 0.], [0., 0.]]),
                      W_1=np.eye(2), w_2=np.array([1., 1.]))


# ---------------------------------------------------------------- toy DAGs
def test_T1_chain_alpha_zero():
    cfg = cfg_dict()
    f = oracle.forward(t1_params(cfg), cfg, oracle.pack(CHAIN), X_T1, EF_T1)
    lay = f["layers"][0]
    # a = 0 -> α = 0 -> e = σ(0) = 1/2 on every channel (P145)
    assert np.array_equal(lay["e"], np.full((2, 2), 0.5))
    # W_m e = (1/2, 0) -> channel softmax = (σ(1/2), 1 - σ(1/2))  (P149 reading A)
    g0 = sig(0.5)
    assert np.allclose(lay["g"], [[g0, 1 - g0], [g0, 1 - g0]], rtol=0, atol=1e-15)
    # node 0 has no in-edge -> 0; node1 <- g ⊙ h̄0; node2 <- g ⊙ h̄1 (all positive)
    h1 = np.array([[0, 0], [g0 * 1, (1 - g0) * 2], [g0 * 3, (1 - g0) * 4]])
    assert np.allclose(lay["h"], h1, rtol=0, atol=1e-15)
    r = h1.mean(axis=0)
    assert np.allclose(f["r"][0], r, atol=1e-15)
    assert abs(f["yhat"][0] - r.sum()) < 1e-14
    gold = json.load(open(GOLDEN))["T1"]
    assert abs(f["yhat"][0] - gold["yhat"]) < 1e-9
    assert np.allclose(lay["h"], gold["h1"], atol=1e-9)


def test_T2_chain_alpha_nonzero():
    cfg = cfg_dict()
    p = t1_params(cfg)
    p.update(a_s0=np.array([1., 0.]), a_d0=np.array([0., 1.]), W_m0=np.eye(2))
    f = oracle.forward(p, cfg, oracle.pack(CHAIN), X_T1, EF_T1)
    lay = f["layers"][0]
    # p = h̄[:,0] = (1,3,5), q = h̄[:,1] = (2,4,6); α(0->1) = 1+4, α(1->2) = 3+6
    assert np.array_equal(lay["alpha"], [5.0, 9.0])
    e = np.array([[sig(0.5), sig(1.0)], [sig(2.7), sig(3.6)]])
    assert np.allclose(lay["e"], e, atol=1e-15)
    # 2-channel softmax of (x, y) = (σ(x - y), σ(y - x))
    g = np.array([[sig(e[0, 0] - e[0, 1]), sig(e[0, 1] - e[0, 0])],
                  [sig(e[1, 0] - e[1, 1]), sig(e[1, 1] - e[1, 0])]])
    h1 = np.array([[0, 0], [g[0, 0] * 1, g[0, 1] * 2], [g[1, 0] * 3, g[1, 1] * 4]])
    assert np.allclose(lay["h"], h1, atol=1e-14)
    gold = json.load(open(GOLDEN))["T2"]
    assert abs(f["yhat"][0] - gold["yhat"]) < 1e-9
    assert np.allclose(lay["h"], gold["h1"], atol=1e-9)


def test_T3_diamond_path_counts():
    cfg = cfg_dict(L=2)
    g = [(4, np.array([0, 0, 1, 2], np.int32), np.array([1, 2, 3, 3], np.int32))]
    X = np.array([[1, 1], [0, 0], [0, 0], [0, 0]], np.float64)
    p = toy_params(cfg, W_u0=np.eye(2), W_u1=np.eye(2), W_1=np.eye(2), w_2=np.ones(2))
    f = oracle.forward(p, cfg, oracle.pack(g), X, np.zeros((4, 2)))
    assert np.array_equal(f["layers"][0]["h"], [[0, 0], [.5, .5], [.5, .5], [0, 0]])
    assert np.array_equal(f["layers"][1]["h"], [[0, 0], [0, 0], [0, 0], [.5, .5]])


def test_batching_T1_plus_pair():
    g2 = (2, np.array([0], np.int32), np.array([1], np.int32))
    pk = oracle.pack(CHAIN + [g2])
    assert pk["node_off"].tolist() == [0, 3, 5]
    assert pk["edge_off"].tolist() == [0, 2, 3]
    cfg = cfg_dict()
    X = np.vstack([X_T1, [[7, 8], [9, 10]]])
    EF = np.vstack([EF_T1, [[0.5, 0.6]]])
    yb = oracle.forward(t1_params(cfg), cfg, pk, X, EF)["yhat"]
    y1 = oracle.forward(t1_params(cfg), cfg, oracle.pack(CHAIN), X_T1, EF_T1)["yhat"]
    assert yb[0] == y1[0]


# ---------------------------------------------------------------- pack
def brute_pack_check(graphs, pk):
    N, E = pk["num_nodes"], pk["num_edges"]
    src, dst = [], []
    off = 0
    for n, s, t in graphs:
        src += (np.asarray(s) + off).tolist()
        dst += (np.asarray(t) + off).tolist()
        off += n
    trip = sorted(zip(dst, src, range(E)))
    assert pk["in_dst"].tolist() == [t for t, _, _ in trip]
    assert pk["in_src"].tolist() == [s for _, s, _ in trip]
    assert pk["in_eid"].tolist() == [e for _, _, e in trip]
    for v in range(N + 1):
        assert pk["in_ptr"][v] == sum(1 for t in dst if t < v)
        assert pk["out_ptr"][v] == sum(1 for s in src if s < v)
    otrip = sorted(zip(src, dst, range(E)))
    for j, (s, t, e) in enumerate(otrip):
        k = pk["out_pos"][j]
        assert pk["in_eid"][k] == e and pk["in_src"][k] == s and pk["in_dst"][k] == t
    assert sorted(pk["out_pos"].tolist()) == list(range(E))
    ng = []
    for b, (n, _, _) in enumerate(graphs):
        ng += [b] * n
    assert pk["node_graph"].tolist() == ng


@pytest.mark.parametrize("seed", range(6))
def test_pack_brute_force(seed):
    b = configs.random_dag_batch(7, seed, max_nodes=9, hub=(seed % 2 == 1))
    # add a multi-edge and an edgeless graph
    graphs = b.graphs + [(3, np.array([0, 0, 1], np.int32), np.array([2, 2, 2], np.int32)),
                         (1, np.zeros(0, np.int32), np.zeros(0, np.int32))]
    pk = oracle.pack(graphs)
    brute_pack_check(graphs, pk)
    for k in ("in_ptr", "in_src", "in_eid", "out_ptr", "out_pos", "node_off"):
        assert pk[k].dtype == np.int32


# ---------------------------------------------------------------- closed forms
def rand_params(cfg, seed, scale=1.0):
    c = weights.ModelConfig(L=cfg["L"], F_n=cfg["F_n"], F_e=cfg["F_e"], d=cfg["d"],
                            d_h=cfg["d_h"], aggr=cfg["aggr"], msg=cfg["msg"])
    flat = weights.init_flat(c, seed).astype(np.float64) * scale
    return oracle.unflatten(cfg, flat)


@pytest.mark.parametrize("seed", range(4))
def test_path_count_closed_form(seed):
    """W_u = I (F_n = d), a = 0, W_m = 0, SUM, X >= 0:  H^i = (A^T)^i X / d^i."""
    d, L = 4, 3
    cfg = cfg_dict(L=L, F_n=d, F_e=3, d=d, d_h=d)
    b = configs.random_dag_batch(3, 100 + seed, max_nodes=10, f_n=d, f_e=3, hub=True)
    X = np.floor(b.node_feat.astype(np.float64) * 8)
    p = rand_params(cfg, seed)
    for i in range(L):
        p[f"W_u{i}"] = np.eye(d)
        p[f"a_s{i}"] = np.zeros(d)
        p[f"a_d{i}"] = np.zeros(d)
        p[f"W_m{i}"] = np.zeros((d, d))
    pk = oracle.pack(b.graphs)
    f = oracle.forward(p, cfg, pk, X, b.edge_feat)
    N = pk["num_nodes"]
    # brute-force path counts: paths[i][u][v] = # length-i paths u -> v
    adj = np.zeros((N, N), np.int64)
    for s, t in zip(pk["in_src"], pk["in_dst"]):
        adj[s, t] += 1
    cnt = np.eye(N, dtype=np.int64)
    for i in range(L):
        cnt = cnt @ adj
        expect = cnt.T.astype(np.float64) @ X / d ** (i + 1)
        assert np.array_equal(f["layers"][i]["h"], expect)
        assert np.array_equal(f["layers"][i]["e"], np.full((pk["num_edges"], d), 0.5))
        assert np.array_equal(f["layers"][i]["g"], np.full((pk["num_edges"], d), 1.0 / d))


def test_sources_are_zero_and_d1_independent_of_edges():
    cfg = cfg_dict(L=2, F_n=5, F_e=3, d=1, d_h=3)
    b = configs.random_dag_batch(5, 9, f_n=5, f_e=3)
    p = rand_params(cfg, 3, scale=3.0)
    pk = oracle.pack(b.graphs)
    f1 = oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)
    f2 = oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat * 5.0 + 1.0)
    assert np.array_equal(f1["yhat"], f2["yhat"])           # softmax of 1 element is 1
    deg = np.diff(pk["in_ptr"])
    for lay in f1["layers"]:
        assert (lay["h"][deg == 0] == 0).all()


def test_head_closed_form_when_W_u_zero():
    cfg = cfg_dict(L=2, F_n=6, F_e=4, d=4, d_h=3)
    b = configs.random_dag_batch(4, 2, f_n=6, f_e=4)
    p = rand_params(cfg, 5)
    p["W_u0"] = np.zeros_like(p["W_u0"])
    p["W_u1"] = np.zeros_like(p["W_u1"])
    f = oracle.forward(p, cfg, oracle.pack(b.graphs), b.node_feat, b.edge_feat)
    b1 = p["b_1"]
    o = np.where(b1 > 0, b1, 0.01 * b1)
    assert np.allclose(f["yhat"], o @ p["w_2"] + p["b_2"][0], rtol=0, atol=1e-15)


def test_mean_equals_sum_on_chains_and_halves_diamond():
    cfg_s = cfg_dict(L=2, F_n=3, F_e=2, d=3, d_h=2)
    cfg_m = dict(cfg_s, aggr=oracle.AGGR_MEAN)
    chain = [(5, np.arange(4, dtype=np.int32), np.arange(1, 5, dtype=np.int32))]
    X = np.arange(15, dtype=np.float64).reshape(5, 3) / 7
    EF = np.arange(8, dtype=np.float64).reshape(4, 2) / 5
    p = rand_params(cfg_s, 4, 2.0)
    ys = oracle.forward(p, cfg_s, oracle.pack(chain), X, EF)["yhat"]
    ym = oracle.forward(p, cfg_m, oracle.pack(chain), X, EF)["yhat"]
    assert np.array_equal(ys, ym)
    cfg = cfg_dict(L=2, aggr=oracle.AGGR_MEAN)
    g = [(4, np.array([0, 0, 1, 2], np.int32), np.array([1, 2, 3, 3], np.int32))]
    X = np.array([[1, 1], [0, 0], [0, 0], [0, 0]], np.float64)
    pp = toy_params(cfg, W_u0=np.eye(2), W_u1=np.eye(2))
    f = oracle.forward(pp, cfg, oracle.pack(g), X, np.zeros((4, 2)))
    assert np.array_equal(f["layers"][1]["h"][3], [.25, .25])   # mean of two (.25,.25)


def test_reading_B_chain_closed_form():
    """NEXT-1 reading B: a single in-edge has weight 1 => h_t = LReLU(h̄_src)."""
    cfg = cfg_dict(L=1, F_n=3, F_e=2, d=4, d_h=2, msg=oracle.MSG_NEIGHBOR_SOFTMAX)
    chain = [(4, np.arange(3, dtype=np.int32), np.arange(1, 4, dtype=np.int32))]
    X = np.arange(12, dtype=np.float64).reshape(4, 3) / 5 - 1
    p = rand_params(cfg, 8, 3.0)
    lay = oracle.forward(p, cfg, oracle.pack(chain), X, np.ones((3, 2)))["layers"][0]
    hb = lay["hbar"]
    expect = np.vstack([np.zeros(4), np.where(hb[:3] > 0, hb[:3], 0.01 * hb[:3])])
    assert np.allclose(lay["h"], expect, rtol=0, atol=1e-15)


# ---------------------------------------------------------------- invariances
@pytest.mark.parametrize("msg", [0, 1])
def test_node_permutation_invariance(msg):
    cfg = cfg_dict(L=3, F_n=80, F_e=4, d=16, d_h=16, msg=msg)
    b = configs.random_dag_batch(4, 21, max_nodes=15, hub=True)
    p = rand_params(cfg, 11)
    for i in range(3):
        p[f"W_u{i}"] *= 16
    y0 = oracle.predict(p, cfg, b.graphs, b.node_feat, b.edge_feat)
    from occu_gen.prng import Rng
    r = Rng(77)
    graphs, feats = [], []
    off = 0
    for (n, s, t) in b.graphs:
        perm = r.permutation(n)
        inv = np.argsort(perm)
        graphs.append((n, perm[s].astype(np.int32), perm[t].astype(np.int32)))
        feats.append(b.node_feat[off:off + n][inv])
        off += n
    y1 = oracle.predict(p, cfg, graphs, np.vstack(feats), b.edge_feat)
    assert np.allclose(y0, y1, rtol=1e-12, atol=0)


def test_batching_invariance_bitwise():
    cfg = cfg_dict(L=3, F_n=80, F_e=4, d=8, d_h=8)
    b = configs.random_dag_batch(6, 31, max_nodes=12, hub=True)
    p = rand_params(cfg, 2)
    yb = oracle.predict(p, cfg, b.graphs, b.node_feat, b.edge_feat)
    for i in range(b.num_graphs):
        s = b.subset([i])
        yi = oracle.predict(p, cfg, s.graphs, s.node_feat, s.edge_feat)
        assert np.allclose(yi[0], yb[i], rtol=1e-13, atol=1e-15)


# ---------------------------------------------------------------- backward
def fd_check(cfg, b, p, names=None, eps_rel=1e-5, tol=2e-6, gb=None):
    """Central differences.  Bound: truncation O(h^2) (relative tol) plus the
    round-off of differencing two float64 losses, ~eps_mach*|loss|/h per entry."""
    pk = oracle.pack(b.graphs)
    loss, grads = oracle.backward(p, cfg, pk, oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat),
                                  b.targets, gb)
    names = names or list(p)
    for name in names:
        w = p[name]
        flat = w.ravel()
        num = np.zeros_like(flat)
        hmin = np.inf
        for j in range(flat.size):
            h = eps_rel * max(1.0, abs(flat[j]))
            hmin = min(hmin, h)
            old = flat[j]
            flat[j] = old + h
            lp = oracle.mse_loss(oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)["yhat"], b.targets, gb)
            flat[j] = old - h
            lm = oracle.mse_loss(oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)["yhat"], b.targets, gb)
            flat[j] = old
            num[j] = (lp - lm) / (2 * h)
        an = grads[name].ravel()
        roundoff = 50 * np.finfo(np.float64).eps * abs(loss) / hmin * np.sqrt(flat.size)
        err = np.linalg.norm(an - num)
        assert err <= tol * np.linalg.norm(num) + roundoff, (name, err, np.linalg.norm(num), roundoff)
        # the gradient must not be vacuous for the weights that matter
    assert any(np.linalg.norm(grads[n]) > 1e-3 for n in names)


@pytest.mark.parametrize("d,L,aggr,msg", [(2, 1, 0, 0), (4, 2, 0, 0), (4, 2, 1, 0), (3, 2, 0, 1)])
def test_backward_finite_differences(d, L, aggr, msg):
    cfg = cfg_dict(L=L, F_n=5, F_e=3, d=d, d_h=3, aggr=aggr, msg=msg)
    b = configs.random_dag_batch(3, 40 + d, max_nodes=7, f_n=5, f_e=3, hub=True)
    p = rand_params(cfg, 6, scale=2.0)
    for i in range(L):
        p[f"W_u{i}"] *= d
    fd_check(cfg, b, p, tol=2e-6)


def torch_forward_loss(p, cfg, pk, X, EF, y):
    torch = pytest.importorskip("torch")
    T = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in p.items()}
    s = torch.tensor(pk["in_src"].astype(np.int64))
    t = torch.tensor(pk["in_dst"].astype(np.int64))
    h = torch.tensor(X, dtype=torch.float64)
    e = torch.tensor(EF, dtype=torch.float64)[torch.tensor(pk["in_eid"].astype(np.int64))]
    lrelu = lambda x: torch.nn.functional.leaky_relu(x, cfg["slope"])
    N = pk["num_nodes"]
    for i in range(cfg["L"]):
        hb = lrelu(h @ T[f"W_u{i}"].T)
        al = hb[s] @ T[f"a_s{i}"] + hb[t] @ T[f"a_d{i}"]
        e = torch.sigmoid(al[:, None] * (e @ T[f"W_e{i}"].T))
        g = torch.softmax(e @ T[f"W_m{i}"].T, dim=1)
        A = torch.zeros(N, hb.shape[1], dtype=torch.float64).index_add(0, t, g * hb[s])
        if cfg["aggr"] == 1:
            A = A / torch.tensor(np.maximum(np.diff(pk["in_ptr"]), 1), dtype=torch.float64)[:, None]
        h = lrelu(A)
        ng = torch.tensor(pk["node_graph"].astype(np.int64))
    nb = torch.tensor(np.diff(pk["node_off"]).astype(np.float64))
    r = torch.zeros(pk["num_graphs"], h.shape[1], dtype=torch.float64).index_add(0, ng, h) / nb[:, None]
    yh = lrelu(r @ T["W_1"].T + T["b_1"]) @ T["w_2"] + T["b_2"][0]
    loss = ((yh - torch.tensor(y, dtype=torch.float64)) ** 2).sum() / len(y)
    loss.backward()
    return float(loss), {k: v.grad.numpy() for k, v in T.items()}


@pytest.mark.parametrize("aggr", [0, 1])
def test_backward_matches_torch_autograd(aggr):
    cfg = cfg_dict(L=3, F_n=80, F_e=4, d=16, d_h=8, aggr=aggr)
    b = configs.random_dag_batch(5, 50, max_nodes=14, hub=True)
    p = rand_params(cfg, 13)
    for i in range(3):
        p[f"W_u{i}"] *= 16
    pk = oracle.pack(b.graphs)
    loss, grads = oracle.backward(p, cfg, pk, oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat),
                                  b.targets)
    tl, tg = torch_forward_loss(p, cfg, pk, b.node_feat, b.edge_feat, b.targets)
    assert abs(loss - tl) <= 1e-12 * abs(tl)
    for k in p:
        assert np.allclose(grads[k], tg[k], rtol=1e-9, atol=1e-14 * max(1, np.abs(tg[k]).max())), k


def test_dp_shard_gradients_sum_to_full_batch():
    cfg = cfg_dict(L=2, F_n=80, F_e=4, d=8, d_h=8)
    b = configs.random_dag_batch(8, 60, max_nodes=10)
    p = rand_params(cfg, 17)
    B = b.num_graphs
    _, g_full = oracle.loss_and_grads(p, cfg, b.graphs, b.node_feat, b.edge_feat, b.targets)
    acc = {k: np.zeros_like(v) for k, v in p.items()}
    for shard in ([0, 3, 5], [1, 2], [4, 6, 7]):
        s = b.subset(shard)
        _, gs = oracle.loss_and_grads(p, cfg, s.graphs, s.node_feat, s.edge_feat, s.targets, B)
        for k in acc:
            acc[k] += gs[k]
    for k in p:
        assert np.allclose(acc[k], g_full[k], rtol=1e-12, atol=1e-16), k


# ---------------------------------------------------------------- Adam
def test_adam_first_step_closed_form():
    rng = np.random.default_rng(0)
    p = {"w": rng.normal(size=20)}
    g = {"w": rng.normal(size=20) * 1e-3}
    lr, wd, eps = 1e-4, 1e-4, 1e-8
    newp, st = oracle.adam_step(p, g, {}, lr, wd)
    gh = g["w"] + wd * p["w"]
    assert np.allclose(newp["w"], p["w"] - lr * gh / (np.abs(gh) + eps), rtol=0, atol=1e-15)
    assert st["t"] == 1


def test_adam_matches_torch_optim():
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(1)
    w0 = rng.normal(size=(5, 3))
    grads = [rng.normal(size=(5, 3)) for _ in range(6)]
    tw = torch.tensor(w0, dtype=torch.float64, requires_grad=True)
    opt = torch.optim.Adam([tw], lr=1e-3, weight_decay=1e-4)
    p, st = {"w": w0.copy()}, {}
    for g in grads:
        tw.grad = torch.tensor(g, dtype=torch.float64)
        opt.step()
        p, st = oracle.adam_step(p, {"w": g}, st, 1e-3, 1e-4)
    assert np.allclose(p["w"], tw.detach().numpy(), rtol=1e-12, atol=1e-15)


# ------------------------------------------------ OCCU_BF16 emulation (R24-R27)
def test_bf16_round_ties_and_library():
    """bf16_round = round-to-nearest-even to 8 significant bits: hand-worked ties and
    torch's own float32 -> bfloat16 conversion (an independent library routine)."""
    import torch
    r = oracle.bf16_round
    assert r(1.0) == 1.0
    assert r(1 + 2 ** -8) == 1.0                        # tie -> even mantissa (1.0)
    assert r(1 + 3 * 2 ** -8) == 1 + 2 ** -6            # tie between 1+2^-7 (odd) and 1+2^-6
    assert r(1 + 2 ** -8 + 2 ** -20) == 1 + 2 ** -7     # above the tie
    assert r(-(1 + 3 * 2 ** -8)) == -(1 + 2 ** -6)
    assert r(0.0) == 0.0 and r(2.0 ** 100) == 2.0 ** 100
    x = np.random.default_rng(5).standard_normal(10000) * np.exp(np.random.default_rng(6).uniform(-20, 20, 10000))
    ref = torch.tensor(x, dtype=torch.float32).to(torch.bfloat16).to(torch.float64).numpy()
    assert np.array_equal(r(x), ref)


def test_forward_bf16_equals_forward_when_rounding_is_exact():
    """T3-style inputs (integers, W_u = I, a = 0, W_m = 0) make every BF16 rounding an
    identity (e' = 1/2, g = 1/d, small dyadic h), so the BF16 forward equals the plain one."""
    d = 4
    cfg = cfg_dict(L=2, F_n=d, F_e=d, d=d, d_h=d)
    graphs = [(4, np.array([0, 0, 1, 2], np.int32), np.array([1, 2, 3, 3], np.int32))]
    X = np.array([[1, 2, 3, 0], [0, 1, 0, 0], [2, 0, 0, 1], [0, 0, 0, 0]], np.float64)
    EF = np.random.default_rng(1).uniform(size=(4, d))
    p = toy_params(cfg, W_u0=np.eye(d), W_u1=np.eye(d), W_e0=np.ones((d, d)), W_e1=np.ones((d, d)),
                   W_1=np.eye(d), w_2=np.ones(d))
    pk = oracle.pack(graphs)
    a = oracle.forward(p, cfg, pk, X, EF)
    b = oracle.forward_bf16(p, cfg, pk, X, EF)
    for i in range(2):
        for k in ("hbar", "p", "q", "e", "g", "h"):
            assert np.array_equal(a["layers"][i][k], b["layers"][i][k]), (i, k)
    assert np.array_equal(a["yhat"], b["yhat"])


def test_forward_bf16_rounds_where_the_mode_says():
    """Random weights: stored h̄, e', g, h are BF16 values; p is computed from the
    unrounded h̄ (so it differs from h̄_bf16·a_s); the whole stays within the BF16 budget."""
    cfg = cfg_dict(L=2, F_n=80, F_e=4, d=16, d_h=16)
    b = configs.random_dag_batch(6, 44, max_nodes=20)
    flat = weights.init_flat(weights.ModelConfig(L=2, d=16, d_h=16), 9)
    p = oracle.unflatten(cfg, flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    f = oracle.forward_bf16(p, cfg, pk, b.node_feat, b.edge_feat)
    g = oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)
    for i in range(2):
        lay = f["layers"][i]
        for k in ("hbar", "e", "g", "h"):
            assert np.array_equal(oracle.bf16_round(lay[k]), lay[k]), (i, k)
        assert not np.array_equal(lay["p"], lay["hbar"] @ p[f"a_s{i}"])
        for k in ("hbar", "p", "e", "h"):
            ref = g["layers"][i][k]
            assert np.linalg.norm(lay[k] - ref) <= 2e-2 * np.linalg.norm(ref), (i, k)


# ------------------------------------------ OCCU_BF16 training backward (R28)
def test_backward_bf16_identity_rounding_is_the_plain_backward():
    """With the rounding replaced by the identity, the BF16-mode forward is forward() and
    backward_bf16's σ'(y) = e'·σ(-αz) equals e'(1 - e'): the gradients must be those of the
    plain backward (itself pinned by finite differences and torch autograd above)."""
    cfg = cfg_dict(L=3, F_n=80, F_e=4, d=16, d_h=8, aggr=0)
    b = configs.random_dag_batch(5, 71, max_nodes=14, hub=True)
    p = rand_params(cfg, 21)
    for i in range(3):
        p[f"W_u{i}"] *= 16
    pk = oracle.pack(b.graphs)
    ident = lambda x: np.asarray(x, np.float64)
    fb = oracle.forward_bf16(p, cfg, pk, b.node_feat, b.edge_feat, rnd=ident)
    fa = oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)
    assert np.allclose(fb["yhat"], fa["yhat"], rtol=1e-13, atol=0)
    lb, gb = oracle.backward_bf16(p, cfg, pk, fb, b.targets)
    la, ga = oracle.backward(p, cfg, pk, fa, b.targets)
    assert abs(lb - la) <= 1e-13 * la
    for k in p:
        assert np.linalg.norm(gb[k] - ga[k]) <= 1e-10 * np.linalg.norm(ga[k]) + 1e-300, k


def test_backward_bf16_exact_when_rounding_is_exact():
    """Integer X, W_u = I, a = 0, an integer W_m with equal row sums and BF16-representable
    W_e / edge features make every BF16 rounding of the mode an identity (e' = 1/2, equal
    logits so g = 1/d, dyadic h, z exact) while W_mᵀ dv, σ' and z still carry gradient
    into a_s, a_d, so the BF16-mode gradients equal the float64 ones."""
    d = 4
    cfg = cfg_dict(L=2, F_n=d, F_e=d, d=d, d_h=d)
    graphs = [(5, np.array([0, 0, 1, 2, 3], np.int32), np.array([1, 2, 3, 3, 4], np.int32))]
    X = np.array([[1, 2, 3, 0], [0, 1, 0, 0], [2, 0, 0, 1], [0, 0, 0, 0], [1, 1, 1, 1]], np.float64)
    rng = np.random.default_rng(3)
    EF = oracle.bf16_round(rng.uniform(size=(5, d)))
    Wm = np.array([[1, 2, 0, -1], [2, -1, 1, 0], [0, 1, -1, 2], [-1, 0, 2, 1]], np.float64)
    p = toy_params(cfg, W_u0=np.eye(d), W_u1=np.eye(d), W_m0=Wm, W_m1=Wm.T.copy(),
                   W_e0=oracle.bf16_round(rng.normal(size=(d, d))),
                   W_e1=oracle.bf16_round(rng.normal(size=(d, d))),
                   W_1=rng.normal(size=(d, d)), b_1=rng.normal(size=d), w_2=rng.normal(size=d))
    y = np.array([0.3])
    pk = oracle.pack(graphs)
    lb, gb = oracle.backward_bf16(p, cfg, pk, oracle.forward_bf16(p, cfg, pk, X, EF), y)
    la, ga = oracle.backward(p, cfg, pk, oracle.forward(p, cfg, pk, X, EF), y)
    assert abs(lb - la) <= 1e-14 * la
    for k in p:
        assert np.allclose(gb[k], ga[k], rtol=1e-12, atol=1e-15), k
    for k in ("W_m0", "W_m1", "a_s1", "a_d0", "W_u0"):      # dW_e = α·(...) = 0 here
        assert np.linalg.norm(ga[k]) > 0, k


def test_backward_bf16_within_the_bf16_budget():
    """Real BF16 roundings: the mode's gradients approximate the exact ones to the BF16
    budget (8 significant bits on stored activations, errors averaging over many terms)."""
    cfg = cfg_dict(L=2, F_n=80, F_e=4, d=16, d_h=16)
    b = configs.random_dag_batch(6, 45, max_nodes=20)
    flat = weights.init_flat(weights.ModelConfig(L=2, d=16, d_h=16), 9)
    p = oracle.unflatten(cfg, flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    lb, gb = oracle.backward_bf16(p, cfg, pk, oracle.forward_bf16(p, cfg, pk, b.node_feat, b.edge_feat), b.targets)
    la, ga = oracle.backward(p, cfg, pk, oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat), b.targets)
    assert abs(lb - la) <= 2e-2 * la
    for k in p:
        assert np.linalg.norm(gb[k] - ga[k]) <= 3e-2 * np.linalg.norm(ga[k]), k


# ------------------------------------------ NEXT-2: Set-Transformer decoder readout
def dec_cfg(k=4, heads=4, d=16, L=2):
    c = cfg_dict(L=L, F_n=80, F_e=4, d=d, d_h=8)
    c.update(readout=1, k=k, heads=heads)
    return c


def dec_params(c, seed):
    wc = weights.ModelConfig(L=c["L"], F_n=c["F_n"], F_e=c["F_e"], d=c["d"], d_h=c["d_h"],
                             readout=1, k=c["k"], heads=c["heads"])
    p = oracle.unflatten(c, weights.init_flat(wc, seed).astype(np.float64))
    for i in range(c["L"]):
        p[f"W_u{i}"] *= 4.0                      # keep node states O(1) through the layers
    rng = np.random.default_rng(seed)
    for m in ("M1_", "M2_"):                      # non-trivial LayerNorm affine parameters
        for ln in ("ln1", "ln2"):
            p[m + ln + "_g"] = 1.0 + 0.3 * rng.standard_normal(c["d"])
            p[m + ln + "_b"] = 0.2 * rng.standard_normal(c["d"])
    return p


def torch_decoder(H, p, c):
    """Independent implementation of Decoder(H) = FFN(SAB(PMA_k(FFN(H)))) with torch's own
    nn.MultiheadAttention and nn.LayerNorm (float64)."""
    torch = pytest.importorskip("torch")
    d, heads = c["d"], c["heads"]
    T = lambda a: torch.tensor(a, dtype=torch.float64)
    F = torch.nn.functional

    def ffn(x, q):
        return F.linear(F.relu(F.linear(x, T(p[q + "W1"]), T(p[q + "b1"]))), T(p[q + "W2"]), T(p[q + "b2"]))

    def mab(X, Y, m):
        att = torch.nn.MultiheadAttention(d, heads, bias=True, batch_first=True, dtype=torch.float64)
        ln1 = torch.nn.LayerNorm(d, eps=1e-5, dtype=torch.float64)
        ln2 = torch.nn.LayerNorm(d, eps=1e-5, dtype=torch.float64)
        with torch.no_grad():
            att.in_proj_weight.copy_(torch.cat([T(p[m + "Wq"]), T(p[m + "Wk"]), T(p[m + "Wv"])]))
            att.in_proj_bias.copy_(torch.cat([T(p[m + "bq"]), T(p[m + "bk"]), T(p[m + "bv"])]))
            att.out_proj.weight.copy_(T(p[m + "Wo"]))
            att.out_proj.bias.copy_(T(p[m + "bo"]))
            ln1.weight.copy_(T(p[m + "ln1_g"])); ln1.bias.copy_(T(p[m + "ln1_b"]))
            ln2.weight.copy_(T(p[m + "ln2_g"])); ln2.bias.copy_(T(p[m + "ln2_b"]))
            a, _ = att(X[None], Y[None], Y[None], need_weights=False)
            Hb = ln1(X + a[0])
            return ln2(Hb + ffn(Hb, m + "F_"))

    with torch.no_grad():
        Z = ffn(T(H), "P_")
        pma = mab(T(p["S"]), Z, "M1_")
        return ffn(mab(pma, pma, "M2_"), "D_").numpy()


@pytest.mark.parametrize("k,heads", [(4, 4), (1, 2), (3, 1)])
def test_decoder_matches_torch_modules(k, heads):
    c = dec_cfg(k=k, heads=heads)
    b = configs.random_dag_batch(4, 77 + k, max_nodes=20, hub=True)
    p = dec_params(c, 5 + k)
    pk = oracle.pack(b.graphs)
    f = oracle.forward(p, c, pk, b.node_feat, b.edge_feat)
    hL = f["layers"][-1]["h"]
    off = pk["node_off"]
    for g in range(pk["num_graphs"]):
        ref = torch_decoder(hL[off[g]:off[g + 1]], p, c)
        assert f["dec"][g].shape == (k, c["d"])
        assert np.allclose(f["dec"][g], ref, rtol=1e-10, atol=1e-12), g
    # the head reads the flattened decoder output
    r = f["dec"].reshape(pk["num_graphs"], -1)
    y = oracle.leaky_relu(r @ p["W_1"].T + p["b_1"], c["slope"]) @ p["w_2"] + p["b_2"][0]
    assert np.array_equal(y, f["yhat"])


def test_decoder_single_key_attention_ignores_query_and_key_maps():
    """Softmax over one key is exactly 1: with k = 1 the SAB's attention output is its value
    projection, so W_q, W_k of MAB2 cannot matter (bitwise); with single-node graphs the same
    holds for MAB1 (PMA)."""
    c = dec_cfg(k=1, heads=2)
    b = configs.random_dag_batch(3, 41, max_nodes=12)
    p = dec_params(c, 9)
    pk = oracle.pack(b.graphs)
    y0 = oracle.forward(p, c, pk, b.node_feat, b.edge_feat)["yhat"]
    q = dict(p)
    q["M2_Wq"] = p["M2_Wq"] * 3.0 + 1.0
    q["M2_Wk"] = -p["M2_Wk"]
    q["M2_bq"] = p["M2_bq"] + 2.0
    assert np.array_equal(oracle.forward(q, c, pk, b.node_feat, b.edge_feat)["yhat"], y0)
    single = [(1, np.zeros(0, np.int32), np.zeros(0, np.int32))] * 3
    nf = np.random.default_rng(2).normal(size=(3, 80))
    ef = np.zeros((0, 4))
    pk1 = oracle.pack(single)
    y1 = oracle.forward(p, c, pk1, nf, ef)["yhat"]
    q = dict(p)
    q["M1_Wq"] = p["M1_Wq"] * 2.0
    q["M1_Wk"] = p["M1_Wk"] - 1.0
    assert np.array_equal(oracle.forward(q, c, pk1, nf, ef)["yhat"], y1)


def test_decoder_readout_node_permutation_and_batching_invariance():
    c = dec_cfg()
    b = configs.random_dag_batch(5, 123, max_nodes=25, hub=True)
    p = dec_params(c, 3)
    y = oracle.predict(p, c, b.graphs, b.node_feat, b.edge_feat)
    for g in range(b.num_graphs):                       # batching (BLAS blocking: ~1 ulp)
        s = b.subset([g])
        assert np.allclose(oracle.predict(p, c, s.graphs, s.node_feat, s.edge_feat), y[g:g + 1],
                           rtol=1e-13, atol=1e-15)
    # relabel nodes inside every graph: PMA pools a set, so ŷ is unchanged up to rounding
    rng = np.random.default_rng(8)
    graphs, nfs, efs = [], [], []
    noff = np.concatenate([[0], np.cumsum([g[0] for g in b.graphs])])
    eoff = np.concatenate([[0], np.cumsum([len(g[1]) for g in b.graphs])])
    for g, (n, s_, t_) in enumerate(b.graphs):
        perm = rng.permutation(n)
        inv = np.argsort(perm)
        graphs.append((n, inv[s_].astype(np.int32), inv[t_].astype(np.int32)))
        nfs.append(b.node_feat[noff[g]:noff[g + 1]][perm])
        efs.append(b.edge_feat[eoff[g]:eoff[g + 1]])
    y2 = oracle.predict(p, c, graphs, np.concatenate(nfs), np.concatenate(efs))
    assert np.allclose(y2, y, rtol=1e-12, atol=1e-14)


# ------------------------------------------ NEXT-3: Graphormer layers (P153-P157)
def gph_cfg(G=2, heads=4, d=16, L=2, readout=0, k=2):
    c = cfg_dict(L=L, F_n=80, F_e=4, d=d, d_h=8)
    c.update(readout=readout, k=k, heads=heads, graphormer=G)
    return c


def gph_params(c, seed):
    wc = weights.ModelConfig(L=c["L"], F_n=c["F_n"], F_e=c["F_e"], d=c["d"], d_h=c["d_h"],
                             readout=c["readout"], k=c["k"], heads=c["heads"],
                             graphormer=c["graphormer"])
    p = oracle.unflatten(c, weights.init_flat(wc, seed).astype(np.float64))
    for i in range(c["L"]):
        p[f"W_u{i}"] *= 4.0
    rng = np.random.default_rng(seed)
    for j in range(c["graphormer"]):              # non-trivial LayerNorm affine parameters
        for ln in ("ln1", "ln2"):
            p[f"G{j}_{ln}_g"] = 1.0 + 0.3 * rng.standard_normal(c["d"])
            p[f"G{j}_{ln}_b"] = 0.2 * rng.standard_normal(c["d"])
    return p


def torch_graphormer(H, p, c, j):
    """Independent Graphormer layer (P155, P157): pre-LN self-attention and FFN blocks with
    residuals, built from torch's nn.LayerNorm and nn.MultiheadAttention (float64)."""
    torch = pytest.importorskip("torch")
    d, heads = c["d"], c["heads"]
    T = lambda a: torch.tensor(a, dtype=torch.float64)
    F = torch.nn.functional
    g = f"G{j}_"
    att = torch.nn.MultiheadAttention(d, heads, bias=True, batch_first=True, dtype=torch.float64)
    ln1 = torch.nn.LayerNorm(d, eps=1e-5, dtype=torch.float64)
    ln2 = torch.nn.LayerNorm(d, eps=1e-5, dtype=torch.float64)
    with torch.no_grad():
        att.in_proj_weight.copy_(torch.cat([T(p[g + "Wq"]), T(p[g + "Wk"]), T(p[g + "Wv"])]))
        att.in_proj_bias.copy_(torch.cat([T(p[g + "bq"]), T(p[g + "bk"]), T(p[g + "bv"])]))
        att.out_proj.weight.copy_(T(p[g + "Wo"]))
        att.out_proj.bias.copy_(T(p[g + "bo"]))
        ln1.weight.copy_(T(p[g + "ln1_g"])); ln1.bias.copy_(T(p[g + "ln1_b"]))
        ln2.weight.copy_(T(p[g + "ln2_g"])); ln2.bias.copy_(T(p[g + "ln2_b"]))
        h = T(H)
        x = ln1(h)
        a, _ = att(x[None], x[None], x[None], need_weights=False)
        hb = a[0] + h
        y = ln2(hb)
        f = F.linear(F.relu(F.linear(y, T(p[g + "F_W1"]), T(p[g + "F_b1"]))), T(p[g + "F_W2"]), T(p[g + "F_b2"]))
        return (f + hb).numpy()


@pytest.mark.parametrize("G,heads,readout", [(2, 4, 0), (1, 2, 0), (2, 4, 1)])
def test_graphormer_matches_torch_modules(G, heads, readout):
    c = gph_cfg(G=G, heads=heads, readout=readout)
    b = configs.random_dag_batch(4, 300 + G + heads, max_nodes=20, hub=True)
    p = gph_params(c, 11 + G)
    pk = oracle.pack(b.graphs)
    f = oracle.forward(p, c, pk, b.node_feat, b.edge_feat)
    off = pk["node_off"]
    h = f["layers"][-1]["h"]
    for j in range(G):
        ref = np.concatenate([torch_graphormer(h[off[g]:off[g + 1]], p, c, j)
                              for g in range(pk["num_graphs"])])
        assert np.allclose(f["gph"][j], ref, rtol=1e-10, atol=1e-12), j
        h = ref
    if readout == 0:          # mean readout of the last Graphormer output, then the head
        r = np.stack([h[off[g]:off[g + 1]].mean(axis=0) for g in range(pk["num_graphs"])])
        y = oracle.leaky_relu(r @ p["W_1"].T + p["b_1"], c["slope"]) @ p["w_2"] + p["b_2"][0]
        assert np.allclose(f["yhat"], y, rtol=1e-12, atol=1e-14)
    else:                     # the decoder reads the Graphormer output
        for g in range(pk["num_graphs"]):
            assert np.allclose(f["dec"][g], torch_decoder(h[off[g]:off[g + 1]], p, c),
                               rtol=1e-10, atol=1e-12)


def test_graphormer_zero_output_maps_is_identity():
    """With W_o = b_o = 0 and the FFN's W2 = b2 = 0 both residual branches vanish: the layer
    is the identity, bitwise (P155, P157 residual form)."""
    c = gph_cfg(G=2)
    b = configs.random_dag_batch(3, 61, max_nodes=15)
    p = gph_params(c, 4)
    for j in range(2):
        for n in ("Wo", "bo", "F_W2", "F_b2"):
            p[f"G{j}_{n}"] = np.zeros_like(p[f"G{j}_{n}"])
    pk = oracle.pack(b.graphs)
    f = oracle.forward(p, c, pk, b.node_feat, b.edge_feat)
    assert np.array_equal(f["gph"][1], f["layers"][-1]["h"])


def test_graphormer_single_node_graph_closed_form():
    """One node: attention over a single key is exactly 1, so MHA(x) = W_o (W_v x + b_v) + b_o
    whatever W_q, W_k (bitwise invariance), and the layer has the closed form below."""
    c = gph_cfg(G=1, heads=2)
    p = gph_params(c, 8)
    single = [(1, np.zeros(0, np.int32), np.zeros(0, np.int32))] * 3
    nf = np.random.default_rng(5).normal(size=(3, 80))
    ef = np.zeros((0, 4))
    pk = oracle.pack(single)
    f = oracle.forward(p, c, pk, nf, ef)
    h = f["layers"][-1]["h"]
    ln = lambda x, g, bb: (x - x.mean(-1, keepdims=True)) / np.sqrt(x.var(-1, keepdims=True) + 1e-5) * g + bb
    x = ln(h, p["G0_ln1_g"], p["G0_ln1_b"])
    hb = (x @ p["G0_Wv"].T + p["G0_bv"]) @ p["G0_Wo"].T + p["G0_bo"] + h
    y = ln(hb, p["G0_ln2_g"], p["G0_ln2_b"])
    ref = np.maximum(y @ p["G0_F_W1"].T + p["G0_F_b1"], 0) @ p["G0_F_W2"].T + p["G0_F_b2"] + hb
    assert np.allclose(f["gph"][0], ref, rtol=1e-12, atol=1e-13)
    q = dict(p)
    q["G0_Wq"] = p["G0_Wq"] * 3.0 - 1.0
    q["G0_Wk"] = -p["G0_Wk"]
    q["G0_bk"] = p["G0_bk"] + 5.0
    assert np.array_equal(oracle.forward(q, c, pk, nf, ef)["gph"][0], f["gph"][0])


def test_graphormer_node_permutation_and_batching_invariance():
    """Self-attention over a graph's node set is permutation-equivariant and never crosses
    graphs: ŷ is invariant to relabelling nodes and equal batched vs one graph at a time."""
    c = gph_cfg(G=2)
    b = configs.random_dag_batch(5, 129, max_nodes=25, hub=True)
    p = gph_params(c, 6)
    y = oracle.predict(p, c, b.graphs, b.node_feat, b.edge_feat)
    for g in range(b.num_graphs):
        s = b.subset([g])
        assert np.allclose(oracle.predict(p, c, s.graphs, s.node_feat, s.edge_feat), y[g:g + 1],
                           rtol=1e-12, atol=1e-14)
    rng = np.random.default_rng(18)
    graphs, nfs, efs = [], [], []
    noff = np.concatenate([[0], np.cumsum([g[0] for g in b.graphs])])
    eoff = np.concatenate([[0], np.cumsum([len(g[1]) for g in b.graphs])])
    for g, (n, s_, t_) in enumerate(b.graphs):
        perm = rng.permutation(n)
        inv = np.argsort(perm)
        graphs.append((n, inv[s_].astype(np.int32), inv[t_].astype(np.int32)))
        nfs.append(b.node_feat[noff[g]:noff[g + 1]][perm])
        efs.append(b.edge_feat[eoff[g]:eoff[g + 1]])
    y2 = oracle.predict(p, c, graphs, np.concatenate(nfs), np.concatenate(efs))
    assert np.allclose(y2, y, rtol=1e-11, atol=1e-13)


def test_graphormer_weights_file_v3_roundtrip(tmp_path):
    c = gph_cfg(G=2, readout=1, k=3)
    wc = weights.ModelConfig(L=c["L"], F_n=80, F_e=4, d=c["d"], d_h=c["d_h"], readout=1, k=3,
                             heads=c["heads"], graphormer=2)
    flat = weights.init_flat(wc, 42)
    path = str(tmp_path / "w.bin")
    weights.write_weights(path, wc, flat)
    cf, p = oracle.read_weights(path)
    assert cf["graphormer"] == 2 and cf["readout"] == 1 and cf["k"] == 3
    assert np.array_equal(oracle.flatten(cf, p), flat.astype(np.float64))
    assert np.all(p["G1_ln2_g"] == 1.0) and np.all(p["G0_ln1_b"] == 0.0)


# ------------------------------------------ NEXT-4: occu-packing consumer (P390-P392)
def read_golden_packing():
    import os
    d = {}
    for ln in open(os.path.join(os.path.dirname(__file__), "golden", "occu_packing_first_fit.txt")):
        if ln.startswith("#") or not ln.strip():
            continue
        k, *v = ln.split()
        d[k] = v
    return (np.array(d["occ"], np.float32), np.array(d["assign"], np.int32), int(d["bins"][0]))


def test_occu_packing_golden_first_fit():
    occ, assign, bins = read_golden_packing()
    a, loads = oracle.occu_packing(occ)
    assert np.array_equal(a, assign) and len(loads) == bins


def test_occu_packing_invariants_and_bounds():
    """Every slot stays within capacity (jobs <= capacity), loads are the sums of their jobs,
    first fit never leaves two slots at most half full (so slots <= 2*sum + 1), and the
    count is at least ceil(sum); equal-size jobs of 1/k fill slots exactly k at a time."""
    rng = np.random.default_rng(4)
    for n in (1, 17, 500):
        occ = rng.random(n).astype(np.float32)
        a, loads = oracle.occu_packing(occ)
        assert np.all(loads <= 1.0)
        assert np.allclose(np.bincount(a, weights=occ.astype(np.float64)), loads, rtol=0, atol=1e-12)
        assert np.sum(loads <= 0.5) <= 1
        assert len(loads) >= np.ceil(occ.astype(np.float64).sum() - 1e-9)
        assert len(loads) <= 2 * occ.astype(np.float64).sum() + 1
    a, loads = oracle.occu_packing(np.full(12, 0.25, np.float32))
    assert np.array_equal(a, np.repeat(np.arange(3), 4))
    a, _ = oracle.occu_packing(np.array([-0.1, 1.3, 0.2], np.float32))   # clamp, oversize alone
    assert np.array_equal(a, [0, 1, 0])


def test_forward_bf16_reading_b_identity_rounding_and_chain_closed_form():
    """Reading B in OCCU_BF16 (R40): with the rounding replaced by the identity, forward_bf16
    is forward() (same steps); with BF16 rounding, a single in-edge still gives weight
    exactly 1 (softmax over one edge), so a chain's h_t = LReLU(h̄_src) holds per layer
    with the BF16-stored h̄."""
    cfg = cfg_dict(L=2, F_n=80, F_e=4, d=16, d_h=8)
    cfg["msg"] = 1
    b = configs.random_dag_batch(5, 91, max_nodes=20, hub=True)
    wc = weights.ModelConfig(L=2, F_n=80, F_e=4, d=16, d_h=8, msg=1)
    p = oracle.unflatten(cfg, weights.init_flat(wc, 3).astype(np.float64))
    pk = oracle.pack(b.graphs)
    f = oracle.forward(p, cfg, pk, b.node_feat, b.edge_feat)
    fb = oracle.forward_bf16(p, cfg, pk, b.node_feat, b.edge_feat, rnd=lambda x: np.asarray(x, np.float64))
    assert np.allclose(fb["yhat"], f["yhat"], rtol=1e-12, atol=1e-14)
    for i in range(2):
        assert np.allclose(fb["layers"][i]["g"], f["layers"][i]["g"], rtol=1e-12, atol=1e-14)
    chain = [(6, np.arange(5, dtype=np.int32), np.arange(1, 6, dtype=np.int32))]
    nf = np.random.default_rng(1).random((6, 80))
    ef = np.random.default_rng(2).random((5, 4))
    pkc = oracle.pack(chain)
    fc = oracle.forward_bf16(p, cfg, pkc, nf, ef)
    for i in range(2):
        lay = fc["layers"][i]
        assert np.array_equal(lay["g"], np.ones_like(lay["g"]))
        assert np.allclose(lay["h_f32"][1:], oracle.leaky_relu(lay["hbar"][:5], cfg["slope"]), rtol=1e-15, atol=0)


def test_mha_fp16_rounded_variant_limits():
    """R42: with the identity as rounding the fp16-operand MHA is the plain MHA (same
    function); with fp16 rounding it stays within fp16's relative precision of it."""
    rng = np.random.default_rng(3)
    d, heads = 16, 4
    p = {f"G_W{w}": rng.standard_normal((d, d)) / 4 for w in "qkvo"}
    p.update({f"G_b{w}": rng.standard_normal(d) / 4 for w in "qkvo"})
    X = rng.standard_normal((11, d))
    ref = oracle.mha(X, X, p, "G_", heads)
    assert np.allclose(oracle.mha(X, X, p, "G_", heads, rnd=lambda x: np.asarray(x, np.float64)), ref,
                       rtol=1e-12, atol=1e-13)
    r16 = oracle.mha(X, X, p, "G_", heads, rnd=oracle.fp16_round)
    assert np.linalg.norm(r16 - ref) <= 4e-3 * np.linalg.norm(ref)
    assert not np.array_equal(r16, ref)


# ------------------------------------------ NEXT-2 / NEXT-3 training: readout-stack backward
def torch_full_loss(p, c, pk, X, EF, y, gb=None):
    """Independent forward of the paper's full model (ANEE -> Graphormer layers -> decoder or
    mean -> head, MSE) built from torch.nn.functional (layer_norm, multi_head_attention_forward,
    linear), differentiated by autograd in float64."""
    torch = pytest.importorskip("torch")
    F = torch.nn.functional
    T = {k: torch.tensor(v, dtype=torch.float64, requires_grad=True) for k, v in p.items()}
    s = torch.tensor(pk["in_src"].astype(np.int64))
    t = torch.tensor(pk["in_dst"].astype(np.int64))
    h = torch.tensor(X, dtype=torch.float64)
    e = torch.tensor(EF, dtype=torch.float64)[torch.tensor(pk["in_eid"].astype(np.int64))]
    lrelu = lambda x: F.leaky_relu(x, c["slope"])
    N, d, heads = pk["num_nodes"], c["d"], c["heads"]
    for i in range(c["L"]):
        hb = lrelu(h @ T[f"W_u{i}"].T)
        al = hb[s] @ T[f"a_s{i}"] + hb[t] @ T[f"a_d{i}"]
        e = torch.sigmoid(al[:, None] * (e @ T[f"W_e{i}"].T))
        g = torch.softmax(e @ T[f"W_m{i}"].T, dim=1)
        h = lrelu(torch.zeros(N, d, dtype=torch.float64).index_add(0, t, g * hb[s]))

    def ffn(x, q):
        return F.linear(F.relu(F.linear(x, T[q + "W1"], T[q + "b1"])), T[q + "W2"], T[q + "b2"])

    def att(Xq, Y, m):
        o, _ = F.multi_head_attention_forward(
            Xq[:, None], Y[:, None], Y[:, None], d, heads,
            torch.cat([T[m + "Wq"], T[m + "Wk"], T[m + "Wv"]]),
            torch.cat([T[m + "bq"], T[m + "bk"], T[m + "bv"]]), None, None, False, 0.0,
            T[m + "Wo"], T[m + "bo"], training=False, need_weights=False)
        return o[:, 0]

    def ln(x, q):
        return F.layer_norm(x, (d,), T[q + "_g"], T[q + "_b"], 1e-5)

    def mab(Xq, Y, m):
        Hb = ln(Xq + att(Xq, Y, m), m + "ln1")
        return ln(Hb + ffn(Hb, m + "F_"), m + "ln2")

    off = pk["node_off"].astype(np.int64)
    rows = []
    for b in range(pk["num_graphs"]):
        H = h[off[b]:off[b + 1]]
        for j in range(c["graphormer"]):
            g_ = f"G{j}_"
            Hb = att(ln(H, g_ + "ln1"), ln(H, g_ + "ln1"), g_) + H
            H = ffn(ln(Hb, g_ + "ln2"), g_ + "F_") + Hb
        if c["readout"] == 1:
            pma = mab(T["S"], ffn(H, "P_"), "M1_")
            rows.append(ffn(mab(pma, pma, "M2_"), "D_").reshape(-1))
        else:
            rows.append(H.mean(dim=0))
    r = torch.stack(rows)
    yh = lrelu(r @ T["W_1"].T + T["b_1"]) @ T["w_2"] + T["b_2"][0]
    nb = len(y) if gb is None else gb
    loss = ((yh - torch.tensor(y, dtype=torch.float64)) ** 2).sum() / nb
    loss.backward()
    return float(loss), {k: v.grad.numpy() for k, v in T.items()}


def _stack_params(c, seed):
    p = gph_params(c, seed)
    rng = np.random.default_rng(seed + 100)
    if c["readout"] == 1:
        for m in ("M1_", "M2_"):
            for ln_ in ("ln1", "ln2"):
                p[m + ln_ + "_g"] = 1.0 + 0.3 * rng.standard_normal(c["d"])
                p[m + ln_ + "_b"] = 0.2 * rng.standard_normal(c["d"])
    return p


@pytest.mark.parametrize("G,heads,readout", [(2, 4, 0), (0, 2, 1), (2, 4, 1), (1, 1, 1)])
def test_readout_stack_backward_matches_torch_autograd(G, heads, readout):
    c = gph_cfg(G=G, heads=heads, readout=readout, k=3)
    b = configs.random_dag_batch(4, 900 + G + heads + readout, max_nodes=16, hub=True)
    p = _stack_params(c, 21 + G)
    pk = oracle.pack(b.graphs)
    loss, grads = oracle.backward(p, c, pk, oracle.forward(p, c, pk, b.node_feat, b.edge_feat),
                                  b.targets, global_batch=7)
    tl, tg = torch_full_loss(p, c, pk, b.node_feat, b.edge_feat, b.targets, gb=7)
    assert abs(loss - tl) <= 1e-12 * abs(tl)
    assert set(grads) == set(p)
    for k in p:
        assert np.allclose(grads[k], tg[k], rtol=1e-8, atol=1e-13 * max(1, np.abs(tg[k]).max())), k


@pytest.mark.parametrize("G,readout", [(1, 1), (2, 0)])
def test_readout_stack_backward_finite_differences(G, readout):
    """Central differences through the whole stack on a tiny model (d = 4, 2 heads, k = 2)."""
    c = gph_cfg(G=G, heads=2, d=4, L=1, readout=readout, k=2)
    c["F_n"], c["F_e"] = 5, 3
    b = configs.random_dag_batch(3, 70 + G, max_nodes=6, f_n=5, f_e=3, hub=True)
    p = _stack_params(c, 31 + G)
    fd_check(c, b, p, tol=2e-6)
