"""CPU ORACLE for DNN-occu's batched ANEE GNN hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this module.  The product path (the C-ABI
library in ``paper_conf_cluster_meiqsgls23_b200/``) never calls it, and this
module imports nothing from the product package.

Plain NumPy, float64 throughout (the paper fixes no precision).  Every function
cites the passage it follows; "P<n>" = /root/reference/PAPER.md line n, "R<k>"
= reading k listed in DESIGN.md §3 (readings of garbled / silent passages).

Computation (per ANEE layer i, P139-P151; R1-R9):
    h̄   = LeakyReLU(h^{i-1} W_u^T)                                 P141
    α_l = a_s·h̄_s + a_d·h̄_d   for edge l = (s, d)                  P145, P147 (R1)
    e^i_l = σ(α_l · (W_e e^{i-1}_l))                                P145 (R2, R3)
    f(u',l') = Softmax_channels(W_m e^i_l') ⊙ h̄_u'                  P149 (R4, reading A)
    h^i_u = LeakyReLU(Σ_{l'=(u',u)} f(u',l'))                       P149 (R8, R9)
optionally Graphormer layers per graph (P153-P157, NEXT-3; R35-R37), then the per-graph
mean readout (north_star; R11) or the Set-Transformer decoder (P159-P205, NEXT-2; R30-R34)
and the MLP head (P125; R12),
MSE loss (P209-P213), Adam (P273; R16).

Parity status: every function here is pinned by tests in tests/test_oracle.py
(hand-derived toy DAGs, closed forms, invariances, finite differences, an
independent torch-autograd implementation, Adam's first-step closed form).
"""
from __future__ import annotations

import struct

import numpy as np

AGGR_SUM, AGGR_MEAN = 0, 1
MSG_CHANNEL_SOFTMAX, MSG_NEIGHBOR_SOFTMAX = 0, 1


# --------------------------------------------------------------------------
# Step P: packing (P49 "DAG", P139 edge l = (u_s, u_d), P149 Σ over l'=(u',u);
# tie-break keys are reading R17).  Integer work: must match the library
# bit for bit.
# --------------------------------------------------------------------------
def pack(graphs):
    """graphs: list of (num_nodes, src[m], dst[m]) with local ids.

    Returns dict of int32 arrays: node_off, edge_off [B+1]; in_ptr [N+1],
    in_src, in_dst, in_eid [E] (edges sorted by key (dst, src, eid));
    out_ptr [N+1], out_pos [E] (edges sorted by key (src, dst, eid); out_pos[j]
    is the in-CSR position of the j-th out-ordered edge); node_graph [N].
    """
    B = len(graphs)
    n_b = np.array([int(g[0]) for g in graphs], dtype=np.int64)
    m_b = np.array([len(g[1]) for g in graphs], dtype=np.int64)
    node_off = np.concatenate([[0], np.cumsum(n_b)]).astype(np.int64)
    edge_off = np.concatenate([[0], np.cumsum(m_b)]).astype(np.int64)
    N, E = int(node_off[-1]), int(edge_off[-1])
    src = np.zeros(E, np.int64)
    dst = np.zeros(E, np.int64)
    for b, (n, s, t) in enumerate(graphs):
        src[edge_off[b]:edge_off[b + 1]] = node_off[b] + np.asarray(s, np.int64)
        dst[edge_off[b]:edge_off[b + 1]] = node_off[b] + np.asarray(t, np.int64)
    eid = np.arange(E, dtype=np.int64)
    in_order = np.lexsort((eid, src, dst))        # primary dst, then src, then eid
    out_order = np.lexsort((eid, dst, src))       # primary src, then dst, then eid
    in_pos_of_eid = np.empty(E, np.int64)
    in_pos_of_eid[in_order] = np.arange(E)
    in_ptr = np.searchsorted(dst[in_order], np.arange(N + 1), side="left")
    out_ptr = np.searchsorted(src[out_order], np.arange(N + 1), side="left")
    node_graph = np.repeat(np.arange(B), n_b)
    i32 = lambda a: np.asarray(a, dtype=np.int32)
    return {
        "num_graphs": B, "num_nodes": N, "num_edges": E,
        "node_off": i32(node_off), "edge_off": i32(edge_off),
        "in_ptr": i32(in_ptr), "in_src": i32(src[in_order]), "in_dst": i32(dst[in_order]),
        "in_eid": i32(in_order), "out_ptr": i32(out_ptr),
        "out_pos": i32(in_pos_of_eid[out_order]), "node_graph": i32(node_graph),
    }


# --------------------------------------------------------------------------
# Weights file; the oracle reads it with its own reader.
# --------------------------------------------------------------------------
def read_weights(path):
    with open(path, "rb") as f:
        raw = f.read()
    if raw[:8] != b"OCCUW001":
        raise ValueError("bad magic")
    version, L, F_n, F_e, d, d_h, aggr, msg = struct.unpack_from("<8I", raw, 8)
    (slope,) = struct.unpack_from("<f", raw, 40)
    cfg = dict(L=L, F_n=F_n, F_e=F_e, d=d, d_h=d_h, aggr=aggr, msg=msg, slope=float(slope))
    hdr = 44
    if version == 2:                      # Set-Transformer decoder readout (NEXT-2)
        cfg["readout"], cfg["k"], cfg["heads"] = struct.unpack_from("<3I", raw, 44)
        hdr = 56
    elif version == 3:                    # + Graphormer layers (NEXT-3)
        cfg["readout"], cfg["k"], cfg["heads"], cfg["graphormer"] = struct.unpack_from("<4I", raw, 44)
        hdr = 60
    flat = np.frombuffer(raw, dtype="<f4", offset=hdr, count=(len(raw) - hdr - 8) // 4)
    return cfg, unflatten(cfg, flat.astype(np.float64))


def param_shapes(cfg):
    """File order; shapes follow P141-P149 (R1, R5) and P125 (R12)."""
    out = []
    for i in range(cfg["L"]):
        d_in = cfg["F_n"] if i == 0 else cfg["d"]
        de_in = cfg["F_e"] if i == 0 else cfg["d"]
        out += [(f"W_u{i}", (cfg["d"], d_in)), (f"W_e{i}", (cfg["d"], de_in)),
                (f"W_m{i}", (cfg["d"], cfg["d"])), (f"a_s{i}", (cfg["d"],)),
                (f"a_d{i}", (cfg["d"],))]
    d, hin = cfg["d"], cfg["d"]
    ffn = lambda p: [(p + "W1", (d, d)), (p + "b1", (d,)), (p + "W2", (d, d)), (p + "b2", (d,))]
    for j in range(cfg.get("graphormer", 0)):
        # Graphormer layer j (P153-P157; R35-R37): LN1, MHA, LN2, FFN
        g = f"G{j}_"
        out += [(g + "ln1_g", (d,)), (g + "ln1_b", (d,))]
        for w in "qkvo":
            out += [(g + "W" + w, (d, d)), (g + "b" + w, (d,))]
        out += [(g + "ln2_g", (d,)), (g + "ln2_b", (d,))] + ffn(g + "F_")
    if cfg.get("readout", 0) == 1:
        # Set-Transformer decoder (P159-P205; R30-R34): seeds, pre-pooling FFN,
        # MAB1 (PMA), MAB2 (SAB), final FFN; the head then reads the flattened k x d output
        out += [("S", (cfg["k"], d))] + ffn("P_")
        for m in ("M1_", "M2_"):
            for w in "qkvo":
                out += [(m + "W" + w, (d, d)), (m + "b" + w, (d,))]
            out += [(m + "ln1_g", (d,)), (m + "ln1_b", (d,))] + ffn(m + "F_")
            out += [(m + "ln2_g", (d,)), (m + "ln2_b", (d,))]
        out += ffn("D_")
        hin = cfg["k"] * d
    out += [("W_1", (cfg["d_h"], hin)), ("b_1", (cfg["d_h"],)),
            ("w_2", (cfg["d_h"],)), ("b_2", (1,))]
    return out


def unflatten(cfg, flat):
    params, off = {}, 0
    for name, shape in param_shapes(cfg):
        n = int(np.prod(shape))
        params[name] = np.array(flat[off:off + n], dtype=np.float64).reshape(shape)
        off += n
    if off != len(flat):
        raise ValueError("weights payload size mismatch")
    return params


def flatten(cfg, params):
    return np.concatenate([np.asarray(params[n], np.float64).ravel()
                           for n, _ in param_shapes(cfg)])


# --------------------------------------------------------------------------
# Elementwise functions (R3 σ = logistic; R7 LeakyReLU slope 0.01).
# --------------------------------------------------------------------------
def leaky_relu(x, slope):
    return np.where(x > 0, x, slope * x)


def leaky_relu_grad(x, slope):
    """PyTorch convention: derivative at 0 is the negative slope (R7)."""
    return np.where(x > 0, 1.0, slope)


def sigmoid(x):
    return 1.0 / (1.0 + np.exp(-x))


def softmax_channels(v):
    """Softmax over the last axis (channels) of each row: reading A of P149 (R4)."""
    mx = v.max(axis=-1, keepdims=True)
    ex = np.exp(v - mx)
    return ex / ex.sum(axis=-1, keepdims=True)


def segment_sum(values, seg_ids, num_segments):
    """Σ of rows per segment, rows added in ascending row order (np.add.at is
    sequential and unbuffered).  Empty segments give 0 (R8)."""
    out = np.zeros((num_segments,) + values.shape[1:], dtype=values.dtype)
    np.add.at(out, seg_ids, values)
    return out


# --------------------------------------------------------------------------
# Step F: forward (P141-P151), readout (north_star, R11), head (P125, R12).
# --------------------------------------------------------------------------
def anee_layer(params, i, cfg, pk, h_prev, e_prev):
    """One ANEE round i (0-based) on the packed batch; edges in in-CSR order.

    Returns the layer's intermediates (all float64).
    """
    slope = cfg["slope"]
    s_k, t_k = pk["in_src"].astype(np.int64), pk["in_dst"].astype(np.int64)
    N = pk["num_nodes"]
    W_u, W_e, W_m = params[f"W_u{i}"], params[f"W_e{i}"], params[f"W_m{i}"]
    a_s, a_d = params[f"a_s{i}"], params[f"a_d{i}"]
    # P141: h̄_u = LeakyReLU(W_u × h_u^{i-1})
    P = h_prev @ W_u.T
    hbar = leaky_relu(P, slope)
    # P145/P147 (R1): a^T (h̄_s || h̄_d) = a_s·h̄_s + a_d·h̄_d, a scalar per edge
    p = hbar @ a_s
    q = hbar @ a_d
    alpha = p[s_k] + q[t_k]
    # P145 (R2): e_l^i = σ(α_l · (W_e × e_l^{i-1}))
    z = e_prev @ W_e.T
    e = sigmoid(alpha[:, None] * z)
    if cfg.get("msg", MSG_CHANNEL_SOFTMAX) == MSG_CHANNEL_SOFTMAX:
        # P149 (R4 reading A): f(u',l') = Softmax(W_m × e_l'^i) ⊙ h̄_u'
        v = e @ W_m.T
        g = softmax_channels(v)
        msg = g * hbar[s_k]
        # P149: h_u^i = LeakyReLU(Σ_{l'=(u',u)} f(u',l'))
        A = segment_sum(msg, t_k, N)
    else:
        # NEXT-1 reading B: per-channel softmax over the in-edges of u
        v = e @ W_m.T
        M = np.full((N, v.shape[1]), -np.inf)
        np.maximum.at(M, t_k, v)
        ex = np.exp(v - M[t_k])
        den = segment_sum(ex, t_k, N)
        g = ex / den[t_k]
        msg = g * hbar[s_k]
        A = segment_sum(msg, t_k, N)
    deg = np.diff(pk["in_ptr"].astype(np.int64))
    if cfg["aggr"] == AGGR_MEAN:
        A = A / np.maximum(deg, 1)[:, None]
    h = leaky_relu(A, slope)
    return dict(P=P, hbar=hbar, p=p, q=q, alpha=alpha, z=z, e=e, v=v, g=g, A=A, h=h)


def forward_anee(params, cfg, pk, node_feat, edge_feat):
    """Full forward with the mean readout.  node_feat [N,F_n] in graph-concatenated order;
    edge_feat [E,F_e] in INPUT edge order (permuted to in-CSR order here, step a1)."""
    h = np.asarray(node_feat, np.float64)
    e = np.asarray(edge_feat, np.float64)[pk["in_eid"].astype(np.int64)]
    layers = []
    for i in range(cfg["L"]):
        lay = anee_layer(params, i, cfg, pk, h, e)
        layers.append(lay)
        h, e = lay["h"], lay["e"]
    out = dict(layers=layers, e0=np.asarray(edge_feat, np.float64)[pk["in_eid"].astype(np.int64)],
               h0=np.asarray(node_feat, np.float64))
    if cfg.get("readout", 0) == 1 or cfg.get("graphormer", 0) > 0:
        return out                        # Graphormer layers / the decoder follow in forward()
    n_b = np.diff(pk["node_off"].astype(np.int64))
    # north_star: segmented per-graph readout, mean over nodes (R11)
    r = segment_sum(h, pk["node_graph"].astype(np.int64), pk["num_graphs"]) / n_b[:, None]
    # P125 MLP head (R12): c = W_1 r + b_1 ; o = LReLU(c) ; ŷ = w_2·o + b_2
    c = r @ params["W_1"].T + params["b_1"]
    o = leaky_relu(c, cfg["slope"])
    yhat = o @ params["w_2"] + params["b_2"][0]
    out.update(r=r, c=c, o=o, yhat=yhat)
    return out


# --------------------------------------------------------------------------
# OCCU_BF16 mode (SURVEY §8(c) "Precision modes"; R24-R27): the same
# forward with the BF16 roundings of the mode applied at the points where the
# mode stores or feeds BF16, every operation itself in float64.  It defines what
# the BF16 path computes up to FP32 summation order.
# --------------------------------------------------------------------------
def bf16_round(x):
    """Round to the nearest bfloat16, ties to even (via float32, as FP32 -> BF16 RN)."""
    b = np.ascontiguousarray(np.asarray(x, np.float64).astype(np.float32)).view(np.uint32)
    b = (b + np.uint32(0x7FFF) + ((b >> np.uint32(16)) & np.uint32(1))) & np.uint32(0xFFFF0000)
    return b.view(np.float32).astype(np.float64)


def forward_bf16(params, cfg, pk, node_feat, edge_feat, rnd=None):
    """Forward of OCCU_BF16: tensor-core GEMM operands (activations and W_u, W_e, W_m) are
    rounded to BF16 (R24); stored h̄, e', g, h are BF16 (R24); p, q come from the unrounded
    h̄ and, like α, σ, the softmax, the message product, the segment sums, the readout (over
    the unrounded last-layer h, R27) and the head, stay unrounded.  The layer-1 edge
    transform with F_e <= 16 is a CUDA-core FP32 step, not a tensor-core GEMM (R27).
    ``rnd`` replaces the rounding function (tests pass the identity to recover forward()).
    The saved fields are the ones the training backward of the mode reads (R28)."""
    r16 = bf16_round if rnd is None else rnd
    slope = cfg["slope"]
    s_k, t_k = pk["in_src"].astype(np.int64), pk["in_dst"].astype(np.int64)
    N = pk["num_nodes"]
    h = np.asarray(node_feat, np.float64)
    e = np.asarray(edge_feat, np.float64)[pk["in_eid"].astype(np.int64)]
    deg = np.diff(pk["in_ptr"].astype(np.int64))
    layers = []
    for i in range(cfg["L"]):
        W_u, W_e, W_m = params[f"W_u{i}"], params[f"W_e{i}"], params[f"W_m{i}"]
        P = r16(h) @ r16(W_u).T                                   # P141, BF16 operands
        hbar_f = leaky_relu(P, slope)
        p = hbar_f @ params[f"a_s{i}"]                            # P145/P147 (R1)
        q = hbar_f @ params[f"a_d{i}"]
        hbar = r16(hbar_f)                                        # stored BF16
        alpha = p[s_k] + q[t_k]
        tensor_core = not (i == 0 and e.shape[1] <= 16)
        z = (r16(e) @ r16(W_e).T) if tensor_core else (e @ W_e.T)   # P145
        e_new = r16(sigmoid(alpha[:, None] * z))                  # stored BF16
        if cfg.get("msg", MSG_CHANNEL_SOFTMAX) == MSG_CHANNEL_SOFTMAX:
            v = e_new @ r16(W_m).T                                # P149
            g = r16(softmax_channels(v))                          # stored BF16 (R24)
        else:
            # reading B (NEXT-1) in OCCU_BF16 (R40): the logits are stored BF16; the softmax
            # over the destination's in-edges and its weights stay unrounded
            v = r16(e_new @ r16(W_m).T)
            M = np.full((N, v.shape[1]), -np.inf)
            np.maximum.at(M, t_k, v)
            ex = np.exp(v - M[t_k])
            g = ex / segment_sum(ex, t_k, N)[t_k]
        A = segment_sum(g * hbar[s_k], t_k, N)                    # P149 (R4)
        if cfg["aggr"] == AGGR_MEAN:
            A = A / np.maximum(deg, 1)[:, None]
        h_f = leaky_relu(A, slope)
        layers.append(dict(P=P, hbar=hbar, p=p, q=q, alpha=alpha, z=z, e=e_new, g=g, A=A,
                           h=r16(h_f), h_f32=h_f))
        h, e = r16(h_f), e_new
    if cfg.get("readout", 0) == 1 or cfg.get("graphormer", 0) > 0:
        # R41: Graphormer layers / the decoder run in FP32 on the BF16-stored last h
        f = dict(layers=layers, h0=np.asarray(node_feat, np.float64),
                 e0=np.asarray(edge_feat, np.float64)[pk["in_eid"].astype(np.int64)])
        # R42: the Graphormer attention takes one fp16 product per step in this mode
        return readout_stack(params, cfg, pk, f, layers[-1]["h"],
                             att_rnd=fp16_round if rnd is None else rnd)
    n_b = np.diff(pk["node_off"].astype(np.int64))
    r = segment_sum(layers[-1]["h_f32"], pk["node_graph"].astype(np.int64), pk["num_graphs"]) / n_b[:, None]
    c = r @ params["W_1"].T + params["b_1"]                       # P125 (R12)
    o = leaky_relu(c, slope)
    yhat = o @ params["w_2"] + params["b_2"][0]
    return dict(layers=layers, h0=np.asarray(node_feat, np.float64),
                e0=np.asarray(edge_feat, np.float64)[pk["in_eid"].astype(np.int64)],
                r=r, c=c, o=o, yhat=yhat)


# --------------------------------------------------------------------------
# NEXT-2: Set-Transformer decoder readout (P159-P205; R30-R34).
#   MAB(X, Y) = LN(H̄ + FFN(H̄)),  H̄ = LN(X + MHA(X, Y, Y))          P159-P161, P191-P193
#   SAB(X) = MAB(X, X)                                               P195-P197
#   PMA_k(H) = MAB(S, FFN(H)),  S ∈ ℝ^{k×d} learnable seeds           P199-P201
#   Decoder(H) = FFN(SAB(PMA_k(H))) ∈ ℝ^{k×d}                         P203-P205
# FFN(x) = W2·ReLU(W1 x + b1) + b2 (R31); MHA with `heads` heads of width d/heads, scaled
# dot-product attention, input / output projections with biases (R32); LN = LayerNorm with
# gain and bias, eps 1e-5, biased variance (R33).  The head reads the flattened k·d output.
# --------------------------------------------------------------------------
def layer_norm(x, g, b, eps=1e-5):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    return (x - mu) / np.sqrt(var + eps) * g + b


def ffn(x, params, p):
    return np.maximum(x @ params[p + "W1"].T + params[p + "b1"], 0.0) @ params[p + "W2"].T + params[p + "b2"]


def mha(X, Y, params, m, heads, rnd=None):
    """Multi-head attention MHA(X, Y, Y): queries from X, keys and values from Y.  rnd (OCCU_BF16
    Graphormer attention, R42): the operands of the two products — Q·log2(e)/√d_h, K, V and the
    unnormalised weights 2^(s - max) — are rounded by rnd; the normaliser is the unrounded sum."""
    Q = X @ params[m + "Wq"].T + params[m + "bq"]
    K = Y @ params[m + "Wk"].T + params[m + "bk"]
    V = Y @ params[m + "Wv"].T + params[m + "bv"]
    dh = Q.shape[1] // heads
    out = np.zeros_like(Q)
    for h in range(heads):
        sl = slice(h * dh, (h + 1) * dh)
        if rnd is None:
            A = softmax_channels(Q[:, sl] @ K[:, sl].T / np.sqrt(dh))     # softmax over the keys
            out[:, sl] = A @ V[:, sl]
        else:
            S = rnd(Q[:, sl] * (np.log2(np.e) / np.sqrt(dh))) @ rnd(K[:, sl]).T
            Pu = np.exp2(S - S.max(axis=1, keepdims=True))
            out[:, sl] = (rnd(Pu) @ rnd(V[:, sl])) / Pu.sum(axis=1, keepdims=True)
    return out @ params[m + "Wo"].T + params[m + "bo"]


def mab(X, Y, params, m, heads):
    Hb = layer_norm(X + mha(X, Y, params, m, heads), params[m + "ln1_g"], params[m + "ln1_b"])
    return layer_norm(Hb + ffn(Hb, params, m + "F_"), params[m + "ln2_g"], params[m + "ln2_b"])


def set_decoder(H, params, heads):
    """Decoder(H) for one graph's node states H [n, d] -> [k, d]."""
    Z = ffn(H, params, "P_")                           # PMA's FFN(H)
    pma = mab(params["S"], Z, params, "M1_", heads)    # PMA_k
    sab = mab(pma, pma, params, "M2_", heads)          # SAB
    return ffn(sab, params, "D_")


def fp16_round(x):
    """Round to the nearest IEEE fp16 (ties to even)."""
    return np.asarray(x, np.float64).astype(np.float16).astype(np.float64)


def graphormer_layer(H, params, j, heads, att_rnd=None):
    """Graphormer layer j over one graph's node states H [n, d] (P153-P157; R35-R37):
        h̄ = MHA(LN(h)) + h,    h' = FFN(LN(h̄)) + h̄
    with self-attention over all n nodes of the graph (MHA(X, X, X), R32 heads)."""
    g = f"G{j}_"
    X = layer_norm(H, params[g + "ln1_g"], params[g + "ln1_b"])
    Hb = mha(X, X, params, g, heads, att_rnd) + H
    Y = layer_norm(Hb, params[g + "ln2_g"], params[g + "ln2_b"])
    return ffn(Y, params, g + "F_") + Hb


def readout_stack(params, cfg, pk, f, hL, att_rnd=None):
    """cfg["graphormer"] Graphormer layers per graph (NEXT-3) on the last ANEE states hL, then
    the readout — the segmented mean (a7) or, with cfg["readout"] == 1, the Set-Transformer
    decoder per graph (NEXT-2) — and the MLP head on the (flattened) readout; fills f."""
    off = pk["node_off"].astype(np.int64)
    B = pk["num_graphs"]
    gph = []
    for j in range(cfg.get("graphormer", 0)):
        hL = np.concatenate([graphormer_layer(hL[off[b]:off[b + 1]], params, j, cfg["heads"], att_rnd)
                             for b in range(B)])
        gph.append(hL)
    f["gph"] = gph
    if cfg.get("readout", 0) == 1:
        D = np.stack([set_decoder(hL[off[b]:off[b + 1]], params, cfg["heads"]) for b in range(B)])
        f["dec"] = D
        r = D.reshape(B, -1)
    else:                                 # segmented mean readout (R11)
        r = segment_sum(hL, pk["node_graph"].astype(np.int64), B) / np.diff(off)[:, None]
    c = r @ params["W_1"].T + params["b_1"]
    o = leaky_relu(c, cfg["slope"])
    f.update(r=r, c=c, o=o, yhat=o @ params["w_2"] + params["b_2"][0])
    return f


# --------------------------------------------------------------------------
# Backward of the readout stack (NEXT-2 / NEXT-3 training; P153-P205 with Adam, P273).
# Hand-derived, float64, in the forward's notation; every function returns the input
# gradient(s) and adds its parameter gradients into `grads`.  Pinned by torch autograd over
# the same forward and by central finite differences (tests/test_oracle.py).
# --------------------------------------------------------------------------
def _acc(grads, name, g):
    grads[name] = grads[name] + g if name in grads else g


def layer_norm_bwd(x, g, dy, eps=1e-5):
    """y = x̂·g + b, x̂ = (x - μ)/sqrt(σ² + eps) per row (R33) -> (dx, dg, db)."""
    mu = x.mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(((x - mu) ** 2).mean(axis=-1, keepdims=True) + eps)
    xh = (x - mu) * rstd
    dxh = dy * g
    dx = rstd * (dxh - dxh.mean(axis=-1, keepdims=True) - xh * (dxh * xh).mean(axis=-1, keepdims=True))
    return dx, (dy * xh).sum(axis=0), dy.sum(axis=0)


def ffn_bwd(x, params, p, dy, grads):
    """FFN(x) = W2·ReLU(W1 x + b1) + b2 (R31)."""
    a = x @ params[p + "W1"].T + params[p + "b1"]
    t = np.maximum(a, 0.0)
    _acc(grads, p + "W2", dy.T @ t)
    _acc(grads, p + "b2", dy.sum(axis=0))
    da = (dy @ params[p + "W2"]) * (a > 0)
    _acc(grads, p + "W1", da.T @ x)
    _acc(grads, p + "b1", da.sum(axis=0))
    return da @ params[p + "W1"]


def mha_bwd(X, Y, params, m, heads, dout, grads):
    """MHA(X, Y, Y) of ``mha`` (R32) -> (dX, dY)."""
    Q = X @ params[m + "Wq"].T + params[m + "bq"]
    K = Y @ params[m + "Wk"].T + params[m + "bk"]
    V = Y @ params[m + "Wv"].T + params[m + "bv"]
    dh = Q.shape[1] // heads
    O = np.zeros_like(Q)
    As = []
    for h in range(heads):
        sl = slice(h * dh, (h + 1) * dh)
        A = softmax_channels(Q[:, sl] @ K[:, sl].T / np.sqrt(dh))
        O[:, sl] = A @ V[:, sl]
        As.append(A)
    _acc(grads, m + "Wo", dout.T @ O)
    _acc(grads, m + "bo", dout.sum(axis=0))
    dO = dout @ params[m + "Wo"]
    dQ, dK, dV = np.zeros_like(Q), np.zeros_like(K), np.zeros_like(V)
    for h in range(heads):
        sl = slice(h * dh, (h + 1) * dh)
        A = As[h]
        dA = dO[:, sl] @ V[:, sl].T
        dV[:, sl] = A.T @ dO[:, sl]
        dS = A * (dA - np.sum(dA * A, axis=1, keepdims=True)) / np.sqrt(dh)
        dQ[:, sl] = dS @ K[:, sl]
        dK[:, sl] = dS.T @ Q[:, sl]
    for w, dW, inp in (("q", dQ, X), ("k", dK, Y), ("v", dV, Y)):
        _acc(grads, m + "W" + w, dW.T @ inp)
        _acc(grads, m + "b" + w, dW.sum(axis=0))
    return dQ @ params[m + "Wq"], dK @ params[m + "Wk"] + dV @ params[m + "Wv"]


def mab_bwd(X, Y, params, m, heads, dout, grads):
    """MAB(X, Y) = LN2(H̄ + FFN(H̄)), H̄ = LN1(X + MHA(X, Y, Y)) -> (dX, dY)."""
    T1 = X + mha(X, Y, params, m, heads)
    Hb = layer_norm(T1, params[m + "ln1_g"], params[m + "ln1_b"])
    T2 = Hb + ffn(Hb, params, m + "F_")
    dT2, dg, db = layer_norm_bwd(T2, params[m + "ln2_g"], dout)
    _acc(grads, m + "ln2_g", dg)
    _acc(grads, m + "ln2_b", db)
    dHb = dT2 + ffn_bwd(Hb, params, m + "F_", dT2, grads)
    dT1, dg, db = layer_norm_bwd(T1, params[m + "ln1_g"], dHb)
    _acc(grads, m + "ln1_g", dg)
    _acc(grads, m + "ln1_b", db)
    dXa, dY = mha_bwd(X, Y, params, m, heads, dT1, grads)
    return dT1 + dXa, dY


def set_decoder_bwd(H, params, heads, dD, grads):
    """Backward of ``set_decoder`` for one graph: dD [k, d] -> dH [n, d] (+ dS, parameters)."""
    Z = ffn(H, params, "P_")
    pma = mab(params["S"], Z, params, "M1_", heads)
    sab = mab(pma, pma, params, "M2_", heads)
    dsab = ffn_bwd(sab, params, "D_", dD, grads)
    dx, dy = mab_bwd(pma, pma, params, "M2_", heads, dsab, grads)
    dS, dZ = mab_bwd(params["S"], Z, params, "M1_", heads, dx + dy, grads)
    _acc(grads, "S", dS)
    return ffn_bwd(H, params, "P_", dZ, grads)


def graphormer_layer_bwd(H, params, j, heads, dout, grads):
    """Backward of ``graphormer_layer`` (P155, P157) for one graph: dout -> dH."""
    g = f"G{j}_"
    X = layer_norm(H, params[g + "ln1_g"], params[g + "ln1_b"])
    Hb = mha(X, X, params, g, heads) + H
    Y = layer_norm(Hb, params[g + "ln2_g"], params[g + "ln2_b"])
    dY = ffn_bwd(Y, params, g + "F_", dout, grads)
    dHb2, dg, db = layer_norm_bwd(Hb, params[g + "ln2_g"], dY)
    _acc(grads, g + "ln2_g", dg)
    _acc(grads, g + "ln2_b", db)
    dHb = dout + dHb2
    dXq, dXkv = mha_bwd(X, X, params, g, heads, dHb, grads)
    dH1, dg, db = layer_norm_bwd(H, params[g + "ln1_g"], dXq + dXkv)
    _acc(grads, g + "ln1_g", dg)
    _acc(grads, g + "ln1_b", db)
    return dHb + dH1


def readout_stack_bwd(params, cfg, pk, fwd, dr, grads):
    """dr = ∂L/∂r (the head's input) -> ∂L/∂h_L of the ANEE stack, through the decoder (or
    the segmented mean) and the Graphormer layers in reverse, per graph."""
    off = pk["node_off"].astype(np.int64)
    B = pk["num_graphs"]
    G = cfg.get("graphormer", 0)
    hL = fwd["layers"][-1]["h"]
    ins = [hL] + list(fwd["gph"][:-1]) if G else []
    top = fwd["gph"][-1] if G else hL
    if cfg.get("readout", 0) == 1:
        dD = dr.reshape(B, cfg["k"], cfg["d"])
        dh = np.concatenate([set_decoder_bwd(top[off[b]:off[b + 1]], params, cfg["heads"], dD[b], grads)
                             for b in range(B)])
    else:
        n_b = np.diff(off)
        gidx = pk["node_graph"].astype(np.int64)
        dh = dr[gidx] / n_b[gidx][:, None]
    for j in range(G - 1, -1, -1):
        dh = np.concatenate([graphormer_layer_bwd(ins[j][off[b]:off[b + 1]], params, j, cfg["heads"],
                                                  dh[off[b]:off[b + 1]], grads) for b in range(B)])
    return dh


def forward(params, cfg, pk, node_feat, edge_feat):
    """forward_anee, then (with Graphormer layers or the decoder readout) readout_stack."""
    f = forward_anee(params, cfg, pk, node_feat, edge_feat)
    if cfg.get("readout", 0) != 1 and cfg.get("graphormer", 0) == 0:
        return f
    return readout_stack(params, cfg, pk, f, f["layers"][-1]["h"])


def predict(params, cfg, graphs, node_feat, edge_feat):
    return forward(params, cfg, pack(graphs), node_feat, edge_feat)["yhat"]


# --------------------------------------------------------------------------
# Step a9: MSE loss (P209-P213), normalised by the GLOBAL batch (R15).
# --------------------------------------------------------------------------
def mse_loss(yhat, y, global_batch=None):
    nb = len(yhat) if global_batch is None else global_batch
    return float(np.sum((np.asarray(yhat, np.float64) - np.asarray(y, np.float64)) ** 2) / nb)


# --------------------------------------------------------------------------
# Step BW: hand-derived backward of the forward above (reading A), float64.
# --------------------------------------------------------------------------
def backward(params, cfg, pk, fwd, y, global_batch=None, dsig=None):
    """dsig(layer dict) -> σ'(y) per edge and channel; default e'(1 - e') (exact
    derivative of σ at y = α z).  backward_bf16 passes e'·σ(-α z) (R28)."""
    slope = cfg["slope"]
    B = pk["num_graphs"]
    nb = B if global_batch is None else global_batch
    s_k, t_k = pk["in_src"].astype(np.int64), pk["in_dst"].astype(np.int64)
    N = pk["num_nodes"]
    grads = {}
    # loss and head
    dy = 2.0 * (fwd["yhat"] - np.asarray(y, np.float64)) / nb
    grads["w_2"] = fwd["o"].T @ dy
    grads["b_2"] = np.array([dy.sum()])
    dc = (dy[:, None] * params["w_2"][None, :]) * leaky_relu_grad(fwd["c"], slope)
    grads["W_1"] = dc.T @ fwd["r"]
    grads["b_1"] = dc.sum(axis=0)
    dr = dc @ params["W_1"]
    if cfg.get("readout", 0) == 1 or cfg.get("graphormer", 0) > 0:
        # NEXT-2 / NEXT-3: through the decoder readout and the Graphormer layers
        dh = readout_stack_bwd(params, cfg, pk, fwd, dr, grads)
    else:
        n_b = np.diff(pk["node_off"].astype(np.int64))
        gidx = pk["node_graph"].astype(np.int64)
        dh = dr[gidx] / n_b[gidx][:, None]
    de_out = None
    deg = np.diff(pk["in_ptr"].astype(np.int64))
    for i in range(cfg["L"] - 1, -1, -1):
        lay = fwd["layers"][i]
        h_prev = fwd["layers"][i - 1]["h"] if i > 0 else fwd["h0"]
        e_prev = fwd["layers"][i - 1]["e"] if i > 0 else fwd["e0"]
        W_u, W_e, W_m = params[f"W_u{i}"], params[f"W_e{i}"], params[f"W_m{i}"]
        a_s, a_d = params[f"a_s{i}"], params[f"a_d{i}"]
        hbar, g, e, z, alpha = lay["hbar"], lay["g"], lay["e"], lay["z"], lay["alpha"]
        dA = dh * leaky_relu_grad(lay["A"], slope)
        if cfg["aggr"] == AGGR_MEAN:
            dA = dA / np.maximum(deg, 1)[:, None]
        dm = dA[t_k]
        dg = dm * hbar[s_k]
        dhbar = segment_sum(dm * g, s_k, N)
        if cfg.get("msg", MSG_CHANNEL_SOFTMAX) == MSG_CHANNEL_SOFTMAX:
            dv = g * (dg - np.sum(g * dg, axis=1, keepdims=True))
        else:
            # segmented (over in-edges of t, per channel) softmax backward
            dv = g * (dg - segment_sum(g * dg, t_k, N)[t_k])
        grads[f"W_m{i}"] = dv.T @ e
        de = dv @ W_m                      # de_k = W_m^T dv_k
        if de_out is not None:
            de = de + de_out
        dyk = de * (e * (1.0 - e) if dsig is None else dsig(lay))
        dalpha = np.sum(dyk * z, axis=1)
        dz = alpha[:, None] * dyk
        grads[f"W_e{i}"] = dz.T @ e_prev
        de_out = dz @ W_e
        dp = segment_sum(dalpha, s_k, N)
        dq = segment_sum(dalpha, t_k, N)
        grads[f"a_s{i}"] = hbar.T @ dp
        grads[f"a_d{i}"] = hbar.T @ dq
        dhbar = dhbar + dp[:, None] * a_s[None, :] + dq[:, None] * a_d[None, :]
        dP = dhbar * leaky_relu_grad(lay["P"], slope)
        grads[f"W_u{i}"] = dP.T @ h_prev
        dh = dP @ W_u
    loss = mse_loss(fwd["yhat"], y, nb)
    return loss, grads


def loss_and_grads(params, cfg, graphs, node_feat, edge_feat, y, global_batch=None):
    pk = pack(graphs)
    fwd = forward(params, cfg, pk, node_feat, edge_feat)
    return backward(params, cfg, pk, fwd, y, global_batch)


def backward_bf16(params, cfg, pk, fwd, y, global_batch=None):
    """Step BW of OCCU_BF16 training (SURVEY §8(c) "Precision modes": all gradients FP32;
    DESIGN.md R28): the hand-derived backward above evaluated on what the BF16 forward
    saved — h̄, e', g and h as BF16 values, z as the mode computes it (BF16 operands on the
    tensor cores), p, q, α, A and the head state unrounded — with the gradient GEMMs against
    the unrounded weights and σ'(y) = e'·σ(-α z) (stored e', recomputed z)."""
    return backward(params, cfg, pk, fwd, y, global_batch,
                    dsig=lambda lay: lay["e"] * sigmoid(-lay["alpha"][:, None] * lay["z"]))


def loss_and_grads_bf16(params, cfg, graphs, node_feat, edge_feat, y, global_batch=None):
    pk = pack(graphs)
    fwd = forward_bf16(params, cfg, pk, node_feat, edge_feat)
    return backward_bf16(params, cfg, pk, fwd, y, global_batch)


# --------------------------------------------------------------------------
# Step O: Adam (P273 "default hyperparameters", lr = weight decay = 1e-4; R16:
# PyTorch torch.optim.Adam semantics, L2 weight decay added to the gradient).
# --------------------------------------------------------------------------
def adam_step(params, grads, state, lr, wd=1e-4, beta1=0.9, beta2=0.999, eps=1e-8):
    """Returns (new_params, new_state); state = dict(t, m{name}, v{name})."""
    t = state.get("t", 0) + 1
    new_p, m_new, v_new = {}, {}, {}
    for name, w in params.items():
        gr = grads[name] + wd * w
        m = beta1 * state.get("m", {}).get(name, np.zeros_like(w)) + (1 - beta1) * gr
        v = beta2 * state.get("v", {}).get(name, np.zeros_like(w)) + (1 - beta2) * gr * gr
        mhat = m / (1 - beta1 ** t)
        vhat = v / (1 - beta2 ** t)
        new_p[name] = w - lr * mhat / (np.sqrt(vhat) + eps)
        m_new[name], v_new[name] = m, v
    return new_p, {"t": t, "m": m_new, "v": v_new}


# --------------------------------------------------------------------------
# NEXT-4 consumer: occu-packing (P390-P392; R38).  "an appropriate packing
# policy for multiple jobs should ensure the cumulative occupancy is at most 100%" (P390);
# "a GPU-occupancy-based bin-packing algorithm (with co-location ensuring GPU occupancy does
# not exceed 100%)" (P392).  Reading R38: first fit in submission order; job j goes to the
# lowest-numbered GPU slot b with load_b + occ_j <= capacity (float64 arithmetic on the
# float32 predictions, loads summed in placement order), else a new slot is opened;
# predictions below 0 count as 0.  Plain O(jobs x slots) loop.
# --------------------------------------------------------------------------
def occu_packing(occ, capacity=1.0):
    occ = np.maximum(np.asarray(occ, np.float32).astype(np.float64), 0.0)
    loads = []
    assign = np.empty(len(occ), np.int32)
    for j, o in enumerate(occ):
        for b, ld in enumerate(loads):
            if ld + o <= capacity:
                loads[b] = ld + o
                assign[j] = b
                break
        else:
            loads.append(o)
            assign[j] = len(loads) - 1
    return assign, np.array(loads, np.float64)
