"""OCCU_BF16 training: per-tensor gradient errors of the GPU path against the oracle's
BF16-mode backward (oracle.backward_bf16) and the plain float64 backward (R28)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu

for (L, d, aggr, wset) in [(2, 64, 0, "unit"), (3, 128, 0, "unit"), (3, 128, 1, "unit"), (3, 128, 0, "default")]:
    c = occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, prec=occu.BF16)
    wc = weights.ModelConfig(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr)
    ocf = dict(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr, msg=0, slope=float(np.float32(0.01)))
    b = configs.random_dag_batch(int(os.environ.get("NG", 24)), 503 + L + aggr, max_nodes=50, hub=True)
    flat = weights.init_flat(wc, 11)
    if wset == "unit":
        flat = weights.unit_scale(wc, flat)
    params = oracle.unflatten(ocf, flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    le, ge = oracle.backward_bf16(params, ocf, pk, oracle.forward_bf16(params, ocf, pk, b.node_feat, b.edge_feat), b.targets)
    lr_, gr = oracle.loss_and_grads(params, ocf, b.graphs, b.node_feat, b.edge_feat, b.targets)
    m = occu.Model(c)
    m.set_params(flat)
    loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets)
    g = weights.unflatten(wc, m.get_grads())
    rel = lambda a, r: float(np.linalg.norm(np.asarray(a, np.float64) - r) / max(np.linalg.norm(r), 1e-300))
    print(f"L={L} d={d} aggr={aggr} {wset}: loss vs emu {abs(loss-le)/le:.2e} vs f64 {abs(loss-lr_)/lr_:.2e}")
    print("  vs emu:", {k: f"{rel(g[k], ge[k]):.1e}" for k in ge})
    print("  vs f64:", {k: f"{rel(g[k], gr[k]):.1e}" for k in gr})
    print("  emu vs f64:", {k: f"{rel(ge[k], gr[k]):.1e}" for k in gr})
