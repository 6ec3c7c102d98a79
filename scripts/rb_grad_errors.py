"""Per-tensor gradient errors (GPU vs float64 oracle) for reading A / B, SUM / MEAN, with the
'wide' weight set of tests/test_gpu_readingb.py (W_m, a_s, a_d x 8)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu

for msg in (0, 1):
    for aggr in (0, 1):
        L, d = 3, 128
        c = occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, msg=msg)
        wc = weights.ModelConfig(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr, msg=msg)
        ocf = dict(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr, msg=msg, slope=float(np.float32(0.01)))
        b = configs.random_dag_batch(24, 950 + L + aggr, max_nodes=50, hub=True)
        flat = weights.init_flat(wc, 11).copy()
        off = 0
        for name, shape in oracle.param_shapes(ocf):
            n = int(np.prod(shape))
            if name.startswith("W_m") or name.startswith("a_"):
                flat[off:off + n] *= 8.0
            off += n
        params = oracle.unflatten(ocf, flat.astype(np.float64))
        lr_, gr = oracle.loss_and_grads(params, ocf, b.graphs, b.node_feat, b.edge_feat, b.targets)
        m = occu.Model(c)
        m.set_params(flat)
        loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets)
        g = weights.unflatten(wc, m.get_grads())
        rel = lambda a, r: float(np.linalg.norm(np.asarray(a, np.float64) - r) / max(np.linalg.norm(r), 1e-300))
        print(f"msg={msg} aggr={aggr}: loss {abs(loss-lr_)/lr_:.2e}", {k: f"{rel(g[k], gr[k]):.1e}" for k in gr})
        for k in gr:
            if not np.isfinite(g[k]).all():
                print("   nonfinite", k, int((~np.isfinite(g[k])).sum()), "of", g[k].size)
