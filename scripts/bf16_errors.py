"""Per-tensor rel-L2 error of the OCCU_BF16 path vs the float64 oracle (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu


def rel(a, b):
    a = np.asarray(a, np.float64); b = np.asarray(b, np.float64)
    return np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-300)


for (L, d, aggr, seed) in [(2, 64, 0, 1), (3, 128, 0, 2), (3, 128, 1, 3)]:
    for ws in ("unit", "default"):
        c = occu.config(L=L, F_n=80, F_e=4, d=d, aggr=aggr, prec=occu.BF16)
        wc = weights.ModelConfig(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr)
        flat = weights.init_flat(wc, seed)
        if ws == "unit":
            flat = weights.unit_scale(wc, flat)
        b = configs.random_dag_batch(40, 300 + seed, max_nodes=60, hub=True)
        m = occu.Model(c); m.set_params(flat); m.keep_intermediates(True)
        y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
        oc = dict(L=L, F_n=80, F_e=4, d=d, d_h=d, aggr=aggr, msg=0, slope=float(np.float32(0.01)))
        pk = oracle.pack(b.graphs)
        ref = oracle.forward(oracle.unflatten(oc, flat.astype(np.float64)), oc, pk, b.node_feat, b.edge_feat)
        N, E, B = pk["num_nodes"], pk["num_edges"], pk["num_graphs"]
        out = []
        for i in range(L):
            lay = ref["layers"][i]
            out.append(f"L{i}: hbar {rel(m.get_tensor(occu.T_HBAR, i, (N, d)), lay['hbar']):.2e} "
                       f"p {rel(m.get_tensor(occu.T_P, i, (N,)), lay['p']):.2e} "
                       f"e {rel(m.get_tensor(occu.T_E, i, (E, d)), lay['e']):.2e} "
                       f"h {rel(m.get_tensor(occu.T_H, i, (N, d)), lay['h']):.2e}")
        print((L, d, aggr, seed, ws), " | ".join(out),
              f"| r {rel(m.get_tensor(occu.T_R, 0, (B, d)), ref['r']):.2e} y {rel(y, ref['yhat']):.2e}")
