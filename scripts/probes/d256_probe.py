"""d = 256 probe: one small predict through the CTA-pair path vs the oracle (prints errors)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from occu_gen import configs, weights  # noqa: E402
from paper_conf_cluster_meiqsgls23_b200 import occu  # noqa: E402

for L, n, mx in ((1, 4, 10), (1, 40, 60), (2, 40, 60), (3, 40, 60)):
    c = occu.config(L=L, F_n=80, F_e=4, d=256)
    wc = weights.ModelConfig(L=L, F_n=80, F_e=4, d=256, d_h=256, aggr=0)
    flat = weights.unit_scale(wc, weights.init_flat(wc, 1))
    b = configs.random_dag_batch(n, 70 + L, max_nodes=mx, hub=True)
    m = occu.Model(c)
    m.set_params(flat)
    m.keep_intermediates(True)
    csr = occu.pack(b.graphs)
    t = time.time()
    y = m.predict(csr, b.node_feat, b.edge_feat)
    torch.cuda.synchronize()
    ocf = dict(L=L, F_n=80, F_e=4, d=256, d_h=256, aggr=0, msg=0, slope=float(np.float32(0.01)))
    params = oracle.unflatten(ocf, flat.astype(np.float64))
    pk = oracle.pack(b.graphs)
    ref = oracle.forward(params, ocf, pk, b.node_feat, b.edge_feat)
    N, E = pk["num_nodes"], pk["num_edges"]
    out = [f"L={L} N={N} E={E} t={time.time() - t:.2f}s"]
    for i in range(L):
        lay = ref["layers"][i]
        for name, tt, shape in (("hbar", occu.T_HBAR, (N, 256)), ("p", occu.T_P, (N,)), ("e", occu.T_E, (E, 256)),
                                ("h", occu.T_H, (N, 256))):
            got = m.get_tensor(tt, i, shape)
            r = np.linalg.norm(got - lay[name]) / max(np.linalg.norm(lay[name]), 1e-30)
            out.append(f"{name}{i}={r:.2e}")
    out.append(f"yhat={np.max(np.abs(y - ref['yhat']) / np.maximum(np.abs(ref['yhat']), 1e-2)):.2e}")
    print(" ".join(out), flush=True)
