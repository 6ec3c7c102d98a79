import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from occu_gen import configs, weights
from paper_conf_cluster_meiqsgls23_b200 import occu
c = occu.config(L=3, F_n=80, F_e=4, d=128, aggr=0)
wc = weights.ModelConfig(L=3, F_n=80, F_e=4, d=128, d_h=128)
ocf = dict(L=3, F_n=80, F_e=4, d=128, d_h=128, aggr=0, msg=0, slope=float(np.float32(0.01)))
b = configs.random_dag_batch(24, 503, max_nodes=50, hub=True)
flat = weights.unit_scale(wc, weights.init_flat(wc, 11))
params = oracle.unflatten(ocf, flat.astype(np.float64))
lref, gref = oracle.loss_and_grads(params, ocf, b.graphs, b.node_feat, b.edge_feat, b.targets)
for path in (0, 1):
    m = occu.Model(c); m.set_kernel_path(path); m.set_params(flat)
    loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets)
    g = weights.unflatten(wc, m.get_grads())
    errs = {k: float(np.linalg.norm(g[k] - gref[k]) / np.linalg.norm(gref[k])) for k in gref}
    print(path, 'loss', abs(loss - lref) / lref, {k: f"{v:.2e}" for k, v in errs.items()})
