"""Helper for tests/test_gpu_ab_switches.py: one compute_grads on a fixed seeded batch, the
flat gradient written to argv[1] (.npy).  Run in a subprocess so that the library's
environment A/B switches (read once per process) take effect."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from occu_gen import configs, weights  # noqa: E402
from paper_conf_cluster_meiqsgls23_b200 import occu  # noqa: E402

prec = occu.BF16 if os.environ.get("AB_PREC") == "bf16" else occu.FP32
aggr = int(os.environ.get("AB_AGGR", "0"))
b = configs.cfg2(16)
c = occu.config(L=3, F_n=80, F_e=4, d=128, aggr=aggr, prec=prec)
wc = weights.ModelConfig(L=3, F_n=80, F_e=4, d=128, d_h=128, aggr=aggr)
m = occu.Model(c)
m.set_params(weights.unit_scale(wc, weights.init_flat(wc, 3)))
y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)          # inference path too
loss = m.compute_grads(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets)
np.save(sys.argv[1], np.concatenate([m.get_grads(), np.array([loss], np.float32), y.astype(np.float32)]))
