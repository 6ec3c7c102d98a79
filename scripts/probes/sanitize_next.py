"""Small runs of the NEXT-row kernels for compute-sanitizer (memcheck / racecheck)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch
from occu_gen import configs, templates
from paper_conf_cluster_meiqsgls23_b200 import occu
b = configs.random_dag_batch(6, 5, max_nodes=150, hub=True)
for cfg in (occu.config(L=2, d=128, graphormer=2, heads=4, readout=occu.READOUT_SET_DECODER, k=4),
            occu.config(L=2, d=64, graphormer=1, heads=2),
            occu.config(L=2, d=128, msg=occu.MSG_NEIGHBOR_SOFTMAX, prec=occu.BF16)):
    m = occu.Model(cfg)
    m.init_weights(3)
    y = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
    print("ok", y[:2])
m = occu.Model(occu.config(L=2, d=64))
m.init_weights(1)
m.set_small_batch_kernel(True)
c1 = configs.cfg1()
print("small", m.predict(occu.pack(c1.graphs), c1.node_feat, c1.edge_feat))
t = m.template(templates.build_template("lenet5"))
csr, nf, ef = m.synthesize([t, t], np.array([[16, 1, 0, 0], [32, 3, 0, 0]], np.float32))
print("synth", m.predict(csr, nf, ef).cpu().numpy())
torch.cuda.synchronize()
