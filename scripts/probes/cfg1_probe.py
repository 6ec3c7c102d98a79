"""Probe: CFG1 forward (small-batch kernel) for ncu."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
dev = torch.device("cuda", 0)
b = configs.cfg1()
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64))
m.init_weights(42)
csr = m.to_device(occu.pack(b.graphs))
nf = torch.from_numpy(b.node_feat).to(dev); ef = torch.from_numpy(b.edge_feat).to(dev)
out = torch.empty(1, device=dev)
for _ in range(5):
    m.predict(csr, nf, ef, out)
torch.cuda.synchronize()
print("done")
