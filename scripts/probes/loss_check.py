"""Probe: FP32 vs BF16 loss / predictions on the same batch (device inputs)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
dev = torch.device("cuda", 0)
b = configs.cfg2(64)
for prec in (occu.FP32, occu.BF16):
    m = occu.Model(occu.config(L=3, d=128, prec=prec))
    m.init_weights(42)
    csr = m.to_device(occu.pack(b.graphs))
    nf = torch.from_numpy(b.node_feat).to(dev); ef = torch.from_numpy(b.edge_feat).to(dev)
    yt = torch.from_numpy(b.targets).to(dev)
    y = m.predict(csr, nf, ef)
    torch.cuda.synchronize()
    yh = m.predict(occu.pack(b.graphs), b.node_feat, b.edge_feat)
    l1 = m.train_step(csr, nf, ef, yt, 1e-3)
    l2 = m.train_step(csr, nf, ef, yt, 1e-3)
    lh = m.train_step(occu.pack(b.graphs), b.node_feat, b.edge_feat, b.targets, 1e-3)
    print(prec, y[:4].tolist(), yh[:4].tolist(), l1, l2, lh, float(((torch.as_tensor(yh) - torch.as_tensor(b.targets))**2).mean()))
