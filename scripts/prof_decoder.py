"""ncu driver: CFG2 inference with the Set-Transformer decoder readout (NEXT-2)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128, readout=occu.READOUT_SET_DECODER, k=4, heads=4))
m.init_weights(42)
b = configs.cfg2(256)
csr = m.to_device(occu.pack(b.graphs))
nf = torch.from_numpy(b.node_feat).cuda(); ef = torch.from_numpy(b.edge_feat).cuda()
for _ in range(2):
    m.predict(csr, nf, ef)
torch.cuda.synchronize()
print("done")
