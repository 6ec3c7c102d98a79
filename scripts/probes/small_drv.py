import os, sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
b1 = configs.cfg1(); dev = torch.device("cuda", 0)
nf = torch.from_numpy(b1.node_feat).to(dev); ef = torch.from_numpy(b1.edge_feat).to(dev)
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64)); m.init_weights(42); m.set_small_batch_kernel(True)
csr = m.to_device(occu.pack(b1.graphs)); out = torch.empty(1, device=dev)
for _ in range(5): m.predict(csr, nf, ef, out)
torch.cuda.synchronize(); print("ok")
