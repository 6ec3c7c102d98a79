import os, sys
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np, torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
b = configs.cfg2(16)
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64)); m.init_weights(1)
nf = torch.from_numpy(b.node_feat).pin_memory(); ef = torch.from_numpy(b.edge_feat).pin_memory()
y = torch.from_numpy(b.targets).pin_memory(); lo = [torch.zeros(1).pin_memory() for _ in range(2)]
g_nn = np.array([g[0] for g in b.graphs], np.int32); g_ne = np.array([len(g[1]) for g in b.graphs], np.int64)
s = np.concatenate([g[1] for g in b.graphs]).astype(np.int32); d = np.concatenate([g[2] for g in b.graphs]).astype(np.int32)
for k in range(6):
    hc = occu.pack_arrays(g_nn, g_ne, s, d)
    m.train_step_async(hc, nf, ef, y, 1e-3, out_loss=lo[k & 1])
m.wait(); print("async ok", float(lo[0][0]), float(lo[1][0]))
