"""Small training steps (FP32 reading A / B, BF16) for compute-sanitizer."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
b = configs.random_dag_batch(5, 9, max_nodes=140, hub=True)
for cfg in (occu.config(L=3, d=128), occu.config(L=2, d=64, aggr=occu.AGGR_MEAN),
            occu.config(L=2, d=128, msg=occu.MSG_NEIGHBOR_SOFTMAX), occu.config(L=3, d=128, prec=occu.BF16)):
    m = occu.Model(cfg)
    m.init_weights(4)
    csr = occu.pack(b.graphs)
    l1 = m.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-3)
    l2 = m.train_step(csr, b.node_feat, b.edge_feat, b.targets, 1e-3)
    print("ok", l1, l2)
torch.cuda.synchronize()
