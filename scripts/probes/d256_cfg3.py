"""d = 256 pair kernels on CFG3-sized inputs (L = 1): per-kernel time and HBM fraction, to
separate small-batch overheads (CFG2-paper) from the kernels' streaming rate."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
b = configs.cfg3(512); dev = torch.device("cuda", 0)
N, E = b.num_nodes, b.num_edges
nf = torch.from_numpy(b.node_feat).to(dev); ef = torch.from_numpy(b.edge_feat).to(dev)
for prec, sa in ((occu.FP32, 4), (occu.BF16, 2)):
    m = occu.Model(occu.config(L=1, F_n=80, F_e=4, d=256, prec=prec)); m.init_weights(42)
    csr = m.to_device(occu.pack(b.graphs)); out = torch.empty(b.num_graphs, device=dev)
    for _ in range(3): m.predict(csr, nf, ef, out)
    torch.cuda.synchronize()
    m.set_profiling(True)
    m.profile_reset()
    for _ in range(5): m.predict(csr, nf, ef, out)
    torch.cuda.synchronize()
    prof = m.profile()
    m.set_profiling(False)
    by = {"gate_tc": 2 * sa * E * 256, "node_tc": 4 * N * 80 + sa * N * 256 + 8 * N,
          "edge_small": 4 * E * 4 + 12 * E + 8 * N + sa * E * 256}
    for k, (ms, n) in prof.items():
        t = ms / 5
        f = by.get(k)
        print(prec, k, round(t * 1e3, 1), "us", (round(f / (t * 1e-3) / 1e9 / 6545.9, 3) if f else ""))
    del m, csr
