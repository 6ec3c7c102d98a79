"""Breakdown of the e2e step (bench.py e2e): host pack, H2D + forward + D2H through occu_predict."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
b = configs.cfg2(256)
m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128)); m.init_weights(42)
pin_nf = torch.from_numpy(b.node_feat).pin_memory(); pin_ef = torch.from_numpy(b.edge_feat).pin_memory()
out = torch.empty(256).pin_memory()
dnf = pin_nf.cuda(); torch.cuda.synchronize()
for it in range(3):
    t0 = time.perf_counter(); hc = occu.pack(b.graphs); t1 = time.perf_counter()
    m.predict(hc, pin_nf, pin_ef, out); t2 = time.perf_counter()
    x = torch.empty_like(pin_nf, device="cuda"); torch.cuda.synchronize(); t3 = time.perf_counter()
    x.copy_(pin_nf, non_blocking=True); torch.cuda.synchronize(); t4 = time.perf_counter()
    print(f"pack {1e3*(t1-t0):.3f} ms  predict(host ptrs) {1e3*(t2-t1):.3f} ms  H2D node_feat alone {1e3*(t4-t3):.3f} ms ({pin_nf.numel()*4/(t4-t3)/1e9:.1f} GB/s)", flush=True)
print("cores", len(os.sched_getaffinity(0)))
