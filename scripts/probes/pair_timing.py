"""Per-role busy / wait cycles of CTA 0 of the d = 256 gate pair kernel (rowgemm_pair_kernel
<EPI_GATE>): builds a -DOCCU_TC_TIMING copy of the library, runs CFG2-paper (L = 1) predicts."""
import ctypes, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
from paper_conf_cluster_meiqsgls23_b200 import build as B
objdir = os.path.join(ROOT, "build", "tc_timing"); os.makedirs(objdir, exist_ok=True)
inc, libd = B.nccl_dirs(); objs = []
for src in B.sources():
    obj = os.path.join(objdir, os.path.basename(src) + ".o")
    flags = ["-DOCCU_TC_TIMING"] if src.endswith(".cu") else []
    cmd = ["nvcc", *(B.ARCH if src.endswith(".cu") else []), "-O3", "-std=c++17", "--expt-relaxed-constexpr", *flags, "-Xcompiler", "-fPIC",
           "-I", os.path.join(ROOT, "include"), "-I", inc] + (["-x", "c++"] if src.endswith(".cpp") else []) + ["-c", src, "-o", obj]
    subprocess.run(cmd, check=True); objs.append(obj)
lib = os.path.join(objdir, "libocc_tct.so")
subprocess.run(["nvcc", *B.ARCH, "-shared", "-o", lib, *objs, "-L", libd, "-l:libnccl.so.2", "-Xlinker", f"-rpath={libd}", "-lcudart"], check=True)
from paper_conf_cluster_meiqsgls23_b200 import occu
occu.LIB_PATH = lib
import numpy as np, torch
from occu_gen import configs
b = configs.cfg2(256); dev = torch.device("cuda", 0)
nf = torch.from_numpy(b.node_feat).to(dev); ef = torch.from_numpy(b.edge_feat).to(dev)
m = occu.Model(occu.config(L=1, F_n=80, F_e=4, d=256)); m.init_weights(42)
csr = m.to_device(occu.pack(b.graphs)); out = torch.empty(256, device=dev)
f = occu.lib().occu_debug_tc_time
for _ in range(3): m.predict(csr, nf, ef, out)
torch.cuda.synchronize()
buf = np.zeros((32, 4), np.uint64)
f(buf.ctypes.data_as(ctypes.c_void_p))          # reset
R = 10
for _ in range(R): m.predict(csr, nf, ef, out)
torch.cuda.synchronize()
f(buf.ctypes.data_as(ctypes.c_void_p))
names = ["producer", "mma"] + [f"conv{i}" for i in range(4)] + [f"epi{i}" for i in range(16)]
for i, n in enumerate(names):
    w, bz, c = (int(x) for x in buf[i, :3])
    if c:
        print(f"{n:9s} wait {w / R / 1e3:8.1f} kcyc  busy {bz / R / 1e3:8.1f} kcyc  per launch")
