"""Stage timestamps (clock64, thread 0) of the single-CTA small-batch forward: builds a
-DOCCU_SMALL_TIMING copy of the library and prints the cycle deltas between barriers."""
import ctypes, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
from paper_conf_cluster_meiqsgls23_b200 import build as B
objdir = os.path.join(ROOT, "build", "small_timing"); os.makedirs(objdir, exist_ok=True)
inc, libd = B.nccl_dirs(); objs = []
for src in B.sources():
    obj = os.path.join(objdir, os.path.basename(src) + ".o")
    flags = ["-DOCCU_SMALL_TIMING"] if src.endswith(".cu") else []
    cmd = ["nvcc", *(B.ARCH if src.endswith(".cu") else []), "-O3", "-std=c++17", "--expt-relaxed-constexpr", *flags, "-Xcompiler", "-fPIC",
           "-I", os.path.join(ROOT, "include"), "-I", inc] + (["-x", "c++"] if src.endswith(".cpp") else []) + ["-c", src, "-o", obj]
    subprocess.run(cmd, check=True); objs.append(obj)
lib = os.path.join(objdir, "libocc_small.so")
subprocess.run(["nvcc", *B.ARCH, "-shared", "-o", lib, *objs, "-L", libd, "-l:libnccl.so.2", "-Xlinker", f"-rpath={libd}", "-lcudart"], check=True)
from paper_conf_cluster_meiqsgls23_b200 import occu
occu.LIB_PATH = lib
import numpy as np, torch
from occu_gen import configs
b1 = configs.cfg1(); dev = torch.device("cuda", 0)
nf = torch.from_numpy(b1.node_feat).to(dev); ef = torch.from_numpy(b1.edge_feat).to(dev)
m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64)); m.init_weights(42); m.set_small_batch_kernel(True)
csr = m.to_device(occu.pack(b1.graphs)); out = torch.empty(1, device=dev)
for _ in range(20): m.predict(csr, nf, ef, out)
torch.cuda.synchronize()
ts = np.zeros(64, np.uint64)
occu.lib().occu_debug_small_ts(ts.ctypes.data_as(ctypes.c_void_p))
ids = (ts >> np.uint64(56)).astype(np.int64)
cyc = (ts & np.uint64(0xFFFFFFFFFFFFFF)).astype(np.int64)
n = int(np.max(np.nonzero(ts)[0])) + 1
print("total cycles", cyc[n - 1] - cyc[0])
for i in range(1, n):
    print(f"sync {ids[i]:2d}: {cyc[i] - cyc[i - 1]:7d} cycles")
