"""Build a timing-instrumented library copy and report per-role wait/busy cycles (CTA 0)."""
import ctypes, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cluster_meiqsgls23_b200 import build as B
objdir = os.path.join(ROOT, "build", "timing"); os.makedirs(objdir, exist_ok=True)
inc, libd = B.nccl_dirs(); objs = []
for src in B.sources():
    obj = os.path.join(objdir, os.path.basename(src) + ".o")
    flags = ["-DOCCU_TC_TIMING"] if src.endswith(".cu") else []
    cmd = ["nvcc", *(B.ARCH if src.endswith(".cu") else []), "-O3", "-std=c++17", *flags, "-Xcompiler", "-fPIC",
           "-I", os.path.join(ROOT, "include"), "-I", inc] + (["-x", "c++"] if src.endswith(".cpp") else []) + ["-c", src, "-o", obj]
    subprocess.run(cmd, check=True); objs.append(obj)
lib = os.path.join(objdir, "libocc_timing.so")
subprocess.run(["nvcc", *B.ARCH, "-shared", "-o", lib, *objs, "-L", libd, "-l:libnccl.so.2", f"-Xlinker", f"-rpath={libd}", "-lcudart"], check=True)
from paper_conf_cluster_meiqsgls23_b200 import occu
occu.LIB_PATH = lib
import numpy as np, torch
from occu_gen import configs
m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128)); m.init_weights(42)
b = configs.cfg2(256)
csr = m.to_device(occu.pack(b.graphs))
nf = torch.from_numpy(b.node_feat).cuda(); ef = torch.from_numpy(b.edge_feat).cuda()
L = occu.lib()
buf = np.zeros((32, 4), np.uint64)
ebuf = np.zeros((32, 4), np.uint64)
m.predict(csr, nf, ef); torch.cuda.synchronize()
L.occu_debug_tc_time(buf.ctypes.data_as(ctypes.c_void_p))   # reset
L.occu_debug_eg_time(ebuf.ctypes.data_as(ctypes.c_void_p))
m.predict(csr, nf, ef); torch.cuda.synchronize()
L.occu_debug_tc_time(buf.ctypes.data_as(ctypes.c_void_p))
L.occu_debug_eg_time(ebuf.ctypes.data_as(ctypes.c_void_p))
names = ["producer", "mma"] + [f"conv{w}" for w in range(8)] + [f"epi{w}" for w in range(16)] + ["-", "-", "-", "-", "setup", "total"]
for title, b in (("rowgemm", buf), ("edgegate", ebuf)):
    print("==", title)
    for k, n in enumerate(names):
        w, bsy, cnt = b[k][0], b[k][1], b[k][2]
        if cnt:
            print(f"{n:9s} launches {cnt} wait {w/cnt:10.0f} busy {bsy/cnt:10.0f} cycles/launch")
