"""Build a traced copy of the library, run one CFG2 edge-GEMM launch, print CTA-0 timeline."""
import ctypes, os, subprocess, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cluster_meiqsgls23_b200 import build as B
# compile traced variant into a separate .so
import glob
objdir = os.path.join(ROOT, "build", "trace")
os.makedirs(objdir, exist_ok=True)
inc, libd = B.nccl_dirs()
objs = []
for src in B.sources():
    obj = os.path.join(objdir, os.path.basename(src) + ".o")
    if src.endswith(".cu"):
        cmd = ["nvcc", *B.ARCH, "-O3", "-std=c++17", "-DOCCU_TC_TRACE", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include"), "-I", inc, "-c", src, "-o", obj]
    else:
        cmd = ["nvcc", "-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include"), "-I", inc, "-x", "c++", "-c", src, "-o", obj]
    subprocess.run(cmd, check=True)
    objs.append(obj)
lib = os.path.join(objdir, "libocc_trace.so")
subprocess.run(["nvcc", *B.ARCH, "-shared", "-o", lib, *objs, "-L", libd, "-l:libnccl.so.2", f"-Xlinker", f"-rpath={libd}", "-lcudart"], check=True)
from paper_conf_cluster_meiqsgls23_b200 import occu
occu.LIB_PATH = lib
import torch
from occu_gen import configs
m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128))
m.init_weights(42)
b = configs.cfg2(256)
csr = m.to_device(occu.pack(b.graphs))
nf = torch.from_numpy(b.node_feat).cuda(); ef = torch.from_numpy(b.edge_feat).cuda()
m.predict(csr, nf, ef); torch.cuda.synchronize()
print("done predict")
L = occu.lib()
L.occu_debug_trace.restype = ctypes.c_int
import numpy as np
buf = np.zeros((4096, 4), np.int64)
n = L.occu_debug_trace(buf.ctypes.data_as(ctypes.c_void_p), 4096)    # reset
m.predict(csr, nf, ef); torch.cuda.synchronize()
n = L.occu_debug_trace(buf.ctypes.data_as(ctypes.c_void_p), 4096)
ev = buf[:n]
# first launch only: stop when producer tile index resets
t0 = ev[:, 0].min()
names = {0: 'prod', 1: 'mma'}
out = []
seen_prod = -1
for t, role, tile, e in ev:
    out.append((t - t0, role, tile, e))
out.sort()
launch_end = None
for i, (t, role, tile, e) in enumerate(out):
    pass
lines = []
for t, role, tile, e in out[:600]:
    lines.append(f"{t:9d} {names.get(role, 'w%d' % (role-2)):5s} tile {tile:3d} ev {e}")
open(os.path.join(ROOT, "gpurun_out", "trace.txt"), "w").write("\n".join(lines))
print("events", n)
