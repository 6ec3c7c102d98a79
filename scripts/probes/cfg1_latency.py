"""CFG1 latency breakdown: eager vs CUDA-graph replay, 9-launch path vs single-CTA kernel,
and the device time of each kernel (library CUDA events)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from occu_gen import configs  # noqa: E402
from paper_conf_cluster_meiqsgls23_b200 import build, occu  # noqa: E402

build.build()
dev = torch.device("cuda", 0)
b1 = configs.cfg1()
nf = torch.from_numpy(b1.node_feat).to(dev)
ef = torch.from_numpy(b1.edge_feat).to(dev)


def lat(fn, reps=1000):
    for _ in range(50):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / reps


for small, path in ((False, 0), (True, 0), (False, 1)):
    side = torch.cuda.Stream(dev)
    m = occu.Model(occu.config(L=2, F_n=80, F_e=4, d=64), device=0, stream=side.cuda_stream)
    m.init_weights(42)
    m.set_small_batch_kernel(small)
    m.set_kernel_path(path)
    csr = m.to_device(occu.pack(b1.graphs))
    out = torch.empty(1, device=dev)
    with torch.cuda.stream(side):
        eager = lat(lambda: m.predict(csr, nf, ef, out))
        for _ in range(3):
            m.predict(csr, nf, ef, out)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=side):
        m.predict(csr, nf, ef, out)
    graph = lat(g.replay)
    m.profile_reset()
    m.set_profiling(True)
    with torch.cuda.stream(side):
        for _ in range(200):
            m.predict(csr, nf, ef, out)
    torch.cuda.synchronize()
    m.set_profiling(False)
    prof = {k: round(v[0] / 200 * 1e3, 2) for k, v in m.profile().items()}
    print(f"path={path} single_cta={small}: eager {eager:.1f} us, graph replay {graph:.1f} us, launches "
          f"{m.last_launch_count()}, kernel us: {prof}")
