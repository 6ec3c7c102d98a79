"""A/B timing of kernel-path variants (per-kernel CUDA events), one GPU.

    python scripts/probes/variants.py [infer|train|both] [--steps K]

infer: CFG2 FP32 / BF16 inference under kernel path 0, path 2 (gate + aggregation fused) and
OCCU_FUSE_EG=1 (edge + gate fused); train: CFG3 FP32 / BF16 training-step breakdown.
"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from occu_gen import configs, weights  # noqa: E402
from paper_conf_cluster_meiqsgls23_b200 import occu  # noqa: E402

STEPS = int(sys.argv[sys.argv.index("--steps") + 1]) if "--steps" in sys.argv else 10
MODE = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("-") else "both"
dev = torch.device("cuda", 0)
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)


def timeit(fn, m, steps=STEPS):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ev = []
    for _ in range(steps):
        flush.fill_(1.0)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        ev.append((a, b))
    torch.cuda.synchronize()
    ms = float(np.mean([a.elapsed_time(b) for a, b in ev]))
    m.profile_reset()
    m.set_profiling(True)
    for _ in range(steps):
        flush.fill_(1.0)
        fn()
    torch.cuda.synchronize()
    m.set_profiling(False)
    prof = {k: v[0] / steps for k, v in m.profile().items()}
    return ms, prof


def show(tag, ms, prof):
    print(f"== {tag}: {ms:.3f} ms/step")
    for k, v in sorted(prof.items(), key=lambda x: -x[1]):
        print(f"   {k:18s} {v:8.3f} ms")
    sys.stdout.flush()


def infer():
    b = configs.cfg2(256)
    hc = occu.pack(b.graphs)
    nf = torch.from_numpy(b.node_feat).to(dev)
    ef = torch.from_numpy(b.edge_feat).to(dev)
    for prec, pname in ((occu.FP32, "f32"), (occu.BF16, "bf16")):
        for tag, path, env in (("path0", 0, {}), ("path2", 2, {}), ("fuse_eg", 0, {"OCCU_FUSE_EG": "1"}),
                               ("fuse_ega", 0, {"OCCU_FUSE_EGA": "1"}), ("path0_again", 0, {})):
            if prec == occu.BF16 and path == 2:
                continue
            os.environ.pop("OCCU_FUSE_EG", None)
            os.environ.pop("OCCU_FUSE_EGA", None)
            os.environ.update(env)
            m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128, prec=prec))
            m.init_weights(42)
            m.set_kernel_path(path)
            csr = m.to_device(hc)
            out = torch.empty(b.num_graphs, device=dev)
            ms, prof = timeit(lambda: m.predict(csr, nf, ef, out), m)
            show(f"CFG2 infer {pname} {tag}", ms, prof)
            del m
    os.environ.pop("OCCU_FUSE_EG", None)
    os.environ.pop("OCCU_FUSE_EGA", None)


def train():
    b = configs.cfg3(512)
    hc = occu.pack(b.graphs)
    nf = torch.from_numpy(b.node_feat).to(dev)
    ef = torch.from_numpy(b.edge_feat).to(dev)
    yt = torch.from_numpy(b.targets).to(dev)
    wc = weights.ModelConfig(L=3, F_n=80, F_e=4, d=128, d_h=128)
    flat = weights.unit_scale(wc, weights.init_flat(wc, 42))
    print(f"CFG3: N={b.num_nodes} E={b.num_edges}")
    for prec, pname in ((occu.FP32, "f32"), (occu.BF16, "bf16")):
        m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128, prec=prec))
        m.set_params(flat)
        csr = m.to_device(hc)
        ms, prof = timeit(lambda: m.train_step(csr, nf, ef, yt, 1e-4, want_loss=False), m)
        show(f"CFG3 train {pname}", ms, prof)
        del m


if __name__ == "__main__":
    from paper_conf_cluster_meiqsgls23_b200 import build
    build.build()
    t0 = time.time()
    if MODE in ("infer", "both"):
        infer()
    if MODE in ("train", "both"):
        train()
    print(f"done in {time.time() - t0:.0f} s")
