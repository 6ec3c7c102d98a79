"""Small driver for ncu: a few CFG2 forward (and optionally train) steps."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from occu_gen import configs  # noqa: E402
from paper_conf_cluster_meiqsgls23_b200 import occu  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--path", type=int, default=0)
ap.add_argument("--train", action="store_true")
ap.add_argument("--graphs", type=int, default=256)
ap.add_argument("--bf16", action="store_true")
ap.add_argument("--graphormer", type=int, default=0)
ap.add_argument("--decoder", action="store_true")
ap.add_argument("--synth", action="store_true", help="inputs synthesized on the device (NEXT-4)")
ap.add_argument("--cfg3", action="store_true", help="CFG3 (512 BERT-base / GPT-2 graphs) instead of CFG2")
ap.add_argument("--d", type=int, default=128)
ap.add_argument("--L", type=int, default=3)
a = ap.parse_args()
dev = torch.device("cuda", 0)
m = occu.Model(occu.config(L=a.L, F_n=80, F_e=4, d=a.d, prec=occu.BF16 if a.bf16 else occu.FP32,
                           graphormer=a.graphormer, heads=4,
                           readout=occu.READOUT_SET_DECODER if a.decoder else occu.READOUT_MEAN))
m.init_weights(42)
m.set_kernel_path(a.path)
b = configs.cfg3(512) if a.cfg3 else configs.cfg2(a.graphs)
csr = m.to_device(occu.pack(b.graphs))
nf = torch.from_numpy(b.node_feat).to(dev)
ef = torch.from_numpy(b.edge_feat).to(dev)
yt = torch.from_numpy(b.targets).to(dev)
if a.synth:
    import numpy as np
    from occu_gen import templates
    t = m.template(templates.build_template("resnet50"))
    grid = configs.cnn_grid()
    hp = np.stack([templates.hp_vector("resnet50", grid[i % len(grid)]) for i in range(a.graphs)]).astype(np.float32)
for _ in range(a.steps):
    if a.synth:
        csr, nf, ef = m.synthesize([t] * a.graphs, hp)
    if a.train:
        m.train_step(csr, nf, ef, yt, 1e-4, want_loss=False)
    else:
        m.predict(csr, nf, ef)
torch.cuda.synchronize()
print("done")
