"""Time CFG2 inference (FP32 and BF16) under the current OCCU_GATHER_* environment."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np
import torch
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu
dev = torch.device("cuda", 0)
b = configs.cfg2(256)
res = {}
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)
for prec, key in ((occu.FP32, "f32"), (occu.BF16, "bf16")):
    m = occu.Model(occu.config(L=3, d=128, prec=prec))
    m.init_weights(42)
    csr = m.to_device(occu.pack(b.graphs))
    nf = torch.from_numpy(b.node_feat).to(dev); ef = torch.from_numpy(b.edge_feat).to(dev)
    out = torch.empty(256, device=dev)
    for _ in range(5):
        m.predict(csr, nf, ef, out)
    m.set_profiling(True); m.profile_reset()
    ts = []
    for _ in range(30):
        flush.fill_(1.0)
        a = torch.cuda.Event(enable_timing=True); z = torch.cuda.Event(enable_timing=True)
        a.record(); m.predict(csr, nf, ef, out); z.record()
        ts.append((a, z))
    torch.cuda.synchronize()
    pr = m.profile()
    res[key] = {"ms": float(np.median([x.elapsed_time(y) for x, y in ts])),
                "gather_ms": pr["gather_segsum"][0] / 30}
print(json.dumps({"env": {k: v for k, v in os.environ.items() if k.startswith("OCCU_GATHER")}, **res}))
