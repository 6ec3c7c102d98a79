import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
# the paper's full model stack, inputs synthesized on the GPU from (family, hyperparameters)
from paper_conf_cluster_meiqsgls23_b200 import occu
from occu_gen import templates
m2 = occu.Model(occu.config(L=3, d=128, graphormer=2, heads=4, readout=occu.READOUT_SET_DECODER, k=4))
m2.init_weights(42)
t = m2.template(templates.build_template("resnet50"))
csr, nf, ef = m2.synthesize([t] * 2, [[16, 3, 0, 0], [64, 1, 0, 0]])   # (batch, cin, seq, hw)
occ = m2.predict(csr, nf, ef)                                          # CUDA tensor [2]
slots, loads = occu.pack_jobs(occ.cpu().numpy())                       # occu-packing (P390-P392)

from paper_conf_cluster_meiqsgls23_b200 import occu
from occu_gen import configs
m = occu.Model(occu.config(L=3, F_n=80, F_e=4, d=128))
m.init_weights(42)
b = configs.cfg2(256)
csr = occu.pack(b.graphs)
y = m.predict(csr, b.node_feat, b.edge_feat)             # host arrays: synchronous
loss = m.train_step(csr, b.node_feat, b.edge_feat, b.targets, lr=1e-4)

print('readme examples ok', occ, slots, y[:2], loss)
