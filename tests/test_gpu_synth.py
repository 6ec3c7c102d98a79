"""GPU tests of on-device feature synthesis (R39): the batch
occu_synthesize builds from family templates equals, per array, what the host path produces
for the same (family, hyperparameter) list — the CSR bit for bit against occu_pack, the Table I
features against the generator (occu_gen.features) to within one float32 ulp (float64 log2 on
the device vs the host's libm), and predictions on the two batches agree."""
import numpy as np
import pytest

from occu_gen import configs, templates
from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu


class _Dev:
    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr,
                                         "data": (C_addr(ptr), False), "version": 3}


def C_addr(p):
    import ctypes
    return ctypes.cast(p, ctypes.c_void_p).value or 0


def dev_ints(ptr, n):
    import torch
    return torch.as_tensor(_Dev(ptr, n, "<i4"), device="cuda").cpu().numpy()


_TMPL = {}


def tmpl(model, fam):
    key = (id(model), fam)
    if key not in _TMPL:
        _TMPL[key] = model.template(templates.build_template(fam))
    return _TMPL[key]


def synth_batch(model, specs):
    ts = [tmpl(model, fam) for fam, _ in specs]
    hp = np.stack([templates.hp_vector(fam, h) for fam, h in specs]).astype(np.float32)
    return model.synthesize(ts, hp)


def ulps(a, b):
    a = np.ascontiguousarray(a, np.float32).view(np.int32).astype(np.int64)
    b = np.ascontiguousarray(b, np.float32).view(np.int32).astype(np.int64)
    return np.abs(a - b)


@pytest.mark.parametrize("n,seed", [(24, 1005), (7, 77)])
def test_synthesized_batch_matches_host_path(n, seed):
    m = occu.Model(occu.config(L=3, d=128))
    m.init_weights(42)
    specs = configs.mixture_specs(n, seed)
    specs[0] = ("lenet5", {"batch": 16, "cin": 1})
    specs[1] = ("bert_base", {"batch": 32, "cin": 3, "seq": 512})
    ref = configs._make(specs, seed=seed)
    csr, nf, ef = synth_batch(m, specs)
    host = occu.pack(ref.graphs)
    hs, ds = host.struct, csr.struct
    assert (ds.num_graphs, ds.num_nodes, ds.num_edges) == (hs.num_graphs, hs.num_nodes, hs.num_edges)
    B, N, E = hs.num_graphs, hs.num_nodes, hs.num_edges
    for name, cnt in (("node_off", B + 1), ("edge_off", B + 1), ("in_ptr", N + 1), ("out_ptr", N + 1),
                      ("in_src", E), ("in_dst", E), ("in_eid", E), ("out_pos", E), ("node_graph", N)):
        got = dev_ints(getattr(ds, name), cnt)
        exp = np.ctypeslib.as_array(getattr(hs, name), shape=(cnt,))
        assert np.array_equal(got, exp), name
    gnf, gef = nf.cpu().numpy(), ef.cpu().numpy()
    assert gnf.shape == ref.node_feat.shape and gef.shape == ref.edge_feat.shape
    assert ulps(gnf, ref.node_feat).max() <= 1
    assert ulps(gef, ref.edge_feat).max() <= 1
    assert np.mean(gnf == ref.node_feat) > 0.999
    # predictions on the synthesized device batch vs the host-built batch
    y_syn = m.predict(csr, nf, ef).cpu().numpy()
    y_host = m.predict(host, ref.node_feat, ref.edge_feat)
    assert np.allclose(y_syn, y_host, rtol=1e-5, atol=1e-7)


def test_synthesize_errors():
    m = occu.Model(occu.config(L=2, d=64))
    t = tmpl(m, "lenet5")
    with pytest.raises(occu.OccuError):
        m.synthesize([t], np.array([[-1, 1, 0, 0]], np.float32))
    with pytest.raises(occu.OccuError):
        m.synthesize([t], np.array([[np.nan, 1, 0, 0]], np.float32))
    m2 = occu.Model(occu.config(L=2, F_n=16, F_e=4, d=64))
    t2 = m2.template(templates.build_template("lenet5"))
    with pytest.raises(occu.OccuError):
        m2.synthesize([t2], np.array([[16, 1, 0, 0]], np.float32))
