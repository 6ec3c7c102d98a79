"""Input-generator tests: determinism, DAG-ness, size anchors, FLOPs closed form."""
import numpy as np
import pytest

from occu_gen import configs, dags, features, prng, weights


def test_splitmix64_reference_vectors():
    # Published splitmix64 outputs for seed 1234567 (Vigna's reference C code).
    splitmix = prng.splitmix64_stream(1234567, 5).tolist()
    assert splitmix == [6457827717110365317, 3203168211198807973, 9817491932198370423,
                        4593380528125082431, 16408922859458223821]
    assert int(prng.splitmix64_stream(0, 1)[0]) == 0xE220A8397B1DCDAF


def test_counter_based_offsets():
    a = prng.uniform01(7, 100)
    b = prng.uniform01(7, 40, offset=60)
    assert np.array_equal(a[60:], b)
    assert (a >= 0).all() and (a < 1).all()


@pytest.mark.parametrize("fam", list(dags.FAMILIES))
def test_families_are_dags(fam):
    g = dags.training_graph(fam)
    assert g.num_nodes >= 13
    assert dags.is_dag(g.num_nodes, g.src, g.dst)
    assert (g.src != g.dst).all()
    assert (g.src < g.dst).all()            # topological node order


def test_size_anchors():
    # SURVEY §8(d) anchors: LeNet-5 ~38/50, ResNet-50 ~512/718 (training graphs)
    g = dags.training_graph("lenet5")
    assert (g.num_nodes, g.num_edges) == (39, 52)
    g = dags.training_graph("resnet50")
    assert (g.num_nodes, g.num_edges) == (514, 721)
    # P239: >30 operator types across the dataset
    types = set()
    for f in dags.FAMILIES:
        types |= set(dags.training_graph(f).node_op.tolist())
    assert len(types) > 30


def test_training_expansion_counts():
    # N = 2 n_fwd + n_params + 1 ; E = 2 m_fwd + n_fwd + n_params + 2
    for fam in ("resnet18", "vit_t", "lstm"):
        fb = dags.build_forward(fam)
        nf = len(fb.ops)
        mf = sum(len(o.inputs) for o in fb.ops)
        npar = sum(len(o.params) for o in fb.ops)
        g = dags.expand_training(fam, fb)
        assert g.num_nodes == 2 * nf + npar + 1
        assert g.num_edges == 2 * mf + nf + npar + 2


def test_conv_flops_closed_form():
    # P131: 2*K*C*R*S*N*P*Q ; ResNet-50 conv1 at N=1, C=3: 236,027,904
    fb = dags.build_forward("resnet50", {"batch": 1, "cin": 3})
    conv1 = next(o for o in fb.ops if o.type == "Conv")
    assert conv1.flops == 236027904.0
    assert conv1.out_shape == (1, 64, 112, 112)


def test_features_shape_and_range():
    b = configs.cfg1()
    assert b.node_feat.shape == (39, features.F_N)
    assert b.edge_feat.shape == (52, features.F_E)
    assert b.node_feat.dtype == np.float32
    assert (b.node_feat >= 0).all() and (b.node_feat <= 1.0).all()
    onehot = b.node_feat[:, :40]
    assert np.array_equal(onehot.sum(axis=1), np.ones(39, np.float32))
    assert (b.node_feat[:, 79] == 0).all()
    assert ((b.targets > 0) & (b.targets < 1)).all()


def test_cfg2_determinism_and_variants():
    b1 = configs.cfg2(8)
    b2 = configs.cfg2(8)
    assert np.array_equal(b1.node_feat, b2.node_feat)
    assert np.array_equal(b1.edge_feat, b2.edge_feat)
    # variants differ in features only, never topology
    assert all(np.array_equal(g[1], b1.graphs[0][1]) for g in b1.graphs)
    assert not np.array_equal(b1.node_feat[:514], b1.node_feat[514:1028])


def test_weights_init_and_file_roundtrip(tmp_path):
    cfg = weights.ModelConfig(L=3, d=128)
    assert weights.num_params(cfg) == 142849
    w = weights.init_flat(cfg, 42)
    assert w.dtype == np.float32
    p = weights.unflatten(cfg, w)
    assert np.abs(p["W_u0"]).max() <= 1 / np.sqrt(80)
    assert np.abs(p["W_m1"]).max() <= 1 / np.sqrt(128)
    path = tmp_path / "w.bin"
    weights.write_weights(str(path), cfg, w)
    raw = path.read_bytes()
    assert raw[:8] == b"OCCUW001"
    assert len(raw) == 8 + 32 + 4 + 4 * w.size + 8
    back = np.frombuffer(raw, "<f4", offset=44, count=w.size)
    assert np.array_equal(back, w)


def test_random_dag_batch():
    b = configs.random_dag_batch(20, 5, hub=True)
    for n, s, t in b.graphs:
        assert dags.is_dag(n, s, t)
        assert (s < t).all() if len(s) else True
    assert b.node_feat.shape[0] == b.num_nodes


def test_feature_templates_exact_for_every_family():
    """NEXT-4 templates (occu_gen/templates.py): every family's hyperparameter-dependent Table I
    quantities are reproduced exactly (float64 ==) by the Newton form at held-out mixture
    hyperparameters, so on-device synthesis can match the generator's features."""
    from occu_gen import templates
    from occu_gen.prng import Rng
    for fam in configs.MIXTURE + ["bert_base"]:
        t = templates.build_template(fam)
        r = Rng(2024)
        templates.verify(t, [configs.mixture_variant(fam, r) for _ in range(2)])
        assert t.node_coef.shape == (t.num_nodes, 22, 12)
        assert np.all(t.node_static[:, 42:76] == 0)


def test_feature_template_verify_rejects_a_non_polynomial_quantity():
    """templates.verify is a real check: perturbing one coefficient (a quantity that the
    Newton form no longer reproduces) is reported."""
    from occu_gen import templates
    t = templates.build_template("lenet5")
    t.node_coef[3, 20, 1] += 1.0                 # FLOPs of node 3: wrong batch slope
    with pytest.raises(ValueError):
        templates.verify(t, [{"batch": 24, "cin": 2}])


def test_feature_template_hp_vector_defaults():
    from occu_gen import templates
    assert list(templates.hp_vector("resnet50", {"batch": 20, "cin": 3})) == [20.0, 3.0, 0.0, 0.0]
    assert list(templates.hp_vector("lstm", {"batch": 128, "seq": 32})) == [128.0, 1.0, 32.0, 0.0]
    assert list(templates.hp_vector("gpt2", {"batch": 16, "cin": 3, "seq": 512})) == [16.0, 3.0, 512.0, 0.0]


def test_mixture_arrays_match_specs():
    from occu_gen import templates
    specs = configs.mixture_specs(300, 1005, start=12345)
    fam, hp = configs.mixture_arrays(300, 1005, start=12345)
    for i, (f, h) in enumerate(specs):
        assert configs.MIXTURE[fam[i]] == f
        assert np.array_equal(hp[i], templates.hp_vector(f, h)), (f, h, hp[i])
    w = configs.family_work()[fam]
    assert np.array_equal(w, configs.spec_work(specs))
