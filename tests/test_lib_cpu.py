"""CPU-side tests of the C-ABI library: it loads, exports every symbol the header
declares, and its host packer (a0) matches the oracle bit for bit."""
import re
import subprocess

import numpy as np
import pytest

import oracle
from occu_gen import configs
from paper_conf_cluster_meiqsgls23_b200 import occu

HEADER = "include/occu.h"


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_cluster_meiqsgls23_b200 import build
    build.build()


def declared_symbols():
    import os
    txt = open(os.path.join(os.path.dirname(__file__), "..", HEADER)).read()
    return sorted(set(re.findall(r"\b(occu_[a-z0-9_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    names = declared_symbols()
    assert len(names) >= 20
    L = occu.lib()
    out = subprocess.run(["nm", "-D", "--defined-only", occu.LIB_PATH], capture_output=True,
                         text=True).stdout
    exported = set(re.findall(r" T (occu_\w+)", out))
    for n in names:
        assert n in exported, n
        assert hasattr(L, n)
    assert set(occu.EXPORTS) <= exported


def test_num_params_matches_layout():
    from occu_gen import weights
    for L, d, fn, fe in [(3, 128, 80, 4), (2, 64, 80, 4), (1, 64, 8, 4)]:
        c = occu.config(L=L, F_n=fn, F_e=fe, d=d)
        assert occu.num_params(c) == weights.num_params(
            weights.ModelConfig(L=L, F_n=fn, F_e=fe, d=d, d_h=d))


def assert_pack_equal(graphs):
    ref = oracle.pack(graphs)
    got = occu.pack(graphs).arrays()
    for k in ("node_off", "edge_off", "in_ptr", "in_src", "in_dst", "in_eid", "out_ptr",
              "out_pos", "node_graph"):
        assert got[k].dtype == np.int32
        assert np.array_equal(got[k], ref[k]), k
    assert (got["num_graphs"], got["num_nodes"], got["num_edges"]) == \
        (ref["num_graphs"], ref["num_nodes"], ref["num_edges"])


@pytest.mark.parametrize("seed", range(8))
def test_pack_bit_exact_random(seed):
    b = configs.random_dag_batch(25, 200 + seed, max_nodes=30, hub=seed % 2 == 0)
    graphs = b.graphs + [(1, np.zeros(0, np.int32), np.zeros(0, np.int32)),
                         (4, np.array([0, 0, 0, 2], np.int32), np.array([3, 3, 3, 3], np.int32))]
    assert_pack_equal(graphs)


def test_pack_bit_exact_cfg2_threaded():
    b = configs.cfg2(64)
    assert_pack_equal(b.graphs)


def test_pack_unsorted_and_shuffled_ids():
    # edges given in arbitrary order, nodes not topologically numbered
    from occu_gen.prng import Rng
    r = Rng(5)
    graphs = []
    for n in (5, 17, 40):
        perm = r.permutation(n)
        s = r.randint(0, n - 2, 3 * n)
        t = s + 1 + np.floor(r.uniform(3 * n) * (n - 1 - s)).astype(np.int64)
        graphs.append((n, perm[s].astype(np.int32), perm[t].astype(np.int32)))
    assert_pack_equal(graphs)


@pytest.mark.parametrize("bad,msg", [
    ([(0, [], [])], "num_nodes"),
    ([(3, [0, 1], [1, 3])], "out of range"),
    ([(3, [0, 1], [1, 1])], "self-loop"),
    ([(3, [-1], [1])], "out of range"),
])
def test_pack_errors(bad, msg):
    graphs = [(n, np.array(s, np.int32), np.array(t, np.int32)) for n, s, t in bad]
    with pytest.raises(occu.OccuError) as ei:
        occu.pack(graphs)
    assert ei.value.status == occu.OCCU_EINVAL
    assert msg in str(ei.value)


def test_pack_empty_batch_rejected():
    with pytest.raises(occu.OccuError):
        occu.pack([])


def test_pack_arrays_matches_pack_and_oracle():
    """pack_arrays (concatenated edge lists) builds the same views as pack (per-graph list):
    bit-exact against the oracle, on a large threaded batch and a ragged small one; errors in
    the multi-threaded validation name the first bad graph."""
    for graphs in (configs.cfg2(96).graphs,
                   configs.random_dag_batch(33, 9, max_nodes=25, hub=True).graphs
                   + [(1, np.zeros(0, np.int32), np.zeros(0, np.int32))]):
        nn = [g[0] for g in graphs]
        ne = [len(g[1]) for g in graphs]
        c = occu.pack_arrays(nn, ne, np.concatenate([g[1] for g in graphs]),
                             np.concatenate([g[2] for g in graphs]))
        got, ref = c.arrays(), oracle.pack(graphs)
        for k in ("node_off", "edge_off", "in_ptr", "in_src", "in_dst", "in_eid", "out_ptr",
                  "out_pos", "node_graph"):
            assert np.array_equal(got[k], ref[k]), k
    graphs = configs.cfg2(40).graphs
    bad = [(n, s.copy(), t.copy()) for n, s, t in graphs]
    bad[31][2][5] = bad[31][1][5]                      # self-loop in graph 31
    with pytest.raises(occu.OccuError) as ei:
        occu.pack(bad)
    assert "graph 31" in str(ei.value) and "self-loop" in str(ei.value)


# ------------------------------------------ NEXT-4: occu-packing through the C-ABI (host)
def test_pack_jobs_matches_oracle_bit_exact():
    rng = np.random.default_rng(11)
    cases = [np.zeros(0, np.float32), np.array([0.3], np.float32),
             rng.random(1000).astype(np.float32),
             (rng.random(3000) * 0.4).astype(np.float32),            # many jobs per slot
             np.concatenate([rng.random(200), [1.5, -0.2, 0.0, 1.0]]).astype(np.float32),
             np.round(rng.random(500) * 8).astype(np.float32) / 8]   # exact ties at capacity
    for occ in cases:
        a, loads = occu.pack_jobs(occ)
        ra, rl = oracle.occu_packing(occ)
        assert np.array_equal(a, ra)
        assert np.array_equal(loads, rl)
    a, _ = occu.pack_jobs(np.full(9, 0.3, np.float32), capacity=0.6)
    assert np.array_equal(a, oracle.occu_packing(np.full(9, 0.3, np.float32), 0.6)[0])


def test_pack_jobs_golden_and_errors():
    import os
    d = {}
    for ln in open(os.path.join(os.path.dirname(__file__), "golden", "occu_packing_first_fit.txt")):
        if ln.strip() and not ln.startswith("#"):
            k, *v = ln.split()
            d[k] = v
    a, loads = occu.pack_jobs(np.array(d["occ"], np.float32))
    assert np.array_equal(a, np.array(d["assign"], np.int32)) and len(loads) == int(d["bins"][0])
    for bad in (np.array([0.1, np.nan], np.float32), np.array([np.inf], np.float32)):
        with pytest.raises(occu.OccuError):
            occu.pack_jobs(bad)
    with pytest.raises(occu.OccuError):
        occu.pack_jobs(np.array([0.1], np.float32), capacity=0.0)
