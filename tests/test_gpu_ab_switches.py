"""The training step's byte-saving variants against the paths they replace (same process
code, A/B by the library's environment switches, each run in its own subprocess):

* LReLU'(h) from the forward's sign bits (default) vs from the stored h rows
  (OCCU_NO_HBITS=1): the same per-element decisions, so the gradient is BITWISE equal;
* dα by the compensated FP32 dot (default) vs float64 FMAs (OCCU_DA_F64=1): both are
  accurate far beyond FP32 rounding of the result, so the gradients agree to ~1e-6.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def grads(tmp_path, tag, **env):
    out = str(tmp_path / f"{tag}.npy")
    e = dict(os.environ)
    e.update(env)
    subprocess.run([sys.executable, os.path.join(HERE, "_ab_grads.py"), out], env=e, check=True,
                   timeout=600)
    return np.load(out)


@pytest.mark.parametrize("prec,aggr", [("f32", 0), ("f32", 1), ("bf16", 0)])
def test_sign_bits_mask_is_bitwise_the_row_mask(tmp_path, prec, aggr):
    a = grads(tmp_path, "bits", AB_PREC=prec, AB_AGGR=str(aggr))
    b = grads(tmp_path, "rows", AB_PREC=prec, AB_AGGR=str(aggr), OCCU_NO_HBITS="1")
    assert np.array_equal(a, b)


def test_dot2_dalpha_matches_float64(tmp_path):
    a = grads(tmp_path, "dot2")
    b = grads(tmp_path, "f64", OCCU_DA_F64="1")
    rel = np.abs(a - b) / np.maximum(np.abs(b), 1e-3 * np.abs(b).max())
    assert rel.max() < 1e-5, rel.max()


@pytest.mark.parametrize("prec,aggr", [("f32", 0), ("f32", 1), ("bf16", 0)])
def test_row_exponent_handoff_is_bitwise_neutral(tmp_path, prec, aggr):
    """DV / DZ / dP row scale exponents written by their producers (gate backward, edge
    backward, node backward) instead of the W_m / W_e / W_u row-GEMM converters' own row-max
    pass: the same exponents of the same stored rows, so the gradient is BITWISE equal."""
    a = grads(tmp_path, "rexp", AB_PREC=prec, AB_AGGR=str(aggr))
    b = grads(tmp_path, "norexp", AB_PREC=prec, AB_AGGR=str(aggr), OCCU_NO_REXP="1")
    assert np.array_equal(a, b)


@pytest.mark.parametrize("prec,aggr", [("f32", 0), ("f32", 1), ("bf16", 0)])
def test_node_bwd_cp_async_ring_is_bitwise_neutral(tmp_path, prec, aggr):
    """The node backward's out-edge rows landed by cp.async in a per-warp shared-memory ring
    (default) vs held in registers (OCCU_NB_NOCPA=1): the same rows summed in the same order."""
    a = grads(tmp_path, "cpa", AB_PREC=prec, AB_AGGR=str(aggr))
    b = grads(tmp_path, "nocpa", AB_PREC=prec, AB_AGGR=str(aggr), OCCU_NB_NOCPA="1")
    assert np.array_equal(a, b)


@pytest.mark.parametrize("prec", ["f32", "bf16"])
def test_edge_bwd_small_cp_async_ring_is_bitwise_neutral(tmp_path, prec):
    """The layer-1 edge backward's e' / de rows landed by cp.async in a per-warp ring (default)
    vs register rows (OCCU_EB_NOCPA=1): the same rows in the same order, BITWISE equal."""
    a = grads(tmp_path, "ebcpa", AB_PREC=prec)
    b = grads(tmp_path, "ebnocpa", AB_PREC=prec, OCCU_EB_NOCPA="1")
    assert np.array_equal(a, b)


@pytest.mark.parametrize("aggr", [0, 1])
def test_broadcast_dh_batched_is_bitwise_neutral(tmp_path, aggr):
    """The head backward's broadcast with 4 nodes per warp step (default, d = 128) vs the
    per-element kernel (OCCU_BDH_V1=1): the same arithmetic per element, BITWISE equal."""
    a = grads(tmp_path, "bdh4", AB_AGGR=str(aggr))
    b = grads(tmp_path, "bdh1", AB_AGGR=str(aggr), OCCU_BDH_V1="1")
    assert np.array_equal(a, b)
