"""Weight-gradient GEMM of the backward (SURVEY §8(c) step BW: dW = Σ_r X[r]ᵀ Y[r], split-K
with a fixed-order reduction) through the occu_test_wgrad hook, against float64 NumPy —
the same kernels occu_train_step launches, at row counts that span one CTA's range, many
32-row stages and a ragged tail, with FP32 Y and (OCCU_BF16 training, R28) BF16 Y."""
import numpy as np
import pytest

from paper_conf_cluster_meiqsgls23_b200 import occu

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("ybf", [False, True], ids=["y_fp32", "y_bf16"])
@pytest.mark.parametrize("A,Bn,R", [(128, 128, 37), (128, 128, 1000), (128, 128, 5003),
                                    (128, 128, 184_576), (64, 64, 7777), (128, 80, 20_000),
                                    (32, 16, 4099), (128, 4, 184_576), (128, 4, 999), (64, 20, 3000)])
def test_wgrad_matches_float64(A, Bn, R, ybf):
    import torch
    if ybf and Bn % 16:
        pytest.skip("BF16 Y rows come from d-wide activations (Bn = d)")
    dev = torch.device("cuda", 0)
    g = torch.Generator().manual_seed(A * 7 + Bn * 3 + R)
    X = torch.randn(R, A, generator=g, dtype=torch.float64)
    Y = torch.rand(R, Bn, generator=g, dtype=torch.float64)
    Xf = X.float()
    Yd = Y.to(torch.bfloat16) if ybf else Y.float()
    m = occu.Model(occu.config(L=1, F_n=80, F_e=4, d=128))
    out = torch.full((A, Bn), float("nan"), dtype=torch.float32, device=dev)
    m.test_wgrad(Xf.to(dev).contiguous(), Yd.to(dev).contiguous(), out, y_bf16=ybf)
    torch.cuda.synchronize()
    ref = Xf.double().numpy().T @ Yd.double().numpy()       # exact inputs the kernel saw
    got = out.cpu().double().numpy()
    err = np.linalg.norm(got - ref) / np.linalg.norm(ref)
    assert np.isfinite(got).all()
    # FP32 accumulation of ~R/148 rows per split (TMEM) plus the fixed-order split sum, and
    # the dropped X_lo·Y_lo term of 3xTF32 (~2^-22): sqrt-n growth of the FP32 rounding
    assert err <= 2e-6 + 5e-8 * np.sqrt(R), err
    # determinism: the split-K reduction has a fixed order
    out2 = torch.empty_like(out)
    m.test_wgrad(Xf.to(dev).contiguous(), Yd.to(dev).contiguous(), out2, y_bf16=ybf)
    torch.cuda.synchronize()
    assert torch.equal(out, out2)
