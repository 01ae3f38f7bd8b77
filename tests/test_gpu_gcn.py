"""GraphConv (dtc_graphconv, NEXT-3, Eq. (2)) on the GPU vs the FP64 oracle
(oracle/gcn.py), through the C ABI.  Tolerance derived in DESIGN.md §2: SpMM rtol + 2e-3
for the TF32 GEMM, on Bound = (|A|·|H|)·|W|."""
import numpy as np
import pytest

import datagen
from datagen import configs
from oracle import gcn as ogcn

from gpu_util import build, dev

pytestmark = pytest.mark.gpu


def _run(f, H, W, b, relu, dtype):
    import torch
    Hd = dev(H.astype(np.float16) if dtype == "fp16" else H.astype(np.float32))
    Y, AH = f.graphconv(Hd, dev(W.astype(np.float32)), None if b is None else dev(b.astype(np.float32)), relu=relu)
    torch.cuda.synchronize()
    return Y.cpu().numpy(), AH.cpu().numpy()


def _check(Y, M, K, rp, ci, v, H, W, b, relu, dtype):
    Yr, Bd, _ = ogcn.graphconv(M, K, rp, ci, v.astype(np.float32), H.astype(np.float32), W, b, relu)
    rtol, atol = ogcn.tolerance(dtype, W)
    err = np.abs(Y.astype(np.float64) - Yr)
    lim = rtol * Bd + atol
    assert np.all(np.isfinite(Y))
    assert np.all(err <= lim), f"max err/limit {float(np.max(err / lim)):.3g}"


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("relu,bias", [(True, True), (False, True), (True, False), (False, False)])
@pytest.mark.parametrize("Fi,Fo", [(16, 7), (64, 128), (128, 64), (33, 40)])
def test_graphconv_random(Fi, Fo, relu, bias, dtype):
    M, K = 517, 389
    seed = Fi * 1000 + Fo
    rp, ci = datagen.random_csr(M, K, 0.04, seed)
    v = datagen.uniform(seed, 1, len(ci))
    H = datagen.uniform(seed, 2, K * Fi).reshape(K, Fi)
    W = datagen.uniform(seed, 3, Fi * Fo).reshape(Fi, Fo)
    b = datagen.uniform(seed, 4, Fo) if bias else None
    if dtype == "fp16":
        v, H = v.astype(np.float16), H.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype)
    Y, _ = _run(f, H, W, b, relu, dtype)
    _check(Y, M, K, rp, ci, v, H, W, b, relu, dtype)


@pytest.mark.parametrize("name,Fi,Fo", [("c1", 128, 128), ("c1", 256, 64), ("c2", 128, 256)])
def test_graphconv_on_configs(name, Fi, Fo):
    """The paper's GCN hidden sizes 128/256 on the Cora/arxiv-shaped graphs."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    H = datagen.uniform(cfg.seed_b, 7, cfg.K * Fi).reshape(cfg.K, Fi)
    W = datagen.uniform(cfg.seed_b, 8, Fi * Fo).reshape(Fi, Fo) * np.float32(1.0 / np.sqrt(Fi))
    b = datagen.uniform(cfg.seed_b, 9, Fo)
    f = build(cfg.M, cfg.K, rp, ci, v)
    Y, AH = _run(f, H, W, b, True, "tf32")
    _check(Y, cfg.M, cfg.K, rp, ci, v, H, W, b, True, "tf32")
    # AH is exactly what dtc_spmm returns (same kernel, same launch shape)
    import torch
    C = f.spmm(dev(H.astype(np.float32)))
    torch.cuda.synchronize()
    assert np.array_equal(AH, C.cpu().numpy())


def test_two_layer_gcn_forward():
    """The paper's 2-layer DTC-GCN forward: ReLU hidden layer, linear output."""
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    F0, F1, F2 = 64, 128, 16
    X = datagen.uniform(11, 1, cfg.K * F0).reshape(cfg.K, F0)
    W1 = datagen.uniform(11, 2, F0 * F1).reshape(F0, F1) * np.float32(0.125)
    b1 = datagen.uniform(11, 3, F1)
    W2 = datagen.uniform(11, 4, F1 * F2).reshape(F1, F2) * np.float32(0.09)
    b2 = datagen.uniform(11, 5, F2)
    f = build(cfg.M, cfg.K, rp, ci, v)
    H1, _ = _run(f, X, W1, b1, True, "tf32")
    _check(H1, cfg.M, cfg.K, rp, ci, v, X, W1, b1, True, "tf32")
    # layer 2 takes the GPU's H1 (errors of layer 1 are inputs here; the oracle reuses them)
    H2, _ = _run(f, H1, W2, b2, False, "tf32")
    _check(H2, cfg.M, cfg.K, rp, ci, v, H1, W2, b2, False, "tf32")


def test_graphconv_rejects_bad_arguments():
    import torch
    from paper_conf_asplos_fan0024_b200 import DtcError
    rp, ci = datagen.random_csr(20, 20, 0.2, 1)
    v = datagen.uniform(1, 1, len(ci))
    f = build(20, 20, rp, ci, v)
    H = torch.zeros((20, 8), device="cuda")
    with pytest.raises(TypeError):
        f.graphconv(H, torch.zeros((7, 4), device="cuda"))
    with pytest.raises(TypeError):
        f.graphconv(H.half(), torch.zeros((8, 4), device="cuda"))
    from paper_conf_asplos_fan0024_b200 import lib
    assert lib().dtc_graphconv(f.handle, H.data_ptr(), 8, 0, 4, 0, 1, 0, 0, 0) != 0
