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


# ------------------------------------------------------------------ backward / training (NEXT-3)
@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("name", ["c1", "c2"])
def test_transposed_format_bit_exact(name, dtype):
    """opts.transpose: the GPU condenses A^T from A's CSR; bit-exact against O2 of the oracle's
    CSR transpose (rows of A^T ascending in the original row)."""
    from gpu_util import assert_format_equal, check_units
    import oracle
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    v = v.astype(np.float16) if dtype == "fp16" else v
    ft = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype, transpose=True)
    assert (ft.M, ft.K, ft.nnz) == (cfg.K, cfg.M, len(ci))
    rp_t, ci_t, v_t = ogcn.csr_transpose(cfg.M, cfg.K, rp, ci, v)
    got = ft.export()
    assert_format_equal(got, oracle.condense(cfg.K, rp_t, ci_t, v_t))
    check_units(got, cfg.K)


def test_transposed_nonsquare_and_empty():
    import oracle
    from gpu_util import assert_format_equal
    M, K = 70, 45
    rp, ci = datagen.random_csr(M, K, 0.08, 5)
    v = datagen.uniform(5, 1, len(ci))
    ft = build(M, K, rp, ci, v, transpose=True)
    rp_t, ci_t, v_t = ogcn.csr_transpose(M, K, rp, ci, v)
    assert_format_equal(ft.export(), oracle.condense(K, rp_t, ci_t, v_t))
    B = datagen.uniform(5, 2, M * 24).reshape(M, 24)
    from gpu_util import spmm, check_tol
    check_tol(spmm(ft, B), K, M, rp_t, ci_t, v_t, B, "tf32")
    f0 = build(M, K, np.zeros(M + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32), transpose=True)
    assert (f0.M, f0.num_tc_blocks) == (K, 0)


def _bw_check(got, ref, bound, rtol, atol=1e-6, what=""):
    err = np.abs(got.astype(np.float64) - ref)
    lim = rtol * bound + atol
    assert np.all(np.isfinite(got)), what
    assert np.all(err <= lim), f"{what}: max err/limit {float(np.max(err / lim)):.3g}"


@pytest.mark.parametrize("relu", [True, False])
@pytest.mark.parametrize("name,Fi,Fo", [("c1", 64, 16), ("c1", 33, 7), ("c2", 128, 64)])
def test_graphconv_backward_vs_oracle(name, Fi, Fo, relu):
    """dtc_graphconv_backward (dW, db, dAH, dH = A^T dAH on the transposed ME-TCF) against the FP64
    chain rule; the ReLU mask is the GPU forward's (both sides take the same sign decision)."""
    import torch
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    H = datagen.uniform(cfg.seed_b, 21, cfg.K * Fi).reshape(cfg.K, Fi)
    W = datagen.uniform(cfg.seed_b, 22, Fi * Fo).reshape(Fi, Fo) * np.float32(1.0 / np.sqrt(Fi))
    b = datagen.uniform(cfg.seed_b, 23, Fo)
    dY = datagen.uniform(cfg.seed_b, 24, cfg.M * Fo).reshape(cfg.M, Fo)
    f = build(cfg.M, cfg.K, rp, ci, v)
    ft = build(cfg.M, cfg.K, rp, ci, v, transpose=True)
    Y, AH = f.graphconv(dev(H), dev(W), dev(b), relu=relu)
    g = f.graphconv_backward(AH, dev(W), Y, dev(dY), relu=relu, At=ft)
    torch.cuda.synchronize()
    Yh = Y.cpu().numpy()
    mask = (Yh > 0).astype(np.float64) if relu else None
    ref = ogcn.graphconv_backward(cfg.M, cfg.K, rp, ci, v, H, W, dY, mask=mask)
    tol = ogcn.backward_tolerance("tf32", cfg.M)
    _bw_check(g["dW"].cpu().numpy(), ref["dW"], ref["bound_dW"], tol["dW"], what="dW")
    _bw_check(g["db"].cpu().numpy(), ref["db"], ref["bound_db"], tol["db"], what="db")
    _bw_check(g["dAH"].cpu().numpy(), ref["dAH"], ref["bound_dAH"], tol["dAH"], what="dAH")
    _bw_check(g["dH"].cpu().numpy(), ref["dH"], ref["bound_dH"], tol["dH"], what="dH")


def test_softmax_xent_vs_oracle():
    import torch
    from paper_conf_asplos_fan0024_b200 import softmax_xent, DtcError
    M, C = 3000, 10
    z = datagen.uniform(3, 1, M * C).reshape(M, C) * np.float32(4.0)
    lab = (np.arange(M) * 7 % C).astype(np.int32)
    loss, dz = softmax_xent(dev(z), dev(lab))
    torch.cuda.synchronize()
    rl, rg = ogcn.softmax_xent(z, lab)
    assert abs(float(loss.item()) - rl) <= 1e-5 * max(1.0, abs(rl))
    assert np.allclose(dz.cpu().numpy(), rg, rtol=1e-5, atol=1e-8)
    with pytest.raises(DtcError):
        softmax_xent(dev(z), dev(np.full(M, C, np.int32)))


def test_gcn2_training_reduces_loss():
    """Two-layer GCN trained for a few SGD steps through the library (forward: dtc_graphconv x 2,
    loss: dtc_softmax_xent, backward: dtc_graphconv_backward x 2 with A^T, update: dtc_sgd_update);
    labels are a learnable function of (A X), so the loss must fall."""
    import torch
    from paper_conf_asplos_fan0024_b200 import GCN2
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    F0, F1, C = 32, 64, 7
    X = datagen.uniform(31, 1, cfg.K * F0).reshape(cfg.K, F0)
    import oracle
    AX = oracle.spmm(cfg.M, cfg.K, rp, ci, v, X, bound=False)
    Wt = datagen.uniform(31, 2, F0 * C).reshape(F0, C)
    labels = np.argmax(AX @ Wt, axis=1).astype(np.int32)
    A = build(cfg.M, cfg.K, rp, ci, v)
    At = build(cfg.M, cfg.K, rp, ci, v, transpose=True)
    net = GCN2(A, At, F0, F1, C, seed=1)
    Xd, Ld = dev(X), dev(labels)
    losses = [float(net.train_step(Xd, Ld, lr=1.0).item()) for _ in range(40)]
    assert all(np.isfinite(losses))
    assert losses[-1] < 0.9 * losses[0], losses[::8]
    assert sum(b > a for a, b in zip(losses, losses[1:])) <= 4, losses   # (near-)monotone descent
