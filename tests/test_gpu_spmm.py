"""S1-S5 (dtc_spmm) on the GPU vs oracle O1, through the C ABI.

Tolerance |dC| <= rtol*(|A|.|B|) + 1e-6 with rtol 2e-3 (TF32) / 1e-2 (FP16)
(BASELINE.json north_star); bit-exact where the arithmetic is exact (P2-P5).
"""
import numpy as np
import pytest

import datagen
import oracle
from datagen import configs

from gpu_util import build, dev, spmm, check_tol, compare_chunked

pytestmark = pytest.mark.gpu


def _torch():
    import torch
    return torch


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("N", [1, 3, 8, 32, 33, 64, 100, 128, 256, 512])
def test_random_tolerance(dtype, N):
    M, K = 700, 900
    rp, ci = datagen.random_csr(M, K, 0.03, N)
    v = datagen.uniform(N, 1, len(ci))
    B = datagen.uniform(N, 2, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype)
    C = spmm(f, B)
    check_tol(C, M, K, rp, ci, v, B, dtype)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("name,N", [("c1", 32), ("c2", 128), ("c1", 256)])
def test_p2_integer_bit_exact(name, N, dtype):
    """P2: |a|,|b| <= 4 integers: exact in TF32/FP16 and in FP32 accumulation."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = datagen.integers(cfg.seed_a, 5, len(ci))
    B = datagen.integers(cfg.seed_b, 6, cfg.K * N).reshape(cfg.K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype)
    C = spmm(f, B)
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v.astype(np.float32), B.astype(np.float32))
    assert np.array_equal(C.astype(np.float64), Cr)


def test_p3_identity_and_p4_permutation():
    M, N = 1000, 64
    B = datagen.uniform(1, 2, M * N).reshape(M, N)
    Bt = B.view(np.uint32) & np.uint32(0xFFFFE000)   # pre-rounded to TF32 by truncation...
    Bt = Bt.view(np.float32)                        # ...so RN(tf32) is the identity on it
    rp = np.arange(M + 1, dtype=np.int32)
    f = build(M, M, rp, np.arange(M, dtype=np.int32), np.ones(M, np.float32))
    assert np.array_equal(spmm(f, Bt), Bt)
    perm = np.random.default_rng(1).permutation(M).astype(np.int32)
    # A = P stored as canonical CSR: row i has the single column perm[i]
    f = build(M, M, rp, perm, np.ones(M, np.float32))
    assert np.array_equal(spmm(f, Bt), Bt[perm])


def test_p5_row_sums():
    cfg = configs.get("c2")
    rp, ci = configs.make_pattern(cfg)
    v = datagen.dyadic(3, 1, len(ci), -1, 1)
    N = 16
    f = build(cfg.M, cfg.K, rp, ci, v)
    C = spmm(f, np.ones((cfg.K, N), np.float32))
    rows = np.repeat(np.arange(cfg.M), np.diff(rp))
    sums = np.zeros(cfg.M)
    np.add.at(sums, rows, v.astype(np.float64))
    for j in range(N):
        assert np.array_equal(C[:, j].astype(np.float64), sums)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_p6_column_independence(dtype):
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = datagen.uniform(3, 2, cfg.K * 64).reshape(cfg.K, 64)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype)
    C64 = spmm(f, B)
    for j in (0, 5, 63):
        C1 = spmm(f, np.ascontiguousarray(B[:, j:j + 1]))
        assert np.array_equal(C1[:, 0], C64[:, j])


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("U", [1, 2, 5])
@pytest.mark.parametrize("N", [96, 256, 258])
def test_split_windows_fixup(U, dtype, N):
    """Tiny work units force many split windows: the deterministic fixup path (N = 256 / 258: the
    TF32 1 KB-slice kernel's transposed tiles, vector and scalar C stores)."""
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = datagen.uniform(4, 2, cfg.K * N).reshape(cfg.K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype, unit_blocks=U)
    assert f.num_split_windows > 0
    C1 = spmm(f, B)
    C2 = spmm(f, B)
    assert np.array_equal(C1, C2)                     # deterministic, counters self-reset
    check_tol(C1, cfg.M, cfg.K, rp, ci, v, B, dtype)


def test_deterministic_and_overwrites_everything():
    torch = _torch()
    cfg = configs.get("c2")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    N = 128
    B = dev(configs.make_B(cfg, N))
    f = build(cfg.M, cfg.K, rp, ci, v)
    C1 = torch.full((cfg.M, N), float("nan"), device="cuda")
    f.spmm(B, C1)
    C2 = torch.full((cfg.M, N), float("nan"), device="cuda")
    f.spmm(B, C2)
    torch.cuda.synchronize()
    assert not torch.isnan(C1).any()
    assert torch.equal(C1, C2)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("N", [258, 300])
def test_misaligned_c_wide_rows(dtype, N):
    """Aligned B (the TMA path with 1 KB slices for TF32), C with an odd leading dimension and start:
    the scalar stores of the transposed TF32 tiles, ragged last column group."""
    torch = _torch()
    M, K = 300, 400
    rp, ci = datagen.random_csr(M, K, 0.05, 11)
    v = datagen.uniform(11, 1, len(ci))
    B = datagen.uniform(11, 2, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype)
    Cbig = torch.full((M, N + 5), float("nan"), device="cuda")
    C = Cbig[:, 1:1 + N]                 # ldc = N + 5, misaligned
    f.spmm(dev(B), C)
    torch.cuda.synchronize()
    check_tol(C.cpu().numpy(), M, K, rp, ci, v, B, dtype)
    assert torch.isnan(Cbig[:, :1]).all() and torch.isnan(Cbig[:, 1 + N:]).all()


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_strided_and_misaligned_scalar_path(dtype):
    torch = _torch()
    M, K, N = 300, 400, 37
    rp, ci = datagen.random_csr(M, K, 0.05, 7)
    v = datagen.uniform(7, 1, len(ci))
    Bf = datagen.uniform(7, 2, K * 50).reshape(K, 50)
    if dtype == "fp16":
        v, Bf = v.astype(np.float16), Bf.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype)
    Bd = dev(Bf)[:, 1:1 + N]             # ldb = 50, misaligned start
    Cbig = torch.full((M, 41), float("nan"), device="cuda")
    C = Cbig[:, 2:2 + N]                 # ldc = 41, misaligned
    f.spmm(Bd, C)
    torch.cuda.synchronize()
    check_tol(C.cpu().numpy(), M, K, rp, ci, v, Bf[:, 1:1 + N], dtype)
    assert torch.isnan(Cbig[:, :2]).all() and torch.isnan(Cbig[:, 2 + N:]).all()


def test_empty_and_tail_windows():
    M, K, N = 37, 20, 8
    rows = {0: [1, 2], 36: [19]}
    rp = np.zeros(M + 1, np.int32)
    ci = []
    for i in range(M):
        ci += rows.get(i, [])
        rp[i + 1] = len(ci)
    ci = np.array(ci, np.int32)
    v = np.array([1.0, 2.0, 3.0], np.float32)
    B = datagen.integers(1, 2, K * N).reshape(K, N)
    f = build(M, K, rp, ci, v)
    C = spmm(f, B)
    Cr, _ = oracle.spmm(M, K, rp, ci, v, B)
    assert np.array_equal(C.astype(np.float64), Cr)
    # all-zero matrix
    f0 = build(M, K, np.zeros(M + 1, np.int32), np.zeros(0, np.int32), np.zeros(0, np.float32))
    assert np.all(spmm(f0, B) == 0)


def test_host_api_matches_device():
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg)
    f = build(cfg.M, cfg.K, rp, ci, v)
    C1 = spmm(f, B)
    C2 = f.spmm_host(B)
    assert np.array_equal(C1, C2)


@pytest.mark.parametrize("name,N", [("c1", 32), ("c2", 128), ("c3", 256), ("c3h", 256),
                                    ("c4", 64), ("c4", 128), ("c4", 256), ("c5", 512)])
def test_config_full_size(name, N, parity_report):
    """Every BASELINE config at full size in the bench launch configuration, EVERY element of C
    compared with O1 (64k-row chunks): within |dC| <= rtol*(|A|.|B|) + 1e-6 (north_star).  The
    worst err/limit per config is printed in the session summary."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=cfg.dtype)
    C = spmm(f, B)
    assert np.isfinite(C).all()
    worst = compare_chunked(C, cfg.M, cfg.K, rp, ci, v, B, cfg.dtype)
    parity_report[f"{name} N={N} {cfg.dtype}"] = (worst, cfg.M * N)


@pytest.mark.parametrize("name,N", [("c2", 128), ("c3", 256), ("c4", 128), ("c5", 512)])
def test_tall_windows_full_size(name, N, parity_report):
    """NEXT-2 layout (32-row windows, two 16-row tiles per TC block sharing the gathered B rows):
    every element of C against O1 at full size."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=cfg.dtype, window_rows=32)
    C = spmm(f, B)
    worst = compare_chunked(C, cfg.M, cfg.K, rp, ci, v, B, cfg.dtype)
    parity_report[f"{name} N={N} {cfg.dtype} tall32"] = (worst, cfg.M * N)


@pytest.mark.parametrize("N", [8, 33, 64, 100])
@pytest.mark.parametrize("U", [0, 2])
def test_tall_windows_narrow_rows(N, U):
    """32-row windows on the 256 B and 512 B slice kernels (B rows <= 256 B, ragged), with and
    without forced splits: C within tolerance of O1, and integer inputs bit-exact."""
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = datagen.uniform(9, 2, cfg.K * N).reshape(cfg.K, N)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype="tf32", window_rows=32, unit_blocks=U)
    check_tol(spmm(f, B), cfg.M, cfg.K, rp, ci, v, B, "tf32")
    vi = np.rint(v * 4).astype(np.float32)
    Bi = np.rint(B * 4).astype(np.float32)
    fi = build(cfg.M, cfg.K, rp, ci, vi, dtype="tf32", window_rows=32, unit_blocks=U)
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, vi, Bi)
    assert np.array_equal(spmm(fi, Bi).astype(np.float64), Cr)


@pytest.mark.parametrize("name,N", [("c3", 256), ("c3h", 256), ("c4", 128), ("c5", 512)])
def test_p2_integer_full_size_exact(name, N, parity_report):
    """P2 at full size: integer A and B (|a|,|b| <= 2 -> every product and partial sum is exact in
    TF32/FP16 and FP32 as long as row sums of |a||b| stay below 2^24; the largest rows here give
    < 2^20), so EVERY GPU entry must EQUAL the FP64 oracle, in the bench's launch configuration."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = datagen.integers(cfg.seed_a, 5, len(ci), -2, 2)
    B = datagen.integers(cfg.seed_b, 6, cfg.K * N, -2, 2).reshape(cfg.K, N)
    if cfg.dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    assert int(np.diff(rp).max()) * 4 < 2 ** 23
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=cfg.dtype)
    C = spmm(f, B)
    compare_chunked(C, cfg.M, cfg.K, rp, ci, v, B, exact=True)
    parity_report[f"{name} N={N} {cfg.dtype} P2 integer"] = (0.0, cfg.M * N)


@pytest.mark.parametrize("chunks", [1, 2, 3, 4, 16])
@pytest.mark.parametrize("dtype,N", [("tf32", 128), ("tf32", 100), ("tf32", 257), ("fp16", 192)])
def test_host_api_column_chunks(chunks, dtype, N):
    """dtc_spmm_host pipelined over column chunks (DTC_OPT_HOST_CHUNKS): C(:, cols) depends only on
    B(:, cols), so every chunking returns what one dtc_spmm over all N columns returns (the
    per-column sum order is the same), and it stays within the O1 tolerance."""
    M, K = 3000, 2500
    rp, ci = datagen.random_csr(M, K, 0.01, N + 7)
    v = datagen.uniform(N, 3, len(ci))
    B = datagen.uniform(N, 4, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype, options={"host_chunks": chunks})
    Cd = spmm(f, B)
    Ch = f.spmm_host(np.ascontiguousarray(B))
    assert f.get_option("last_host_mode") == 2 * min(chunks, (N + 31) // 32)
    check_tol(Ch, M, K, rp, ci, v, B, dtype)
    assert np.array_equal(Cd, Ch)
    # a second call reuses the staging buffers, streams and events
    Ch2 = f.spmm_host(np.ascontiguousarray(B))
    assert np.array_equal(Ch, Ch2)


@pytest.mark.parametrize("zc", [0, 1])
@pytest.mark.parametrize("chunks", [1, 2, 4])
def test_host_api_pinned_zero_copy(zc, chunks):
    """dtc_spmm_host with pinned torch buffers; DTC_OPT_HOST_ZERO_COPY=1 stores C straight into the
    mapped host buffer (no copy-out).  Same C as dtc_spmm, bit for bit, including a padded ldc."""
    import torch
    M, K, N = 4000, 3500, 128
    rp, ci = datagen.random_csr(M, K, 0.01, 11)
    v = datagen.uniform(N, 5, len(ci))
    B = datagen.uniform(N, 6, K * N).reshape(K, N)
    f = build(M, K, rp, ci, v, options={"host_zero_copy": zc, "host_chunks": chunks})
    Cd = spmm(f, B)
    Bh = torch.from_numpy(B).pin_memory()
    Ch = torch.full((M, N), float("nan"), dtype=torch.float32).pin_memory()
    f.spmm_host(Bh, Ch)
    assert f.get_option("last_host_mode") == 2 * chunks + zc
    assert np.array_equal(Ch.numpy(), Cd)
    Cw = torch.full((M, N + 4), -7.0, dtype=torch.float32).pin_memory()   # ldc = N + 4
    f.spmm_host(Bh, Cw[:, :N])
    assert np.array_equal(Cw[:, :N].numpy(), Cd)
    assert torch.all(Cw[:, N:] == -7.0)


def test_binding_rejects_mismatched_buffers():
    """the binding validates what the C ABI cannot see (host extents, K rows, dtype,
    device), raising instead of letting a kernel or a copy run past a buffer."""
    import torch
    M, K, N = 200, 300, 16
    rp, ci = datagen.random_csr(M, K, 0.05, 3)
    v = datagen.uniform(3, 1, len(ci))
    f = build(M, K, rp, ci, v)
    good = np.zeros((K, N), np.float32)
    for bad in (np.zeros((K - 1, N), np.float32), np.zeros((K, N), np.float16), np.zeros((K, N), np.float64)):
        with pytest.raises((TypeError, ValueError)):
            f.spmm_host(bad)
    for badC in (np.zeros((M - 1, N), np.float32), np.zeros((M, N), np.float64), np.zeros((M, N + 1), np.float32)):
        with pytest.raises((TypeError, ValueError)):
            f.spmm_host(good, badC)
    with pytest.raises(ValueError):
        f.spmm(torch.zeros((K + 5, N), device="cuda"))
    with pytest.raises(TypeError):
        f.spmm(torch.zeros((K, N), device="cuda"), torch.zeros((M, N + 1), device="cuda"))
    f16 = build(M, K, rp, ci, v, dtype="fp16")
    with pytest.raises(TypeError):
        f16.spmm_host(good)


@pytest.mark.parametrize("zc", [0, 1])
@pytest.mark.parametrize("dtype,N", [("tf32", 128), ("fp16", 96), ("tf32", 37)])
def test_host_async_stream_matches_device(zc, dtype, N):
    """dtc_spmm_host_async: a stream of 5 products with different B (alternating pinned host buffers,
    as a serving loop would), waited once at the end; every C equals dtc_spmm bit for bit."""
    import torch
    M, K = 3000, 2500
    rp, ci = datagen.random_csr(M, K, 0.01, N + 3)
    v = datagen.uniform(N, 7, len(ci))
    f = build(M, K, rp, ci, v, dtype=dtype, options={"host_zero_copy": zc})
    Bs, refs, Cs = [], [], []
    for j in range(5):
        B = datagen.uniform(N + j, 8, K * N).reshape(K, N)
        if dtype == "fp16":
            B = B.astype(np.float16)
        Bs.append(torch.from_numpy(B).pin_memory())
        refs.append(spmm(f, B))
        Cs.append(torch.full((M, N), float("nan"), dtype=torch.float32).pin_memory())
    for j in range(5):
        f.spmm_host_async(Bs[j], Cs[j])
    f.wait()
    for j in range(5):
        assert np.array_equal(Cs[j].numpy(), refs[j])
    assert f.get_option("last_host_mode") == 2 + zc
