"""Every dtc_spmm launch variant (per-handle options, include/dtc.h DTC_OPT_*) against oracle O1.

The library default is covered by test_gpu_spmm.py at every config; this module runs the
same parity bar (tolerance of BASELINE.json north_star, bit-exact for the exact-arithmetic
pins P2/P3/P9) on each variant -- the register-gather fallback kernel, the padded TMA kernel
one CTA per unit, persistent, without first-batch records, and with 512-byte slices forced --
so an ablation number in profiles/ is never a number of an incorrect kernel.
"""
import numpy as np
import pytest

import datagen
import oracle
from datagen import configs

from gpu_util import build as _build, dev, spmm, check_tol

pytestmark = pytest.mark.gpu

VARIANTS = {
    "ldg": {"kernel": "ldg"},
    "pad": {"kernel": "pad"},
    "pers": {"kernel": "pad", "persistent": 1},
    "nofirst": {"kernel": "pad", "first_records": 0},
    "slice512": {"kernel": "pad", "slice_bytes": 512},
    "tall": {},   # NEXT-2: 32-row windows (build option window_rows=32; TF32)
}


@pytest.fixture(params=list(VARIANTS))
def path(request):
    return request.param


def build(*a, path=None, **kw):
    if path == "tall":
        if kw.get("dtype", "tf32") != "tf32":
            pytest.skip("tall windows are TF32")
        kw["window_rows"] = 32
    f = _build(*a, options=VARIANTS[path] if path else None, **kw)
    return f


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("N", [1, 8, 33, 64, 128, 200, 512])
def test_random_tolerance(path, dtype, N):
    M, K = 500, 700
    rp, ci = datagen.random_csr(M, K, 0.04, N + 11)
    v = datagen.uniform(N, 1, len(ci))
    B = datagen.uniform(N, 2, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype, path=path)
    check_tol(spmm(f, B), M, K, rp, ci, v, B, dtype)
    # the variant really ran: TMA needs a 16-byte row pitch (contiguous B: N*elt % 16 == 0),
    # else the register gather
    elt = 2 if dtype == "fp16" else 4
    want = 1 if path == "ldg" or (N * elt) % 16 else 4
    if path == "tall":
        want = 4   # tall windows always run the padded kernel (B staged when TMA cannot describe it)
    assert f.get_option("last_kernel") == want


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("name,N,U", [("c1", 32, 0), ("c1", 256, 0), ("c2", 128, 0), ("c1", 96, 2)])
def test_p2_integer_bit_exact(path, name, N, U, dtype):
    """P2 (small integers: exact in TF32/FP16 and FP32), incl. split windows (U=2)."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = datagen.integers(cfg.seed_a, 5, len(ci))
    B = datagen.integers(cfg.seed_b, 6, cfg.K * N).reshape(cfg.K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype, unit_blocks=U, path=path)
    C = spmm(f, B)
    assert np.array_equal(C, spmm(f, B))
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v.astype(np.float32), B.astype(np.float32))
    assert np.array_equal(C.astype(np.float64), Cr)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_p9_dense_blocks_exact(path, dtype):
    """P9: fully dense A (every TC block holds 128 non-zeros, every mask bit set), M and K
    not multiples of 16 / 8 (ragged last window and last block), integer values."""
    M, K, N = 45, 29, 72
    rp = (np.arange(M + 1) * K).astype(np.int32)
    ci = np.tile(np.arange(K, dtype=np.int32), M)
    v = datagen.integers(9, 1, M * K)
    B = datagen.integers(9, 2, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype, path=path)
    C = spmm(f, B)
    ref = v.astype(np.float64).reshape(M, K) @ B.astype(np.float64)
    assert np.array_equal(C.astype(np.float64), ref)


def test_p3_identity_and_empty_windows(path):
    M, N = 1000, 64
    B = datagen.uniform(1, 2, M * N).reshape(M, N)
    Bt = (B.view(np.uint32) & np.uint32(0xFFFFE000)).view(np.float32)   # TF32-representable
    keep = np.ones(M, bool)
    keep[100:180] = False                                              # 5 empty windows
    rp = np.concatenate([[0], np.cumsum(keep)]).astype(np.int32)
    ci = np.nonzero(keep)[0].astype(np.int32)
    f = build(M, M, rp, ci, np.ones(len(ci), np.float32), path=path)
    ref = Bt * keep[:, None]
    assert np.array_equal(spmm(f, Bt), ref)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_strided_misaligned(path, dtype):
    import torch
    M, K, N = 300, 400, 37
    rp, ci = datagen.random_csr(M, K, 0.05, 7)
    v = datagen.uniform(7, 1, len(ci))
    Bf = datagen.uniform(7, 2, K * 50).reshape(K, 50)
    if dtype == "fp16":
        v, Bf = v.astype(np.float16), Bf.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype, path=path)
    Bd = dev(Bf)[:, 1:1 + N]
    Cbig = torch.full((M, 41), float("nan"), device="cuda")
    C = Cbig[:, 2:2 + N]
    f.spmm(Bd, C)
    torch.cuda.synchronize()
    check_tol(C.cpu().numpy(), M, K, rp, ci, v, Bf[:, 1:1 + N], dtype)
    assert torch.isnan(Cbig[:, :2]).all() and torch.isnan(Cbig[:, 2 + N:]).all()


def test_row_perm_original_order(path):
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = datagen.integers(cfg.seed_a, 5, len(ci))
    N = 64
    B = datagen.integers(cfg.seed_b, 6, cfg.K * N).reshape(cfg.K, N)
    perm = np.random.default_rng(3).permutation(cfg.M).astype(np.int32)
    f = build(cfg.M, cfg.K, rp, ci, v, row_perm=dev(perm), path=path)
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B)
    assert np.array_equal(spmm(f, B).astype(np.float64), Cr)


@pytest.mark.parametrize("name,U", [("c2", 0), ("c2", 16), ("c1", 2)])
def test_persistent_bit_identical(name, U):
    """Persistent and one-CTA-per-unit launches compute every unit in the same order."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, cfg.N)
    f = build(cfg.M, cfg.K, rp, ci, v, unit_blocks=U, path="pad")
    C0 = spmm(f, B)
    f.set_option("persistent", 1)
    C1 = spmm(f, B)
    assert np.array_equal(C0, C1)


@pytest.mark.parametrize("name,U", [("c2", 16), ("c1", 2)])
def test_unit_order_split_first(name, U):
    """F4 default order: split-window pieces first (window order), then whole-window units;
    same units as strict window order and the same C bit for bit."""
    from gpu_util import check_units
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, cfg.N)
    f0 = build(cfg.M, cfg.K, rp, ci, v, unit_blocks=U)
    f1 = build(cfg.M, cfg.K, rp, ci, v, unit_blocks=U, window_order=True)
    e0, e1 = f0.export(), f1.export()
    check_units(e0, cfg.M)
    u0, u1 = e0["units"], e1["units"]
    assert sorted(map(tuple, u0)) == sorted(map(tuple, u1))
    sp = u0[:, 4] >= 0
    k = int(sp.sum())
    assert k > 0 and np.all(sp[:k]) and not np.any(sp[k:])
    assert np.all(np.diff(u0[:k, 2]) >= 0) and np.all(np.diff(u0[k:, 2]) >= 0)   # window (block) order inside
    assert np.all(np.diff(u1[:, 2]) >= 0)
    assert np.array_equal(spmm(f0, B), spmm(f1, B))


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
@pytest.mark.parametrize("N", [1024, 1100, 2048])
def test_persistent_many_column_groups(dtype, N):
    """Wide B (several CTA column groups, each with its own dynamic unit counter), split windows:
    persistent == one-CTA-per-unit bit for bit, and within tolerance of the oracle."""
    M, K = 600, 500
    rp, ci = datagen.random_csr(M, K, 0.08, N)
    v = datagen.uniform(N, 1, len(ci))
    B = datagen.uniform(N, 2, K * N).reshape(K, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(M, K, rp, ci, v, dtype=dtype, unit_blocks=4, path="pad")
    C0 = spmm(f, B)
    f.set_option("persistent", 1)
    C1 = spmm(f, B)
    C2 = spmm(f, B)       # counters reset by the previous launch
    assert np.array_equal(C0, C1) and np.array_equal(C1, C2)
    check_tol(C1, M, K, rp, ci, v, B, dtype)


@pytest.mark.parametrize("name,U,dtype,N", [("c2", 0, "tf32", 128), ("c2", 16, "tf32", 512), ("c1", 2, "tf32", 32),
                                            ("c1", 2, "fp16", 256), ("c1", 0, "tf32", 33)])
def test_first_batch_records_bit_identical(name, U, dtype, N):
    """DTC_OPT_FIRST_RECORDS: the CTA's first batch from the per-unit side record (ids, TCOffset
    bounds, first-window end) computes exactly what the unit-record path computes, and matches O1."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    if dtype == "fp16":
        v, B = v.astype(np.float16), B.astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=dtype, unit_blocks=U)
    f.set_option("first_records", 0)
    C0 = spmm(f, B)
    f.set_option("first_records", 1)
    C1 = spmm(f, B)
    C2 = spmm(f, B)
    assert np.array_equal(C0, C1) and np.array_equal(C1, C2)
    check_tol(C1, cfg.M, cfg.K, rp, ci, v, B, dtype)


@pytest.mark.parametrize("U", [0, 1, 3])
@pytest.mark.parametrize("name,N", [("c1", 64), ("c1", 256), ("c2", 128)])
def test_fp16_block_pairs_exact(name, N, U):
    """FP16 m16n8k16 over pairs of TC blocks of one window (odd tails and unit/split boundaries take
    m16n8k8): integer inputs are exact either way, so C must equal O1 bit for bit, and the padded
    kernel must equal the register-gather kernel (k8 per block) bit for bit."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = datagen.integers(cfg.seed_a, 7, len(ci)).astype(np.float16)
    B = datagen.integers(cfg.seed_b, 8, cfg.K * N).reshape(cfg.K, N).astype(np.float16)
    f = build(cfg.M, cfg.K, rp, ci, v, dtype="fp16", unit_blocks=U)
    C = spmm(f, B)
    assert f.get_option("last_kernel") == 4
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v.astype(np.float32), B.astype(np.float32))
    assert np.array_equal(C.astype(np.float64), Cr)
    f.set_option("kernel", "ldg")
    assert np.array_equal(spmm(f, B), C)


def test_options_roundtrip_and_errors():
    from paper_conf_asplos_fan0024_b200 import DtcError
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v)
    defaults = {"kernel": 0, "persistent": 0, "first_records": 1, "host_chunks": 0, "host_zero_copy": -1,
                "slice_bytes": 0}
    for k, x in defaults.items():
        assert f.get_option(k) == x
    for k, bad in (("kernel", 2), ("persistent", 5), ("host_chunks", 17), ("host_zero_copy", 2),
                   ("slice_bytes", 256), ("last_kernel", 1)):
        with pytest.raises(DtcError):
            f.set_option(k, bad)
    f.set_option("host_chunks", 3)
    assert f.get_option("host_chunks") == 3
