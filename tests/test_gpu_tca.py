"""Format build with a row permutation (dtc_build_opts_t.row_perm, e.g. the TCA order):
the condensed arrays equal the oracle condensation of the permuted CSR, and dtc_spmm
returns C in the ORIGINAL row order (P:253 Reid + DESIGN.md C19)."""
import numpy as np
import pytest

import datagen
import oracle
import paper_conf_asplos_fan0024_b200 as dtc
from datagen import configs

from gpu_util import dev, assert_format_equal, spmm, check_tol

pytestmark = pytest.mark.gpu


def _permute(rp, ci, v, perm):
    deg = np.diff(rp)[perm]
    nrp = np.zeros(len(perm) + 1, np.int32)
    nrp[1:] = np.cumsum(deg)
    idx = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in perm]).astype(np.int64)
    return nrp, ci[idx], v[idx]


def _shuffled(name, seed=5):
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    perm0 = np.random.default_rng(seed).permutation(cfg.M)
    v = configs.make_values(cfg, len(ci))
    srp, sci, sv = _permute(rp, ci, v, perm0)
    return cfg, srp, sci, sv


@pytest.mark.parametrize("name", ["c1", "c2"])
@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_tca_build_and_spmm(name, dtype):
    cfg, rp, ci, v = _shuffled(name)
    perm = dtc.tca_reorder(cfg.M, cfg.K, rp, ci)
    vv = v.astype(np.float16) if dtype == "fp16" else v
    f = dtc.Format.build(dev(rp), dev(ci), dev(vv), cfg.M, cfg.K, dtype=dtype, row_perm=dev(perm))
    prp, pci, pv = _permute(rp, ci, vv, perm)
    assert_format_equal(f.export(), oracle.condense(cfg.M, prp, pci, pv))
    N = 64
    B = datagen.uniform(3, 2, cfg.K * N).reshape(cfg.K, N)
    if dtype == "fp16":
        B = B.astype(np.float16)
    C = spmm(f, B)
    check_tol(C, cfg.M, cfg.K, rp, ci, vv, B, dtype)   # original row order


def test_tca_integer_exact_and_split_units():
    cfg, rp, ci, _ = _shuffled("c2", 7)
    v = datagen.integers(2, 5, len(ci))
    perm = dtc.tca_reorder(cfg.M, cfg.K, rp, ci)
    N = 128
    B = datagen.integers(3, 6, cfg.K * N).reshape(cfg.K, N)
    Cr, _ = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B)
    for U in (0, 3):
        f = dtc.Format.build(dev(rp), dev(ci), dev(v), cfg.M, cfg.K, row_perm=dev(perm), unit_blocks=U)
        assert np.array_equal(spmm(f, B).astype(np.float64), Cr)


def test_invalid_permutation_rejected():
    rp, ci = datagen.random_csr(50, 40, 0.1, 1)
    v = datagen.uniform(1, 1, len(ci))
    bad = np.arange(50, dtype=np.int32)
    bad[3] = 4   # duplicate
    with pytest.raises(dtc.DtcError) as e:
        dtc.Format.build(dev(rp), dev(ci), dev(v), 50, 40, row_perm=dev(bad))
    assert e.value.status == dtc.DTC_ERR_INVALID
    bad[3] = 50  # out of range
    with pytest.raises(dtc.DtcError):
        dtc.Format.build(dev(rp), dev(ci), dev(v), 50, 40, row_perm=dev(bad))
