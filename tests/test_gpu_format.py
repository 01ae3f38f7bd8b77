"""F0-F4 on the GPU vs the oracle's reference condensation: bit-exact ME-TCF."""
import numpy as np
import pytest

import datagen
import oracle
from datagen import configs
from paper_conf_asplos_fan0024_b200 import DtcError, DTC_ERR_UNSORTED, DTC_ERR_DUPLICATE, DTC_ERR_RANGE, \
    DTC_ERR_INVALID

from gpu_util import build, assert_format_equal, check_units

pytestmark = pytest.mark.gpu

CASES = [
    (1, 1, 1.0, 1), (15, 9, 0.3, 2), (16, 8, 1.0, 3), (17, 40, 0.2, 4), (40, 70, 0.05, 5),
    (48, 130, 0.5, 6), (333, 3000, 0.01, 7), (64, 12, 0.0, 8), (200, 200, 0.9, 9), (1000, 50, 0.3, 10),
    (4097, 9000, 0.002, 11), (100, 100000, 0.004, 12),
]


@pytest.mark.parametrize("path", [0, 1, 2])
@pytest.mark.parametrize("M,K,density,seed", CASES)
def test_random_bit_exact(M, K, density, seed, path):
    rp, ci = datagen.random_csr(M, K, density, seed)
    v = datagen.uniform(seed, 1, len(ci))
    f = build(M, K, rp, ci, v, dedup_path=path)
    got = f.export()
    assert_format_equal(got, oracle.condense(M, rp, ci, v))
    check_units(got, M)


@pytest.mark.parametrize("dtype", ["tf32", "fp16"])
def test_fp16_values_permuted_bitwise(dtype):
    rp, ci = datagen.random_csr(300, 500, 0.05, 3)
    v = datagen.uniform(3, 1, len(ci))
    vv = v.astype(np.float16) if dtype == "fp16" else v
    f = build(300, 500, rp, ci, vv, dtype=dtype)
    assert_format_equal(f.export(), oracle.condense(300, rp, ci, vv))


def _rows_csr(M, rows):
    rp = [0]
    ci = []
    for i in range(M):
        c = sorted(rows.get(i, []))
        ci += c
        rp.append(len(ci))
    return np.array(rp, np.int32), np.array(ci, np.int32)


@pytest.mark.parametrize("path", [0, 2])
def test_edge_cases(path):
    # empty matrix, empty windows between full ones, a dense long row (> 2048 nnz -> bitmap path)
    for M, K, rows in [
        (5, 7, {}),
        (64, 64, {0: [1], 40: [63], 63: list(range(64))}),
        (40, 6000, {3: list(range(0, 6000, 2)), 17: list(range(5000, 5100)), 39: [5999]}),
        (33, 10, {i: [i % 10] for i in range(33)}),
    ]:
        rp, ci = _rows_csr(M, rows)
        v = datagen.uniform(M, 1, len(ci))
        f = build(M, K, rp, ci, v, dedup_path=path)
        got = f.export()
        assert_format_equal(got, oracle.condense(M, rp, ci, v))
        check_units(got, M)


@pytest.mark.parametrize("U", [1, 2, 3, 8])
def test_forced_splits_schedule(U):
    cfg = configs.get("c1")
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v, unit_blocks=U)
    got = f.export()
    check_units(got, cfg.M)
    assert f.num_split_windows > 0


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c3h", "c4", "c5"])
def test_config_bit_exact(name):
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=cfg.dtype)
    got = f.export()
    assert_format_equal(got, oracle.condense(cfg.M, rp, ci, v))
    check_units(got, cfg.M)


def test_invalid_inputs():
    rp = np.array([0, 2, 4], np.int32)
    v = np.ones(4, np.float32)
    for ci, code in [
        (np.array([1, 0, 2, 3], np.int32), DTC_ERR_UNSORTED),
        (np.array([1, 1, 2, 3], np.int32), DTC_ERR_DUPLICATE),
        (np.array([0, 1, 2, 9], np.int32), DTC_ERR_RANGE),
        (np.array([0, 1, -1, 3], np.int32), DTC_ERR_RANGE),
    ]:
        with pytest.raises(DtcError) as e:
            build(2, 5, rp, ci, v)
        assert e.value.status == code
    with pytest.raises(DtcError) as e:
        build(2, 5, np.array([0, 3, 2], np.int32), np.array([0, 1, 2], np.int32), np.ones(3, np.float32))
    assert e.value.status == DTC_ERR_INVALID


@pytest.mark.parametrize("name", ["c1", "c2", "c3", "c4", "c5"])
def test_tall_window_format_bit_exact(name):
    """NEXT-2 layout (window_rows = 32): the GPU builder equals O2 applied to 32-row windows
    (oracle.condense(window=32), pinned by the brute force and the decode round trip)."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v, dtype=cfg.dtype, window_rows=32)
    assert f.window_rows == 32
    got = f.export()
    assert_format_equal(got, oracle.condense(cfg.M, rp, ci, v, window=32))
    check_units(got, cfg.M)


def test_tall_window_fp16_unsupported():
    from paper_conf_asplos_fan0024_b200 import DtcError, DTC_ERR_UNSUPPORTED
    rp, ci = datagen.random_csr(40, 40, 0.1, 1)
    v = datagen.uniform(1, 1, len(ci))
    with pytest.raises(DtcError) as e:
        build(40, 40, rp, ci, v, dtype="fp16", window_rows=32)
    assert e.value.status == DTC_ERR_UNSUPPORTED


@pytest.mark.parametrize("name,N,want", [("c4", 256, 32), ("c4", 128, 16), ("c2", 256, 16), ("c1", 512, 16)])
def test_selector_picks_window_height(name, N, want):
    """Selector (selector=1, window_rows=0): 32-row windows exactly when T32 <= 0.65 T16 and the
    gathered rows are >= 1 KB (n_hint x 4 B); the counts come from O2 at both heights."""
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v, selector=2, n_hint=N)
    _, t16 = oracle.condense_count(cfg.M, rp, ci, 16)
    _, t32 = oracle.condense_count(cfg.M, rp, ci, 32)
    expect = 32 if (N * 4 >= 1024 and t32 <= 0.65 * t16) else 16
    assert f.window_rows == expect == want
    assert_format_equal(f.export(), oracle.condense(cfg.M, rp, ci, v, window=expect))


@pytest.mark.parametrize("U", [16, 64, 256])
@pytest.mark.parametrize("guided", [1, -1])
@pytest.mark.parametrize("name", ["c2", "c4"])
def test_selector_plans_the_builders_units(name, U, guided):
    """The Selector simulates exactly the units F4 emits: its unit count for (U, guided) equals the
    builder's, and its simulated makespan equals dtc_selector_simulate over the exported units."""
    import paper_conf_asplos_fan0024_b200 as dtc
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    f = build(cfg.M, cfg.K, rp, ci, v, unit_blocks=U, guided=guided)
    e = f.export()
    m = dtc.sched_model("tf32", cfg.N)
    plan = dtc.selector_plan(e["row_window_offset"], m, [U], guided=guided)
    p = [x for x in plan["plans"] if x["makespan_ns"] >= 0][0]
    assert p["num_units"] == f.num_units
    assert p["makespan_ns"] == pytest.approx(dtc.selector_simulate(e["units"], m), rel=1e-12)
