"""Selector diagnostic (NEXT-4, §4.5.2): the oracle's makespan simulation
pinned by hand-worked schedules and closed forms, and the native dtc_selector_ar (host,
no GPU) equal to it on random and config-shaped windows."""
import numpy as np
import pytest

import paper_conf_asplos_fan0024_b200 as dtc
from oracle import selector as osel


def rwo_of(lengths):
    return np.concatenate([[0], np.cumsum(lengths)]).astype(np.int32)


def test_eq1_paper_example():
    # 128 SMs, occupancy 6; SM 0 first holds blocks 0,128,...,640 and block
    # 768 is the next one it receives (C20 precedence)
    first_wave = [b for b in range(768) if osel.eq1_sm(b, 128) == 0]
    assert first_wave == [0, 128, 256, 384, 512, 640]
    assert osel.eq1_sm(768, 128) == 0
    assert sorted(osel.eq1_sm(b, 128) for b in range(128)) == list(range(128))   # bijective on a wave
    assert sorted(osel.eq1_sm(b, 148) for b in range(148)) == list(range(148))


def test_hand_worked_schedule_two_sms():
    # S=2 -> sm = b mod 2.  SM0: 3, 2, 5 on 2 slots -> 3 | 2+5 = 7.  SM1: 1 | 2 -> 2.
    rwo = rwo_of([3, 1, 2, 2, 5])
    assert osel.makespan_base(rwo, 2, 2) == 7
    assert osel.makespan_balanced(rwo, 2, 2) == 13 / 4
    assert osel.approximation_ratio(rwo, 2, 2) == pytest.approx(7 / 3.25)


def test_hand_worked_schedule_four_sms():
    # S=4, O=1: b -> 0,2,1,3,0,2: SM0 1+5, SM2 2+6, SM1 3, SM3 4 -> makespan 8
    rwo = rwo_of([1, 2, 3, 4, 5, 6])
    assert osel.makespan_base(rwo, 4, 1) == 8
    assert osel.makespan_balanced(rwo, 4, 1) == 21 / 4


def test_uniform_windows_have_ar_one():
    # the paper's "naturally balanced" case: every SM slot receives the same work
    for S, O, k, c in ((128, 6, 3, 4), (148, 4, 2, 7), (8, 2, 5, 1)):
        rwo = rwo_of([c] * (S * O * k))
        assert osel.makespan_base(rwo, S, O) == k * c
        assert osel.approximation_ratio(rwo, S, O) == 1.0
        assert not osel.select_balanced(rwo, S, O)


def test_single_heavy_window_ar_is_slots():
    rwo = rwo_of([0] * 37 + [6000] + [0] * 100)
    assert osel.makespan_base(rwo, 128, 6) == 6000
    assert osel.approximation_ratio(rwo, 128, 6) == pytest.approx(768.0)
    assert osel.select_balanced(rwo, 128, 6)


@pytest.mark.parametrize("S,O", [(2, 1), (2, 2), (4, 3), (128, 6), (148, 6), (148, 1)])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_native_matches_oracle(S, O, seed):
    rng = np.random.default_rng(seed)
    W = int(rng.integers(0, 3000))
    lengths = rng.pareto(1.5, W).astype(np.int64) % 500
    rwo = rwo_of(lengths)
    got = dtc.selector_ar(rwo, S, O)
    assert got["makespan_base"] == osel.makespan_base(rwo, S, O)
    assert got["makespan_balanced"] == pytest.approx(osel.makespan_balanced(rwo, S, O), rel=1e-15)
    assert got["ar"] == pytest.approx(osel.approximation_ratio(rwo, S, O), rel=1e-12)


@pytest.mark.parametrize("name", ["c1", "c2"])
def test_native_matches_oracle_on_configs(name):
    import oracle
    from datagen import configs
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    ref = oracle.condense(cfg.M, rp, ci, np.ones(len(ci), np.float32))
    rwo = ref["row_window_offset"]
    got = dtc.selector_ar(rwo, 148, 6)
    assert got["makespan_base"] == osel.makespan_base(rwo, 148, 6)
    assert got["ar"] == pytest.approx(osel.approximation_ratio(rwo, 148, 6), rel=1e-12)


def test_native_rejects_bad_arguments():
    rwo = rwo_of([1, 2])
    for S, O in ((3, 1), (0, 1), (148, 0)):
        with pytest.raises(dtc.DtcError):
            dtc.selector_ar(rwo, S, O)
    with pytest.raises(dtc.DtcError):
        dtc.selector_ar(np.array([0, 5, 3], np.int32), 2, 1)
