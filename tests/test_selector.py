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


# ------------------------------------------------------------------ B200 Selector (NEXT-4, reading C26)
def _units(nbs, split=None):
    """dtc_format_export unit records: whole-window units of the given block counts, or split pieces
    (split = list of (window, piece, npieces) per unit)."""
    out, b = [], 0
    for k, nb in enumerate(nbs):
        sid, piece, npc = (-1, 0, 1) if split is None or split[k] is None else (split[k][0], split[k][1], split[k][2])
        out.append([k, k + 1, b, b + nb, sid, piece, npc, 0])
        b += nb
    return np.array(out, dtype=np.int32)


def test_b200_simulate_hand_worked():
    """List scheduling in unit order on S x O slots, earliest-free slot (lowest on ties):
    1 SM x 2 slots, block 1 ns, no CTA cost: [3,1,2,2,5] -> s0: 3, s1: 1, s1: 3, s0 (tie at 3): 5,
    s1: 8 -> makespan 8; with cta_ns = 1 every unit costs 1 more: s0 4, s1 2, s1 5, s0 7, s1 11."""
    m = dtc.make_model(1, 2, 0.0, 1.0, 0.0)
    assert dtc.selector_simulate(_units([3, 1, 2, 2, 5]), m) == 8.0
    m = dtc.make_model(1, 2, 1.0, 1.0, 0.0)
    assert dtc.selector_simulate(_units([3, 1, 2, 2, 5]), m) == 11.0


def test_b200_simulate_split_fixup_chain():
    """The last piece of a window split into np pieces pays fixup_ns x (G + ceil(np/G)),
    G = np for np <= 4 else ceil(sqrt(np)): 4 pieces of 2 blocks on 4 slots -> 2 + (4 + 1) x 10."""
    m = dtc.make_model(2, 2, 0.0, 1.0, 10.0)
    sp = [(0, p, 4) for p in range(4)]
    assert dtc.selector_simulate(_units([2, 2, 2, 2], sp), m) == 2.0 + 50.0
    sp9 = [(0, p, 9) for p in range(9)]       # G = 3 -> chain 3 + 3 = 6
    m1 = dtc.make_model(9, 1, 0.0, 1.0, 1.0)
    assert dtc.selector_simulate(_units([1] * 9, sp9), m1) == 1.0 + 6.0


def test_b200_plan_closed_forms():
    """Closed-form cases of the plan.  4096 windows of 8 blocks on 888 slots with a CTA cost of 1e6:
    U=16 gives 2048 units = 3 waves (3 x (1e6 + 16)), U=64 512 units and U=256 128 units = one wave
    each (1e6 + 64 and 1e6 + 256) -> U=64.  One 300-block window on one slot: every split finishes
    at 300 (no CTA cost), ties go to the larger U."""
    rwo = np.arange(0, 8 * 4096 + 1, 8, dtype=np.int32)
    r = dtc.selector_plan(rwo, dtc.make_model(148, 6, 1e6, 1.0, 0.0), [16, 64, 256], guided=-1)
    ms = {p["unit_blocks"]: p["makespan_ns"] for p in r["plans"] if p["makespan_ns"] >= 0}
    assert ms == {16: 3 * (1e6 + 16), 64: 1e6 + 64, 256: 1e6 + 256}
    assert r["best"]["unit_blocks"] == 64
    rwo2 = np.array([0, 300], dtype=np.int32)          # one 300-block window, 1 slot: splitting cannot help
    r2 = dtc.selector_plan(rwo2, dtc.make_model(1, 1, 0.0, 1.0, 0.0), [16, 512], guided=-1)
    assert r2["best"]["makespan_ns"] == 300.0 and r2["best"]["unit_blocks"] == 512
