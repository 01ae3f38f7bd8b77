"""Calibrate p_local per G1 config so MeanNnzTC hits the SURVEY §8(d) target.

Run once; the resulting p_local values are frozen in datagen/configs.py.
Uses only datagen/ and the oracle's condensation count (oracle/).
    python tests/tools/calibrate.py c1 c2 c3 c5
"""
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))

from datagen import configs  # noqa: E402
import oracle  # noqa: E402


def mean_nnz_tc(cfg, p):
    rp, ci = configs.make_pattern(cfg, p_local=p)
    _, T = oracle.condense_count(cfg.M, rp, ci)
    return len(ci) / T


def main(names):
    for name in names:
        cfg = configs.get(name)
        target = cfg.mean_nnz_tc_target
        lo, hi = 0.0, 0.99
        best = None
        for it in range(10):
            mid = 0.5 * (lo + hi)
            m = mean_nnz_tc(cfg, mid)
            print(f"{name} p_local={mid:.4f} MeanNnzTC={m:.3f} (target {target})", flush=True)
            if best is None or abs(m - target) < abs(best[1] - target):
                best = (mid, m)
            if abs(m - target) / target < 0.02:
                break
            if m < target:
                lo = mid
            else:
                hi = mid
        print(f"RESULT {name} p_local={best[0]:.4f} MeanNnzTC={best[1]:.3f}", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["c1", "c2", "c3", "c5"])
