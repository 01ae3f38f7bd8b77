"""NEXT-2 measurement: how many gathered B rows would co-scheduled windows share?

For groups of G consecutive row windows (the candidates for one CTA pair / cluster, or one taller
tile), compare the gathered rows of separate windows, sum_w u_w, with the union of the group's
columns |U_w1 u ... u U_wG| (what a cluster multicast of the union, or a G*16-row tile, would
gather once).  Prints, per config and G, the fraction of gathered rows such sharing would save.

    python tools/window_overlap.py c2 c3 c4 c5
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def group_union(rp, ci, M, rows_per_group):
    """sum over groups of rows_per_group consecutive rows of |unique columns|."""
    nb = (M + rows_per_group - 1) // rows_per_group
    g = np.repeat(np.arange(M) // rows_per_group, np.diff(rp))
    key = g.astype(np.int64) * (int(ci.max()) + 1) + ci
    return int(np.unique(key).size), nb


def main():
    from datagen import configs
    for name in sys.argv[1:] or ["c2", "c3", "c4", "c5"]:
        cfg = configs.get(name)
        rp, ci = configs.make_pattern(cfg)
        base, W = group_union(rp, ci, cfg.M, 16)
        out = [f"{name}: sum_w u_w = {base} over {W} windows (mean {base / W:.0f})"]
        for G in (2, 4, 8):
            u, _ = group_union(rp, ci, cfg.M, 16 * G)
            out.append(f"G={G}: union {u} -> saves {100 * (1 - u / base):.1f}% of gathered rows")
        print("; ".join(out), flush=True)


if __name__ == "__main__":
    main()
