"""Per-CTA timeline of the TMA-path SpMM kernel (dtc_format_set_trace) -- diagnostics, not product code.

The paper's per-SM busy/idle method (Fig. 3; Fig. 15) on B200:
    python tools/trace_cta.py c2 [--unit-blocks U] [--out gpurun_out/trace_c2.npz]
One L2-flushed dtc_spmm over the config; prints the kernel span, CTA waves, the startup latency
of a CTA (start -> first B stage landed), per-block time, and per-SM busy fraction.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--unit-blocks", type=int, default=0)
    ap.add_argument("--out", default="")
    ap.add_argument("--persistent", type=int, default=0)
    a = ap.parse_args()
    import torch
    from datagen import configs
    import paper_conf_asplos_fan0024_b200 as dtc
    cfg = configs.get(a.config)
    N = cfg.N
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    B = configs.make_B(cfg, N)
    f = dtc.Format.build(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(v).cuda(),
                         cfg.M, cfg.K, dtype=cfg.dtype, unit_blocks=a.unit_blocks)
    f.set_option("persistent", a.persistent)
    Bd = torch.from_numpy(B).cuda()
    C = torch.empty((cfg.M, N), device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    cap = f.num_units * 8
    tr = torch.zeros((cap, 8), dtype=torch.int64, device="cuda")
    for _ in range(3):
        f.spmm(Bd, C)
    flush.zero_()
    torch.cuda.synchronize()
    f.set_trace(tr)
    f.spmm(Bd, C)
    torch.cuda.synchronize()
    f.set_trace(None)
    t = tr.cpu().numpy()
    t = t[t[:, 2] > 0]
    t0 = t[:, 2].min()
    start, issue, data, cdone, nb, pdone = (t[:, 2] - t0, t[:, 3] - t0, t[:, 4] - t0, t[:, 5] - t0, t[:, 6],
                                             t[:, 7] - t0)
    has = nb > 0
    span = max(cdone.max(), pdone.max())
    life = cdone - start
    print(f"{a.config}: {len(t)} CTAs, span {span / 1e3:.1f} us, T={int(nb.sum())} blocks")
    q = lambda x: np.percentile(x, [5, 50, 95]).round(0).astype(int).tolist()
    print("  CTA lifetime ns p5/50/95:", q(life))
    print("  start -> first TMA issue ns:", q(issue[has] - start[has]))
    print("  first issue -> first data ns:", q(data[has] - issue[has]))
    print("  first data -> consumer done ns:", q(cdone[has] - data[has]))
    per_blk = (cdone[has] - data[has]) / np.maximum(nb[has], 1)
    print("  steady ns per block:", q(per_blk))
    sm = t[:, 1]
    busy = np.zeros(sm.max() + 1)
    np.add.at(busy, sm, life)
    res = np.bincount(sm)
    conc = busy / span
    print(f"  per-SM summed CTA-time / span (avg resident CTAs): p5/50/95 {np.percentile(conc, [5, 50, 95]).round(2).tolist()}")
    last_start = start.max()
    print(f"  last CTA start at {last_start / 1e3:.1f} us ({100 * last_start / span:.0f}% of span); "
          f"tail after it {(span - last_start) / 1e3:.1f} us")
    # resident-CTA profile over time (10 buckets)
    edges = np.linspace(0, span, 11)
    prof = [int(np.sum((start < e1) & (cdone > e0))) for e0, e1 in zip(edges[:-1], edges[1:])]
    print("  CTAs alive per span decile:", prof)
    if a.out:
        np.savez(a.out, trace=t)


if __name__ == "__main__":
    main()
