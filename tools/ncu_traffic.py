"""One dtc_spmm launch per workload, for bench.py's in-run ncu DRAM-traffic capture.

    ncu --metrics dram__bytes_read.sum,... -k regex:k_spmm_(pad|ldg) python tools/ncu_traffic.py \
        --cache DIR --legs c3:256,c2:128,...

Patterns come from DIR/<cfg>.rp.npy / .ci.npy (written by bench.py in the same run), values and B
from the seeded generators; the format is built exactly as bench.py builds it (default options),
then ONE dtc_spmm per leg is launched, in leg order (ncu replays each launch with caches flushed).
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cache", required=True)
    ap.add_argument("--legs", required=True)
    a = ap.parse_args()
    import torch
    from datagen import configs
    import paper_conf_asplos_fan0024_b200 as dtc
    dev = torch.device("cuda", 0)
    for item in a.legs.split(","):
        name, _, n = item.partition(":")
        cfg = configs.get(name)
        N = int(n)
        base = os.path.join(a.cache, name)
        if os.path.exists(base + ".rp.npy"):
            rp, ci = np.load(base + ".rp.npy"), np.load(base + ".ci.npy")
        else:
            rp, ci = configs.make_pattern(cfg)
        v = configs.make_values(cfg, len(ci))
        B = configs.make_B(cfg, N)
        f = dtc.Format.build(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev), torch.from_numpy(v).to(dev),
                             cfg.M, cfg.K, dtype=cfg.dtype)
        Bd = torch.from_numpy(B).to(dev)
        C = torch.empty((cfg.M, N), dtype=torch.float32, device=dev)
        f.spmm(Bd, C)
        torch.cuda.synchronize()
        f.close()
        del Bd, C
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
