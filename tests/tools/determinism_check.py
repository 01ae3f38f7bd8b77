"""Determinism + exactness check of dtc_spmm on a config with integer inputs (three runs vs O1 on the
first 200k rows) -- the check that found the early A-slot release race; usage: determinism_check.py c4 256 [U]."""
import sys, os, numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import datagen, oracle
from datagen import configs
import paper_conf_asplos_fan0024_b200 as dtc
name = sys.argv[1] if len(sys.argv) > 1 else "c4"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 256
U = int(sys.argv[3]) if len(sys.argv) > 3 else 0
cfg = configs.get(name)
rp, ci = configs.make_pattern(cfg)
v = datagen.integers(cfg.seed_a, 5, len(ci), -2, 2)
B = datagen.integers(cfg.seed_b, 6, cfg.K * N, -2, 2).reshape(cfg.K, N)
f = dtc.Format.build(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(v).cuda(), cfg.M, cfg.K, unit_blocks=U)
Bd = torch.from_numpy(B).cuda()
Cs = [f.spmm(Bd).cpu().numpy() for _ in range(3)]
print("deterministic:", all(np.array_equal(Cs[0], c) for c in Cs[1:]), "units", f.num_units, "U", f.unit_blocks)
r1 = min(cfg.M, 200000)
Cr = oracle.spmm(cfg.M, cfg.K, rp, ci, v, B, 0, r1, bound=False)
for k, C in enumerate(Cs):
    bad = np.flatnonzero((C[:r1] != Cr).any(axis=1))
    print(k, "bad rows", len(bad), bad[:10])
    if len(bad):
        r = bad[0]; cols = np.flatnonzero(C[r] != Cr[r]); print("  row", r, "bad cols", cols[:20], "got", C[r, cols[:4]], "want", Cr[r, cols[:4]])
e = f.export(); u = e["units"]; rwo = e["row_window_offset"]
if len(bad):
    w = bad[0] // 16
    k = np.flatnonzero((u[:, 0] <= w) & (u[:, 1] > w))
    print("window", w, "blocks", rwo[w], rwo[w+1], "unit(s)", u[k][:3])
