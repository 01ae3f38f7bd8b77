"""Time Format.build (wall, synchronised) per config: first call and repeats."""
import sys, os, time, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from datagen import configs
from paper_conf_asplos_fan0024_b200 import Format
out = {}
for name in sys.argv[1:] or ["c2", "c3", "c4", "c5"]:
    cfg = configs.get(name)
    rp, ci = configs.make_pattern(cfg)
    v = configs.make_values(cfg, len(ci))
    rpd, cid, vd = torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(), torch.from_numpy(v).cuda()
    ts = []
    for it in range(4):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        f = Format.build(rpd, cid, vd, cfg.M, cfg.K, dtype=cfg.dtype)
        torch.cuda.synchronize(); ts.append((time.perf_counter() - t0) * 1e3)
        f.close()
    out[name] = [round(x, 2) for x in ts]
    print(name, "build ms:", out[name], flush=True)
