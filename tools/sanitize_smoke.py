"""Small SpMM runs for compute-sanitizer (memcheck / racecheck / synccheck)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import datagen
from datagen import configs
from paper_conf_asplos_fan0024_b200 import Format

cfg = configs.get("c1")
rp, ci = configs.make_pattern(cfg)
for path in ("auto", "ldg", "pers"):
  for dtype in ("tf32", "fp16"):
    v = configs.make_values(cfg, len(ci))
    for N in ((32, 37, 128, 256, 512) if path == "auto" else (37, 128)):
        B = datagen.uniform(1, 2, cfg.K * N).reshape(cfg.K, N)
        if dtype == "fp16":
            v, B = v.astype(np.float16), B.astype(np.float16)
        for U in (0, 3):
            f = Format.build(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda(),
                             torch.from_numpy(v if dtype == "fp16" else v.astype(np.float32)).cuda(),
                             cfg.M, cfg.K, dtype=dtype, unit_blocks=U)
            f.set_option("kernel", "ldg" if path == "ldg" else "auto")
            f.set_option("persistent", 1 if path == "pers" else 0)
            C = f.spmm(torch.from_numpy(B).cuda())
            torch.cuda.synchronize()
            f.close()
print("sanitize smoke done")
