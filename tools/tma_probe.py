"""Run the gather4 hardware probe on the GPU box (python tools/tma_probe.py)."""
import ctypes
import os
import subprocess
import sys

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "libtma_probe.so")


def build():
    subprocess.check_call(["nvcc", "-O2", "-shared", "-Xcompiler", "-fPIC", "-gencode", "arch=compute_100a,code=sm_100a",
                           os.path.join(HERE, "tma_probe.cu"), "-o", SO])


def main():
    import torch
    if not os.path.exists(SO):
        build()
    L = ctypes.CDLL(SO)
    L.tma_probe.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64] + [ctypes.c_int] * 9 + \
        [ctypes.c_void_p, ctypes.c_char_p]
    K, N = 1000, 256
    B = (torch.arange(K * N, dtype=torch.float32).reshape(K, N)).cuda()
    Bh = (torch.arange(K * N, dtype=torch.float32).reshape(K, N) % 2048).half().cuda()
    out = torch.zeros(1024, dtype=torch.int32, device="cuda")
    msg = ctypes.create_string_buffer(256)
    for elt, box_cols, box_rows, sw, col0, rows in [
        (4, 32, 1, 128, 64, (5, 7, 999, 0)),
        (4, 32, 1, 128, 64, (5, -1, 1000, 3)),
        (4, 32, 1, 0, 64, (5, 7, 9, 11)),
        (4, 128, 1, 0, 0, (1, 2, 3, 4)),
        (4, 32, 4, 128, 64, (5, 7, 9, 11)),
        (2, 64, 1, 128, 64, (5, -1, 2000000, 3)),
    ]:
        src = B if elt == 4 else Bh
        out.zero_()
        rc = L.tma_probe(src.data_ptr(), K, N, elt, box_cols, box_rows, sw, col0, *rows, out.data_ptr(), msg)
        print(f"elt={elt} box=({box_cols},{box_rows}) sw={sw} col0={col0} rows={rows}: rc={rc} {msg.value.decode()}")
        if rc != 0:
            continue
        raw = out.cpu().numpy().view(np.uint32)
        nbytes = 4 * box_cols * elt
        words = raw[: nbytes // 4]
        if elt == 4:
            vals = words.view(np.float32).reshape(4, box_cols)
        else:
            vals = words.view(np.float16).reshape(4, box_cols)
        # expected (unswizzled)
        for r in range(4):
            row = rows[r]
            exp = np.zeros(box_cols) if (row < 0 or row >= K) else src[row, col0:col0 + box_cols].float().cpu().numpy()
            got = vals[r].astype(np.float64)
            if sw == 128:
                # undo 128B swizzle: 16B chunk c of row r stored at chunk c ^ (r & 7) (smem row = 128B)
                per = 16 // elt
                un = np.zeros_like(got)
                for c in range(box_cols // per):
                    sc = c ^ (r & 7)
                    un[c * per:(c + 1) * per] = got[sc * per:(sc + 1) * per]
                got = un
            ok = np.array_equal(got, exp)
            print(f"   row{r} ({row}): {'OK' if ok else 'MISMATCH'} got[:8]={got[:8]} exp[:8]={exp[:8]}")
        print("   tail sentinel word:", hex(int(raw[nbytes // 4])) if nbytes // 4 < 1024 else "-")
    sys.stdout.flush()


if __name__ == "__main__":
    main()
