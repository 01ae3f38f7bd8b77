"""The C-ABI library loads and exports every symbol include/dtc.h declares; the
host-only entry points (status strings, the window partitioner) behave.  No
compute call is made here (no GPU in this container)."""
import ctypes
import os
import re
import subprocess
import sys

import numpy as np
import pytest

import paper_conf_asplos_fan0024_b200 as dtc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_header_symbol():
    L = dtc.lib()
    names = dtc.exported_symbols()
    assert len(names) >= 15
    for n in names:
        assert hasattr(L, n), n
    out = subprocess.check_output(["nm", "-D", "--defined-only", dtc.library_path()]).decode()
    defined = set(re.findall(r"\bT (dtc_\w+)", out))
    assert set(names) <= defined


def test_library_is_sm100a_only():
    out = subprocess.run(["cuobjdump", "--list-elf", dtc.library_path()], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out)


def test_status_strings():
    L = dtc.lib()
    assert L.dtc_status_string(0) == b"DTC_OK"
    assert L.dtc_status_string(-3) == b"DTC_ERR_DUPLICATE"
    assert L.dtc_status_string(-99) == b"DTC_ERR_UNKNOWN"
    assert b"sm_100a" in L.dtc_version()


def test_partition_windows_prefix_rule():
    rwo = np.array([0, 3, 3, 10, 11, 20], np.int32)
    assert dtc.partition_windows(rwo, 1).tolist() == [0, 5]
    # smallest w with rwo[w] >= ceil(r*T/P)
    assert dtc.partition_windows(rwo, 2).tolist() == [0, 3, 5]
    assert dtc.partition_windows(rwo, 3).tolist() == [0, 3, 5, 5]


@pytest.mark.parametrize("world", [1, 2, 4, 8])
def test_partition_windows_balances_blocks(world):
    rng = np.random.default_rng(world)
    nb = rng.integers(0, 40, size=5000)
    rwo = np.concatenate([[0], np.cumsum(nb)]).astype(np.int32)
    wb = dtc.partition_windows(rwo, world)
    assert wb[0] == 0 and wb[-1] == 5000 and np.all(np.diff(wb) >= 0)
    T = rwo[-1]
    loads = [rwo[wb[r + 1]] - rwo[wb[r]] for r in range(world)]
    assert sum(loads) == T
    assert max(loads) <= T / world + nb.max() + 1


def test_partition_rejects_bad_args():
    with pytest.raises(dtc.DtcError):
        dtc.partition_windows(np.array([0], np.int32), 0)


def test_header_documents_every_entry_point():
    txt = open(os.path.join(ROOT, "include", "dtc.h")).read()
    for n in dtc.exported_symbols():
        assert re.search(r"\b" + n + r"\s*\(", txt)
    assert "PAPER.md:180" in txt and "PAPER.md:68" in txt


def test_product_path_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_fan0024_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cuh", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in src.replace("no oracle", ""), f


def test_default_spmm_kernels_do_not_spill():
    """The padded-row kernels dtc_spmm launches by default (vector C path, untraced) keep the per-block
    MMA sequence in registers: no local-memory access between the first and the last HMMA of any
    instantiation.  A few loop-invariant words may sit on the stack (unit fields and row offsets,
    reloaded per unit or window): at most 16 bytes for TF32 16-row kernels (the 512 B-slice one runs
    7 CTAs per SM on 80 registers), 24 for the FP16 block-pair and TF32 32-row kernels."""
    lib = dtc.library_path()
    out = subprocess.run(["cuobjdump", "-res-usage", lib], capture_output=True, text=True).stdout
    lines = out.splitlines()
    names = []
    for i, line in enumerate(lines):
        m = re.search(r"Function (_ZN3dtc10k_spmm_padILi(\d)ELi\d+ELi\d+ELb1ELi(\d)ELb0E\S*):", line)
        if m:
            names.append(m.group(1))
            stack = int(re.search(r"STACK:(\d+)", lines[i + 1]).group(1))
            local = int(re.search(r"LOCAL:(\d+)", lines[i + 1]).group(1))
            limit = 16 if (m.group(2) == "0" and m.group(3) == "1") else 24
            assert stack <= limit and local <= limit, (m.group(1)[:60], lines[i + 1])
    assert len(names) >= 6
    sass = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
    for name in names:
        body = sass.split("Function : " + name, 1)[1].split("Function : ", 1)[0].splitlines()
        mma = [k for k, l in enumerate(body) if "HMMA" in l]
        assert mma, name[:60]
        hot = body[mma[0]:mma[-1] + 1]
        assert not [l for l in hot if "LDL" in l or "STL" in l], name[:60]


def test_missing_library_fails_loudly(tmp_path):
    """No CPU fallback: with libdtc.so absent the binding raises on the first call into the path."""
    code = ("import sys, paper_conf_asplos_fan0024_b200 as d\n"
            "try:\n    d.lib()\nexcept ImportError as e:\n    print('raised', 'no CPU fallback' in str(e)); sys.exit(0)\n"
            "sys.exit(3)\n")
    env = dict(os.environ, DTC_LIBRARY=str(tmp_path / "libdtc.so"))
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-c", code], env=env, cwd=root, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    assert "raised True" in r.stdout
