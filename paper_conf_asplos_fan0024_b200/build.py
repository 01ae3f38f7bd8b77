"""Build libdtc.so in-tree: nvcc for sm_100a only (no PTX JIT fallback, no other arch)."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
SO = os.path.join(HERE, "libdtc.so")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_paths():
    import importlib.util
    spec = importlib.util.find_spec("nvidia")
    base = list(spec.submodule_search_locations)[0]
    inc = os.path.join(base, "nccl", "include")
    lib = os.path.join(base, "nccl", "lib")
    if not os.path.exists(os.path.join(inc, "nccl.h")):
        raise RuntimeError("nccl.h not found under " + inc)
    return inc, lib


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def needs_build() -> bool:
    if not os.path.exists(SO):
        return True
    t = os.path.getmtime(SO)
    deps = sources() + glob.glob(os.path.join(CSRC, "*.h")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        [os.path.join(ROOT, "include", "dtc.h")]
    return any(os.path.getmtime(p) > t for p in deps)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    if out is None and not force and not needs_build():
        return SO
    target = out or SO
    inc, lib = nccl_paths()
    nvcc = os.environ.get("NVCC", "nvcc")
    cmd = [nvcc, "-O3", "-std=c++17", "-lineinfo", "--expt-relaxed-constexpr", *ARCH,
           "-shared", "-Xcompiler", "-fPIC", "-cudart", "static",
           "-I", os.path.join(ROOT, "include"), "-I", inc,
           *[f"-D{d}" for d in defines], *sources(), "-o", target + ".tmp",
           "-L", lib, "-l:libnccl.so.2", "-Xlinker", "-rpath=" + lib, "-lcublasLt"]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(SO)
