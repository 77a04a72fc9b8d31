"""Build libspinfer.so in-tree with nvcc for sm_100a (no JIT cache, no torch extension)."""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "libspinfer.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
    "-shared", "-cudart", "static",
]


def sources():
    return sorted(glob.glob(os.path.join(PKG, "csrc", "*.cu")))


def deps():
    return sources() + sorted(glob.glob(os.path.join(PKG, "csrc", "*.cuh"))) + [os.path.join(ROOT, "include", "spinfer.h")]


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in deps())


LIB_INSTR = os.path.join(PKG, "libspinfer_instr.so")   # experiments only (stage trace, debug modes)
LIB_DBG = os.path.join(PKG, "libspinfer_dbg.so")       # experiments only (debug modes, no trace)


def build(force: bool = False, verbose: bool = False, instrumented: int = 0) -> str:
    out = {0: LIB, 1: LIB_INSTR, 2: LIB_DBG}[int(instrumented)]
    if not force and not instrumented and up_to_date():
        return LIB
    cmd = [NVCC, *NVCC_FLAGS, "-I", os.path.join(ROOT, "include"), *sources(), "-o", out + ".tmp"]
    if instrumented:
        cmd.append(f"-DSPINFER_INSTRUMENT={int(instrumented)}")
    if verbose:
        cmd[1:1] = ["-Xptxas", "-v"]
    subprocess.check_call(cmd)
    os.replace(out + ".tmp", out)
    return out


if __name__ == "__main__":
    print(build(force=True, verbose="-v" in sys.argv,
                instrumented=1 if "--instrumented" in sys.argv else 2 if "--debug-modes" in sys.argv else 0))
