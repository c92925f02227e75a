"""Build libabft.so (nvcc, sm_100a) in-tree.  No JIT cache: the .so lives in
the package directory so it travels to the GPU box with the repo."""
from __future__ import annotations

import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libabft.so")
ROOT = os.path.dirname(PKG)

def nccl_dir() -> str:
    """NCCL headers + library: the wheel torch itself loads (one libnccl.so.2
    per process), else the system copy."""
    try:
        import nvidia
        for base in list(nvidia.__path__):
            d = os.path.join(base, "nccl")
            if os.path.exists(os.path.join(d, "include", "nccl.h")):
                return d
    except Exception:  # noqa: BLE001
        pass
    return "/usr"


def nccl_flags() -> list:
    d = nccl_dir()
    inc, lib = os.path.join(d, "include"), os.path.join(d, "lib")
    if d == "/usr":
        lib = "/usr/lib/x86_64-linux-gnu"
    return ["-I" + inc, "-L" + lib, "-Xlinker", "-rpath," + lib, "-l:libnccl.so.2"]


NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-ffp-contract=off",
    "-fmad=false",            # no FMA contraction anywhere (R1)
    "-Xcompiler", "-fPIC", "-shared",
    "-cudart", "static",
]


def sources():
    out = [os.path.join(ROOT, "include", "abft.h")]
    for f in sorted(os.listdir(CSRC)):
        if f.endswith((".cu", ".cuh", ".inc", ".h")):
            out.append(os.path.join(CSRC, f))
    return out


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def nvcc() -> str:
    for c in ("/usr/local/cuda/bin/nvcc", "nvcc"):
        if os.path.sep not in c or os.path.exists(c):
            return c
    return "nvcc"


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    cmd = [nvcc(), *NVCC_FLAGS, "-o", LIB + ".tmp", os.path.join(CSRC, "abft.cu"), *nccl_flags()]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    return LIB


if __name__ == "__main__":
    build(force=True, verbose=True)
    print(LIB)
