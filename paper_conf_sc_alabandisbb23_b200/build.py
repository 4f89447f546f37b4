"""Build libeclscc.so in-tree with nvcc for sm_100a (no JIT cache: the .so travels with the
repo snapshot to the GPU box)."""
from __future__ import annotations

import glob
import os
import subprocess
import sysconfig

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libeclscc.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def nccl_dirs() -> tuple[str, str]:
    """NCCL headers + library shipped with torch's nvidia-nccl wheel (2.28.x)."""
    site = sysconfig.get_paths()["purelib"]
    base = os.path.join(site, "nvidia", "nccl")
    return os.path.join(base, "include"), os.path.join(base, "lib")


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")))


def deps() -> list[str]:
    return sources() + sorted(glob.glob(os.path.join(CSRC, "*.cuh"))) + sorted(
        glob.glob(os.path.join(CSRC, "*.h"))) + [os.path.join(ROOT, "include", "ecl_scc.h")]


def build(force: bool = False, verbose: bool = False) -> str:
    if os.environ.get("ECL_PROF") == "1" or os.environ.get("ECL_NVCC_EXTRA"):
        force = True
    if not force and os.path.exists(LIB):
        t = os.path.getmtime(LIB)
        if all(os.path.getmtime(d) <= t for d in deps()):
            return LIB
    inc, lib = nccl_dirs()
    tmp = LIB + f".tmp{os.getpid()}"
    extra = ["-DECL_PROF"] if os.environ.get("ECL_PROF") == "1" else []
    extra += os.environ.get("ECL_NVCC_EXTRA", "").split()       # development: variant -D flags
    cmd = [NVCC, "-O3", "-std=c++17", *ARCH, "-lineinfo", *extra, "-Xcompiler", "-fPIC", "-shared",
           "-I", os.path.join(ROOT, "include"), "-I", inc, "-o", tmp, *sources(),
           "-L", lib, "-l:libnccl.so.2", f"-Xlinker", f"-rpath={lib}"]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force=True, verbose=True))
