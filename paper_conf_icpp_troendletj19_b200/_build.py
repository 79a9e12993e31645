"""Build the in-tree shared libraries with nvcc for sm_100a.

libtq.so    <- csrc/*.cu           (the product: kernels + C ABI of include/tq.h)

The .so lands next to this file so it travels with the repo snapshot to the
GPU box (git-ignored, not gpurun-ignored).
"""
from __future__ import annotations

import glob
import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libtq.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xcompiler", "-O2",
         "-shared", "-diag-suppress", "128"]


def sources() -> list[str]:
    return sorted(glob.glob(os.path.join(HERE, "csrc", "*.cu")))


def deps() -> list[str]:
    return (sources() + glob.glob(os.path.join(HERE, "csrc", "*.cuh"))
            + glob.glob(os.path.join(ROOT, "include", "*")))


def up_to_date(lib: str, inputs: list[str]) -> bool:
    if not os.path.exists(lib):
        return False
    t = os.path.getmtime(lib)
    return all(os.path.getmtime(d) <= t for d in inputs)


def build(force: bool = False, verbose: bool = False, out: str | None = None, defines=()) -> str:
    """Build libtq.so (or, for A/B experiments, `out` with extra -D `defines`)."""
    lib = out or LIB
    if not force and up_to_date(lib, deps()):
        return lib
    tmp = lib + f".tmp{os.getpid()}"
    cmd = [NVCC, *ARCH, *FLAGS, *(f"-D{d}" for d in defines), "-I", os.path.join(ROOT, "include"), "-o", tmp,
           *sources()]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
        print(" ".join(cmd))
    subprocess.check_call(cmd)
    os.replace(tmp, lib)
    return lib


if __name__ == "__main__":
    import sys
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))


def build_user_kernel(src: str, out: str, force: bool = False) -> str:
    """Build a standalone user-kernel library against the public headers
    (include/tq.h, include/tq_device.cuh) -- e.g. the device-API test kernel
    tests/csrc/devapi_test.cu -> tests/libtqdevapi.so."""
    inputs = [src] + glob.glob(os.path.join(ROOT, "include", "*"))
    if not force and up_to_date(out, inputs):
        return out
    tmp = out + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, *FLAGS, "-I", os.path.join(ROOT, "include"), "-o", tmp, src])
    os.replace(tmp, out)
    return out
