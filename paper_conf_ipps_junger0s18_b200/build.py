"""Build the in-tree shared libraries with nvcc for sm_100a (no JIT, no torch extension):

  paper_conf_ipps_junger0s18_b200/libwarpdrive.so   the product (C-ABI, include/warpdrive.h)
  wdgen/libwdgen.so                                  device-side input generator (bench/tests)

The multi-GPU exchange is peer-memory stores/loads inside the kernels (CUDA IPC for one
process per GPU), so the library links only the CUDA runtime.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
COMMON = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
          "-Xptxas", "-warn-spills"]

LIB = os.path.join(PKG, "libwarpdrive.so")
GENLIB = os.path.join(ROOT, "wdgen", "libwdgen.so")


def _stale(out, srcs):
    if not os.path.exists(out):
        return True
    t = os.path.getmtime(out)
    return any(os.path.getmtime(s) > t for s in srcs)


def _run(cmd, verbose):
    if verbose:
        print(" ".join(cmd), file=sys.stderr)
    subprocess.check_call(cmd)


def build(force: bool = False, verbose: bool = False, extra: list[str] | None = None) -> None:
    srcs = [os.path.join(PKG, "csrc", "warpdrive.cu"), os.path.join(PKG, "csrc", "wd_device.cuh"),
            os.path.join(ROOT, "include", "warpdrive.h")]
    if force or _stale(LIB, srcs):
        tmp = LIB + f".tmp{os.getpid()}"
        _run([NVCC, *ARCH, *COMMON, *(extra or []), "-I", os.path.join(ROOT, "include"),
              "-o", tmp, srcs[0]], verbose)
        os.replace(tmp, LIB)
    gsrc = [os.path.join(ROOT, "wdgen", "wdgen.cu")]
    if force or _stale(GENLIB, gsrc):
        tmp = GENLIB + f".tmp{os.getpid()}"
        _run([NVCC, *ARCH, *COMMON, "-o", tmp, gsrc[0]], verbose)
        os.replace(tmp, GENLIB)


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
