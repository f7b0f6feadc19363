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
COMMON_C = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xptxas", "-warn-spills"]
COMMON = COMMON_C + ["-shared"]

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


UNITS = ["warpdrive", "probe_g1", "probe_g2", "probe_g4", "probe_g8", "probe_g16", "probe_g32"]


def build(force: bool = False, verbose: bool = False, extra: list[str] | None = None) -> None:
    """Compile the translation units of libwarpdrive.so in parallel (the probe dispatch is
    instantiated once per |g| in probe_g<G>.cu), then link."""
    from concurrent.futures import ThreadPoolExecutor
    csrc = os.path.join(PKG, "csrc")
    headers = [os.path.join(csrc, "wd_device.cuh"), os.path.join(csrc, "wd_host.cuh"),
               os.path.join(ROOT, "include", "warpdrive.h")]
    objdir = os.path.join(ROOT, "build", "obj")
    os.makedirs(objdir, exist_ok=True)
    objs, jobs = [], []
    for u in UNITS:
        src, obj = os.path.join(csrc, u + ".cu"), os.path.join(objdir, u + ".o")
        objs.append(obj)
        if force or extra or _stale(obj, [src, *headers]):
            tmp = obj + f".tmp{os.getpid()}"
            jobs.append((obj, tmp, [NVCC, *ARCH, *COMMON_C, *(extra or []), "-I",
                                    os.path.join(ROOT, "include"), "-c", "-o", tmp, src]))

    def one(job):
        obj, tmp, cmd = job
        _run(cmd, verbose)
        os.replace(tmp, obj)

    with ThreadPoolExecutor(max_workers=max(1, min(len(jobs), os.cpu_count() or 1))) as ex:
        list(ex.map(one, jobs))
    if jobs or _stale(LIB, objs):
        tmp = LIB + f".tmp{os.getpid()}"
        _run([NVCC, *ARCH, "-shared", "-o", tmp, *objs], verbose)
        os.replace(tmp, LIB)
    gsrc = [os.path.join(ROOT, "wdgen", "wdgen.cu")]
    if force or _stale(GENLIB, gsrc):
        tmp = GENLIB + f".tmp{os.getpid()}"
        _run([NVCC, *ARCH, *COMMON, "-o", tmp, gsrc[0]], verbose)
        os.replace(tmp, GENLIB)


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
