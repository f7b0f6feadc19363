"""Device-side generator (wdgen/libwdgen.so): the same counter-based streams as
wdgen/__init__.py, written straight into CUDA tensors.  Generator only."""
from __future__ import annotations

import ctypes as C
import os

_LIB = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libwdgen.so")
_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(_LIB)
        u64, p = C.c_uint64, C.c_void_p
        L.wdgen_unique_keys.argtypes = [p, u64, u64, u64, p]
        L.wdgen_values.argtypes = [p, u64, u64, u64, p]
        L.wdgen_uniform_keys.argtypes = [p, u64, u64, u64, p]
        L.wdgen_interleaved_queries.argtypes = [p, u64, u64, u64, u64, p]
        L.wdgen_mixed_queries.argtypes = [p, p, u64, u64, u64, C.c_double, u64, p]
        L.wdgen_zipf_keys.argtypes = [p, u64, u64, u64, u64, p]
        _lib = L
    return _lib


def _s():
    import torch
    return torch.cuda.current_stream().cuda_stream


def _chk(r):
    if r != 0:
        raise RuntimeError(f"wdgen kernel launch failed (cudaError {r})")


def _new(n, dtype=None):
    import torch
    return torch.empty(int(n), dtype=dtype or torch.int32, device="cuda")


def unique_keys(n, seed, start=0, out=None):
    out = _new(n) if out is None else out
    _chk(lib().wdgen_unique_keys(out.data_ptr(), start, n, seed, _s()))
    return out


def values(n, seed, start=0, out=None):
    out = _new(n) if out is None else out
    _chk(lib().wdgen_values(out.data_ptr(), start, n, seed, _s()))
    return out


def uniform_keys(n, seed, start=0, out=None):
    out = _new(n) if out is None else out
    _chk(lib().wdgen_uniform_keys(out.data_ptr(), start, n, seed, _s()))
    return out


def interleaved_queries(n_present, seed, start=0, count=None, out=None):
    count = 2 * n_present - start if count is None else count
    out = _new(count) if out is None else out
    _chk(lib().wdgen_interleaved_queries(out.data_ptr(), n_present, start, count, seed, _s()))
    return out


def mixed_queries(n_table, count, hit_frac, seed, start=0, out=None, hits=None):
    import torch
    out = _new(count) if out is None else out
    hp = hits.data_ptr() if hits is not None else None
    _chk(lib().wdgen_mixed_queries(out.data_ptr(), hp, n_table, start, count, float(hit_frac),
                                   seed, _s()))
    return out


def zipf_keys(n, universe, seed, start=0, out=None):
    out = _new(n) if out is None else out
    _chk(lib().wdgen_zipf_keys(out.data_ptr(), start, n, universe, seed, _s()))
    return out
