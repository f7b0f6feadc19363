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
        L.wdgen_check_unique.argtypes = [p, p, p, u64, u64, u64, u64, p, p]
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


def check_unique(q, vals_out, found_out, n_present, key_seed, val_seed, chunk=1 << 28):
    """Closed-form check of EVERY query on the device (test harness): query k must report
    found iff pi_s^-1(k) < n_present, with value values(pi_s^-1(k)) (else WD_NOT_FOUND).
    vals_out / found_out may be None.  Returns (mismatches, first mismatching position or
    None, found count).  Generator arithmetic only (wdgen), no code of the method."""
    import torch
    res = torch.tensor([0, -1, 0], dtype=torch.int64, device=q.device)
    n = q.numel()
    for o in range(0, n, chunk):
        c = min(chunk, n - o)
        r = torch.tensor([0, -1, 0], dtype=torch.int64, device=q.device)
        vp = vals_out[o:o + c].data_ptr() if vals_out is not None else None
        fp = found_out[o:o + c].data_ptr() if found_out is not None else None
        _chk(lib().wdgen_check_unique(q[o:o + c].data_ptr(), vp, fp, c, n_present, key_seed,
                                      val_seed, r.data_ptr(), _s()))
        bad, first, found = r.tolist()
        res[0] += bad
        res[2] += found
        if bad and res[1].item() == -1:
            res[1] = o + first
    bad, first, found = res.tolist()
    return int(bad), (int(first) if bad else None), int(found)
