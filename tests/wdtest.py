"""Shared helpers for the GPU parity tests (test harness only)."""
from __future__ import annotations

import numpy as np


def to_dev(a: np.ndarray):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


def from_dev(t) -> np.ndarray:
    return t.cpu().numpy().view(np.uint32)


def capacity_for(n: int, alpha: float) -> int:
    """C13: c = ceil(n / alpha)."""
    import math
    return int(math.ceil(n / alpha))


def gpu_roundtrip(table, keys: np.ndarray, vals: np.ndarray, queries: np.ndarray, host=False):
    """insert keys->vals, then retrieve queries; returns (vals_out, found_out) as numpy."""
    import torch
    if host:
        kk, vv, qq = (torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).pin_memory()
                      for a in (keys, vals, queries))
        table.insert(kk, vv)
        ov = torch.empty(qq.numel(), dtype=torch.int32).pin_memory()
        of = torch.empty(qq.numel(), dtype=torch.uint8).pin_memory()
        table.retrieve(qq, ov, of)
        torch.cuda.synchronize()
        return ov.numpy().view(np.uint32).copy(), of.numpy().copy()
    table.insert(to_dev(keys), to_dev(vals))
    ov, of = table.retrieve(to_dev(queries))
    torch.cuda.synchronize()
    return from_dev(ov), of.cpu().numpy()
