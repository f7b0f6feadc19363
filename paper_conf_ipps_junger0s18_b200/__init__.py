"""paper_conf_ipps_junger0s18_b200 — B200-native WarpDrive hot path (Python binding).

A thin ctypes binding over libwarpdrive.so (C-ABI in include/warpdrive.h): argument
marshalling only.  Every step of the hot path runs in the library's sm_100a kernels;
there is NO CPU fallback — importing this package without the built library raises.

    import paper_conf_ipps_junger0s18_b200 as wd
    t = wd.Table(capacity=int(n / 0.95), group_size=4)
    t.insert(keys, vals)                   # torch tensors (cuda or pinned cpu) or numpy
    vals_out, found = t.retrieve(queries)

The module-level functions carry the C names (wd_create, wd_insert, ...) and take raw
integers (pointers, stream handles); `Table` adds tensor/array marshalling.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# WD_LIBRARY: measurement hook for A/B runs of two builds (tools/); default is in-tree
LIB_PATH = os.environ.get("WD_LIBRARY") or os.path.join(_HERE, "libwarpdrive.so")

WD_OK, WD_ERR_INVALID_ARG, WD_ERR_OUT_OF_MEMORY, WD_ERR_CUDA, WD_ERR_NCCL = 0, 1, 2, 3, 4
WD_ERR_TABLE_FULL, WD_ERR_RESERVED_KEY, WD_ERR_EXCHANGE, WD_ERR_UNSUPPORTED = 5, 6, 7, 8
WD_EMPTY_KEY = 0xFFFFFFFF
WD_NOT_FOUND = 0xFFFFFFFF

WD_OPT_GROUP_SIZE, WD_OPT_P_MAX, WD_OPT_BATCH, WD_OPT_SERIAL = 0, 1, 2, 3
WD_OPT_KEYS_IN_FLIGHT, WD_OPT_PART_SEED, WD_OPT_PART_MODE, WD_OPT_PROBE_MODE = 4, 5, 6, 7
WD_OPT_KERNEL_FLAGS, WD_OPT_SLOTS_PER_LANE, WD_OPT_SPAN, WD_OPT_SLICES = 8, 9, 10, 11
WD_OPT_EXCHANGE = 12
WD_OPT_PHASE_TIMING = 13
WD_OPT_AUTO_REBUILD = 15
WD_OPT_QUERY_GROUP_SIZE = 16
WD_OPT_INSERT_GROUP_SIZE = 17
PHASES = ["h2d", "group", "multisplit", "exchange", "probe", "reverse", "unpermute", "d2h",
          "probe_query"]
EXCHANGE_FUSED, EXCHANGE_COPY, EXCHANGE_NCCL = 0, 1, 2
WD_OPT_N_SHARDS, WD_OPT_RANK, WD_OPT_LOCAL_SHARDS, WD_OPT_LAUNCHES = 100, 101, 102, 103
WD_OPT_GROUP_SIZE_USED = 104
WD_OPT_REGION_ALIGN = 105
WD_RANK_HANDLE_BYTES = 256
# int (*)(uint64_t* value, int op, void* ctx)
ALLREDUCE_FN = C.CFUNCTYPE(C.c_int, C.POINTER(C.c_uint64), C.c_int, C.c_void_p)

EXPORTS = ["wd_create", "wd_create_loopback", "wd_create_rank", "wd_rank_handle",
           "wd_rank_connect",
           "wd_destroy", "wd_clear", "wd_insert", "wd_retrieve", "wd_size", "wd_capacity",
           "wd_sync", "wd_set_option", "wd_get_option", "wd_last_error", "wd_error_string",
           "wd_last_error_message", "wd_shard_capacity", "wd_dump", "wd_counters", "wd_erase",
           "wd_rebuild", "wd_insert_sharded", "wd_retrieve_sharded", "wd_phase_times",
           "wd_probe_counts"]


class WarpDriveError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_name(status)}: {msg}")
        self.status = status


def _name(s):
    try:
        return _lib.wd_error_string(s).decode()
    except Exception:  # pragma: no cover
        return str(s)


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python __graft_entry__.py build` "
                          "(or paper_conf_ipps_junger0s18_b200/build.py); there is no fallback")
    L = C.CDLL(LIB_PATH)
    u64, i32, p, i64 = C.c_uint64, C.c_int, C.c_void_p, C.c_int64
    sig = {
        "wd_create": ([u64, i32, i32], p),
        "wd_create_loopback": ([u64, i32, i32], p),
        "wd_create_rank": ([u64, i32, i32, i32], p),
        "wd_rank_handle": ([p, p], i32),
        "wd_rank_connect": ([p, p, p, p], i32),
        "wd_destroy": ([p], None),
        "wd_clear": ([p, p], i32),
        "wd_insert": ([p, p, p, u64, p], i32),
        "wd_retrieve": ([p, p, p, p, u64, p], i32),
        "wd_size": ([p], u64),
        "wd_capacity": ([p], u64),
        "wd_sync": ([p], i32),
        "wd_set_option": ([p, i32, i64], i32),
        "wd_get_option": ([p, i32], i64),
        "wd_last_error": ([], i32),
        "wd_error_string": ([i32], C.c_char_p),
        "wd_last_error_message": ([], C.c_char_p),
        "wd_shard_capacity": ([p, i32], u64),
        "wd_dump": ([p, i32, p], i32),
        "wd_counters": ([p, i32, p], i32),
        "wd_erase": ([p, p, p, u64, p], i32),
        "wd_rebuild": ([p, C.c_uint32, p], i32),
        "wd_insert_sharded": ([p, p, p, p, p], i32),
        "wd_retrieve_sharded": ([p, p, p, p, p, p], i32),
        "wd_phase_times": ([p, p, p], i32),
        "wd_probe_counts": ([p, i32, p], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    return L


_lib = _load()

# C-named thin wrappers (raw ints: pointers and cudaStream_t handles)
for _n in EXPORTS:
    globals()[_n] = getattr(_lib, _n)


def _check(status: int):
    if status != WD_OK:
        raise WarpDriveError(status, _lib.wd_last_error_message().decode())


def _addr(x, itemsize: int | None = None, what: str = "buffer", min_len: int | None = None):
    """(pointer, nelem, is_cuda) of a torch tensor / numpy array / None.  The C-ABI takes
    uint32 keys / values and uint8 found flags: `itemsize` is checked (any 4-byte integer
    dtype is reinterpreted bit for bit; int64 or 1-2-byte keys would be misread), and an
    output must hold at least `min_len` elements."""
    if x is None:
        return None, 0, False
    if isinstance(x, np.ndarray):
        if not x.flags.c_contiguous:
            raise ValueError(f"{what}: must be C-contiguous")
        if itemsize is not None and (x.dtype.itemsize != itemsize or x.dtype.kind not in "iu"):
            raise TypeError(f"{what}: need a {itemsize}-byte integer dtype, got {x.dtype}")
        p, n, cuda = x.ctypes.data, x.size, False
    else:
        import torch
        if not isinstance(x, torch.Tensor):
            raise TypeError(f"unsupported buffer type {type(x)}")
        if not x.is_contiguous():
            raise ValueError(f"{what}: must be contiguous")
        if itemsize is not None and (x.element_size() != itemsize or x.dtype.is_floating_point
                                     or x.dtype.is_complex or x.dtype == torch.bool):
            raise TypeError(f"{what}: need a {itemsize}-byte integer dtype, got {x.dtype}")
        p, n, cuda = x.data_ptr(), x.numel(), x.is_cuda
    if min_len is not None and n < min_len:
        raise ValueError(f"{what}: {n} elements, need at least {min_len}")
    return p, n, cuda


def _stream(stream, dev_hint=None):
    if stream is None:
        import torch
        if not torch.cuda.is_available():
            return 0
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Table:
    """One WarpDrive hash table (single GPU, loopback shards, single-process multi-GPU or
    one shard per rank).  All methods are asynchronous on `stream` except size/sync/dump."""

    def __init__(self, capacity: int, n_gpus: int = 1, group_size: int = 4, *,
                 loopback_shards: int | None = None, rank: int | None = None,
                 world: int | None = None, process_group=None, batch: int | None = None,
                 exchange: int | None = None):
        """rank/world: one process per GPU (torchrun); the exchange handles are all-gathered
        and the host collective is run over `process_group` (torch.distributed)."""
        self._cb = None
        if loopback_shards is not None:
            h = _lib.wd_create_loopback(int(capacity), int(loopback_shards), int(group_size))
        elif rank is not None:
            assert world is not None
            h = _lib.wd_create_rank(int(capacity), int(rank), int(world), int(group_size))
        else:
            h = _lib.wd_create(int(capacity), int(n_gpus), int(group_size))
        if not h:
            raise WarpDriveError(_lib.wd_last_error(), _lib.wd_last_error_message().decode())
        self._h = h
        if batch is not None:
            self.set_option(WD_OPT_BATCH, batch)
        if exchange is not None:        # rank mode: before the handles are exchanged
            self.set_option(WD_OPT_EXCHANGE, exchange)
        if rank is not None:
            self._connect(process_group)

    def _connect(self, group):
        from . import dist as wdist
        blob = (C.c_uint8 * WD_RANK_HANDLE_BYTES)()
        _check(_lib.wd_rank_handle(self._h, C.addressof(blob)))
        blobs = wdist.allgather_bytes(bytes(blob), group)
        allb = (C.c_uint8 * (WD_RANK_HANDLE_BYTES * len(blobs))).from_buffer_copy(b"".join(blobs))

        def _allreduce(vptr, op, ctx):
            try:
                vptr[0] = wdist.allreduce_u64(int(vptr[0]), int(op), group)
                return 0
            except Exception:  # pragma: no cover - reported as WD_ERR_EXCHANGE
                return 1

        self._cb = ALLREDUCE_FN(_allreduce)   # keep alive as long as the table
        _check(_lib.wd_rank_connect(self._h, C.addressof(allb), self._cb, None))

    # -- lifetime
    def close(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.wd_destroy(self._h)
            self._h = None

    def __del__(self):
        self.close()

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    @property
    def handle(self):
        return self._h

    # -- hot path
    def clear(self, stream=None):
        _check(_lib.wd_clear(self._h, _stream(stream)))

    def insert(self, keys, vals, stream=None):
        kp, n, kc = _addr(keys, 4, "keys")
        vp, nv, vc = _addr(vals, 4, "vals")
        if n != nv:
            raise ValueError("keys and vals differ in length")
        _check(_lib.wd_insert(self._h, kp, vp, n, _stream(stream)))

    def retrieve(self, keys, vals_out=None, found_out=None, stream=None):
        kp, n, kc = _addr(keys, 4, "keys")
        if vals_out is None and found_out is None:
            import torch
            dev = keys.device if isinstance(keys, torch.Tensor) else None
            if dev is not None:
                pin = dev.type == "cpu" and keys.is_pinned()
                vals_out = torch.empty(n, dtype=torch.int32, device=dev, pin_memory=pin)
                found_out = torch.empty(n, dtype=torch.uint8, device=dev, pin_memory=pin)
            else:
                vals_out = np.empty(n, np.uint32)
                found_out = np.empty(n, np.uint8)
        vp, _, _ = _addr(vals_out, 4, "vals_out", n)
        fp, _, _ = _addr(found_out, 1, "found_out", n)
        _check(_lib.wd_retrieve(self._h, kp, vp, fp, n, _stream(stream)))
        return vals_out, found_out

    def _local(self):
        return self.get_option(WD_OPT_LOCAL_SHARDS)

    def insert_sharded(self, keys, vals, streams=None):
        """Device-sided cascade: keys[r] / vals[r] are local shard r's
        portion, on its device; streams[r] (optional) is a stream of that device."""
        L = self._local()
        if len(keys) != L or len(vals) != L:
            raise ValueError(f"need {L} portions (one per local shard)")
        kp = (C.c_void_p * L)(*[_addr(k, 4, "keys")[0] for k in keys])
        vp = (C.c_void_p * L)(*[_addr(v, 4, "vals")[0] for v in vals])
        ns = [_addr(k, 4)[1] for k in keys]
        if ns != [_addr(v, 4)[1] for v in vals]:
            raise ValueError("keys and vals differ in length")
        n = (C.c_uint64 * L)(*ns)
        sp = (C.c_void_p * L)(*[_stream(x) for x in streams]) if streams is not None else None
        _check(_lib.wd_insert_sharded(self._h, kp, vp, n, sp))

    def retrieve_sharded(self, keys, vals_out, found_out, streams=None):
        L = self._local()
        if not (len(keys) == len(vals_out) == len(found_out) == L):
            raise ValueError(f"need {L} portions (one per local shard)")
        ns = [_addr(k, 4)[1] for k in keys]
        kp = (C.c_void_p * L)(*[_addr(k, 4, "keys")[0] for k in keys])
        vp = (C.c_void_p * L)(*[_addr(v, 4, "vals_out", n)[0] for v, n in zip(vals_out, ns)])
        fp = (C.c_void_p * L)(*[_addr(f, 1, "found_out", n)[0] for f, n in zip(found_out, ns)])
        sp = (C.c_void_p * L)(*[_stream(x) for x in streams]) if streams is not None else None
        _check(_lib.wd_retrieve_sharded(self._h, kp, vp, fp, (C.c_uint64 * L)(*ns), sp))
        return vals_out, found_out

    def erase(self, keys, found_out=None, stream=None):
        """P:91 deletion; found_out[i] = 1 for the occurrence that removed keys[i]."""
        kp, n, kc = _addr(keys, 4, "keys")
        if found_out is None:
            import torch
            if isinstance(keys, torch.Tensor):
                pin = keys.device.type == "cpu" and keys.is_pinned()
                found_out = torch.empty(n, dtype=torch.uint8, device=keys.device, pin_memory=pin)
            else:
                found_out = np.empty(n, np.uint8)
        fp, _, _ = _addr(found_out, 1, "found_out", n)
        _check(_lib.wd_erase(self._h, kp, fp, n, _stream(stream)))
        return found_out

    def rebuild(self, seed: int, stream=None):
        """re-insert the live entries into a fresh table with hash seed `seed`."""
        _check(_lib.wd_rebuild(self._h, int(seed) & 0xFFFFFFFF, _stream(stream)))

    # -- queries of state
    def size(self) -> int:
        s = _lib.wd_size(self._h)
        if s == 2**64 - 1:
            _check(_lib.wd_last_error() or WD_ERR_CUDA)
        return int(s)

    def capacity(self) -> int:
        return int(_lib.wd_capacity(self._h))

    def sync(self) -> int:
        """Wait; returns the sticky device-side status (0 = WD_OK) without raising."""
        return int(_lib.wd_sync(self._h))

    def set_option(self, opt: int, value: int):
        _check(_lib.wd_set_option(self._h, int(opt), int(value)))

    def get_option(self, opt: int) -> int:
        return int(_lib.wd_get_option(self._h, int(opt)))

    def shard_capacity(self, shard: int = 0) -> int:
        return int(_lib.wd_shard_capacity(self._h, shard))

    def dump(self, shard: int = 0) -> np.ndarray:
        out = np.empty(self.shard_capacity(shard), np.uint64)
        _check(_lib.wd_dump(self._h, shard, out.ctypes.data))
        return out

    def counters(self, shard: int = 0) -> dict:
        out = np.zeros(6, np.uint64)
        _check(_lib.wd_counters(self._h, shard, out.ctypes.data))
        return {"new": int(out[0]), "failed": int(out[1]), "reserved": int(out[2]),
                "exchange_errors": int(out[3]), "last_failed_key": int(out[4]),
                "erased": int(out[5])}

    def phase_times(self) -> dict:
        """Per-phase CUDA-event milliseconds since the last call (WD_OPT_PHASE_TIMING = 1);
        synchronizes and resets.  {phase: (ms, intervals)}"""
        ms = (C.c_double * len(PHASES))()
        cnt = (C.c_uint64 * len(PHASES))()
        _check(_lib.wd_phase_times(self._h, C.addressof(ms), C.addressof(cnt)))
        return {p: (ms[i], int(cnt[i])) for i, p in enumerate(PHASES)}

    def probe_counts(self, shard: int = 0) -> dict:
        """Windows / 128-B lines / CAS attempts / CAS lost / keys of the probe launches since
        the last call (a -DWD_COUNT_PROBES build only; else WarpDriveError UNSUPPORTED)."""
        out = np.zeros(5, np.uint64)
        _check(_lib.wd_probe_counts(self._h, shard, out.ctypes.data))
        return dict(zip(("windows", "lines", "cas", "cas_lost", "keys"), (int(x) for x in out)))

    @property
    def launches(self) -> int:
        return self.get_option(WD_OPT_LAUNCHES)
