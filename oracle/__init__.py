"""oracle — CPU oracle for the WarpDrive hot path (ctypes wrapper over wd_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs, never by the product package.  It shares no code
with the CUDA path; its only shared dependency is the input generator `wdgen`.

Every function cites the PAPER.md passage it follows (see wd_oracle.c's header).
Parity status per function:
  fmix32, mueller ............ pinned (MurmurHash3 published vectors, Mueller's inverse)
  partition .................. pinned (range/uniformity; Fig. 4 mode k mod m)
  Map (insert/retrieve/size) . pinned (brute-force dictionary on tiny inputs, closed form)
  multisplit, table_scans .... pinned (brute force / permutation + histogram invariants)
  replay (Fig. 3) ............ pinned (single-region closed forms, |g|-independence P:89)
  expected_unique ............ pinned (generator closed form; cross-checked vs Map)
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

import wdgen

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "wd_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

EMPTY_KEY = 0xFFFFFFFF
NOT_FOUND = 0xFFFFFFFF


def build(force: bool = False) -> str:
    """Compile wd_oracle.c with plain gcc -O2 (no vectorisation tricks, single thread)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class _Stats(C.Structure):
    _fields_ = [(n, C.c_uint64) for n in
                ("ops", "windows", "sectors", "new_keys", "updates", "failures", "found",
                 "max_windows", "lines")]

    def as_dict(self):
        return {n: int(getattr(self, n)) for n, _ in self._fields_}


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        u32, u64, p = C.c_uint32, C.c_uint64, C.c_void_p
        L.or_fmix32.argtypes = [u32]; L.or_fmix32.restype = u32
        L.or_mueller.argtypes = [u32]; L.or_mueller.restype = u32
        L.or_partition.argtypes = [u32, u32, u32, C.c_int]; L.or_partition.restype = u32
        L.or_map_create.argtypes = [u64, C.c_int]; L.or_map_create.restype = p
        L.or_map_destroy.argtypes = [p]; L.or_map_destroy.restype = None
        L.or_map_insert.argtypes = [p, p, p, u64]; L.or_map_insert.restype = u64
        L.or_map_retrieve.argtypes = [p, p, p, p, u64]; L.or_map_retrieve.restype = None
        L.or_map_size.argtypes = [p]; L.or_map_size.restype = u64
        L.or_map_pair_status_many.argtypes = [p, p, p, p, u64]
        L.or_map_pair_status_many.restype = None
        L.or_multisplit.argtypes = [p, u64, u32, u32, C.c_int, p, p]
        L.or_multisplit.restype = None
        L.or_table_scans.argtypes = [p, u32, p, p]; L.or_table_scans.restype = None
        L.or_replay_insert.argtypes = [p, u64, u32, C.c_int, u32, u32, p, p, u64, C.POINTER(_Stats)]
        L.or_replay_insert.restype = None
        L.or_replay_query.argtypes = [p, u64, u32, C.c_int, u32, u32, p, p, p, u64,
                                      C.POINTER(_Stats), C.c_int]
        L.or_replay_query.restype = None
        L.or_replay_rebuild.argtypes = [p, p, u64, u32, C.c_int, u32, u32, C.POINTER(_Stats)]
        L.or_replay_rebuild.restype = None
        L.or_replay_base_seed.argtypes = [u32, u32, u64, u32, u32]
        L.or_replay_base_seed.restype = u64
        L.or_region_align.argtypes = []; L.or_region_align.restype = u64
        assert L.or_region_align() == REGION_ALIGN
        L.or_map_erase.argtypes = [p, p, p, u64]; L.or_map_erase.restype = u64
        L.or_replay_base.argtypes = [u32, u32, u64]; L.or_replay_base.restype = u64
        L.or_physical_capacity.argtypes = [u64]; L.or_physical_capacity.restype = u64
        L.or_physical_capacity_a.argtypes = [u64, u64]; L.or_physical_capacity_a.restype = u64
        for f in (L.or_fmix32_many, L.or_mueller_many):
            f.argtypes = [p, p, u64]; f.restype = None
        L.or_partition_many.argtypes = [p, p, u64, u32, u32, C.c_int]
        L.or_partition_many.restype = None
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


# ---------------------------------------------------------------- (1) hashes
def fmix32(x) -> int:
    return int(lib().or_fmix32(int(x) & 0xFFFFFFFF))


def mueller(x) -> int:
    return int(lib().or_mueller(int(x) & 0xFFFFFFFF))


def fmix32_many(x) -> np.ndarray:
    a = _u32(x); y = np.empty_like(a)
    lib().or_fmix32_many(_ptr(a), _ptr(y), a.size)
    return y


def mueller_many(x) -> np.ndarray:
    a = _u32(x); y = np.empty_like(a)
    lib().or_mueller_many(_ptr(a), _ptr(y), a.size)
    return y


# ---------------------------------------------------------------- (2) p(k) (C15)
PART_HASH, PART_MOD = 0, 1


def partition(keys, m: int, seed: int, mode: int = PART_HASH) -> np.ndarray:
    k = _u32(keys).ravel()
    d = np.empty_like(k)
    lib().or_partition_many(_ptr(k), _ptr(d), k.size, m, seed, mode)
    return d


# ---------------------------------------------------------------- (3) the map
class Map:
    """The exact map f: K -> V with upsert and the reserved key (C8)."""

    def __init__(self, expected_keys: int, dup_mode: bool = False):
        self._h = lib().or_map_create(int(expected_keys), int(dup_mode))
        self.dup = dup_mode

    def close(self):
        if self._h:
            lib().or_map_destroy(self._h)
            self._h = None

    __del__ = close

    def insert(self, keys, vals) -> int:
        k, v = _u32(keys), _u32(vals)
        assert k.shape == v.shape
        return int(lib().or_map_insert(self._h, _ptr(k), _ptr(v), k.size))

    def retrieve(self, keys):
        k = _u32(keys)
        vals = np.empty(k.size, np.uint32)
        found = np.empty(k.size, np.uint8)
        lib().or_map_retrieve(self._h, _ptr(k), _ptr(vals), _ptr(found), k.size)
        return vals, found

    def size(self) -> int:
        return int(lib().or_map_size(self._h))

    def erase(self, keys):
        """P:91 deletion; returns found (uint8 per key: was present and is now removed)."""
        k = _u32(keys)
        found = np.empty(k.size, np.uint8)
        lib().or_map_erase(self._h, _ptr(k), _ptr(found), k.size)
        return found

    def pair_status(self, keys, vals) -> np.ndarray:
        """0: (k,v) never inserted; 1: inserted in some call; 2: in k's last call."""
        k, v = _u32(keys), _u32(vals)
        out = np.empty(k.size, np.int8)
        lib().or_map_pair_status_many(self._h, _ptr(k), _ptr(v), _ptr(out), k.size)
        return out


# ---------------------------------------------------------------- (4) multisplit
def multisplit(keys, m: int, seed: int, mode: int = PART_HASH):
    """Stable partition by p(k): returns (counts[m], perm[n]) with perm[i] the output
    position of input i (partitions concatenated in order 0..m-1, Fig. 4)."""
    k = _u32(keys)
    counts = np.zeros(m, np.uint64)
    perm = np.zeros(k.size, np.uint64)
    lib().or_multisplit(_ptr(k), k.size, m, seed, mode, _ptr(counts), _ptr(perm))
    return counts, perm


# ---------------------------------------------------------------- (5) T scans
def table_scans(T):
    T = np.ascontiguousarray(T, dtype=np.uint64)
    m = T.shape[0]
    send_off = np.zeros((m, m), np.uint64)
    recv_off = np.zeros((m, m), np.uint64)
    lib().or_table_scans(_ptr(T), m, _ptr(send_off), _ptr(recv_off))
    return send_off, recv_off


# ---------------------------------------------------------------- (6) Fig. 3 replay
TOMB_WORD = 0xFFFFFFFEFFFFFFFF
# reading C2': region starts are multiples of A slots, A a property of the
# table, the same for every |g| used on it (the probing scheme must not depend on |g|):
# A = 4 (one 32-byte sector) by default, A = 16 (one 128-byte line) for a table created
# with |g| >= 16, so that its 128-byte windows never straddle two lines
REGION_ALIGN = 4
LINE_ALIGN = 16


def region_align_for(group_size: int) -> int:
    """A of a table created with |g| = group_size (0 = dynamic |g|: the default A)."""
    return LINE_ALIGN if int(group_size) >= 16 else REGION_ALIGN


def n_regions(c: int, align: int = REGION_ALIGN) -> int:
    """nb, the number of region starts of a c-slot table (eq. 3's modulus)."""
    return (int(c) - 32) // int(align) + 1


class Replay:
    """Sequential single-group replay of Fig. 3 on a c-slot table (c >= 32, c % A == 0,
    A = align) with hash seed `seed` (P:161 translated variants; P:63 rebuild with a
    distinct one)."""

    def __init__(self, capacity: int, group_size: int, p_max: int = 1024, seed: int = 0,
                 align: int = REGION_ALIGN):
        assert align in (REGION_ALIGN, LINE_ALIGN)
        assert capacity >= 32 and capacity % align == 0
        assert group_size in (1, 2, 4, 8, 16, 32)
        self.c, self.G, self.pmax, self.seed = int(capacity), int(group_size), int(p_max), int(seed)
        self.align = int(align)
        self.table = np.full(self.c, np.uint64(0xFFFFFFFFFFFFFFFF), np.uint64)
        self.ins = _Stats()
        self.qry = _Stats()

    def insert(self, keys, vals):
        k, v = _u32(keys), _u32(vals)
        lib().or_replay_insert(_ptr(self.table), self.c, self.align, self.G, self.pmax, self.seed, _ptr(k),
                               _ptr(v), k.size, C.byref(self.ins))

    def query(self, keys, stats: _Stats | None = None, erase: bool = False):
        k = _u32(keys)
        vals = np.empty(k.size, np.uint32)
        found = np.empty(k.size, np.uint8)
        st = stats if stats is not None else self.qry
        lib().or_replay_query(_ptr(self.table), self.c, self.align, self.G, self.pmax, self.seed, _ptr(k),
                              _ptr(vals), _ptr(found), k.size, C.byref(st), int(erase))
        return vals, found

    def erase(self, keys):
        """P:91 deletion: matching slots become tombstones (reading C9'); returns found."""
        return self.query(keys, _Stats(), erase=True)[1]

    def rebuild(self, seed: int):
        """re-insert every live slot (slot order) into a fresh table with `seed`."""
        old = self.table.copy()
        self.seed = int(seed)
        self.table = np.full(self.c, np.uint64(0xFFFFFFFFFFFFFFFF), np.uint64)
        st = _Stats()
        lib().or_replay_rebuild(_ptr(old), _ptr(self.table), self.c, self.align, self.G, self.pmax,
                                self.seed, C.byref(st))
        return st

    @staticmethod
    def base(k: int, p: int, capacity: int, seed: int = 0, align: int = REGION_ALIGN) -> int:
        return int(lib().or_replay_base_seed(int(k), int(p), int(capacity), int(seed), int(align)))


def physical_capacity(c: int, align: int = REGION_ALIGN) -> int:
    """Slots a table of requested capacity c must have so that eq. 3 has full period
    (nb = (c-32)/A + 1 prime, A = align; reading C13')."""
    return int(lib().or_physical_capacity_a(int(c), int(align)))


# ---------------------------------------------------------------- closed form (generator)
def expected_unique(queries, n_inserted: int, key_seed: int, val_seed: int):
    """Unique-mode answer without a table: key k was inserted iff its generator index
    pi^{-1}(k) < n_inserted, and then its value is values(index) (SURVEY §8(c) 'what pins
    each part').  Exact for every query at any size."""
    q = _u32(queries)
    idx = wdgen.key_index(q, key_seed).astype(np.uint64)
    found = (idx < np.uint64(n_inserted)) & (q != np.uint32(EMPTY_KEY))
    vals = np.full(q.size, NOT_FOUND, np.uint32)
    if found.any():
        z = wdgen.stream(val_seed, wdgen.TAG_VAL, idx[found])
        vals[found] = (z & np.uint64(0xFFFFFFFF)).astype(np.uint32)
    return vals, found.astype(np.uint8)
