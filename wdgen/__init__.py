"""wdgen — seeded, index-addressable input generators (numpy side).

This module is the ONLY code shared by the oracle (`oracle/`) and the CUDA path
(`paper_conf_ipps_junger0s18_b200/`).  It holds none of the method's arithmetic
(no table hash, no probing, no partition function): it only produces the
synthetic workloads of the paper's experiments (§V-A):

* unique keys     — "sampled without replacement ... equivalent to a Fisher-Yates
                    shuffle": k_i = pi_s(i), pi_s a keyed bijection on
                    [0, 2^32-1) (the reserved sentinel 0xFFFFFFFF is excluded);
* absent keys     — pi_s(n + j), disjoint from the first n unique keys;
* uniform keys    — "drawn with replacement from a uniform distribution";
* arbitrary 4-byte values, 0xFFFFFFFF included on purpose.

The same counter-based generator is implemented a second time in CUDA in
`wdgen/wdgen.cu` (device-side generation for the large configs, never timed,
P:175 "test data generation ... omitted"); `tests/test_gen.py` checks the two
agree element by element.

pi_s is a 4-round Feistel network on two 16-bit halves whose round function is
splitmix64, cycle-walked once to skip 0xFFFFFFFF.  Its inverse gives the
closed-form "is key k present, and with which value" answer used at full sizes.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "EMPTY_KEY", "splitmix64", "stream", "perm32", "perm32_inv", "unique_keys",
    "key_index", "values", "uniform_keys", "interleaved_queries", "mixed_queries",
    "TAG_VAL", "TAG_UNI", "TAG_MIX", "TAG_PERM", "zipf_ranks", "zipf_keys", "TAG_ZIPF",
]

EMPTY_KEY = 0xFFFFFFFF
_M64 = (1 << 64) - 1

# stream tags (distinct sub-streams of one seed)
TAG_PERM = 0x5045524D  # "PERM"
TAG_VAL = 0x56414C55   # "VALU"
TAG_UNI = 0x554E4946   # "UNIF"
TAG_MIX = 0x4D495851   # "MIXQ"
TAG_ZIPF = 0x5A495046  # "ZIPF"

_U64 = np.uint64


def splitmix64(z):
    """splitmix64 finalizer (Steele/Lea/Flood) on numpy uint64 arrays or Python ints."""
    if isinstance(z, (int, np.integer)) and not isinstance(z, np.ndarray):
        z = (int(z) + 0x9E3779B97F4A7C15) & _M64
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
        return z ^ (z >> 31)
    z = np.asarray(z, dtype=_U64)
    with np.errstate(over="ignore"):
        z = z + _U64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> _U64(30))) * _U64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> _U64(27))) * _U64(0x94D049BB133111EB)
    return z ^ (z >> _U64(31))


def _stream_key(seed: int, tag: int) -> int:
    return splitmix64((int(seed) ^ (int(tag) << 32)) & _M64)


def stream(seed: int, tag: int, idx):
    """Counter-based stream: splitmix64(stream_key(seed, tag) + idx) (uint64)."""
    k = _stream_key(seed, tag)
    idx = np.asarray(idx, dtype=_U64)
    with np.errstate(over="ignore"):
        return splitmix64(idx + _U64(k))


def _round_keys(seed: int):
    base = _stream_key(seed, TAG_PERM)
    return [splitmix64((base + r) & _M64) for r in range(4)]


def _feistel(x, rk, inverse=False):
    x = np.asarray(x, dtype=np.uint32).astype(_U64)
    L = x >> _U64(16)
    R = x & _U64(0xFFFF)
    rounds = range(3, -1, -1) if inverse else range(4)
    for r in rounds:
        if not inverse:
            F = splitmix64(R ^ _U64(rk[r])) & _U64(0xFFFF)
            L, R = R, L ^ F
        else:
            F = splitmix64(L ^ _U64(rk[r])) & _U64(0xFFFF)
            L, R = R ^ F, L
    return ((L << _U64(16)) | R).astype(np.uint32)


def perm32(x, seed: int):
    """pi_s: bijection on [0, 2^32-1) (uint32 in, uint32 out, never 0xFFFFFFFF)."""
    rk = _round_keys(seed)
    y = _feistel(x, rk)
    bad = y == np.uint32(EMPTY_KEY)
    if np.any(bad):  # cycle-walk: the single excluded point is skipped once
        y = np.where(bad, _feistel(np.full(y.shape, EMPTY_KEY, np.uint32), rk), y)
    return y


def perm32_inv(y, seed: int):
    """Inverse of perm32 on [0, 2^32-1)."""
    rk = _round_keys(seed)
    x = _feistel(y, rk, inverse=True)
    bad = x == np.uint32(EMPTY_KEY)
    if np.any(bad):
        x = np.where(bad, _feistel(np.full(x.shape, EMPTY_KEY, np.uint32), rk, inverse=True), x)
    return x


def unique_keys(n: int, seed: int, start: int = 0):
    """k_i = pi_s(i) for i in [start, start+n): pairwise distinct, never the sentinel."""
    assert start + n <= EMPTY_KEY
    return perm32(np.arange(start, start + n, dtype=np.uint64).astype(np.uint32), seed)


def key_index(keys, seed: int):
    """pi_s^{-1}: the generator index of a key (closed-form presence test: index < n)."""
    return perm32_inv(np.asarray(keys, dtype=np.uint32), seed)


def values(n: int, seed: int, start: int = 0):
    """v_i = lo32(stream(seed, VAL, i)); any uint32 including 0xFFFFFFFF."""
    z = stream(seed, TAG_VAL, np.arange(start, start + n, dtype=_U64))
    return (z & _U64(0xFFFFFFFF)).astype(np.uint32)


def uniform_keys(n: int, seed: int, start: int = 0):
    """Uniform draws with replacement: lo32(z), or hi32(z) if lo32 is the sentinel."""
    z = stream(seed, TAG_UNI, np.arange(start, start + n, dtype=_U64))
    lo = (z & _U64(0xFFFFFFFF)).astype(np.uint32)
    hi = (z >> _U64(32)).astype(np.uint32)
    k = np.where(lo == np.uint32(EMPTY_KEY), hi, lo)
    return np.where(k == np.uint32(EMPTY_KEY), np.uint32(0), k).astype(np.uint32)


def interleaved_queries(n_present: int, seed: int, start: int = 0, count: int | None = None):
    """Config-1 query stream: query j is pi_s(j//2) for even j (present) and
    pi_s(n_present + j//2) for odd j (absent).  Returns keys for j in [start, start+count)."""
    if count is None:
        count = 2 * n_present - start
    j = np.arange(start, start + count, dtype=np.uint64)
    idx = (j >> np.uint64(1)) + (j & np.uint64(1)) * np.uint64(n_present)
    return perm32(idx.astype(np.uint32), seed)


def mixed_queries(n_table: int, count: int, hit_frac: float, seed: int, start: int = 0):
    """Config-4 query mix: query j is a hit with probability hit_frac.
    hit  -> pi_s(r mod n_table); miss -> pi_s(n_table + r mod (2^32-1-n_table)),
    r = hi32(stream(seed, MIX, j)); hit iff lo32 < hit_frac * 2^32."""
    z = stream(seed, TAG_MIX, np.arange(start, start + count, dtype=_U64))
    lo = z & _U64(0xFFFFFFFF)
    r = z >> _U64(32)
    thr = _U64(min(int(hit_frac * 4294967296.0), 4294967296))
    hit = lo < thr
    n_abs = _U64(EMPTY_KEY - n_table)
    idx = np.where(hit, r % _U64(max(n_table, 1)), _U64(n_table) + r % n_abs)
    return perm32(idx.astype(np.uint32), seed), hit


ZIPF_S = 1.0 + 1e-6     # s = 1 + 10^-6
ZIPF_ATTEMPTS = 8


def _zipf_consts(universe: int, expo: float):
    h = lambda x: np.exp(-expo * np.log(x))                                   # noqa: E731
    hi = lambda x: _zh2((1.0 - expo) * np.log(x)) * np.log(x)                  # noqa: E731
    hinv = lambda x: np.exp(_zh1(np.maximum(x * (1.0 - expo), -1.0)) * x)      # noqa: E731
    c1 = hi(np.float64(1.5)) - 1.0
    cn = hi(np.float64(universe) + 0.5)
    sq = 2.0 - hinv(hi(np.float64(2.5)) - h(np.float64(2.0)))
    return h, hi, hinv, c1, cn, sq


def _zh1(x):  # log1p(x)/x
    x = np.asarray(x, np.float64)
    small = np.abs(x) <= 1e-8
    xs = np.where(small, 1.0, x)
    return np.where(small, 1 - x * (0.5 - x * (1.0 / 3 - 0.25 * x)), np.log1p(xs) / xs)


def _zh2(x):  # expm1(x)/x
    x = np.asarray(x, np.float64)
    small = np.abs(x) <= 1e-8
    xs = np.where(small, 1.0, x)
    return np.where(small, 1 + x * 0.5 * (1 + x * (1.0 / 3) * (1 + 0.25 * x)), np.expm1(xs) / xs)


def zipf_ranks(n: int, universe: int, seed: int, start: int = 0, expo: float = ZIPF_S):
    """Zipf ranks k in [1, universe] with P(k) proportional to k^-s ("the
    multiplicity of a key with rank k is smaller than the one of the most common key by a
    factor of k^-s"; s = 1 + 1e-6).  Exact sampler: rejection-inversion (Hormann &
    Derflinger 1996).  Sample i uses the uniforms hi53(stream(seed, ZIPF, 8 i + j)) for
    attempts j < 8; a sample still rejected after 8 attempts (probability < 1e-9) keeps its
    last candidate.  Implemented identically in wdgen.cu (float64)."""
    h, hi, hinv, c1, cn, sq = _zipf_consts(universe, expo)
    idx = np.arange(start, start + n, dtype=_U64)
    k_out = np.zeros(n, np.uint64)
    todo = np.ones(n, bool)
    for j in range(ZIPF_ATTEMPTS):
        z = stream(seed, TAG_ZIPF, idx * _U64(ZIPF_ATTEMPTS) + _U64(j))
        uu = (z >> _U64(11)).astype(np.float64) * (1.0 / 9007199254740992.0)
        u = cn + uu * (c1 - cn)
        x = hinv(u)
        k = np.floor(x + 0.5)
        k = np.clip(k, 1, universe)
        acc = (k - x <= sq) | (u >= hi(k + 0.5) - h(k))
        take = todo & (acc | (j == ZIPF_ATTEMPTS - 1))
        k_out[take] = k[take].astype(np.uint64)
        todo &= ~take
        if not todo.any():
            break
    return k_out


def zipf_keys(n: int, universe: int, seed: int, start: int = 0):
    """Zipf-distributed keys: rank r -> key pi_s(r - 1) (distinct ranks, distinct keys)."""
    r = zipf_ranks(n, universe, seed, start)
    return perm32((r - _U64(1)).astype(np.uint32), seed)
