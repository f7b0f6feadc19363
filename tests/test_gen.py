"""Generator pins (CPU): wdgen is shared by oracle and CUDA path, so it is pinned first."""
import json
import math
import os

import numpy as np

import wdgen

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "hash_vectors.json")))
GAMMA = 0x9E3779B97F4A7C15


def test_splitmix64_reference_sequence():
    # SplitMix64 seeded with 0: output_k = mix(k * gamma); our splitmix64(z) = mix(z + gamma)
    want = [int(h, 16) for h in GOLD["splitmix64_seed0_first3"]]
    got = [wdgen.splitmix64((k * GAMMA) & (2**64 - 1)) for k in range(3)]
    assert got == want
    arr = wdgen.splitmix64(np.array([(k * GAMMA) & (2**64 - 1) for k in range(3)], np.uint64))
    assert [int(x) for x in arr] == want


def test_perm32_is_bijection_on_samples():
    rng = np.random.default_rng(1)
    x = rng.integers(0, 2**32 - 1, size=1 << 20, dtype=np.uint64).astype(np.uint32)
    for seed in (0, 7, 123456789):
        y = wdgen.perm32(x, seed)
        assert not np.any(y == np.uint32(wdgen.EMPTY_KEY))
        assert np.array_equal(wdgen.perm32_inv(y, seed), x)


def test_unique_keys_distinct_and_sentinel_free():
    n = 1 << 21
    k = wdgen.unique_keys(n, seed=3)
    assert k.dtype == np.uint32 and k.size == n
    assert np.unique(k).size == n
    assert not np.any(k == np.uint32(0xFFFFFFFF))
    # absent keys pi(n + j) are disjoint from the present ones
    a = wdgen.unique_keys(n, seed=3, start=n)
    assert np.intersect1d(k, a).size == 0
    # index-addressable: a slice equals the corresponding part of the whole
    assert np.array_equal(wdgen.unique_keys(1000, 3, start=5000), k[5000:6000])


def test_cycle_walk_excludes_sentinel_exactly():
    # find the preimage of the sentinel under the raw Feistel network for some seed and
    # check that index maps to pi(0xFFFFFFFF) instead (one cycle-walk step)
    seed = 11
    rk = wdgen._round_keys(seed)
    pre = int(wdgen._feistel(np.array([0xFFFFFFFF], np.uint32), rk, inverse=True)[0])
    y = int(wdgen.perm32(np.array([pre], np.uint32), seed)[0])
    assert y != 0xFFFFFFFF
    assert y == int(wdgen._feistel(np.array([0xFFFFFFFF], np.uint32), rk)[0])
    assert int(wdgen.perm32_inv(np.array([y], np.uint32), seed)[0]) == pre


def test_uniform_keys_bootstrap_ratio():
    # P:156 / P:181: the number of distinct keys among n uniform draws from 2^32 values
    # is 2^32 (1 - exp(-n / 2^32)) in expectation.  Check within 6 sigma.
    n = 1 << 24
    k = wdgen.uniform_keys(n, seed=5)
    assert not np.any(k == np.uint32(0xFFFFFFFF))
    d = np.unique(k).size
    N = 2.0**32
    mean = N * (1 - math.exp(-n / N))
    var = N * math.exp(-n / N) * (1 - (1 + n / N) * math.exp(-n / N))  # occupancy variance
    assert abs(d - mean) < 6 * math.sqrt(var) + 1
    # P:181 closed form: 2^27 draws -> ~98.45% distinct
    assert abs((1 - math.exp(-2**27 / N)) * N / 2**27 - 0.98454) < 1e-5


def test_values_cover_full_range_and_are_indexable():
    v = wdgen.values(1 << 20, seed=9)
    assert v.dtype == np.uint32
    assert np.unique(v).size > 0.999 * v.size
    assert np.array_equal(wdgen.values(10, 9, start=100), v[100:110])


def test_query_streams():
    n = 1000
    q = wdgen.interleaved_queries(n, seed=2)
    k = wdgen.unique_keys(2 * n, seed=2)
    assert np.array_equal(q[0::2], k[:n]) and np.array_equal(q[1::2], k[n:])
    mq, hit = wdgen.mixed_queries(5000, 20000, 0.5, seed=4)
    idx = wdgen.key_index(mq, 4).astype(np.int64)
    assert np.array_equal(idx < 5000, hit)
    assert abs(hit.mean() - 0.5) < 0.02
    mq0, hit0 = wdgen.mixed_queries(5000, 2000, 0.0, seed=4)
    mq1, hit1 = wdgen.mixed_queries(5000, 2000, 1.0, seed=4)
    assert not hit0.any() and hit1.all()


def test_zipf_frequencies_match_power_law():
    # multiplicity of rank k ~ k^-s.  Exact sampler: frequencies within 6 sigma of
    # p_k = k^-s / H_{N,s} for a small universe; keys are distinct per rank.
    N, n, s = 1000, 1 << 21, 1.0 + 1e-6
    r = wdgen.zipf_ranks(n, N, seed=3)
    assert r.min() >= 1 and r.max() <= N
    H = sum(k ** -s for k in range(1, N + 1))
    cnt = np.bincount(r.astype(np.int64), minlength=N + 1)[1:]
    for k in (1, 2, 3, 5, 10, 50, 200, 1000):
        p = k ** -s / H
        assert abs(cnt[k - 1] - n * p) < 6 * math.sqrt(n * p * (1 - p)) + 1, k
    keys = wdgen.zipf_keys(1 << 16, 2**32 - 1, seed=4)
    ranks = wdgen.zipf_ranks(1 << 16, 2**32 - 1, seed=4)
    # rank -> key is injective (pi_s), so equal keys <=> equal ranks
    assert np.unique(keys).size == np.unique(ranks).size
    assert not np.any(keys == np.uint32(0xFFFFFFFF))
