"""Full-size parity with EVERY query checked (BASELINE configs 2-5 on one B200).

The checks are closed forms of the seeded generator, evaluated on the device by
wdgen.gpu.check_unique (generator arithmetic only; pinned against oracle.expected_unique in
tests/test_gpu_gen.py): a key is present iff its generator index pi_s^-1(k) < n, and then its
value is values(pi_s^-1(k)).  Duplicate mode is checked against the sorted list of every
drawn (key, value) pair on the device: found-ness exactly, and each returned value must be
one of the values drawn for its key.  No sample: every query of every
call below is compared.  Marked gpu."""
import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

KS, VS = 0x5EED, 0xBEEF     # the bench's seeds (bench.py KEY_SEED / VAL_SEED)


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg
    return wd, gg, torch


def _check_all(gg, q, vout, fout, n_present, ks=KS, vs=VS, expect_found=None):
    bad, first, found = gg.check_unique(q, vout, fout, n_present, ks, vs)
    assert bad == 0, f"{bad} of {q.numel()} queries differ from the closed form (first at {first})"
    if expect_found is not None:
        assert found == expect_found, (found, expect_found)
    return found


def _roundtrip_all(wd, gg, torch, t, n, keys, n_absent=1 << 26, ks=KS, vs=VS):
    """retrieve all n keys (insert order, like bench.py) and n_absent never-inserted keys;
    every answer against the closed form"""
    vout = torch.empty(n, dtype=torch.int32, device="cuda")
    fout = torch.empty(n, dtype=torch.uint8, device="cuda")
    t.retrieve(keys, vout, fout)
    _check_all(gg, keys, vout, fout, n, ks, vs, expect_found=n)
    if n_absent:
        absent = gg.unique_keys(n_absent, ks, start=n)
        t.retrieve(absent, vout[:n_absent], fout[:n_absent])
        _check_all(gg, absent, vout[:n_absent], fout[:n_absent], n, ks, vs, expect_found=0)
    assert t.sync() == 0, wd._lib.wd_last_error_message()


def test_bench_configuration_every_query(env):
    # the exact configuration bench.py times: 2^28 unique pairs, alpha 0.95, |g| = 16,
    # auto slice-grouped insert (16 slices over 2^26-pair chunks), default V / K, queries
    # in insert order (scrambled chunk order inside the kernel) — plus a second insert of
    # the same keys with new values (upsert) and 2^26 absent keys
    wd, gg, torch = env
    n = 1 << 28
    keys, vals = gg.unique_keys(n, KS), gg.values(n, VS)
    with wd.Table(int(math.ceil(n / 0.95)), 1, 16) as t:
        for rep in range(2):                       # clear + insert + retrieve, twice
            t.clear()
            l0 = t.launches
            t.insert(keys, vals)
            assert t.launches - l0 > 1             # the sliced path ran
            assert t.sync() == 0 and t.size() == n
            _roundtrip_all(wd, gg, torch, t, n, keys)
        vs2 = VS + 1                               # upsert: every key gets a new value
        t.insert(keys, gg.values(n, vs2))
        assert t.size() == n
        _roundtrip_all(wd, gg, torch, t, n, keys, n_absent=0, vs=vs2)


@pytest.mark.parametrize("alpha", [0.8, 0.9, 0.95, 0.99])
@pytest.mark.parametrize("G", [1, 2, 4, 8, 16, 32])
def test_config2_grid_every_query(env, alpha, G):
    # BASELINE config 2: 2^28 pairs, the full alpha x |g| grid; every query of the
    # retrieve of all keys and of 2^26 absent keys
    wd, gg, torch = env
    n = 1 << 28
    keys, vals = gg.unique_keys(n, KS), gg.values(n, VS)
    with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
        t.insert(keys, vals)
        del vals
        assert t.sync() == 0 and t.size() == n
        for qg in (0, -1):          # queries with the table's |g| (the paper's), and the default
            t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, qg)
            _roundtrip_all(wd, gg, torch, t, n, keys)


def test_config3_single_gpu_every_query(env):
    # BASELINE config 3 at m = 1: every non-sentinel 4-byte key (n = 2^32 - 1, C14) into a
    # 4.52e9-slot table (36 GB, 64-bit slot indices) at alpha 0.95, |g| = 4; all 2^32 - 1
    # keys queried back (chunks of 2^28), every answer checked; plus the reserved key
    wd, gg, torch = env
    free, _ = torch.cuda.mem_get_info()
    if free < 100e9:
        pytest.skip("needs ~90 GB of device memory")
    n = (1 << 32) - 1
    with pytest.raises(RuntimeError):
        gg.unique_keys(1, KS, start=n)             # generator index 2^32 - 1 does not exist
    keys = gg.unique_keys(n, 111)
    vals = gg.values(n, 112)
    with wd.Table(int(math.ceil(n / 0.95)), 1, 4) as t:
        t.insert(keys, vals)
        del vals
        assert t.sync() == 0 and t.size() == n
        C = 1 << 28
        vout = torch.empty(C, dtype=torch.int32, device="cuda")
        fout = torch.empty(C, dtype=torch.uint8, device="cuda")
        total = 0
        for o in range(0, n, C):
            c = min(C, n - o)
            t.retrieve(keys[o:o + c], vout[:c], fout[:c])
            total += _check_all(gg, keys[o:o + c], vout[:c], fout[:c], n, 111, 112, expect_found=c)
        assert total == n
        rq = torch.full((5,), -1, dtype=torch.int32, device="cuda")     # 0xFFFFFFFF
        t.retrieve(rq, vout[:5], fout[:5])
        _check_all(gg, rq, vout[:5], fout[:5], n, 111, 112, expect_found=0)
        assert t.sync() == wd.WD_ERR_RESERVED_KEY
        assert t.size() == n


@pytest.mark.parametrize("G", [4, 16])
def test_config4_query_mix_every_query(env, G):
    # BASELINE config 4 on one GPU: a 2^31-key table (c = 2,260,509,104 slots, 18 GB) and
    # 2^32 queries per hit fraction h in {0, 0.5, 1} (chunks of 2^30); found must equal the
    # generator's hit flag and every value the closed form
    wd, gg, torch = env
    free, _ = torch.cuda.mem_get_info()
    if free < 50e9:
        pytest.skip("needs ~40 GB of device memory")
    n = 1 << 31
    keys, vals = gg.unique_keys(n, KS), gg.values(n, VS)
    with wd.Table(2_260_509_104, 1, G) as t:
        t.insert(keys, vals)
        del keys, vals
        assert t.sync() == 0 and t.size() == n
        C = 1 << 30
        q = torch.empty(C, dtype=torch.int32, device="cuda")
        hits = torch.empty(C, dtype=torch.uint8, device="cuda")
        vout = torch.empty(C, dtype=torch.int32, device="cuda")
        fout = torch.empty(C, dtype=torch.uint8, device="cuda")
        for h in (0.0, 0.5, 1.0):
            found = 0
            for o in range(0, 1 << 32, C):
                gg.mixed_queries(n, C, h, KS, start=o, out=q, hits=hits)
                t.retrieve(q, vout, fout)
                found += _check_all(gg, q, vout, fout, n)
                assert bool((fout == hits).all())
            if h == 0.0:
                assert found == 0
            elif h == 1.0:
                assert found == 1 << 32
            else:
                assert abs(found / 2**32 - 0.5) < 1e-3
        assert t.sync() == 0


def _pairs_sorted(torch, keys, vals):
    p = ((keys.to(torch.int64) & 0xFFFFFFFF) << 32) | (vals.to(torch.int64) & 0xFFFFFFFF)
    return torch.sort(p).values


def _check_dup(torch, keys, vout, fout, pairs, uniq):
    """duplicate mode: found iff the key was drawn; a found value is one of the key's drawn
    values (membership of (k, v) in the sorted pair list)"""
    k64 = keys.to(torch.int64) & 0xFFFFFFFF
    pos = torch.searchsorted(uniq, k64).clamp(max=uniq.numel() - 1)
    drawn = uniq[pos] == k64
    assert bool((fout.to(torch.bool) == drawn).all()), "found != drawn"
    got = (k64 << 32) | (vout.to(torch.int64) & 0xFFFFFFFF)
    sel = drawn
    g = got[sel]
    pp = torch.searchsorted(pairs, g).clamp(max=pairs.numel() - 1)
    assert bool((pairs[pp] == g).all()), "a returned value was never drawn for its key"
    nf = vout[~sel]
    assert bool((nf == -1).all()), "not-found value must be WD_NOT_FOUND"


@pytest.mark.parametrize("host", [True, False])
def test_config5_scaled_duplicates_every_query(env, host):
    # BASELINE config 5 scaled to one GPU: 2^30 uniform draws WITH replacement (duplicate
    # keys) into a table sized for the expected distinct count at alpha 0.95 (C13);
    # host=True streams them from pinned host memory (a11, batches of 2^22), host=False
    # from HBM.  Every draw is queried back plus 2^24 fresh uniform keys (mostly absent):
    # found exactly, every value among the drawn ones, size = #distinct.
    wd, gg, torch = env
    n = 1 << 30
    keys, vals = gg.uniform_keys(n, KS), gg.values(n, VS)
    uniq = torch.unique(keys.to(torch.int64) & 0xFFFFFFFF)      # sorted
    distinct = uniq.numel()
    expect = 2**32 * (1 - math.exp(-n / 2**32))
    assert abs(distinct - expect) < 5 * math.sqrt(expect)       # P:156 bootstrap ratio
    pairs = _pairs_sorted(torch, keys, vals)
    extra = gg.uniform_keys(1 << 24, KS + 7)
    with wd.Table(int(math.ceil(expect / 0.95)), 1, 8, batch=1 << 22) as t:
        if host:
            hk = torch.empty(n, dtype=torch.int32, pin_memory=True)
            hv = torch.empty(n, dtype=torch.int32, pin_memory=True)
            hk.copy_(keys)
            hv.copy_(vals)
            del vals
            t.insert(hk, hv)
            hvo = torch.empty(n, dtype=torch.int32, pin_memory=True)
            hfo = torch.empty(n, dtype=torch.uint8, pin_memory=True)
            t.retrieve(hk, hvo, hfo)
            torch.cuda.synchronize()
            vout, fout = hvo.cuda(), hfo.cuda()
            del hk, hv, hvo, hfo
        else:
            t.insert(keys, vals)
            del vals
            vout = torch.empty(n, dtype=torch.int32, device="cuda")
            fout = torch.empty(n, dtype=torch.uint8, device="cuda")
            t.retrieve(keys, vout, fout)
        assert t.sync() == 0 and t.size() == distinct
        assert bool((fout == 1).all())
        _check_dup(torch, keys, vout, fout, pairs, uniq)
        ve = torch.empty(extra.numel(), dtype=torch.int32, device="cuda")
        fe = torch.empty(extra.numel(), dtype=torch.uint8, device="cuda")
        t.retrieve(extra, ve, fe)
        _check_dup(torch, extra, ve, fe, pairs, uniq)
        assert t.sync() == 0
