"""Deletion (tombstones, reading C9') and rebuild with a distinct hash:
GPU (through the C-ABI) against the oracle."""
import numpy as np
import pytest

import oracle
import wdgen
from wdtest import capacity_for, from_dev, gpu_roundtrip, to_dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def wd():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    return wd


def _erase(t, keys, host=False):
    import torch
    if host:
        return np.asarray(t.erase(np.ascontiguousarray(keys)))
    f = t.erase(to_dev(keys))
    torch.cuda.synchronize()
    return f.cpu().numpy()


def _check_found_once(found, erase_keys, present_before):
    # exactly one occurrence of each present key reports found; absent keys never
    for k in np.unique(erase_keys):
        occ = found[erase_keys == k]
        assert occ.sum() == (1 if k in present_before else 0), k


@pytest.mark.parametrize("G,V", [(4, 1), (8, 4), (4, 4), (1, 1), (32, 8)])
def test_erase_and_reinsert_parity(wd, G, V):
    n = 150_000
    keys, vals = wdgen.unique_keys(n, 81), wdgen.values(n, 82)
    er = np.concatenate([keys[::3], keys[::3][:1000], wdgen.unique_keys(2000, 81, start=n)])
    again = np.concatenate([keys[::3][:20_000], wdgen.unique_keys(5000, 81, start=2 * n)])
    again_v = wdgen.values(again.size, 83)
    q = np.concatenate([keys, again[-5000:], wdgen.unique_keys(3000, 81, start=3 * n)])
    m = oracle.Map(2 * n)
    m.insert(keys, vals)
    with wd.Table(capacity_for(n, 0.8), 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)   # queries / erases with this |g| and V
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.insert(to_dev(keys), to_dev(vals))
        f = _erase(t, er)
        _check_found_once(f, er, set(keys.tolist()))
        m.erase(er)
        assert t.size() == m.size()
        assert t.counters()["erased"] == n - m.size()
        t.insert(to_dev(again), to_dev(again_v))
        m.insert(again, again_v)
        ov, of = t.retrieve(to_dev(q))
        gv, gf = from_dev(ov), of.cpu().numpy()
        assert t.sync() == 0 and t.size() == m.size()
    ev, ef = m.retrieve(q)
    assert np.array_equal(gf, ef) and np.array_equal(gv, ev)


@pytest.mark.parametrize("G,V", [(4, 1), (8, 4), (2, 2), (16, 8), (16, 4)])
def test_erase_rebuild_serial_layout(wd, G, V):
    # serial mode: insert, erase, rebuild — the slot words (incl. tombstones) equal the
    # oracle's sequential replay bit for bit at every stage
    n = 3000
    A = oracle.region_align_for(G)
    c = oracle.physical_capacity(4000, A)
    keys, vals = wdgen.unique_keys(n, 91), wdgen.values(n, 92)
    er = keys[1::2]
    r = oracle.Replay(c, G, p_max=oracle.n_regions(c, A), align=A)
    r.insert(keys, vals)
    r.erase(er)
    with wd.Table(4000, 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)   # queries / erases with this |g| and V
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_SERIAL, 1)
        t.insert(to_dev(keys), to_dev(vals))
        _erase(t, er)
        assert np.array_equal(t.dump(), r.table)
        assert int(np.sum(t.dump() == np.uint64(oracle.TOMB_WORD))) == er.size
        t.rebuild(0xC0FFEE)
        r.rebuild(0xC0FFEE)
        assert np.array_equal(t.dump(), r.table)
        assert t.size() == n - er.size


def test_rebuild_preserves_map_and_frees_tombstones(wd):
    import torch
    n = 200_000
    keys, vals = wdgen.unique_keys(n, 93), wdgen.values(n, 94)
    with wd.Table(capacity_for(n, 0.95), 1, 8) as t:
        t.insert(to_dev(keys), to_dev(vals))
        _erase(t, keys[: n // 2])
        assert int(np.sum(t.dump() == np.uint64(oracle.TOMB_WORD))) == n // 2
        t.rebuild(12345)
        torch.cuda.synchronize()
        sl = t.dump()
        assert not np.any(sl == np.uint64(oracle.TOMB_WORD))
        assert t.size() == n - n // 2 and t.sync() == 0
        # the freed space is usable again: fill back to alpha ~ 0.95
        more = wdgen.unique_keys(n // 2, 93, start=n)
        t.insert(to_dev(more), to_dev(wdgen.values(more.size, 95)))
        q = np.concatenate([keys, more])
        gv, gf = gpu_roundtrip(t, np.zeros(0, np.uint32), np.zeros(0, np.uint32), q)
        assert t.sync() == 0
    assert np.all(gf[: n // 2] == 0) and np.all(gf[n // 2:] == 1)
    assert np.array_equal(gv[n // 2: n], vals[n // 2:])


@pytest.mark.parametrize("m", [3])
def test_erase_loopback_and_host(wd, m):
    n = 60_000
    keys, vals = wdgen.unique_keys(n, 96), wdgen.values(n, 97)
    er = np.concatenate([keys[::4], wdgen.unique_keys(500, 96, start=n)])
    with wd.Table(capacity_for(n, 0.85), group_size=4, loopback_shards=m, batch=7000) as t:
        t.insert(to_dev(keys), to_dev(vals))
        f = _erase(t, er, host=True)                     # host pointers through the cascade
        _check_found_once(f, er, set(keys.tolist()))
        assert t.size() == n - keys[::4].size
        gv, gf = gpu_roundtrip(t, np.zeros(0, np.uint32), np.zeros(0, np.uint32), keys)
        t.rebuild(7)
        gv2, gf2 = gpu_roundtrip(t, np.zeros(0, np.uint32), np.zeros(0, np.uint32), keys)
    want = np.ones(n, np.uint8); want[::4] = 0
    assert np.array_equal(gf, want) and np.array_equal(gf2, want)
    assert np.array_equal(gv[want == 1], vals[want == 1]) and np.array_equal(gv2, gv)


@pytest.mark.parametrize("G,shards", [(4, 1), (16, 1), (8, 3)])
def test_auto_rebuild_on_table_full(wd, G, shards):
    # an insert that cannot find an empty slot while n < c triggers a reconstruction
    # with a distinct hash.  Tombstones (reading C9': not reused before a rebuild) fill the
    # table: without WD_OPT_AUTO_REBUILD the later insert fails (sticky TABLE_FULL), with it
    # the table rebuilds, re-inserts the keys left behind and ends exact.
    n = 60_000
    keys, vals = wdgen.unique_keys(n, 201), wdgen.values(n, 202)
    more = wdgen.unique_keys(n // 2, 201, start=n)
    mvals = wdgen.values(n // 2, 203)
    cap = capacity_for(n, 0.97)
    kw = {"loopback_shards": shards} if shards > 1 else {}
    results = {}
    for auto in (0, 1):
        with wd.Table(cap, group_size=G, **kw) if shards > 1 else wd.Table(cap, 1, G) as t:
            if shards > 1:
                t.set_option(wd.WD_OPT_BATCH, 10_000)
            t.set_option(wd.WD_OPT_AUTO_REBUILD, auto)
            assert t.get_option(wd.WD_OPT_AUTO_REBUILD) == auto
            t.insert(to_dev(keys), to_dev(vals))
            _erase(t, keys[: n // 2])                      # half the table becomes tombstones
            assert t.sync() == 0 and t.size() == n - n // 2
            if auto:
                t.insert(to_dev(more), to_dev(mvals))      # recovers: no error
            else:
                t.insert(to_dev(more), to_dev(mvals))
            st = t.sync()
            results[auto] = st
            if auto:
                assert st == 0, wd._lib.wd_last_error_message()
                assert t.size() == n
                q = np.concatenate([keys, more])
                gv, gf = gpu_roundtrip(t, np.zeros(0, np.uint32), np.zeros(0, np.uint32), q)
                want = np.concatenate([np.zeros(n // 2, np.uint8), np.ones(n - n // 2 + n // 2, np.uint8)])
                assert np.array_equal(gf, want)
                assert np.array_equal(gv[n // 2: n], vals[n // 2:]) and np.array_equal(gv[n:], mvals)
    assert results[0] == wd.WD_ERR_TABLE_FULL
