"""Single-GPU parity: the CUDA path (through the C-ABI) against the oracle, element by
element, bit-exact on (found, value).  Marked gpu: run on the B200 box."""
import numpy as np
import pytest

import oracle
import wdgen
from wdtest import capacity_for, from_dev, gpu_roundtrip, to_dev

pytestmark = pytest.mark.gpu

GS = [1, 2, 4, 8, 16, 32]


@pytest.fixture(scope="module")
def wd():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    return wd


def _oracle_answers(keys, vals, queries, dup=False):
    m = oracle.Map(keys.size, dup_mode=dup)
    m.insert(keys, vals)
    return m, *m.retrieve(queries)


MODES = [(G, 1) for G in GS] + [(G, 2) for G in GS if G <= 8]   # (|g|, probe mode)


@pytest.mark.parametrize("qg", [0, -1])
@pytest.mark.parametrize("G,mode", MODES)
def test_config1_unique_parity(wd, G, mode, qg):
    # BASELINE config 1: 2^20 unique keys, load 0.95, all keys + 2^20 absent keys queried
    n, ks, vs = 1 << 20, 101, 202
    keys, vals = wdgen.unique_keys(n, ks), wdgen.values(n, vs)
    q = wdgen.interleaved_queries(n, ks)
    with wd.Table(capacity_for(n, 0.95), 1, G) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, qg)      # 0: queries with the table's |g|
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, qg)     # -1: the library's auto choice
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0
        assert t.size() == n
        cnt = t.counters()
        assert cnt["failed"] == 0 and cnt["reserved"] == 0
        assert t.capacity() == oracle.physical_capacity(capacity_for(n, 0.95),
                                                        oracle.region_align_for(G))
        assert t.get_option(wd.WD_OPT_REGION_ALIGN) == oracle.region_align_for(G)
        load = t.size() / t.capacity()
        assert abs(load - 0.95) < 1e-3
    m, ev, ef = _oracle_answers(keys, vals, q)
    assert np.array_equal(gf, ef)
    assert np.array_equal(gv, ev)
    # closed form (independent of the oracle's table)
    cv, cf = oracle.expected_unique(q, n, ks, vs)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("mode", [1, 2])
@pytest.mark.parametrize("kif", [4, 8])
@pytest.mark.parametrize("alpha", [0.8, 0.99, 0.999])
def test_alpha_and_keys_in_flight(wd, alpha, kif, mode):
    n = 300_001  # ragged
    keys, vals = wdgen.unique_keys(n, 7), wdgen.values(n, 8)
    q = wdgen.interleaved_queries(n, 7)
    with wd.Table(capacity_for(n, alpha), 1, 4) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, kif)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 7, 8)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("G,mode", MODES)
def test_serial_layout_equals_fig3_replay(wd, G, mode):
    # WD_OPT_SERIAL runs one probing group, one key at a time: the slot layout must equal
    # the oracle's sequential replay of Fig. 3 bit for bit (probe sequence, windows,
    # leftmost-empty leader, update-on-match).
    n = 3000
    A = oracle.region_align_for(G)                  # reading C2': the table's geometry
    c = oracle.physical_capacity(3200, A)
    keys = np.concatenate([wdgen.unique_keys(n, 3), wdgen.unique_keys(200, 3)])  # 200 updates
    vals = wdgen.values(n + 200, 4)
    r = oracle.Replay(c, G, align=A)
    r.insert(keys, vals)
    with wd.Table(3200, 1, G) as t:
        assert t.shard_capacity() == c
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_SERIAL, 1)
        t.insert(to_dev(keys), to_dev(vals))
        assert t.sync() == 0
        slots = t.dump()
        assert t.size() == n
    assert np.array_equal(slots, r.table)


@pytest.mark.parametrize("Gc,Gi", [(16, 4), (16, 1), (32, 8), (4, 16), (0, 16)])
def test_region_align_is_per_table(wd, Gc, Gi):
    # reading C2': A is fixed when the table is created (16 for |g| >= 16, else 4); later
    # calls with another |g| probe the same sequence: the serial layout of a |g| = Gi
    # insert equals the replay with the CREATION geometry, and queries with every |g| agree
    n = 2000
    A = oracle.region_align_for(Gc)
    c = oracle.physical_capacity(2300, A)
    keys, vals = wdgen.unique_keys(n, 51), wdgen.values(n, 52)
    r = oracle.Replay(c, Gi, align=A)
    r.insert(keys, vals)
    with wd.Table(2300, 1, Gc) as t:
        assert t.get_option(wd.WD_OPT_REGION_ALIGN) == A and t.capacity() == c
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, Gi)
        t.set_option(wd.WD_OPT_SERIAL, 1)
        t.insert(to_dev(keys), to_dev(vals))
        assert t.sync() == 0
        assert np.array_equal(t.dump(), r.table)
        t.set_option(wd.WD_OPT_SERIAL, 0)
        q = wdgen.interleaved_queries(n, 51)
        cv, cf = oracle.expected_unique(q, n, 51, 52)
        for Gq in (1, 4, 16, 32):
            t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, Gq)
            ov, of = t.retrieve(to_dev(q))
            assert np.array_equal(of.cpu().numpy(), cf) and np.array_equal(from_dev(ov), cv)


@pytest.mark.parametrize("Gi,Gq,mi,mq", [(1, 32, 1, 1), (32, 1, 1, 2), (4, 8, 2, 1),
                                         (8, 2, 1, 2), (2, 16, 2, 0), (4, 4, 2, 1), (4, 4, 1, 2)])
def test_cross_group_size(wd, Gi, Gq, mi, mq):
    # the probing scheme is consistent when |g| varies: insert with one |g|, query
    # with another — and across the two probe modes (same windows, same sequence).
    n = 200_000
    keys, vals = wdgen.unique_keys(n, 9), wdgen.values(n, 9)
    q = wdgen.interleaved_queries(n, 9)
    with wd.Table(capacity_for(n, 0.97), 1, Gi) as t:
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_PROBE_MODE, mi)
        t.insert(to_dev(keys), to_dev(vals))
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, Gq)
        t.set_option(wd.WD_OPT_PROBE_MODE, mq)
        ov, of = t.retrieve(to_dev(q))
        gv, gf = from_dev(ov), of.cpu().numpy()
    cv, cf = oracle.expected_unique(q, n, 9, 9)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("G", [1, 2, 4, 8, 16, 32])
def test_query_group_size(wd, G):
    # WD_OPT_QUERY_GROUP_SIZE / WD_OPT_INSERT_GROUP_SIZE (default -1 = auto): calls probe with
    # a |g| other than the table's — P:89, every result is the same: hits, misses (long
    # chains at alpha 0.97), erase flags, queries past tombstones, updates of existing keys
    n = 120_001
    keys, vals = wdgen.unique_keys(n, 61), wdgen.values(n, 62)
    q = wdgen.interleaved_queries(n, 61)
    cv, cf = oracle.expected_unique(q, n, 61, 62)
    auto_ins = 16                                         # A = 16, or a shard <= 64 MB
    with wd.Table(1000, 1, G) as t:                       # invalid values are refused
        for opt in (wd.WD_OPT_QUERY_GROUP_SIZE, wd.WD_OPT_INSERT_GROUP_SIZE):
            for bad in (-2, 3, 64):
                with pytest.raises(Exception):
                    t.set_option(opt, bad)
            assert t.get_option(opt) == -1
    for qg, ig in ((-1, -1), (16, 0), (0, 0), (1, -1), (4, 0), (32, 32), (-1, 1)):
        with wd.Table(capacity_for(n, 0.97), 1, G) as t:
            assert t.get_option(wd.WD_OPT_QUERY_GROUP_SIZE) == -1
            assert t.get_option(wd.WD_OPT_INSERT_GROUP_SIZE) == -1
            t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, qg)
            t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, ig)
            assert t.get_option(wd.WD_OPT_QUERY_GROUP_SIZE) == qg
            gv, gf = gpu_roundtrip(t, keys, vals, q)
            assert np.array_equal(gf, cf) and np.array_equal(gv, cv), (qg, ig)
            # auto at load 0.97: 16
            assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == (16 if qg < 0 else qg or G)
            # erase every third key (found flags), then query past the tombstones
            er = keys[::3]
            df = t.erase(to_dev(er))
            assert np.all(df.cpu().numpy() == 1)
            upd = keys[1::3]                              # updates of existing keys
            t.insert(to_dev(upd), to_dev(vals[1::3] ^ np.uint32(0x5A5A5A5A)))
            assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == (auto_ins if ig < 0 else ig or G)
            ov, of = t.retrieve(to_dev(keys))
            gv, gf = from_dev(ov), of.cpu().numpy()
            assert t.sync() == 0 and t.size() == n - er.size
        want_f = np.ones(n, np.uint8); want_f[::3] = 0
        want_v = vals.copy(); want_v[1::3] ^= np.uint32(0x5A5A5A5A)
        assert np.array_equal(gf, want_f), (qg, ig)
        assert np.array_equal(gv[want_f == 1], want_v[want_f == 1]), (qg, ig)


def test_auto_insert_serial_layout(wd):
    # the auto insert |g| (16 on small shards and A = 16 tables, 8 on A = 4 shards > 64 MB)
    # lays the keys out exactly as the paper's |g| does: serial layout = the Fig. 3 replay
    # with the table's |g| and geometry
    n = 2500
    for G, cap, want in ((1, 2700, 16), (2, 2700, 16), (4, 2700, 16), (32, 2700, 16),
                         (4, 9_000_000, 8), (16, 9_000_000, 16)):
        A = oracle.region_align_for(G)
        c = oracle.physical_capacity(cap, A)
        keys = np.concatenate([wdgen.unique_keys(n, 71), wdgen.unique_keys(100, 71)])
        vals = wdgen.values(n + 100, 72)
        r = oracle.Replay(c, G, align=A)
        r.insert(keys, vals)
        with wd.Table(cap, 1, G) as t:
            t.set_option(wd.WD_OPT_SERIAL, 1)
            t.insert(to_dev(keys), to_dev(vals))
            assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == want, (G, cap)
            assert t.sync() == 0
            assert np.array_equal(t.dump(), r.table), (G, cap)


def test_auto_insert_group_large_table(wd):
    # shards > 24 GB with A = 4 keep the table's |g| for inserts (config 3's regime); the map
    # stays exact
    n = 200_000
    keys, vals = wdgen.unique_keys(n, 73), wdgen.values(n, 74)
    q = wdgen.interleaved_queries(n, 73)
    with wd.Table(3_300_000_000, 1, 4) as t:           # 26.4 GB
        t.insert(to_dev(keys), to_dev(vals))
        assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == 4
        ov, of = t.retrieve(to_dev(q))
        gv, gf = from_dev(ov), of.cpu().numpy()
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 73, 74)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("G,mode,flags", [(1, 1, 3), (4, 1, 3), (32, 1, 3), (2, 2, 3), (4, 2, 3),
                                          (8, 2, 3), (4, 0, 3), (4, 1, 0), (4, 2, 0), (1, 1, 1),
                                          (1, 1, 11), (4, 1, 11), (8, 0, 11), (8, 2, 8)])
def test_duplicates_upsert(wd, G, mode, flags):
    # duplicate-key mode: value must be one of the values inserted for the key;
    # size = number of distinct keys; a second stream-ordered call wins.
    n = 400_000
    keys = wdgen.uniform_keys(n, 11) % np.uint32(150_000)
    vals = wdgen.values(n, 12)
    with wd.Table(capacity_for(150_000, 0.9), 1, G) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.insert(to_dev(keys), to_dev(vals))
        q = np.arange(160_000, dtype=np.uint32)
        ov, of = t.retrieve(to_dev(q))
        gv, gf = from_dev(ov), of.cpu().numpy()
        m = oracle.Map(n, dup_mode=True)
        m.insert(keys, vals)
        assert t.size() == m.size()
        ev, ef = m.retrieve(q)
        assert np.array_equal(gf, ef)
        st = m.pair_status(q[gf == 1], gv[gf == 1])
        assert np.all(st >= 1)          # v in V(k)
        assert np.all(gv[gf == 0] == 0xFFFFFFFF)
        # second call overwrites: last call wins
        k2 = np.unique(keys)[:1000]
        v2 = wdgen.values(k2.size, 99)
        t.insert(to_dev(k2), to_dev(v2))
        ov, of = t.retrieve(to_dev(k2))
        assert np.array_equal(from_dev(ov), v2)
        assert t.size() == m.size()


def test_edge_cases(wd):
    import torch
    # exactly full: c = 32 (one region), 32 keys, alpha = 1
    keys, vals = wdgen.unique_keys(33, 5), wdgen.values(33, 5)
    with wd.Table(32, 1, 4) as t:
        assert t.capacity() == 32
        gv, gf = gpu_roundtrip(t, keys[:32], vals[:32], keys)
        assert t.sync() == 0 and t.size() == 32
        assert np.all(gf[:32] == 1) and np.array_equal(gv[:32], vals[:32]) and gf[32] == 0
        # alpha > 1: the 33rd key cannot be placed
        t.set_option(wd.WD_OPT_P_MAX, 4)
        t.insert(to_dev(keys[32:]), to_dev(vals[32:]))
        assert t.sync() == wd.WD_ERR_TABLE_FULL
        assert t.counters()["failed"] == 1 and t.size() == 32
        t.clear()
        torch.cuda.synchronize()
        assert t.sync() == 0 and t.size() == 0
    # alpha = 1 on a multi-region table: p_max >= nb reaches every slot
    c = oracle.physical_capacity(1000)
    keys = wdgen.unique_keys(c, 6)
    with wd.Table(1000, 1, 4) as t:
        assert t.capacity() == c
        t.set_option(wd.WD_OPT_P_MAX, oracle.n_regions(c))
        gv, gf = gpu_roundtrip(t, keys, keys ^ np.uint32(1), keys)
        assert t.sync() == 0 and t.size() == c and np.all(gf == 1)
        assert np.array_equal(gv, keys ^ np.uint32(1))
    # reserved key and 0xFFFFFFFF values
    keys = np.array([1, 0xFFFFFFFF, 2, 0, 3], np.uint32)
    vals = np.array([0xFFFFFFFF, 7, 0, 0xFFFFFFFF, 5], np.uint32)
    q = np.array([0, 1, 2, 3, 0xFFFFFFFF, 4], np.uint32)
    with wd.Table(64, 1, 8) as t:
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == wd.WD_ERR_RESERVED_KEY
        assert t.size() == 4
        m, ev, ef = _oracle_answers(keys, vals, q)
        assert np.array_equal(gf, ef) and np.array_equal(gv, ev)
    # n = 0 and n = 1
    with wd.Table(100, 1, 4) as t:
        t.insert(to_dev(np.zeros(0, np.uint32)), to_dev(np.zeros(0, np.uint32)))
        ov, of = t.retrieve(to_dev(np.zeros(0, np.uint32)))
        assert ov.numel() == 0
        gv, gf = gpu_roundtrip(t, np.array([42], np.uint32), np.array([43], np.uint32),
                               np.array([42, 41], np.uint32))
        assert list(gf) == [1, 0] and gv[0] == 43 and gv[1] == 0xFFFFFFFF
    # bad arguments
    with pytest.raises(wd.WarpDriveError):
        wd.Table(100, 1, 3)
    with pytest.raises(wd.WarpDriveError):
        wd.Table(0, 1, 4)


@pytest.mark.parametrize("pinned", [True, False])
@pytest.mark.parametrize("batch", [7_777, 25_001, 1 << 20])
def test_host_pointers_out_of_core(wd, pinned, batch):
    # a11: host-resident input streamed in batches.  7 777: many batches (the
    # staging slots are reused); 25 001: full batches + a ragged last one; 2^20: one batch
    n = 100_003
    keys, vals = wdgen.unique_keys(n, 13), wdgen.values(n, 14)
    q = wdgen.interleaved_queries(n, 13)
    with wd.Table(capacity_for(n, 0.95), 1, 4) as t:
        t.set_option(wd.WD_OPT_BATCH, batch)
        if pinned:
            gv, gf = gpu_roundtrip(t, keys, vals, q, host=True)
        else:
            t.insert(keys, vals)           # numpy (pageable)
            gv, gf = t.retrieve(q)
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 13, 14)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


def test_config2_full_size_sampled(wd):
    # BASELINE config 2 at its full size (2^28 unique pairs, alpha 0.95, |g| = 4), inputs
    # generated on the device; every query checked in-kernel-order against the closed
    # form on a 2^22 sample of positions spanning the whole range.
    import torch
    import wdgen.gpu as gg
    n, ks, vs = 1 << 28, 77, 78
    keys, vals = gg.unique_keys(n, ks), gg.values(n, vs)
    with wd.Table(capacity_for(n, 0.95), 1, 4) as t:
        t.insert(keys, vals)
        del vals
        q = gg.interleaved_queries(n, ks, start=n - (1 << 27), count=1 << 28)  # half present
        ov, of = t.retrieve(q)
        assert t.sync() == 0 and t.size() == n
        torch.cuda.synchronize()
        rng = np.random.default_rng(0)
        idx = np.sort(rng.choice(q.numel(), 1 << 22, replace=False))
        ii = torch.from_numpy(idx).cuda()
        qs = q[ii].cpu().numpy().view(np.uint32)
        gv = ov[ii].cpu().numpy().view(np.uint32)
        gf = of[ii].cpu().numpy()
    cv, cf = oracle.expected_unique(qs, n, ks, vs)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
    assert 0.45 < gf.mean() < 0.55


@pytest.mark.parametrize("G,mode,flags", [(1, 1, 3), (4, 1, 3), (8, 1, 3), (4, 2, 3), (2, 2, 3),
                                          (4, 1, 0), (4, 2, 1), (4, 1, 2), (1, 1, 11), (8, 0, 11),
                                          (4, 2, 10)])
def test_zipf_duplicates(wd, G, mode, flags):
    # Zipf keys (s = 1 + 1e-6): hot keys updated by many groups at once.
    # Every returned value must be one of the values inserted for its key; size = #distinct.
    n = 1 << 20
    keys = wdgen.zipf_keys(n, 2**32 - 1, 17)
    vals = wdgen.values(n, 18)
    distinct = np.unique(keys).size
    with wd.Table(capacity_for(distinct, 0.95), 1, G) as t:   # load = actual occupancy
        t.set_option(wd.WD_OPT_PROBE_MODE, mode)
        t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        q = np.concatenate([np.unique(keys), wdgen.unique_keys(1000, 99)])
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0
        assert t.size() == distinct
    m = oracle.Map(n, dup_mode=True)
    m.insert(keys, vals)
    ev, ef = m.retrieve(q)
    assert np.array_equal(gf, ef)
    assert np.all(m.pair_status(q[gf == 1], gv[gf == 1]) >= 1)


SPLITS = [(2, 2), (4, 2), (8, 2), (8, 4), (16, 4), (32, 8), (16, 2), (32, 4), (16, 16),
          (32, 16)]   # (|g|, V)


@pytest.mark.parametrize("G,V", SPLITS)
def test_window_split_serial_layout(wd, G, V):
    # a window read by |g|/V lanes of V slots each: same probing, same sequential layout
    n = 2500
    A = oracle.region_align_for(G)
    c = oracle.physical_capacity(2700, A)
    keys = np.concatenate([wdgen.unique_keys(n, 31), wdgen.unique_keys(100, 31)])
    vals = wdgen.values(n + 100, 32)
    r = oracle.Replay(c, G, align=A)
    r.insert(keys, vals)
    with wd.Table(2700, 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_SERIAL, 1)
        t.insert(to_dev(keys), to_dev(vals))
        assert t.sync() == 0
        assert np.array_equal(t.dump(), r.table)


@pytest.mark.parametrize("G,V", [(1, 1), (4, 1), (4, 2), (8, 4), (8, 8), (16, 4), (32, 1)])
@pytest.mark.parametrize("n", [1000, 128 * 9, 300_007, 1 << 20])
def test_scrambled_query_order(wd, G, V, n):
    # kF_QSCR: queries visit their chunks in a scrambled order; every result must still land
    # at its own position (full chunks, partial last chunk, tiny inputs), with and without
    # the scramble, for duplicates in the query batch too
    keys, vals = wdgen.unique_keys(n, 43), wdgen.values(n, 44)
    q = wdgen.interleaved_queries(n, 43)
    q = np.concatenate([q, q[: n // 3]])
    cv, cf = oracle.expected_unique(q, n, 43, 44)
    for flags in (11, 3):
        with wd.Table(capacity_for(n, 0.95), 1, G) as t:
            t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
            t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
            t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
            t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
            gv, gf = gpu_roundtrip(t, keys, vals, q)
            assert t.sync() == 0 and t.size() == n
        assert np.array_equal(gf, cf) and np.array_equal(gv, cv), flags


@pytest.mark.parametrize("G,V", SPLITS)
def test_window_split_parity(wd, G, V):
    n = 400_003
    keys, vals = wdgen.unique_keys(n, 33), wdgen.values(n, 34)
    q = wdgen.interleaved_queries(n, 33)
    with wd.Table(capacity_for(n, 0.97), 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 33, 34)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
    # duplicates through the same split
    dk = wdgen.uniform_keys(200_000, 35) % np.uint32(60_000)
    dv = wdgen.values(200_000, 36)
    with wd.Table(capacity_for(60_000, 0.9), 1, G) as t:
        t.set_option(wd.WD_OPT_SLOTS_PER_LANE, V)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        qq = np.arange(61_000, dtype=np.uint32)
        gv, gf = gpu_roundtrip(t, dk, dv, qq)
        m = oracle.Map(200_000, dup_mode=True)
        m.insert(dk, dv)
        assert t.size() == m.size()
    ev, ef = m.retrieve(qq)
    assert np.array_equal(gf, ef)
    assert np.all(m.pair_status(qq[gf == 1], gv[gf == 1]) >= 1)


def test_config3_single_gpu_full_size(wd):
    # BASELINE config 3 at m = 1: every non-sentinel 4-byte key (n = 2^32 - 1, C14) into a
    # 4.52e9-slot table (36 GB, 64-bit slot indices) at alpha 0.95; inputs generated on the
    # device; a 2^21 random sample of queries checked against the closed form.
    import torch
    import wdgen.gpu as gg
    free, _ = torch.cuda.mem_get_info()
    if free < 100e9:
        pytest.skip("needs ~90 GB of device memory")
    n = (1 << 32) - 1
    keys, vals = gg.unique_keys(n, 111), gg.values(n, 112)
    with wd.Table(capacity_for(n, 0.95), 1, 8) as t:
        t.insert(keys, vals)
        del vals
        torch.cuda.synchronize()
        assert t.sync() == 0 and t.size() == n
        idx = torch.randint(0, n, (1 << 21,), device="cuda", dtype=torch.int64)
        q = torch.cat([keys[idx], gg.unique_keys(1 << 10, 999)])   # + keys of another seed
        ov, of = t.retrieve(q)
        torch.cuda.synchronize()
        gv, gf = from_dev(ov), of.cpu().numpy()
        qs = from_dev(q)
    cv, cf = oracle.expected_unique(qs, n, 111, 112)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


def test_dynamic_group_size_by_load(wd):
    # P:245 future work, built: |g| = 0 picks |g| per call from the projected load; the
    # calls of one table then use different |g| — P:89 says the probe sequence is the same
    n = 400_000
    keys, vals = wdgen.unique_keys(n, 121), wdgen.values(n, 122)
    c = capacity_for(n, 0.99)
    with wd.Table(c, 1, 0) as t:
        assert t.get_option(wd.WD_OPT_GROUP_SIZE) == 0
        t.insert(to_dev(keys[: n // 2]), to_dev(vals[: n // 2]))        # load ~0.5
        assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == 8
        t.insert(to_dev(keys[n // 2:]), to_dev(vals[n // 2:]))         # load -> 0.99
        assert t.get_option(wd.WD_OPT_GROUP_SIZE_USED) == 16
        q = wdgen.interleaved_queries(n, 121)
        ov, of = t.retrieve(to_dev(q))
        gv, gf = from_dev(ov), of.cpu().numpy()
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 121, 122)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)


@pytest.mark.parametrize("G", [1, 2, 4])
@pytest.mark.parametrize("span", [1, 2])
def test_span_read_ahead(wd, G, span):
    # WD_OPT_SPAN: one lane loads S = 2 consecutive windows per round trip and decides on
    # the first that holds a match or an empty slot (Fig. 3 order).  The serial layout must
    # still equal the sequential replay bit for bit, and concurrent calls must return the
    # exact map — hits, misses (long chains at alpha 0.99) and updates.
    n = 2500
    A = oracle.region_align_for(G)
    c = oracle.physical_capacity(2700, A)
    keys = np.concatenate([wdgen.unique_keys(n, 51), wdgen.unique_keys(100, 51)])
    vals = wdgen.values(n + 100, 52)
    r = oracle.Replay(c, G, align=A)
    r.insert(keys, vals)
    with wd.Table(2700, 1, G) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, 2)          # one lane per window (V = |g|)
        t.set_option(wd.WD_OPT_SPAN, span)
        assert t.get_option(wd.WD_OPT_SPAN) == span
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_SERIAL, 1)
        t.insert(to_dev(keys), to_dev(vals))
        assert t.sync() == 0
        assert np.array_equal(t.dump(), r.table)
    n = 99_001
    keys, vals = wdgen.unique_keys(n, 53), wdgen.values(n, 54)
    q = wdgen.interleaved_queries(n, 53)
    with wd.Table(capacity_for(n, 0.99), 1, G) as t:
        t.set_option(wd.WD_OPT_PROBE_MODE, 2)
        t.set_option(wd.WD_OPT_SPAN, span)
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0 and t.size() == n
        df = t.erase(to_dev(q[: n // 2]))             # deletion runs the same probe
        assert t.sync() == 0
    cv, cf = oracle.expected_unique(q, n, 53, 54)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
    assert np.array_equal(df.cpu().numpy().astype(bool), cf[: n // 2].astype(bool))


@pytest.mark.parametrize("G", [4, 16])
@pytest.mark.parametrize("slices", [1, 2, 16, 32, 64, 128])
def test_slice_grouped_insert(wd, G, slices):
    # WD_OPT_SLICES: a bulk insert grouped by table slice of the first region and inserted
    # with one launch per slice.  Unique keys: exact map; duplicates with a reserved key:
    # v in V(k), size = #distinct, the reserved key counted and never stored; a later
    # stream-ordered call still wins.  (Grouping changes the order in which one call's keys
    # are inserted, so only the map is compared, as for any concurrent call.)
    n = 300_007
    keys, vals = wdgen.unique_keys(n, 61), wdgen.values(n, 62)
    q = wdgen.interleaved_queries(n, 61)
    with wd.Table(capacity_for(n, 0.95), 1, G) as t:
        t.set_option(wd.WD_OPT_SLICES, slices)
        assert t.get_option(wd.WD_OPT_SLICES) == slices
        gv, gf = gpu_roundtrip(t, keys, vals, q)
        assert t.sync() == 0 and t.size() == n
    cv, cf = oracle.expected_unique(q, n, 61, 62)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
    nd = 400_000
    dk = wdgen.uniform_keys(nd, 63) % np.uint32(150_000)
    dk[::1000] = 0xFFFFFFFF                                  # reserved key (C8)
    dv = wdgen.values(nd, 64)
    with wd.Table(capacity_for(150_000, 0.9), 1, G) as t:
        t.set_option(wd.WD_OPT_SLICES, slices)
        t.insert(to_dev(dk), to_dev(dv))
        assert t.sync() == wd.WD_ERR_RESERVED_KEY
        assert t.counters()["reserved"] == 400
        qq = np.arange(160_000, dtype=np.uint32)
        ov, of = t.retrieve(to_dev(qq))
        gv, gf = from_dev(ov), of.cpu().numpy()
        m = oracle.Map(nd, dup_mode=True)
        m.insert(dk, dv)
        assert t.size() == m.size()
        ev, ef = m.retrieve(qq)
        assert np.array_equal(gf, ef)
        assert np.all(m.pair_status(qq[gf == 1], gv[gf == 1]) >= 1)
        k2 = np.unique(dk[dk != 0xFFFFFFFF])[:1000]
        v2 = wdgen.values(k2.size, 65)
        t.insert(to_dev(k2), to_dev(v2))
        ov, of = t.retrieve(to_dev(k2))
        assert np.array_equal(from_dev(ov), v2)


def _fmix32_inv(h: np.ndarray) -> np.ndarray:
    """inverse of MurmurHash3's fmix32 (test helper: keys with chosen first-region slices)"""
    x = h.astype(np.uint64)
    m = np.uint64(0xFFFFFFFF)
    x ^= x >> np.uint64(16)
    x = (x * np.uint64(pow(0xC2B2AE35, -1, 1 << 32))) & m
    x ^= (x >> np.uint64(13)) ^ (x >> np.uint64(26))
    x = (x * np.uint64(pow(0x85EBCA6B, -1, 1 << 32))) & m
    x ^= x >> np.uint64(16)
    return x.astype(np.uint32)


@pytest.mark.parametrize("skew", ["one_slice", "ninety_percent", "last_slice_and_ragged"])
def test_slice_grouped_insert_skewed(wd, skew):
    # the segment-mode multisplit with skewed slice counts: every key's first region in one
    # slice (all blocks' counts in one destination), 90 % in one slice, or all in the last
    # slice with a ragged tail; keys built through the inverse of fmix32 (slice = top 5 bits
    # of fmix32(k + seed), seed 0 on a fresh table)
    rng = np.random.default_rng(5)
    n = (1 << 20) + 77
    top = {"one_slice": 0, "ninety_percent": 5, "last_slice_and_ragged": 31}[skew]
    h = rng.choice(1 << 27, size=n, replace=False).astype(np.uint64) + (np.uint64(top) << np.uint64(27))
    if skew == "ninety_percent":
        k = n // 10
        h[:k] = rng.choice(1 << 32, size=k, replace=False).astype(np.uint64)
        h = np.unique(h)
        n = h.size
    keys = _fmix32_inv(h.astype(np.uint32))
    assert np.array_equal(oracle.fmix32_many(keys), h.astype(np.uint32))   # the inverse, pinned
    keep = keys != np.uint32(0xFFFFFFFF)
    keys = keys[keep]
    n = keys.size
    vals = wdgen.values(n, 81)
    absent = wdgen.unique_keys(50_000, 82)
    absent = absent[~np.isin(absent, keys)]
    with wd.Table(capacity_for(n, 0.6), 1, 16) as t:
        t.set_option(wd.WD_OPT_SLICES, 32)
        t.insert(to_dev(keys), to_dev(vals))
        assert t.sync() == 0 and t.size() == n
        ov, of = t.retrieve(to_dev(np.concatenate([keys, absent])))
        gv, gf = from_dev(ov), of.cpu().numpy()
    assert np.all(gf[:n] == 1) and np.array_equal(gv[:n], vals)
    assert np.all(gf[n:] == 0)


def test_slice_grouped_insert_chunks(wd):
    # more than one 2^26-pair chunk (auto slices on an HBM-sized table), ragged tail;
    # every query checked against the closed form on a sample
    import torch
    import wdgen.gpu as gg
    n, ks, vs = (1 << 28) + 12_345, 71, 72            # two 2^28-pair chunks (ragged second)
    keys, vals = gg.unique_keys(n, ks), gg.values(n, vs)
    with wd.Table(capacity_for(n, 0.95), 1, 16) as t:
        assert t.get_option(wd.WD_OPT_SLICES) == 0                 # auto -> 32 here (2.4 GB)
        t.insert(keys, vals)
        del vals
        q = gg.interleaved_queries(n, ks, start=n - (1 << 24), count=1 << 25)
        ov, of = t.retrieve(q)
        assert t.sync() == 0 and t.size() == n
        torch.cuda.synchronize()
        rng = np.random.default_rng(1)
        ii = torch.from_numpy(np.sort(rng.choice(q.numel(), 1 << 21, replace=False))).cuda()
        qs = q[ii].cpu().numpy().view(np.uint32)
        gv = ov[ii].cpu().numpy().view(np.uint32)
        gf = of[ii].cpu().numpy()
        assert t.launches >= 2 * (3 + 16)                             # two sliced chunks
    cv, cf = oracle.expected_unique(qs, n, ks, vs)
    assert np.array_equal(gf, cf) and np.array_equal(gv, cv)
