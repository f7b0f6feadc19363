"""Seeded randomized parity through the C-ABI: random sizes (ragged, tiny, empty), loads,
table |g|, per-call insert / query |g| (reading C24), slice grouping, probe modes, keys in
flight, duplicate fractions, the reserved key, erase and re-insert, host or device buffers,
loopback shards, exchange modes and batch sizes.  Every case replays its calls on the oracle's map (P:31 exact map,
P:185 upsert, P:91 delete) and compares every query: found flags exactly, values exactly for
keys inserted once per call and v in V(k) for keys a call inserted several times."""
import numpy as np
import pytest

from wdtest import capacity_for, from_dev, to_dev

pytestmark = pytest.mark.gpu

N_CASES = 160
GS = (1, 2, 4, 8, 16, 32)


@pytest.fixture(scope="module")
def wd():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_junger0s18_b200 as wd
    return wd


def _case(seed):
    r = np.random.default_rng(seed)
    c = {
        "n": int(r.choice([0, 1, 31, 1000, int(r.integers(2, 300_000))])),
        "alpha": float(r.uniform(0.5, 0.97)),
        "G": int(r.choice(GS)),
        "ig": int(r.choice([-1, 0] + list(GS))),
        "qg": int(r.choice([-1, 0] + list(GS))),
        "slices": int(r.choice([0, 1, 2, 8, 32])),
        "mode": int(r.choice([0, 1, 2])),
        "kif": int(r.choice([0, 0, 2, 4])),
        "dup": float(r.choice([0.0, 0.0, 0.3, 0.9])),
        "reserved": bool(r.random() < 0.2),
        "erase": float(r.choice([0.0, 0.25])),
        "host": bool(r.random() < 0.3),
        "shards": int(r.choice([1, 1, 1, 2, 3])),
        "exchange": int(r.choice([0, 1])),   # fused peer stores / copy engine (cascade only)
        "batch": int(r.choice([0, 5000, 1 << 16])),
    }
    if c["shards"] > 1:
        c["slices"] = 0                      # the cascade has no slice grouping
    return c


def _as_input(a, host):
    import torch
    if host:
        return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).pin_memory()
    return to_dev(a)


@pytest.mark.parametrize("seed", range(N_CASES))
def test_fuzz_parity(wd, seed):
    import torch
    import oracle
    import wdgen
    c = _case(1000 + seed)
    n = c["n"]
    rng = np.random.default_rng(seed)
    distinct = max(1, int(n * (1.0 - c["dup"])))
    keys = wdgen.uniform_keys(n, 7 + seed) % np.uint32(distinct) if c["dup"] > 0 \
        else wdgen.unique_keys(n, 7 + seed)
    keys = keys.astype(np.uint32)
    if c["reserved"] and n:
        keys[rng.integers(0, n, size=max(1, n // 1000))] = 0xFFFFFFFF
    vals = wdgen.values(n, 9 + seed)
    # room for the distinct keys plus what the erase step re-inserts: tombstones are not
    # reused (reading C9'), so every re-inserted key takes a new slot (<= half of the erased
    # keys + 100 absent ones)
    cap = capacity_for(int(distinct * (1 + c["erase"] / 2)) + 150, c["alpha"]) + 64
    kw = {"loopback_shards": c["shards"], "exchange": c["exchange"]} if c["shards"] > 1 else {}
    m = oracle.Map(max(n, 1) * 2, dup_mode=True)
    with (wd.Table(cap, group_size=c["G"], **kw) if kw else wd.Table(cap, 1, c["G"])) as t:
        t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, c["ig"])
        t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, c["qg"])
        if c["shards"] == 1:
            t.set_option(wd.WD_OPT_SLICES, c["slices"])
        t.set_option(wd.WD_OPT_PROBE_MODE, c["mode"])
        if c["kif"]:
            t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, c["kif"])
        if c["batch"]:
            t.set_option(wd.WD_OPT_BATCH, c["batch"])        # pipeline / cascade batches
        if n:
            t.insert(_as_input(keys, c["host"]), _as_input(vals, c["host"]))
        m.insert(keys, vals)
        # erase a subset (present and absent keys), then re-insert part of it with new values
        er = np.zeros(0, np.uint32)
        if c["erase"] and n:
            er = np.unique(keys[keys != 0xFFFFFFFF])
            er = er[: int(er.size * c["erase"])]
            er = np.unique(np.concatenate([er, wdgen.unique_keys(200, 3 + seed, start=1 << 30)]))
            f = t.erase(to_dev(er))
            torch.cuda.synchronize()
            want = m.erase(er)
            assert np.array_equal(f.cpu().numpy().astype(bool), want.astype(bool)), c
            back = er[: er.size // 2][::-1].copy()
            bv = wdgen.values(back.size, 11 + seed)
            t.insert(to_dev(back), to_dev(bv))
            m.insert(back, bv)
        q = np.concatenate([keys[: 50_000], er, wdgen.unique_keys(5000, 13 + seed, start=1 << 31)])
        if q.size == 0:
            q = np.array([5, 7], np.uint32)
        if c["host"]:
            qq = _as_input(q, True)
            ov = torch.empty(q.size, dtype=torch.int32).pin_memory()
            of = torch.empty(q.size, dtype=torch.uint8).pin_memory()
            t.retrieve(qq, ov, of)
            torch.cuda.synchronize()
            gv, gf = ov.numpy().view(np.uint32).copy(), of.numpy().copy()
        else:
            ov, of = t.retrieve(to_dev(q))
            gv, gf = from_dev(ov), of.cpu().numpy()
        st = t.sync()
        expect_st = wd.WD_ERR_RESERVED_KEY if (c["reserved"] and n) else 0
        assert st == expect_st, (c, st, wd._lib.wd_last_error_message())
        assert t.size() == m.size(), c
    ev, ef = m.retrieve(q)
    assert np.array_equal(gf, ef), c
    assert np.all(gv[gf == 0] == 0xFFFFFFFF), c
    hit = gf == 1
    assert np.all(m.pair_status(q[hit], gv[hit]) >= 1), c          # v in V(k)
    if c["dup"] == 0.0:
        assert np.array_equal(gv[hit], ev[hit]), c                   # unique: exact
