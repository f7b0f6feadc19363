"""Multi-GPU paths on >= 2 PHYSICAL devices (skipped on a one-GPU box; they run wherever
torch.cuda.device_count() >= 2): the single-process table over n_gpus devices (wd_create
with n_gpus > 1: per-device shards, peer access over NVLink, host input split into
portions) and its device-sided _sharded calls, and one process per GPU
(rank mode, CUDA IPC peer mappings, cross-device epoch flags).  Every query is checked
against the generator's closed form."""
import math
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

KS, VS = 501, 502


def _ndev():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


needs2 = pytest.mark.skipif(_ndev() < 2, reason="needs >= 2 CUDA devices")


@needs2
@pytest.mark.parametrize("G,exchange", [(4, 0), (16, 0), (16, 1), (16, 2)])
def test_single_process_multi_gpu_host_input(G, exchange):
    import torch
    import oracle
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen
    m = min(_ndev(), 8)
    n = 1_000_003
    keys, vals = wdgen.unique_keys(n, KS), wdgen.values(n, VS)
    q = wdgen.interleaved_queries(n, KS)
    torch.cuda.set_device(0)
    with wd.Table(int(math.ceil(n / 0.9)), m, G, exchange=exchange) as t:
        assert t.get_option(wd.WD_OPT_N_SHARDS) == m
        t.set_option(wd.WD_OPT_BATCH, 1 << 18)           # several batches per shard
        kk = torch.from_numpy(keys.view(np.int32)).pin_memory()
        vv = torch.from_numpy(vals.view(np.int32)).pin_memory()
        t.insert(kk, vv)
        qq = torch.from_numpy(q.view(np.int32)).pin_memory()
        ov = torch.empty(q.size, dtype=torch.int32).pin_memory()
        of = torch.empty(q.size, dtype=torch.uint8).pin_memory()
        t.retrieve(qq, ov, of)
        torch.cuda.synchronize()
        assert t.sync() == 0, wd._lib.wd_last_error_message()
        assert t.size() == n
        seed = t.get_option(wd.WD_OPT_PART_SEED)
        for d in range(m):                                 # shard d holds p(k) = d
            sl = t.dump(d)
            k = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
            k = k[k != np.uint32(0xFFFFFFFF)]
            assert np.all(oracle.partition(k, m, seed) == d)
    cv, cf = oracle.expected_unique(q, n, KS, VS)
    assert np.array_equal(of.numpy(), cf) and np.array_equal(ov.numpy().view(np.uint32), cv)


@needs2
@pytest.mark.parametrize("exchange", [0, 1, 2])
def test_single_process_multi_gpu_sharded_device_input(exchange):
    import torch
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg
    m = min(_ndev(), 8)
    n_local = 1 << 22
    n = n_local * m
    torch.cuda.set_device(0)
    with wd.Table(int(math.ceil(n / 0.95)), m, 16, exchange=exchange) as t:
        keys, vals, q, vo, fo, st = [], [], [], [], [], []
        for r in range(m):
            with torch.cuda.device(r):
                keys.append(gg.unique_keys(n_local, KS, start=r * n_local))
                vals.append(gg.values(n_local, VS, start=r * n_local))
                q.append(gg.interleaved_queries(n, KS, start=2 * r * n_local, count=2 * n_local))
                vo.append(torch.empty(2 * n_local, dtype=torch.int32, device=f"cuda:{r}"))
                fo.append(torch.empty(2 * n_local, dtype=torch.uint8, device=f"cuda:{r}"))
                st.append(torch.cuda.current_stream(r))
        with pytest.raises(Exception):
            t.insert(keys[0], vals[0])                     # whole-table call: host memory only
        t.insert_sharded(keys, vals, st)
        t.retrieve_sharded(q, vo, fo, st)
        for r in range(m):
            torch.cuda.synchronize(r)
        assert t.sync() == 0 and t.size() == n
        for r in range(m):
            with torch.cuda.device(r):
                bad, first, found = gg.check_unique(q[r], vo[r], fo[r], n, KS, VS)
            assert bad == 0 and found == n_local, (r, bad, first, found)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_worker(rank, world, port, q, n_local, G, exchange):
    try:
        import torch
        import torch.distributed as dist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(rank)                       # one process per PHYSICAL GPU
        import paper_conf_ipps_junger0s18_b200 as wd
        import wdgen.gpu as gg
        n = world * n_local
        keys = gg.unique_keys(n_local, KS, start=rank * n_local)
        vals = gg.values(n_local, VS, start=rank * n_local)
        t = wd.Table(int(math.ceil(n / 0.95)), group_size=G, rank=rank, world=world,
                     batch=1 << 20, exchange=exchange)
        t.insert(keys, vals)
        qk = gg.interleaved_queries(n, KS, start=2 * rank * n_local, count=2 * n_local)
        vo = torch.empty(2 * n_local, dtype=torch.int32, device="cuda")
        fo = torch.empty(2 * n_local, dtype=torch.uint8, device="cuda")
        t.retrieve(qk, vo, fo)
        torch.cuda.synchronize()
        st, size = t.sync(), t.size()
        bad, first, found = gg.check_unique(qk, vo, fo, n, KS, VS)
        ok = st == 0 and size == n and bad == 0 and found == n_local
        t.close()
        dist.destroy_process_group()
        q.put((rank, "ok" if ok else f"st={st} size={size} bad={bad} first={first} found={found}"))
    except Exception:
        import traceback
        q.put((rank, traceback.format_exc()))


@needs2
@pytest.mark.parametrize("G,exchange", [(4, 0), (16, 0), (16, 1), (16, 2)])
def test_rank_mode_physical_gpus(G, exchange):
    import torch.multiprocessing as mp
    world = min(_ndev(), 8)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_worker, args=(r, world, port, q, 3_000_017, G, exchange))
             for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {r: "ok" for r in range(world)}, res
