"""One process per GPU (rank mode), exercised with 2 processes sharing the single B200
of the test box: exchange arenas mapped with CUDA IPC, handles all-gathered and the host
collective run over torch.distributed (gloo), data moved by the multisplit/unpermute
kernels through the peer mappings, epoch flags across processes.  Results must equal
the closed form (every query) — the same cascade bench.py runs under torchrun."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, n_local, batch, G, exchange=0):
    try:
        import torch
        import torch.distributed as dist
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        import oracle
        import paper_conf_ipps_junger0s18_b200 as wd
        import wdgen
        seed = 41
        keys = wdgen.unique_keys(n_local, seed, start=rank * n_local)
        vals = wdgen.values(n_local, seed + 1, start=rank * n_local)
        cap = int(np.ceil(world * n_local / 0.9))
        t = wd.Table(cap, group_size=G, rank=rank, world=world, batch=batch, exchange=exchange)
        dk = torch.from_numpy(keys.view(np.int32)).cuda()
        dv = torch.from_numpy(vals.view(np.int32)).cuda()
        t.insert(dk, dv)
        qk, _ = wdgen.mixed_queries(world * n_local, n_local // 2 + rank, 0.5, seed,
                                    start=rank * n_local)
        ov, of = t.retrieve(torch.from_numpy(qk.view(np.int32)).cuda())
        torch.cuda.synchronize()
        st = t.sync()
        size = t.size()
        gv, gf = ov.cpu().numpy().view(np.uint32), of.cpu().numpy()
        ev, ef = oracle.expected_unique(qk, world * n_local, seed, seed + 1)
        ok = st == 0 and size == world * n_local and np.array_equal(gf, ef) and np.array_equal(gv, ev)
        # every key on this shard belongs to it
        sl = t.dump(0)
        kk = (sl & np.uint64(0xFFFFFFFF)).astype(np.uint32)
        kk = kk[kk != np.uint32(0xFFFFFFFF)]
        ok = ok and np.all(oracle.partition(kk, world, t.get_option(wd.WD_OPT_PART_SEED)) == rank)
        t.close()
        dist.destroy_process_group()
        q.put((rank, "ok" if ok else f"mismatch st={st} size={size} found={gf.sum()}/{ef.sum()}"))
    except Exception:
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("G,exchange", [(4, 0), (4, 1), (16, 1)])
def test_rank_mode_two_processes_one_gpu(G, exchange):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, 50_000, 8_192, G, exchange))
             for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
