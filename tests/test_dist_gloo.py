"""World-size-2 tests of the N>1 host logic on CPU (gloo, 127.0.0.1):
  * the rank-mode plumbing of the binding (handle all-gather, host allreduce, max-over-ranks
    timing) — paper_conf_ipps_junger0s18_b200.dist;
  * the distributed cascade's semantics at the oracle level: multisplit on each
    rank -> transposition of T -> per-rank maps; every rank ends with exactly its partition
    and the union answers every query like one global map ("transparent scaling", P:7)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    return dist


def _plumbing(rank, world, port, q):
    try:
        dist = _init(rank, world, port)
        from paper_conf_ipps_junger0s18_b200 import dist as wdist
        blobs = wdist.allgather_bytes(bytes([rank]) * 128)
        assert [b[0] for b in blobs] == list(range(world)) and all(len(b) == 128 for b in blobs)
        assert wdist.allreduce_u64(rank + 5, wdist.WD_REDUCE_SUM) == sum(r + 5 for r in range(world))
        assert wdist.allreduce_u64(10 * rank + 3, wdist.WD_REDUCE_MAX) == 10 * (world - 1) + 3
        assert wdist.max_over_ranks(1.5 * rank) == 1.5 * (world - 1)
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))


def _cascade(rank, world, port, q):
    try:
        dist = _init(rank, world, port)
        import oracle
        import wdgen
        n_local, seed, pseed = 20_000, 33, 0x9E3779B9
        keys = wdgen.unique_keys(n_local, seed, start=rank * n_local)
        vals = wdgen.values(n_local, seed, start=rank * n_local)
        counts, perm = oracle.multisplit(keys, world, pseed)          # a6: row of T
        order = np.empty(n_local, np.int64)
        order[perm.astype(np.int64)] = np.arange(n_local)
        ks, vs = keys[order], vals[order]
        rows = [None] * world
        dist.all_gather_object(rows, counts.tolist())                  # a7: T
        T = np.array(rows, np.uint64)
        send_off, recv_off = oracle.table_scans(T)
        parts = [(ks[int(send_off[rank, d]):int(send_off[rank, d] + T[rank, d])],
                  vs[int(send_off[rank, d]):int(send_off[rank, d] + T[rank, d])])
                 for d in range(world)]
        allparts = [None] * world
        dist.all_gather_object(allparts, parts)                        # a8: transposition
        mk = np.concatenate([allparts[g][rank][0] for g in range(world)])
        mv = np.concatenate([allparts[g][rank][1] for g in range(world)])
        assert mk.size == int(T[:, rank].sum())                        # column of T
        assert int(recv_off[rank, world - 1] + T[world - 1, rank]) == mk.size
        assert np.all(oracle.partition(mk, world, pseed) == rank)
        local = oracle.Map(mk.size)
        local.insert(mk, mv)                                           # a9
        # query cascade (a6, a8, a9, a10): every rank asks about a mix of keys
        qk, _ = wdgen.mixed_queries(world * n_local, 5000, 0.5, seed, start=rank * 5000)
        dst = oracle.partition(qk, world, pseed)
        asks = [None] * world
        dist.all_gather_object(asks, [qk[dst == d] for d in range(world)])
        answers = [local.retrieve(asks[g][rank]) for g in range(world)]
        back = [None] * world
        dist.all_gather_object(back, answers)
        gv = np.empty(qk.size, np.uint32); gf = np.empty(qk.size, np.uint8)
        for d in range(world):                                          # unpermute
            gv[dst == d], gf[dst == d] = back[d][rank]
        ev, ef = oracle.expected_unique(qk, world * n_local, seed, seed)
        assert np.array_equal(gf, ef) and np.array_equal(gv, ev)
        dist.destroy_process_group()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))


@pytest.mark.parametrize("fn", [_plumbing, _cascade])
def test_world2_gloo(fn):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=fn, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
