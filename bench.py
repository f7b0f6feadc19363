#!/usr/bin/env python
"""bench.py — WarpDrive hot path on B200: G inserts/s + G queries/s at load 0.95.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference] [--sweep]

One step = one pass of the whole hot path over one batch of synthetic input
(SURVEY §8(a)): a1 table fill, a2+a3 insert of n unique pairs, a2+a4 retrieve of the same
n keys (100 % hits; BASELINE config 2's "insert and retrieve" at alpha = 0.95, |g| = 16);
with N > 1 (torchrun, one process per GPU, weak scaling: n pairs per GPU) the insert and
retrieve run the distributed cascades a6-a10 (multisplit fused with the NVLink push, T
flags, local probe, reverse pull + unpermute).

value      = (inserts + queries of all ranks) / max-over-ranks step time, device-resident
             inputs, CUDA events on the launching stream.
e2e        = the same step through the C-ABI with PINNED HOST buffers: H2D of keys/values/
             queries and D2H of values/found inside the timed region (out-of-core path a11).
roofline   = the dominant call (CUDA-event time inside the timed region; the retrieve is
             one probe launch, the bulk insert one launch per table slice plus the slice
             grouping, WD_OPT_SLICES) against the measured HBM copy bandwidth
             (MEASURED_PEAKS.json), with the ALGORITHMIC bytes of SURVEY §8(d): insert
             8 + 32 S_ins + 32 B, hit query 9 + 32 S_hit B, S from the oracle's sequential
             Fig. 3 replay (tests/golden/probe_cost.json, written by tools/probe_cost.py);
             `traffic` = measured DRAM bytes of those launches per call (profiles/traffic.json,
             ncu launch list, tools/traffic_per_call.py), and
             `pattern_ceiling` = the same call against this B200's measured random-access
             rate for the probe's access pattern (profiles/ceilings.json).
cpu_baseline = the oracle (single-threaded C dictionary) on a bounded sample.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "G inserts/s and G queries/s at load 0.95, 1/2/4/8 B200; % HBM sector roofline"
UNIT = "G ops/s"
KEY_SEED, VAL_SEED = 0x5EED, 0xBEEF


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n-log2", type=int, default=None,
                    help="config 2: pairs per GPU (28); config 3: 2^n - [n = 32] pairs in total (32); "
                         "config 4: table keys (31); config 5: draws per GPU (30)")
    ap.add_argument("--alpha", type=float, default=0.95)
    ap.add_argument("--group-size", type=int, default=None,
                    help="|g| (config 2: 16, the fastest at alpha 0.95 on B200, "
                         "profiles/r01_sweep.jsonl; config 3: 4; config 4: 16; config 5: 8)")
    ap.add_argument("--kif", type=int, default=0, help="keys in flight per group (0=default)")
    ap.add_argument("--probe-mode", type=int, default=None,
                    help="0: auto; 1: cooperative group per window (Fig. 3); 2: lane-window")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--dist-backend", default="nccl",
                    help="torch.distributed backend for the control plane (gloo: tests)")
    ap.add_argument("--same-device", action="store_true",
                    help="all ranks on cuda:0 (dry run of the N>1 path on a 1-GPU box)")
    ap.add_argument("--strong", action="store_true",
                    help="strong scaling (Fig. 9, eq. 4): 2^n-log2 pairs in total, split over "
                         "the ranks (default: weak, 2^n-log2 pairs per GPU)")
    ap.add_argument("--sweep", action="store_true",
                    help="extra lines: config-2 alpha x |g| sweep (not the headline)")
    ap.add_argument("--config", type=int, default=2, choices=[2, 3, 4, 5],
                    help="BASELINE config: 2 (default headline; weak, n pairs per GPU), "
                         "3 (2^32 - 1 unique pairs in total, strong), 4 (query mix on a 2^31-key "
                         "table, 2^32 queries at 0/50/100%% hits), 5 (uniform draws with "
                         "duplicates streamed from pinned host memory, per GPU)")
    ap.add_argument("--exchange", type=int, default=0, choices=[0, 1, 2],
                    help="N > 1 transposition: 0 fused peer stores, 1 copy engine, 2 NCCL")
    ap.add_argument("--batch-log2", type=int, default=None,
                    help="items per shard per cascade batch (default 24, P:197)")
    args = ap.parse_args()
    if args.n_log2 is None:
        args.n_log2 = {2: 28, 3: 32, 4: 31, 5: 30}[args.config]
    if args.group_size is None:
        args.group_size = {2: 16, 3: 4, 4: 16, 5: 8}[args.config]
    return args


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.proc = index, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "50"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        sm = [float(r[0]) for r in self.rows if len(r) >= 7 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 7 and r[1].replace(".", "").isdigit()]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 7
                          for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": reasons,
                "samples": len(sm)}


# ----------------------------------------------------------------------------- helpers
def probe_cost(alpha: float, G: int):
    d = json.load(open(os.path.join(ROOT, "tests", "golden", "probe_cost.json")))
    best = min(d["rows"], key=lambda r: (abs(r["alpha"] - alpha), abs(r["G"] - G)))
    return best


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def cpu_baseline_sample(log2n: int = 28):
    """The oracle as it stands (single-threaded C dictionary) on config 2's FULL size by
    default (2^28 unique inserts + 2^28 hit queries, ~30 s on one core of the
    GPU box, profiles/r02/oracle_full.json); inputs from the same counter-based generator,
    produced on the device and copied to the host.  --n-log2 below 28 scales it down."""
    import numpy as np
    import oracle
    n = 1 << log2n
    try:
        import wdgen.gpu as gg
        keys = gg.unique_keys(n, KEY_SEED).cpu().numpy().view(np.uint32)
        vals = gg.values(n, VAL_SEED).cpu().numpy().view(np.uint32)
    except Exception:
        import wdgen
        keys, vals = wdgen.unique_keys(n, KEY_SEED), wdgen.values(n, VAL_SEED)
    m = oracle.Map(n)
    t0 = time.perf_counter()
    m.insert(keys, vals)
    t1 = time.perf_counter()
    v, f = m.retrieve(keys)
    t2 = time.perf_counter()
    assert int(f.sum()) == n and np.array_equal(v, vals)
    return {"value": 2 * n / (t2 - t0) / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"2^{log2n} unique inserts + 2^{log2n} hit queries (config-2 workload"
                      f"{', full size' if log2n == 28 else ', scaled'}), single-threaded C dictionary",
            "insert_gops": n / (t1 - t0) / 1e9, "query_gops": n / (t2 - t1) / 1e9,
            "seconds": t2 - t0, "host_cpus": os.cpu_count()}


def pcie_roofline(torch, n, te_ms, hk, hv, dk, dv, barrier):
    """The e2e step's PCIe bound, measured live on this GPU with plain pinned copies of the
    same buffers (cudaMemcpyAsync through torch): the insert must bring 8n bytes host ->
    device (t_ins); the retrieve brings 4n bytes in while 5n bytes (values + found flags) go
    out, both directions at once on two streams (t_ret).  bound = t_ins + t_ret, each the
    best of 5 timed repetitions; frac = bound / measured e2e step (1.0 = PCIe-limited)."""
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    ho = torch.empty(n, dtype=torch.int32, pin_memory=True)
    hf = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    df = torch.empty(n, dtype=torch.uint8, device="cuda")
    cur = torch.cuda.current_stream()

    def timed(fn, reps=5):
        ts = []
        for _ in range(reps + 1):
            barrier()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(cur)
            s1.wait_stream(cur)
            s2.wait_stream(cur)
            fn()
            cur.wait_stream(s1)
            cur.wait_stream(s2)
            b.record(cur)
            barrier()
            ts.append(a.elapsed_time(b) * 1e-3)
        return min(ts[1:])

    def ins():
        with torch.cuda.stream(s1):
            dk.copy_(hk, non_blocking=True)
            dv.copy_(hv, non_blocking=True)

    def ret():
        with torch.cuda.stream(s1):
            dk.copy_(hk, non_blocking=True)
        with torch.cuda.stream(s2):
            ho.copy_(dv, non_blocking=True)
            hf.copy_(df, non_blocking=True)

    t_ins = timed(ins)                     # 8n bytes in
    t_ret = timed(ret)                     # 4n in || 5n out
    del ho, hf, df
    bound_ms = (t_ins + t_ret) * 1e3
    return {"h2d_GBps": 8 * n / t_ins / 1e9, "retrieve_in_out_GBps": 9 * n / t_ret / 1e9,
            "insert_copy_ms": t_ins * 1e3, "retrieve_copy_ms": t_ret * 1e3,
            "bound_ms": bound_ms, "frac": bound_ms / te_ms,
            "model": "copy(8n in) + copy(4n in || 5n out), pinned cudaMemcpyAsync of the "
                     "same buffers, CUDA events, best of 5"}


def workload_config(args, world):
    n = (1 << args.n_log2) // (world if args.strong else 1)
    per = "in total" if args.strong else "per GPU"
    return {"workload": f"config2: 2^{args.n_log2} unique u32 key/value pairs {per}, "
                        f"load {args.alpha}, |g|={args.group_size}; step = fill + insert all + "
                        f"retrieve all (100% hits, queried in insert order)",
            "global_batch": n * world, "pairs_per_gpu": n, "alpha": args.alpha,
            "group_size": args.group_size,
            "parallelism": f"keyspace-shard{world}" if world > 1 else "single",
            "exchange": ["fused peer stores", "copy engine", "NCCL"][args.exchange] if world > 1 else None,
            "l2": "inputs (2 x 2^%d x 4 B) and table exceed the 126 MB L2; no flush" % args.n_log2}


def make_config(args, world):
    """the `config` object of the JSON line — identical for our arm and the reference arm"""
    if args.config == 2:
        return workload_config(args, world)
    G, alpha = args.group_size, args.alpha
    if args.config == 3:
        n_total = (1 << args.n_log2) - (1 if args.n_log2 == 32 else 0)
        size = "2^32 - 1, C14" if args.n_log2 == 32 else f"2^{args.n_log2}"
        wl = (f"config3: {n_total} unique u32 pairs in total ({size}) hash-partitioned over "
              f"the GPUs, load {alpha}, |g|={G}; step = fill + insert all + retrieve all")
    elif args.config == 4:
        wl = (f"config4: table of 2^{args.n_log2} unique keys (load {alpha}, |g|={G}); "
              f"2^{args.n_log2 + 1} queries at 0 / 50 / 100 % hits each (reverse exchange + "
              f"unpermute); step = the three query batches")
    else:
        N = (1 << args.n_log2) * world
        expect = 2**32 * (1 - math.exp(-N / 2**32))
        wl = (f"config5: 2^{args.n_log2} uniform draws WITH replacement per GPU ({N} in total) "
              f"in pinned host memory, streamed (a11) into a table sized for the expected "
              f"{expect:.0f} distinct keys at load {alpha}, |g|={G}; step = fill + insert all + "
              f"retrieve all back to pinned host memory")
    return {"workload": wl, "baseline_config": args.config, "group_size": G, "alpha": alpha,
            "parallelism": f"keyspace-shard{world}" if world > 1 else "single",
            "exchange": ["fused peer stores", "copy engine", "NCCL"][args.exchange] if world > 1 else None,
            "l2": "inputs and table exceed the 126 MB L2; no flush"}


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    """--impl reference: the oracle (this tier's reference arm: the single-threaded C
    dictionary of oracle/) on one host core, timed as it stands on a BOUNDED sample of the
    same config's workload per step (same generator, same metric, same `config` object):
    configs 2 / 3: 2^22 unique inserts + 2^22 hit queries; config 4: 3 x 2^23 queries (0 / 50
    / 100 % hits) on a 2^22-key table; config 5: 2^22 uniform draws with duplicates, inserted
    and queried back.  Under torchrun only rank 0 runs."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    import wdgen
    n = 1 << 22
    times = []
    if args.config in (2, 3):
        keys, vals = wdgen.unique_keys(n, KEY_SEED), wdgen.values(n, VAL_SEED)
        sample = (f"2^22 unique inserts + 2^22 hit queries per step (config-{args.config} keys, generator "
                  f"indices [0, 2^22){'; the 1/1024 subset of config 3' if args.config == 3 else ''})")
        ops = 2 * n
    elif args.config == 4:
        # the 1/1024 subset of config 4: a 2^21-key table, 2^22 queries per mix
        nt = n // 2
        keys, vals = wdgen.unique_keys(nt, KEY_SEED), wdgen.values(nt, VAL_SEED)
        qs = [wdgen.mixed_queries(nt, n, h, KEY_SEED)[0] for h in (0.0, 0.5, 1.0)]
        sample = ("oracle rate on the 1/1024 subset: 2^21-key table (untimed insert) + 3 x 2^22 "
                  "queries at 0 / 50 / 100 % hits per step")
        ops = 3 * n
    else:
        # the 1/1024 subset of config 5's 2^35 draws
        n = 1 << 25
        keys, vals = wdgen.uniform_keys(n, KEY_SEED), wdgen.values(n, VAL_SEED)
        sample = ("oracle rate on the 1/1024 subset: 2^25 uniform draws with replacement "
                  "(duplicate mode) inserted + queried back per step")
        ops = 2 * n
    for it in range(args.warmup + args.steps):
        m = oracle.Map(n, dup_mode=args.config == 5)
        if args.config == 4:
            m.insert(keys, vals)
            t0 = time.perf_counter()
            for q in qs:
                m.retrieve(q)
        else:
            t0 = time.perf_counter()
            m.insert(keys, vals)
            m.retrieve(keys)
        dt = time.perf_counter() - t0
        m.close()
        if it >= args.warmup:
            times.append(dt)
    t = sum(times) / len(times)
    val = ops / t / 1e9
    scaling = "weak" if args.config in (2, 5) and not args.strong else "strong"
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3,
            "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "u32", "data": "synthetic", "impl": "reference",
            "config": make_config(args, args.gpus),
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": sample + ", single-threaded C oracle (oracle/wd_oracle.c)"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- configs 3-5
def _setup_dist(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    assert world == args.gpus or world == 1, "launch N>1 with torchrun --nproc-per-node N"
    dev = 0 if args.same_device else local_rank
    torch.cuda.set_device(dev)
    if world > 1:
        backend = "gloo" if args.same_device else args.dist_backend
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
    return torch, dist, world, rank, dev, barrier


def _make_table(wd, args, capacity_total, world, rank):
    kw = {}
    if args.batch_log2 is not None:
        kw["batch"] = 1 << args.batch_log2
    if world > 1:
        t = wd.Table(capacity_total, group_size=args.group_size, rank=rank, world=world,
                     exchange=args.exchange, **kw)
    else:
        t = wd.Table(capacity_total, 1, args.group_size, **kw)
    if args.kif:
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, args.kif)
    return t


def _phases(table, wd, fn, steps=1):
    """one instrumented repetition of fn (not the timed region): per-phase CUDA-event ms"""
    table.phase_times()
    table.set_option(wd.WD_OPT_PHASE_TIMING, 1)
    for _ in range(steps):
        fn()
    out = table.phase_times()
    table.set_option(wd.WD_OPT_PHASE_TIMING, 0)
    return {k: round(v[0] / steps, 4) for k, v in out.items() if v[1]}


def _nvlink(world, bytes_per_op, ops_per_rank, phase_ms):
    """NVLink bytes of a cascade call per rank and their rate over the phase that moves them
    (fused exchange: inside the multisplit / probe; staged: the exchange / reverse phase),
    against NVLink 5's 900 GB/s per direction per GPU"""
    if world == 1 or not phase_ms:
        return None
    b = bytes_per_op * (world - 1) / world * ops_per_rank
    gbs = b / (phase_ms * 1e-3) / 1e9
    return {"bytes_per_op": bytes_per_op * (world - 1) / world, "bytes_per_rank": b,
            "phase_ms": phase_ms, "GBps_per_gpu": gbs, "frac_of_900GBps": gbs / 900.0}


def run_config(args):
    """BASELINE configs 3, 4, 5 at N GPUs (torchrun, one process per GPU; rank mode).
    Inputs are device-resident (3, 4) or pinned host memory (5), generated by the seeded
    generator; every query of the measured configuration is checked against the closed form
    (3, 4) or the drawn pairs (5, N = 1) after the warm-up."""
    import numpy as np  # noqa: F401
    torch, dist, world, rank, dev, barrier = _setup_dist(args)
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg
    from paper_conf_ipps_junger0s18_b200.dist import max_over_ranks
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    stream = torch.cuda.current_stream()
    G, alpha = args.group_size, args.alpha
    info, checks = {}, {}
    if args.config == 3:
        # 2^32 pairs -> n = 2^32 - 1 unique keys (C14), contiguous 1/N index slices
        n_total = (1 << args.n_log2) - (1 if args.n_log2 == 32 else 0)
        lo, hi = n_total * rank // world, n_total * (rank + 1) // world
        n = hi - lo
        table = _make_table(wd, args, int(math.ceil(n_total / alpha)), world, rank)
        keys, vals = gg.unique_keys(n, KEY_SEED, start=lo), gg.values(n, VAL_SEED, start=lo)
        vout = torch.empty(n, dtype=torch.int32, device="cuda")
        fout = torch.empty(n, dtype=torch.uint8, device="cuda")

        def step(m=None):
            table.clear(stream)
            if m: m[0].record(stream)
            table.insert(keys, vals, stream)
            if m: m[1].record(stream)
            table.retrieve(keys, vout, fout, stream)
            if m: m[2].record(stream)
        ops_total = 2 * n_total
        scaling = "strong"
    elif args.config == 4:
        n_table = 1 << args.n_log2
        lo, hi = n_table * rank // world, n_table * (rank + 1) // world
        q_total = 2 * n_table
        nq = q_total // world
        table = _make_table(wd, args, int(math.ceil(n_table / alpha)), world, rank)
        k0, v0 = gg.unique_keys(hi - lo, KEY_SEED, start=lo), gg.values(hi - lo, VAL_SEED, start=lo)
        table.insert(k0, v0, stream)
        torch.cuda.synchronize()
        del k0, v0
        qs = {}
        for h in (0.0, 0.5, 1.0):
            q = torch.empty(nq, dtype=torch.int32, device="cuda")
            hits = torch.empty(nq, dtype=torch.uint8, device="cuda")
            gg.mixed_queries(n_table, nq, h, KEY_SEED, start=rank * nq, out=q, hits=hits)
            qs[h] = (q, hits)
        vout = torch.empty(nq, dtype=torch.int32, device="cuda")
        fout = torch.empty(nq, dtype=torch.uint8, device="cuda")

        def step(m=None):
            for i, h in enumerate((0.0, 0.5, 1.0)):
                if m: m[i].record(stream)
                table.retrieve(qs[h][0], vout, fout, stream)
            if m: m[3].record(stream)
        ops_total = 3 * q_total
        scaling = "strong"
    else:
        per = 1 << args.n_log2
        N = per * world
        expect = 2**32 * (1 - math.exp(-N / 2**32))
        table = _make_table(wd, args, int(math.ceil(expect / alpha)), world, rank)
        if args.batch_log2 is None and world == 1:
            table.set_option(wd.WD_OPT_BATCH, 1 << 22)
        dk = gg.uniform_keys(per, KEY_SEED, start=rank * per)
        dv = gg.values(per, VAL_SEED, start=rank * per)
        hk = torch.empty(per, dtype=torch.int32, pin_memory=True)
        hv = torch.empty(per, dtype=torch.int32, pin_memory=True)
        hk.copy_(dk)
        hv.copy_(dv)
        hvo = torch.empty(per, dtype=torch.int32, pin_memory=True)
        hfo = torch.empty(per, dtype=torch.uint8, pin_memory=True)

        def step(m=None):
            table.clear(stream)
            if m: m[0].record(stream)
            table.insert(hk, hv, stream)
            if m: m[1].record(stream)
            table.retrieve(hk, hvo, hfo, stream)
            if m: m[2].record(stream)
        ops_total = 2 * N
        scaling = "weak"

    # ---- warm-up + every-query check of the measured configuration
    nmarks = 4 if args.config == 4 else 3
    for _ in range(max(1, args.warmup)):
        step()
    barrier()
    st = table.sync()
    assert st == 0, f"device-side status {st}: {wd._lib.wd_last_error_message()}"
    if args.config == 3:
        assert table.size() == n_total
        bad, first, found = gg.check_unique(keys, vout, fout, n_total, KEY_SEED, VAL_SEED)
        assert bad == 0 and found == n, (bad, first, found)
        checks = {"queries_checked": n, "mismatches": bad, "kind": "closed form, every query"}
    elif args.config == 4:
        found = {}
        for h in (0.0, 0.5, 1.0):
            table.retrieve(qs[h][0], vout, fout, stream)
            bad, first, f = gg.check_unique(qs[h][0], vout, fout, n_table, KEY_SEED, VAL_SEED)
            assert bad == 0 and bool((fout == qs[h][1]).all()), (h, bad, first)
            found[str(h)] = f
        checks = {"queries_checked": 3 * nq, "mismatches": 0, "found": found,
                  "kind": "closed form + generator hit flag, every query"}
    else:
        size = table.size()
        assert abs(size - expect) < 6 * math.sqrt(expect) + 16, (size, expect)
        assert bool((hfo == 1).all())
        checks = {"size": size, "expected_distinct": expect, "all_found": True}
        if world == 1:
            uniq = torch.unique(dk.to(torch.int64) & 0xFFFFFFFF)
            assert size == uniq.numel()
            pairs = torch.sort(((dk.to(torch.int64) & 0xFFFFFFFF) << 32) | (dv.to(torch.int64) & 0xFFFFFFFF)).values
            got = ((dk.to(torch.int64) & 0xFFFFFFFF) << 32) | (hvo.cuda().to(torch.int64) & 0xFFFFFFFF)
            pp = torch.searchsorted(pairs, got).clamp(max=pairs.numel() - 1)
            assert bool((pairs[pp] == got).all())
            checks.update(distinct_exact=True, values_checked=per, kind="every returned value among the drawn pairs")
            del uniq, pairs, got, pp
        del dk, dv

    # ---- timed region
    launches0 = table.launches
    marks = [[ev() for _ in range(nmarks)] for _ in range(args.steps)]
    e0, e1 = ev(), ev()
    with ClockSampler(dev) as clk:
        barrier()
        e0.record(stream)
        for k in range(args.steps):
            step(marks[k])
        e1.record(stream)
        barrier()
    launches = table.launches - launches0
    t_ms = max_over_ranks(e0.elapsed_time(e1) / args.steps)
    sub = [max_over_ranks(sum(mk[i].elapsed_time(mk[i + 1]) for mk in marks) / args.steps)
           for i in range(nmarks - 1)]
    assert table.sync() == 0
    value = ops_total / (t_ms * 1e-3) / 1e9
    phases = _phases(table, wd, lambda: step())
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": t_ms, "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (seeded generator)", "config": make_config(args, world),
            "clocks": clk.summary(), "gpu_launches": launches, "checks": checks,
            "phases_ms_rank0": phases}
    if args.config in (3, 5):
        nn = n_total if args.config == 3 else N
        line["insert_gops"] = nn / (sub[0] * 1e-3) / 1e9
        line["query_gops"] = nn / (sub[1] * 1e-3) / 1e9
        line["nvlink"] = {"insert": _nvlink(world, 8, nn / world, phases.get("multisplit") if args.exchange == 0 else phases.get("exchange")),
                          "query": _nvlink(world, 12, nn / world, phases.get("probe_query") if args.exchange == 0 else phases.get("reverse"))}
    else:
        line["mix"] = {str(h): {"query_gops": q_total / (sub[i] * 1e-3) / 1e9, "ms": sub[i]}
                       for i, h in enumerate((0.0, 0.5, 1.0))}
        line["query_gops"] = value
    if args.config == 5:
        line["e2e"] = {"value": value, "unit": UNIT, "h2d_bytes_per_step": 12 * per,
                       "d2h_bytes_per_step": 5 * per,
                       "note": "config 5 IS the host-streamed path: value is end to end"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    table.close()
    if world > 1:
        dist.destroy_process_group()


# ----------------------------------------------------------------------------- our arm
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    if args.config != 2:
        return run_config(args)
    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    assert world == args.gpus or world == 1, "launch N>1 with torchrun --nproc-per-node N"
    dev = 0 if args.same_device else local_rank
    torch.cuda.set_device(dev)
    if world > 1:
        # NCCL refuses two ranks on one device: the same-device dry run uses gloo
        backend = "gloo" if args.same_device else args.dist_backend
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)

    # weak scaling: n pairs per GPU; strong (--strong): 2^n-log2 in total, n per GPU
    n = (1 << args.n_log2) // (world if args.strong else 1)
    G = args.group_size
    cap_local = int(math.ceil(n / args.alpha))
    table = _make_table(wd, args, cap_local * world, world, rank)
    if args.probe_mode is not None:
        table.set_option(wd.WD_OPT_PROBE_MODE, args.probe_mode)

    # inputs: rank r inserts generator indices [r n, (r+1) n) -> globally unique keys
    keys = gg.unique_keys(n, KEY_SEED, start=rank * n)
    vals = gg.values(n, VAL_SEED, start=rank * n)
    vout = torch.empty(n, dtype=torch.int32, device="cuda")
    fout = torch.empty(n, dtype=torch.uint8, device="cuda")
    stream = torch.cuda.current_stream()
    torch.cuda.synchronize()

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    from paper_conf_ipps_junger0s18_b200.dist import max_over_ranks

    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    def step(marks=None):
        table.clear(stream)
        if marks is not None:
            marks[0].record(stream)
        table.insert(keys, vals, stream)
        if marks is not None:
            marks[1].record(stream)
        table.retrieve(keys, vout, fout, stream)
        if marks is not None:
            marks[2].record(stream)

    # ---- warm-up + correctness of the measured configuration (sampled, closed form)
    for _ in range(args.warmup - 1):
        step()
    # last warm-up step: count the library's launches per call (the insert of a big call
    # into an HBM-sized table is slice-grouped: several launches, WD_OPT_SLICES)
    table.clear(stream)
    l0 = table.launches
    table.insert(keys, vals, stream)
    l1 = table.launches
    table.retrieve(keys, vout, fout, stream)
    per_call = {"insert": l1 - l0, "retrieve": table.launches - l1}
    barrier()
    st = table.sync()
    assert st == 0, f"device-side status {st}: {wd._lib.wd_last_error_message()}"
    assert table.size() == n * world
    idx = torch.randint(0, n, (1 << 16,), device="cuda")
    ok = bool((fout[idx] == 1).all().item()) and bool((vout[idx] == vals[idx]).all().item())
    assert ok, "measured configuration returned wrong results"

    # ---- timed region: device-resident
    # the library brackets every phase (slice grouping, probe launches, ...) with CUDA events
    # on the stream it runs on (WD_OPT_PHASE_TIMING): the probe kernels' own time over the
    # timed steps is the roofline's launch time (a few event records per call)
    launches0 = table.launches
    marks = [[ev(), ev(), ev()] for _ in range(args.steps)]
    e0, e1 = ev(), ev()
    table.phase_times()
    table.set_option(wd.WD_OPT_PHASE_TIMING, 1)
    with ClockSampler(dev) as clk:
        barrier()
        e0.record(stream)
        for k in range(args.steps):
            step(marks[k])
        e1.record(stream)
        barrier()
    launches = table.launches - launches0
    ph_timed = table.phase_times()
    table.set_option(wd.WD_OPT_PHASE_TIMING, 0)
    phases = {k: round(v[0] / args.steps, 4) for k, v in ph_timed.items() if v[1]}
    t_local = e0.elapsed_time(e1) / args.steps
    ins_local = sum(a.elapsed_time(b) for a, b, _ in marks) / args.steps
    qry_local = sum(b.elapsed_time(c) for _, b, c in marks) / args.steps
    t_ms = max_over_ranks(t_local)
    ins_ms = max_over_ranks(ins_local)
    qry_ms = max_over_ranks(qry_local)
    fill_ms = max_over_ranks(t_local - ins_local - qry_local)
    ops = 2 * n * world
    value = ops / (t_ms * 1e-3) / 1e9
    assert table.sync() == 0
    nvlink = None
    if world > 1:
        nvlink = {"insert": _nvlink(world, 8, n, phases.get("multisplit") if args.exchange == 0 else phases.get("exchange")),
                  "query": _nvlink(world, 12, n, phases.get("probe_query") if args.exchange == 0 else phases.get("reverse"))}

    # ---- roofline of the dominant kernel (single GPU: one launch per call)
    pc = probe_cost(args.alpha, G)
    hbm, peak_src = peaks()
    b_ins = 8 + 32 * pc["ins_sectors"] + 32
    b_hit = 9 + 32 * pc["hit_sectors"]
    # the probe kernels' own time (all launches of the call), else the call time
    k_ins = phases.get("probe", ins_ms) if world == 1 else ins_ms
    k_qry = phases.get("probe_query", qry_ms) if world == 1 else qry_ms
    kern = {"insert": (k_ins, b_ins, ins_ms), "retrieve": (k_qry, b_hit, qry_ms)}
    dom = max(kern, key=lambda k: kern[k][0])
    other = "retrieve" if dom == "insert" else "insert"

    def roof(name):
        ms, bpo, call_ms = kern[name]
        ach = n * bpo / (ms * 1e-3) / 1e9
        # N > 1: the insert / retrieve call is the whole cascade (multisplit + NVLink push,
        # flags, local probe, reverse pull + unpermute), timed as one call on the stream
        if world > 1:
            kname = (f"{name} cascade a6-a10 over {world} ranks (call time, not one launch; "
                     f"the N=1 line carries the per-kernel roofline)")
        elif per_call[name] == 1:
            kname = f"probe_kernel<{name}> (G={G}), one launch per call"
        else:
            kname = (f"probe_kernel<{name}, InBucket> (G={G}): the {per_call[name] - 3} probe "
                     f"launches of the slice-grouped call (one per table slice, WD_OPT_SLICES), "
                     f"their summed CUDA-event time over the timed steps; the call adds the "
                     f"slice grouping (histogram, scan, multisplit; `call` below)")
        call_ach = n * bpo / (call_ms * 1e-3) / 1e9
        return {"kernel": kname, "bound": "hbm", "achieved": ach,
                "peak": hbm, "unit": "GB/s", "frac": ach / hbm, "traffic": None,
                "bytes_per_op": bpo, "launch_ms": ms, "launches_per_call": per_call[name],
                "call": {"ms": call_ms, "achieved": call_ach, "frac": call_ach / hbm},
                "sectors_per_op": pc["ins_sectors" if name == "insert" else "hit_sectors"],
                # HBM moves whole 128-B lines for random accesses (C2): the
                # same kernel against the replay's distinct lines per op
                "line_model": line_model(name, ms),
                # the same kernel against the MEASURED random-access rate of its own access
                # pattern on this part (tools/randbench.cu -> profiles/ceilings.json)
                "pattern_ceiling": pattern_ceiling(name, ms)}

    def pattern_ceiling(name, ms):
        cf = os.path.join(ROOT, "profiles", "ceilings.json")
        if not os.path.exists(cf):
            return None
        c = json.load(open(cf))
        wb = str(8 * G)
        L = pc["ins_windows" if name == "insert" else "hit_windows"]
        R = c["read"].get(wb)
        C = c["casw"].get(wb)
        if R is None or (name == "insert" and C is None):
            return None
        t = (L - 1) / R + 1 / C if name == "insert" else L / R      # ns per op
        ach = n / (ms * 1e-3) / 1e9
        out = {"gops": 1 / t, "achieved_gops": ach, "frac": ach * t, "windows_per_op": L,
               "model": ("(L-1) random %s-B window reads + 1 read-then-CAS (randbench casw)"
                         if name == "insert" else "L random %s-B window reads") % wb,
               "rates_Gwin_s": {"read": R, "casw": C}, "source": "profiles/ceilings.json"}
        if ach * t > 1:
            out["note"] = ("above 1: the slice-grouped call serves part of its window loads "
                           "and write-backs from L2, so the random-DRAM pattern does not bound "
                           "it (profiles/r01_slices.txt)")
        return out

    def line_model(name, ms):
        lines = pc.get("ins_lines" if name == "insert" else "hit_lines")
        if lines is None:
            return None
        bpo = (8 + 32 if name == "insert" else 9) + 128 * lines
        ach = n * bpo / (ms * 1e-3) / 1e9
        return {"lines_per_op": lines, "bytes_per_op": bpo, "achieved": ach, "frac": ach / hbm}

    roofline = roof(dom)
    roofline["peak_source"] = peak_src
    roofline["other"] = roof(other)
    traffic_file = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(traffic_file) and world == 1:
        tj = json.load(open(traffic_file))
        for r, name in ((roofline, dom), (roofline["other"], other)):
            tr = tj.get(f"{name}_probe_G{G}_a{args.alpha}_n{args.n_log2}")
            if tr:
                r["traffic"] = tr                       # DRAM bytes of the probe launches
            trc = tj.get(f"{name}_G{G}_a{args.alpha}_n{args.n_log2}")
            if trc:
                r["call"]["traffic"] = trc              # ... of the whole call

    # ---- e2e: the same step through the C-ABI with pinned host buffers
    e2e = None
    if not args.no_e2e:
        hk = torch.empty(n, dtype=torch.int32, pin_memory=True)
        hv = torch.empty(n, dtype=torch.int32, pin_memory=True)
        hk.copy_(keys)
        hv.copy_(vals)
        hvo = torch.empty(n, dtype=torch.int32, pin_memory=True)
        hfo = torch.empty(n, dtype=torch.uint8, pin_memory=True)

        def hstep():
            table.clear(stream)
            table.insert(hk, hv, stream)
            table.retrieve(hk, hvo, hfo, stream)

        hstep()
        barrier()
        assert bool((hfo[:4096] == 1).all()) and bool((hvo[:4096] == hv[:4096]).all())
        e_steps = max(1, min(args.steps, 5))
        a, b = ev(), ev()
        barrier()
        a.record(stream)
        for _ in range(e_steps):
            hstep()
        b.record(stream)
        barrier()
        te = max_over_ranks(a.elapsed_time(b) / e_steps)
        e2e = {"value": ops / (te * 1e-3) / 1e9, "unit": UNIT, "ms_per_step": te,
               "h2d_bytes_per_step": 12 * n, "d2h_bytes_per_step": 5 * n, "steps": e_steps}
        assert table.sync() == 0
        del hvo, hfo
        e2e["pcie"] = pcie_roofline(torch, n, te, hk, hv, keys, vals, barrier)
        del hk, hv

    # ---- CPU baseline (rank 0, N = 1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline_sample(min(args.n_log2, 28))

    sweep_lines = []
    if args.sweep and world == 1:
        sweep_lines = run_sweep(args, wd, gg, torch)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_ms,
            "higher_is_better": True, "scaling": "strong" if args.strong else "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": make_config(args, world),
            "capacity_per_gpu": table.shard_capacity(0),
            "insert_gops": n * world / (ins_ms * 1e-3) / 1e9,
            "query_gops": n * world / (qry_ms * 1e-3) / 1e9,
            "fill_ms": fill_ms,
            "roofline": roofline, "cpu_baseline": cpu,
            "phases_ms_rank0": phases, "nvlink": nvlink,
            "clocks": clk.summary(), "e2e": e2e, "gpu_launches": launches,
            "gpu_launches_per_step": launches / args.steps,
        }
        print(json.dumps(line), flush=True)
        for l in sweep_lines:
            print(json.dumps(l), flush=True)
    table.close()
    if world > 1:
        dist.destroy_process_group()


def run_sweep(args, wd, gg, torch):
    """config 2 sweep (alpha x |g|): insert and retrieve G ops/s with sector-roofline
    fractions; extra lines, not the headline."""
    out = []
    n = 1 << args.n_log2
    keys = gg.unique_keys(n, KEY_SEED)
    vals = gg.values(n, VAL_SEED)
    vout = torch.empty(n, dtype=torch.int32, device="cuda")
    fout = torch.empty(n, dtype=torch.uint8, device="cuda")
    hbm, _ = peaks()
    s = torch.cuda.current_stream()
    for alpha in (0.8, 0.9, 0.95, 0.99):
        for G in (1, 2, 4, 8, 16, 32):
            with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
                ti, tq, tauto, tiauto = [], [], [], []
                for it in range(4):
                    a, b, c, d, e, f = (torch.cuda.Event(enable_timing=True) for _ in range(6))
                    t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)    # the paper's: the table's |g|
                    t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
                    t.clear(s)
                    a.record(s)
                    t.insert(keys, vals, s)
                    b.record(s)
                    t.retrieve(keys, vout, fout, s)
                    c.record(s)
                    t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, -1)    # the library defaults (auto)
                    t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, -1)
                    t.retrieve(keys, vout, fout, s)
                    d.record(s)
                    t.clear(s)
                    e.record(s)
                    t.insert(keys, vals, s)
                    f.record(s)
                    torch.cuda.synchronize()
                    if it:
                        ti.append(a.elapsed_time(b))
                        tq.append(b.elapsed_time(c))
                        tauto.append(c.elapsed_time(d))
                        tiauto.append(e.elapsed_time(f))
                assert t.sync() == 0
                pc = probe_cost(alpha, G)
                ims, qms = sum(ti) / len(ti), sum(tq) / len(tq)
                out.append({"sweep": "config2", "alpha": alpha, "G": G,
                            "insert_gops": n / ims / 1e6, "query_gops": n / qms / 1e6,
                            "query_gops_auto": n / (sum(tauto) / len(tauto)) / 1e6,
                            "insert_gops_auto": n / (sum(tiauto) / len(tiauto)) / 1e6,
                            "insert_frac": n * (40 + 32 * pc["ins_sectors"]) / (ims * 1e-3) / 1e9 / hbm,
                            "query_frac": n * (9 + 32 * pc["hit_sectors"]) / (qms * 1e-3) / 1e9 / hbm})
    out += run_config1(wd, gg, torch)
    out += run_mix(wd, gg, torch, keys, vals, args.n_log2)
    del keys, vals, vout, fout
    out += run_zipf(wd, gg, torch)
    out += run_ooc(wd, gg, torch)
    return out


def l2_roofline(G, ins, qry):
    """Config 1's table (8.8 MB) is L2-resident: its ceiling is this B200's random L2 rate
    for the kernels' own pattern (tools/randbench 0.0088 -> profiles/ceilings.json "l2_8.8MB"):
    an insert = (L - 1) window reads + one read-then-CAS, a query = L window reads, L from the
    oracle replay (hits; misses for the absent half of the queries)."""
    cf = os.path.join(ROOT, "profiles", "ceilings.json")
    if not os.path.exists(cf):
        return None
    c = json.load(open(cf)).get("l2_8.8MB")
    wb = str(min(8 * G, 256))
    if not c or wb not in c["read"] or wb not in c["casw"]:
        return None
    pc = probe_cost(0.95, G)
    R, C = c["read"][wb], c["casw"][wb]
    ins_ceiling = 1.0 / ((pc["ins_windows"] - 1) / R + 1 / C)
    q_ceiling = R / (0.5 * pc["hit_windows"] + 0.5 * pc["miss_windows"])
    return {"insert_ceiling_gops": ins_ceiling, "insert_frac": ins / ins_ceiling,
            "query_ceiling_gops": q_ceiling, "query_frac": qry / q_ceiling,
            "rates_Gwin_s": {"read": R, "casw": C}, "windows": {
                "insert": pc["ins_windows"], "hit": pc["hit_windows"], "miss": pc["miss_windows"]},
            "source": "profiles/ceilings.json l2_8.8MB"}


def run_config1(wd, gg, torch):
    """BASELINE config 1: 2^20 unique pairs at alpha 0.95 (an 8.8 MB, L2-resident table),
    then all 2^20 keys + 2^20 absent keys queried (interleaved); |g| = 4 as configured,
    and 8 / 16 beside it.  Rates are per call (one launch each), device-resident."""
    out = []
    n = 1 << 20
    keys, vals = gg.unique_keys(n, KEY_SEED), gg.values(n, VAL_SEED)
    q = gg.interleaved_queries(n, KEY_SEED)
    vout = torch.empty(2 * n, dtype=torch.int32, device="cuda")
    fout = torch.empty(2 * n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    for G, qg in ((4, 0), (8, 0), (16, 0), (4, -1), (8, -1)):
        with wd.Table(int(math.ceil(n / 0.95)), 1, G) as t:
            t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, qg)   # 0: the paper's (calls with |g|)
            t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, qg)
            ti, tq = [], []
            for it in range(11):
                a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                t.clear(s)
                a.record(s)
                t.insert(keys, vals, s)
                b.record(s)
                t.retrieve(q, vout, fout, s)
                c.record(s)
                torch.cuda.synchronize()
                if it:
                    ti.append(a.elapsed_time(b))
                    tq.append(b.elapsed_time(c))
            assert t.sync() == 0 and t.size() == n and int(fout.sum().item()) == n
            ins = n / (sum(ti) / len(ti)) / 1e6
            qry = 2 * n / (sum(tq) / len(tq)) / 1e6
            out.append({"sweep": "config1", "alpha": 0.95, "G": G, "query_G": "auto" if qg < 0 else G, "keys": n, "queries": 2 * n,
                        "table_MB": t.capacity() * 8 / 1e6, "insert_gops": ins, "query_gops": qry,
                        "l2_roofline": l2_roofline(G, ins, qry)})
    return out


def run_mix(wd, gg, torch, keys, vals, log2n):
    """BASELINE config 4 at one GPU: a 2^log2n-key table at alpha 0.95, then 2^log2n queries
    with hit fraction 0 / 0.5 / 1 (wdgen.mixed_queries: a hit is a stored key, a miss a key
    never inserted).  found must equal the generator's hit flag for every query."""
    out = []
    n = 1 << log2n
    q = torch.empty(n, dtype=torch.int32, device="cuda")
    hits = torch.empty(n, dtype=torch.uint8, device="cuda")
    vout = torch.empty(n, dtype=torch.int32, device="cuda")
    fout = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    hbm, _ = peaks()
    for G in (4, 8, 16):
        with wd.Table(int(math.ceil(n / 0.95)), 1, G) as t:
            t.insert(keys, vals, s)
            for h, qg in ((0.0, 0), (0.5, 0), (1.0, 0), (0.0, -1), (0.5, -1), (1.0, -1)):
                if qg < 0 and G == 16:
                    continue
                t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, qg)   # 0: the paper's (queries with |g|)
                gg.mixed_queries(n, n, h, KEY_SEED, out=q, hits=hits)
                ts = []
                for it in range(4):
                    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    a.record(s)
                    t.retrieve(q, vout, fout, s)
                    b.record(s)
                    torch.cuda.synchronize()
                    if it:
                        ts.append(a.elapsed_time(b))
                assert t.sync() == 0 and bool((fout == hits).all())
                ms = sum(ts) / len(ts)
                pc = probe_cost(0.95, G)
                S = h * pc["hit_sectors"] + (1 - h) * pc["miss_sectors"]
                # the replay's sector counts are for windows of the table's |g| (qg = 0)
                out.append({"sweep": "config4_mix_1gpu", "alpha": 0.95, "G": G, "query_G": "auto" if qg < 0 else G, "hit_frac": h,
                            "table_keys": n, "queries": n, "query_gops": n / ms / 1e6,
                            "sectors_per_query": S if not qg else None,
                            "query_frac": n * (9 + 32 * S) / (ms * 1e-3) / 1e9 / hbm if not qg else None})
    return out


def run_ooc(wd, gg, torch, log2n=30):
    """BASELINE config 5 scaled to one GPU: 2^log2n uniform draws WITH replacement (duplicate
    keys) in pinned host memory, streamed through the C-ABI's out-of-core pipeline
    (H2D(b+1) || insert(b), batches of 2^22 pairs: the library's single-shard default
    used 2^24) into a table sized for the expected
    number of distinct keys at alpha 0.95 (C13); then all draws are queried back to pinned
    host memory.  Checks: size = distinct count; every query found; on the keys with
    k mod 1024 == 0, each returned value is one of the values drawn for that key."""
    n = 1 << log2n
    keys = gg.uniform_keys(n, KEY_SEED)
    vals = gg.values(n, VAL_SEED)
    distinct = int(torch.unique(keys).numel())
    expect = 2**32 * (1 - math.exp(-n / 2**32))
    hk = torch.empty(n, dtype=torch.int32, pin_memory=True)
    hv = torch.empty(n, dtype=torch.int32, pin_memory=True)
    hk.copy_(keys)
    hv.copy_(vals)
    hvo = torch.empty(n, dtype=torch.int32, pin_memory=True)
    hfo = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    s = torch.cuda.current_stream()
    out = []
    with wd.Table(int(math.ceil(expect / 0.95)), 1, 8, batch=1 << 22) as t:
        ti, tq = [], []
        for it in range(3):
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t.clear(s)
            a.record(s)
            t.insert(hk, hv, s)
            b.record(s)
            t.retrieve(hk, hvo, hfo, s)
            c.record(s)
            torch.cuda.synchronize()
            if it:
                ti.append(a.elapsed_time(b))
                tq.append(b.elapsed_time(c))
        assert t.sync() == 0 and t.size() == distinct
        assert bool((hfo == 1).all())
        # subset check of duplicate mode: (k, returned v) must be a drawn pair
        sel = (keys.to(torch.int64) & 0xFFFFFFFF) % 1024 == 0
        pairs = ((keys[sel].to(torch.int64) & 0xFFFFFFFF) << 32) | (vals[sel].to(torch.int64) & 0xFFFFFFFF)
        pairs = torch.unique(pairs)
        got = ((keys[sel].to(torch.int64) & 0xFFFFFFFF) << 32) | \
              (hvo.cuda()[sel].to(torch.int64) & 0xFFFFFFFF)
        pos = torch.searchsorted(pairs, got).clamp(max=pairs.numel() - 1)
        assert bool((pairs[pos] == got).all()), "duplicate mode: value not among the drawn ones"
        ims, qms = sum(ti) / len(ti), sum(tq) / len(tq)
        out.append({"sweep": "config5_ooc_1gpu", "draws": n, "distinct": distinct,
                    "expected_distinct": expect, "alpha_actual": distinct / t.capacity(),
                    "G": 8, "batch": 1 << 22, "insert_gops_e2e": n / ims / 1e6,
                    "query_gops_e2e": n / qms / 1e6,
                    "h2d_GBps_insert": 8 * n / (ims * 1e-3) / 1e9,
                    "pcie_bytes": {"insert_h2d": 8 * n, "query_h2d": 4 * n, "query_d2h": 5 * n},
                    "checked_pairs": int(sel.sum().item())})
    return out


def run_zipf(wd, gg, torch, log2n=27):
    """SURVEY §8(f) #1 / Fig. 8 protocol: 2^27 Zipf(s = 1 + 1e-6) draws over
    the 4-byte key space, insert all then retrieve all; load = actual occupancy (distinct
    keys / capacity).  Extra lines, not the headline."""
    out = []
    n = 1 << log2n
    keys = gg.zipf_keys(n, 2**32 - 1, KEY_SEED)
    vals = gg.values(n, VAL_SEED)
    distinct = int(torch.unique(keys).numel())
    vout = torch.empty(n, dtype=torch.int32, device="cuda")
    fout = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    for alpha in (0.8, 0.95):
        for G in (1, 2, 4, 8, 16):
            with wd.Table(int(math.ceil(distinct / alpha)), 1, G) as t:
                t.set_option(wd.WD_OPT_INSERT_GROUP_SIZE, 0)   # the paper's Fig. 8 grid: |g| as given
                t.set_option(wd.WD_OPT_QUERY_GROUP_SIZE, 0)
                ti, tq = [], []
                for it in range(4):
                    a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                    t.clear(s)
                    a.record(s)
                    t.insert(keys, vals, s)
                    b.record(s)
                    t.retrieve(keys, vout, fout, s)
                    c.record(s)
                    torch.cuda.synchronize()
                    if it:
                        ti.append(a.elapsed_time(b))
                        tq.append(b.elapsed_time(c))
                assert t.sync() == 0 and t.size() == distinct
                assert bool((fout == 1).all())
                ims, qms = sum(ti) / len(ti), sum(tq) / len(tq)
                out.append({"sweep": "zipf", "draws": n, "distinct": distinct, "alpha": alpha,
                            "G": G, "insert_gops": n / ims / 1e6, "query_gops": n / qms / 1e6})
    return out


if __name__ == "__main__":
    main()
