"""Insert / retrieve rates of one configuration (measurement tool, one JSON line per run).

    python tools/rates.py LOG2N G [alpha] [key=value ...]

keys: slices=<WD_OPT_SLICES>, v=<WD_OPT_SLOTS_PER_LANE>, k=<WD_OPT_KEYS_IN_FLIGHT>,
span=<WD_OPT_SPAN>, ig=<WD_OPT_INSERT_GROUP_SIZE>, reps=<timed repetitions>, qg=<|g| of the retrieve calls> (any |g| probes
the same sequence; default the table's).  The kernel variant follows the environment
(WD_PROBE_KERNEL=classic for the round-1 kernel).  Device-resident unique keys; every query
checked against the closed form after the timed runs."""
import json
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402

OPT = {"slices": wd.WD_OPT_SLICES, "v": wd.WD_OPT_SLOTS_PER_LANE, "k": wd.WD_OPT_KEYS_IN_FLIGHT,
       "ig": wd.WD_OPT_INSERT_GROUP_SIZE,
       "span": wd.WD_OPT_SPAN, "mode": wd.WD_OPT_PROBE_MODE,
       "flags": wd.WD_OPT_KERNEL_FLAGS}


def main():
    lg, G = int(sys.argv[1]), int(sys.argv[2])
    alpha = float(sys.argv[3]) if len(sys.argv) > 3 and "=" not in sys.argv[3] else 0.95
    kv = dict(a.split("=") for a in sys.argv[3:] if "=" in a)
    reps = int(kv.pop("reps", 5))
    qg = int(kv.pop("qg", G))
    qmode = kv.pop("q", "")                 # inter: config 1 (all keys + as many absent,
    inter = qmode == "inter"                # interleaved); miss: absent keys only
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 11), gg.values(n, 12)
    qk = gg.interleaved_queries(n, 11) if inter else (gg.unique_keys(n, 11, start=n) if qmode == "miss" else keys)
    nq = qk.numel()
    vo = torch.empty(nq, dtype=torch.int32, device="cuda")
    fo = torch.empty(nq, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
        for k, v in kv.items():
            t.set_option(OPT[k], int(v))
        ti, tq = [], []
        for r in range(reps + 1):
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t.clear(s)
            t.set_option(wd.WD_OPT_GROUP_SIZE, G)
            a.record(s)
            t.insert(keys, vals, s)
            b.record(s)
            t.set_option(wd.WD_OPT_GROUP_SIZE, qg)
            t.retrieve(qk, vo, fo, s)
            c.record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(a.elapsed_time(b))
                tq.append(b.elapsed_time(c))
        assert t.sync() == 0 and t.size() == n
        t.phase_times()
        t.set_option(wd.WD_OPT_PHASE_TIMING, 1)
        t.clear(s)
        t.set_option(wd.WD_OPT_GROUP_SIZE, G)
        t.insert(keys, vals, s)
        t.set_option(wd.WD_OPT_GROUP_SIZE, qg)
        ph_ins = {k: round(v[0], 4) for k, v in t.phase_times().items() if v[1]}
        t.retrieve(qk, vo, fo, s)
        ph_q = {k: round(v[0], 4) for k, v in t.phase_times().items() if v[1]}
        t.set_option(wd.WD_OPT_PHASE_TIMING, 0)
        bad, first, found = gg.check_unique(qk, vo, fo, n, 11, 12)
        assert bad == 0 and found == (0 if qmode == "miss" else n)
        ims, qms = sum(ti) / len(ti), sum(tq) / len(tq)
        print(json.dumps({"n_log2": lg, "G": G, "query_G": qg, "alpha": alpha, "opts": kv,
                          "env": {k: v for k, v in os.environ.items() if k.startswith("WD_")},
                          "table_MB": t.capacity() * 8 / 1e6,
                          "insert_gops": n / ims / 1e6, "query_gops": nq / qms / 1e6, "queries": nq,
                          "insert_ms": ims, "query_ms": qms, "insert_phases_ms": ph_ins,
                          "query_phases_ms": ph_q}), flush=True)


if __name__ == "__main__":
    main()
