"""Insert / retrieve rates of one configuration (measurement tool, one JSON line per run).

    python tools/rates.py LOG2N G [alpha] [key=value ...]

keys: slices=<WD_OPT_SLICES>, v=<WD_OPT_SLOTS_PER_LANE>, k=<WD_OPT_KEYS_IN_FLIGHT>,
span=<WD_OPT_SPAN>, reps=<timed repetitions>.  The kernel variant follows the environment
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
       "span": wd.WD_OPT_SPAN, "mode": wd.WD_OPT_PROBE_MODE}


def main():
    lg, G = int(sys.argv[1]), int(sys.argv[2])
    alpha = float(sys.argv[3]) if len(sys.argv) > 3 and "=" not in sys.argv[3] else 0.95
    kv = dict(a.split("=") for a in sys.argv[3:] if "=" in a)
    reps = int(kv.pop("reps", 5))
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 11), gg.values(n, 12)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
        for k, v in kv.items():
            t.set_option(OPT[k], int(v))
        ti, tq = [], []
        for r in range(reps + 1):
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t.clear(s)
            a.record(s)
            t.insert(keys, vals, s)
            b.record(s)
            t.retrieve(keys, vo, fo, s)
            c.record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(a.elapsed_time(b))
                tq.append(b.elapsed_time(c))
        assert t.sync() == 0 and t.size() == n
        bad, first, found = gg.check_unique(keys, vo, fo, n, 11, 12)
        assert bad == 0 and found == n
        ims, qms = sum(ti) / len(ti), sum(tq) / len(tq)
        print(json.dumps({"n_log2": lg, "G": G, "alpha": alpha, "opts": kv,
                          "kernel": os.environ.get("WD_PROBE_KERNEL", "lean"),
                          "table_MB": t.capacity() * 8 / 1e6,
                          "insert_gops": n / ims / 1e6, "query_gops": n / qms / 1e6,
                          "insert_ms": ims, "query_ms": qms}), flush=True)


if __name__ == "__main__":
    main()
