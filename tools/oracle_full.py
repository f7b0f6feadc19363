"""The oracle (oracle/wd_oracle.c: single-threaded C dictionary, the tier's CPU baseline) at
BASELINE config 2's FULL size on the GPU box's host (SURVEY §8(d) "configs 1-2 run at full
size"): 2^28 unique inserts then 2^28 hit queries, inputs from the same seeded generator,
every answer checked against the closed form.  bench.py's cpu_baseline keeps a bounded sample
(the run must stay within minutes); this records the full-size rate beside it.

    python tools/oracle_full.py [LOG2N]     # one JSON line"""
import json
import os
import platform
import sys
import time

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import wdgen  # noqa: E402


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
    n = 1 << lg
    t0 = time.perf_counter()
    keys, vals = wdgen.unique_keys(n, 0x5EED), wdgen.values(n, 0xBEEF)
    tg = time.perf_counter() - t0
    m = oracle.Map(n)
    t1 = time.perf_counter()
    m.insert(keys, vals)
    t2 = time.perf_counter()
    v, f = m.retrieve(keys)
    t3 = time.perf_counter()
    ok = bool(f.all()) and np.array_equal(v, vals) and m.size() == n
    cpu = ""
    try:
        cpu = next(l.split(":", 1)[1].strip() for l in open("/proc/cpuinfo") if l.startswith("model name"))
    except Exception:
        cpu = platform.processor()
    print(json.dumps({"tool": "oracle_full", "workload": f"config2: 2^{lg} unique inserts + 2^{lg} hit queries",
                      "insert_gops": n / (t2 - t1) / 1e9, "query_gops": n / (t3 - t2) / 1e9,
                      "value_gops": 2 * n / (t3 - t1) / 1e9, "seconds": t3 - t1,
                      "generation_s": tg, "cores": 1, "host_cpus": os.cpu_count(), "cpu": cpu,
                      "exact": ok}), flush=True)


if __name__ == "__main__":
    main()
