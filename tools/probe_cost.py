"""Write tests/golden/probe_cost.json: windows, distinct 32-byte sectors and distinct
128-byte lines per op of the
sequential Fig. 3 replay (oracle only) for alpha x |g|, at n = 2^22 unique keys.

These are the ALGORITHMIC sector counts S of SURVEY §8(d) (the bytes the method must move
per op on a table >> L2): insert/hit = 8 B input + 32 S_ins (+32 B dirty sector for an
insert), miss = 9 B + 32 S_miss.  bench.py reads this file; it never imports the oracle
for the GPU measurement.  Re-run after any change to oracle/wd_oracle.c's replay.
"""
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import wdgen  # noqa: E402


def main(n=1 << 22):
    keys, vals = wdgen.unique_keys(n, 1), wdgen.values(n, 2)
    absent = wdgen.unique_keys(n // 4, 1, start=n)
    out = {"_source": "tools/probe_cost.py: oracle.Replay (sequential Fig. 3, readings C1/C2, "
                      "32-slot regions starting at multiples of A = 4 slots, A = 16 for |g| >= 16 (C2'), "
                      "prime region count), "
                      "n = %d unique keys, p_max = 1024" % n,
           "rows": []}
    for alpha in (0.8, 0.9, 0.95, 0.99):
        c = oracle.physical_capacity(int(math.ceil(n / alpha)))
        for G in (1, 2, 4, 8, 16, 32):
            A = oracle.region_align_for(G)      # the geometry the library gives a |g| table
            c = oracle.physical_capacity(int(math.ceil(n / alpha)), A)
            r = oracle.Replay(c, G, align=A)
            r.insert(keys, vals)
            st_hit = oracle._Stats()
            r.query(keys[::4], st_hit)  # spread over insertion order
            st_miss = oracle._Stats()
            r.query(absent, st_miss)
            row = {"alpha": alpha, "G": G, "align": A,
                   "ins_windows": r.ins.windows / n, "ins_sectors": r.ins.sectors / n,
                   "hit_windows": st_hit.windows / st_hit.ops, "hit_sectors": st_hit.sectors / st_hit.ops,
                   "miss_windows": st_miss.windows / st_miss.ops,
                   "miss_sectors": st_miss.sectors / st_miss.ops,
                   "ins_lines": r.ins.lines / n, "hit_lines": st_hit.lines / st_hit.ops,
                   "miss_lines": st_miss.lines / st_miss.ops,
                   "max_ins_windows": int(r.ins.max_windows)}
            out["rows"].append(row)
            print(row, flush=True)
    path = os.path.join(ROOT, "tests", "golden", "probe_cost.json")
    json.dump(out, open(path, "w"), indent=1)
    print("wrote", path)


if __name__ == "__main__":
    main()
