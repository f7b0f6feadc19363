"""Capacity sweep without the key-space saturation of tools/size_sweep.py:
random unique keys (generator subsets) at a FIXED load alpha = 0.5 from 2^25 to 2^31 keys, i.e.
tables of 0.5 GB to 34 GB, so no point contains most of the 4-byte key space (at most 50 %).
Insert / retrieve rates per size; every query checked against the closed form on the device.
    python tools/size_sweep2.py [G] [alpha]"""
import json, math, os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402
import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402

G = int(sys.argv[1]) if len(sys.argv) > 1 else 16
alpha = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
for lg in (25, 27, 28, 29, 30, 31):
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 11), gg.values(n, 12)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
        ti, tq = [], []
        for r in range(3):
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t.clear(s); a.record(s); t.insert(keys, vals, s); b.record(s); t.retrieve(keys, vo, fo, s); c.record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
        assert t.sync() == 0 and t.size() == n
        bad, first, found = gg.check_unique(keys, vo, fo, n, 11, 12)
        print(json.dumps({"n_log2": lg, "G": G, "alpha": alpha, "table_GB": t.capacity() * 8 / 1e9,
                          "key_space_fraction": n / 2**32,
                          "insert_gops": n / (sum(ti) / len(ti)) / 1e6,
                          "query_gops": n / (sum(tq) / len(tq)) / 1e6, "every_query_ok": bad == 0}), flush=True)
    del keys, vals, vo, fo
    torch.cuda.empty_cache()
