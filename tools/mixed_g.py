import math, os, sys, json
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
n = 1 << 28
keys, vals = gg.unique_keys(n, 11), gg.values(n, 12)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for gi, gq in ((16, 16), (8, 16), (4, 16)):
    with wd.Table(int(math.ceil(n / 0.95)), 1, 16) as t:
        ti, tq = [], []
        for r in range(4):
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            t.clear(s)
            t.set_option(wd.WD_OPT_GROUP_SIZE, gi)
            a.record(s); t.insert(keys, vals, s); b.record(s)
            t.set_option(wd.WD_OPT_GROUP_SIZE, gq)
            t.retrieve(keys, vo, fo, s); c.record(s)
            torch.cuda.synchronize()
            if r: ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
        assert t.sync() == 0 and t.size() == n
        assert gg.check_unique(keys, vo, fo, n, 11, 12)[0] == 0
        print(json.dumps({"insert_G": gi, "query_G": gq, "align": t.get_option(wd.WD_OPT_REGION_ALIGN),
                          "insert_gops": n / (sum(ti)/len(ti)) / 1e6, "query_gops": n / (sum(tq)/len(tq)) / 1e6,
                          "step_ms": (sum(ti)+sum(tq))/len(ti)}), flush=True)
