import math, os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
n = 1 << 28
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
t = wd.Table(int(math.ceil(n / 0.95)), 1, 8)
s = torch.cuda.current_stream()
def run(ki, kq, reps=4):
    ti, tq = [], []
    for r in range(reps + 1):
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        t.clear(s)
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, ki)
        a.record(s); t.insert(keys, vals, s); b.record(s)
        t.set_option(wd.WD_OPT_KEYS_IN_FLIGHT, kq)
        t.retrieve(keys, vo, fo, s); c.record(s)
        torch.cuda.synchronize()
        if r: ti.append(a.elapsed_time(b)); tq.append(b.elapsed_time(c))
    print(f"insert K={ki}: {n/(sum(ti)/len(ti))/1e6:6.2f}   retrieve K={kq}: {n/(sum(tq)/len(tq))/1e6:6.2f}", flush=True)
for ki, kq in [(4, 4), (2, 4), (0, 0), (2, 2), (4, 4), (2, 4)]:
    run(ki, kq)
