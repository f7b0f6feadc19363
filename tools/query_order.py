"""Diagnostic: does the query rate depend on the query order relative to the insert order?
(Keys inserted concurrently may share lines; querying them concurrently again means
concurrent misses on the same 128-B line.)"""
import math, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
G = int(sys.argv[1]) if len(sys.argv) > 1 else 4
n = 1 << 28
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
g = torch.Generator(device="cuda"); g.manual_seed(7)
perm = torch.randperm(n, device="cuda", generator=g)
orders = {"insert order": keys, "shuffled": keys[perm].contiguous(), "reversed": keys.flip(0).contiguous(),
          "shifted by 2^20": torch.roll(keys, 1 << 20).contiguous()}
def tq(t, q):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t.retrieve(q, vo, fo)
    a.record()
    for _ in range(5):
        t.retrieve(q, vo, fo)
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / 5
for G_ in (G,):
    t = wd.Table(int(math.ceil(n / 0.95)), 1, G)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(); t.insert(keys, vals); b.record(); torch.cuda.synchronize()
    ti = a.elapsed_time(b)
    for QF in (3, 11):   # query without / with the scrambled chunk order (kF_QSCR)
        t.set_option(wd.WD_OPT_KERNEL_FLAGS, QF)
        res = {k: tq(t, q) for k, q in orders.items()}
        print(f"G={G} insert ({ti:.1f} ms), query flags={QF}: " + "  ".join(f"{k}: {v:.2f} ms" for k, v in res.items()), flush=True)
    t.close()
