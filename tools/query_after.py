"""Diagnostic driver for ncu: build a 2^28 table with kernel flags F, then retrieve all keys twice."""
import math, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
F = int(sys.argv[1]); G = int(sys.argv[2]) if len(sys.argv) > 2 else 4
n = 1 << 28
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
t = wd.Table(int(math.ceil(n / 0.95)), 1, G)
t.set_option(wd.WD_OPT_KERNEL_FLAGS, F)
t.insert(keys, vals)
for _ in range(2):
    t.retrieve(keys, vo, fo)
torch.cuda.synchronize()
