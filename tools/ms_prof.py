"""Measurement tool: one loopback cascade insert + retrieve (m shards on one GPU) for ncu
captures of the exchange kernels (multisplit / unpermute).
    python tools/ms_prof.py [log2 n] [m] [log2 batch]"""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
m = int(sys.argv[2]) if len(sys.argv) > 2 else 8
lb = int(sys.argv[3]) if len(sys.argv) > 3 else 24
n = 1 << lg
keys, vals = gg.unique_keys(n, 3), gg.values(n, 4)
with wd.Table(int(math.ceil(n / 0.95)), group_size=16, loopback_shards=m, batch=1 << lb) as t:
    for _ in range(2):
        t.clear()
        t.insert(keys, vals)
        v, f = t.retrieve(keys)
    torch.cuda.synchronize()
    assert t.sync() == 0 and t.size() == n and bool((f == 1).all())
print("ok")
