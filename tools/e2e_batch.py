"""Measurement tool: the bench's e2e step (pinned host buffers through the C-ABI) split into
its insert and retrieve calls, for several pipeline batch sizes, next to the PCIe copy
time of the same bytes.   python tools/e2e_batch.py [log2 n]"""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
n = 1 << lg
keys, vals = gg.unique_keys(n, 0x5EED), gg.values(n, 0xBEEF)
hk = torch.empty(n, dtype=torch.int32, pin_memory=True); hk.copy_(keys)
hv = torch.empty(n, dtype=torch.int32, pin_memory=True); hv.copy_(vals)
hvo = torch.empty(n, dtype=torch.int32, pin_memory=True)
hfo = torch.empty(n, dtype=torch.uint8, pin_memory=True)
s = torch.cuda.current_stream()
ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
# plain copies of the same bytes
a, b = ev(), ev()
a.record(s); keys.copy_(hk, non_blocking=True); vals.copy_(hv, non_blocking=True); b.record(s)
torch.cuda.synchronize()
print(f"H2D 8n = {8 * n / 1e9:.2f} GB: {a.elapsed_time(b):.2f} ms", flush=True)
for lb in (20, 21, 22, 23, 24, 25):
    with wd.Table(int(math.ceil(n / 0.95)), 1, 16, batch=1 << lb) as t:
        ti, tq = [], []
        for r in range(4):
            e = [ev() for _ in range(3)]
            t.clear(s)
            e[0].record(s); t.insert(hk, hv, s); e[1].record(s); t.retrieve(hk, hvo, hfo, s); e[2].record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(e[0].elapsed_time(e[1])); tq.append(e[1].elapsed_time(e[2]))
        assert t.sync() == 0 and t.size() == n
    mi, mq = sum(ti) / len(ti), sum(tq) / len(tq)
    print(f"batch 2^{lb}: insert {mi:7.2f} ms  retrieve {mq:7.2f} ms  step {mi + mq:7.2f} ms "
          f"({2 * n / (mi + mq) / 1e6:.2f} G ops/s)", flush=True)
