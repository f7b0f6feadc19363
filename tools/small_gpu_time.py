"""Measurement tool: device time of one insert / retrieve call on small (L2-resident)
tables, with the host-side cost of the call hidden behind a GPU sleep queued first
(torch.cuda._sleep), next to the plain event timing that includes it.

    python tools/small_gpu_time.py [log2 n ...]
"""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402


def run(lg, G, hide):
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    ti, tq = [], []
    with wd.Table(int(math.ceil(n / 0.95)), 1, G) as t:
        for r in range(6):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            t.clear(s)
            if hide:
                torch.cuda._sleep(2_000_000)
            ev[0].record(s)
            t.insert(keys, vals, s)
            ev[1].record(s)
            if hide:
                torch.cuda._sleep(2_000_000)
            ev[2].record(s)
            t.retrieve(keys, vo, fo, s)
            ev[3].record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(ev[0].elapsed_time(ev[1]))
                tq.append(ev[2].elapsed_time(ev[3]))
        assert t.sync() == 0 and t.size() == n
    mi, mq = sum(ti) / len(ti), sum(tq) / len(tq)
    return mi * 1e3, mq * 1e3, n / mi / 1e6, n / mq / 1e6


if __name__ == "__main__":
    for lg in [int(x) for x in sys.argv[1:]] or [16, 18, 20, 22]:
        for G in (4, 8, 16):
            for hide in (False, True):
                a, b, c, d = run(lg, G, hide)
                print(f"n=2^{lg} G={G} {'device-only' if hide else 'with host'}: insert {a:8.1f} us "
                      f"({c:5.2f} G/s)  retrieve {b:8.1f} us ({d:5.2f} G/s)", flush=True)
