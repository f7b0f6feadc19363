"""Measurement tool: WD_OPT_SPAN 1 vs 2 (one lane per window) on small and large tables —
device time per insert / retrieve call (host cost hidden behind a GPU sleep) and config 1
(2^20 keys, |g| = 4, 2^21 interleaved queries with half misses).
    python tools/span_bench.py"""
import math
import os
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch  # noqa: E402

import paper_conf_ipps_junger0s18_b200 as wd  # noqa: E402
import wdgen.gpu as gg  # noqa: E402


def run(lg, G, span, mixed=False, reps=5):
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
    q = gg.interleaved_queries(n, 1) if mixed else keys
    vo = torch.empty(q.numel(), dtype=torch.int32, device="cuda")
    fo = torch.empty(q.numel(), dtype=torch.uint8, device="cuda")
    s = torch.cuda.current_stream()
    ti, tq = [], []
    with wd.Table(int(math.ceil(n / 0.95)), 1, G) as t:
        t.set_option(wd.WD_OPT_SPAN, span)
        for r in range(reps + 1):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            t.clear(s)
            torch.cuda._sleep(1_000_000)
            ev[0].record(s); t.insert(keys, vals, s); ev[1].record(s)
            torch.cuda._sleep(1_000_000)
            ev[2].record(s); t.retrieve(q, vo, fo, s); ev[3].record(s)
            torch.cuda.synchronize()
            if r:
                ti.append(ev[0].elapsed_time(ev[1])); tq.append(ev[2].elapsed_time(ev[3]))
        assert t.sync() == 0 and t.size() == n
        assert int(fo.sum().item()) == n
    mi, mq = sum(ti) / len(ti) * 1e3, sum(tq) / len(tq) * 1e3
    return mi, mq, n / mi / 1e3, q.numel() / mq / 1e3


if __name__ == "__main__":
    for lg, mixed in [(16, False), (18, False), (20, False), (20, True), (22, False), (22, True), (26, False)]:
        for G in (1, 2, 4):
            for span in (1, 2):
                a, b, c, d = run(lg, G, span, mixed)
                print(f"n=2^{lg}{' config1-queries' if mixed else ''} G={G} S={span}: insert {a:8.1f} us "
                      f"({c:6.2f} G/s)  retrieve {b:8.1f} us ({d:6.2f} G/s)", flush=True)
