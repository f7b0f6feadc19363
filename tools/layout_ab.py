"""Diagnostic: why do queries run faster on a table built with the speculative insert
(flags 7) than on one built with flags 3?  Two tables alive at once; compare layouts and
query times, then rebuild table B with flags 3 and re-time."""
import math, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 28
G = int(sys.argv[2]) if len(sys.argv) > 2 else 4
n = 1 << lg
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
cap = int(math.ceil(n / 0.95))

def tq(t, what):
    ts = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s); t.retrieve(keys, vo, fo, s); b.record(s); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print(f"{what}: query ms {['%.2f' % x for x in ts]}", flush=True)

def ins(t, flags, what):
    t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t.clear(s); a.record(s); t.insert(keys, vals, s); b.record(s); torch.cuda.synchronize()
    print(f"{what}: insert flags={flags} {a.elapsed_time(b):.2f} ms", flush=True)

A = wd.Table(cap, 1, G); B = wd.Table(cap, 1, G)
ins(A, 3, "A"); ins(B, 7, "B")
tq(A, "A(3)"); tq(B, "B(7)"); tq(A, "A(3)"); tq(B, "B(7)")
da, db = A.dump(), B.dump()
print(f"layout: identical slots {np.mean(da == db):.6f}", flush=True)
del da, db
ins(B, 3, "B"); tq(B, "B(3)")
ins(A, 7, "A"); tq(A, "A(7)")
ins(A, 5, "A"); tq(A, "A(5: spec, no L1)")
ins(A, 6, "A"); tq(A, "A(6: spec+xchg, no L1)")
ins(A, 2, "A"); tq(A, "A(2)")
