import math, os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg

def fmix32(x):
    x = x.astype(np.uint64)
    x ^= x >> np.uint64(16); x = (x * np.uint64(0x85EBCA6B)) & np.uint64(0xFFFFFFFF)
    x ^= x >> np.uint64(13); x = (x * np.uint64(0xC2B2AE35)) & np.uint64(0xFFFFFFFF)
    x ^= x >> np.uint64(16)
    return x

def stats(t, G):
    d = t.dump()
    c = d.size
    nb = (c - 32) // 4 + 1
    idx = np.nonzero((d & np.uint64(0xFFFFFFFF)) != np.uint64(0xFFFFFFFF))[0].astype(np.uint64)
    k = d[idx] & np.uint64(0xFFFFFFFF)
    b0 = (fmix32(k) * np.uint64(nb)) >> np.uint64(32)
    off = idx.astype(np.int64) - 4 * b0.astype(np.int64)
    inr0 = (off >= 0) & (off < 32)
    win = off[inr0] // G + 1
    return inr0.mean(), win.mean(), (off[inr0] == 0).mean()

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 26
n = 1 << lg
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
for G in (8, 4):
    for flags in (3, 7, 3, 7):
        t = wd.Table(int(math.ceil(n / 0.95)), 1, G)
        t.set_option(wd.WD_OPT_KERNEL_FLAGS, flags)
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        ev[0].record(s); t.insert(keys, vals, s); ev[1].record(s)
        t.retrieve(keys, vo, fo, s); ev[2].record(s); t.retrieve(keys, vo, fo, s); ev[3].record(s)
        torch.cuda.synchronize()
        r0, w, z = stats(t, G)
        print(f"n=2^{lg} G={G} flags={flags}: insert {ev[0].elapsed_time(ev[1]):7.2f} ms  query {ev[1].elapsed_time(ev[2]):6.2f} / {ev[2].elapsed_time(ev[3]):6.2f} ms"
              f"  region0 {r0:.4f}  mean window (region 0) {w:.3f}  at slot 0 of own window seq {z:.3f}", flush=True)
        t.close()
