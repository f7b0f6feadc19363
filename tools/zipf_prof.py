import math, os, sys
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, R)
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
n = 1 << int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 25
G = int(sys.argv[2]) if len(sys.argv) > 2 else 4
mode = int(sys.argv[3]) if len(sys.argv) > 3 else 0
keys = gg.zipf_keys(n, 2**32 - 1, 5); vals = gg.values(n, 6)
distinct = int(torch.unique(keys).numel())
t = wd.Table(int(math.ceil(distinct / 0.95)), 1, G)
t.set_option(wd.WD_OPT_PROBE_MODE, mode)
s = torch.cuda.current_stream()
for it in range(2):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t.clear(s); a.record(s); t.insert(keys, vals, s); b.record(s); torch.cuda.synchronize()
    print(f"n={n} distinct={distinct} G={G} mode={mode}: insert {n / a.elapsed_time(b) / 1e6:.3f} G/s", flush=True)
