"""Diagnostic: query rate and SM clock / power on tables built with flags 3 vs 7."""
import math, os, sys, subprocess, time, threading
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_junger0s18_b200 as wd
import wdgen.gpu as gg
G = int(sys.argv[1]) if len(sys.argv) > 1 else 4
n = 1 << 28
keys, vals = gg.unique_keys(n, 1), gg.values(n, 2)
vo = torch.empty(n, dtype=torch.int32, device="cuda"); fo = torch.empty(n, dtype=torch.uint8, device="cuda")
tabs = {}
for F in (3, 7):
    t = wd.Table(int(math.ceil(n / 0.95)), 1, G)
    t.set_option(wd.WD_OPT_KERNEL_FLAGS, F)
    t.insert(keys, vals)
    tabs[F] = t
torch.cuda.synchronize()
for F in (3, 7, 3, 7):
    p = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=clocks.sm,clocks.mem,power.draw,temperature.gpu,temperature.memory",
                          "--format=csv,noheader,nounits", "-lms", "100"], stdout=subprocess.PIPE, text=True)
    rows = []
    th = threading.Thread(target=lambda: [rows.append(l.strip()) for l in p.stdout], daemon=True); th.start()
    time.sleep(0.3)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(100):
        tabs[F].retrieve(keys, vo, fo)
    b.record(); torch.cuda.synchronize()
    p.terminate(); p.wait()
    print(f"flags={F}: query {a.elapsed_time(b) / 100:.2f} ms; samples {rows[3:8]} ... {rows[-3:]}", flush=True)
