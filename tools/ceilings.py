"""Write profiles/ceilings.json from a tools/randbench.cu run (profiles/r01_randbench.txt):
the measured random-access rates of this B200 for the probe kernels' own access pattern,
which bench.py turns into a per-op ceiling next to the copy-peak roofline.

    python tools/ceilings.py profiles/r01_randbench.txt

Model: a retrieve that needs L windows costs L independent random window
reads; an insert costs (L - 1) window reads plus one window read followed by a successful
CAS in it (randbench `casw`, the dirty line is written back later).  Rates are for windows
of the headline geometry (|g| = 16, 128-byte windows on 128-byte lines) and for 32/64-byte
windows (|g| = 4/8) in a 2.26 GB buffer (the config-2 table size)."""
import json
import re
import sys

src = sys.argv[1] if len(sys.argv) > 1 else "profiles/r01_randbench.txt"
rx = re.compile(r"^([\d.]+)GB (read|cas|casw)\s+W=\s*(\d+)B align=\s*(\d+)B D=\d+ :\s+([\d.]+) Gwin/s")
out = {"source": src, "buffer_GB": 2.26, "read": {}, "casw": {}}
for line in open(src):
    m = rx.match(line)
    if not m or abs(float(m.group(1)) - 2.26) > 0.01:
        continue
    kind, wb, ab, rate = m.group(2), int(m.group(3)), int(m.group(4)), float(m.group(5))
    if kind in ("read", "casw") and wb == ab:
        out[kind][str(wb)] = rate
json.dump(out, open("profiles/ceilings.json", "w"), indent=1)
print(json.dumps(out))
