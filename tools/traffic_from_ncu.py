"""Write profiles/traffic.json entries from an `ncu --set full` report of bench.py:
dram__bytes_read.sum + dram__bytes_write.sum per probe-kernel launch (the roofline's
`traffic` field).  Usage: python tools/traffic_from_ncu.py <report.ncu-rep> <G> [alpha] [log2n]"""
import csv
import io
import json
import os
import subprocess
import sys

rep, G = sys.argv[1], int(sys.argv[2])
alpha = float(sys.argv[3]) if len(sys.argv) > 3 else 0.95
lg = int(sys.argv[4]) if len(sys.argv) > 4 else 28
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, data = rows[0], rows[2:]
ki, r, w = hdr.index("Kernel Name"), hdr.index("dram__bytes_read.sum"), hdr.index("dram__bytes_write.sum")
units = rows[1]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
out = json.load(open(path)) if os.path.exists(path) else {}
for d in data:
    name = d[ki]
    op = "insert" if ", (bool)1," in name or ", 1, " in name else "retrieve"
    t = float(d[r]) * scale[units[r]] + float(d[w]) * scale[units[w]]
    out[f"{op}_G{G}_a{alpha}_n{lg}"] = t
    print(op, name[:60], t / 1e9, "GB")
out["_source"] = ("ncu --set full --clock-control none (profiles/r01_ncu_summary.md), "
                  "dram__bytes_read.sum + dram__bytes_write.sum per launch, 2^28 ops")
json.dump(out, open(path, "w"), indent=1)
