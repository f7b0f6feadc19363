"""Per-call DRAM traffic and launch shares from an ncu launch list of bench.py
(--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum).

A bench step is fill_kernel, the insert call (one probe launch, or for a slice-grouped
insert: per chunk a histogram, a scan, the multisplit and one probe launch per slice), then
the retrieve probe launch.  Writes profiles/traffic.json entries per CALL (read + write
bytes, mean over the steps in the list) and prints the kernels' shares of the step time.

    python tools/traffic_per_call.py launches.csv G [alpha] [log2n]"""
import collections
import csv
import json
import os
import sys

path, G = sys.argv[1], int(sys.argv[2])
alpha = float(sys.argv[3]) if len(sys.argv) > 3 else 0.95
lg = int(sys.argv[4]) if len(sys.argv) > 4 else 28
rows = list(csv.reader(open(path)))
hdr, recs = None, collections.OrderedDict()
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        key = (d["ID"], d["Kernel Name"])
        recs.setdefault(key, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
kern = [(name, m) for (_, name), m in recs.items()]
steps, cur, phase = [], None, None
for name, m in kern:
    if name.startswith("wd::fill_kernel"):
        cur = {"insert": [], "retrieve": [], "fill": [(name, m)]}
        steps.append(cur)
        phase = "insert"
        continue
    if cur is None or not name.startswith(("wd::", "void wd::")):
        continue
    if "probe_kernel" in name and ", 0, " in name.split("<", 1)[1].split(">")[0] + ", ":
        cur["retrieve"].append((name, m))
        phase = "done"
    elif phase == "insert":
        cur["insert"].append((name, m))
steps = [s for s in steps if s["insert"] and s["retrieve"]]
out_path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
out = json.load(open(out_path)) if os.path.exists(out_path) else {}
tot = collections.Counter()
for call in ("insert", "retrieve"):
    b = [sum(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0) for _, m in s[call]) for s in steps]
    t = [sum(m["gpu__time_duration.sum"] for _, m in s[call]) for s in steps]
    out[f"{call}_G{G}_a{alpha}_n{lg}"] = sum(b) / len(b)
    bp = [sum(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
              for name, m in s[call] if "probe_kernel" in name) for s in steps]
    out[f"{call}_probe_G{G}_a{alpha}_n{lg}"] = sum(bp) / len(bp)   # the probe launches only
    print(f"{call}: {len(steps)} steps, {sum(len(s[call]) for s in steps) / len(steps):.0f} launches/call, "
          f"{sum(t) / len(t) / 1e6:.2f} ms, {sum(b) / len(b) / 1e9:.2f} GB DRAM per call")
for s in steps:
    for call in ("fill", "insert", "retrieve"):
        for name, m in s[call]:
            short = name.split("(")[0].replace("void ", "")
            tot[short] += m["gpu__time_duration.sum"]
allt = sum(tot.values())
for k, v in tot.most_common():
    print(f"  {k:70s} {v / len(steps) / 1e6:8.3f} ms/step  {100 * v / allt:5.1f} %")
out["_source"] = ("ncu launch list of bench.py (gpu__time_duration, dram__bytes_read/write per "
                  "launch), summed per call: tools/traffic_per_call.py")
json.dump(out, open(out_path, "w"), indent=1)
