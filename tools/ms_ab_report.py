"""Summarise gpurun_out/msab_<lib>.csv launch lists: mean per-launch time (us) and DRAM MB of
the exchange kernels.   python tools/ms_ab_report.py lib ..."""
import collections
import csv
import sys

for l in sys.argv[1:]:
    rows = list(csv.reader(open(f"gpurun_out/msab_{l}.csv")))
    hdr, agg = None, collections.defaultdict(lambda: collections.defaultdict(list))
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            agg[d["Kernel Name"][:30]][d["Metric Name"].split("__")[1][:12]].append(
                float(d["Metric Value"].replace(",", "")))
    print("==", l)
    for k, m in agg.items():
        if "multisplit" in k or "unpermute" in k:
            print(f"  {k:30s} " + " ".join(f"{n}={sum(v) / len(v) / (1e3 if 'time' in n else 1e6):.1f}"
                                           for n, v in m.items()))
