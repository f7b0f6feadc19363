"""Probe accounting under concurrency vs the sequential Fig. 3 replay (measurement tool).

Builds (once) a -DWD_COUNT_PROBES variant of the library into build/count/ and runs, for
the config-2 grid (2^28 keys by default, alpha x |g|): one bulk insert (slice-grouped like the
bench), one retrieve of all keys (hits) and one of 2^26 absent keys (misses).  Reports
windows, distinct 128-B lines and CAS per op next to the replay's figures
(tests/golden/probe_cost.json, written by tools/probe_cost.py from the oracle's replay).

    python tools/probe_counts.py [LOG2N]       # one JSON line per (alpha, |g|)
"""
import json
import math
import os
import subprocess
import sys

R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(R, "build", "count", "libwarpdrive.so")


def build():
    if os.path.exists(LIB):
        return
    import importlib.util
    spec = importlib.util.spec_from_file_location("_b", os.path.join(R, "paper_conf_ipps_junger0s18_b200", "build.py"))
    b = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(b)
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    from concurrent.futures import ThreadPoolExecutor
    objs = [os.path.join(R, "build", "count", u + ".o") for u in b.UNITS]

    def one(uo):
        u, o = uo
        subprocess.check_call([b.NVCC, *b.ARCH, *b.COMMON_C, "-DWD_COUNT_PROBES", "-I",
                               os.path.join(R, "include"), "-c", "-o", o,
                               os.path.join(R, "paper_conf_ipps_junger0s18_b200", "csrc", u + ".cu")])
    with ThreadPoolExecutor(max_workers=os.cpu_count() or 1) as ex:
        list(ex.map(one, zip(b.UNITS, objs)))
    subprocess.check_call([b.NVCC, *b.ARCH, "-shared", "-o", LIB, *objs])


def main():
    lg = int(sys.argv[1]) if len(sys.argv) > 1 and sys.argv[1].isdigit() else 28
    if "--build-only" in sys.argv:
        build()
        return
    build()
    os.environ["WD_LIBRARY"] = LIB
    sys.path.insert(0, R)
    import torch
    import paper_conf_ipps_junger0s18_b200 as wd
    import wdgen.gpu as gg
    gold = json.load(open(os.path.join(R, "tests", "golden", "probe_cost.json")))["rows"]
    n = 1 << lg
    keys, vals = gg.unique_keys(n, 21), gg.values(n, 22)
    miss = gg.unique_keys(n // 4, 21, start=n)
    vo = torch.empty(n, dtype=torch.int32, device="cuda")
    fo = torch.empty(n, dtype=torch.uint8, device="cuda")
    for alpha in (0.8, 0.9, 0.95, 0.99):
        for G in (1, 2, 4, 8, 16, 32):
            with wd.Table(int(math.ceil(n / alpha)), 1, G) as t:
                t.probe_counts()
                t.insert(keys, vals)
                ci = t.probe_counts()
                t.retrieve(keys, vo, fo)
                ch = t.probe_counts()
                t.retrieve(miss, vo[: miss.numel()], fo[: miss.numel()])
                cm = t.probe_counts()
                assert t.sync() == 0 and t.size() == n
                A = t.get_option(wd.WD_OPT_REGION_ALIGN)
            g = min(gold, key=lambda r: (abs(r["alpha"] - alpha), abs(r["G"] - G), abs(r["align"] - A)))
            per = lambda c, k: c[k] / max(c["keys"], 1)   # noqa: E731
            print(json.dumps({
                "n_log2": lg, "alpha": alpha, "G": G, "align": A,
                "insert": {"windows": per(ci, "windows"), "lines": per(ci, "lines"),
                           "cas": per(ci, "cas"), "cas_lost": per(ci, "cas_lost"), "keys": ci["keys"]},
                "hit": {"windows": per(ch, "windows"), "lines": per(ch, "lines"), "keys": ch["keys"]},
                "miss": {"windows": per(cm, "windows"), "lines": per(cm, "lines"), "keys": cm["keys"]},
                "replay": {k: g.get(k) for k in ("ins_windows", "ins_lines", "hit_windows", "hit_lines",
                                                  "miss_windows", "miss_lines", "align")}}), flush=True)


if __name__ == "__main__":
    main()
