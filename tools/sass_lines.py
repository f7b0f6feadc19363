"""Attribute an ncu SASS source page to CUDA source lines (measurement tool).

ncu's `--page source --print-source sass --csv` lists every SASS instruction of a kernel with
its executed-instruction count and stall samples, but not the source line.  nvdisasm -g
prints the line of every instruction offset.  This joins the two:

    python tools/sass_lines.py SOURCE_SASS.csv CUBIN KERNEL_SUBSTRING [top]

and prints, per source line of wd_device.cuh, the share of executed warp instructions and of
stall samples, plus the line text."""
import collections
import csv
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def disasm_lines(cubin, mangled_sub):
    out = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
    secs = re.split(r"\n//-+ \.text\.", out)
    res = {}
    for sec in secs:
        name = sec.split(" ", 1)[0]
        if not all(p in name for p in mangled_sub):
            continue
        cur = None
        m = {}
        for ln in sec.splitlines():
            f = re.search(r'//## File "([^"]+)", line (\d+)', ln)
            if f:
                cur = (os.path.basename(f.group(1)), int(f.group(2)))
                continue
            a = re.match(r"\s+/\*([0-9a-f]{4,})\*/", ln)
            if a:
                m[int(a.group(1), 16)] = cur
        res[name] = m
    return res


def ncu_sections(path):
    rows = list(csv.reader(open(path)))
    secs, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            secs.append(cur)
        elif r and r[0] == "Address":
            cur["hdr"] = r
        elif cur is not None and r:
            cur["rows"].append(r)
    return secs


def main():
    csvp, cubin, ksub = sys.argv[1], sys.argv[2], sys.argv[3]
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    mangled = ksub.split(",")
    dl = disasm_lines(cubin, mangled)
    assert len(dl) == 1, f"{len(dl)} kernels match {mangled}: {list(dl)[:4]}"
    offs = next(iter(dl.values()))
    readable = {"InSoA": "InSoA", "InBucket": "InBucket"}
    want = [k for k in readable if any(k in x for x in mangled)]
    sec = next(s for s in ncu_sections(csvp) if all(w in s["name"] for w in want) and
               ("(bool)1" if "Lb1E" in ksub else "(bool)0") in s["name"])
    h = sec["hdr"]
    ie, smp = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    base = int(sec["rows"][0][0], 16)
    inst, stall = collections.Counter(), collections.Counter()
    for r in sec["rows"]:
        off = int(r[0], 16) - base
        key = offs.get(off)
        inst[key] += float(r[ie] or 0)
        stall[key] += float(r[smp] or 0)
    ti, ts = sum(inst.values()), sum(stall.values())
    src = open(os.path.join(ROOT, "paper_conf_ipps_junger0s18_b200", "csrc", "wd_device.cuh")).read().splitlines()
    print(f"{sec['name'][:100]}\n total warp instructions {ti:.4g}, stall samples {ts:.4g}")
    for key, v in inst.most_common(top):
        text = src[key[1] - 1].strip()[:80] if key and key[0] == "wd_device.cuh" else ""
        print(f"{100 * v / ti:5.1f}% inst {100 * stall[key] / ts:5.1f}% stall  {key}  {text}")


if __name__ == "__main__":
    main()
