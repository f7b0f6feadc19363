"""Scaling efficiency per eq. 4 of the paper from bench.py JSON lines.

    E_s(n, m) = tau(n, 1) / (m tau(n, m))        strong: n pairs in total (bench.py --strong)
    E_w(n, m) = tau(n, 1) / tau(m n, m)          weak:   n pairs per GPU (bench.py default)

With value = ops / tau (ops = 2 x pairs: insert + retrieve), both reduce to
E(m) = value(m) / (m value(1)).  Lines are grouped by their "scaling" field; the insert and
query rates get their own efficiencies.

    python tools/scaling.py SCALE.json [more.json ...]
"""
import json
import sys


def efficiencies(lines):
    out = {}
    for kind in ("weak", "strong"):
        runs = {d["n_gpus"]: d for d in lines if d.get("scaling") == kind and "impl" not in d}
        if 1 not in runs:
            continue
        base = runs[1]
        out[kind] = {m: {k: d[k] / (m * base[k]) for k in ("value", "insert_gops", "query_gops")
                         if k in d and k in base}
                     for m, d in sorted(runs.items())}
    return out


def main(paths):
    lines = []
    for p in paths:
        for line in open(p):
            line = line.strip()
            if line.startswith("{"):
                d = json.loads(line)
                if "metric" in d and "n_gpus" in d:
                    lines.append(d)
    for kind, rows in efficiencies(lines).items():
        print(f"{kind} scaling (eq. 4): " + ", ".join(
            f"m={m}: E={r['value']:.3f} (insert {r.get('insert_gops', float('nan')):.3f}, "
            f"query {r.get('query_gops', float('nan')):.3f})" for m, r in rows.items()))


if __name__ == "__main__":
    main(sys.argv[1:])
