"""Summarise an ncu --csv launch list: per-launch and per-kernel durations/metrics."""
import csv
import sys
from collections import defaultdict


def load(path):
    lines = [l for l in open(path) if l.startswith('"')]
    rows = list(csv.reader(lines))
    hdr = rows[0]
    ii, ki, mi, vi = (hdr.index(x) for x in ("ID", "Kernel Name", "Metric Name", "Metric Value"))
    L = defaultdict(dict)
    for r in rows[1:]:
        i = int(r[ii])
        L[i]["name"] = r[ki]
        try:
            L[i][r[mi]] = float(r[vi].replace(",", ""))
        except ValueError:
            L[i][r[mi]] = r[vi]
    return L


def short(name):
    n = name.split("(")[0]
    return n.replace("void ", "").replace("<unnamed>::", "")[:40]


if __name__ == "__main__":
    L = load(sys.argv[1])
    thr = float(sys.argv[2]) if len(sys.argv) > 2 else 50.0  # us
    tot = defaultdict(lambda: [0, 0.0])
    for i in sorted(L):
        d = L[i]
        t = d.get("gpu__time_duration.sum", 0.0) / 1e3
        k = short(d["name"])
        tot[k][0] += 1
        tot[k][1] += t
        if t > thr:
            extra = {m.split("__")[1][:28]: d[m] for m in d if m not in ("name", "gpu__time_duration.sum")}
            print(f"{i:5d} {k:40s} {t:10.1f} us  {extra}")
    print("--- per kernel (launches, total us)")
    for k, (c, t) in sorted(tot.items(), key=lambda kv: -kv[1][1])[:20]:
        print(f"{k:40s} {c:6d} {t:12.1f}")
