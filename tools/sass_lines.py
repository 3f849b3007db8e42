"""Attribute ncu per-SASS-instruction counts (source page CSV, --print-source sass) to
CUDA source lines via nvdisasm line info of the kernel in a cubin.

usage: python tools/sass_lines.py SASS.csv CUBIN KERNEL_SUBSTR [metric]"""
import collections
import csv
import re
import subprocess
import sys

csvp, cubin, ksub = sys.argv[1:4]
metric = sys.argv[4] if len(sys.argv) > 4 else "Instructions Executed"
rows = list(csv.reader(open(csvp)))
i = 0
while i < len(rows) and (not rows[i] or rows[i][0] != "Address"):
    i += 1
hdr = rows[i]
data = []
for r in rows[i + 1:]:
    if r and r[0] in ("Address", "Kernel Name"):
        break  # next kernel section
    if len(r) == len(hdr):
        data.append(dict(zip(hdr, r)))
base = int(data[0]["Address"], 16)


def f(x):
    try:
        return float(x.replace(",", ""))
    except Exception:
        return 0.0


dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
# find function
lines = dis.splitlines()
start = None
for j, l in enumerate(lines):
    if l.startswith(".text.") and ksub in l:
        start = j
        break
if start is None:
    # function labels
    for j, l in enumerate(lines):
        if ksub in l and l.rstrip().endswith(":") and "text" in l:
            start = j
            break
cur = None
off2line = {}
for l in lines[start + 1:]:
    if l.startswith(".text.") or l.startswith("\t.section"):
        break
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (m.group(1).split("/")[-1], int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if m and cur:
        off2line[int(m.group(1), 16)] = cur
agg = collections.Counter()
for d in data:
    off = int(d["Address"], 16) - base
    agg[off2line.get(off, ("?", 0))] += f(d.get(metric, "0"))
tot = sum(agg.values())
print(f"total {metric}: {tot:.4g}")
for (fn, ln), v in agg.most_common(40):
    print(f"{v / tot * 100:5.1f}%  {fn}:{ln}")
