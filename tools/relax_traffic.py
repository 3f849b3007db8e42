"""Fold an ncu --csv launch log of the relax kernels (gpu__time_duration, dram bytes) of one
64-source query into profiles/round2/relax_traffic_<CFG>.json, the `traffic` of bench.py's
roofline: DRAM bytes per bench step = per-query bytes x queries per step / 64.

usage: python tools/relax_traffic.py LOG.csv CFG CALLS_PER_STEP [K]"""
import collections
import csv
import json
import os
import sys

log, cfg, per_step = sys.argv[1], sys.argv[2], float(sys.argv[3])
kq = int(sys.argv[4]) if len(sys.argv) > 4 else 64
rows = [r for r in csv.reader(open(log)) if len(r) > 10]
hdr = rows[0]
ix = {k: i for i, k in enumerate(hdr)}
acc = collections.defaultdict(lambda: collections.Counter())
for r in rows[1:]:
    if r[ix["Metric Name"]] not in ("gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum"):
        continue
    name = r[ix["Kernel Name"]].split("(")[0].replace("void ", "").replace("<unnamed>::", "")
    unit = r[ix["Metric Unit"]]
    v = float(r[ix["Metric Value"]].replace(",", ""))
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-6, "usecond": 1e-3, "ns": 1e-6, "us": 1e-3, "ms": 1.0,
             "msecond": 1.0}.get(unit, 1.0)
    key = r[ix["Metric Name"]]
    acc[name][key] += v * scale
    if key == "gpu__time_duration.sum":
        acc[name]["launches"] += 1
tot = collections.Counter()
for k in acc.values():
    tot.update(k)
dram = tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]
out = {
    "config": cfg,
    "dram_bytes_per_subbatch": dram,
    "dram_bytes_per_step": dram * per_step,
    "ncu_ms_per_subbatch": tot["gpu__time_duration.sum"],
    "ncu_GBps": dram / (tot["gpu__time_duration.sum"] / 1e3) / 1e9 if tot["gpu__time_duration.sum"] else None,
    "per_kernel": {k: {"launches": int(v["launches"]), "ms": round(v["gpu__time_duration.sum"], 3),
                       "dram_GB": round((v["dram__bytes_read.sum"] + v["dram__bytes_write.sum"]) / 1e9, 3)}
                   for k, v in acc.items()},
    "source": (f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum over every "
               f"k_eat_(activate|big|chain) launch of one {kq}-source EAT call (tools/prof_query.py --config {cfg} "
               f"--k {kq}), serialised cold-cache replay; x{per_step:g} such calls per bench step"),
}
dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "round2",
                   f"relax_traffic_{cfg}.json")
json.dump(out, open(dst, "w"), indent=1)
print(json.dumps(out, indent=1))
