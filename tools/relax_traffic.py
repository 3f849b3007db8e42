"""Relax-phase DRAM traffic per bench step from ncu launch lists of one EAT and one
LD batch (tools/prof_query.py), written to profiles/<round>/relax_traffic_<cfg>.json
for bench.py's roofline "traffic" field.

    ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
        -k regex:"k_eat_(activate|big|chain)" --csv --log-file eat.csv python tools/prof_query.py --problem eat
    (same for ld) ; python tools/relax_traffic.py C2 eat.csv ld.csv profiles/round1
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from launches import load  # noqa: E402

cfg, files, outdir = sys.argv[1], sys.argv[2:-1], sys.argv[-1]
tot_b = tot_t = 0.0
n = 0
for f in files:
    L = load(f)
    for d in L.values():
        tot_b += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
        tot_t += d.get("gpu__time_duration.sum", 0.0)
        n += 1
res = {"config": cfg, "bytes_per_step": tot_b, "kernel_ns_per_step_under_ncu": tot_t, "launches": n,
       "batches": [os.path.basename(f) for f in files],
       "source": "ncu dram__bytes_read.sum + dram__bytes_write.sum over k_eat_(activate|big|chain), "
                 "one EAT and one LD batch of the bench step (cold-cache, serialised replay)"}
os.makedirs(outdir, exist_ok=True)
json.dump(res, open(os.path.join(outdir, f"relax_traffic_{cfg}.json"), "w"), indent=1)
print(res)
