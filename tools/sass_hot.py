"""Hottest SASS instructions of an ncu source page (--print-source sass) CSV:
by warp-stall samples and by L2 sectors."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
i = 0
while i < len(rows) and (not rows[i] or rows[i][0] != "Address"):
    i += 1
hdr = rows[i]
data = [dict(zip(hdr, r)) for r in rows[i + 1:] if len(r) == len(hdr)]


def f(x):
    try:
        return float(x.replace(",", ""))
    except Exception:
        return 0.0


tot_s = sum(f(d["Warp Stall Sampling (All Samples)"]) for d in data)
tot_l2 = sum(f(d["L2 Theoretical Sectors Global"]) for d in data)
print(f"total stall samples {tot_s:.0f}, total L2 theoretical sectors {tot_l2:.3e}")
print("--- by stall samples")
for d in sorted(data, key=lambda d: -f(d["Warp Stall Sampling (All Samples)"]))[:int(sys.argv[2]) if len(sys.argv) > 2 else 20]:
    st = {k[6:]: d[k] for k in d if k.startswith("stall_") and f(d[k]) > 0.05 * f(d["Warp Stall Sampling (All Samples)"])}
    print(f"{d['Address']:>6} {f(d['Warp Stall Sampling (All Samples)'])/tot_s*100:5.1f}%  L2 {f(d['L2 Theoretical Sectors Global']):>12.0f}  {d['Source'][:70]:70s} {st}")
print("--- by L2 sectors")
for d in sorted(data, key=lambda d: -f(d["L2 Theoretical Sectors Global"]))[:15]:
    print(f"{d['Address']:>6} {f(d['L2 Theoretical Sectors Global'])/tot_l2*100:5.1f}%  ideal {f(d['L2 Theoretical Sectors Global Ideal']):>12.0f}  {d['Source'][:80]}")
