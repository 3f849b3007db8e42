"""Which phase of the bench step carries the occasional slow steps?  (diagnostic)

Runs the C2 bench step (create, build, 64 EAT, 64 LD, close) 200 times with a
synchronize after each phase and prints, per phase, the median and the five worst
wall times, plus the steps whose total exceeds 1.25x the median.
"""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 200
ge = tgsynth.make_graph(cfg, device="cuda")
src = tgsynth.config_sources(cfg, ge, k=64)
outs = {p: torch.empty((64, ge.n), dtype=torch.int32, device="cuda") for p in ("eat", "ld")}
phases = {k: [] for k in ("create", "build", "eat", "ld", "close", "total")}
torch.cuda.synchronize()
for it in range(iters):
    t = [time.perf_counter()]
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    torch.cuda.synchronize(); t.append(time.perf_counter())
    g.build()
    torch.cuda.synchronize(); t.append(time.perf_counter())
    g.query("eat", src, (0, tg.TG_TMAX), out=outs["eat"])
    torch.cuda.synchronize(); t.append(time.perf_counter())
    g.query("ld", src, (0, tg.TG_TMAX), out=outs["ld"])
    torch.cuda.synchronize(); t.append(time.perf_counter())
    g.close()
    torch.cuda.synchronize(); t.append(time.perf_counter())
    for i, k in enumerate(("create", "build", "eat", "ld", "close")):
        phases[k].append((t[i + 1] - t[i]) * 1e3)
    phases["total"].append((t[-1] - t[0]) * 1e3)
rep = {}
for k, v in phases.items():
    v2 = v[10:]
    rep[k] = {"median": round(statistics.median(v2), 3), "worst": [round(x, 2) for x in sorted(v2)[-5:]]}
med = statistics.median(phases["total"][10:])
slow = [i for i, x in enumerate(phases["total"]) if i >= 10 and x > 1.25 * med]
rep["slow_steps"] = [{k: round(phases[k][i], 2) for k in phases} for i in slow[:12]]
rep["n_slow"] = len(slow)
print(json.dumps(rep))
