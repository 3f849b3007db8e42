"""Profiling driver: build a config graph once and run query batches (for ncu).

    python tools/prof_query.py --config C2 --problem eat --k 64 --reps 1
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--problem", default="eat")
ap.add_argument("--k", type=int, default=64)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--sub-batch", type=int, default=0)
ap.add_argument("--shortcuts", type=int, default=1)
ap.add_argument("--walk-min", type=int, default=0)
ap.add_argument("--relabel", type=int, default=0)
ap.add_argument("--stats", type=int, default=0)
ap.add_argument("--lib", default="")
ap.add_argument("--opt", action="append", default=[], help="key=value library option")
a = ap.parse_args()
if a.lib:
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as _T
    _T.load_library(a.lib)

ge = tgsynth.make_graph(a.config, device="cuda")
cfg = tgsynth.CONFIGS[a.config]
w = ge.w if cfg["kind"] == "wikitalk" else None
g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, w, device=0)
g.set_option("relabel", a.relabel)
if a.problem != "ld":
    g.set_option("mirror", 0)
if a.walk_min:
    g.set_option("walk_min", a.walk_min)
g.build()
if a.sub_batch:
    g.set_option("sub_batch", a.sub_batch)
g.set_option("shortcuts", a.shortcuts)
g.set_option("stats", a.stats)
for kv in a.opt:
    g.set_option(kv.split("=")[0], int(kv.split("=")[1]))
src = tgsynth.config_sources(a.config, ge, k=a.k)
win = cfg["windows"][0]
out = torch.empty((len(src), ge.n), dtype=torch.int32, device="cuda")
for i in range(a.reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    g.query(a.problem, src, win, out=out)
    torch.cuda.synchronize()
    print(f"rep {i}: {(time.perf_counter() - t0) * 1e3:.2f} ms  stats={g.last_stats()}", flush=True)
