"""Query-only timing of EAT / LD batches on one config for one library build
(tuning experiments: compare -D variants of libtempgraph.so on the same graph).

usage: python tools/variant_bench.py LIB.so [CONFIG] [k] [--pred] [--check]
Prints one line per problem: median ms per batch over 5 runs (CUDA events).
--check compares the outputs against the default library's EAT rows (same graph).
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as T  # noqa: E402

lib = sys.argv[1]
args = [a for a in sys.argv[2:] if not a.startswith("--")]
cfg = args[0] if args else "C2"
k = int(args[1]) if len(args) > 1 else 64
with_pred = "--pred" in sys.argv
opts = {}
for a in sys.argv[2:]:
    if a.startswith("--opt="):  # --opt=key:value
        kk, vv = a[6:].split(":")
        opts[kk] = int(vv)
T.load_library(lib)
ge = tgsynth.make_graph(cfg, device="cuda")
src = tgsynth.config_sources(cfg, ge, k=k)
torch.cuda.synchronize()
torch.cuda.empty_cache()
g = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
for kk, vv in opts.items():
    g.set_option(kk, vv)
g.build()
out = torch.empty((k, ge.n), dtype=torch.int32, device="cuda")
pred = torch.empty((k, ge.n), dtype=torch.int32, device="cuda") if with_pred else None
win = tgsynth.CONFIGS[cfg]["windows"][0]
res = {}
problems = [a[len("--problems="):] for a in sys.argv if a.startswith("--problems=")]
problems = problems[0].split(",") if problems else ["eat", "ld"]
if "ld" not in problems:
    pass
for p in problems:
    ts = []
    for it in range(7):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        if with_pred:
            T.tg_query(g.h, T.PROBLEMS[p], src, win, out, pred)
        else:
            g.query(p, src, win, out=out)
        e1.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    res[p] = (statistics.median(ts), min(ts), out.clone())
    print(f"{os.path.basename(lib)} {cfg} k={k} pred={int(with_pred)} {opts} {p}: median {res[p][0]:.3f} ms "
          f"min {res[p][1]:.3f} ms", flush=True)
if "--check" in sys.argv:
    ref = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    ref.set_option("packed_state", 1)
    ref.build()
    for p in problems:
        o2 = torch.empty_like(out)
        ref.query(p, src, win, out=o2)
        print(f"check {p}: {'OK' if torch.equal(o2, res[p][2]) else 'MISMATCH'} (vs packed-state path)", flush=True)
