"""Query-only timing of FP / SP batches on one config for one library build.
usage: python tools/spfp_bench.py LIB.so [CONFIG] [k]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as T  # noqa: E402

lib = sys.argv[1]
cfg = sys.argv[2] if len(sys.argv) > 2 else "C3"
k = int(sys.argv[3]) if len(sys.argv) > 3 else 16
T.load_library(lib)
ge = tgsynth.make_graph(cfg, device="cuda")
src = tgsynth.config_sources(cfg, ge, k=k)
w = ge.w if tgsynth.CONFIGS[cfg]["kind"] == "wikitalk" else None
g = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, w, device=0).build()
out = torch.empty((k, ge.n), dtype=torch.int32, device="cuda")
win = tgsynth.CONFIGS[cfg]["windows"][0]
for p in ("fp", "sp"):
    ts = []
    for it in range(7):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        g.query(p, src, win, out=out)
        e1.record()
        torch.cuda.synchronize()
        if it >= 2:
            ts.append(e0.elapsed_time(e1))
    print(f"{os.path.basename(lib)} {cfg} k={k} {p}: median {statistics.median(ts):.3f} ms checksum "
          f"{int(out.to(torch.int64).sum())}", flush=True)
