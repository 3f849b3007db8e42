"""Build-phase timing of one library variant: create + build_chains (fwd + mirror) from
device-resident edges, median of 7 after 2 warm-ups (CUDA events), plus per-kernel totals
of one build (in-library event profiling).  --check compares the chain export with the
default library's.

usage: python tools/build_bench.py LIB.so [CONFIG] [--check]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tgsynth  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as T  # noqa: E402

lib = sys.argv[1]
args = [a for a in sys.argv[2:] if not a.startswith("--")]
cfg = args[0] if args else "C2"
T.load_library(lib)
ge = tgsynth.make_graph(cfg, device="cuda")
torch.cuda.synchronize()
ts = []
for it in range(9):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if it == 8:
        T.tg_profile_enable(True)
    e0.record()
    g = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.build()
    e1.record()
    torch.cuda.synchronize()
    if it >= 2 and it < 8:
        ts.append(e0.elapsed_time(e1))
    if it == 8:
        r = T.tg_profile_report()
        top = sorted(r.items(), key=lambda kv: -kv[1][1])[:8]
        print("  kernels:", ", ".join(f"{k} {v[1]:.3f}" for k, v in top))
    if it < 8:
        g.close()
print(f"{os.path.basename(lib)} {cfg} build (create + fwd + mirror): median {statistics.median(ts):.3f} ms "
      f"min {min(ts):.3f} ms", flush=True)
if "--check" in sys.argv:
    import hashlib
    h = hashlib.sha1()
    for mir in (False, True):
        ex = g.export_chains(mirrored=mir)
        for key in sorted(ex):
            h.update(np.ascontiguousarray(ex[key]).tobytes())
    print("  chain export digest:", h.hexdigest())
