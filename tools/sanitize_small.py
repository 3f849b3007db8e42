"""Small end-to-end workload for compute-sanitizer (all problems, partitions, host/device buffers)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

ge = tgsynth.make_graph("C1", device="cuda", scale_shift=-3)
for opts in ({}, {"walk_min": 2}, {"partitions": 3}):
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, ge.w, device=0)
    for k, v in opts.items():
        g.set_option(k, v)
    g.build()
    src = list(range(40))
    for p in ("eat", "ld", "reach") + (() if opts.get("partitions") else ("fp", "sp")):
        g.query(p, src, (10, 900))
    if not opts:
        g.query("eat", list(range(64)), (0, 1000))   # u32 states, 64-query extract fast path
        g.query("ld", [5], (0, 1000))                # single-query batch
    host = torch.empty((3, ge.n), dtype=torch.int32)
    tg.tg_query(g.h, tg.TG_EAT, [0, 1, 2], (0, 1000), host)
    g.close()
torch.cuda.synchronize()
print("sanitize workload done")
