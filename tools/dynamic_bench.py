"""Dynamic temporal graphs (§5.6): the cost of a batch of
edge insertions with incremental re-transformation against a from-scratch build of the
same edges, and the SP query after each batch (the paper's Fig. 21 workload shape).

usage: python tools/dynamic_bench.py [CONFIG] [batch] [batches]
Prints one JSON line: per-batch insert+re-transform ms (CUDA events), full-build ms of
the final edge list, and an SP / EAT query time after the last batch."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
batch = int(sys.argv[2]) if len(sys.argv) > 2 else 100_000
nb = int(sys.argv[3]) if len(sys.argv) > 3 else 5
ge = tgsynth.make_graph(cfg, device="cuda")
m0 = ge.m - nb * batch  # the graph before the insertions; the batches are its last edges
u, v, t, d = ge.u, ge.v, ge.t, ge.dur
w = ge.w if tgsynth.CONFIGS[cfg]["kind"] == "wikitalk" else None


def ev():
    return torch.cuda.Event(enable_timing=True)


g = tg.Graph(ge.n, u[:m0], v[:m0], t[:m0], d[:m0], None if w is None else w[:m0], device=0)
g.set_option("dynamic", 1)
g.set_option("mirror", 0)
g.build()
srcs = tgsynth.config_sources(cfg, ge)[:16]
win = tgsynth.CONFIGS[cfg]["windows"][0]
ins_ms = []
for b in range(nb):
    lo, hi = m0 + b * batch, m0 + (b + 1) * batch
    e0, e1 = ev(), ev()
    torch.cuda.synchronize()
    e0.record()
    g.insert_edges(u[lo:hi], v[lo:hi], t[lo:hi], d[lo:hi], None if w is None else w[lo:hi])
    e1.record()
    torch.cuda.synchronize()
    ins_ms.append(e0.elapsed_time(e1))
q = {}
for p in ("eat", "sp"):
    g.query(p, srcs, win)
    e0, e1 = ev(), ev()
    torch.cuda.synchronize()
    e0.record()
    g.query(p, srcs, win)
    e1.record()
    torch.cuda.synchronize()
    q[p] = e0.elapsed_time(e1)
full = []
for _ in range(3):
    e0, e1 = ev(), ev()
    torch.cuda.synchronize()
    e0.record()
    g2 = tg.Graph(ge.n, u, v, t, d, w, device=0)
    g2.set_option("mirror", 0)
    g2.build()
    e1.record()
    torch.cuda.synchronize()
    full.append(e0.elapsed_time(e1))
    g2.close()
print(json.dumps({"config": cfg, "m_final": ge.m, "batch": batch, "batches": nb,
                  "insert_retransform_ms": [round(x, 3) for x in ins_ms],
                  "insert_median_ms": statistics.median(ins_ms[1:] or ins_ms),
                  "full_create_build_ms_median": statistics.median(full),
                  "query_ms_after": {p: round(x, 3) for p, x in q.items()}, "query_sources": len(srcs)}))
