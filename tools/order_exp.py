"""Experiment: does the composition of the 64-query sub-batches matter?  Times the C4
1024-source EAT job (query only, CUDA events) with the sources in the job's order and
sorted by a per-source key (out-degree descending / ascending, first departure time).

usage: python tools/order_exp.py [CONFIG] [k]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
k = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
ge = tgsynth.make_graph(cfg, device="cuda")
job = tgsynth.config_sources(cfg, ge, k=k)
deg = torch.bincount(ge.u.long(), minlength=ge.n)
tmin = torch.full((ge.n,), 2**31 - 1, dtype=torch.int64, device="cuda").scatter_reduce(
    0, ge.u.long(), ge.t.long(), reduce="amin")
src = torch.tensor(job, device="cuda")
orders = {
    "job": job,
    "deg_desc": [job[i] for i in torch.argsort(-deg[src], stable=True).tolist()],
    "deg_asc": [job[i] for i in torch.argsort(deg[src], stable=True).tolist()],
    "tmin_asc": [job[i] for i in torch.argsort(tmin[src], stable=True).tolist()],
}
g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
g.set_option("mirror", 0)
g.build()
out = torch.empty((k, ge.n), dtype=torch.int32, device="cuda")
win = tgsynth.CONFIGS[cfg]["windows"][0]
for name, srcs in orders.items():
    ts = []
    for rep in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        g.query("eat", srcs, win, out=out)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{cfg} k={k} order={name}: {min(ts):.1f} ms (reps {[round(x, 1) for x in ts]})", flush=True)
