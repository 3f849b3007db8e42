"""Experiment: sub-batch scheduling keys beyond the library's (first departure time >= alpha).
The library's own ordering is switched off (option order_sources = 0) and the job is passed
in each candidate order; query-only CUDA-event timing of the whole job (best of 3).

usage: python tools/order_exp2.py [CONFIG] [k]"""
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
u, t = ge.u.long(), ge.t.long()
n = ge.n
deg = torch.bincount(u, minlength=n).double()
big = 2**40
tmin = torch.full((n,), big, dtype=torch.int64, device="cuda").scatter_reduce(0, u, t, reduce="amin")
tmax = torch.full((n,), -1, dtype=torch.int64, device="cuda").scatter_reduce(0, u, t, reduce="amax")
tsum = torch.zeros(n, dtype=torch.float64, device="cuda").index_add_(0, u, t.double())
tmean = tsum / deg.clamp(min=1)
src = torch.tensor(job, device="cuda")
keys = {
    "tmin": tmin[src].double(),
    "tmin_then_deg": tmin[src].double() * 1e7 - deg[src],
    "tmean": tmean[src],
    "tmin_bucket256_deg": (tmin[src] // 256).double() * 1e7 - deg[src],
    "tmin_plus_gap": tmin[src].double() + (tmax[src] - tmin[src]).double() / deg[src].clamp(min=1),
}
g = tg.Graph(n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
g.set_option("mirror", 0)
g.set_option("order_sources", 0)
g.build()
out = torch.empty((k, n), dtype=torch.int32, device="cuda")
win = tgsynth.CONFIGS[cfg]["windows"][0]
for name, key in keys.items():
    order = torch.argsort(key, stable=True).tolist()
    srcs = [job[i] for i in order]
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        g.query("eat", srcs, win, out=out)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{cfg} k={k} key={name}: {min(ts):.1f} ms", flush=True)
