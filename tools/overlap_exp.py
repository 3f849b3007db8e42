"""Overlap experiment: two independent graph handles (same edges) answer halves of one
source job concurrently from two host threads on two CUDA streams, against one handle
answering the whole job.  python tools/overlap_exp.py CONFIG K [scale_shift]"""
import os
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as T  # noqa: E402

cfg, k = sys.argv[1], int(sys.argv[2])
shift = int(sys.argv[3]) if len(sys.argv) > 3 else 0
if len(sys.argv) > 4:
    T.load_library(sys.argv[4])
ge = tgsynth.make_graph(cfg, device="cuda", scale_shift=shift)
job = tgsynth.config_sources(cfg, ge, k=k)
win = tgsynth.CONFIGS[cfg]["windows"][0]
gs = []
for i in range(2):
    g = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("mirror", 0)
    g.build()
    gs.append(g)
outs = [torch.empty((k // 2, ge.n), dtype=torch.int32, device="cuda") for _ in range(2)]
out = torch.empty((k, ge.n), dtype=torch.int32, device="cuda")
streams = [torch.cuda.Stream() for _ in range(2)]
# the two halves: interleaved blocks of 64 in schedule order are not known here; halves of
# the caller's order (each handle schedules its own half)
halves = [job[: k // 2], job[k // 2:]]


def one():
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    gs[0].query("eat", job, win, out=out)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1)


def two():
    torch.cuda.synchronize()
    import time
    t0 = time.perf_counter()
    th = []
    for i in range(2):
        def run(i=i):
            with torch.cuda.stream(streams[i]):
                gs[i].query("eat", halves[i], win, out=outs[i], stream=streams[i].cuda_stream)
            streams[i].synchronize()
        th.append(threading.Thread(target=run))
    for t in th:
        t.start()
    for t in th:
        t.join()
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) * 1e3


for rep in range(3):
    a = one()
    b = two()
    print(f"{cfg} shift {shift} k={k}: one handle {a:.1f} ms, two handles concurrently {b:.1f} ms", flush=True)
ok = torch.equal(out[: k // 2], outs[0]) and torch.equal(out[k // 2:], outs[1])
print("rows equal:", ok)
