"""Time the config's whole source job (query only, CUDA events, best of 3) for several
libraries / options: python tools/job_exp.py CONFIG K LIB[:opt=val,...] ..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph as T  # noqa: E402

cfg, k = sys.argv[1], int(sys.argv[2])
ge = tgsynth.make_graph(cfg, device="cuda")
job = tgsynth.config_sources(cfg, ge, k=k)
win = tgsynth.CONFIGS[cfg]["windows"][0]
out = torch.empty((k, ge.n), dtype=torch.int32, device="cuda")
for spec in sys.argv[3:]:
    lib, _, opts = spec.partition(":")
    T._lib = None
    T.load_library(lib)
    g = T.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("mirror", 0)
    for kv in filter(None, opts.split(",")):
        kk, vv = kv.split("=")
        g.set_option(kk, int(vv))
    g.build()
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        g.query("eat", job, win, out=out)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{cfg} k={k} {os.path.basename(lib)} {opts or '-'}: {min(ts):.1f} ms ({k / min(ts) * 1e3:.1f} q/s)", flush=True)
    g.close()
    T.tg_release_cached_memory()  # this library's block cache (the next library has its own)
    torch.cuda.empty_cache()
