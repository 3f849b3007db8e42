"""Wall-clock breakdown of one bench step (create / build / queries / destroy)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import tgsynth  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
ge = tgsynth.make_graph(cfg, device="cuda")
src = tgsynth.config_sources(cfg, ge, k=64)
out = torch.empty((64, ge.n), dtype=torch.int32, device="cuda")
hu, hv, ht, hd = (x.cpu().pin_memory() for x in (ge.u, ge.v, ge.t, ge.dur))
prof = len(sys.argv) > 2
for mode in ("device", "host", "device"):
    for it in range(3):
        if prof:
            tg.tg_profile_enable(True)
        arrs = (ge.u, ge.v, ge.t, ge.dur) if mode == "device" else (hu, hv, ht, hd)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        g = tg.Graph(ge.n, *arrs, None, device=0)
        torch.cuda.synchronize(); t1 = time.perf_counter()
        g.build()
        torch.cuda.synchronize(); t2 = time.perf_counter()
        g.query("eat", src, (0, tg.TG_TMAX), out=out)
        torch.cuda.synchronize(); t3 = time.perf_counter()
        g.query("ld", src, (0, tg.TG_TMAX), out=out)
        torch.cuda.synchronize(); t4 = time.perf_counter()
        g.close()
        torch.cuda.synchronize(); t5 = time.perf_counter()
        print(f"{mode:6s} it{it}: create {1e3*(t1-t0):7.1f} build {1e3*(t2-t1):7.1f} (lib {g.info() if False else ''}) "
              f"eat {1e3*(t3-t2):6.1f} ld {1e3*(t4-t3):6.1f} destroy {1e3*(t5-t4):6.1f} ms", flush=True)
        if prof:
            r = tg.tg_profile_report()
            print("   kernels ms:", round(sum(v[1] for v in r.values()), 2), "launches", sum(v[0] for v in r.values()))
