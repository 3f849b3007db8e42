"""Certify every row of the BASELINE configs at full size (EAT / LD) on the device with the
fixpoint + witness + min-id conditions of tests/props.py, in the bench's launch
configuration (64-source sub-batches); writes a JSON summary.

usage: python tools/certify_full.py OUT.json [C2 C3 C4 C5]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import tgsynth  # noqa: E402
from tests import props  # noqa: E402
import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as tg  # noqa: E402
from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph  # noqa: E402

out_path = sys.argv[1]
cfgs = sys.argv[2:] or ["C2", "C3", "C4", "C5"]
summary = {"check": "tests/props.py fixpoint + witness + min-id tie rule, every row", "configs": {}}
for cfg in cfgs:
    t0 = time.time()
    tempgraph.load_library().tg_release_cached_memory()
    torch.cuda.empty_cache()
    ge = tgsynth.make_graph(cfg, device="cuda")
    spec = tgsynth.CONFIGS[cfg]
    weighted = spec["kind"] == "wikitalk"
    if not weighted:
        ge.w = None
    torch.cuda.empty_cache()
    problems = [p for p in spec["problems"] if p in ("eat", "ld")]
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, ge.w, device=0)
    if "ld" not in problems:
        g.set_option("mirror", 0)
    if cfg == "C5":
        g.set_option("partitions", 8)
    g.build()
    srcs = tgsynth.config_sources(cfg, ge, k=4 if cfg == "C5" else None)
    rows = 0
    for win in spec["windows"]:
        for p in problems:
            for b0 in range(0, len(srcs), 64):
                batch = srcs[b0:b0 + 64]
                vals, pred = g.query(p, batch, win, with_pred=True)
                u32 = g.query(p, batch, win)  # the bench path (u32 states, no preds)
                torch.cuda.synchronize()
                assert torch.equal(vals, u32), f"{cfg} {p}: packed and u32-state values differ"
                chk = props.check_eat_row if p == "eat" else props.check_ld_row
                for r, x in enumerate(batch):
                    chk(ge.u, ge.v, ge.t, ge.dur, ge.n, x, win, vals[r], pred[r])
                rows += len(batch)
                del vals, pred, u32
    g.close()
    summary["configs"][cfg] = {"n": ge.n, "m": ge.m, "problems": problems, "windows": spec["windows"],
                               "sources": len(srcs), "rows_certified": rows, "seconds": round(time.time() - t0, 1),
                               "result": "all rows pass"}
    print(cfg, summary["configs"][cfg], flush=True)
    del ge
json.dump(summary, open(out_path, "w"), indent=1)
