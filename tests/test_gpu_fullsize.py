"""BASELINE.json configs at full size, in the launch configuration bench.py times
(64-source sub-batches per rank), certified row by row on the device with the
fixpoint + witness + tie-rule conditions of tests/props.py (which determine EAT / LD
rows uniquely; pinned against the oracle in tests/test_props_cpu.py).  The u32-state
path (no preds, what the bench times) must give the same values as the packed path."""
import pytest

import tgsynth
from tests import props

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


@pytest.fixture(scope="module")
def tg(cuda_ok):
    import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as m
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import _build
    _build.build()
    return m


def _certify(tg, ge, g, srcs, win, problems=("eat", "ld"), rows=None):
    import torch
    for p in problems:
        out, pred = g.query(p, srcs, win, with_pred=True)
        vals = g.query(p, srcs, win)  # bench path: u32 states, no preds
        torch.cuda.synchronize()
        assert torch.equal(out, vals), f"{p}: packed and u32-state values differ"
        for r in (range(len(srcs)) if rows is None else rows):
            chk = props.check_eat_row if p == "eat" else props.check_ld_row
            chk(ge.u, ge.v, ge.t, ge.dur, ge.n, srcs[r], win, out[r], pred[r])
        del out, pred, vals


def test_c2_full_all_rows(tg):
    """configs[1]: all 64 rows of the EAT and LD batches, both windows."""
    ge = tgsynth.make_graph("C2", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0).build()
    srcs = tgsynth.config_sources("C2", ge)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        _certify(tg, ge, g, srcs, win)
    g.close()


def test_c3_full_all_rows(tg):
    """configs[2]: all 16 EAT / LD rows (skewed timestamps, weights given)."""
    ge = tgsynth.make_graph("C3", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, ge.w, device=0).build()
    srcs = tgsynth.config_sources("C3", ge)
    for win in tgsynth.CONFIGS["C3"]["windows"]:
        _certify(tg, ge, g, srcs, win)
    g.close()


def test_c4_full_one_rank_batch(tg):
    """configs[3] (R-MAT 2^24 / 512 M edges): one rank's 64-source EAT batch of the
    1024-source job (rank 0 of 16 blocks), every row certified."""
    import torch
    ge = tgsynth.make_graph("C4", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("mirror", 0)  # EAT only: the mirror is built lazily
    g.build()
    srcs = tgsynth.config_sources("C4", ge)[:64]
    _certify(tg, ge, g, srcs, tgsynth.CONFIGS["C4"]["windows"][0], problems=("eat",))
    g.close()
    del ge
    torch.cuda.empty_cache()


def test_c5_full_vertex_partitioned(tg):
    """configs[4] (Chung-Lu, 41.7 M vertices / 1.47 B edges): the single-source EAT of
    the 8-GPU vertex-range mode, run as 8 logical vertex-range partitions on one GPU
    (same partitioned build and per-round exchange, shared state), certified."""
    import torch
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph
    tempgraph.load_library().tg_release_cached_memory()  # blocks cached by earlier tests
    torch.cuda.empty_cache()
    free, _ = torch.cuda.mem_get_info()
    if free < 150 * (1 << 30):
        pytest.skip(f"needs ~150 GB of free device memory ({free >> 30} GB free)")
    ge = tgsynth.make_graph("C5", device="cuda")
    ge.w = None  # weights unused (EAT); 5.9 GB back before the build
    torch.cuda.empty_cache()
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("partitions", 8)
    g.set_option("mirror", 0)
    g.build()
    srcs = tgsynth.config_sources("C5", ge)
    _certify(tg, ge, g, srcs, tgsynth.CONFIGS["C5"]["windows"][0], problems=("eat",))
    g.close()
    del ge
    torch.cuda.empty_cache()
