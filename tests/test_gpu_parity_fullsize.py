"""BASELINE.json configs at full size, in the launch configuration bench.py times
(64-source sub-batches per rank), certified row by row on the device with the
fixpoint + witness + tie-rule conditions of tests/props.py (which determine EAT / LD
rows uniquely; pinned against the oracle in tests/test_props_cpu.py).  The u32-state
path (no preds, what the bench times) must give the same values as the packed path."""
import numpy as np
import pytest

import oracle
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
    win = tgsynth.CONFIGS["C5"]["windows"][0]
    _certify(tg, ge, g, srcs, win, problems=("eat",))
    g.close()
    # the cross-rank algorithm (private state per partition, min exchange every round,
    # frontier from the exchanged state): the max-degree source's row element by element
    # against the oracle, values and preds
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("partitions", 8)
    g.set_option("exchange", 1)
    g.set_option("mirror", 0)
    g.build()
    out, pred = g.query("eat", srcs[:1], win, with_pred=True)
    out, pred = tg.as_u32(out)[0], tg.as_u32(pred)[0]
    g.close()
    n, u, v, t, d, _ = ge.numpy()
    del ge
    torch.cuda.empty_cache()
    A, P, _ = oracle.eat(oracle.Graph(n, u, v, t, d), srcs[0], *win)
    np.testing.assert_array_equal(out, A)
    np.testing.assert_array_equal(pred, P)


def test_c4_rows_vs_oracle(tg):
    """configs[3] at full size in the bench's launch configuration (u32 states, 64-source
    sub-batch): two rows element by element against the oracle."""
    import torch
    ge = tgsynth.make_graph("C4", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0)
    g.set_option("mirror", 0)
    g.build()
    srcs = tgsynth.config_sources("C4", ge)[:64]
    win = tgsynth.CONFIGS["C4"]["windows"][0]
    out = tg.as_u32(g.query("eat", srcs, win))
    g.close()
    n, u, v, t, d, _ = ge.numpy()
    del ge
    torch.cuda.empty_cache()
    og = oracle.Graph(n, u, v, t, d)
    for r in (0, 63):
        np.testing.assert_array_equal(out[r], oracle.eat(og, srcs[r], *win)[0], err_msg=f"C4 row {r}")


def test_c2_weighted_sp_fp_sampled(tg):
    """SP / FP / LDS on a high-reach graph at full C2 size (16.8 M edges, w ~ U[1,100]):
    sampled rows of a 4-source batch element by element against the oracle."""
    ge = tgsynth.make_graph("C2", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, ge.w, device=0)
    g.set_option("mirror", 0)
    g.build()
    srcs = tgsynth.config_sources("C2", ge)[:4]
    win = tgsynth.CONFIGS["C2"]["windows"][1]
    rows = {p: tg.as_u32(g.query(p, srcs, win)) for p in ("sp", "fp", "lds")}
    g.close()
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d, w)
    for r in (0, 3):
        np.testing.assert_array_equal(rows["sp"][r], oracle.sp(og, srcs[r], *win), err_msg=f"SP row {r}")
        np.testing.assert_array_equal(rows["fp"][r], oracle.fp(og, srcs[r], *win), err_msg=f"FP row {r}")
        np.testing.assert_array_equal(rows["lds"][r], oracle.lds(og, srcs[r], *win), err_msg=f"LDS row {r}")


def test_c2_streamed_full(tg):
    """configs[1] as an out-of-memory graph (8 time blocks of ~2.1 M edges streamed from
    host memory): the bench's 64-source EAT batch equals the device-resident graph's."""
    import torch
    ge = tgsynth.make_graph("C2", device="cuda")
    srcs = tgsynth.config_sources("C2", ge)
    win = tgsynth.CONFIGS["C2"]["windows"][0]
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0).build()
    ref = g.query("eat", srcs, win)
    g.close()
    hu, hv, ht, hd = (x.cpu() for x in (ge.u, ge.v, ge.t, ge.dur))
    gs = tg.Graph(ge.n, hu, hv, ht, hd, None, device=0, block_edges=ge.m // 8 + 1).build()
    assert gs.info()["n_blocks"] >= 8
    out = gs.query("eat", srcs, win)
    torch.cuda.synchronize()
    assert torch.equal(out, ref)
    gs.close()
