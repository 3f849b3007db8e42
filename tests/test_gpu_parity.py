"""GPU parity: the CUDA path (through the C-ABI) against the oracle, element by
element, bit-exact (all quantities are integers).
"""
import json
import os

import numpy as np
import pytest

import oracle
import tgsynth

pytestmark = pytest.mark.gpu

NONE = 0xFFFFFFFF
GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "figure1.json")


@pytest.fixture(scope="module")
def tg(cuda_ok):
    import paper_conf_asplos_0003wh0dhwy0lyl25_b200 as m
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import _build
    _build.build()
    return m


def _gpu_graph(tg, n, u, v, t, lam, w=None, **opts):
    import torch
    f = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).cuda()
    g = tg.Graph(n, f(u), f(v), f(t), f(lam), None if w is None else f(w), device=0)
    for k, val in opts.items():
        g.set_option(k, val)
    return g.build()


def _check_rows(tg, g, og, problem, sources, win, with_pred=True, stats=False):
    u32 = tg.as_u32
    if problem in ("eat", "ld", "reach"):
        out, pred = g.query(problem, sources, win, with_pred=True)
    else:
        out, pred = g.query(problem, sources, win), None
    out = u32(out)
    pred = u32(pred) if pred is not None else None
    per = g.last_stats(len(sources)).get("per_query_relax") if stats else None
    for r, x in enumerate(sources):
        if problem == "eat":
            A, P, W = oracle.eat(og, x, *win)
            np.testing.assert_array_equal(out[r], A, err_msg=f"EAT x={x} win={win}")
            np.testing.assert_array_equal(pred[r], P, err_msg=f"EAT pred x={x} win={win}")
            if per is not None:
                assert int(per[r]) == W, f"first-touch: relaxations {per[r]} != W {W}"
        elif problem == "ld":
            L, S, _ = oracle.ld(og, x, *win)
            np.testing.assert_array_equal(out[r], L, err_msg=f"LD x={x} win={win}")
            np.testing.assert_array_equal(pred[r], S, err_msg=f"LD succ x={x} win={win}")
        elif problem == "reach":
            np.testing.assert_array_equal(out[r], oracle.reach(og, x, *win))
        elif problem == "sp":
            np.testing.assert_array_equal(out[r], oracle.sp(og, x, *win), err_msg=f"SP x={x} win={win}")
        elif problem == "fp":
            np.testing.assert_array_equal(out[r], oracle.fp(og, x, *win), err_msg=f"FP x={x} win={win}")


# --------------------------------------------------------------------------- Figure 1
def test_figure1(tg):
    d = json.load(open(GOLDEN))
    ix = {s: i for i, s in enumerate(d["vertices"])}
    E = d["edges"]
    arr = lambda k: np.array([e[k] if k >= 2 else ix[e[k]] for e in E], np.uint32)
    n = len(ix)
    g = _gpu_graph(tg, n, arr(0), arr(1), arr(2), arr(3))
    og = oracle.Graph(n, arr(0), arr(1), arr(2), arr(3))
    for q in d["queries"]:
        _check_rows(tg, g, og, q["problem"], [ix[q["source"]]], tuple(q["window"]))
    ch = g.export_chains()
    got = [ch["chain_edges"][ch["chain_off"][i]:ch["chain_off"][i + 1]].tolist() for i in range(len(ch["chain_off"]) - 1)]
    assert got == d["chains"]["edge_sequences"]


# --------------------------------------------------------------------------- random graphs
@pytest.mark.parametrize("seed", range(40))
def test_tiny_random_all_problems(tg, seed):
    n, u, v, t, lam, w = tgsynth.tiny_random(seed, n_max=9, m_max=30, t_max=12)
    g = _gpu_graph(tg, n, u, v, t, lam, w, stats=1)
    og = oracle.Graph(n, u, v, t, lam, w)
    srcs = list(range(n))
    for win in [(0, 100), (2, 9), (3, 3)]:
        for p in ("eat", "ld", "reach", "sp", "fp"):
            _check_rows(tg, g, og, p, srcs, win, stats=(p == "eat"))


def test_relabel_option(tg):
    """Internal vertex relabelling (descending in-degree) is invisible to callers:
    values, preds and exported chains equal the oracle."""
    n, u, v, t, lam, w = tgsynth.tiny_random(4242, n_max=50, m_max=700, t_max=30, lam_max=4)
    g = _gpu_graph(tg, n, u, v, t, lam, w, relabel=1, stats=1)
    og = oracle.Graph(n, u, v, t, lam, w)
    for p in ("eat", "ld", "reach", "sp", "fp"):
        _check_rows(tg, g, og, p, list(range(min(n, 20))), (2, 10**6), stats=(p == "eat"))
    off, ce = oracle.chains(og)
    sc = oracle.shortcuts(og, off, ce)
    ch = g.export_chains()
    np.testing.assert_array_equal(ch["chain_off"], off)
    np.testing.assert_array_equal(ch["chain_edges"], ce)
    for k in ("tail_v", "arr", "elapsed", "sum_w"):
        np.testing.assert_array_equal(ch[k], sc[k], err_msg=k)


@pytest.mark.parametrize("walk_min", [2, 6])
def test_walk_threshold(tg, walk_min):
    """Every chain walked (walk_min = 2) and the default threshold give identical,
    exact results and the same first-touch work."""
    for seed in range(4):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 900, n_max=60, m_max=900, t_max=40, lam_max=4)
        g = _gpu_graph(tg, n, u, v, t, lam, w, walk_min=walk_min, stats=1)
        og = oracle.Graph(n, u, v, t, lam, w)
        for p in ("eat", "ld", "sp", "fp"):
            _check_rows(tg, g, og, p, list(range(min(n, 12))), (0, 10**6), stats=(p == "eat"))


@pytest.mark.parametrize("seed", range(6))
def test_medium_random(tg, seed):
    rng = np.random.default_rng(seed)
    n, m = 3000, 40000
    u = rng.integers(0, n, m).astype(np.uint32)
    v = rng.integers(0, n, m).astype(np.uint32)
    t = rng.integers(0, 500, m).astype(np.uint32)
    lam = rng.integers(1, 8, m).astype(np.uint32)
    w = rng.integers(0, 20, m).astype(np.uint32)
    g = _gpu_graph(tg, n, u, v, t, lam, w, stats=1, sub_batch=7)
    og = oracle.Graph(n, u, v, t, lam, w)
    srcs = [int(x) for x in rng.choice(n, 24, replace=False)]
    for win in [(0, 10**6), (100, 300)]:
        for p in ("eat", "ld", "sp", "fp"):
            _check_rows(tg, g, og, p, srcs, win, stats=(p == "eat"))


def test_chains_match_alg1_random(tg):
    for seed in range(20):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 500, n_max=40, m_max=400, t_max=30, lam_max=5)
        g = _gpu_graph(tg, n, u, v, t, lam, w)
        og = oracle.Graph(n, u, v, t, lam, w)
        off, ce = oracle.chains(og)
        sc = oracle.shortcuts(og, off, ce)
        ch = g.export_chains()
        np.testing.assert_array_equal(ch["chain_off"], off)
        np.testing.assert_array_equal(ch["chain_edges"], ce)
        for k in ("tail_v", "arr", "elapsed", "sum_w"):
            np.testing.assert_array_equal(ch[k], sc[k], err_msg=k)


# --------------------------------------------------------------------------- configs
def test_c1_full(tg):
    """configs[0]: R-MAT 2^14 V / 2^18 E, t in [0,1000), EAT from 0 (+ all problems)."""
    ge = tgsynth.make_graph("C1")
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, stats=1)
    og = oracle.Graph(n, u, v, t, d, w)
    off, ce = oracle.chains(og)
    ch = g.export_chains()
    np.testing.assert_array_equal(ch["chain_off"], off)
    np.testing.assert_array_equal(ch["chain_edges"], ce)
    for win in tgsynth.CONFIGS["C1"]["windows"]:
        for p in ("eat", "ld", "sp", "fp", "reach"):
            _check_rows(tg, g, og, p, [0, 1, 17, 4000], win, stats=(p == "eat"))


def test_c2_small_batch(tg):
    """configs[1] shape at 1/16 scale: EAT + LD, 64-source batch, several tiles + ragged sub-batch."""
    ge = tgsynth.make_graph("C2", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, stats=1, sub_batch=24)
    og = oracle.Graph(n, u, v, t, d, w)
    srcs = tgsynth.config_sources("C2", ge)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        _check_rows(tg, g, og, "eat", srcs, win, stats=True)
        _check_rows(tg, g, og, "ld", srcs[:16], win)


@pytest.mark.parametrize("k", [40, 64, 65])
def test_two_query_groups(tg, k):
    """Sub-batches spanning two 32-query groups (a partial second group at 40, full at
    64, and 64 + a ragged 1-query sub-batch at 65): packed (pred) and u32-state (values
    only, the bench path) rows against the oracle."""
    import torch
    ge = tgsynth.make_graph("C2", scale_shift=-5)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d)
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C2", ge, k=k)
    win = tgsynth.CONFIGS["C2"]["windows"][1]
    for p in ("eat", "ld"):
        _check_rows(tg, g, og, p, srcs, win)
        vals = tg.as_u32(g.query(p, srcs, win))
        torch.cuda.synchronize()
        for r in (0, k // 2, k - 1):
            ref = (oracle.eat if p == "eat" else oracle.ld)(og, srcs[r], *win)[0]
            np.testing.assert_array_equal(vals[r], ref, err_msg=f"u32-state {p} row {r}")


def test_union_work_count(tg):
    """W_union (distinct slots relaxed by any query of the sub-batch, the bench's
    algorithmic-bytes input) equals the union of the oracle's usable valid edges."""
    ge = tgsynth.make_graph("C2", scale_shift=-5)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, stats=1)
    og = oracle.Graph(n, u, v, t, d, w)
    srcs = tgsynth.config_sources("C2", ge, k=40)
    win = (1000, 50000)
    g.query("eat", srcs, win)
    st = g.last_stats(len(srcs))
    used = np.zeros(len(u), bool)
    valid = (t >= win[0]) & (t.astype(np.int64) + d <= win[1])
    for x in srcs:
        A, _, _ = oracle.eat(og, x, *win)
        used |= valid & (A[u] != NONE) & (A[u] <= t)
    assert st["slots_union"] == int(used.sum())
    assert st["slots_relaxed"] >= st["slots_union"]


def test_c3_small_all_problems(tg):
    """configs[2] shape at 1/16 scale: wiki-talk-shaped, all four problems."""
    ge = tgsynth.make_graph("C3", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, stats=1)
    og = oracle.Graph(n, u, v, t, d, w)
    srcs = tgsynth.config_sources("C3", ge)
    for win in tgsynth.CONFIGS["C3"]["windows"]:
        for p in ("eat", "ld", "sp", "fp"):
            _check_rows(tg, g, og, p, srcs[:8], win, stats=(p == "eat"))


@pytest.mark.slow
def test_c2_full_sampled_rows(tg):
    """configs[1] at full size in the bench's launch configuration: 64-source EAT and
    LD batches; a seeded sample of rows is compared with the oracle row by row."""
    import torch
    ge = tgsynth.make_graph("C2", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, None, device=0).build()
    srcs = tgsynth.config_sources("C2", ge)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        out, pred = g.query("eat", srcs, win, with_pred=True)
        lout, lpred = g.query("ld", srcs, win, with_pred=True)
        torch.cuda.synchronize()
        for r in (0, 13, 63):
            A, P, _ = oracle.eat(og, srcs[r], *win)
            np.testing.assert_array_equal(tg.as_u32(out[r]), A)
            np.testing.assert_array_equal(tg.as_u32(pred[r]), P)
            L, S, _ = oracle.ld(og, srcs[r], *win)
            np.testing.assert_array_equal(tg.as_u32(lout[r]), L)
            np.testing.assert_array_equal(tg.as_u32(lpred[r]), S)


@pytest.mark.slow
def test_c3_full_sampled_rows(tg):
    """configs[2] at full size: wiki-talk-shaped graph, all four problems, sampled rows."""
    import torch
    ge = tgsynth.make_graph("C3", device="cuda")
    g = tg.Graph(ge.n, ge.u, ge.v, ge.t, ge.dur, ge.w, device=0).build()
    srcs = tgsynth.config_sources("C3", ge)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d, w)
    for win in tgsynth.CONFIGS["C3"]["windows"]:
        res = {p: g.query(p, srcs, win) for p in ("eat", "ld", "fp", "sp")}
        torch.cuda.synchronize()
        for r in (0, 7):
            x = srcs[r]
            np.testing.assert_array_equal(tg.as_u32(res["eat"][r]), oracle.eat(og, x, *win)[0])
            np.testing.assert_array_equal(tg.as_u32(res["ld"][r]), oracle.ld(og, x, *win)[0])
            np.testing.assert_array_equal(tg.as_u32(res["fp"][r]), oracle.fp(og, x, *win))
            np.testing.assert_array_equal(tg.as_u32(res["sp"][r]), oracle.sp(og, x, *win))


# --------------------------------------------------------------------------- edge cases
def test_edge_cases(tg):
    # no edges
    g = _gpu_graph(tg, 5, np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    og = oracle.Graph(5, [], [], [], [])
    for p in ("eat", "ld", "sp", "fp", "reach"):
        _check_rows(tg, g, og, p, [0, 4], (0, 10))
    # one vertex, self-loops and duplicates
    u = np.array([0, 0, 0], np.uint32); t = np.array([1, 1, 3], np.uint32); lam = np.array([1, 1, 2], np.uint32)
    g = _gpu_graph(tg, 1, u, u, t, lam)
    og = oracle.Graph(1, u, u, t, lam)
    for p in ("eat", "ld", "sp", "fp", "reach"):
        _check_rows(tg, g, og, p, [0], (0, 10))


def test_long_chain_and_hub(tg):
    # a path 0 -> 1 -> ... -> L (one long chain) plus a hub with many out-edges at one time
    L = 5000
    u = list(range(L)); v = list(range(1, L + 1)); t = list(range(L)); lam = [1] * L
    H = 20000
    u += [0] * H; v += list(np.random.default_rng(0).integers(1, L + 1, H)); t += [0] * H; lam += [3] * H
    u, v, t, lam = (np.array(a, np.uint32) for a in (u, v, t, lam))
    g = _gpu_graph(tg, L + 1, u, v, t, lam, stats=1, walk_min=2)
    og = oracle.Graph(L + 1, u, v, t, lam)
    for win in [(0, 10**6), (0, 2500), (7, 4000)]:
        for p in ("eat", "ld", "sp", "fp"):
            _check_rows(tg, g, og, p, [0, 1, 2500], win, stats=(p == "eat"))
    assert g.info()["max_chain_len"] >= 2


def test_host_and_device_buffers_agree(tg):
    import torch
    n, u, v, t, lam, w = tgsynth.tiny_random(7, n_max=30, m_max=300, t_max=20)
    g = _gpu_graph(tg, n, u, v, t, lam, w)
    srcs = list(range(min(n, 5)))
    dev = g.query("eat", srcs, (0, 100))
    host = torch.empty((len(srcs), n), dtype=torch.int32)
    tg.tg_query(g.h, tg.TG_EAT, srcs, (0, 100), host)
    assert torch.equal(dev.cpu(), host)


def test_abi_errors_on_gpu(tg):
    n = 5
    u = np.array([0, 1, 2, 3], np.uint32); v = np.array([1, 2, 3, 4], np.uint32)
    t = np.array([1, 2, 3, 4], np.uint32); lam = np.array([1, 1, 1, 1], np.uint32)
    import torch
    f = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).cuda()
    with pytest.raises(tg.TGError) as e:
        tg.Graph(n, f(u), f(np.full_like(v, n)), f(t), f(lam))
    assert e.value.status == 2
    with pytest.raises(tg.TGError) as e:
        tg.Graph(n, f(u), f(v), f(t), f(np.zeros_like(lam)))
    assert e.value.status == 1
    big = np.full_like(t, 0x7FFFFFFE)
    if len(t):
        with pytest.raises(tg.TGError) as e:
            tg.Graph(n, f(u), f(v), f(big), f(lam))
        assert e.value.status == 2
    g = tg.Graph(n, f(u), f(v), f(t), f(lam))
    out = torch.empty((1, n), dtype=torch.int32, device="cuda")
    with pytest.raises(tg.TGError) as e:
        tg.tg_query(g.h, tg.TG_EAT, [0], (0, 10), out)  # before build
    assert e.value.status == 5
    g.build()
    with pytest.raises(tg.TGError) as e:
        tg.tg_query(g.h, tg.TG_EAT, [0], (10, 0), out)
    assert e.value.status == 1
    with pytest.raises(tg.TGError) as e:
        tg.tg_query(g.h, tg.TG_EAT, [n], (0, 10), out)
    assert e.value.status == 2
    with pytest.raises(tg.TGError) as e:
        tg.tg_query(g.h, tg.TG_SHORTEST, [0], (0, 10), out, pred=out)
    assert e.value.status == 1


# --------------------------------------------------------------------------- vertex-range partitions
@pytest.mark.parametrize("parts", [2, 3, 5])
def test_logical_partitions_random(tg, parts):
    """Multi-GPU mode 1 (vertex-range partitions + state exchange) run as logical
    partitions on one GPU: bit-exact, including preds and first-touch W."""
    for seed in range(6):
        rng = np.random.default_rng(seed + 77)
        n, m = 400, 5000
        u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
        t = rng.integers(0, 300, m).astype(np.uint32); lam = rng.integers(1, 6, m).astype(np.uint32)
        g = _gpu_graph(tg, n, u, v, t, lam, partitions=parts, stats=1)
        og = oracle.Graph(n, u, v, t, lam)
        srcs = [int(x) for x in rng.choice(n, 40, replace=False)]
        for win in [(0, 10**6), (30, 200)]:
            for p in ("eat", "ld", "reach"):
                _check_rows(tg, g, og, p, srcs, win, stats=(p == "eat"))


def test_logical_partitions_c1(tg):
    ge = tgsynth.make_graph("C1")
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, partitions=4, mirror=0)  # LD mirror built on first use
    og = oracle.Graph(n, u, v, t, d, w)
    for win in tgsynth.CONFIGS["C1"]["windows"]:
        _check_rows(tg, g, og, "eat", [0, 5, 99], win)
        _check_rows(tg, g, og, "ld", [0, 5], win)
    with pytest.raises(tg.TGError):
        g.query("sp", [0], (0, 10))  # partitioned graphs answer EAT/LD/REACH only


@pytest.mark.parametrize("exchange", [0, 1])
def test_nccl_comm_world1_vertex_range(tg, exchange):
    """Mode 1 through an NCCL communicator of world 1 (one GPU available).  With
    exchange = 1 the rank runs the cross-rank round exactly as in a multi-GPU run:
    per-round ncclAllReduce(min) of the states, k_part_frontier (next frontier derived
    from the exchanged state) and ncclAllReduce(sum) of the frontier count.  With
    exchange = 0 a world of 1 shares its state like logical partitions (no NCCL call
    in the round loop)."""
    import torch
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import distributed as tgd
    ge = tgsynth.make_graph("C2", scale_shift=-6)
    n, u, v, t, d, w = ge.numpy()
    comm = tgd.make_comm(0, 1, 0)
    f = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).cuda()
    g = tg.Graph(n, f(u), f(v), f(t), f(d), device=0)
    g.set_option("exchange", exchange)
    tg.tg_graph_attach_comm(g.h, comm, 1)
    g.build()
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C2", ge, k=8)
    _check_rows(tg, g, og, "eat", srcs, (0, 10**9))
    _check_rows(tg, g, og, "ld", srcs, (0, 10**9))
    _check_values(tg, g, og, "reach", srcs, (1000, 40000))
    g.close()
    tg.tg_comm_destroy(comm)


@pytest.mark.parametrize("parts", [2, 3, 8])
def test_exchange_partitions_random(tg, parts):
    """The multi-rank vertex-range algorithm (P:L313 rounds) inside one
    process: every logical partition relaxes its own chains into a PRIVATE state copy,
    the copies are combined by an elementwise min after every round (what
    ncclAllReduce(min) leaves on every rank), and each partition derives its next
    frontier from the combined state (k_part_frontier).  Bit-exact with preds and
    first-touch W, packed and u32 states."""
    for seed in range(5):
        rng = np.random.default_rng(seed + 177)
        n, m = 300 + 50 * seed, 4000
        u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
        t = rng.integers(0, 300, m).astype(np.uint32); lam = rng.integers(1, 6, m).astype(np.uint32)
        g = _gpu_graph(tg, n, u, v, t, lam, partitions=parts, exchange=1, stats=1, sub_batch=37)
        og = oracle.Graph(n, u, v, t, lam)
        srcs = [int(x) for x in rng.choice(n, 40, replace=False)]
        for win in [(0, 10**6), (30, 200)]:
            for p in ("eat", "ld", "reach"):
                _check_rows(tg, g, og, p, srcs, win, stats=(p == "eat"))
                _check_values(tg, g, og, p, srcs, win)
        g.close()


def test_exchange_partitions_c1(tg):
    ge = tgsynth.make_graph("C1")
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d, w)
    for parts in (2, 8):
        g = _gpu_graph(tg, n, u, v, t, d, w, partitions=parts, exchange=1)
        for win in tgsynth.CONFIGS["C1"]["windows"]:
            _check_rows(tg, g, og, "eat", [0, 5, 99], win)
            _check_rows(tg, g, og, "ld", [0, 5], win)
            _check_values(tg, g, og, "eat", [0, 7], win)
        g.close()


def test_exchange_partitions_c5_eighth(tg):
    """C5-shaped (Chung-Lu, lambda ~ U[1,15]) at 1/8 scale, 8 partitions, single-source
    EAT as in the C5 configuration: values and preds against the oracle."""
    ge = tgsynth.make_graph("C5", device="cuda", scale_shift=-3)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C5", ge, k=2)
    g = _gpu_graph(tg, n, u, v, t, d, partitions=8, exchange=1, mirror=0)
    _check_rows(tg, g, og, "eat", srcs, (0, 10**9))
    _check_values(tg, g, og, "eat", srcs, (0, 10**9))
    g.close()


# --------------------------------------------------------------------------- state width / schedules
def _check_values(tg, g, og, problem, sources, win):
    """Values only (pred = NULL: the engines keep u32 arrival states, not packed words)."""
    out = tg.as_u32(g.query(problem, sources, win))
    for r, x in enumerate(sources):
        if problem == "eat":
            exp = oracle.eat(og, x, *win)[0]
        elif problem == "ld":
            exp = oracle.ld(og, x, *win)[0]
        else:
            exp = oracle.reach(og, x, *win)
        np.testing.assert_array_equal(out[r], exp, err_msg=f"{problem} (no pred) x={x} win={win}")


@pytest.mark.parametrize("seed", range(4))
def test_unpacked_state_values(tg, seed):
    """Without pred the EAT family runs on u32 arrival states; values equal the oracle
    (the packed path is covered by every test that asks for preds)."""
    n, u, v, t, lam, w = tgsynth.tiny_random(seed + 3100, n_max=80, m_max=1500, t_max=60, lam_max=6)
    g = _gpu_graph(tg, n, u, v, t, lam, w, sub_batch=5)
    og = oracle.Graph(n, u, v, t, lam, w)
    srcs = list(range(min(n, 17)))
    for win in [(0, 10**6), (5, 40)]:
        for p in ("eat", "ld", "reach"):
            _check_values(tg, g, og, p, srcs, win)


def test_unpacked_state_c2_small(tg):
    ge = tgsynth.make_graph("C2", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w)
    og = oracle.Graph(n, u, v, t, d, w)
    srcs = tgsynth.config_sources("C2", ge)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        _check_values(tg, g, og, "eat", srcs, win)
        _check_values(tg, g, og, "ld", srcs[:16], win)


@pytest.mark.parametrize("seed,sub_batch", [(0, 64), (1, 40), (2, 9), (3, 33)])
def test_arrival_bound_filter_random(tg, seed, sub_batch):
    """Option ub_filter=2 forces the per-(vertex, 8 queries) arrival bounds that prune
    (edge, query) pairs (auto-enabled only for states >= 1 GiB): values and preds stay
    equal to the oracle, with full and ragged 8-query blocks and one or two groups."""
    n, u, v, t, lam, w = tgsynth.tiny_random(seed + 4100, n_max=120, m_max=3000, t_max=300, lam_max=9)
    g = _gpu_graph(tg, n, u, v, t, lam, w, sub_batch=sub_batch, ub_filter=2)
    og = oracle.Graph(n, u, v, t, lam, w)
    srcs = [i % n for i in range(70)]
    for win in [(0, 10**6), (20, 200), (7, 7)]:
        _check_rows(tg, g, og, "eat", srcs, win)
        _check_rows(tg, g, og, "ld", srcs[:24], win)
        for p in ("eat", "ld", "reach"):
            _check_values(tg, g, og, p, srcs, win)


def test_arrival_bound_filter_c2_small(tg):
    ge = tgsynth.make_graph("C2", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, w, ub_filter=2)
    og = oracle.Graph(n, u, v, t, d, w)
    srcs = tgsynth.config_sources("C2", ge)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        _check_values(tg, g, og, "eat", srcs, win)
        _check_rows(tg, g, og, "eat", srcs[:8], win)
        _check_values(tg, g, og, "ld", srcs[:16], win)


@pytest.mark.parametrize("graph_loop", [0, 2])
def test_round_loop_modes(tg, graph_loop):
    """GAC rounds driven by the host (checks every round_group rounds) or by the device in
    a CUDA-graph WHILE loop (the default): same rows and preds; packed and u32 states
    alternate on one handle (the cached loop graph is keyed by the state width)."""
    ge = tgsynth.make_graph("C2", scale_shift=-5)
    n, u, v, t, d, w = ge.numpy()
    g = _gpu_graph(tg, n, u, v, t, d, graph_loop=graph_loop)
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C2", ge, k=40)
    rounds = []
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        for p in ("eat", "ld"):
            _check_rows(tg, g, og, p, srcs, win)
            rounds.append(g.last_stats()["rounds"])
            _check_values(tg, g, og, p, srcs, win)
        for p in ("sp", "fp"):  # the SP/FP node-state engine's loop (same two modes)
            _check_rows(tg, g, og, p, srcs[:6], win)
            rounds.append(g.last_stats()["rounds"])
    assert min(rounds) >= 1


def test_two_query_lanes(tg):
    """Sub-batches rotating over 2 or 4 query lanes (scratch sets + streams, option lanes;
    2 is the default for device outputs) give the same rows as one lane, for EAT, LD and
    REACH, with scheduled (reordered) sources, a ragged last sub-batch and preds."""
    import torch
    ge = tgsynth.make_graph("C2", scale_shift=-5)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C2", ge, k=200)
    res = {}
    for lanes in (1, 2, 4):
        g = _gpu_graph(tg, n, u, v, t, d, lanes=lanes, graph_loop=2)
        for win in tgsynth.CONFIGS["C2"]["windows"]:
            for p in ("eat", "ld", "reach"):
                o = g.query(p, srcs, win)
                o2, pr = g.query(p, srcs, win, with_pred=True)
                torch.cuda.synchronize()
                res[(lanes, win, p)] = (tg.as_u32(o), tg.as_u32(o2), tg.as_u32(pr), g.last_stats()["rounds"])
        # host outputs (pinned staging ring on a copy stream; one lane)
        win = tgsynth.CONFIGS["C2"]["windows"][0]
        h = torch.empty((len(srcs), n), dtype=torch.int32).pin_memory()
        g.query("eat", srcs, win, out=h)
        res[(lanes, "host")] = tg.as_u32(h)
    for key in [k for k in res if k[0] > 1 and k[1] != "host"]:
        a, b = res[key], res[(1,) + key[1:]]
        for x, y in zip(a[:3], b[:3]):
            np.testing.assert_array_equal(x, y)
        # (round counts are not compared: which round a relaxation lands in depends on the
        # timing of concurrent claims and stale-safe reads; the fixpoint does not)
        assert a[3] >= 1 and b[3] >= 1
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        vals = res[(2, win, "eat")][0]
        for r in (0, 63, 64, 127, 128, 199):
            np.testing.assert_array_equal(vals[r], oracle.eat(og, srcs[r], *win)[0])
    for lanes in (2, 4):
        np.testing.assert_array_equal(res[(lanes, "host")], res[(1, "host")])
        np.testing.assert_array_equal(res[(lanes, "host")], res[(1, tgsynth.CONFIGS["C2"]["windows"][0], "eat")][0])


# --------------------------------------------------------------------------- bit-lane reachability (f2)
def _check_reach(tg, g, og, sources, win, host=False):
    import torch
    if host:
        out = torch.empty((len(sources), og.n), dtype=torch.int32)
        tg.tg_query(g.h, tg.TG_REACH, sources, win, out)
    else:
        out = g.query("reach", sources, win)
    out = tg.as_u32(out)
    for r, x in enumerate(sources):
        np.testing.assert_array_equal(out[r], oracle.reach(og, x, *win), err_msg=f"REACH x={x} win={win}")


@pytest.mark.parametrize("seed", range(8))
def test_reach_bitlane_random(tg, seed):
    """pred = NULL runs TG_REACH on the bit-lane engine (64 sources per u64 word over
    the departure nodes): equal to the oracle's reachability
    for 100 sources (two words), several windows incl. alpha == omega."""
    n, u, v, t, lam, w = tgsynth.tiny_random(seed + 6100, n_max=120, m_max=2500, t_max=60, lam_max=6)
    og = oracle.Graph(n, u, v, t, lam, w)
    for opts in ({}, {"walk_min": 2}, {"relabel": 1}):
        g = _gpu_graph(tg, n, u, v, t, lam, w, reach_bits=1, **opts)
        srcs = list(range(min(n, 100)))
        for win in [(0, 10**6), (5, 40), (7, 7), (20, 21)]:
            _check_reach(tg, g, og, srcs, win)
        g.close()


def test_reach_bitlane_hubs_and_host(tg):
    """A hub with thousands of departure nodes (long wait-edge scans, queued edge chunks),
    long chains, duplicates and self-loops; host-memory output."""
    rng = np.random.default_rng(61)
    n = 700
    parts = []
    # hub 0: 6000 out-edges at distinct-ish times; chains 1 -> 2 -> ... -> 60 at increasing times
    parts.append((np.zeros(6000), rng.integers(0, n, 6000), rng.integers(0, 3000, 6000), rng.integers(1, 4, 6000)))
    parts.append((np.arange(1, 61), np.arange(2, 62), np.arange(1, 61) * 3, np.full(60, 2)))
    parts.append((rng.integers(0, n, 9000), rng.integers(0, n, 9000), rng.integers(0, 3000, 9000),
                  rng.integers(1, 9, 9000)))
    parts.append((np.full(50, 5), np.full(50, 5), np.arange(50), np.ones(50)))  # self-loops
    u, v, t, lam = (np.concatenate([p[i] for p in parts]).astype(np.uint32) for i in range(4))
    og = oracle.Graph(n, u, v, t, lam)
    g = _gpu_graph(tg, n, u, v, t, lam, walk_min=2, reach_bits=1)
    srcs = [0, 1, 5] + [int(x) for x in rng.choice(n, 70, replace=False)]
    for win in [(0, 10**6), (100, 2000)]:
        _check_reach(tg, g, og, srcs, win)
        _check_reach(tg, g, og, srcs[:9], win, host=True)
    g.close()


def test_reach_bitlane_c2_small(tg):
    ge = tgsynth.make_graph("C2", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d)
    srcs = tgsynth.config_sources("C2", ge)
    for bits in (1, 0):
        g = _gpu_graph(tg, n, u, v, t, d, reach_bits=bits)
        for win in tgsynth.CONFIGS["C2"]["windows"]:
            _check_reach(tg, g, og, srcs, win)
        g.close()


# --------------------------------------------------------------------------- f4: LDS, top-K, summaries
@pytest.mark.parametrize("seed", range(10))
def test_lds_random(tg, seed):
    """Single-source latest departure (reading R5) on the FP node-state engine: equal to
    the oracle's one-pass scan, several windows, walk thresholds and relabelling."""
    n, u, v, t, lam, w = tgsynth.tiny_random(seed + 7300, n_max=60, m_max=900, t_max=40, lam_max=5)
    og = oracle.Graph(n, u, v, t, lam, w)
    for opts in ({}, {"walk_min": 2, "relabel": 1}):
        g = _gpu_graph(tg, n, u, v, t, lam, w, **opts)
        srcs = list(range(min(n, 20)))
        for win in [(0, 10**6), (4, 30), (9, 9)]:
            out = tg.as_u32(g.query("lds", srcs, win))
            for r, x in enumerate(srcs):
                np.testing.assert_array_equal(out[r], oracle.lds(og, x, *win), err_msg=f"LDS x={x} win={win}")
        g.close()


def test_lds_c1(tg):
    ge = tgsynth.make_graph("C1")
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d, w)
    g = _gpu_graph(tg, n, u, v, t, d, w)
    for win in tgsynth.CONFIGS["C1"]["windows"]:
        out = tg.as_u32(g.query("lds", [0, 3, 77], win))
        for r, x in enumerate([0, 3, 77]):
            np.testing.assert_array_equal(out[r], oracle.lds(og, x, *win), err_msg=f"LDS C1 x={x} win={win}")
    g.close()


@pytest.mark.parametrize("problem", ["eat", "fp", "sp"])
def test_topk_and_summary(tg, problem):
    """top-K nearest (ties by vertex id, source and unreached excluded, padding) and the
    (reached, sum) row summary against the oracle rows; device and host outputs."""
    import torch
    rng = np.random.default_rng(7)
    n, m = 2000, 30000
    u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
    t = rng.integers(0, 400, m).astype(np.uint32); lam = rng.integers(1, 8, m).astype(np.uint32)
    w = rng.integers(0, 9, m).astype(np.uint32)
    og = oracle.Graph(n, u, v, t, lam, w)
    g = _gpu_graph(tg, n, u, v, t, lam, w)
    srcs = [int(x) for x in rng.choice(n, 40, replace=False)]
    fn = {"eat": lambda x, win: oracle.eat(og, x, *win)[0], "fp": lambda x, win: oracle.fp(og, x, *win),
          "sp": lambda x, win: oracle.sp(og, x, *win)}[problem]
    for win, K in [((0, 10**6), 50), ((100, 200), 3000)]:
        ov, oval = g.topk(problem, srcs, K, win)
        ov, oval = tg.as_u32(ov), tg.as_u32(oval)
        hv = torch.empty((len(srcs), K), dtype=torch.int32)
        hx = torch.empty((len(srcs), K), dtype=torch.int32)
        tg.tg_query_topk(g.h, tg.PROBLEMS[problem], srcs, win, K, hv, hx)
        cnt, sm = g.summary(problem, srcs, win)
        for r, x in enumerate(srcs):
            row = fn(x, win)
            ev, ex = oracle.topk(row, x, K)
            np.testing.assert_array_equal(ov[r], ev, err_msg=f"top-K vertices x={x}")
            np.testing.assert_array_equal(oval[r], ex, err_msg=f"top-K values x={x}")
            np.testing.assert_array_equal(tg.as_u32(hv[r]), ev)
            np.testing.assert_array_equal(tg.as_u32(hx[r]), ex)
            assert (int(cnt[r]), int(sm[r])) == oracle.summary(row, x)
    g.close()


# --------------------------------------------------------------------------- f3: dynamic insertions
def _t32(a):
    import torch
    return torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32)).cuda()


@pytest.mark.parametrize("seed", range(4))
def test_insert_edges_incremental(tg, seed):
    """Batches of insertions into a built graph: after each batch the
    incrementally re-transformed chains equal Alg. 1 / Alg. 2 of the oracle on the whole
    edge list (ids continue), and every problem equals the oracle."""
    rng = np.random.default_rng(seed + 4400)
    n = 300
    m0 = 3000
    cols = lambda m, tmax: (rng.integers(0, n, m), rng.integers(0, n, m), rng.integers(0, tmax, m),
                            rng.integers(1, 7, m), rng.integers(0, 9, m))
    U, V, T, L, W = (np.asarray(c, np.uint32) for c in cols(m0, 200))
    g = _gpu_graph(tg, n, U, V, T, L, W, dynamic=1, reach_bits=1)
    for b, (k, tmax) in enumerate([(500, 200), (1200, 400), (1, 50), (800, 600)]):
        bu, bv, bt, bl, bw = (np.asarray(c, np.uint32) for c in cols(k, tmax))
        g.insert_edges(_t32(bu), _t32(bv), _t32(bt), _t32(bl), _t32(bw))
        U, V, T, L, W = (np.concatenate([a, c]) for a, c in zip((U, V, T, L, W), (bu, bv, bt, bl, bw)))
        og = oracle.Graph(n, U, V, T, L, W)
        off, ce = oracle.chains(og)
        sc = oracle.shortcuts(og, off, ce)
        ch = g.export_chains()
        np.testing.assert_array_equal(ch["chain_off"], off, err_msg=f"batch {b}")
        np.testing.assert_array_equal(ch["chain_edges"], ce, err_msg=f"batch {b}")
        for key in ("tail_v", "arr", "elapsed", "sum_w"):
            np.testing.assert_array_equal(ch[key], sc[key], err_msg=key)
        gr, _ = oracle.mirror(og)
        moff, mce = oracle.chains(gr)
        mch = g.export_chains(mirrored=True, shortcuts=False)
        np.testing.assert_array_equal(mch["chain_edges"], mce)
        srcs = [int(x) for x in rng.choice(n, 12, replace=False)]
        for win in [(0, 10**6), (40, 300)]:
            for p in ("eat", "ld", "sp", "fp", "reach"):
                _check_rows(tg, g, og, p, srcs, win)
            _check_reach(tg, g, og, srcs, win)
    g.close()


def test_insert_edges_errors_and_unbuilt(tg):
    rng = np.random.default_rng(3)
    n, m = 50, 400
    U, V, T, L = (rng.integers(0, n, m).astype(np.uint32), rng.integers(0, n, m).astype(np.uint32),
                  rng.integers(0, 90, m).astype(np.uint32), rng.integers(1, 4, m).astype(np.uint32))
    f = _t32
    # built without "dynamic": refused
    g = _gpu_graph(tg, n, U, V, T, L)
    with pytest.raises(tg.TGError) as e:
        g.insert_edges(f(U[:5]), f(V[:5]), f(T[:5]), f(L[:5]))
    assert e.value.status == 5
    g.close()
    # unbuilt: edges appended, the first build sees all of them; a bad batch rolls back
    g = tg.Graph(n, f(U), f(V), f(T), f(L), None, device=0)
    g.set_option("dynamic", 1)
    g.insert_edges(f(V[:100]), f(U[:100]), f(T[:100] + 5), f(L[:100]))
    with pytest.raises(tg.TGError) as e:
        g.insert_edges(f(np.array([n], np.uint32)), f(U[:1]), f(T[:1]), f(L[:1]))  # endpoint out of range
    assert e.value.status == 2
    g.build()
    U2, V2 = np.concatenate([U, V[:100]]), np.concatenate([V, U[:100]])
    T2, L2 = np.concatenate([T, T[:100] + 5]), np.concatenate([L, L[:100]])
    og = oracle.Graph(n, U2, V2, T2, L2)
    _check_rows(tg, g, og, "eat", list(range(10)), (0, 10**6))
    _check_rows(tg, g, og, "ld", list(range(10)), (0, 10**6))
    g.close()


# --------------------------------------------------------------------------- f1: out-of-memory graphs
def _streamed(tg, n, u, v, t, lam, w=None, block_edges=64, **opts):
    import torch
    f = lambda a: torch.from_numpy(np.ascontiguousarray(a, np.uint32).view(np.int32))  # HOST tensors
    g = tg.Graph(n, f(u), f(v), f(t), f(lam), None if w is None else f(w), device=0, block_edges=block_edges)
    for k, val in opts.items():
        g.set_option(k, val)
    return g.build()


@pytest.mark.parametrize("seed", range(6))
def test_streamed_blocks_random(tg, seed):
    """Graphs cut into time blocks (§4.5), transformed per block, kept in host
    memory and streamed through two device slots: EAT values, preds and first-touch W,
    REACH, equal to the oracle for block sizes from a few edges to the whole graph."""
    rng = np.random.default_rng(seed + 5100)
    n, m = 200 + 40 * seed, 3000
    u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
    t = rng.integers(0, 120 + 400 * (seed % 2), m).astype(np.uint32); lam = rng.integers(1, 9, m).astype(np.uint32)
    og = oracle.Graph(n, u, v, t, lam)
    srcs = [int(x) for x in rng.choice(n, 37, replace=False)]
    for be in (1, 37, 500, 10**6):
        g = _streamed(tg, n, u, v, t, lam, block_edges=be, stats=1)
        info = g.info()
        assert info["n_blocks"] >= 1 and (be >= m or info["n_blocks"] > 1)
        for win in [(0, 10**6), (30, 90), (50, 50)]:
            _check_rows(tg, g, og, "eat", srcs, win, stats=True)
            _check_values(tg, g, og, "eat", srcs, win)
            _check_values(tg, g, og, "reach", srcs, win)
        with pytest.raises(tg.TGError) as e:
            g.query("ld", srcs[:2], (0, 100))
        assert e.value.status == 5
        g.close()


def test_streamed_c2_small_and_host_out(tg):
    import torch
    ge = tgsynth.make_graph("C2", scale_shift=-4)
    n, u, v, t, d, w = ge.numpy()
    og = oracle.Graph(n, u, v, t, d)
    g = _streamed(tg, n, u, v, t, d, block_edges=100_000)
    assert g.info()["n_blocks"] >= 10
    srcs = tgsynth.config_sources("C2", ge)
    for win in tgsynth.CONFIGS["C2"]["windows"]:
        _check_values(tg, g, og, "eat", srcs, win)
    hout = torch.empty((8, n), dtype=torch.int32)
    tg.tg_query(g.h, tg.TG_EAT, srcs[:8], (0, 10**9), hout)
    for r, x in enumerate(srcs[:8]):
        np.testing.assert_array_equal(tg.as_u32(hout[r]), oracle.eat(og, x, 0, 10**9)[0])
    g.close()


# --------------------------------------------------------------------------- sub-batch scheduling
@pytest.mark.parametrize("seed", range(3))
def test_source_scheduling_rows(tg, seed):
    """Sources of a call are scheduled into sub-batches by first departure time; every
    query's values, preds and first-touch W must land in the caller's row (device and host
    outputs, ragged last sub-batch, sub-batch sizes 64 and 20, duplicate sources)."""
    import torch
    rng = np.random.default_rng(seed + 8800)
    n, m = 500, 9000
    u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
    t = rng.integers(0, 400, m).astype(np.uint32); lam = rng.integers(1, 9, m).astype(np.uint32)
    og = oracle.Graph(n, u, v, t, lam)
    srcs = [int(x) for x in rng.choice(n, 150, replace=True)]
    for sb in (0, 20):
        g = _gpu_graph(tg, n, u, v, t, lam, stats=1, sub_batch=sb)
        for win in [(0, 10**6), (50, 300)]:
            for p in ("eat", "ld", "reach"):
                _check_rows(tg, g, og, p, srcs, win, stats=(p == "eat"))
                _check_values(tg, g, og, p, srcs, win)
            hout = torch.empty((len(srcs), n), dtype=torch.int32)
            hpred = torch.empty((len(srcs), n), dtype=torch.int32)
            tg.tg_query(g.h, tg.TG_EAT, srcs, win, hout, hpred)
            for r, x in enumerate(srcs):
                A, P, _ = oracle.eat(og, x, *win)
                np.testing.assert_array_equal(tg.as_u32(hout[r]), A)
                np.testing.assert_array_equal(tg.as_u32(hpred[r]), P)
            tg.tg_query(g.h, tg.TG_LD, srcs, win, hout)
            for r, x in enumerate(srcs):
                np.testing.assert_array_equal(tg.as_u32(hout[r]), oracle.ld(og, x, *win)[0])
            # node-state engines (sub-batches <= 32): scheduled rows, device and host outputs
            few = srcs[:70]
            for p, fn in (("sp", oracle.sp), ("fp", oracle.fp), ("lds", oracle.lds)):
                dout = tg.as_u32(g.query(p, few, win))
                tg.tg_query(g.h, tg.PROBLEMS[p], few, win, hout[:len(few)])
                for r, x in enumerate(few):
                    exp = fn(og, x, *win)
                    np.testing.assert_array_equal(dout[r], exp, err_msg=f"{p} row {r}")
                    np.testing.assert_array_equal(tg.as_u32(hout[r]), exp, err_msg=f"{p} host row {r}")
        g.close()


def test_streamed_edge_cases(tg):
    """Out-of-memory graphs: no edges; every edge at one departure time (one block larger
    than block_edges); a window that excludes every block."""
    n = 40
    g = _streamed(tg, n, *(np.zeros(0, np.uint32) for _ in range(4)), block_edges=4)
    out = tg.as_u32(g.query("eat", [0, 3], (5, 9)))
    assert out[0, 0] == 5 and out[1, 3] == 5 and (out[0, 1:] == NONE).all()
    g.close()
    rng = np.random.default_rng(12)
    m = 500
    u = rng.integers(0, n, m).astype(np.uint32); v = rng.integers(0, n, m).astype(np.uint32)
    t = np.full(m, 7, np.uint32); lam = rng.integers(1, 4, m).astype(np.uint32)
    og = oracle.Graph(n, u, v, t, lam)
    g = _streamed(tg, n, u, v, t, lam, block_edges=16)
    for win in [(0, 100), (8, 100), (0, 7)]:
        _check_rows(tg, g, og, "eat", list(range(n)), win)
    g.close()
