"""Pins for the oracle (CPU only): values the paper fixes (Figure-1 fixture),
brute force over legal walks, an explicit time-expanded-DAG DP, closed forms
from textbook special cases, and invariants.  None of these re-types the
oracle's scan.
"""
import json
import os

import numpy as np
import pytest
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import shortest_path

import oracle
import tgsynth
from tests.pins import NONE, brute_force, brute_force_ld, brute_force_lds, gx_dp

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "figure1.json")


def fig1():
    d = json.load(open(GOLDEN))
    names = d["vertices"]
    ix = {s: i for i, s in enumerate(names)}
    E = d["edges"]
    g = oracle.Graph(len(names), [ix[a] for a, _, _, _ in E], [ix[b] for _, b, _, _ in E],
                     [e[2] for e in E], [e[3] for e in E])
    return d, g, ix


# --------------------------------------------------------------------------- Figure 1
def _expect(n, ix, values, default=NONE):
    exp = np.full(n, default, np.uint32)
    for k, val in values.items():
        exp[ix[k]] = val
    return exp


def test_figure1_queries():
    d, g, ix = fig1()
    for q in d["queries"]:
        x = ix[q["source"]]
        a, o = q["window"]
        exp = _expect(g.n, ix, q["values"])
        if q["problem"] == "eat":
            A, P, _ = oracle.eat(g, x, a, o)
            np.testing.assert_array_equal(A, exp)
            if "pred" in q:
                np.testing.assert_array_equal(P, _expect(g.n, ix, q["pred"]))
        elif q["problem"] == "ld":
            L, S, _ = oracle.ld(g, x, a, o)
            np.testing.assert_array_equal(L, exp)
            np.testing.assert_array_equal(S, _expect(g.n, ix, q["pred"]))
        elif q["problem"] == "sp":
            np.testing.assert_array_equal(oracle.sp(g, x, a, o), exp)
        elif q["problem"] == "fp":
            np.testing.assert_array_equal(oracle.fp(g, x, a, o), exp)


def test_figure1_legality_statements():
    _, g, ix = fig1()
    # P:L106 / P:L121 / P:L140: from C the walk (C,B,5,6) -> (B,A,3,4) is illegal; A unreached.
    A, _, _ = oracle.eat(g, ix["C"])
    assert A[ix["A"]] == NONE and A[ix["B"]] == 6 and A[ix["D"]] == 7
    # from root (B,3) the chain (B,3)->(C,5)->(B,6)->(D,7) reaches C, B and D.
    A, _, _ = oracle.eat(g, ix["B"], 3, 100)
    assert A[ix["C"]] == 4 and A[ix["D"]] == 7


def test_figure1_chains_alg1():
    d, g, _ = fig1()
    off, edges = oracle.chains(g)
    got = [edges[off[i]:off[i + 1]].tolist() for i in range(len(off) - 1)]
    assert got == d["chains"]["edge_sequences"]


def test_figure1_shortcuts_alg2():
    # Chain (B,3)->(C,5)->(B,6)->(D,7): shortcut (B,3)->(D,7), sum of W_e = 3,
    # elapsed 7-3 = 4; the one-edge chain (I,4)->(J,5) is its own shortcut (Alg. 2 line 8).
    d, g, _ = fig1()
    off, edges = oracle.chains(g)
    sc = oracle.shortcuts(g, off, edges)
    seqs = d["chains"]["edge_sequences"]
    k = seqs.index([4, 1, 2])
    assert (sc["tail_v"][k], sc["arr"][k], sc["sum_w"][k], sc["elapsed"][k], sc["len"][k]) == (3, 7, 3, 4, 3)
    k = seqs.index([0])
    assert (sc["tail_v"][k], sc["arr"][k], sc["sum_w"][k], sc["len"][k]) == (7, 5, 1, 1)


# --------------------------------------------------------------------------- brute force
def _windows(seed):
    rng = np.random.default_rng(seed + 12345)
    a = int(rng.integers(0, 4))
    o = int(rng.integers(a, 13))
    return [(0, 100), (a, o)]


@pytest.mark.parametrize("block", range(8))
def test_bruteforce_eat_sp_fp(block):
    for seed in range(block * 150, (block + 1) * 150):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed)
        g = oracle.Graph(n, u, v, t, lam, w)
        for (a, o) in _windows(seed):
            for x in range(min(n, 3)):
                bf = brute_force(n, u, v, t, lam, w, x, a, o)
                A, P, W = oracle.eat(g, x, a, o)
                assert A.tolist() == bf["eat"], (seed, x, a, o)
                assert P.tolist() == bf["eat_pred"], (seed, x, a, o)
                assert oracle.sp(g, x, a, o).tolist() == bf["sp"], (seed, x, a, o)
                assert oracle.fp(g, x, a, o).tolist() == bf["fp"], (seed, x, a, o)
                # W = valid edges whose tail is reached by the departure time
                Wbf = sum(1 for e in range(len(u)) if t[e] >= a and int(t[e]) + int(lam[e]) <= o
                          and bf["eat"][u[e]] != NONE and bf["eat"][u[e]] <= t[e])
                assert W == Wbf


@pytest.mark.parametrize("block", range(4))
def test_bruteforce_ld(block):
    for seed in range(block * 100, (block + 1) * 100):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 50000, n_max=6, m_max=12)
        g = oracle.Graph(n, u, v, t, lam, w)
        for (a, o) in _windows(seed):
            for x in range(min(n, 2)):
                L, S, _ = oracle.ld(g, x, a, o)
                bL, bS = brute_force_ld(n, u, v, t, lam, w, x, a, o)
                assert L.tolist() == bL and S.tolist() == bS, (seed, x, a, o)


@pytest.mark.parametrize("block", range(4))
def test_bruteforce_lds(block):
    """Single-source latest departure (f4, reading R5) against walk enumeration."""
    for seed in range(block * 150, (block + 1) * 150):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 81000)
        g = oracle.Graph(n, u, v, t, lam, w)
        for (a, o) in _windows(seed):
            for x in range(min(n, 3)):
                assert oracle.lds(g, x, a, o).tolist() == brute_force_lds(n, u, v, t, lam, w, x, a, o), \
                    (seed, x, a, o)


def test_lds_closed_form_via_eat():
    """LDS(v) = max departure time s >= alpha of x with EAT_{x,[s,omega]}(v) reached
    (a path leaving x at s or later exists), for every v != x."""
    for seed in range(200):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 9100, n_max=8, m_max=20, t_max=12)
        g = oracle.Graph(n, u, v, t, lam, w)
        for x in range(min(n, 2)):
            a, o = 1, 14
            best = np.full(n, NONE, np.int64)
            for s in sorted({int(tt) for uu, tt in zip(u, t) if uu == x and tt >= a}):
                A, _, _ = oracle.eat(g, x, s, o)
                best[A != NONE] = s  # ascending s: the last reaching s wins
            best[x] = o
            np.testing.assert_array_equal(oracle.lds(g, x, a, o), best.astype(np.uint32))


def test_topk_and_summary_plain():
    """top-K / summary of a row: hand-checked cases (ties by vertex id, the source and
    unreached excluded, padding)."""
    row = np.array([0, 5, NONE, 3, 5, 1, 3], np.uint32)
    vs, vals = oracle.topk(row, 0, 4)
    assert vs.tolist() == [5, 3, 6, 1] and vals.tolist() == [1, 3, 3, 5]
    vs, vals = oracle.topk(row, 5, 9)
    assert vs.tolist() == [0, 3, 6, 1, 4, NONE, NONE, NONE, NONE]
    assert vals.tolist()[:5] == [0, 3, 3, 5, 5]
    assert oracle.summary(row, 0) == (5, 5 + 3 + 5 + 1 + 3)


@pytest.mark.parametrize("block", range(4))
def test_gx_dp_agrees(block):
    """Larger random graphs than brute force can enumerate: explicit G_X DP."""
    for seed in range(block * 40, (block + 1) * 40):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 90000, n_max=30, m_max=160, t_max=40, lam_max=6, w_max=9)
        g = oracle.Graph(n, u, v, t, lam, w)
        for (a, o) in [(0, 1000), (5, 30)]:
            for x in range(min(n, 3)):
                dp = gx_dp(n, u, v, t, lam, w, x, a, o)
                A, _, _ = oracle.eat(g, x, a, o)
                assert A.tolist() == dp["eat"]
                assert oracle.sp(g, x, a, o).tolist() == dp["sp"]
                assert oracle.fp(g, x, a, o).tolist() == dp["fp"]


# --------------------------------------------------------------------------- closed forms
def _static_random(seed, n, p):
    rng = np.random.default_rng(seed)
    E = [(i, j) for i in range(n) for j in range(n) if i != j and rng.random() < p]
    return E


@pytest.mark.parametrize("seed", range(12))
def test_always_available_is_static_bfs(seed):
    """Every static edge available at every integer time, duration 1, D > n:
    EAT = FP = hop distance, SP (w = 1) = hop distance, LD = D - hops to target."""
    n = 9
    E = _static_random(seed, n, 0.2)
    D = n + 3
    nn, u, v, t, lam = tgsynth.always_available(n, E, D)
    g = oracle.Graph(nn, u, v, t, lam)
    adj = csr_matrix((np.ones(len(E)), ([a for a, _ in E], [b for _, b in E])), shape=(n, n)) if E else csr_matrix((n, n))
    hops = shortest_path(adj, unweighted=True, directed=True)
    for x in range(n):
        exp = np.array([NONE if np.isinf(h) else int(h) for h in hops[x]], np.uint32)
        A, _, _ = oracle.eat(g, x, 0, D)
        np.testing.assert_array_equal(A, exp)
        np.testing.assert_array_equal(oracle.fp(g, x, 0, D), exp)
        np.testing.assert_array_equal(oracle.sp(g, x, 0, D), exp)
        L, _, _ = oracle.ld(g, x, 0, D)
        expL = np.array([NONE if np.isinf(h) else D - int(h) for h in hops[:, x]], np.uint32)
        np.testing.assert_array_equal(L, expL)


@pytest.mark.parametrize("seed", range(12))
def test_always_available_sp_is_dijkstra(seed):
    n = 8
    E = _static_random(seed + 100, n, 0.3)
    D = n + 2
    nn, u, v, t, lam = tgsynth.always_available(n, E, D)
    rng = np.random.default_rng(seed)
    wE = rng.integers(0, 10, len(E))
    w = np.repeat(wE, D).astype(np.uint32)  # same weight at every time copy
    g = oracle.Graph(nn, u, v, t, lam, w)
    if E:
        # parallel static edges do not occur (i != j, each pair once)
        adj = csr_matrix((wE.astype(float) + 1e-9, ([a for a, _ in E], [b for _, b in E])), shape=(n, n))
    else:
        adj = csr_matrix((n, n))
    dist = shortest_path(adj, directed=True)
    for x in range(n):
        exp = np.array([NONE if np.isinf(d) else int(round(d)) for d in dist[x]], np.uint32)
        np.testing.assert_array_equal(oracle.sp(g, x, 0, D), exp)


@pytest.mark.parametrize("seed", range(12))
def test_topological_time_dag(seed):
    """Static DAG i<j with t = i, duration 1: every static path is legal, so
    SP = static Dijkstra, reachability = static reachability, and
    EAT(v) = 1 + min{p reachable (or x) : (p, v) in E}."""
    n, u, v, t, lam, w = tgsynth.topo_time_dag(seed, 12, 0.25)
    g = oracle.Graph(n, u, v, t, lam, w)
    adjw = csr_matrix((w.astype(float) + 1e-9, (u, v)), shape=(n, n))
    dist = shortest_path(adjw, directed=True)
    for x in range(n):
        exp = np.array([NONE if np.isinf(d) else int(round(d)) for d in dist[x]], np.uint32)
        np.testing.assert_array_equal(oracle.sp(g, x, 0, 10**6), exp)
        reach = ~np.isinf(dist[x])
        np.testing.assert_array_equal(oracle.reach(g, x, 0, 10**6).astype(bool), reach)
        A, _, _ = oracle.eat(g, x, 0, 10**6)
        for y in range(n):
            if y == x:
                assert A[y] == 0
                continue
            preds = [int(p) for p, q in zip(u, v) if q == y and reach[p]]
            assert A[y] == (NONE if not preds else 1 + min(preds))


def test_fp_closed_form_via_eat():
    """FP(v) = min over departure times s >= alpha of x of (EAT_{x,[s,omega]}(v) - s)."""
    for seed in range(200):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 7000, n_max=8, m_max=20, t_max=12)
        g = oracle.Graph(n, u, v, t, lam, w)
        for x in range(min(n, 2)):
            a, o = 1, 14
            best = np.full(n, NONE, np.int64)
            for s in sorted({int(tt) for uu, tt in zip(u, t) if uu == x and tt >= a}):
                A, _, _ = oracle.eat(g, x, s, o)
                r = A != NONE
                best[r] = np.minimum(best[r], A[r].astype(np.int64) - s)
            best[x] = 0
            np.testing.assert_array_equal(oracle.fp(g, x, a, o), best.astype(np.uint32))


# --------------------------------------------------------------------------- invariants
def test_pred_paths_are_legal():
    for seed in range(300):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 3000, n_max=10, m_max=30, t_max=10)
        g = oracle.Graph(n, u, v, t, lam, w)
        x, a, o = 0, 1, 12
        A, P, _ = oracle.eat(g, x, a, o)
        for y in range(n):
            if y == x or A[y] == NONE:
                assert P[y] == NONE
                continue
            path, cur = [], y
            while cur != x:
                e = P[cur]
                assert v[e] == cur and t[e] + lam[e] == A[cur] and t[e] >= a and t[e] + lam[e] <= o
                path.append(e)
                cur = int(u[e])
                assert len(path) <= n
            path.reverse()
            for e1, e2 in zip(path, path[1:]):
                assert t[e1] + lam[e1] <= t[e2]  # legal and strictly increasing departures
                assert t[e1] < t[e2]


def test_window_monotone_and_edge_order_invariant():
    rng = np.random.default_rng(5)
    for seed in range(200):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 4000, n_max=10, m_max=30, t_max=12)
        g = oracle.Graph(n, u, v, t, lam, w)
        A1, _, _ = oracle.eat(g, 0, 0, 15)
        A2, _, _ = oracle.eat(g, 0, 0, 9)
        assert np.all((A2 >= A1) | (A2 == NONE))
        assert np.all(A2[A1 == NONE] == NONE)
        perm = rng.permutation(len(u))
        gp = oracle.Graph(n, u[perm], v[perm], t[perm], lam[perm], w[perm])
        for f in (oracle.sp, oracle.fp):
            np.testing.assert_array_equal(f(g, 0, 0, 15), f(gp, 0, 0, 15))
        Ap, Pp, _ = oracle.eat(gp, 0, 0, 15)
        np.testing.assert_array_equal(A1, Ap)


def test_ld_mirror_identity():
    """Reading A5: LD(G,x,[a,o])(v) = C - EAT(G^R,x,[max(0,C-o), C-a])(v), succ = pred."""
    for seed in range(400):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 6000, n_max=8, m_max=18, t_max=10)
        if len(u) == 0:
            continue
        g = oracle.Graph(n, u, v, t, lam, w)
        gr, C = oracle.mirror(g)
        for (a, o) in [(0, 100), (2, 8), (0, C), (C + 1, C + 5)]:
            x = seed % n
            L, S, _ = oracle.ld(g, x, a, o)
            if a > C:
                exp = np.full(n, NONE, np.uint32); exp[x] = o
                np.testing.assert_array_equal(L, exp)
                continue
            A, P, _ = oracle.eat(gr, x, max(0, C - o), C - a)
            exp = np.where(A == NONE, NONE, C - A.astype(np.int64)).astype(np.uint32)
            exp[x] = o
            np.testing.assert_array_equal(L, exp)
            np.testing.assert_array_equal(S, P)


def _departure_nodes(u, t):
    return sorted(set(zip(u.tolist(), t.tolist())))


def test_chains_alg1_invariants():
    """Def. 1/2: chains partition the edges; consecutive edges are
    joined at the tail's first departure at or after arrival; every chain starts
    at a hub; inner vertices are non-hubs; every chain ends at a hub or a sink."""
    for seed in range(300):
        n, u, v, t, lam, w = tgsynth.tiny_random(seed + 8000, n_max=8, m_max=25, t_max=10)
        g = oracle.Graph(n, u, v, t, lam, w)
        off, ce = oracle.chains(g)
        m = len(u)
        assert sorted(ce.tolist()) == list(range(m))
        nodes = _departure_nodes(u, t)
        deps = {}
        for (a, tt) in nodes:
            deps.setdefault(a, []).append(tt)

        def snap(e):
            arr = int(t[e]) + int(lam[e])
            later = [tt for tt in deps.get(int(v[e]), []) if tt >= arr]
            return (int(v[e]), min(later)) if later else None

        indeg = {nd: 0 for nd in nodes}
        outdeg = {nd: 0 for nd in nodes}
        for e in range(m):
            outdeg[(int(u[e]), int(t[e]))] += 1
            s = snap(e)
            if s is not None:
                indeg[s] += 1
        hub = {nd: indeg[nd] == 0 or indeg[nd] >= 2 or outdeg[nd] >= 2 for nd in nodes}
        heads = []
        for c in range(len(off) - 1):
            seq = ce[off[c]:off[c + 1]].tolist()
            h = (int(u[seq[0]]), int(t[seq[0]]))
            assert hub[h]
            heads.append((h[0], h[1], seq[0]))
            for e1, e2 in zip(seq, seq[1:]):
                s = snap(e1)
                assert s == (int(u[e2]), int(t[e2])) and not hub[s]
            s = snap(seq[-1])
            assert s is None or hub[s]
        assert heads == sorted(heads)


def test_c1_scale_runs():
    """The C1 workload (configs[0]) finishes in seconds on the oracle."""
    ge = tgsynth.make_graph("C1")
    n, u, v, t, d, w = ge.numpy()
    g = oracle.Graph(n, u, v, t, d, w)
    A, P, W = oracle.eat(g, 0)
    assert (A != NONE).sum() > 1000 and W > 0.5 * len(u)
    off, ce = oracle.chains(g)
    assert off[-1] == len(u)


def test_time_order_is_stable_sort():
    """The oracle's counting sort (oracle_time_order) is the stable sort by t of P:L123's
    time order: identical to numpy's stable argsort, ties (many equal t) in input order,
    times spanning both 16-bit digits."""
    rng = np.random.default_rng(5)
    for m, hi in [(0, 1), (1, 5), (1000, 4), (50_000, 1 << 16), (50_000, 1 << 31), (20_000, 70_000)]:
        t = rng.integers(0, hi, m).astype(np.uint32)
        z = np.zeros(m, np.uint32)
        g = oracle.Graph(4, z, z, t, z + 1)
        np.testing.assert_array_equal(g.order, np.argsort(t, kind="stable"))
