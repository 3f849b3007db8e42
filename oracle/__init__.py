"""TempGraph oracle -- TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU implementation of the hot path's results,
written from /root/reference/PAPER.md (cited P:L<line>).  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl
reference`` legs may import this package.  It shares no code with the CUDA path
(``paper_conf_asplos_0003wh0dhwy0lyl25_b200/``) and neither imports the other.

Functions (all inputs are numpy uint32 edge arrays u, v, t, lam[, w]):

* ``eat``   earliest arrival, one-pass ascending-time scan
* ``ld``    latest departure to a target (reading A5), descending-time scan
* ``sp``    shortest path, P:L115 (dist = sum W_e), Pareto-list scan
* ``fp``    fastest path, P:L114 (duration = end - start, reading A6), Pareto-list scan
* ``reach`` reachability, P:L112 (= EAT reached)
* ``lds``   single-source latest departure (reading R5), Pareto-list scan
* ``topk`` / ``summary``  top-K nearest / (reached, sum) of a row (f4), plain numpy
* ``chains``     Alg. 1 chain partition of the transformed DAG
* ``shortcuts``  Alg. 2 shortcut generation
* ``mirror``     the reversed-time graph used by reading A5's identity (pins only)

Pins: tests/test_oracle_pins.py (brute force, G_X DP, closed forms, Figure-1).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

NONE = 0xFFFFFFFF
_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (the checker, not the product)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        u32, u64, i64 = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int64
        for name in ("oracle_eat", "oracle_ld"):
            f = getattr(lib, name)
            f.restype = i64
            f.argtypes = [u32, u64, P, P, P, P, P, u32, u32, u32, P, P]
        lib.oracle_time_order.restype = ctypes.c_int
        lib.oracle_time_order.argtypes = [u64, P, P]
        lib.oracle_sp.restype = ctypes.c_int
        lib.oracle_sp.argtypes = [u32, u64, P, P, P, P, P, P, u32, u32, u32, P]
        lib.oracle_fp.restype = ctypes.c_int
        lib.oracle_fp.argtypes = [u32, u64, P, P, P, P, P, u32, u32, u32, P]
        lib.oracle_lds.restype = ctypes.c_int
        lib.oracle_lds.argtypes = [u32, u64, P, P, P, P, P, u32, u32, u32, P]
        lib.oracle_chains.restype = i64
        lib.oracle_chains.argtypes = [u32, u64, P, P, P, P, P, P, P]
        lib.oracle_shortcuts.restype = None
        lib.oracle_shortcuts.argtypes = [i64, P, P, P, P, P, P, P, P, P, P, P, P]
        _lib = lib
    return _lib


def _u32(a):
    return np.ascontiguousarray(a, dtype=np.uint32)


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


class Graph:
    """Edge-list temporal graph: e = (u, v, t, t + lam[, w]).

    ``w`` defaults to ``lam`` (reading A7).  Sorting is done once with numpy
    (a library primitive) for ``order_ut`` by (u, t, id); ``order`` (by t, ties in
    input order) is the C counting sort ``oracle_time_order`` (pinned against
    numpy's stable argsort).
    """

    def __init__(self, n, u, v, t, lam, w=None):
        self.n = int(n)
        self.u, self.v, self.t, self.lam = _u32(u), _u32(v), _u32(t), _u32(lam)
        self.w = _u32(lam if w is None else w)
        self.m = int(self.u.shape[0])
        self._order = None
        self._order_ut = None

    @property
    def order(self):
        if self._order is None:
            order = np.empty(max(self.m, 1), np.int64)
            if _load().oracle_time_order(self.m, _p(self.t), _p(order)) != 0:
                raise MemoryError
            self._order = order[: self.m]
        return self._order

    @property
    def order_ut(self):
        if self._order_ut is None:
            ids = np.arange(self.m, dtype=np.int64)
            self._order_ut = np.ascontiguousarray(np.lexsort((ids, self.t, self.u)), dtype=np.int64)
        return self._order_ut

    def _args(self):
        return (self.n, self.m, _p(self.u), _p(self.v), _p(self.t), _p(self.lam))


def _check_query(g, x, alpha, omega):
    if not (0 <= x < g.n):
        raise ValueError("source out of range")
    if alpha > omega:
        raise ValueError("alpha > omega")


def eat(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Earliest arrival from x. Returns (A, pred, W)."""
    _check_query(g, x, alpha, omega)
    lib = _load()
    A = np.empty(g.n, np.uint32)
    P = np.empty(g.n, np.uint32)
    W = lib.oracle_eat(*g._args(), _p(g.order), x, alpha, omega, _p(A), _p(P))
    return A, P, int(W)


def ld(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Latest departure towards target x (reading A5). Returns (L, succ, W)."""
    _check_query(g, x, alpha, omega)
    lib = _load()
    L = np.empty(g.n, np.uint32)
    S = np.empty(g.n, np.uint32)
    W = lib.oracle_ld(*g._args(), _p(g.order), x, alpha, omega, _p(L), _p(S))
    return L, S, int(W)


def sp(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Shortest (minimum sum of w) legal path lengths from x."""
    _check_query(g, x, alpha, omega)
    lib = _load()
    out = np.empty(g.n, np.uint32)
    if lib.oracle_sp(*g._args(), _p(g.w), _p(g.order), x, alpha, omega, _p(out)) != 0:
        raise MemoryError
    return out


def fp(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Fastest (minimum end - start) legal path durations from x."""
    _check_query(g, x, alpha, omega)
    lib = _load()
    out = np.empty(g.n, np.uint32)
    if lib.oracle_fp(*g._args(), _p(g.order), x, alpha, omega, _p(out)) != 0:
        raise MemoryError
    return out


def lds(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Single-source latest departure (reading R5): for every v the latest departure
    from x (first edge, >= alpha) of a legal path reaching v by omega; x itself: omega."""
    _check_query(g, x, alpha, omega)
    lib = _load()
    out = np.empty(g.n, np.uint32)
    if lib.oracle_lds(*g._args(), _p(g.order), x, alpha, omega, _p(out)) != 0:
        raise MemoryError
    return out


def topk(row: np.ndarray, x: int, K: int):
    """Top-K nearest of a query row: the K reached vertices v != x
    with the smallest values, ties by vertex id; padded with (NONE, NONE).
    Returns (vertices, values) as uint32[K]."""
    row = np.asarray(row, np.uint32)
    cand = np.nonzero(row != NONE)[0]
    cand = cand[cand != x]
    order = np.lexsort((cand, row[cand]))[:K]
    vs = np.full(K, NONE, np.uint32)
    vals = np.full(K, NONE, np.uint32)
    vs[: len(order)] = cand[order]
    vals[: len(order)] = row[cand[order]]
    return vs, vals


def summary(row: np.ndarray, x: int):
    """Closeness-style row summary (f4, all-source batches): (number of reached
    vertices v != x, sum of their values) -- exact integers."""
    row = np.asarray(row, np.uint32)
    mask = row != NONE
    mask[x] = False
    return int(mask.sum()), int(row[mask].astype(np.uint64).sum())


def reach(g: Graph, x: int, alpha: int = 0, omega: int = 0x7FFFFFFE):
    """Reachability: 1 where a legal path exists, else 0."""
    A, _, _ = eat(g, x, alpha, omega)
    return (A != NONE).astype(np.uint32)


def chains(g: Graph):
    """Alg. 1 chains. Returns (chain_off int64[nc+1], chain_edges uint32[m])."""
    lib = _load()
    off = np.empty(g.m + 1, np.int64)
    edges = np.empty(max(g.m, 1), np.uint32)
    nc = lib.oracle_chains(*g._args(), _p(g.order_ut), _p(off), _p(edges))
    if nc < 0:
        raise RuntimeError(f"oracle_chains failed ({nc})")
    return off[: nc + 1].copy(), edges[: g.m].copy()


def shortcuts(g: Graph, chain_off, chain_edges):
    """Alg. 2 shortcuts, one per chain in chain order."""
    lib = _load()
    nc = int(chain_off.shape[0] - 1)
    off = np.ascontiguousarray(chain_off, np.int64)
    ce = _u32(chain_edges) if g.m else np.zeros(1, np.uint32)
    out = {k: np.empty(max(nc, 1), np.uint32) for k in ("tail_v", "arr", "last_id", "elapsed", "len")}
    sum_w = np.empty(max(nc, 1), np.uint64)
    lib.oracle_shortcuts(nc, _p(off), _p(ce), _p(g.v), _p(g.t), _p(g.lam), _p(g.w),
                         _p(out["tail_v"]), _p(out["arr"]), _p(out["last_id"]), _p(sum_w),
                         _p(out["elapsed"]), _p(out["len"]))
    res = {k: a[:nc].copy() for k, a in out.items()}
    res["sum_w"] = sum_w[:nc].copy()
    return res


def mirror(g: Graph):
    """Reading A5: G^R maps e=(u,v,t,lam) to (v,u,C-(t+lam),lam), C = max(t+lam)."""
    C = int((g.t.astype(np.int64) + g.lam).max()) if g.m else 0
    gr = Graph(g.n, g.v, g.u, (C - (g.t.astype(np.int64) + g.lam)).astype(np.uint32), g.lam, g.w)
    return gr, C
