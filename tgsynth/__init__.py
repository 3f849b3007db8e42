"""Seeded synthetic temporal-graph inputs (shared by tests, bench and smoke).

This module holds NO arithmetic of the method (no sorting into chains, no path
scans).  It only draws edge lists (u, v, t_start, duration, weight), sources and
windows with the shapes of the paper's workloads (Table 2; §5.1
P:L371) as fixed in DESIGN.md "Input recipe".

Randomness is a counter-based 32-bit hash of (seed, stream, index), written with
torch int64 ops that never overflow, so the same call gives the same bits on the
CPU and on a CUDA device.  Every array is returned as a torch.int32 tensor on the
requested device (values are non-negative and < 2^31, so they read as uint32 in
the C-ABI unchanged).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np
import torch

TMAX = 0x7FFFFFFE  # max t + duration accepted by the boundary (include/tg.h)
M32 = 0xFFFFFFFF


# --------------------------------------------------------------------------- hashing
def _mul32(x: torch.Tensor, c: int) -> torch.Tensor:
    """(x * c) mod 2^32 for 0 <= x < 2^32 without int64 overflow."""
    lo, hi = c & 0xFFFF, c >> 16
    return (x * lo + (((x * hi) & 0xFFFF) << 16)) & M32


def _mix32(x: torch.Tensor) -> torch.Tensor:
    x = x ^ (x >> 16)
    x = _mul32(x, 0x7FEB352D)
    x = x ^ (x >> 15)
    x = _mul32(x, 0x846CA68B)
    return x ^ (x >> 16)


def hash32(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """Counter-based hash in [0, 2^32) of (seed, stream, idx); idx int64 >= 0."""
    dev = idx.device
    s = torch.tensor([(seed * 0x9E3779B1 + stream * 0x85EBCA77 + 0x165667B1) & M32], dtype=torch.int64, device=dev)
    k = _mix32(_mix32(s) ^ (stream & M32))
    lo = idx & M32
    hi = idx >> 32
    return _mix32(_mix32(hi ^ k) ^ lo)


def uniform_int(seed, stream, idx, lo: int, hi: int) -> torch.Tensor:
    """Integers uniform in [lo, hi) (hi - lo < 2^31)."""
    span = hi - lo
    assert 0 < span < 2**31
    return lo + ((hash32(seed, stream, idx) * span) >> 32)


def uniform_float(seed, stream, idx) -> torch.Tensor:
    """float64 in (0, 1)."""
    return (hash32(seed, stream, idx).double() + 0.5) / 4294967296.0


# --------------------------------------------------------------------------- graphs
@dataclass
class TemporalEdges:
    n: int
    u: torch.Tensor
    v: torch.Tensor
    t: torch.Tensor
    dur: torch.Tensor
    w: torch.Tensor
    meta: dict = field(default_factory=dict)

    @property
    def m(self) -> int:
        return int(self.u.shape[0])

    def to(self, device):
        return TemporalEdges(self.n, self.u.to(device), self.v.to(device), self.t.to(device),
                             self.dur.to(device), self.w.to(device), dict(self.meta))

    def numpy(self):
        f = lambda a: None if a is None else a.cpu().numpy().astype(np.uint32)
        return self.n, f(self.u), f(self.v), f(self.t), f(self.dur), f(self.w)


def _chunks(m, chunk):
    for b in range(0, m, chunk):
        yield b, min(m, b + chunk)


def rmat_endpoints(scale: int, m: int, seed: int, a=0.57, b=0.19, c=0.19, relabel=False,
                   device="cpu", chunk=1 << 24):
    """Graph500 R-MAT (a,b,c,d) quadrant descent, one hash draw per level."""
    A = int(a * 2**32)
    AB = int((a + b) * 2**32)
    ABC = int((a + b + c) * 2**32)
    u = torch.empty(m, dtype=torch.int32, device=device)
    v = torch.empty(m, dtype=torch.int32, device=device)
    for s, e in _chunks(m, chunk):
        idx = torch.arange(s, e, dtype=torch.int64, device=device)
        uu = torch.zeros(e - s, dtype=torch.int64, device=device)
        vv = torch.zeros(e - s, dtype=torch.int64, device=device)
        for lvl in range(scale):
            r = hash32(seed, 1000 + lvl, idx)
            bu = (r >= AB).long()
            bv = ((r >= A) & (r < AB)).long() | (r >= ABC).long()
            uu = uu * 2 + bu
            vv = vv * 2 + bv
        u[s:e] = uu.int()
        v[s:e] = vv.int()
    if relabel:
        n = 1 << scale
        perm = torch.argsort(hash32(seed, 99, torch.arange(n, dtype=torch.int64, device=device)), stable=True)
        perm = perm.int()
        u = perm[u.long()]
        v = perm[v.long()]
    return u, v


def chung_lu_endpoints(n: int, m: int, seed: int, exponent=2.0, device="cpu", chunk=1 << 24):
    """Directed Chung-Lu: endpoints drawn proportionally to power-law weights
    w_i = floor(2^40 / (i+1)^(1/(exponent-1))) + 1, in-weights on a seeded
    permutation of the out-weights (integer inverse-CDF sampling)."""
    p = 1.0 / (exponent - 1.0)
    i = np.arange(n, dtype=np.float64)
    wt = np.floor(2.0**40 / np.power(i + 1.0, p)).astype(np.int64) + 1
    cum = torch.from_numpy(np.cumsum(wt)).to(device)
    total = int(cum[-1].item())
    perm_in = torch.argsort(hash32(seed, 98, torch.arange(n, dtype=torch.int64, device=device)), stable=True).int()
    perm_out = torch.argsort(hash32(seed, 97, torch.arange(n, dtype=torch.int64, device=device)), stable=True).int()
    u = torch.empty(m, dtype=torch.int32, device=device)
    v = torch.empty(m, dtype=torch.int32, device=device)
    for s, e in _chunks(m, chunk):
        idx = torch.arange(s, e, dtype=torch.int64, device=device)
        for stream, dst, perm in ((2000, u, perm_out), (2001, v, perm_in)):
            r = ((hash32(seed, stream, idx) << 30) ^ hash32(seed, stream + 10, idx)) % total
            k = torch.searchsorted(cum, r, right=True).clamp_(max=n - 1)
            dst[s:e] = perm[k]
    return u, v


def uniform_times(m, seed, t_hi, dur_lo, dur_hi, w_lo=1, w_hi=101, device="cpu", chunk=1 << 24):
    t = torch.empty(m, dtype=torch.int32, device=device)
    dur = torch.empty(m, dtype=torch.int32, device=device)
    w = torch.empty(m, dtype=torch.int32, device=device)
    for s, e in _chunks(m, chunk):
        idx = torch.arange(s, e, dtype=torch.int64, device=device)
        t[s:e] = uniform_int(seed, 3000, idx, 0, t_hi).int()
        dur[s:e] = uniform_int(seed, 3001, idx, dur_lo, dur_hi + 1).int()
        w[s:e] = uniform_int(seed, 3002, idx, w_lo, w_hi).int()
    return t, dur, w


def wikitalk_times(u, n, m, seed, T=200_448_000, device="cpu"):
    """Per-vertex activity centre c_u = floor(T * U^(1/3)) (activity grows over time);
    t = clamp(c_u + Laplace(0, T/100), 0, T-1); duration 1; w ~ U[1, 100]."""
    vid = torch.arange(n, dtype=torch.int64, device=device)
    c = torch.floor(T * torch.pow(uniform_float(seed, 4000, vid), 1.0 / 3.0)).long()
    idx = torch.arange(m, dtype=torch.int64, device=device)
    q = uniform_float(seed, 4001, idx) - 0.5
    lap = -(T / 100.0) * torch.sign(q) * torch.log1p(-2.0 * q.abs())
    t = (c[u.long()].double() + lap).round().clamp(0, T - 1).long().int()
    dur = torch.ones(m, dtype=torch.int32, device=device)
    w = uniform_int(seed, 4002, idx, 1, 101).int()
    return t, dur, w


def pick_sources(u: torch.Tensor, n: int, k: int, seed: int, include_max_outdeg=False):
    """k distinct seeded sources with out-degree >= 1."""
    deg = torch.bincount(u.long(), minlength=n)
    order = torch.argsort(hash32(seed, 77, torch.arange(n, dtype=torch.int64, device=u.device)), stable=True)
    cand = order[deg[order] > 0]
    picked = cand[:k].tolist()
    if include_max_outdeg:
        top = int(torch.argmax(deg).item())
        picked = [top] + [x for x in picked if x != top][: k - 1]
    return [int(x) for x in picked]


# --------------------------------------------------------------------------- configs
CONFIGS = {
    # BASELINE.json configs[0..4]; recipe in DESIGN.md "Input recipe"
    "C1": dict(kind="rmat", scale=14, ef=16, relabel=False, t_hi=1000, dur=(1, 16), seed=1,
               k=1, windows=[(0, TMAX), (250, 750)], problems=["eat", "ld", "fp", "sp"]),
    "C2": dict(kind="rmat", scale=20, ef=16, relabel=True, t_hi=1 << 16, dur=(1, 16), seed=2,
               k=64, windows=[(0, TMAX), (1 << 14, 3 << 14)], problems=["eat", "ld"]),
    "C3": dict(kind="wikitalk", n=1_140_149, m=7_833_140, seed=3, k=16,
               windows=[(0, TMAX), (100_224_000, 200_448_000)], problems=["eat", "ld", "fp", "sp"]),
    "C4": dict(kind="rmat", scale=24, ef=32, relabel=True, t_hi=1 << 16, dur=(1, 16), seed=4,
               k=1024, windows=[(0, TMAX)], problems=["eat"]),
    "C5": dict(kind="chunglu", n=41_652_230, m=1_468_365_182, t_hi=1 << 16, dur=(1, 15), seed=5,
               k=1, windows=[(0, TMAX)], problems=["eat"]),
}


def make_graph(name: str, device="cpu", scale_shift: int = 0) -> TemporalEdges:
    """Generate config `name`; scale_shift < 0 shrinks the graph (for fast tests)."""
    cfg = CONFIGS[name]
    seed = cfg["seed"]
    if cfg["kind"] == "rmat":
        scale = cfg["scale"] + scale_shift
        n = 1 << scale
        m = n * cfg["ef"]
        u, v = rmat_endpoints(scale, m, seed, relabel=cfg["relabel"], device=device)
        t, dur, w = uniform_times(m, seed, cfg["t_hi"], *cfg["dur"], device=device)
    elif cfg["kind"] == "wikitalk":
        f = 2.0**scale_shift
        n = max(16, int(cfg["n"] * f))
        m = max(16, int(cfg["m"] * f))
        u, v = chung_lu_endpoints(n, m, seed, device=device)
        t, dur, w = wikitalk_times(u, n, m, seed, device=device)
    elif cfg["kind"] == "chunglu":
        f = 2.0**scale_shift
        n = max(16, int(cfg["n"] * f))
        m = max(16, int(cfg["m"] * f))
        u, v = chung_lu_endpoints(n, m, seed, device=device)
        t, dur, w = uniform_times(m, seed, cfg["t_hi"], *cfg["dur"], device=device)
    else:
        raise ValueError(cfg["kind"])
    return TemporalEdges(n, u, v, t, dur, w, meta=dict(config=name, seed=seed, scale_shift=scale_shift))


def config_sources(name: str, g: TemporalEdges, k: int | None = None):
    cfg = CONFIGS[name]
    k = cfg["k"] if k is None else k
    if name == "C1":
        return [0][:k]
    return pick_sources(g.u, g.n, k, cfg["seed"], include_max_outdeg=(cfg["kind"] != "rmat"))


# --------------------------------------------------------------------------- tiny graphs for pins
def tiny_random(seed: int, n_max=7, m_max=14, t_max=8, lam_max=3, w_max=5):
    """Tiny seeded graphs for brute-force pins (numpy arrays)."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, n_max + 1))
    m = int(rng.integers(0, m_max + 1))
    u = rng.integers(0, n, m).astype(np.uint32)
    v = rng.integers(0, n, m).astype(np.uint32)
    t = rng.integers(0, t_max, m).astype(np.uint32)
    lam = rng.integers(1, lam_max + 1, m).astype(np.uint32)
    w = rng.integers(0, w_max + 1, m).astype(np.uint32)
    return n, u, v, t, lam, w


def always_available(n_static: int, static_edges, D: int):
    """Every static edge (a, b) present at every integer t in [0, D) with duration 1."""
    u, v, t = [], [], []
    for (a, b) in static_edges:
        for tt in range(D):
            u.append(a); v.append(b); t.append(tt)
    m = len(u)
    return (n_static, np.array(u, np.uint32), np.array(v, np.uint32), np.array(t, np.uint32),
            np.ones(m, np.uint32))


def topo_time_dag(seed: int, n: int, p: float, w_max=9):
    """Random static DAG on 0..n-1 (edges i<j), each edge departs at t = i, duration 1."""
    rng = np.random.default_rng(seed)
    u, v = [], []
    for i in range(n):
        for j in range(i + 1, n):
            if rng.random() < p:
                u.append(i); v.append(j)
    m = len(u)
    u = np.array(u, np.uint32); v = np.array(v, np.uint32)
    return n, u, v, u.copy(), np.ones(m, np.uint32), rng.integers(0, w_max + 1, m).astype(np.uint32)


FIGURE1_NAMES = ["A", "B", "C", "D", "F", "H", "I", "J", "K"]
