"""Independent pins for the oracle (test side only; no oracle code is reused).

* brute_force: enumerates every legal walk inside the window
  on tiny graphs and takes min/max of the problem's objective literally.
* gx_dp: a textbook dynamic programme over an explicit time-expanded DAG
  (vertex copies at every event time, wait edges between consecutive copies,
  one travel edge per temporal edge) -- the transformation of P:L123 written
  with explicit wait edges (reading A11).
"""
from __future__ import annotations

from collections import defaultdict

NONE = 0xFFFFFFFF


def _walks_from(n, u, v, t, lam, w, x, alpha, omega):
    """All legal walks starting at x; yields (edge list). Departures strictly increase
    because lam >= 1, so the enumeration terminates."""
    m = len(u)
    out = defaultdict(list)
    for e in range(m):
        if t[e] >= alpha and int(t[e]) + int(lam[e]) <= omega:
            out[int(u[e])].append(e)
    stack = [(x, alpha, [])]  # (vertex, earliest departure allowed, path)
    while stack:
        cur, ready, path = stack.pop()
        for e in out[cur]:
            if t[e] >= ready:
                p2 = path + [e]
                yield p2
                stack.append((int(v[e]), int(t[e]) + int(lam[e]), p2))


def brute_force(n, u, v, t, lam, w, x, alpha, omega):
    """Returns dict with eat, eat_pred, sp, fp per vertex, by enumerating walks."""
    eat = [NONE] * n
    pred = [NONE] * n
    sp = [NONE] * n
    fp = [NONE] * n
    eat[x] = alpha
    sp[x] = 0
    fp[x] = 0
    for path in _walks_from(n, u, v, t, lam, w, x, alpha, omega):
        last = path[-1]
        y = int(v[last])
        if y == x:
            continue
        end = int(t[last]) + int(lam[last])
        start = int(t[path[0]])
        dist = sum(int(w[e]) for e in path)
        if end < eat[y] or (end == eat[y] and last < pred[y]):
            eat[y] = end
            pred[y] = last
        sp[y] = min(sp[y], dist)
        fp[y] = min(fp[y], end - start)
    return dict(eat=eat, eat_pred=pred, sp=sp, fp=fp)


def brute_force_lds(n, u, v, t, lam, w, x, alpha, omega):
    """Single-source latest departure (reading R5): for every v != x the max start over
    legal walks x -> v in the window; x itself gets omega."""
    L = [NONE] * n
    L[x] = omega
    for path in _walks_from(n, u, v, t, lam, w, x, alpha, omega):
        y = int(v[path[-1]])
        if y == x:
            continue
        st = int(t[path[0]])
        if L[y] == NONE or st > L[y]:
            L[y] = st
    return L


def brute_force_ld(n, u, v, t, lam, w, x, alpha, omega):
    """Latest departure towards target x (reading A5): for every v != x, the max
    start over legal walks v -> x in the window; succ = min first-edge id."""
    L = [NONE] * n
    S = [NONE] * n
    L[x] = omega
    for s in range(n):
        if s == x:
            continue
        for path in _walks_from(n, u, v, t, lam, w, s, alpha, omega):
            if int(v[path[-1]]) != x:
                continue
            st = int(t[path[0]])
            f = path[0]
            if L[s] == NONE or st > L[s] or (st == L[s] and f < S[s]):
                L[s] = st
                S[s] = f
    return L, S


def gx_dp(n, u, v, t, lam, w, x, alpha, omega):
    """DP over the explicit time-expanded DAG.  Node = (vertex, time) for every
    departure/arrival event (plus (x, alpha)); wait edges join consecutive copies
    of a vertex; travel edges (u,t)->(v,t+lam) for valid temporal edges.
    Returns eat, sp, fp per vertex."""
    m = len(u)
    valid = [e for e in range(m) if t[e] >= alpha and int(t[e]) + int(lam[e]) <= omega]
    times = defaultdict(set)
    times[x].add(alpha)
    for e in valid:
        times[int(u[e])].add(int(t[e]))
        times[int(v[e])].add(int(t[e]) + int(lam[e]))
    nodes = sorted(((tt, vv) for vv, ts in times.items() for tt in ts))
    INF = float("inf")
    dist = {nd: INF for nd in nodes}     # SP
    ls = {nd: -INF for nd in nodes}      # latest start (FP)
    reach = {nd: False for nd in nodes}  # EAT
    for tt in times[x]:
        if tt >= alpha:
            dist[(tt, x)] = 0
            ls[(tt, x)] = tt
            reach[(tt, x)] = True
    travel = defaultdict(list)
    for e in valid:
        travel[(int(t[e]), int(u[e]))].append(e)
    prev_of = {}
    for vv, ts in times.items():
        s = sorted(ts)
        for a, b in zip(s, s[1:]):
            prev_of[(b, vv)] = (a, vv)
    eat = [NONE] * n
    sp = [NONE] * n
    fp = [NONE] * n
    eat[x] = alpha
    sp[x] = 0
    fp[x] = 0
    # topological order = ascending time (wait and travel edges go strictly forward;
    # a wait predecessor (a,vv) has a < tt so it is final when (tt,vv) is visited)
    incoming = defaultdict(list)
    for e in valid:
        incoming[(int(t[e]) + int(lam[e]), int(v[e]))].append(e)
    for nd in nodes:
        tt, vv = nd
        if nd in prev_of:
            p = prev_of[nd]
            dist[nd] = min(dist[nd], dist[p])
            ls[nd] = max(ls[nd], ls[p])
            reach[nd] = reach[nd] or reach[p]
        for e in incoming[nd]:
            src = (int(t[e]), int(u[e]))
            if reach[src]:
                reach[nd] = True
                d = dist[src] + int(w[e])
                dist[nd] = min(dist[nd], d)
                ls[nd] = max(ls[nd], ls[src])
                if vv != x:
                    eat[vv] = min(eat[vv], tt)
                    sp[vv] = min(sp[vv], d)
                    fp[vv] = min(fp[vv], tt - ls[src])
    return dict(eat=eat, sp=sp, fp=fp)
