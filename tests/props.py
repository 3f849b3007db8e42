"""Full-size correctness certificates for EAT / LD rows, evaluated with torch on the
device (test infrastructure; independent of the CUDA path and of oracle/).

At BASELINE sizes the sequential oracle cannot produce whole rows, so a row is checked
against conditions that together determine it uniquely (PAPER.md P:L106-116 problem
statement; readings A1-A5, A9 of SURVEY §8(c)):

EAT row of source x in [alpha, omega]  (A[v] = earliest arrival, P[v] = pred edge id)
  (e1) A[x] = alpha, P[x] = NONE.
  (e2) Fixpoint: no valid edge e = (u, v, t, lam) with A[u] <= t leaves A[v] > t + lam.
       By induction over a legal path's edges, A is <= the true EAT everywhere.
  (e3) Witness: every reached v != x has P[v] = a valid edge into v with A[u] <= t and
       t + lam = A[v].  Following P strictly decreases time (lam >= 1) and ends at x, so
       A[v] is the arrival of a legal path: A >= the true EAT.  With (e2): A is exact.
  (e4) Tie rule (A9): P[v] is the smallest id among the edges satisfying (e3).
LD row of target x in [alpha, omega]  (L[u] = latest departure, S[u] = first edge id)
  (l1) L[x] = omega, S[x] = NONE.
  (l2) Fixpoint: every valid edge e = (u, v, t, lam), u != x, with L[v] reached and
       t + lam <= L[v] has L[u] reached and L[u] >= t.
  (l3) Witness: every reached u != x has S[u] = a valid edge out of u with L[v] reached,
       t + lam <= L[v] and t = L[u].
  (l4) Tie rule: S[u] is the smallest id among the edges satisfying (l3).
Edges are processed in chunks so that the int64 temporaries stay a few GB.
"""
import torch

NONE = 0xFFFFFFFF


def _i64(x):
    """uint32 bits carried in an int32 tensor -> int64 values."""
    return x.to(torch.int64) & 0xFFFFFFFF


def check_eat_row(u, v, t, d, n, x, win, A, P, chunk=1 << 26):
    """u, v, t, d: int32 device tensors [m] (uint32 bits); A, P: int32 [n] (uint32 bits)."""
    alpha, omega = win
    A = _i64(A)
    P = _i64(P)
    assert int(A[x]) == alpha and int(P[x]) == NONE, "(e1) source value / pred"
    m = u.shape[0]
    best = torch.full((n,), 1 << 40, dtype=torch.int64, device=A.device)  # min id among witnesses
    for c0 in range(0, m, chunk):
        cu, cv = _i64(u[c0:c0 + chunk]), _i64(v[c0:c0 + chunk])
        ct, cd = _i64(t[c0:c0 + chunk]), _i64(d[c0:c0 + chunk])
        arr = ct + cd
        usable = (ct >= alpha) & (arr <= omega) & (A[cu] <= ct)
        bad = usable & (A[cv] > arr)
        assert not bool(bad.any()), f"(e2) fixpoint violated at edge {c0 + int(bad.nonzero()[0])}"
        tight = usable & (A[cv] == arr) & (cv != x)
        ids = torch.arange(c0, c0 + cu.shape[0], dtype=torch.int64, device=A.device)
        best.scatter_reduce_(0, cv[tight], ids[tight], reduce="amin")
    reached = (A != NONE)
    reached[x] = False
    if bool(reached.any()):
        assert bool((P[reached] != NONE).all()), "(e3) reached vertex without pred"
        assert torch.equal(P[reached], best[reached]), "(e3/e4) pred is not the min-id witness"
    unreached = A == NONE
    assert bool((P[unreached] == NONE).all()), "unreached vertex with a pred"


def check_ld_row(u, v, t, d, n, x, win, L, S, chunk=1 << 26):
    alpha, omega = win
    L = _i64(L)
    S = _i64(S)
    assert int(L[x]) == omega and int(S[x]) == NONE, "(l1) target value / succ"
    m = u.shape[0]
    best_t = torch.full((n,), -1, dtype=torch.int64, device=L.device)
    for c0 in range(0, m, chunk):
        cu, cv = _i64(u[c0:c0 + chunk]), _i64(v[c0:c0 + chunk])
        ct, cd = _i64(t[c0:c0 + chunk]), _i64(d[c0:c0 + chunk])
        arr = ct + cd
        ok = (ct >= alpha) & (arr <= omega) & (L[cv] != NONE) & (arr <= L[cv]) & (cu != x)
        bad = ok & ((L[cu] == NONE) | (L[cu] < ct))
        assert not bool(bad.any()), f"(l2) fixpoint violated at edge {c0 + int(bad.nonzero()[0])}"
        best_t.scatter_reduce_(0, cu[ok], ct[ok], reduce="amax")
    reached = L != NONE
    reached[x] = False
    assert torch.equal(L[reached], best_t[reached]), "(l2/l3) latest departure is not attained"
    best = torch.full((n,), 1 << 40, dtype=torch.int64, device=L.device)
    for c0 in range(0, m, chunk):
        cu, cv = _i64(u[c0:c0 + chunk]), _i64(v[c0:c0 + chunk])
        ct, cd = _i64(t[c0:c0 + chunk]), _i64(d[c0:c0 + chunk])
        arr = ct + cd
        ok = (ct >= alpha) & (arr <= omega) & (L[cv] != NONE) & (arr <= L[cv]) & (cu != x) & (L[cu] == ct)
        ids = torch.arange(c0, c0 + cu.shape[0], dtype=torch.int64, device=L.device)
        best.scatter_reduce_(0, cu[ok], ids[ok], reduce="amin")
    if bool(reached.any()):
        assert torch.equal(S[reached], best[reached]), "(l3/l4) succ is not the min-id witness"
    assert bool((S[L == NONE] == NONE).all()), "unreached vertex with a succ"
