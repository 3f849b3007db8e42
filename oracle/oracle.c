/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, sequential CPU implementation of what the TempGraph hot path
 * computes.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header,
 * table or helper with the CUDA path (paper_conf_asplos_0003wh0dhwy0lyl25_b200/csrc).
 *
 * Citations are to /root/reference/PAPER.md as P:L<line> (section).
 *
 * Definitions followed (§2.1 "Temporal Graph" / "Temporal Path Problems"):
 *   edge e = (u, v, t, t') with t' = t + lambda, lambda = duration >= 1 (reading A2);
 *   a path e_1..e_k is legal iff t'_i <= t_{i+1}                          (reading A1);
 *   a query (x, [alpha, omega]) admits paths with alpha <= start(P) and end(P) <= omega
 *   (reading A3): an edge is valid iff t >= alpha and t + lambda <= omega.
 *   EAT  = min end(P)
 *   FP   = min duration(P) = end(P)-start(P) (reading A6)
 *   SP   = min dist(P) = sum of w_e          (reading A7)
 *   LD   = single-target latest departure    (reading A5; not in the paper, north star)
 * The algorithms are the "universal single scan over the transformed DAG along
 * topological order" of P:L123 (§2.1 "Transformation-based Execution"), in the
 * per-edge time-ordered form: edges are visited in ascending departure time t;
 * since lambda >= 1 no edge departing at t can enable another edge departing at t,
 * so the order among equal t is irrelevant.
 *
 * All values are uint32.  ORACLE_NONE = 0xFFFFFFFF marks "unreached" / "no pred".
 * The caller supplies `order`: edge indices sorted by t ascending, ties in input
 * order (oracle_time_order below: a textbook stable counting sort; pinned against
 * numpy.argsort(kind="stable") in tests/test_oracle_pins.py).
 *
 * Alg. 1 (§4.1) and Alg. 2 (§4.2) are written out for the
 * chain / shortcut parity of the transformer and skeleton generator.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_NONE 0xFFFFFFFFu

static int valid_edge(uint32_t t, uint32_t lam, uint32_t alpha, uint32_t omega) {
    /* P:L110 window [start, end]: start <= start(P), end(P) <= end (reading A3). */
    return t >= alpha && (uint64_t)t + lam <= (uint64_t)omega;
}

/* ------------------------------------------------------------------------- */
/* Stable sort of the edge indices by departure time (the "topological order" of
 * P:L123): two counting-sort passes (LSD) over the low and the high 16 bits of t.
 * Counting sort is stable, so after both passes edges are ordered by t with ties
 * in input order.  Returns -1 if the scratch allocation fails. */
int oracle_time_order(uint64_t m, const uint32_t *t, int64_t *order) {
    int64_t *tmp = (int64_t *)malloc((m ? m : 1) * sizeof(int64_t));
    uint64_t *cnt = (uint64_t *)malloc(65537 * sizeof(uint64_t));
    if (!tmp || !cnt) { free(tmp); free(cnt); return -1; }
    for (uint64_t i = 0; i < m; i++) tmp[i] = (int64_t)i;
    int64_t *src = tmp, *dst = order;
    for (int pass = 0; pass < 2; pass++) {
        const int shift = 16 * pass;
        memset(cnt, 0, 65537 * sizeof(uint64_t));
        for (uint64_t i = 0; i < m; i++) cnt[((t[src[i]] >> shift) & 0xFFFFu) + 1]++;
        for (int d = 0; d < 65536; d++) cnt[d + 1] += cnt[d];
        for (uint64_t i = 0; i < m; i++) dst[cnt[(t[src[i]] >> shift) & 0xFFFFu]++] = src[i];
        int64_t *x = src; src = dst; dst = x;
    }
    /* two passes: the result is back in tmp's partner -- src now points at it */
    if (src != order) memcpy(order, src, m * sizeof(int64_t));
    free(tmp);
    free(cnt);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Earliest-arrival.  Returns W = number of valid edges e with
 * A[u] <= t at scan time (the work count of the measurement).
 * pred = the smallest edge id among valid edges with A[u] <= t and
 * t + lambda == A[v] (reading A9). */
int64_t oracle_eat(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
                   const uint32_t *t, const uint32_t *lam, const int64_t *order,
                   uint32_t x, uint32_t alpha, uint32_t omega,
                   uint32_t *A, uint32_t *P) {
    int64_t W = 0;
    for (uint32_t i = 0; i < n; i++) { A[i] = ORACLE_NONE; P[i] = ORACLE_NONE; }
    A[x] = alpha;
    for (uint64_t k = 0; k < m; k++) {
        int64_t e = order[k];
        if (t[e] >= omega) break; /* lambda >= 1: nothing departing at >= omega can be valid */
        if (!valid_edge(t[e], lam[e], alpha, omega)) continue;
        if (A[u[e]] != ORACLE_NONE && A[u[e]] <= t[e]) {
            uint32_t arr = t[e] + lam[e];
            W++;
            if (v[e] != x && (arr < A[v[e]] || (arr == A[v[e]] && (uint32_t)e < P[v[e]]))) {
                A[v[e]] = arr;
                P[v[e]] = (uint32_t)e;
            }
        }
    }
    return W;
}

/* ------------------------------------------------------------------------- */
/* Latest-departure to a single target x (reading A5).  L[v] = latest departure
 * time t_1 >= alpha of a legal path from v that reaches x with end <= omega.
 * S[v] = the smallest id among first edges achieving L[v].  Scan in descending
 * t; NONE compares as -infinity. */
int64_t oracle_ld(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
                  const uint32_t *t, const uint32_t *lam, const int64_t *order,
                  uint32_t x, uint32_t alpha, uint32_t omega,
                  uint32_t *L, uint32_t *S) {
    int64_t W = 0;
    for (uint32_t i = 0; i < n; i++) { L[i] = ORACLE_NONE; S[i] = ORACLE_NONE; }
    L[x] = omega;
    for (uint64_t k = m; k-- > 0;) {
        int64_t e = order[k];
        if (t[e] < alpha) break;
        if (!valid_edge(t[e], lam[e], alpha, omega)) continue;
        uint32_t lv = L[v[e]];
        if (lv != ORACLE_NONE && (uint64_t)t[e] + lam[e] <= lv) {
            W++;
            uint32_t a = u[e];
            if (a != x && (L[a] == ORACLE_NONE || t[e] > L[a] || (t[e] == L[a] && (uint32_t)e < S[a]))) {
                L[a] = t[e];
                S[a] = (uint32_t)e;
            }
        }
    }
    return W;
}

/* ------------------------------------------------------------------------- */
/* Pareto lists used by SP and FP: per vertex, pairs (a, val) sorted by a
 * ascending.  For SP val = dist, strictly decreasing with a; for FP val = latest
 * start, strictly increasing with a. */
typedef struct { uint32_t a; uint32_t val; } pair_t;
typedef struct { pair_t *p; uint32_t len, cap; } plist_t;

/* index of the last pair with a <= q, or -1 */
static int64_t plist_floor(const plist_t *L, uint32_t q) {
    int64_t lo = 0, hi = (int64_t)L->len; /* first index with a > q */
    while (lo < hi) {
        int64_t mid = (lo + hi) / 2;
        if (L->p[mid].a <= q) lo = mid + 1; else hi = mid;
    }
    return lo - 1;
}

static void plist_insert_at(plist_t *L, int64_t pos, int64_t erase_end, pair_t x) {
    /* replace [pos, erase_end) by x */
    int64_t nerase = erase_end - pos;
    if (nerase == 0) {
        if (L->len == L->cap) {
            L->cap = L->cap ? L->cap * 2 : 4;
            L->p = (pair_t *)realloc(L->p, (size_t)L->cap * sizeof(pair_t));
        }
        memmove(L->p + pos + 1, L->p + pos, (size_t)(L->len - pos) * sizeof(pair_t));
        L->len++;
    } else if (nerase > 1) {
        memmove(L->p + pos + 1, L->p + erase_end, (size_t)(L->len - erase_end) * sizeof(pair_t));
        L->len -= (uint32_t)(nerase - 1);
    }
    L->p[pos] = x;
}

/* SP: (a', d') dominates (a, d) iff a' <= a and d' <= d. */
static void sp_insert(plist_t *L, uint32_t a, uint32_t d) {
    int64_t f = plist_floor(L, a);
    if (f >= 0 && L->p[f].val <= d) return; /* dominated (d decreasing: floor has min d among a' <= a) */
    int64_t pos = f + 1;                     /* first pair with a' > a ... */
    if (f >= 0 && L->p[f].a == a) pos = f;   /* ... or the equal-a pair (which has larger d) */
    int64_t end = pos;
    while (end < (int64_t)L->len && L->p[end].val >= d) end++; /* pairs it dominates */
    pair_t x = {a, d};
    plist_insert_at(L, pos, end, x);
}

/* FP: (a', s') dominates (a, s) iff a' <= a and s' >= s. */
static void fp_insert(plist_t *L, uint32_t a, uint32_t s) {
    int64_t f = plist_floor(L, a);
    if (f >= 0 && L->p[f].val >= s) return;
    int64_t pos = f + 1;
    if (f >= 0 && L->p[f].a == a) pos = f;
    int64_t end = pos;
    while (end < (int64_t)L->len && L->p[end].val <= s) end++;
    pair_t x = {a, s};
    plist_insert_at(L, pos, end, x);
}

/* Shortest path (dist(P) = sum of W_e).  out[v] = min dist,
 * out[x] = 0, unreached = NONE.  Returns 0, or -1 on allocation failure. */
int oracle_sp(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
              const uint32_t *t, const uint32_t *lam, const uint32_t *w, const int64_t *order,
              uint32_t x, uint32_t alpha, uint32_t omega, uint32_t *out) {
    plist_t *Ls = (plist_t *)calloc(n, sizeof(plist_t));
    if (!Ls) return -1;
    for (uint32_t i = 0; i < n; i++) out[i] = ORACLE_NONE;
    sp_insert(&Ls[x], alpha, 0);
    for (uint64_t k = 0; k < m; k++) {
        int64_t e = order[k];
        if (t[e] >= omega) break;
        if (!valid_edge(t[e], lam[e], alpha, omega)) continue;
        int64_t f = plist_floor(&Ls[u[e]], t[e]);
        if (f < 0) continue;
        uint32_t d = Ls[u[e]].p[f].val + w[e];
        sp_insert(&Ls[v[e]], t[e] + lam[e], d);
        if (d < out[v[e]]) out[v[e]] = d;
    }
    out[x] = 0;
    for (uint32_t i = 0; i < n; i++) free(Ls[i].p);
    free(Ls);
    return 0;
}

/* Fastest path (duration(P) = end(P) - start(P), reading A6). */
int oracle_fp(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
              const uint32_t *t, const uint32_t *lam, const int64_t *order,
              uint32_t x, uint32_t alpha, uint32_t omega, uint32_t *out) {
    plist_t *Ls = (plist_t *)calloc(n, sizeof(plist_t));
    if (!Ls) return -1;
    for (uint32_t i = 0; i < n; i++) out[i] = ORACLE_NONE;
    for (uint64_t k = 0; k < m; k++) {
        int64_t e = order[k];
        if (t[e] >= omega) break;
        if (!valid_edge(t[e], lam[e], alpha, omega)) continue;
        if (u[e] == x) fp_insert(&Ls[x], t[e], t[e]); /* a path may start here, now */
        int64_t f = plist_floor(&Ls[u[e]], t[e]);
        if (f < 0) continue;
        uint32_t s = Ls[u[e]].p[f].val;
        uint32_t arr = t[e] + lam[e];
        fp_insert(&Ls[v[e]], arr, s);
        if (arr - s < out[v[e]]) out[v[e]] = arr - s;
    }
    out[x] = 0;
    for (uint32_t i = 0; i < n; i++) free(Ls[i].p);
    free(Ls);
    return 0;
}

/* Single-SOURCE latest departure (the variant named by reading A5;
 * DESIGN.md reading R5): out[v] = the latest start(P) (departure of the first edge,
 * >= alpha) over legal paths P from x to v with end(P) <= omega; out[x] = omega;
 * unreached = NONE.  The same one-pass scan as FP: the floor of L_u at t is
 * the latest start among paths that are at u by time t (latest starts increase with
 * the arrival in a Pareto list), so every relaxation offers its start to v. */
int oracle_lds(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
               const uint32_t *t, const uint32_t *lam, const int64_t *order,
               uint32_t x, uint32_t alpha, uint32_t omega, uint32_t *out) {
    plist_t *Ls = (plist_t *)calloc(n, sizeof(plist_t));
    if (!Ls) return -1;
    for (uint32_t i = 0; i < n; i++) out[i] = ORACLE_NONE;
    for (uint64_t k = 0; k < m; k++) {
        int64_t e = order[k];
        if (t[e] >= omega) break;
        if (!valid_edge(t[e], lam[e], alpha, omega)) continue;
        if (u[e] == x) fp_insert(&Ls[x], t[e], t[e]); /* a path may start here, now */
        int64_t f = plist_floor(&Ls[u[e]], t[e]);
        if (f < 0) continue;
        uint32_t s = Ls[u[e]].p[f].val;
        fp_insert(&Ls[v[e]], t[e] + lam[e], s);
        if (out[v[e]] == ORACLE_NONE || s > out[v[e]]) out[v[e]] = s;
    }
    out[x] = omega;
    for (uint32_t i = 0; i < n; i++) free(Ls[i].p);
    free(Ls);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Alg. 1 "Chain-based Transformation on CPU" (§4.1) on the
 * transformed DAG of P:L123 / P:L204 as fixed by reading A11:
 *   DAG vertex = departure node (v, tau): a distinct (u, t) pair of some edge;
 *   edge e = (u,v,t,lambda) is a DAG edge (u,t) -> (v, tau) with tau the first
 *   departure time of v at or after t+lambda; if there is none the edge ends at a
 *   sink (v, t+lambda), which has no outgoing edges.
 *   Hub (Def. 2): in-degree 0, in-degree >= 2, or out-degree >= 2.
 * Each hub is a root; for each of its outgoing edges ChainPartitioning follows
 * the unique outgoing edge of each non-hub vertex until a hub or a sink.
 * Chains are emitted as edge-id sequences, roots in (u, t) order and each root's
 * outgoing edges in id order (chains from one root are consecutive).
 *
 * order_ut: edge ids sorted by (u, t, id) (numpy.lexsort, a library sort).
 * Outputs: chain_off[0..nchains], chain_edges[0..m).  Returns nchains, or -1. */
int64_t oracle_chains(uint32_t n, uint64_t m, const uint32_t *u, const uint32_t *v,
                      const uint32_t *t, const uint32_t *lam, const int64_t *order_ut,
                      int64_t *chain_off, uint32_t *chain_edges) {
    /* departure nodes */
    int64_t *node_of = (int64_t *)malloc((m ? m : 1) * sizeof(int64_t));   /* per edge id */
    int64_t *node_first = (int64_t *)malloc((m + 1) * sizeof(int64_t));     /* first position in order_ut */
    uint32_t *node_t = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    int64_t *vfirst = (int64_t *)malloc(((size_t)n + 1) * sizeof(int64_t)); /* nodes of v: [vfirst[v], vfirst[v+1]) */
    if (!node_of || !node_first || !node_t || !vfirst) return -1;
    int64_t nn = 0;
    for (uint32_t i = 0; i <= n; i++) vfirst[i] = -1;
    for (uint64_t k = 0; k < m; k++) {
        int64_t e = order_ut[k];
        if (k == 0 || u[e] != u[order_ut[k - 1]] || t[e] != t[order_ut[k - 1]]) {
            node_first[nn] = (int64_t)k;
            node_t[nn] = t[e];
            if (vfirst[u[e]] < 0) vfirst[u[e]] = nn;
            nn++;
        }
        node_of[e] = nn - 1;
    }
    node_first[nn] = (int64_t)m;
    vfirst[n] = nn;
    for (int64_t i = (int64_t)n - 1; i >= 0; i--) if (vfirst[i] < 0) vfirst[i] = vfirst[i + 1];

    /* DAG edge heads: tail node of each edge (or -1 for a sink) */
    int64_t *tail = (int64_t *)malloc((m ? m : 1) * sizeof(int64_t));
    uint32_t *indeg = (uint32_t *)calloc(nn ? nn : 1, sizeof(uint32_t));
    if (!tail || !indeg) return -1;
    for (uint64_t e = 0; e < m; e++) {
        uint64_t a = (uint64_t)t[e] + lam[e];
        int64_t lo = vfirst[v[e]], hi = vfirst[v[e] + 1];
        while (lo < hi) { int64_t mid = (lo + hi) / 2; if (node_t[mid] >= a) hi = mid; else lo = mid + 1; }
        tail[e] = (lo < vfirst[v[e] + 1]) ? lo : -1;
        if (tail[e] >= 0) indeg[tail[e]]++;
    }
    /* hub-vertex set H */
    char *hub = (char *)malloc(nn ? nn : 1);
    if (!hub) return -1;
    for (int64_t j = 0; j < nn; j++) {
        int64_t outdeg = node_first[j + 1] - node_first[j];
        hub[j] = (indeg[j] == 0 || indeg[j] >= 2 || outdeg >= 2);
    }
    /* Transformation((v_root, t_root), Ch) for every hub root, in node order */
    int64_t nch = 0, q = 0;
    for (int64_t j = 0; j < nn; j++) {
        if (!hub[j]) continue;
        for (int64_t k = node_first[j]; k < node_first[j + 1]; k++) { /* each outgoing neighbour */
            int64_t e = order_ut[k];
            chain_off[nch++] = q;                 /* NewChain: record the offset */
            /* ChainPartitioning: insert the edge, follow non-hub vertices */
            for (;;) {
                chain_edges[q++] = (uint32_t)e;
                int64_t nx = tail[e];
                if (nx < 0 || hub[nx]) break;      /* sink or hub: the chain ends */
                e = order_ut[node_first[nx]];      /* the unique outgoing edge of a non-hub */
            }
        }
    }
    chain_off[nch] = q;
    free(node_of); free(node_first); free(node_t); free(vfirst); free(tail); free(indeg); free(hub);
    return (q == (int64_t)m) ? nch : -2; /* -2: chains do not cover every edge once */
}

/* Alg. 2 "Shortcut Generation" (§4.2): per chain Ch_l the shortcut
 * S_l from its head (v_x, t_x) to its tail with weights folded over its edges:
 * sum of W_e (SP), the tail arrival, the elapsed time arr_last - t_first,
 * and the chain length.  A one-edge chain uses the edge itself (line 8). */
void oracle_shortcuts(int64_t nchains, const int64_t *chain_off, const uint32_t *chain_edges,
                      const uint32_t *v, const uint32_t *t, const uint32_t *lam, const uint32_t *w,
                      uint32_t *sc_tail_v, uint32_t *sc_arr, uint32_t *sc_last_id,
                      uint64_t *sc_sum_w, uint32_t *sc_elapsed, uint32_t *sc_len) {
    for (int64_t l = 0; l < nchains; l++) {
        int64_t b = chain_off[l], e = chain_off[l + 1];
        uint32_t first = chain_edges[b], last = chain_edges[e - 1];
        uint64_t sw = 0;
        if (e - b > 1) {
            for (int64_t k = b; k < e; k++) sw += w[chain_edges[k]]; /* GenerateShortcut fold */
        } else {
            sw = w[first]; /* S_l <- W_e */
        }
        sc_tail_v[l] = v[last];
        sc_arr[l] = t[last] + lam[last];
        sc_last_id[l] = last;
        sc_sum_w[l] = sw;
        sc_elapsed[l] = t[last] + lam[last] - t[first];
        sc_len[l] = (uint32_t)(e - b);
    }
}
