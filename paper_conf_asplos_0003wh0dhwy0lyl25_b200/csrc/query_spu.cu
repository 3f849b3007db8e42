// query_spu.cu -- SHORTEST / FASTEST / single-source LATEST DEPARTURE on (node, query-group)
// units (sm_100a): the unit/pair design of the EAT engine applied to the node-state problems.
//
// Paper: §3.1 and Alg. 3 with Table 1's hooks:
// VInitial (root 0 / others +inf for SP), GenerateShortcut (sum of W_e for SP, the
// chain's start-preserving hop for FP), Propagate (min(dst, src + w)).
//
// The state lives on departure nodes (v, tau) of the transformed DAG (reading A11), now
// interleaved over the sub-batch: dn[j * S + q] (SP: distance; FP / LDS: key = 0xFFFFFFFE -
// latest start, so every problem is a min), vout[v * S + q].  The frontier is a bitmap of
// nodes with one bit per query (a unit = a node and its <= 32 queries), so the queries that
// improved the same node in a round share one pass over its out-edges:
//   activate (warp per unit, lanes = queries): the unit's improved lanes relax the node's
//     out-edges -- one broadcast 16-byte occurrence record per edge, the head row of vout
//     and the tail node's row of dn read coalesced, the improving lanes' bits ORed into the
//     tail node's frontier word with one atomic per edge -- and then walk the wait edges
//     (v, tau_i) -> (v, tau_{i+1}): every lane carries its value to the vertex's later nodes
//     until it meets a node that is already as good (that node's own value is being
//     propagated past it), relaxing the out-edges of the nodes it improved on the way.
//     Walks longer than WALK_INLINE nodes continue as WALK_SEG-node segments, walked in
//     parallel (waiting from a node to ANY later node is legal, so every segment applies the
//     carried values on its own and stops per lane at its first node that is as good).
//   walked chains (>= walk_min edges) are followed slot by slot with the lanes whose tail
//     node improved ((min,+) for SP, the preserved latest start for FP / LDS), the shortcut
//     to the tail first (Alg. 3 line 6).
// Every update is a plain (stale-safe) read + a reduction: values only decrease.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "tg_internal.cuh"

namespace {

constexpr int UT = 256;
constexpr uint32_t WALK_INLINE = 32;  // wait-walk nodes a unit's warp walks itself
constexpr uint32_t WALK_SEG = 128;    // nodes per queued wait segment

struct SpuP {
    const uint32_t *vnode_off, *node_t, *node_u, *node_eoff, *occ_slot;
    const uint4 *occ_spr;
    const int4 *slots;
    const uint32_t *slot_w, *slot_tn;
    const uint2 *lc;
    const int4 *sc;
    const unsigned long long *sc_sumw;
    uint32_t *dn, *vout;
    uint32_t *fb[2];   // frontier words by round parity, one per node (bit = query)
    uint4 *segq;       // {record, first node, end node, lane mask}
    uint32_t *segd;    // [record * 32 + lane] carried value
    uint64_t segcap;
    uint2 *walkq;      // nodes improved by wait walks in this round: {node, lanes}
    uint64_t walkcap;
    RoundCtl *ctl;
    uint32_t round, S;
    uint64_t nnodes;
    uint32_t alpha, omega;
    int use_sc, stats;
    unsigned long long *cnt;  // stats: [0] (slot, query) relaxations [1] (wait node, query) steps
};

// the value a path carries onto the next node (cand) and the vertex output it offers (val)
template <int MODE>
__device__ __forceinline__ void offer(uint32_t cur, uint32_t arr, uint32_t w, uint32_t &cand, uint32_t &val) {
    if (MODE == 1) { cand = cur; val = arr - (0xFFFFFFFEu - cur); }  // duration = end - start (A6)
    else if (MODE == 2) { cand = cur; val = cur; }                     // LDS: the latest start
    else { cand = cur + w; val = cand; }                               // Propagate: src + w
}

// One edge (or chain) step for the lanes in `lanes`, each carrying `cur`: vertex output of
// the head, tail node state, tail frontier bit.  Returns the lanes whose tail improved.
template <int MODE>
__device__ __forceinline__ uint32_t step_edge(const SpuP &P, uint32_t lanes, uint32_t cur, uint32_t v, uint32_t arr,
                                              uint32_t w, uint32_t tn, uint32_t &cand, uint32_t *fout) {
    const int lane = threadIdx.x & 31;
    const bool on = (lanes >> lane) & 1u;
    uint32_t val;
    offer<MODE>(cur, arr, w, cand, val);
    if (on) {
        uint32_t *vo = P.vout + (size_t)v * P.S + lane;
        if (__ldcg(vo) > val) atomicMin(vo, val);
    }
    if (P.stats && lane == 0) atomicAdd(P.cnt + 0, (unsigned long long)__popc(lanes));
    if (tn == TG_NONE) return 0u;
    bool imp = false;
    if (on) {
        uint32_t *d = P.dn + (size_t)tn * P.S + lane;
        imp = __ldcg(d) > cand;
        if (imp) atomicMin(d, cand);
    }
    const uint32_t im = __ballot_sync(0xffffffffu, imp);
    if (im && lane == 0) atomicOr(fout + tn, im);  // one frontier atomic per edge
    return im;
}

// Relax out-occurrence p for the lanes in `lanes` holding `cur`.
template <int MODE>
__device__ __forceinline__ void relax_occ(const SpuP &P, uint32_t p, uint32_t lanes, uint32_t cur, uint32_t *fout) {
    const uint4 rc = __ldg(P.occ_spr + p);  // broadcast: every lane reads the same record
    if (!(rc.y >> 31)) {  // not on a walked chain: one edge
        if (rc.y > P.omega) return;
        uint32_t cand;
        step_edge<MODE>(P, lanes, cur, rc.x, rc.y, rc.w, rc.z, cand, fout);
        return;
    }
    uint32_t s = __ldg(P.occ_slot + p);
    int4 sl = tg_ld_slot(P.slots + s);
    if ((uint32_t)sl.y > P.omega) return;
    const uint32_t l = (uint32_t)sl.w;
    const uint2 info = __ldg(P.lc + l);
    const uint32_t s_end = info.x + info.y;
    if (P.use_sc && s == info.x) {
        // skeleton: Propagate(S_l) head -> tail with the shortcut weight (Alg. 2 / Alg. 3 line 6)
        const int4 scv = __ldg(P.sc + l);
        if ((uint32_t)scv.y <= P.omega) {
            uint32_t cand;
            const uint32_t w = MODE == 0 ? (uint32_t)__ldg(P.sc_sumw + l) : 0u;
            step_edge<MODE>(P, lanes, cur, (uint32_t)scv.x, (uint32_t)scv.y, w, __ldg(P.slot_tn + s_end - 1), cand, fout);
        }
    }
    // ChainEngine: slot by slot with the lanes whose tail node improved
    for (;;) {
        uint32_t cand;
        const uint32_t w = MODE == 0 ? __ldg(P.slot_w + s) : 0u;
        lanes = step_edge<MODE>(P, lanes, cur, (uint32_t)sl.x, (uint32_t)sl.y, w, __ldg(P.slot_tn + s), cand, fout);
        if (!lanes || ++s >= s_end) return;
        cur = cand;
        sl = tg_ld_slot(P.slots + s);  // the chain's next edge departs from that tail node
        if ((uint32_t)sl.y > P.omega) return;
    }
}

template <int MODE>
__device__ __forceinline__ void relax_node(const SpuP &P, uint32_t j, uint32_t lanes, uint32_t cur, uint32_t *fout) {
    const uint32_t p0 = __ldg(P.node_eoff + j), p1 = __ldg(P.node_eoff + j + 1);
    for (uint32_t p = p0; p < p1; p++) relax_occ<MODE>(P, p, lanes, cur, fout);
}

// A node the wait walk improved: its out-edges are relaxed in the same round by
// k_spu_expand (queue of {node, lanes}); a full queue falls back to the next frontier.
__device__ __forceinline__ void walked_node(const SpuP &P, uint32_t j, uint32_t lanes, uint32_t *fout) {
    const int lane = threadIdx.x & 31;
    if (lane != 0) return;
    const uint32_t k = atomicAdd(&P.ctl->cnt[P.round & (TG_RING - 1)][2], 1u);
    if (k < P.walkcap) P.walkq[k] = make_uint2(j, lanes);
    else atomicOr(fout + j, lanes);
}

// Wait walk over nodes [j, jend) of one vertex with per-lane carried values d: a lane stops
// at its first node that is already as good (that node's value is being propagated past
// it); every node it improves is queued for k_spu_expand.  Four node rows are read ahead
// (independent loads; only the stop rule is sequential).  Returns the node the walk stopped
// at (jend if it reached the end); `lanes` keeps the lanes still walking.
__device__ __forceinline__ uint32_t wait_walk(const SpuP &P, uint32_t j, uint32_t jend, uint32_t &lanes, uint32_t d,
                                              uint32_t budget, uint32_t *fout) {
    const int lane = threadIdx.x & 31;
    uint32_t steps = 0;
    while (j < jend && lanes) {
        uint32_t tt[4], x[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t jj = j + k;
            tt[k] = jj < jend ? __ldg(P.node_t + jj) : P.omega;
            x[k] = (jj < jend && ((lanes >> lane) & 1u)) ? __ldcg(P.dn + (size_t)jj * P.S + lane) : 0u;
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            if (!lanes || j >= jend) break;
            if (steps == budget) return j;
            if (tt[k] >= P.omega) return jend;  // nothing valid departs at >= omega
            const bool imp = ((lanes >> lane) & 1u) && x[k] > d;
            if (imp) atomicMin(P.dn + (size_t)j * P.S + lane, d);
            if (P.stats && lane == 0) atomicAdd(P.cnt + 1, (unsigned long long)__popc(lanes));
            lanes = __ballot_sync(0xffffffffu, imp);
            if (lanes) walked_node(P, j, lanes, fout);
            j++;
            steps++;
        }
    }
    return jend;
}

// Activation: a warp loads 32 frontier words (nodes), then for each improved node the lanes
// are its queries: relax its out-edges, walk its wait edges.
template <int MODE>
__global__ void __launch_bounds__(UT) k_spu_activate(SpuP P) {
    const uint32_t r = P.round;
    uint32_t *fin = P.fb[r & 1], *fout = P.fb[(r + 1) & 1];
    if (blockIdx.x == 0 && threadIdx.x < 4) P.ctl->cnt[(r + 1) & (TG_RING - 1)][threadIdx.x] = 0;
    uint32_t *seg_cnt = &P.ctl->cnt[r & (TG_RING - 1)][1];
    const int lane = threadIdx.x & 31;
    uint32_t my_units = 0;
    const uint64_t N = P.nnodes;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t jb = gw * 32; jb < N; jb += nw * 32) {
        const uint64_t ji = jb + lane;
        uint32_t word = ji < N ? fin[ji] : 0u;
        if (word) fin[ji] = 0u;  // consume
        uint32_t pending = __ballot_sync(0xffffffffu, word != 0);
        my_units += lane == 0 ? __popc(pending) : 0u;
        while (pending) {
            const int o = __ffs(pending) - 1;
            pending &= pending - 1;
            const uint32_t j = (uint32_t)(jb + o);
            const uint32_t lanes = __shfl_sync(0xffffffffu, word, o);
            const uint32_t d = ((lanes >> lane) & 1u) ? __ldcg(P.dn + (size_t)j * P.S + lane) : TG_NONE;
            relax_node<MODE>(P, j, lanes, d, fout);
            const uint32_t vend = __ldg(P.vnode_off + __ldg(P.node_u + j) + 1);
            uint32_t walking = lanes;  // lanes still carrying their value (the walk narrows it)
            const uint32_t stop = wait_walk(P, j + 1, vend, walking, d, WALK_INLINE, fout);
            if (stop < vend && walking) {
                // the rest of the vertex's nodes as segments walked by other warps
                const uint32_t nseg = (vend - stop + WALK_SEG - 1) / WALK_SEG;
                uint32_t k = 0;
                if (lane == 0) k = atomicAdd(seg_cnt, nseg);
                k = __shfl_sync(0xffffffffu, k, 0);
                if ((uint64_t)k + nseg <= P.segcap) {
                    for (uint32_t c = 0; c < nseg; c++) {
                        P.segd[(size_t)(k + c) * 32 + lane] = d;
                        if (lane == 0)
                            P.segq[k + c] = make_uint4(k + c, stop + c * WALK_SEG, min(vend, stop + (c + 1) * WALK_SEG), walking);
                    }
                } else {
                    // queue full: reserved entries empty, the walk finishes here
                    for (uint32_t c = lane; c < nseg && k + c < P.segcap; c += 32) P.segq[k + c] = make_uint4(0, 0, 0, 0);
                    wait_walk(P, stop, vend, walking, d, 0xFFFFFFFFu, fout);
                }
            }
        }
    }
    if (lane == 0 && my_units) atomicAdd(&P.ctl->cnt[r & (TG_RING - 1)][3], my_units);
}

__global__ void __launch_bounds__(UT) k_spu_segments(SpuP P) {
    const uint32_t r = P.round;
    uint32_t *fout = P.fb[(r + 1) & 1];
    const uint32_t B = (uint32_t)min((uint64_t)*(volatile uint32_t *)&P.ctl->cnt[r & (TG_RING - 1)][1], P.segcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < B; it += nw) {
        const uint4 c = P.segq[it];
        if (c.y >= c.z) continue;
        const uint32_t d = P.segd[(size_t)c.x * 32 + lane];
        uint32_t walking = c.w;
        wait_walk(P, c.y, c.z, walking, d, 0xFFFFFFFFu, fout);
    }
}

// Out-edges of the nodes the wait walks improved in this round, with their current values.
template <int MODE>
__global__ void __launch_bounds__(UT) k_spu_expand(SpuP P) {
    const uint32_t r = P.round;
    uint32_t *fout = P.fb[(r + 1) & 1];
    const uint32_t B = (uint32_t)min((uint64_t)*(volatile uint32_t *)&P.ctl->cnt[r & (TG_RING - 1)][2], P.walkcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < B; it += nw) {
        const uint2 c = P.walkq[it];
        const uint32_t d = ((c.y >> lane) & 1u) ? __ldcg(P.dn + (size_t)c.x * P.S + lane) : TG_NONE;
        relax_node<MODE>(P, c.x, c.y, d, fout);
    }
}

// VInitial: the source's departure nodes tau in [alpha, omega) get 0 (SP) / key of LS = tau
// (FP, LDS) and enter the frontier.
template <int MODE>
__global__ void k_spu_init(SpuP P, const uint32_t *srcs, uint32_t S) {
    const uint32_t q = blockIdx.y;
    if (q >= S) return;
    const uint32_t x = srcs[q];
    const uint32_t a = P.vnode_off[x], b = P.vnode_off[x + 1];
    const uint32_t j0 = tg_lower_bound(P.node_t, a, b, P.alpha);
    uint32_t *fout = P.fb[1];  // round 1's frontier
    for (uint32_t j = j0 + blockIdx.x * blockDim.x + threadIdx.x; j < b; j += gridDim.x * blockDim.x) {
        const uint32_t tau = P.node_t[j];
        if (tau >= P.omega) break;
        P.dn[(size_t)j * P.S + q] = MODE ? (0xFFFFFFFEu - tau) : 0u;
        atomicOr(fout + j, 1u << q);
    }
}

__global__ void k_spu_ctl(RoundCtl *ctl) {
    for (int i = 0; i < TG_RING; i++)
        for (int j = 0; j < 4; j++) ctl->cnt[i][j] = 0;
}

// rows of the caller: out[row(q)][v] from vout[v][q]; LDS un-keys, sources get 0 / omega
__global__ void k_spu_extract(const uint32_t *__restrict__ vout, uint32_t n, uint32_t S, uint32_t stride,
                              const uint32_t *__restrict__ srcs, uint32_t *__restrict__ out,
                              const uint32_t *__restrict__ perm, int lds, uint32_t omega,
                              const uint32_t *__restrict__ rows) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint32_t vi = perm ? perm[v] : v;
        for (uint32_t q = 0; q < S; q++) {
            const uint32_t x = vout[(size_t)vi * stride + q];
            const size_t row = rows ? rows[q] : q;
            uint32_t y;
            if (lds) y = (v == srcs[q]) ? omega : (x == TG_NONE ? TG_NONE : 0xFFFFFFFEu - x);
            else y = (v == srcs[q]) ? 0u : x;
            __stcs(out + row * n + v, y);
        }
    }
}

__global__ void k_spu_records(const uint2 *__restrict__ occ_rec, const uint32_t *__restrict__ occ_slot,
                              const uint32_t *__restrict__ slot_tn, const uint32_t *__restrict__ slot_w, uint64_t m,
                              uint4 *__restrict__ out) {
    for (uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p < m; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint2 r = occ_rec[p];
        const uint32_t s = occ_slot[p];
        out[p] = make_uint4(r.x, r.y, slot_tn[s], slot_w[s]);
    }
}

}  // namespace

// Sub-batch of the unit engine: up to 32 queries (one frontier word per node), fewer when
// the interleaved node state would exceed 16 GiB.
static uint32_t spu_sub_batch(tg_graph *g, uint32_t k) {
    if (g->opt_sub_batch > 0) return (uint32_t)std::min<int64_t>(std::min<int64_t>(g->opt_sub_batch, 32), k);
    const uint64_t nn = std::max<uint64_t>(g->fwd.nnodes, 1);
    uint64_t S = 32;  // node state + vertex output within a 16 GiB budget
    while (S > 1 && (nn + g->n) * S * 4 > (16ull << 30)) S >>= 1;
    return (uint32_t)std::min<uint64_t>(S, k);
}

static tg_status spu_scratch(tg_graph *g, uint32_t S) {
    UnitScratch &U = g->us;
    const uint64_t nn = g->fwd.nnodes, n = g->n;
    if (U.dn && U.S >= S && U.nn == nn && U.n == n) return TG_OK;
    TG_TRY_CUDA(cudaDeviceSynchronize());
    U.arena.free_all();
    tg_pinned_put(U.h_ctr);
    U = UnitScratch{};
    U.S = S;
    U.nn = nn;
    U.n = n;
    DevArena &A = U.arena;
    TG_TRY(A.alloc((void **)&U.dn, std::max<uint64_t>(nn, 1) * S * 4));
    TG_TRY(A.alloc((void **)&U.vout, n * S * 4));
    for (int i = 0; i < 2; i++) TG_TRY(A.alloc((void **)&U.fb[i], std::max<uint64_t>(nn, 1) * 4));
    U.segcap = std::min<uint64_t>(nn / WALK_SEG + 65536, 1ull << 24);
    TG_TRY(A.alloc((void **)&U.segq, U.segcap * 16));
    TG_TRY(A.alloc((void **)&U.segd, U.segcap * 32 * 4));
    U.walkcap = std::min<uint64_t>(nn + 65536, 1ull << 26);
    TG_TRY(A.alloc((void **)&U.walkq, U.walkcap * 8));
    TG_TRY(A.alloc((void **)&U.ctl, sizeof(RoundCtl)));
    TG_TRY(A.alloc((void **)&U.cnt, 64));
    TG_TRY(A.alloc((void **)&U.srcs, 32 * 4));
    TG_TRY(A.alloc((void **)&U.srcs_int, 32 * 4));
    TG_TRY(A.alloc((void **)&U.rows, 32 * 4));
    TG_TRY_CUDA(tg_pinned_get((void **)&U.h_ctr));
    U.bytes = A.total;
    return TG_OK;
}

template <int MODE>
static tg_status spu_rounds(tg_graph *g, uint32_t Sb, uint32_t alpha, uint32_t omega, cudaStream_t s, uint32_t *rounds_out) {
    UnitScratch &U = g->us;
    ChainGraph &c = g->fwd;
    const uint64_t n = g->n, nn = c.nnodes;
    TG_TRY_CUDA(cudaMemsetAsync(U.vout, 0xFF, n * U.S * 4, s));
    if (nn) {
        TG_TRY_CUDA(cudaMemsetAsync(U.dn, 0xFF, nn * U.S * 4, s));
        TG_TRY_CUDA(cudaMemsetAsync(U.fb[0], 0, nn * 4, s));
        TG_TRY_CUDA(cudaMemsetAsync(U.fb[1], 0, nn * 4, s));
    }
    *rounds_out = 0;
    if (g->m == 0 || alpha >= omega) return TG_OK;
    SpuP P{};
    P.vnode_off = c.vnode_off; P.node_t = c.node_t; P.node_u = c.node_u; P.node_eoff = c.node_eoff;
    P.occ_slot = c.occ_slot; P.occ_spr = c.occ_spr; P.slots = c.slots; P.slot_w = c.slot_w; P.slot_tn = c.slot_tn;
    P.lc = c.lc; P.sc = c.sc; P.sc_sumw = c.sc_sumw;
    P.dn = U.dn; P.vout = U.vout; P.fb[0] = U.fb[0]; P.fb[1] = U.fb[1];
    P.segq = U.segq; P.segd = U.segd; P.segcap = U.segcap; P.ctl = U.ctl;
    P.walkq = U.walkq; P.walkcap = U.walkcap;
    P.S = U.S; P.nnodes = nn; P.alpha = alpha; P.omega = omega;
    P.use_sc = (int)g->opt_shortcuts; P.stats = (int)g->opt_stats; P.cnt = U.cnt;
    TG_LAUNCH(k_spu_ctl, 1, 1, 0, s, U.ctl);
    {
        dim3 grid(64, Sb);  // a hub source has many departure nodes
        TG_LAUNCH(k_spu_init<MODE>, grid, 256, 0, s, P, U.srcs_int, Sb);
    }
    const uint32_t grid = tg_grid_persistent(8);
    const int group = (int)std::max<int64_t>(1, g->opt_round_group);
    uint32_t r = 1;
    for (;;) {
        for (int k = 0; k < group; k++, r++) {
            P.round = r;
            TG_LAUNCH_RELAX(k_spu_activate<MODE>, grid, UT, 0, s, P);
            TG_LAUNCH_RELAX(k_spu_segments, grid, UT, 0, s, P);
            TG_LAUNCH_RELAX(k_spu_expand<MODE>, grid, UT, 0, s, P);
        }
        TG_TRY_CUDA(cudaMemcpyAsync(U.h_ctr, U.ctl, sizeof(RoundCtl), cudaMemcpyDeviceToHost, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        const RoundCtl *h = (const RoundCtl *)U.h_ctr;
        const uint32_t last = r - 1;
        if (h->cnt[last & (TG_RING - 1)][3] == 0) {
            // the group's first round that consumed no frontier word did no work
            uint32_t first = last;
            for (uint32_t q = last + 1 - (uint32_t)group; q < last; q++)
                if (q >= 1 && h->cnt[q & (TG_RING - 1)][3] == 0) { first = q; break; }
            *rounds_out = first - 1;
            return TG_OK;
        }
        if (r > 10000000) { tg_set_error("SP/FP rounds did not converge"); return TG_ERR_CUDA; }
    }
}

tg_status tg_run_spu(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                     bool out_dev, cudaStream_t s) {
    const int mode = (p == TG_FASTEST) ? 1 : (p == TG_LD_SOURCE ? 2 : 0);
    ChainGraph &c = g->fwd;
    if (!c.occ_spr && g->m) {
        TG_TRY(c.arena.alloc((void **)&c.occ_spr, g->m * 16));
        TG_LAUNCH(k_spu_records, (unsigned)std::min<uint64_t>((g->m + 255) / 256, 148ull * 32), 256, 0, s, c.occ_rec,
                  c.occ_slot, c.slot_tn, c.slot_w, g->m, c.occ_spr);
    }
    const uint32_t S = spu_sub_batch(g, k);
    TG_TRY(spu_scratch(g, S));
    UnitScratch &U = g->us;
    const uint64_t n = g->n;
    // host outputs: one staging buffer of S rows (copied out per sub-batch)
    if (!out_dev && !U.stage) TG_TRY(U.arena.alloc((void **)&U.stage, (uint64_t)U.S * n * 4));
    g->last = tg_query_stats{};
    const uint64_t launches0 = g_tg_launches;
    std::vector<uint32_t> order, srcs_sched(k);
    TG_TRY(tg_schedule_sources(g, c, sources, k, w.t_alpha,
                               g->opt_order_sources && k > S && g->m > 0 && w.t_alpha < w.t_omega, order, s));
    for (uint32_t i = 0; i < k; i++) srcs_sched[i] = sources[order[i]];
    for (uint32_t b0 = 0; b0 < k; b0 += S) {
        const uint32_t Sb = std::min(S, k - b0);
        TG_TRY(tg_load_sources_to(g, srcs_sched.data() + b0, Sb, U.srcs, U.srcs_int, s));
        TG_TRY_CUDA(cudaMemcpyAsync(U.rows, order.data() + b0, Sb * 4, cudaMemcpyHostToDevice, s));
        if (g->opt_stats) TG_TRY_CUDA(cudaMemsetAsync(U.cnt, 0, 16, s));
        uint32_t rounds = 0;
        if (mode == 1) TG_TRY((spu_rounds<1>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        else if (mode == 2) TG_TRY((spu_rounds<2>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        else TG_TRY((spu_rounds<0>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        g->last.rounds = std::max(g->last.rounds, rounds);
        g->last.sub_batches++;
        if (g->opt_stats) {
            unsigned long long h[2];
            TG_TRY_CUDA(cudaMemcpyAsync(h, U.cnt, 16, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            g->last.slots_relaxed += h[0];
            g->last.slots_union += h[1];
        }
        // device outputs: rows straight to the caller's rows; host: staging rows 0.., then per row
        const unsigned xg = (unsigned)std::min<uint64_t>((n + 255) / 256, 148ull * 8);
        TG_LAUNCH(k_spu_extract, xg, 256, 0, s, U.vout, g->n, Sb, U.S, U.srcs, out_dev ? out : U.stage,
                  g->relabeled ? g->perm : (const uint32_t *)nullptr, mode == 2 ? 1 : 0, w.t_omega,
                  out_dev ? (const uint32_t *)U.rows : (const uint32_t *)nullptr);
        if (!out_dev)
            for (uint32_t q = 0; q < Sb; q++)
                TG_TRY_CUDA(cudaMemcpyAsync(out + (size_t)order[b0 + q] * n, U.stage + (size_t)q * n, n * 4,
                                            cudaMemcpyDeviceToHost, s));
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    g->last.kernel_launches = g_tg_launches - launches0;
    return TG_OK;
}
