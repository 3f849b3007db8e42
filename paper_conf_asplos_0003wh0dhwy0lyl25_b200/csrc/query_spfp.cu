// query_spfp.cu -- GAC execution for SHORTEST and FASTEST paths (sm_100a).
//
// Paper: §3.1 and Alg. 3 with the per-problem hooks of
// Table 1: VInitial (root 0 / others +inf for SP),
// GenerateShortcut (sum of W_e for SP, the chain's start-preserving hop for FP,
// P:L185), Propagate (min(dst, src + w)).
//
// Unlike EAT, a chain vertex's state here depends on WHEN the path arrived, so
// the state lives on departure nodes (v, tau) of the transformed DAG (reading
// A11): dnode[q][j] = min distance (SP) or max latest start LS (FP, stored as
// key = 0xFFFFFFFE - LS so both are atomicMin).  Waiting at a vertex is the
// implicit wait edge (v, tau_i) -> (v, tau_{i+1}); it is propagated by a short
// forward scan over the vertex's later departure nodes when a node improves.
//
// Round: frontier = improved nodes.  Activate: wait-propagate each improved node
// over later nodes of its vertex (stop at the first node that is already as
// good), then expand the out-edges of all improved nodes warp-cooperatively.
// Compute: from each entered slot walk the chain ((min,+) for SP, max for FP),
// atomicMin on tail node states and on the per-vertex output; stop where the
// tail node does not improve (whoever improved it pushed it).
#include <cooperative_groups.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cstring>
#include <string>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

tg_status tg_ensure_scratch(tg_graph *g, uint32_t S, bool nodes_state);
uint32_t tg_pick_sub_batch(tg_graph *g, uint32_t k, bool nodes_state);

namespace {

constexpr int QT = 256;
constexpr uint32_t BIG_T = 256;
constexpr uint32_t CHUNK = 1024;
constexpr uint32_t WAIT_INLINE = 32;  // wait-propagation steps a lane does inline; longer walks go to k_spfp_wait
#ifndef TG_WAIT_SEG
#define TG_WAIT_SEG 128  // C3: FP 2.45 -> 0.89 ms, SP 2.95 -> 0.90 ms per 16 queries (1024: 1.18, 256: 0.92, 64: 0.89)
#endif
constexpr uint32_t WAIT_SEG = TG_WAIT_SEG;  // nodes per queued wait segment (one warp each)

struct SpP {
    const uint32_t *vnode_off, *node_t, *node_u, *node_eoff, *occ_slot, *occ_node;
    const uint4 *occ_spr;
    const int4 *slots;
    const uint32_t *slot_w, *slot_tn;
    const uint2 *lc;
    const int4 *sc;
    const unsigned long long *sc_sumw;
    uint32_t *dnode, *vout, *mark;
    uint32_t n;
    uint64_t nnodes;
    uint32_t alpha, omega;
    int use_sc;
    RoundCtl *ctl;
    uint32_t round, stamp;  // round of this launch and its dedupe stamp (host counters)
    uint32_t dev_round;     // 1: graph loop -- round = RoundCtl::round, stamp = RoundCtl::stamp + round
    unsigned long long *fr0, *fr1;
    uint4 *bigq;
    uint64_t bigcap;
    uint4 *waitq;  // long wait-propagation walks {q, next node, vertex end, value}
    uint64_t waitcap;
    unsigned long long *cnt;  // stats: [0] chain-slot relaxations [1] wait-edge steps
    int stats;
};

struct RoundV {
    uint32_t r;
    uint32_t stamp;
    const unsigned long long *fin;
    uint32_t fin_n;
    unsigned long long *fout;
    uint32_t *fout_cnt, *big_cnt, *wait_cnt;
};

__device__ __forceinline__ RoundV round_view(const SpP &P) {
    RoundV R;
    const uint32_t r = P.dev_round ? *(volatile const uint32_t *)&P.ctl->round : P.round;
    R.r = r;
    R.stamp = P.dev_round ? *(volatile const uint32_t *)&P.ctl->stamp + r : P.stamp;
    R.fin = (r & 1) ? P.fr1 : P.fr0;
    R.fout = (r & 1) ? P.fr0 : P.fr1;
    R.fin_n = *(volatile uint32_t *)&P.ctl->cnt[r & 3][0];
    R.fout_cnt = &P.ctl->cnt[(r + 1) & 3][0];
    R.big_cnt = &P.ctl->cnt[r & 3][1];
    R.wait_cnt = &P.ctl->cnt[r & 3][2];
    return R;
}

// Counters of later rounds, cleared by the first kernel of round r: round r+2's
// (its input count is written during round r+1) and round r+1's work-queue counts.
// The host reads round r+1's input count after round r; it is cleared again only in
// round r+3.
__device__ __forceinline__ void clear_later_rounds(const SpP &P, const RoundV &R) {
    if (blockIdx.x != 0) return;
    const uint32_t r = R.r;
    if (threadIdx.x < 4) P.ctl->cnt[(r + 2) & 3][threadIdx.x] = 0;
    else if (threadIdx.x < 6) P.ctl->cnt[(r + 1) & 3][threadIdx.x - 3] = 0;
}

__device__ __forceinline__ void push_node(const SpP &P, const RoundV &R, uint32_t q, uint32_t j) {
    const size_t i = (size_t)q * P.nnodes + j;
    if (atomicExch(P.mark + i, R.stamp) != R.stamp) {
        cg::coalesced_group g = cg::coalesced_threads();
        uint32_t base = 0;
        if (g.thread_rank() == 0) base = atomicAdd(R.fout_cnt, g.size());
        base = g.shfl(base, 0);
        R.fout[base + g.thread_rank()] = ((unsigned long long)q << 32) | j;
    }
}

// Walk the chain from slot s (entered with head-node value cur).
template <int MODE, bool ST>
__device__ void spfp_walk(const SpP &P, const RoundV &R, uint32_t q, uint32_t s, uint32_t s_end, uint32_t cur) {
    uint32_t *dn = P.dnode + (size_t)q * P.nnodes;
    uint32_t *vo = P.vout + (size_t)q * P.n;
    for (; s < s_end; s++) {
        if (ST) atomicAdd(P.cnt + 0, 1ull);
        const int4 sl = tg_ld_slot(P.slots + s);
        const uint32_t arr = (uint32_t)sl.y;
        if (arr > P.omega) return;
        uint32_t cand;
        uint32_t val;
        if (MODE == 1) {
            cand = cur;                          // latest start is preserved along the path
            val = arr - (0xFFFFFFFEu - cur);     // duration = end - start (reading A6)
        } else if (MODE == 2) {
            cand = cur;                          // LDS: the latest start reaching v (key = ~LS)
            val = cur;
        } else {
            cand = cur + __ldg(P.slot_w + s);    // Propagate: src + w
            val = cand;
        }
        if (vo[sl.x] > val) atomicMin(vo + sl.x, val);  // stale read is an upper bound
        const uint32_t tn = __ldg(P.slot_tn + s);
        if (tn == TG_NONE) return;  // sink
        if (__ldcg(dn + tn) <= cand) return;  // not improved (stale read is an upper bound)
        // improved as far as this read knows: min (a reduction) and push; a concurrent
        // better value only makes this walk redundant (push dedupes by stamp)
        atomicMin(dn + tn, cand);
        push_node(P, R, q, tn);     // wait propagation + other out-edges next round
        cur = cand;
    }
}

template <int MODE, bool ST>
__device__ __forceinline__ void spfp_edge(const SpP &P, const RoundV &R, uint32_t q, uint32_t p) {
    // occurrence-ordered record {v, arrival | walked flag, tail node, w}: an edge that is
    // not on a walked chain needs nothing else (no slot, weight or tail-node gathers)
    const uint4 rc = __ldg(P.occ_spr + p);
    const uint32_t j = __ldg(P.occ_node + p);
    const uint32_t cur = __ldcg(P.dnode + (size_t)q * P.nnodes + j);
    if (cur == TG_NONE) return;
    if (!(rc.y >> 31)) {
        const uint32_t arr = rc.y;
        if (arr > P.omega) return;
        if (ST) atomicAdd(P.cnt + 0, 1ull);
        uint32_t cand, val;
        if (MODE == 1) { cand = cur; val = arr - (0xFFFFFFFEu - cur); }
        else if (MODE == 2) { cand = cur; val = cur; }
        else { cand = cur + rc.w; val = cand; }
        uint32_t *vo = P.vout + (size_t)q * P.n;
        if (vo[rc.x] > val) atomicMin(vo + rc.x, val);
        const uint32_t tn = rc.z;
        if (tn == TG_NONE) return;
        uint32_t *dn = P.dnode + (size_t)q * P.nnodes;
        if (__ldcg(dn + tn) <= cand) return;
        atomicMin(dn + tn, cand);
        push_node(P, R, q, tn);
        return;
    }
    const uint32_t s = __ldg(P.occ_slot + p);
    const int4 sl = tg_ld_slot(P.slots + s);
    if ((uint32_t)sl.y > P.omega) return;
    uint32_t s_end = s + 1;
    if ((uint32_t)sl.w != TG_SINGLE) {
        const uint32_t l = (uint32_t)sl.w;
        const uint2 info = __ldg(P.lc + l);
        s_end = info.x + info.y;
        if (P.use_sc && s == info.x) {
            // skeleton: Propagate(S_l) head -> tail with the shortcut weight (Alg. 2 / Alg. 3 line 6)
            const int4 scv = __ldg(P.sc + l);
            if ((uint32_t)scv.y <= P.omega) {
                const uint32_t tn = __ldg(P.slot_tn + s_end - 1);
                uint32_t cand;
                if (MODE == 1) {
                    cand = cur;
                    atomicMin(P.vout + (size_t)q * P.n + scv.x, (uint32_t)scv.y - (0xFFFFFFFEu - cur));
                } else if (MODE == 2) {
                    cand = cur;
                    atomicMin(P.vout + (size_t)q * P.n + scv.x, cur);
                } else {
                    cand = cur + (uint32_t)__ldg(P.sc_sumw + l);
                    atomicMin(P.vout + (size_t)q * P.n + scv.x, cand);
                }
                if (tn != TG_NONE && __ldcg(P.dnode + (size_t)q * P.nnodes + tn) > cand) {
                    atomicMin(P.dnode + (size_t)q * P.nnodes + tn, cand);
                    push_node(P, R, q, tn);
                }
            }
        }
    }
    spfp_walk<MODE, ST>(P, R, q, s, s_end, cur);
}

template <int MODE, bool ST>
__global__ void __launch_bounds__(QT) k_spfp_activate(SpP P) {
    const RoundV R = round_view(P);
    clear_later_rounds(P, R);
    const uint32_t F = R.fin_n;
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t base = gw * 32; base < F; base += nw * 32) {
        const uint32_t i = base + lane;
        uint32_t q = 0, e0 = 0, cnt = 0;
        if (i < F) {
            const unsigned long long it = R.fin[i];
            q = (uint32_t)(it >> 32);
            const uint32_t j = (uint32_t)it;
            uint32_t *dn = P.dnode + (size_t)q * P.nnodes;
            const uint32_t d = __ldcg(dn + j);
            const uint32_t u = __ldg(P.node_u + j);
            const uint32_t vend = __ldg(P.vnode_off + u + 1);
            // wait edges: later departure nodes of u inherit d (reading A11);
            // the first WAIT_INLINE nodes here, the rest by a warp in k_spfp_wait
            uint32_t jend = j + 1;
            bool more = false;
            // plain (stale-safe) reads, 4 nodes in flight: a node already at <= d stops the
            // walk (its own value is being propagated past it); a stale read that misses a
            // concurrent improvement only costs a redundant min.  The mins are reductions.
            for (uint32_t steps = 0; jend < vend;) {
                uint32_t tt[4], dd[4];
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const uint32_t jj = jend + k;
                    tt[k] = jj < vend ? __ldg(P.node_t + jj) : P.omega;
                    dd[k] = jj < vend ? __ldcg(dn + jj) : 0u;
                }
                bool stop = false;
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    if (stop) continue;
                    // no valid out-edge departs at >= omega; a node at <= d ends the walk
                    if (tt[k] >= P.omega || dd[k] <= d || steps == WAIT_INLINE) { stop = true; continue; }
                    if (ST) atomicAdd(P.cnt + 1, 1ull);
                    atomicMin(dn + jend, d);
                    jend++;
                    steps++;
                }
                if (stop) break;
            }
            // the inline budget ran out with nodes left: the rest goes to k_spfp_wait
            if (jend - (j + 1) == WAIT_INLINE && jend < vend) {
                const uint32_t tt = __ldg(P.node_t + jend), dd = __ldcg(dn + jend);
                more = tt < P.omega && dd > d;
            }
            if (more) {
                // the rest of the walk as WAIT_SEG-node segments, walked by different warps in
                // parallel: waiting from node j to ANY later node is legal, so every segment
                // applies d on its own and stops at its first node that is already as good
                // (that node's own value is being propagated past it)
                const uint32_t nseg = (vend - jend + WAIT_SEG - 1) / WAIT_SEG;
                const uint32_t k = atomicAdd(R.wait_cnt, nseg);
                // all or nothing: a partly queued walk would let its first segments write d
                // into the nodes the retry walk starts from
                const bool fits = (uint64_t)k + nseg <= P.waitcap;
                for (uint32_t c = 0; c < nseg && k + c < P.waitcap; c++)
                    P.waitq[k + c] = fits ? make_uint4(q, jend + c * WAIT_SEG, min(vend, jend + (c + 1) * WAIT_SEG), d)
                                          : make_uint4(q, vend, vend, d);  // reserved, empty
                if (!fits) push_node(P, R, q, jend - 1);  // queue full: continue next round
            }
            e0 = __ldg(P.node_eoff + j);
            cnt = __ldg(P.node_eoff + jend) - e0;
        }
        if (cnt > BIG_T) {
            const uint32_t nch = (cnt + CHUNK - 1) / CHUNK;
            const uint32_t k = atomicAdd(R.big_cnt, nch);
            for (uint32_t c = 0; c < nch; c++) {
                const uint32_t b0 = e0 + c * CHUNK, b1 = min(e0 + cnt, b0 + CHUNK);
                if (k + c < P.bigcap) P.bigq[k + c] = make_uint4(q, b0, b1, 0);
                else for (uint32_t p = b0; p < b1; p++) spfp_edge<MODE, ST>(P, R, q, p);
            }
            cnt = 0;
        }
        uint32_t incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        const uint32_t excl = incl - cnt;
        for (uint32_t gb = 0; gb < total; gb += 32) {
            const uint32_t g = gb + lane;
            uint32_t own = 0;
#pragma unroll
            for (int b = 16; b; b >>= 1) {
                const uint32_t v = __shfl_sync(0xffffffffu, incl, own + b - 1);
                if (v <= g) own += b;
            }
            own &= 31;
            const uint32_t oe0 = __shfl_sync(0xffffffffu, e0, own);
            const uint32_t oex = __shfl_sync(0xffffffffu, excl, own);
            const uint32_t oq = __shfl_sync(0xffffffffu, q, own);
            if (g < total) spfp_edge<MODE, ST>(P, R, oq, oe0 + (g - oex));
        }
    }
}

// Long wait-propagation walks: warp per walk, 32 later departure nodes of the
// vertex per step (atomicMin with the walk's value); the improved prefix's
// out-edges are queued as chunks for k_spfp_big of the same round.  Nodes past the
// first non-improving one that still improved (legal: waiting is transitive) are
// pushed to the next frontier.
template <int MODE, bool ST>
__global__ void __launch_bounds__(QT) k_spfp_wait(SpP P) {
    const RoundV R = round_view(P);
    const uint32_t NW = (uint32_t)min((uint64_t)*(volatile uint32_t *)R.wait_cnt, P.waitcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < NW; it += nw) {
        const uint4 c = P.waitq[it];
        const uint32_t q = c.x, vend = c.z, d = c.w;
        uint32_t *dn = P.dnode + (size_t)q * P.nnodes;
        const uint32_t jstart = c.y;
        uint32_t j = jstart;
        for (;;) {
            const uint32_t jj = j + lane;
            bool stop = true, improved = false;
            if (jj < vend && __ldg(P.node_t + jj) < P.omega) {
                if (ST) atomicAdd(P.cnt + 1, 1ull);
                improved = __ldcg(dn + jj) > d;  // plain read: stale-safe (see the inline walk)
                if (improved) atomicMin(dn + jj, d);
                stop = !improved;
            }
            const uint32_t sm = __ballot_sync(0xffffffffu, stop);
            const uint32_t first = sm ? (uint32_t)(__ffs(sm) - 1) : 32u;
            if (improved && (uint32_t)lane > first) push_node(P, R, q, jj);
            j += first;
            if (first < 32) break;
        }
        // out-edges of the improved nodes [jstart, j)
        if (j > jstart) {
            const uint32_t e0 = __ldg(P.node_eoff + jstart), e1 = __ldg(P.node_eoff + j);
            const uint32_t nch = (e1 - e0 + CHUNK - 1) / CHUNK;
            uint32_t k = 0;
            if (lane == 0) k = atomicAdd(R.big_cnt, nch);
            k = __shfl_sync(0xffffffffu, k, 0);
            for (uint32_t cc = lane; cc < nch; cc += 32) {
                const uint32_t b0 = e0 + cc * CHUNK, b1 = min(e1, b0 + CHUNK);
                if (k + cc < P.bigcap) P.bigq[k + cc] = make_uint4(q, b0, b1, 0);
                else for (uint32_t pp = b0; pp < b1; pp++) spfp_edge<MODE, ST>(P, R, q, pp);
            }
        }
    }
}

template <int MODE, bool ST>
__global__ void __launch_bounds__(QT) k_spfp_big(SpP P) {
    const RoundV R = round_view(P);
    const uint32_t B = (uint32_t)min((uint64_t)*(volatile uint32_t *)R.big_cnt, P.bigcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < B; it += nw) {
        const uint4 c = P.bigq[it];
        for (uint32_t p = c.y + lane; p < c.z; p += 32) spfp_edge<MODE, ST>(P, R, c.x, p);
    }
}

// VInitial: the source's departure nodes tau >= alpha get 0 (SP) / LS = tau (FP).
// round control for a new loop (before k_spfp_init pushes into buffer 1)
__global__ void k_spfp_ctl_init(RoundCtl *ctl, uint32_t stamp_base) {
    for (int i = 0; i < 4; i++)
        for (int j = 0; j < 4; j++) ctl->cnt[i][j] = 0;
    ctl->round = 1;
    ctl->stamp = stamp_base;  // graph loop: round r's stamp = stamp_base + r
}

// Graph loop: ends round r; the loop stops when the next round's input is empty.
__global__ void k_spfp_round_next(RoundCtl *ctl, cudaGraphConditionalHandle h, uint32_t limit) {
    if (threadIdx.x != 0) return;
    const uint32_t r = ctl->round;
    if (ctl->cnt[(r + 1) & 3][0] == 0 || r >= limit) {
        ctl->last = r;
        cudaGraphSetConditional(h, 0);
    } else {
        ctl->round = r + 1;
    }
}

template <int MODE>
__global__ void k_spfp_init(SpP P, const uint32_t *srcs, uint32_t S) {
    const RoundV R = round_view(P);
    const uint32_t q = blockIdx.y;
    if (q >= S) return;
    const uint32_t x = srcs[q];
    const uint32_t a = P.vnode_off[x], b = P.vnode_off[x + 1];
    const uint32_t j0 = tg_lower_bound(P.node_t, a, b, P.alpha);
    for (uint32_t j = j0 + blockIdx.x * blockDim.x + threadIdx.x; j < b; j += gridDim.x * blockDim.x) {
        const uint32_t tau = P.node_t[j];
        if (tau >= P.omega) break;
        P.dnode[(size_t)q * P.nnodes + j] = MODE ? (0xFFFFFFFEu - tau) : 0u;
        push_node(P, R, q, j);
    }
}

// SP / FP: the per-vertex minimum (source 0); LDS: latest start = ~key (source omega)
// the node-state engines' occurrence records (built once per direction, on first use)
__global__ void k_spfp_records(const uint2 *__restrict__ occ_rec, const uint32_t *__restrict__ occ_slot,
                               const uint32_t *__restrict__ slot_tn, const uint32_t *__restrict__ slot_w, uint64_t m,
                               uint4 *__restrict__ out) {
    for (uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p < m; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint2 r = occ_rec[p];
        const uint32_t s = occ_slot[p];
        out[p] = make_uint4(r.x, r.y, slot_tn[s], slot_w[s]);
    }
}

__global__ void k_spfp_extract(const uint32_t *__restrict__ vout, uint32_t n, const uint32_t *__restrict__ srcs,
                               uint32_t *__restrict__ out, const uint32_t *__restrict__ perm, int lds,
                               uint32_t omega, const uint32_t *__restrict__ rows) {
    const uint32_t q = blockIdx.y;
    const uint32_t src = srcs[q];  // caller's vertex ids
    const size_t row = rows ? rows[q] : q;  // the caller's row of this query
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const size_t i = row * n + v;
        const uint32_t x = vout[(size_t)q * n + (perm ? perm[v] : v)];
        if (lds) out[i] = (v == src) ? omega : (x == TG_NONE ? TG_NONE : 0xFFFFFFFEu - x);
        else out[i] = (v == src) ? 0u : x;
    }
}

}  // namespace

// The rounds of one SP/FP/LDS sub-batch as one CUDA graph with a conditional WHILE node
// (as the EAT family's, query_eat.cu): round number and stamp on the device, the loop ends
// when the next round's frontier is empty.  Cached on the handle by launch parameters.
template <int MODE>
static tg_status spfp_graph_rounds(tg_graph *g, QueryScratch &Q, const SpP &P, uint32_t grid, cudaStream_t s,
                                   uint32_t *rounds) {
    constexpr uint32_t LIMIT = 10000000;
    unsigned char key[sizeof(SpP) + 9];
    std::memcpy(key, &P, sizeof(SpP));
    std::memcpy(key + sizeof(SpP), &grid, 4);
    const int32_t mode = MODE;
    std::memcpy(key + sizeof(SpP) + 4, &mode, 4);
    key[sizeof(SpP) + 8] = 'S';  // the SP/FP/LDS loop
    cudaGraphExec_t exec = tg_rg_find(key, sizeof(key));
    cudaGraph_t graph = nullptr;
    bool owned = false;
    if (!exec) {
        TG_TRY_CUDA(cudaGraphCreate(&graph, 0));
        cudaGraphConditionalHandle h;
        cudaError_t e = cudaGraphConditionalHandleCreate(&h, graph, 1, cudaGraphCondAssignDefault);
        cudaGraphNodeParams cp = {};
        cp.type = cudaGraphNodeTypeConditional;
        cp.conditional.handle = h;
        cp.conditional.type = cudaGraphCondTypeWhile;
        cp.conditional.size = 1;
        cudaGraphNode_t node;
        if (e == cudaSuccess) e = cudaGraphAddNode(&node, graph, nullptr, 0, &cp);
        if (e == cudaSuccess) {
            cudaGraph_t body = cp.conditional.phGraph_out[0];
            cudaStream_t cs;
            e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
            if (e == cudaSuccess) {
                e = cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal);
                if (e == cudaSuccess) {
                    k_spfp_activate<MODE, false><<<grid, QT, 0, cs>>>(P);
                    k_spfp_wait<MODE, false><<<grid, QT, 0, cs>>>(P);
                    k_spfp_big<MODE, false><<<grid, QT, 0, cs>>>(P);
                    k_spfp_round_next<<<1, 32, 0, cs>>>(Q.ctl, h, LIMIT);
                    cudaGraph_t out = nullptr;
                    const cudaError_t e2 = cudaStreamEndCapture(cs, &out);
                    e = e2 != cudaSuccess ? e2 : cudaGetLastError();
                }
                cudaStreamDestroy(cs);
            }
        }
        if (e == cudaSuccess) e = cudaGraphInstantiate(&exec, graph, 0);
        if (e != cudaSuccess) {
            cudaGraphDestroy(graph);
            tg_set_error(std::string("SP/FP round graph: ") + cudaGetErrorString(e));
            return TG_ERR_CUDA;
        }
        owned = !tg_rg_add(key, sizeof(key), graph, exec);
    }
    cudaEvent_t ev0 = (g_tg_profile && g_tg_profile <= 2) ? tg_prof_begin(s) : nullptr;
    TG_TRY_CUDA(cudaGraphLaunch(exec, s));
    if (ev0) tg_prof_end("k_spfp_rounds (graph loop: k_spfp_activate + k_spfp_wait + k_spfp_big per round)", s, ev0);
    TG_TRY_CUDA(cudaMemcpyAsync(Q.h_ctr, Q.ctl, sizeof(RoundCtl), cudaMemcpyDeviceToHost, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    if (owned) {
        cudaGraphExecDestroy(exec);
        cudaGraphDestroy(graph);
    }
    const RoundCtl *hc = (const RoundCtl *)Q.h_ctr;
    const uint32_t last = hc->last;
    g_tg_launches += 4ull * last;
    if (hc->cnt[(last + 1) & 3][0] != 0) { tg_set_error("SP/FP rounds did not converge"); return TG_ERR_CUDA; }
    *rounds = last;
    return TG_OK;
}

template <int MODE>
static tg_status spfp_rounds(tg_graph *g, uint32_t Sb, uint32_t alpha, uint32_t omega, cudaStream_t s,
                             uint32_t *rounds_out) {
    QueryScratch &Q = g->qs;
    ChainGraph &c = g->fwd;
    const uint64_t n = g->n, nn = c.nnodes;
    if (!c.occ_spr && g->m) {
        TG_TRY(c.arena.alloc((void **)&c.occ_spr, g->m * 16));
        TG_LAUNCH(k_spfp_records, (unsigned)std::min<uint64_t>((g->m + 255) / 256, 148ull * 32), 256, 0, s, c.occ_rec,
                  c.occ_slot, c.slot_tn, c.slot_w, g->m, c.occ_spr);
    }
    TG_TRY_CUDA(cudaMemsetAsync(Q.vout, 0xFF, Sb * n * 4, s));
    if (nn) TG_TRY_CUDA(cudaMemsetAsync(Q.dnode, 0xFF, Sb * nn * 4, s));
    if (g->m == 0 || alpha >= omega) { *rounds_out = 0; return TG_OK; }
    SpP P{};
    P.vnode_off = c.vnode_off; P.node_t = c.node_t; P.node_u = c.node_u; P.node_eoff = c.node_eoff;
    P.occ_slot = c.occ_slot; P.occ_node = c.occ_node; P.occ_spr = c.occ_spr; P.slots = c.slots; P.slot_w = c.slot_w; P.slot_tn = c.slot_tn;
    P.lc = c.lc; P.sc = c.sc; P.sc_sumw = c.sc_sumw;
    P.dnode = Q.dnode; P.vout = Q.vout; P.mark = Q.mark; P.n = g->n; P.nnodes = nn;
    P.alpha = alpha; P.omega = omega; P.use_sc = (int)g->opt_shortcuts;
    P.ctl = Q.ctl; P.fr0 = Q.fr[0]; P.fr1 = Q.fr[1];
    P.bigq = Q.bigq; P.bigcap = Q.bigcap;
    P.waitq = Q.chq; P.waitcap = Q.chcap;
    P.cnt = Q.relax_cnt; P.stats = (int)g->opt_stats;
    // rounds and dedupe stamps are host counters passed with each launch (graph loop: on
    // the device, round r's stamp = the base + r); stamps only grow (marks of earlier
    // rounds and loops never match)
    const uint32_t stamp0 = ++Q.stamp;
    TG_LAUNCH(k_spfp_ctl_init, 1, 1, 0, s, Q.ctl, stamp0);
    {
        P.round = 0;  // k_spfp_init pushes with round 0's view: output buffer 1, count cnt[1][0]
        P.stamp = stamp0;
        dim3 grid(64, Sb);  // a hub source has many departure nodes
        TG_LAUNCH(k_spfp_init<MODE>, grid, 256, 0, s, P, Q.srcs_int, Sb);
    }
    const uint32_t grid = tg_grid_persistent(8);
    static const bool trace0 = getenv("TG_TRACE") != nullptr;
    if (g->opt_graph_loop && tg_graph_loop_allowed() && tg_graph_loop_worth(g) && !trace0 && !P.stats) {
        P.round = 0;
        P.stamp = 0;
        P.dev_round = 1;
        TG_TRY(spfp_graph_rounds<MODE>(g, Q, P, grid, s, rounds_out));
        Q.stamp = stamp0 + *rounds_out + 2;  // the loop used stamp0 + 1 .. stamp0 + rounds + 1
        return TG_OK;
    }
    const int group = (int)std::max<int64_t>(1, g->opt_round_group);
    uint32_t rounds = 0;
    uint32_t r = 1;
    static const bool trace = getenv("TG_TRACE") != nullptr;
    cudaEvent_t tev[4] = {};
    if (trace)
        for (auto &e : tev) cudaEventCreate(&e);
    for (;;) {
        for (int k = 0; k < (trace ? 1 : group); k++, r++) {
            P.round = r;
            P.stamp = ++Q.stamp;
            if (trace) cudaEventRecord(tev[0], s);
            if (P.stats) TG_LAUNCH_RELAX((k_spfp_activate<MODE, true>), grid, QT, 0, s, P);
            else TG_LAUNCH_RELAX((k_spfp_activate<MODE, false>), grid, QT, 0, s, P);
            if (trace) cudaEventRecord(tev[1], s);
            if (P.stats) TG_LAUNCH_RELAX((k_spfp_wait<MODE, true>), grid, QT, 0, s, P);
            else TG_LAUNCH_RELAX((k_spfp_wait<MODE, false>), grid, QT, 0, s, P);
            if (trace) cudaEventRecord(tev[2], s);
            if (P.stats) TG_LAUNCH_RELAX((k_spfp_big<MODE, true>), grid, QT, 0, s, P);
            else TG_LAUNCH_RELAX((k_spfp_big<MODE, false>), grid, QT, 0, s, P);
            if (trace) cudaEventRecord(tev[3], s);
        }
        TG_TRY_CUDA(cudaMemcpyAsync(Q.h_ctr, Q.ctl, sizeof(RoundCtl), cudaMemcpyDeviceToHost, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        const RoundCtl *h = (const RoundCtl *)Q.h_ctr;
        if (trace) {
            float ms[3] = {0, 0, 0};
            for (int i = 0; i < 3; i++) cudaEventElapsedTime(&ms[i], tev[i], tev[i + 1]);
            const uint32_t last = r - 1;
            fprintf(stderr, "[tg] %s S=%u round %u: frontier %u wait-walks %u big-chunks %u | activate %.3f wait %.3f "
                    "big %.3f ms\n", MODE == 0 ? "SP" : (MODE == 1 ? "FP" : "LDS"), Sb, last, h->cnt[last & 3][0], h->cnt[last & 3][2],
                    h->cnt[last & 3][1], ms[0], ms[1], ms[2]);
        }
        // r is the next round: its input count was written by the round just finished
        if (h->cnt[r & 3][0] == 0) { rounds = r - 1; break; }
        if (r > 10000000) { tg_set_error("SP/FP rounds did not converge"); return TG_ERR_CUDA; }
    }
    if (trace)
        for (auto &e : tev) cudaEventDestroy(e);
    *rounds_out = rounds;
    return TG_OK;
}

tg_status tg_run_spfp(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                      bool out_dev, cudaStream_t s) {
    const int mode = (p == TG_FASTEST) ? 1 : (p == TG_LD_SOURCE ? 2 : 0);
    const uint32_t S = tg_pick_sub_batch(g, k, true);
    TG_TRY(tg_ensure_scratch(g, S, true));
    QueryScratch &Q = g->qs;
    const uint64_t n = g->n;
    TG_TRY(tg_sink_begin(g, !out_dev, false));
    g->last = tg_query_stats{};
    const uint64_t launches0 = g_tg_launches;
    // sub-batch scheduling by first departure time (query_eat.cu tg_schedule_sources)
    std::vector<uint32_t> order, srcs_sched(k);
    TG_TRY(tg_schedule_sources(g, g->fwd, sources, k, w.t_alpha,
                               g->opt_order_sources && k > S && g->m > 0 && w.t_alpha < w.t_omega, order, s));
    for (uint32_t i = 0; i < k; i++) srcs_sched[i] = sources[order[i]];
    for (uint32_t b0 = 0; b0 < k; b0 += S) {
        const uint32_t Sb = std::min(S, k - b0);
        TG_TRY(tg_load_sources(g, srcs_sched.data() + b0, Sb, s));
        bool consecutive = true;
        for (uint32_t q = 0; q < Sb; q++) consecutive = consecutive && order[b0 + q] == b0 + q;
        const uint32_t *rows = nullptr;
        if (!consecutive && out_dev) {
            TG_TRY_CUDA(cudaMemcpyAsync(Q.rows, order.data() + b0, Sb * 4, cudaMemcpyHostToDevice, s));
            rows = Q.rows;
        }
        uint32_t rounds = 0;
        if (g->opt_stats) TG_TRY_CUDA(cudaMemsetAsync(Q.relax_cnt, 0, 16, s));
        if (mode == 1) TG_TRY((spfp_rounds<1>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        else if (mode == 2) TG_TRY((spfp_rounds<2>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        else TG_TRY((spfp_rounds<0>(g, Sb, w.t_alpha, w.t_omega, s, &rounds)));
        g->last.rounds = std::max(g->last.rounds, rounds);
        if (g->opt_stats) {  // chain-slot relaxations and wait-edge steps (bench roofline)
            unsigned long long h[2];
            TG_TRY_CUDA(cudaMemcpyAsync(h, Q.relax_cnt, 16, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            g->last.slots_relaxed += h[0];
            g->last.slots_union += h[1];
        }
        g->last.sub_batches++;
        const uint32_t bi = b0 / S;  // sub-batch index (staging buffer bi & 1 for host outputs)
        uint32_t *o = out_dev ? (rows ? out : out + (size_t)b0 * n) : nullptr, *no_pred = nullptr;
        TG_TRY(tg_sink_target(g, bi, !out_dev, false, &o, &no_pred, s));
        dim3 grid((unsigned)std::min<uint64_t>((n + 255) / 256, 1024), Sb);
        TG_LAUNCH(k_spfp_extract, grid, 256, 0, s, Q.vout, g->n, Q.srcs, o, g->relabeled ? g->perm : (const uint32_t *)nullptr,
                  mode == 2 ? 1 : 0, w.t_omega, rows);
        if (consecutive || out_dev)
            TG_TRY(tg_sink_flush(g, bi, out_dev ? nullptr : out + (size_t)b0 * n, nullptr, (size_t)Sb * n * 4, s));
        else
            TG_TRY(tg_sink_flush_rows(g, bi, out, nullptr, order.data() + b0, Sb, n, s));
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    TG_TRY(tg_sink_end(g));
    g->last.kernel_launches = g_tg_launches - launches0;
    return TG_OK;
}
