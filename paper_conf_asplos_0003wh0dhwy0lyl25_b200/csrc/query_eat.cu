// query_eat.cu -- Generate-Activate-Compute execution for EAT / LD / REACH (sm_100a).
//
// Paper: Alg. 3 "Shortcut-guided Hybrid Parallel Execution" (§4.3),
// SkeletonEngine = activation (lines 1-12), ChainEngine = chain relaxation
// (lines 13-23).  Design for B200:
//
// state    st[q][v] = (arrival << 32 | pred edge id), relaxed with 64-bit atomicMin,
//          so the min word carries EAT and the smallest optimal edge id (reading A9).
// frontier (q, u) items whose arrival improved in the previous round.
// Activate (k_eat_activate, the "skeleton engine"): for an improved vertex u
//          (old -> new arrival), the out-edges of u departing in [max(new, alpha),
//          old) become usable for the first time.  They are found by binary search
//          in u's departure nodes and expanded warp-cooperatively (warp scan +
//          shuffle binary search); large ranges are split into chunks
//          (k_eat_big).  For each newly usable occurrence:
//            one-edge chain  -> relaxed at once (RemoveChain: 2-vertex
//                               chains are done by the skeleton engine);
//            longer chain    -> atomicMin on the chain's entry position per query;
//                               on the first entry the tail is relaxed through
//                               the shortcut (Alg. 2; Propagate(S_l), Alg. 3
//                               line 6); the newly entered slots [pos, old) are
//                               walked inline when short, else queued.
// Compute  (k_eat_chain, the "chain engine"): one warp per queued chain segment,
//          lanes over consecutive 16-byte slots (coalesced 512 B per step).
// Every usable valid slot is relaxed exactly once per query ("first touch"):
// activation ranges of a vertex are disjoint over rounds and chain entries only
// move backwards, so slot visits == the one-pass work count W.
#include <cooperative_groups.h>

#include <algorithm>
#include <vector>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

namespace {

constexpr int QT = 256;                 // threads per block
constexpr uint32_t BIG_T = 256;         // ranges above this are split into chunks
constexpr uint32_t CHUNK = 1024;        // edges per chunk (one warp)
constexpr uint32_t INLINE_WALK = 16;    // chain segments up to this length are walked inline

struct EatP {
    const uint32_t *vnode_off, *node_t, *node_eoff, *occ_slot;
    const int4 *slots;
    const uint2 *lc;
    const int4 *sc;
    unsigned long long *st;
    uint32_t *act, *mark, *entry;
    uint32_t n;
    uint64_t nlong;
    uint32_t alpha, omega, stamp;
    int use_sc, stats;
    const unsigned long long *fin;
    const uint32_t *fin_cnt;
    unsigned long long *fout;
    uint32_t *fout_cnt;
    uint4 *bigq;
    uint32_t *big_cnt;
    uint64_t bigcap;
    uint4 *chq;
    uint32_t *ch_cnt;
    uint64_t chcap;
    unsigned long long *relax_cnt;
};

__device__ __forceinline__ void eat_relax(const EatP &P, uint32_t q, uint32_t v, uint32_t arr, uint32_t id) {
    const size_t i = (size_t)q * P.n + v;
    const unsigned long long pk = ((unsigned long long)arr << 32) | id;
    const unsigned long long old = atomicMin(P.st + i, pk);
    if (P.stats) atomicAdd(P.relax_cnt + q, 1ull);
    if (arr < (uint32_t)(old >> 32)) {
        if (atomicExch(P.mark + i, P.stamp) != P.stamp) {
            cg::coalesced_group g = cg::coalesced_threads();
            uint32_t base = 0;
            if (g.thread_rank() == 0) base = atomicAdd(P.fout_cnt, g.size());
            base = g.shfl(base, 0);
            P.fout[base + g.thread_rank()] = ((unsigned long long)q << 32) | v;
        }
    }
}

// relax chain slots [s_begin, s_end) sequentially (stop at the window end)
__device__ __forceinline__ void eat_walk(const EatP &P, uint32_t q, uint32_t s_begin, uint32_t s_end) {
    for (uint32_t s = s_begin; s < s_end; s++) {
        int4 sl = tg_ld_slot(P.slots + s);
        if ((uint32_t)sl.y > P.omega) break;  // arrivals increase strictly along a chain
        eat_relax(P, q, (uint32_t)sl.x, (uint32_t)sl.y, (uint32_t)sl.z);
    }
}

// A newly usable occurrence p (sorted-edge position) for query q.
__device__ __forceinline__ void eat_edge(const EatP &P, uint32_t q, uint32_t p) {
    const uint32_t s = __ldg(P.occ_slot + p);
    const int4 sl = tg_ld_slot(P.slots + s);
    const uint32_t arr = (uint32_t)sl.y;
    if (arr > P.omega) return;
    if ((uint32_t)sl.w == TG_SINGLE) {
        eat_relax(P, q, (uint32_t)sl.x, arr, (uint32_t)sl.z);
        return;
    }
    const uint32_t l = (uint32_t)sl.w;
    const uint2 info = __ldg(P.lc + l);  // {first slot, length}
    const uint32_t pos = s - info.x;
    const uint32_t old = atomicMin(P.entry + (size_t)q * P.nlong + l, pos);
    if (pos >= old) return;  // already entered at or before pos
    uint32_t end = min(old, info.y);
    if (old == TG_NONE && P.use_sc) {
        // first entry: Propagate along the shortcut head -> tail (Alg. 3 line 6)
        const int4 scv = __ldg(P.sc + l);
        if ((uint32_t)scv.y <= P.omega) {
            eat_relax(P, q, (uint32_t)scv.x, (uint32_t)scv.y, (uint32_t)scv.z);
            end = info.y - 1;
        }
    }
    if (pos >= end) return;
    eat_relax(P, q, (uint32_t)sl.x, arr, (uint32_t)sl.z);
    const uint32_t s1 = info.x + end;
    if (s1 - (s + 1) > INLINE_WALK) {
        uint32_t k = atomicAdd(P.ch_cnt, 1u);
        if (k < P.chcap) {
            P.chq[k] = make_uint4(q, s + 1, s1, 0);
            return;
        }
    }
    eat_walk(P, q, s + 1, s1);
}

__global__ void __launch_bounds__(QT) k_eat_activate(EatP P) {
    const uint32_t F = *P.fin_cnt;
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t base = gw * 32; base < F; base += nw * 32) {
        const uint32_t i = base + lane;
        uint32_t q = 0, e0 = 0, cnt = 0;
        if (i < F) {
            const unsigned long long it = P.fin[i];
            q = (uint32_t)(it >> 32);
            const uint32_t u = (uint32_t)it;
            const size_t si = (size_t)q * P.n + u;
            const uint32_t now = (uint32_t)(__ldcg(P.st + si) >> 32);
            const uint32_t old = atomicMin(P.act + si, now);
            if (now < old) {
                const uint32_t lo_t = max(now, P.alpha);
                const uint32_t hi_t = min(old, P.omega);  // t + duration <= omega needs t < omega
                if (lo_t < hi_t) {
                    const uint32_t a = __ldg(P.vnode_off + u), b = __ldg(P.vnode_off + u + 1);
                    const uint32_t j0 = tg_lower_bound(P.node_t, a, b, lo_t);
                    const uint32_t j1 = tg_lower_bound(P.node_t, j0, b, hi_t);
                    e0 = __ldg(P.node_eoff + j0);
                    cnt = __ldg(P.node_eoff + j1) - e0;
                }
            }
        }
        if (cnt > BIG_T) {
            const uint32_t nch = (cnt + CHUNK - 1) / CHUNK;
            const uint32_t k = atomicAdd(P.big_cnt, nch);
            for (uint32_t c = 0; c < nch; c++) {
                const uint32_t b0 = e0 + c * CHUNK, b1 = min(e0 + cnt, b0 + CHUNK);
                if (k + c < P.bigcap) P.bigq[k + c] = make_uint4(q, b0, b1, 0);
                else for (uint32_t p = b0; p < b1; p++) eat_edge(P, q, p);  // never expected: bigcap is a bound
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
            uint32_t own = 0;  // number of lanes whose inclusive prefix <= g == owner lane
#pragma unroll
            for (int b = 16; b; b >>= 1) {
                const uint32_t v = __shfl_sync(0xffffffffu, incl, own + b - 1);
                if (v <= g) own += b;
            }
            own &= 31;
            const uint32_t oe0 = __shfl_sync(0xffffffffu, e0, own);
            const uint32_t oex = __shfl_sync(0xffffffffu, excl, own);
            const uint32_t oq = __shfl_sync(0xffffffffu, q, own);
            if (g < total) eat_edge(P, oq, oe0 + (g - oex));
        }
    }
}

__global__ void __launch_bounds__(QT) k_eat_big(EatP P) {
    const uint32_t B = (uint32_t)min((uint64_t)*P.big_cnt, P.bigcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < B; it += nw) {
        const uint4 c = P.bigq[it];
        for (uint32_t p = c.y + lane; p < c.z; p += 32) eat_edge(P, c.x, p);
    }
}

// ChainEngine: warp per queued chain segment, lanes over consecutive slots.
__global__ void __launch_bounds__(QT) k_eat_chain(EatP P) {
    const uint32_t C = (uint32_t)min((uint64_t)*P.ch_cnt, P.chcap);
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t it = gw; it < C; it += nw) {
        const uint4 c = P.chq[it];
        for (uint32_t b = c.y; b < c.z; b += 32) {
            const uint32_t s = b + lane;
            bool stop = false;
            if (s < c.z) {
                const int4 sl = tg_ld_slot(P.slots + s);
                if ((uint32_t)sl.y > P.omega) stop = true;
                else eat_relax(P, c.x, (uint32_t)sl.x, (uint32_t)sl.y, (uint32_t)sl.z);
            }
            if (__any_sync(0xffffffffu, stop)) break;
        }
    }
}

__global__ void k_eat_init(unsigned long long *st, uint32_t n, const uint32_t *srcs, uint32_t S, uint32_t alpha,
                           unsigned long long *fr, uint32_t *fr_cnt, int push) {
    // VInitial (Table 1): every state INF (memset), the source = (alpha, no pred)
    for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < S; q += gridDim.x * blockDim.x) {
        st[(size_t)q * n + srcs[q]] = ((unsigned long long)alpha << 32) | TG_NONE;
        if (push) fr[q] = ((unsigned long long)q << 32) | srcs[q];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) *fr_cnt = push ? S : 0;
}

// mode 0 = EAT, 1 = LD (mirror: value = C - time; target = omega), 2 = REACH
__global__ void k_eat_extract(const unsigned long long *__restrict__ st, uint32_t n, const uint32_t *__restrict__ srcs,
                              int mode, uint32_t C, uint32_t omega, uint32_t *__restrict__ out,
                              uint32_t *__restrict__ pred) {
    const uint32_t q = blockIdx.y;
    const uint32_t src = srcs[q];
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const size_t i = (size_t)q * n + v;
        const unsigned long long pk = st[i];
        const bool reached = pk != ~0ull;
        const uint32_t t = (uint32_t)(pk >> 32), id = (uint32_t)pk;
        uint32_t val, pr = reached ? id : TG_NONE;
        if (mode == 0) {
            val = reached ? t : TG_UNREACHED;
        } else if (mode == 1) {
            val = (v == src) ? omega : (reached ? C - t : TG_UNREACHED);
            if (v == src) pr = TG_NONE;
        } else {
            val = reached ? 1u : 0u;
        }
        out[i] = val;
        if (pred) pred[i] = pr;
    }
}

}  // namespace

static tg_status ensure_scratch(tg_graph *g, uint32_t S, bool nodes_state) {
    QueryScratch &Q = g->qs;
    const uint64_t nlong = std::max(g->fwd.nlong, g->mir.nlong);
    const uint64_t nnodes = std::max(g->fwd.nnodes, g->mir.nnodes);
    if (Q.S >= S && Q.n == g->n && Q.nlong >= nlong && (!nodes_state || Q.nodes_state)) return TG_OK;
    Q.arena.free_all();
    if (Q.h_ctr) { cudaFreeHost(Q.h_ctr); Q.h_ctr = nullptr; }
    Q = QueryScratch{};
    const uint64_t n = g->n, m = g->m;
    Q.S = S;
    Q.n = g->n;
    Q.nlong = nlong;
    Q.nnodes = nnodes;
    Q.nodes_state = nodes_state;
    DevArena &A = Q.arena;
    TG_TRY(A.alloc((void **)&Q.st, S * n * 8));
    TG_TRY(A.alloc((void **)&Q.act, S * n * 4));
    const uint64_t mark_len = S * std::max<uint64_t>(n, nodes_state ? nnodes : 0);
    TG_TRY(A.alloc((void **)&Q.mark, mark_len * 4));
    TG_TRY_CUDA(cudaMemset(Q.mark, 0, mark_len * 4));
    TG_TRY(A.alloc((void **)&Q.entry, std::max<uint64_t>(S * nlong, 1) * 4));
    Q.fcap = S * std::max<uint64_t>(n, nodes_state ? nnodes : 0) + 64;
    TG_TRY(A.alloc((void **)&Q.fr[0], Q.fcap * 8));
    TG_TRY(A.alloc((void **)&Q.fr[1], Q.fcap * 8));
    Q.bigcap = S * (m / CHUNK + std::max<uint64_t>(n, nnodes) / BIG_T + 2) + 1024;
    TG_TRY(A.alloc((void **)&Q.bigq, Q.bigcap * 16));
    Q.chcap = S * nlong + (1u << 20);
    TG_TRY(A.alloc((void **)&Q.chq, Q.chcap * 16));
    TG_TRY(A.alloc((void **)&Q.ctr, 64));
    TG_TRY_CUDA(cudaMemset(Q.ctr, 0, 64));
    TG_TRY_CUDA(cudaMallocHost((void **)&Q.h_ctr, 64));
    TG_TRY(A.alloc((void **)&Q.srcs, S * 4));
    TG_TRY(A.alloc((void **)&Q.relax_cnt, S * 8));
    if (nodes_state) {
        TG_TRY(A.alloc((void **)&Q.dnode, std::max<uint64_t>(S * nnodes, 1) * 4));
        TG_TRY(A.alloc((void **)&Q.vout, S * n * 4));
    }
    return TG_OK;
}

uint32_t tg_pick_sub_batch(tg_graph *g, uint32_t k, bool nodes_state) {
    if (g->opt_sub_batch > 0) return (uint32_t)std::min<int64_t>(g->opt_sub_batch, k);
    const uint64_t n = g->n;
    const uint64_t nlong = std::max(g->fwd.nlong, g->mir.nlong);
    const uint64_t nnodes = std::max(g->fwd.nnodes, g->mir.nnodes);
    uint64_t per = n * (8 + 4 + 4 + 16) + nlong * (4 + 16) + g->m / CHUNK * 16 + 64;
    if (nodes_state) per += nnodes * (4 + 4 + 16) + n * 4;
    const uint64_t budget = 6ull << 30;  // device bytes for per-query state
    uint64_t S = std::max<uint64_t>(1, budget / per);
    S = std::min<uint64_t>(S, 256);
    return (uint32_t)std::min<uint64_t>(S, k);
}

tg_status tg_ensure_scratch(tg_graph *g, uint32_t S, bool nodes_state) { return ensure_scratch(g, S, nodes_state); }

// Run the GAC rounds of one sub-batch on direction cg; returns rounds used.
static tg_status eat_rounds(tg_graph *g, const ChainGraph &cgr, uint32_t S, uint32_t alpha, uint32_t omega,
                            bool any_work, cudaStream_t s, uint32_t *rounds_out) {
    QueryScratch &Q = g->qs;
    const uint64_t n = g->n;
    TG_TRY_CUDA(cudaMemsetAsync(Q.st, 0xFF, S * n * 8, s));
    TG_TRY_CUDA(cudaMemsetAsync(Q.act, 0xFF, S * n * 4, s));
    if (cgr.nlong) TG_TRY_CUDA(cudaMemsetAsync(Q.entry, 0xFF, S * cgr.nlong * 4, s));
    if (g->opt_stats) TG_TRY_CUDA(cudaMemsetAsync(Q.relax_cnt, 0, S * 8, s));
    const bool work = any_work && g->m > 0 && alpha < omega;
    TG_LAUNCH(k_eat_init, (S + 255) / 256, 256, 0, s, Q.st, g->n, Q.srcs, S, alpha, Q.fr[1], Q.ctr + 4, work ? 1 : 0);
    uint32_t rounds = 0;
    if (work) {
        EatP P{};
        P.vnode_off = cgr.vnode_off; P.node_t = cgr.node_t; P.node_eoff = cgr.node_eoff; P.occ_slot = cgr.occ_slot;
        P.slots = cgr.slots; P.lc = cgr.lc; P.sc = cgr.sc;
        P.st = Q.st; P.act = Q.act; P.mark = Q.mark; P.entry = Q.entry;
        P.n = g->n; P.nlong = cgr.nlong; P.alpha = alpha; P.omega = omega;
        P.use_sc = (int)g->opt_shortcuts; P.stats = (int)g->opt_stats;
        P.bigq = Q.bigq; P.bigcap = Q.bigcap; P.chq = Q.chq; P.chcap = Q.chcap; P.relax_cnt = Q.relax_cnt;
        const uint32_t grid = tg_grid_persistent(8);
        const int group = (int)std::max<int64_t>(1, g->opt_round_group);
        uint32_t r = 1;
        for (;;) {
            for (int k = 0; k < group; k++, r++) {
                const int in = r & 1, outp = (r + 1) & 1;
                // counters: ctr[par*4 + 0] = frontier count of buffer par; [1] big; [2] chain
                TG_TRY_CUDA(cudaMemsetAsync(Q.ctr + outp * 4, 0, 4, s));
                TG_TRY_CUDA(cudaMemsetAsync(Q.ctr + in * 4 + 1, 0, 8, s));
                if (++g->qs_epoch == 0) {  // stamp wrapped: clear marks
                    TG_TRY_CUDA(cudaMemsetAsync(Q.mark, 0, (uint64_t)Q.S * n * 4, s));
                    g->qs_epoch = 1;
                }
                P.stamp = g->qs_epoch;
                P.fin = Q.fr[in]; P.fin_cnt = Q.ctr + in * 4;
                P.fout = Q.fr[outp]; P.fout_cnt = Q.ctr + outp * 4;
                P.big_cnt = Q.ctr + in * 4 + 1; P.ch_cnt = Q.ctr + in * 4 + 2;
                TG_LAUNCH(k_eat_activate, grid, QT, 0, s, P);
                TG_LAUNCH(k_eat_big, grid, QT, 0, s, P);
                TG_LAUNCH(k_eat_chain, grid, QT, 0, s, P);
            }
            // r is the next round; its input count is ctr[(r & 1) * 4]
            TG_TRY_CUDA(cudaMemcpyAsync(Q.h_ctr, Q.ctr, 32, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            if (Q.h_ctr[(r & 1) * 4] == 0) break;
            if (r > 1000000) { tg_set_error("GAC rounds did not converge"); return TG_ERR_CUDA; }
        }
        rounds = r - 1;
    }
    *rounds_out = rounds;
    return TG_OK;
}

tg_status tg_run_eat_family(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w,
                            uint32_t *out, uint32_t *pred, bool out_dev, bool pred_dev, cudaStream_t s) {
    const bool ld = (p == TG_LD);
    const ChainGraph &cgr = ld ? g->mir : g->fwd;
    uint32_t alpha = w.t_alpha, omega = w.t_omega;
    bool any_work = true;
    const uint32_t C = g->max_arr;
    if (ld) {
        // reading A5: LD(G,x,[a,o]) = C - EAT(G^R, x, [max(0, C-o), C-a]); a > C -> only the target
        if (alpha > C) { any_work = false; alpha = 0; omega = 0; }
        else { uint32_t a2 = (omega >= C) ? 0u : C - omega; omega = C - alpha; alpha = a2; }
    }
    const uint32_t S = tg_pick_sub_batch(g, k, false);
    TG_TRY(ensure_scratch(g, S, false));
    QueryScratch &Q = g->qs;
    const uint64_t n = g->n;
    if (!out_dev && !Q.out_stage) TG_TRY(Q.arena.alloc((void **)&Q.out_stage, (uint64_t)Q.S * n * 4));
    if (pred && !pred_dev && !Q.pred_stage) TG_TRY(Q.arena.alloc((void **)&Q.pred_stage, (uint64_t)Q.S * n * 4));
    g->last = tg_query_stats{};
    if (g->opt_stats) {
        delete[] g->last_relax;
        g->last_relax = new uint64_t[k];
        g->last_relax_len = k;
    }
    const uint64_t launches0 = g_tg_launches;
    const int mode = ld ? 1 : (p == TG_REACH ? 2 : 0);
    for (uint32_t b0 = 0; b0 < k; b0 += S) {
        const uint32_t Sb = std::min(S, k - b0);
        TG_TRY_CUDA(cudaMemcpyAsync(Q.srcs, sources + b0, Sb * 4, cudaMemcpyHostToDevice, s));
        uint32_t rounds = 0;
        TG_TRY(eat_rounds(g, cgr, Sb, alpha, omega, any_work, s, &rounds));
        g->last.rounds = std::max(g->last.rounds, rounds);
        g->last.sub_batches++;
        uint32_t *o = out_dev ? out + (size_t)b0 * n : Q.out_stage;
        uint32_t *pr = pred ? (pred_dev ? pred + (size_t)b0 * n : Q.pred_stage) : nullptr;
        dim3 grid((unsigned)std::min<uint64_t>((n + 255) / 256, 1024), Sb);
        TG_LAUNCH(k_eat_extract, grid, 256, 0, s, Q.st, g->n, Q.srcs, mode, C, w.t_omega, o, pr);
        if (!out_dev) TG_TRY_CUDA(cudaMemcpyAsync(out + (size_t)b0 * n, Q.out_stage, (size_t)Sb * n * 4, cudaMemcpyDeviceToHost, s));
        if (pred && !pred_dev) TG_TRY_CUDA(cudaMemcpyAsync(pred + (size_t)b0 * n, Q.pred_stage, (size_t)Sb * n * 4, cudaMemcpyDeviceToHost, s));
        if (g->opt_stats) {
            std::vector<unsigned long long> h(Sb);
            TG_TRY_CUDA(cudaMemcpyAsync(h.data(), Q.relax_cnt, Sb * 8, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            for (uint32_t q = 0; q < Sb; q++) { g->last_relax[b0 + q] = h[q]; g->last.slots_relaxed += h[q]; }
        }
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    g->last.kernel_launches = g_tg_launches - launches0;
    return TG_OK;
}
