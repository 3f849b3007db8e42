// build.cu -- chain-based temporal graph transformation on the GPU (sm_100a).
//
// Paper: §4.1 "Chain-based Temporal Graph Transformation" (Alg. 1),
// §4.2 "Skeleton-graph Generation" (Alg. 2), storage P:L273 (Fig. 8).
// The paper runs Alg. 1 on CPU threads (DFS from each hub); here every step is a
// data-parallel kernel:
//   1. key = (u << tbits) | t, stable radix sort with edge-id payload  -> edges in (u, t, id) order
//   2. segmentation into departure nodes (v, tau) = distinct (u, t)   (DAG vertices, reading A11)
//   3. snap: tail node of each edge = first departure of v at or after t + duration (binary search)
//   4. in-degree histogram, hub flags (Def. 2, P:L174 / P:L225)
//   5. successor of each edge through non-hub nodes; chain heads = out-edges of hubs
//   6. chain lengths (walk), scan -> slot offsets, scatter 16-byte slots chain-major
//   7. shortcut per long chain (Alg. 2 fold) and the occurrence index (replaces the
//      GPU hash table of: sorted-edge position -> slot)
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>

#include "tg_internal.cuh"

namespace {

constexpr int BT = 256;

inline unsigned blocks_for(uint64_t n, int per_thread = 1) {
    uint64_t b = (n + (uint64_t)BT * per_thread - 1) / ((uint64_t)BT * per_thread);
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, 148ull * 64));
}

#define GRID_STRIDE(i, n) for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < (n); \
                               i += (uint64_t)gridDim.x * blockDim.x)

__global__ void k_make_keys(const uint32_t *__restrict__ u, const uint32_t *__restrict__ t, uint64_t m, int tbits,
                            unsigned long long *__restrict__ keys, uint32_t *__restrict__ ids) {
    GRID_STRIDE(i, m) {
        keys[i] = ((unsigned long long)u[i] << tbits) | t[i];
        ids[i] = (uint32_t)i;
    }
}

// keys of edges given in sorted order (ids[i]): the same (u << tbits | t) encoding
__global__ void k_keys_of_order(const uint32_t *__restrict__ ids, const uint32_t *__restrict__ u,
                                const uint32_t *__restrict__ t, uint64_t m, int tbits,
                                unsigned long long *__restrict__ keys, uint32_t *__restrict__ out_ids) {
    GRID_STRIDE(i, m) {
        const uint32_t e = ids[i];
        keys[i] = ((unsigned long long)u[e] << tbits) | t[e];
        out_ids[i] = e;
    }
}

// departure-node boundaries in (u, t)-sorted order
__global__ void k_node_flags(const unsigned long long *__restrict__ keys, uint64_t m, uint32_t *__restrict__ flag) {
    GRID_STRIDE(p, m) flag[p] = (p == 0 || keys[p] != keys[p - 1]) ? 1u : 0u;
}

// node_of[p] (exclusive-scanned flags, adjusted) and per-node arrays
__global__ void k_nodes(const unsigned long long *__restrict__ keys, uint64_t m, int tbits,
                        uint32_t *__restrict__ node_of /* in: excl scan of flags */,
                        uint32_t *__restrict__ node_t, uint32_t *__restrict__ node_u,
                        uint32_t *__restrict__ node_eoff) {
    const unsigned long long tmask = (1ull << tbits) - 1ull;
    GRID_STRIDE(p, m) {
        unsigned long long k = keys[p];
        bool head = (p == 0 || k != keys[p - 1]);
        uint32_t j = node_of[p];
        if (head) {
            node_t[j] = (uint32_t)(k & tmask);
            node_u[j] = (uint32_t)(k >> tbits);
            node_eoff[j] = (uint32_t)p;
            node_of[p] = j;
        } else {
            node_of[p] = j - 1;
        }
    }
}

// vnode_off[w] = first node of vertex w (CSR over vertices; empty vertices repeat)
__global__ void k_vnode_off(const uint32_t *__restrict__ node_u, uint64_t nn, uint32_t n,
                            uint32_t *__restrict__ vnode_off) {
    GRID_STRIDE(j, nn + 1) {
        int64_t prev = (j == 0) ? -1 : (int64_t)node_u[j - 1];
        int64_t cur = (j == nn) ? (int64_t)n : (int64_t)node_u[j];
        for (int64_t w = prev + 1; w <= cur; w++) vnode_off[w] = (uint32_t)j;
    }
}

// AoS edge records in input order, {v, arrival, w, t}: one 16-byte gather per
// sorted edge instead of several 4-byte ones
__global__ void k_records(const uint32_t *__restrict__ V, const uint32_t *__restrict__ T,
                          const uint32_t *__restrict__ DUR, const uint32_t *__restrict__ W, uint64_t m,
                          uint4 *__restrict__ rec) {
    GRID_STRIDE(i, m) rec[i] = make_uint4(V[i], T[i] + DUR[i], W[i], T[i]);
}

// snap each sorted edge to its tail departure node; count in-degrees.  The edge's
// record is gathered once here (the sort permutation's only random 16-byte read) and
// written out in sorted order for the chain scatter.  Each thread carries SNAP_ILP
// edges through the dependent loads and the binary searches in lockstep (memory-level
// parallelism for a latency-bound kernel).
#ifndef TG_SNAP_GROUPED
#define TG_SNAP_GROUPED 1  // regroup the snap searches by head vertex (k_snap_grouped)
#endif
#ifndef TG_SNAP_ILP
#define TG_SNAP_ILP 2  // 1, 2, 4 measured equal within 1 %; 8 slower
#endif
__global__ void k_snap(const uint32_t *__restrict__ sid, uint64_t m, const uint4 *__restrict__ rec,
                       const uint32_t *__restrict__ vnode_off, const uint32_t *__restrict__ node_t,
                       uint32_t *__restrict__ tn, uint32_t *__restrict__ indeg, uint4 *__restrict__ srec) {
    constexpr int K = TG_SNAP_ILP;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t p0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; p0 < m; p0 += stride * K) {
        uint32_t lo[K], hi[K], end[K], arr[K];
        uint4 r[K];
#pragma unroll
        for (int j = 0; j < K; j++) {
            const uint64_t p = p0 + j * stride;
            r[j] = make_uint4(0, 0, 0, 0);
            if (p < m) r[j] = rec[sid[p]];
        }
#pragma unroll
        for (int j = 0; j < K; j++) {
            const uint64_t p = p0 + j * stride;
            lo[j] = hi[j] = 0;
            arr[j] = r[j].y;
            if (p < m) {
                if (srec) srec[p] = r[j];
                lo[j] = vnode_off[r[j].x];
                hi[j] = vnode_off[r[j].x + 1];
            }
            end[j] = hi[j];
        }
        // lower bound of the arrival among the head's departure times, K searches interleaved
        bool busy = true;
        while (busy) {
            busy = false;
#pragma unroll
            for (int j = 0; j < K; j++) {
                if (lo[j] < hi[j]) {
                    const uint32_t mid = lo[j] + ((hi[j] - lo[j]) >> 1);
                    if (node_t[mid] < arr[j]) lo[j] = mid + 1; else hi[j] = mid;
                    busy = true;
                }
            }
        }
#pragma unroll
        for (int j = 0; j < K; j++) {
            const uint64_t p = p0 + j * stride;
            if (p >= m) continue;
            const uint32_t x = (lo[j] < end[j]) ? lo[j] : TG_NONE;
            tn[p] = x;
            if (x != TG_NONE) atomicAdd(&indeg[x], 1u);
        }
    }
}

// Grouped snap (the default): the sorted edges' (head, arrival) keys are regrouped by head
// vertex (a radix sort on the head bits only), so the binary searches of one vertex's
// departure times run next to each other and hit cache -- the per-edge searches of
// k_snap are dependent DRAM round trips, deep ones for R-MAT hubs (C4 direction:
// 128 ms, of which 17 ms is the record gather; grouped: 68 ms, the C4 forward + mirror build
// 507 -> 390 ms).  Results are those of k_snap (chain export digests equal).
__global__ void k_snap_keys(const uint32_t *__restrict__ sid, uint64_t m, const uint4 *__restrict__ rec,
                            uint4 *__restrict__ srec, unsigned long long *__restrict__ key2,
                            uint32_t *__restrict__ val2) {
    GRID_STRIDE(p, m) {
        const uint4 r = rec[sid[p]];
        if (srec) srec[p] = r;
        key2[p] = ((unsigned long long)r.x << 32) | r.y;  // (head v, arrival)
        val2[p] = (uint32_t)p;
    }
}

__global__ void k_snap_grouped(const unsigned long long *__restrict__ key2, const uint32_t *__restrict__ val2,
                               uint64_t m, const uint32_t *__restrict__ vnode_off,
                               const uint32_t *__restrict__ node_t, uint32_t *__restrict__ tn,
                               uint32_t *__restrict__ indeg) {
    GRID_STRIDE(i, m) {
        const unsigned long long k = key2[i];
        const uint32_t v = (uint32_t)(k >> 32), arr = (uint32_t)k;
        uint32_t lo = vnode_off[v], hi = vnode_off[v + 1];
        const uint32_t end = hi;
        while (lo < hi) {
            const uint32_t mid = lo + ((hi - lo) >> 1);
            if (node_t[mid] < arr) lo = mid + 1; else hi = mid;
        }
        const uint32_t x = lo < end ? lo : TG_NONE;
        tn[val2[i]] = x;
        // edges of one head arrive together: one atomic per distinct node of the warp
        const uint32_t same = __match_any_sync(__activemask(), x);
        if (x != TG_NONE && (threadIdx.x & 31) == (uint32_t)(__ffs(same) - 1)) atomicAdd(&indeg[x], (uint32_t)__popc(same));
    }
}

// hub (Def. 2): in-degree 0, in-degree >= 2, or out-degree >= 2
__global__ void k_hubs(const uint32_t *__restrict__ indeg, const uint32_t *__restrict__ node_eoff, uint64_t nn,
                       unsigned char *__restrict__ hub) {
    GRID_STRIDE(j, nn) {
        uint32_t outdeg = node_eoff[j + 1] - node_eoff[j];
        hub[j] = (indeg[j] != 1u || outdeg >= 2u) ? 1 : 0;
    }
}

// chain heads = out-edges of hubs; successor through a non-hub tail node
__global__ void k_succ(const uint32_t *__restrict__ node_of, const uint32_t *__restrict__ tn, uint64_t m,
                       const unsigned char *__restrict__ hub, const uint32_t *__restrict__ node_eoff,
                       uint32_t *__restrict__ head, uint32_t *__restrict__ succ) {
    GRID_STRIDE(p, m) {
        head[p] = hub[node_of[p]] ? 1u : 0u;
        uint32_t r = tn[p];
        succ[p] = (r != TG_NONE && !hub[r]) ? node_eoff[r] : TG_NONE;
    }
}

// ChainPartitioning (Alg. 1 lines 8-19) as a walk from each head: chain length
__global__ void k_chain_len(const uint32_t *__restrict__ head, const uint32_t *__restrict__ cidx,
                            const uint32_t *__restrict__ succ, uint64_t m, uint32_t *__restrict__ chain_len,
                            uint32_t *__restrict__ maxlen) {
    uint32_t mx = 0;
    GRID_STRIDE(p, m) {
        if (!head[p]) continue;
        uint32_t len = 1;
        for (uint32_t q = succ[p]; q != TG_NONE; q = succ[q]) len++;
        chain_len[cidx[p]] = len;
        mx = max(mx, len);
    }
    for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    if ((threadIdx.x & 31) == 0) atomicMax(maxlen, mx);
}

__global__ void k_long_flags(const uint32_t *__restrict__ chain_len, uint64_t nc, uint32_t *__restrict__ lflag) {
    GRID_STRIDE(c, nc) lflag[c] = chain_len[c] >= 2 ? 1u : 0u;
}

// Scatter slots chain-major and generate shortcuts (Alg. 2): one thread per chain.
__global__ void k_chain_scatter(const uint32_t *__restrict__ head, const uint32_t *__restrict__ cidx,
                                const uint32_t *__restrict__ succ, uint64_t m,
                                const uint32_t *__restrict__ chain_first, const uint32_t *__restrict__ chain_len,
                                const uint32_t *__restrict__ lidx, const uint32_t *__restrict__ sid,
                                const uint4 *__restrict__ srec, const uint4 *__restrict__ rec,
                                const uint32_t *__restrict__ tn, const uint32_t *__restrict__ node_of,
                                int4 *__restrict__ slots, uint32_t *__restrict__ slot_w,
                                uint32_t *__restrict__ slot_tn, uint32_t *__restrict__ occ_slot,
                                uint2 *__restrict__ occ_rec, uint2 *__restrict__ lc, int4 *__restrict__ sc,
                                unsigned long long *__restrict__ sc_sumw, uint32_t *__restrict__ sc_elapsed,
                                const uint32_t *__restrict__ id_map, uint32_t walk_min) {
    GRID_STRIDE(p, m) {
        if (!head[p]) continue;
        uint32_t c = cidx[p];
        uint32_t first = chain_first[c];
        uint32_t len = chain_len[c];
        const uint32_t l = (len >= 2) ? lidx[c] : TG_SINGLE;
        // slots of chains shorter than walk_min are marked SINGLE: the query engines
        // relax them edge by edge through their own occurrences (RemoveChain, P:L322,
        // generalised); longer chains are walked.  lc/sc are generated for every chain.
        const uint32_t cw = (len >= walk_min) ? l : TG_SINGLE;
        uint32_t s = first;
        uint32_t q = p;
        unsigned long long sumw = 0;
        uint4 r0 = make_uint4(0, 0, 0, 0), r = r0;
        uint32_t e = 0;
        while (q != TG_NONE) {
            e = sid[q];
            r = srec ? srec[q] : rec[e];  // the edge's record (in sorted order when k_snap wrote it)
            if (q == p) r0 = r;
            slots[s] = make_int4((int)r.x, (int)r.y, (int)(id_map ? id_map[e] : e), (int)cw);
            slot_w[s] = r.z;
            slot_tn[s] = tn[q];
            occ_slot[q] = s;
            // occurrence-ordered {head, arrival | walked-chain flag}: the activation reads a
            // vertex's newly usable out-edges as one contiguous run (P:L344's coalescing of
            // the chains leaving one vertex) instead of index + scattered 16-byte slot
            occ_rec[q] = make_uint2(r.x, r.y | (cw != TG_SINGLE ? 0x80000000u : 0u));
            sumw += r.z;  // GenerateShortcut: accumulate W_e (Alg. 2 line 5)
            s++;
            q = succ[q];
        }
        if (len >= 2) {  // r / e now hold the chain's last edge
            lc[l] = make_uint2(first, len);
            const uint32_t lid = id_map ? id_map[e] : e;
            sc[l] = make_int4((int)r.x, (int)r.y, (int)lid, (int)node_of[p]);
            sc_sumw[l] = sumw;
            sc_elapsed[l] = r.y - r0.w;
        }
    }
}

__global__ void k_validate(const uint32_t *__restrict__ u, const uint32_t *__restrict__ v,
                           const uint32_t *__restrict__ t, const uint32_t *__restrict__ dur,
                           const uint32_t *__restrict__ w, uint64_t m, uint32_t n, uint32_t *__restrict__ res) {
    // res: [0] flags (1 range id, 2 duration 0, 4 t+dur > TMAX), [1] max t, [2] max arr, [3] max w, [4] min t
    uint32_t flags = 0, mt = 0, ma = 0, mw = 0, mn = 0xFFFFFFFFu;
    GRID_STRIDE(i, m) {
        uint32_t a = u[i], b = v[i], tt = t[i], d = dur[i];
        if (a >= n || b >= n) flags |= 1u;
        if (d == 0) flags |= 2u;
        unsigned long long arr = (unsigned long long)tt + d;
        if (arr > TG_TMAX) flags |= 4u;
        mt = max(mt, tt);
        mn = min(mn, tt);
        ma = max(ma, (uint32_t)min(arr, 0xFFFFFFFFull));
        mw = max(mw, w ? w[i] : d);
    }
    for (int o = 16; o; o >>= 1) {
        flags |= __shfl_xor_sync(0xffffffffu, flags, o);
        mt = max(mt, __shfl_xor_sync(0xffffffffu, mt, o));
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        ma = max(ma, __shfl_xor_sync(0xffffffffu, ma, o));
        mw = max(mw, __shfl_xor_sync(0xffffffffu, mw, o));
    }
    if ((threadIdx.x & 31) == 0) {
        if (flags) atomicOr(&res[0], flags);
        atomicMax(&res[1], mt);
        atomicMax(&res[2], ma);
        atomicMax(&res[3], mw);
        atomicMin(&res[4], mn);
    }
}

// vertex-range partitions: keep edges whose key vertex (u forward, v mirror) is in [vb, ve)
__global__ void k_range_flags(const uint32_t *__restrict__ key, uint64_t m, uint32_t vb, uint32_t ve,
                              uint32_t *__restrict__ flag) {
    GRID_STRIDE(i, m) flag[i] = (key[i] >= vb && key[i] < ve) ? 1u : 0u;
}

__global__ void k_range_compact(const uint32_t *__restrict__ key, uint64_t m, uint32_t vb, uint32_t ve,
                                const uint32_t *__restrict__ pos, const uint32_t *__restrict__ u,
                                const uint32_t *__restrict__ v, const uint32_t *__restrict__ t,
                                const uint32_t *__restrict__ dur, const uint32_t *__restrict__ w,
                                uint32_t *__restrict__ ou, uint32_t *__restrict__ ov, uint32_t *__restrict__ ot,
                                uint32_t *__restrict__ odur, uint32_t *__restrict__ ow, uint32_t *__restrict__ oid) {
    GRID_STRIDE(i, m) {
        if (key[i] < vb || key[i] >= ve) continue;
        const uint32_t j = pos[i];
        ou[j] = u[i]; ov[j] = v[i]; ot[j] = t[i]; odur[j] = dur[i]; ow[j] = w[i]; oid[j] = (uint32_t)i;
    }
}

// ---- internal vertex order: descending in-degree (hot relaxation targets share L2 lines)
__global__ void k_indeg_hist(const uint32_t *__restrict__ v, uint64_t m, uint32_t *__restrict__ cnt) {
    GRID_STRIDE(i, m) atomicAdd(&cnt[v[i]], 1u);
}

__global__ void k_degree_keys(const uint32_t *__restrict__ cnt, uint32_t n, unsigned long long *__restrict__ keys,
                              uint32_t *__restrict__ ids) {
    GRID_STRIDE(i, n) {
        keys[i] = 0xFFFFFFFFull - cnt[i];
        ids[i] = (uint32_t)i;
    }
}

__global__ void k_perm_from_order(const uint32_t *__restrict__ order, uint32_t n, uint32_t *__restrict__ perm,
                                  uint32_t *__restrict__ iperm) {
    GRID_STRIDE(i, n) {
        perm[order[i]] = (uint32_t)i;
        iperm[i] = order[i];
    }
}

__global__ void k_apply_perm(const uint32_t *__restrict__ u, const uint32_t *__restrict__ v, uint64_t m,
                             const uint32_t *__restrict__ perm, uint32_t *__restrict__ ru, uint32_t *__restrict__ rv) {
    GRID_STRIDE(i, m) {
        ru[i] = perm[u[i]];
        rv[i] = perm[v[i]];
    }
}

__global__ void k_map_sources(const uint32_t *__restrict__ src, uint32_t k, const uint32_t *__restrict__ perm,
                              uint32_t *__restrict__ out) {
    GRID_STRIDE(i, k) out[i] = perm ? perm[src[i]] : src[i];
}

__global__ void k_mirror(const uint32_t *__restrict__ t, const uint32_t *__restrict__ dur, uint64_t m, uint32_t C,
                         uint32_t *__restrict__ mt) {
    // reading A5: e = (u,v,t,lam) -> (v,u, C - (t + lam), lam)
    GRID_STRIDE(i, m) mt[i] = C - (t[i] + dur[i]);
}

}  // namespace

// validation of a chunk of edges, accumulated into res[5] (device; initialised to
// {0, 0, 0, 0, 0xFFFFFFFF}); w may be NULL (weight = duration)
tg_status tg_validate_launch(const uint32_t *u, const uint32_t *v, const uint32_t *t, const uint32_t *dur,
                             const uint32_t *w, uint64_t m, uint32_t n, uint32_t *res, cudaStream_t s) {
    if (m) TG_LAUNCH(k_validate, blocks_for(m, 4), BT, 0, s, u, v, t, dur, w, m, n, res);
    return TG_OK;
}

tg_status tg_validate_edges(tg_graph *g, cudaStream_t s) {
    uint32_t *res = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&res, 5 * 4, s));
    uint32_t init[5] = {0, 0, 0, 0, 0xFFFFFFFFu};
    TG_TRY_CUDA(cudaMemcpyAsync(res, init, sizeof(init), cudaMemcpyHostToDevice, s));
    TG_TRY(tg_validate_launch(g->d_u, g->d_v, g->d_t, g->d_dur, g->d_w, g->m, g->n, res, s));
    uint32_t h[5];
    TG_TRY_CUDA(cudaMemcpyAsync(h, res, sizeof(h), cudaMemcpyDeviceToHost, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    TG_TRY_CUDA(cudaFreeAsync(res, s));
    return tg_validate_finish(g, h);
}

tg_status tg_validate_finish(tg_graph *g, const uint32_t *h) {
    if (h[0] & 1u) { tg_set_error("edge endpoint >= n_vertices"); return TG_ERR_RANGE; }
    if (h[0] & 2u) { tg_set_error("edge duration 0 (durations must be >= 1, reading A2)"); return TG_ERR_INVALID; }
    if (h[0] & 4u) { tg_set_error("t + duration > TG_TMAX"); return TG_ERR_RANGE; }
    g->max_t = h[1];
    g->max_arr = h[2];
    g->max_w = h[3];
    g->min_t = g->m ? h[4] : 0;
    // SP distances: a legal path has strictly increasing departures (duration >= 1),
    // so at most min(m, max_t - min_t + 1) edges; its distance fits in uint32 if
    // that bound times max_w stays below 2^32 - 1.
    unsigned long long maxlen = std::min<unsigned long long>(g->m, (unsigned long long)g->max_t - g->min_t + 1);
    g->sp_ok = (unsigned __int128)maxlen * g->max_w < 0xFFFFFFFFull;
    return TG_OK;
}

static int bits_for(uint64_t x) {  // bits to represent values in [0, x]
    int b = 0;
    while (b < 64 && (x >> b) != 0) b++;
    return std::max(b, 1);
}

// TG_TRACE_BUILD=1: synchronise at the build's section boundaries and print the host
// time of each section to stderr (diagnostics of slow builds; off by default)
static void bmark(cudaStream_t s, const char *label) {
    static const bool on = getenv("TG_TRACE_BUILD") != nullptr;
    if (!on) return;
    static std::chrono::steady_clock::time_point last;
    cudaStreamSynchronize(s);
    const auto now = std::chrono::steady_clock::now();
    if (label) fprintf(stderr, "build-trace %s %.3f\n", label, std::chrono::duration<double, std::milli>(now - last).count());
    last = now;
}

tg_status tg_build_direction(tg_graph *g, ChainGraph *cg, uint64_t m, const uint32_t *u, const uint32_t *v,
                             const uint32_t *t, const uint32_t *dur, const uint32_t *w, const uint32_t *id_map,
                             uint32_t tmax, cudaStream_t s, const uint32_t *presorted) {
    const uint32_t n = g->n;
    cg->n = n;
    cg->m = m;
    bmark(s, nullptr);
    DevArena &A = cg->arena;
    if (g->opt_dynamic) A.slack_pct = 10;  // insertions re-transform into slightly larger arrays
    TG_TRY(A.alloc((void **)&cg->vnode_off, ((size_t)n + 1) * 4));
    if (m == 0) {
        TG_TRY_CUDA(cudaMemsetAsync(cg->vnode_off, 0, ((size_t)n + 1) * 4, s));
        TG_TRY(A.alloc((void **)&cg->chain_first, 4));
        TG_TRY_CUDA(cudaMemsetAsync(cg->chain_first, 0, 4, s));
        return TG_OK;
    }
    // ---- 1. sort by (u, t, id); tmax bounds this direction's t (known from validation).
    const uint32_t maxt = tmax;
    const int tbits = bits_for(maxt);
    const int ubits = bits_for(n - 1);
    unsigned long long *keys = nullptr;
    uint32_t *sid = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&keys, m * 8, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&sid, m * 4, s));
    if (presorted) {
        // an insertion merged the new edges into the kept order: keys by gather
        TG_LAUNCH(k_keys_of_order, blocks_for(m, 4), BT, 0, s, presorted, u, t, m, tbits, keys, sid);
    } else {
        TG_LAUNCH(k_make_keys, blocks_for(m, 4), BT, 0, s, u, t, m, tbits, keys, sid);
        unsigned long long *sk;
        uint32_t *sv;
        TG_TRY(tg_radix_sort_pairs(keys, sid, m, tbits + ubits, &sk, &sv, s));
    }
    if (g->opt_dynamic) {
        TG_TRY(A.alloc((void **)&cg->order, m * 4));
        TG_TRY_CUDA(cudaMemcpyAsync(cg->order, sid, m * 4, cudaMemcpyDeviceToDevice, s));
    }

    bmark(s, "sort");
    // ---- 2. departure nodes
    uint32_t *node_of = nullptr, *d_cnt = nullptr;
    TG_TRY(A.alloc((void **)&cg->occ_node, m * 4));
    node_of = cg->occ_node;
    TG_TRY_CUDA(tg_malloc_async((void **)&d_cnt, 16, s));
    TG_LAUNCH(k_node_flags, blocks_for(m, 4), BT, 0, s, keys, m, node_of);
    TG_TRY(tg_exclusive_scan_u32(node_of, node_of, m, d_cnt, s, nullptr));
    uint32_t h_cnt = 0;
    TG_TRY_CUDA(cudaMemcpyAsync(&h_cnt, d_cnt, 4, cudaMemcpyDeviceToHost, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    // the scan's total excludes the first flag (exclusive); nodes = total of flags
    // k_nodes turns excl-scan values into node ids: head p -> j = excl[p], others excl[p]-1.
    {
        // number of nodes = excl[m-1] + flag[m-1]; recompute on host from the two values
        uint32_t last_excl = 0;
        unsigned long long k_last = 0, k_prev = 0;
        TG_TRY_CUDA(cudaMemcpyAsync(&last_excl, node_of + (m - 1), 4, cudaMemcpyDeviceToHost, s));
        TG_TRY_CUDA(cudaMemcpyAsync(&k_last, keys + (m - 1), 8, cudaMemcpyDeviceToHost, s));
        if (m >= 2) TG_TRY_CUDA(cudaMemcpyAsync(&k_prev, keys + (m - 2), 8, cudaMemcpyDeviceToHost, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        bool last_head = (m == 1) || (k_last != k_prev);
        cg->nnodes = (uint64_t)last_excl + (last_head ? 1 : 0);
    }
    const uint64_t nn = cg->nnodes;
    TG_TRY(A.alloc((void **)&cg->node_t, nn * 4));
    TG_TRY(A.alloc((void **)&cg->node_u, nn * 4));
    TG_TRY(A.alloc((void **)&cg->node_eoff, (nn + 1) * 4));
    // k_nodes: for heads excl == node id; for non-heads excl == node id + 1
    TG_LAUNCH(k_nodes, blocks_for(m, 4), BT, 0, s, keys, m, tbits, node_of, cg->node_t, cg->node_u, cg->node_eoff);
    {
        uint32_t mm = (uint32_t)m;
        TG_TRY_CUDA(cudaMemcpyAsync(cg->node_eoff + nn, &mm, 4, cudaMemcpyHostToDevice, s));
    }
    TG_LAUNCH(k_vnode_off, blocks_for(nn + 1, 4), BT, 0, s, cg->node_u, nn, n, cg->vnode_off);
    TG_TRY_CUDA(cudaFreeAsync(keys, s));

    bmark(s, "nodes");
    // ---- 3./4. snap, in-degree, hubs
    uint32_t *tn = nullptr, *indeg = nullptr;
    uint4 *rec = nullptr;
    unsigned char *hub = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&tn, m * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&rec, m * 16, s));
    TG_LAUNCH(k_records, blocks_for(m, 4), BT, 0, s, v, t, dur, w, m, rec);
    TG_TRY_CUDA(tg_malloc_async((void **)&indeg, nn * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&hub, nn, s));
    TG_TRY_CUDA(cudaMemsetAsync(indeg, 0, nn * 4, s));
    // sorted copy of the records for the chain scatter, when the device has room for it
    // (a 1.47 B-edge partitioned build does not): otherwise the scatter gathers again
    uint4 *srec = nullptr;
    {
        // memory the stream-ordered pool holds but does not use serves the copy without
        // asking the driver: cudaMemGetInfo stalls the host for 10-100 ms at times on
        // the virtualised GPU boxes (TG_TRACE_BUILD), so it is only the fallback
        size_t fr = 0, tot = 0;
        bool room = false;
        int dev = 0;
        cudaGetDevice(&dev);
        cudaMemPool_t pool = nullptr;
        uint64_t reserved = 0, used = 0;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess &&
            cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &reserved) == cudaSuccess &&
            cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &used) == cudaSuccess)
            room = reserved >= used && reserved - used >= m * 16 + (1ull << 20);
        else
            pool = nullptr;
        cudaGetLastError();
        if (!room) {
            cudaMemGetInfo(&fr, &tot);
            room = fr > m * 16 + (4ull << 30);
        }
        if (room && tg_malloc_async((void **)&srec, m * 16, s) != cudaSuccess) {
            cudaGetLastError();
            srec = nullptr;
        }
        // the pool's unused reserve may be fragmented: if the copy made the pool grow, keep
        // the old 4 GB device headroom for the arrays this build still allocates, else fall
        // back to the gather path
        uint64_t reserved2 = 0;
        if (srec && pool && cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &reserved2) == cudaSuccess &&
            reserved2 > reserved) {
            cudaMemGetInfo(&fr, &tot);
            if (fr < (4ull << 30)) {
                cudaFreeAsync(srec, s);
                srec = nullptr;
            }
        }
        cudaGetLastError();
    }
    bmark(s, "memgetinfo");
    {
        // grouped snap when its sort buffers fit (24 B per edge), else the direct searches
        unsigned long long *key2 = nullptr;
        uint32_t *val2 = nullptr;
        // (small graphs: the searches already hit cache -- C2's 16.8 M edges: 9.4 vs 9.8 ms)
        bool grouped = TG_SNAP_GROUPED != 0 && m >= (1ull << 25);
        if (grouped && (tg_malloc_async((void **)&key2, m * 8, s) != cudaSuccess ||
                        tg_malloc_async((void **)&val2, m * 4, s) != cudaSuccess)) {
            cudaGetLastError();
            if (key2) cudaFreeAsync(key2, s);
            key2 = nullptr;
            grouped = false;
        }
        tg_status sst = TG_OK;
        if (grouped) {
            TG_LAUNCH(k_snap_keys, blocks_for(m, 4), BT, 0, s, sid, m, rec, srec, key2, val2);
            sst = tg_radix_sort_pairs_bits(key2, val2, m, 32, bits_for(n - 1), s);
            if (sst == TG_OK)
                TG_LAUNCH(k_snap_grouped, blocks_for(m, 4), BT, 0, s, key2, val2, m, cg->vnode_off, cg->node_t, tn,
                          indeg);
            cudaFreeAsync(key2, s);
            cudaFreeAsync(val2, s);
        }
        if (sst == TG_ERR_NOMEM) {  // the sort's scratch did not fit: direct searches
            cudaGetLastError();
            grouped = false;
        } else if (sst != TG_OK) {
            return sst;
        }
        if (!grouped)
            TG_LAUNCH(k_snap, blocks_for(m, 4 * TG_SNAP_ILP), BT, 0, s, sid, m, rec, cg->vnode_off, cg->node_t, tn,
                      indeg, srec);
    }
    if (srec) {
        TG_TRY_CUDA(cudaFreeAsync(rec, s));
        rec = nullptr;
    }
    TG_LAUNCH(k_hubs, blocks_for(nn, 4), BT, 0, s, indeg, cg->node_eoff, nn, hub);
    TG_TRY_CUDA(cudaFreeAsync(indeg, s));

    bmark(s, "snap_hubs");
    // ---- 5. heads / successors; chain ids in (head u, head t, first id) order
    uint32_t *head = nullptr, *succ = nullptr, *cidx = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&head, m * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&succ, m * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&cidx, m * 4, s));
    TG_LAUNCH(k_succ, blocks_for(m, 4), BT, 0, s, node_of, tn, m, hub, cg->node_eoff, head, succ);
    TG_TRY(tg_exclusive_scan_u32(head, cidx, m, d_cnt, s, nullptr));
    uint32_t nch = 0;
    TG_TRY_CUDA(cudaMemcpyAsync(&nch, d_cnt, 4, cudaMemcpyDeviceToHost, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    cg->nchains = nch;

    bmark(s, "chains");
    // ---- 6. chain lengths, slot offsets, long-chain numbering
    uint32_t *chain_len = nullptr, *lidx = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&chain_len, (uint64_t)nch * 4 + 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&lidx, (uint64_t)nch * 4 + 4, s));
    TG_TRY_CUDA(cudaMemsetAsync(d_cnt + 2, 0, 4, s));
    TG_LAUNCH(k_chain_len, blocks_for(m, 4), BT, 0, s, head, cidx, succ, m, chain_len, d_cnt + 2);
    TG_TRY(A.alloc((void **)&cg->chain_first, ((uint64_t)nch + 1) * 4));
    TG_TRY(tg_exclusive_scan_u32(chain_len, cg->chain_first, nch, cg->chain_first + nch, s, nullptr));
    TG_LAUNCH(k_long_flags, blocks_for(nch, 4), BT, 0, s, chain_len, nch, lidx);
    TG_TRY(tg_exclusive_scan_u32(lidx, lidx, nch, d_cnt + 1, s, nullptr));
    uint32_t h2[3] = {0, 0, 0};
    TG_TRY_CUDA(cudaMemcpyAsync(h2, d_cnt, 12, cudaMemcpyDeviceToHost, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    cg->nlong = h2[1];
    cg->maxlen = h2[2];
    const uint64_t L = cg->nlong;

    TG_TRY(A.alloc((void **)&cg->slots, m * 16));
    TG_TRY(A.alloc((void **)&cg->slot_w, m * 4));
    TG_TRY(A.alloc((void **)&cg->slot_tn, m * 4));
    TG_TRY(A.alloc((void **)&cg->occ_slot, m * 4));
    TG_TRY(A.alloc((void **)&cg->occ_rec, m * 8));
    TG_TRY(A.alloc((void **)&cg->lc, std::max<uint64_t>(L, 1) * 8));
    TG_TRY(A.alloc((void **)&cg->sc, std::max<uint64_t>(L, 1) * 16));
    TG_TRY(A.alloc((void **)&cg->sc_sumw, std::max<uint64_t>(L, 1) * 8));
    TG_TRY(A.alloc((void **)&cg->sc_elapsed, std::max<uint64_t>(L, 1) * 4));
    TG_LAUNCH(k_chain_scatter, blocks_for(m, 4), BT, 0, s, head, cidx, succ, m, cg->chain_first, chain_len, lidx, sid,
              srec, rec, tn, node_of, cg->slots, cg->slot_w, cg->slot_tn, cg->occ_slot, cg->occ_rec, cg->lc, cg->sc,
              cg->sc_sumw, cg->sc_elapsed, id_map, (uint32_t)std::max<int64_t>(2, g->opt_walk_min));

    for (void *p : {(void *)sid, (void *)d_cnt, (void *)tn, (void *)srec, (void *)rec, (void *)hub,
                    (void *)head, (void *)succ, (void *)cidx, (void *)chain_len, (void *)lidx})
        if (p) TG_TRY_CUDA(cudaFreeAsync(p, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    bmark(s, "scatter");
    return TG_OK;
}

tg_status tg_relabel(tg_graph *g, cudaStream_t s) {
    const uint64_t m = g->m;
    const uint32_t n = g->n;
    DevArena &A = g->arena;
    TG_TRY(A.alloc((void **)&g->perm, (uint64_t)n * 4));
    TG_TRY(A.alloc((void **)&g->iperm, (uint64_t)n * 4));
    TG_TRY(A.alloc((void **)&g->d_ru, std::max<uint64_t>(m, 1) * 4));
    TG_TRY(A.alloc((void **)&g->d_rv, std::max<uint64_t>(m, 1) * 4));
    uint32_t *cnt = nullptr, *ids = nullptr;
    unsigned long long *keys = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&cnt, (uint64_t)n * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&ids, (uint64_t)n * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&keys, (uint64_t)n * 8, s));
    TG_TRY_CUDA(cudaMemsetAsync(cnt, 0, (uint64_t)n * 4, s));
    if (m) TG_LAUNCH(k_indeg_hist, blocks_for(m, 4), BT, 0, s, g->d_v, m, cnt);
    TG_LAUNCH(k_degree_keys, blocks_for(n, 4), BT, 0, s, cnt, n, keys, ids);
    unsigned long long *sk;
    uint32_t *sv;
    TG_TRY(tg_radix_sort_pairs(keys, ids, n, 32, &sk, &sv, s));  // stable: ties keep vertex order
    TG_LAUNCH(k_perm_from_order, blocks_for(n, 4), BT, 0, s, ids, n, g->perm, g->iperm);
    if (m) TG_LAUNCH(k_apply_perm, blocks_for(m, 4), BT, 0, s, g->d_u, g->d_v, m, g->perm, g->d_ru, g->d_rv);
    TG_TRY_CUDA(cudaFreeAsync(cnt, s));
    TG_TRY_CUDA(cudaFreeAsync(ids, s));
    TG_TRY_CUDA(cudaFreeAsync(keys, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    g->relabeled = true;
    return TG_OK;
}

tg_status tg_load_sources_to(tg_graph *g, const uint32_t *sources, uint32_t k, uint32_t *d_srcs, uint32_t *d_int,
                             cudaStream_t s) {
    TG_TRY_CUDA(cudaMemcpyAsync(d_srcs, sources, (uint64_t)k * 4, cudaMemcpyHostToDevice, s));
    TG_LAUNCH(k_map_sources, 1, 64, 0, s, d_srcs, k, g->relabeled ? g->perm : nullptr, d_int);
    return TG_OK;
}

tg_status tg_load_sources(tg_graph *g, const uint32_t *sources, uint32_t k, cudaStream_t s) {
    return tg_load_sources_to(g, sources, k, g->qs.srcs, g->qs.srcs_int, s);
}

tg_status tg_build_mirror(tg_graph *g, cudaStream_t s) {
    const uint32_t *U = g->relabeled ? g->d_ru : g->d_u, *V = g->relabeled ? g->d_rv : g->d_v;
    // reading A5: G^R maps (u, v, t, lam) to (v, u, C - (t + lam), lam), C = max(t + lam)
    // mirrored departures C - (t + lam) <= C - min_t - 1
    const uint32_t mir_tmax = g->max_arr - g->min_t;
    if (g->m == 0) return tg_build_direction(g, &g->mir, 0, V, U, g->d_t, g->d_dur, g->d_w, nullptr, 0, s);
    uint32_t *mt = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&mt, g->m * 4, s));
    TG_LAUNCH(k_mirror, blocks_for(g->m, 4), BT, 0, s, g->d_t, g->d_dur, g->m, g->max_arr, mt);
    tg_status st = tg_build_direction(g, &g->mir, g->m, V, U, mt, g->d_dur, g->d_w, nullptr, mir_tmax, s);
    cudaFreeAsync(mt, s);
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    return st;
}

// One vertex-range partition [vb, ve): forward chains over the edges leaving the
// range, mirror chains over the edges entering it (the mirror's sources).
// Slots keep the original edge ids (id map).
tg_status tg_build_partition(tg_graph *g, ChainGraph *fwd, ChainGraph *mir, uint32_t vb, uint32_t ve, cudaStream_t s,
                             int dirs) {
    const uint64_t m = g->m;
    uint32_t *mt = nullptr, *flag = nullptr, *cnt = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&flag, std::max<uint64_t>(m, 1) * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&cnt, 4, s));
    if (dirs & 2) {
        TG_TRY_CUDA(tg_malloc_async((void **)&mt, std::max<uint64_t>(m, 1) * 4, s));
        if (m) TG_LAUNCH(k_mirror, blocks_for(m, 4), BT, 0, s, g->d_t, g->d_dur, m, g->max_arr, mt);
    }
    for (int dir = 0; dir < 2; dir++) {
        if (!((dirs >> dir) & 1)) continue;  // bit 0 forward, bit 1 mirror
        // forward: (u, v, t); mirror: (v, u, C - t - dur)
        const uint32_t *key = dir == 0 ? g->d_u : g->d_v;
        const uint32_t *uu = dir == 0 ? g->d_u : g->d_v;
        const uint32_t *vv = dir == 0 ? g->d_v : g->d_u;
        const uint32_t *tt = dir == 0 ? g->d_t : mt;
        uint32_t ms = 0;
        if (m) {
            TG_LAUNCH(k_range_flags, blocks_for(m, 4), BT, 0, s, key, m, vb, ve, flag);
            TG_TRY(tg_exclusive_scan_u32(flag, flag, m, cnt, s, nullptr));
            TG_TRY_CUDA(cudaMemcpyAsync(&ms, cnt, 4, cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
        }
        uint32_t *sub = nullptr;  // 6 arrays of ms
        TG_TRY_CUDA(tg_malloc_async((void **)&sub, std::max<uint64_t>(ms, 1) * 4 * 6, s));
        uint32_t *su = sub, *sv = sub + ms, *st = sub + 2 * (uint64_t)ms, *sd = sub + 3 * (uint64_t)ms,
                 *sw = sub + 4 * (uint64_t)ms, *sid = sub + 5 * (uint64_t)ms;
        if (ms)
            TG_LAUNCH(k_range_compact, blocks_for(m, 4), BT, 0, s, key, m, vb, ve, flag, uu, vv, tt, g->d_dur, g->d_w,
                      su, sv, st, sd, sw, sid);
        tg_status r = tg_build_direction(g, dir == 0 ? fwd : mir, ms, su, sv, st, sd, sw, sid,
                                         dir == 0 ? g->max_t : g->max_arr - g->min_t, s);
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        cudaFreeAsync(sub, s);
        if (r != TG_OK) return r;
    }
    if (mt) cudaFreeAsync(mt, s);
    cudaFreeAsync(flag, s);
    cudaFreeAsync(cnt, s);
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    return TG_OK;
}
