// dynamic.cu -- batched edge insertion with incremental re-transformation
// (§5.6: dynamic temporal graphs as batches of 100 K edge
// insertions, each followed by re-transformation and queries).
//
// With option "dynamic" the build keeps each direction's edge order (ids sorted by
// (u, t, id); the mirror's by (v, C - t - lambda, id)).  An insertion appends the
// batch to the edge arrays and, for a built graph, re-transforms incrementally:
//   1. only the batch is radix-sorted (k log-passes over the batch, not over m);
//   2. the kept order and the sorted batch are merged (one pass: every element's
//      output position = its own rank + its rank in the other sequence, found by a
//      binary search; equal keys keep the kept edges first = ascending ids);
//   3. departure nodes, snap, hubs, chains, shortcuts and the occurrence index are
//      regenerated from the merged order (tg_build_direction with `presorted`).
// The mirror's order is unaffected by a larger C (C - a keeps its order), so its
// kept order is merged the same way.
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>

#include "tg_internal.cuh"

tg_status tg_validate_edges(tg_graph *g, cudaStream_t s);
tg_status tg_radix_sort_pairs(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                              unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s);

namespace {

constexpr int BT = 256;
inline unsigned nblocks(uint64_t n) { return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + BT - 1) / BT, 148ull * 32)); }

__device__ __forceinline__ unsigned long long key_of(const uint32_t *u, const uint32_t *t, uint32_t e, int tbits) {
    return ((unsigned long long)u[e] << tbits) | t[e];
}

// keys of the batch ids [m_old, m_new)
__global__ void k_batch_keys(const uint32_t *__restrict__ u, const uint32_t *__restrict__ t, uint64_t m_old,
                             uint64_t k, int tbits, unsigned long long *__restrict__ keys, uint32_t *__restrict__ ids) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < k; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t e = (uint32_t)(m_old + i);
        keys[i] = key_of(u, t, e, tbits);
        ids[i] = e;
    }
}

// merge: kept order A (ids, keys by gather) and the sorted batch B (keys, ids) into out
__global__ void k_merge_kept(const uint32_t *__restrict__ A, uint64_t na, const unsigned long long *__restrict__ bk,
                             uint64_t nb, const uint32_t *__restrict__ u, const uint32_t *__restrict__ t, int tbits,
                             uint32_t *__restrict__ out) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < na; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t e = A[i];
        const unsigned long long k = key_of(u, t, e, tbits);
        uint64_t lo = 0, hi = nb;  // batch elements strictly before: key < k (equal keys: kept first)
        while (lo < hi) {
            const uint64_t mid = (lo + hi) >> 1;
            if (bk[mid] < k) lo = mid + 1; else hi = mid;
        }
        out[i + lo] = e;
    }
}

__global__ void k_merge_batch(const uint32_t *__restrict__ A, uint64_t na, const unsigned long long *__restrict__ bk,
                              const uint32_t *__restrict__ bid, uint64_t nb, const uint32_t *__restrict__ u,
                              const uint32_t *__restrict__ t, int tbits, uint32_t *__restrict__ out) {
    for (uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nb; j += (uint64_t)gridDim.x * blockDim.x) {
        const unsigned long long k = bk[j];
        uint64_t lo = 0, hi = na;  // kept elements before: key <= k
        while (lo < hi) {
            const uint64_t mid = (lo + hi) >> 1;
            if (key_of(u, t, A[mid], tbits) <= k) lo = mid + 1; else hi = mid;
        }
        out[j + lo] = bid[j];
    }
}

__global__ void k_mirror_times(const uint32_t *__restrict__ t, const uint32_t *__restrict__ dur, uint64_t m, uint32_t C,
                               uint32_t *__restrict__ mt) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x)
        mt[i] = C - (t[i] + dur[i]);
}

// TG_TRACE_BUILD=1: synchronise at the insertion's section boundaries and print the
// host time of each section (diagnostics)
void dmark(const char *label) {
    static const bool on = getenv("TG_TRACE_BUILD") != nullptr;
    if (!on) return;
    static std::chrono::steady_clock::time_point last;
    cudaDeviceSynchronize();
    const auto now = std::chrono::steady_clock::now();
    if (label) fprintf(stderr, "insert-trace %s %.3f\n", label, std::chrono::duration<double, std::milli>(now - last).count());
    last = now;
}

int bits_of(uint64_t x) {
    int b = 0;
    while (b < 64 && (x >> b) != 0) b++;
    return std::max(b, 1);
}

}  // namespace

// merged order of one direction: U/T are the direction's (head, departure) arrays over
// all m_new edges; kept = the previous order of the first m_old ids
static tg_status merged_order(const uint32_t *U, const uint32_t *T, uint32_t tmax, uint32_t n, const uint32_t *kept,
                              uint64_t m_old, uint64_t m_new, uint32_t *out, cudaStream_t s) {
    const uint64_t k = m_new - m_old;
    const int tbits = bits_of(tmax), ubits = bits_of(n - 1);
    unsigned long long *bk = nullptr;
    uint32_t *bid = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&bk, std::max<uint64_t>(k, 1) * 8, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&bid, std::max<uint64_t>(k, 1) * 4, s));
    k_batch_keys<<<nblocks(k), BT, 0, s>>>(U, T, m_old, k, tbits, bk, bid);
    g_tg_launches++;
    unsigned long long *sk;
    uint32_t *sv;
    TG_TRY(tg_radix_sort_pairs(bk, bid, k, tbits + ubits, &sk, &sv, s));
    k_merge_kept<<<nblocks(m_old), BT, 0, s>>>(kept, m_old, bk, k, U, T, tbits, out);
    k_merge_batch<<<nblocks(k), BT, 0, s>>>(kept, m_old, bk, bid, k, U, T, tbits, out);
    g_tg_launches += 2;
    TG_TRY_CUDA(cudaGetLastError());
    TG_TRY_CUDA(cudaFreeAsync(bk, s));
    TG_TRY_CUDA(cudaFreeAsync(bid, s));
    return TG_OK;
}

extern "C" tg_status tg_graph_insert_edges(tg_graph *g, uint64_t k, const uint32_t *u, const uint32_t *v,
                                           const uint32_t *t_start, const uint32_t *duration, const uint32_t *weight) {
    if (!g) { tg_set_error("graph is NULL"); return TG_ERR_INVALID; }
    if (k == 0) return TG_OK;
    if (!u || !v || !t_start || !duration) { tg_set_error("edge array is NULL"); return TG_ERR_INVALID; }
    if (g->m + k >= 0xFFFFFFFFull) { tg_set_error("n_edges must stay < 2^32 - 1"); return TG_ERR_RANGE; }
    if (g->nparts > 0 || g->comm || g->relabeled) {
        tg_set_error("insertion into partitioned / relabelled graphs is not supported");
        return TG_ERR_STATE;
    }
    const bool weighted = g->d_w != g->d_dur;
    if ((weight != nullptr) != weighted && g->m > 0) {
        tg_set_error("the batch must carry weights iff the graph was created with weights");
        return TG_ERR_INVALID;
    }
    if (g->built && !g->opt_dynamic) {
        tg_set_error("insertion into a built graph needs option \"dynamic\" = 1 before tg_build_chains");
        return TG_ERR_STATE;
    }
    int prev = -1;
    cudaGetDevice(&prev);
    if (prev != g->device) cudaSetDevice(g->device);
    cudaStream_t s = 0;
    TG_TRY_CUDA(cudaDeviceSynchronize());
    dmark(nullptr);
    const uint64_t m_old = g->m, m_new = g->m + k;
    // 1. the new edge arrays: the kept edges, then the batch (ids m_old .. m_new - 1)
    DevArena na;
    na.slack_pct = 10;  // the next insertion's edge arrays come from the cache
    uint32_t *nu = nullptr, *nv = nullptr, *nt = nullptr, *nd = nullptr, *nw = nullptr;
    uint32_t **dst[5] = {&nu, &nv, &nt, &nd, &nw};
    const uint32_t *oldp[5] = {g->d_u, g->d_v, g->d_t, g->d_dur, g->d_w};
    const uint32_t *src[5] = {u, v, t_start, duration, weight};
    for (int i = 0; i < 5; i++) {
        if (i == 4 && !(weighted || (m_old == 0 && weight))) { nw = nd; break; }  // w = duration (reading A7)
        tg_status st = na.alloc((void **)dst[i], m_new * 4);
        if (st != TG_OK) { na.free_all(); return st; }
        if (m_old) TG_TRY_CUDA(cudaMemcpyAsync(*dst[i], oldp[i], m_old * 4, cudaMemcpyDeviceToDevice, s));
        TG_TRY_CUDA(cudaMemcpyAsync(*dst[i] + m_old, src[i], k * 4, cudaMemcpyDefault, s));
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    dmark("copy");
    // swap in; validation over all edges (updates max t / arrival / weight, the SP bound)
    std::swap(g->arena, na);
    g->d_u = nu; g->d_v = nv; g->d_t = nt; g->d_dur = nd; g->d_w = nw;
    const uint64_t m_keep = g->m;
    g->m = m_new;
    tg_status vs = tg_validate_edges(g, s);
    if (vs != TG_OK) {
        // roll back to the kept edges
        std::swap(g->arena, na);
        g->d_u = (uint32_t *)oldp[0]; g->d_v = (uint32_t *)oldp[1]; g->d_t = (uint32_t *)oldp[2];
        g->d_dur = (uint32_t *)oldp[3]; g->d_w = (uint32_t *)oldp[4];
        g->m = m_keep;
        na.free_all();
        tg_validate_edges(g, s);
        return vs;
    }
    na.free_all();  // the old edge arrays
    dmark("validate");
    // query scratch is sized by m / nodes: rebuilt lazily by the next query
    TG_TRY_CUDA(cudaDeviceSynchronize());
    g->qs.arena.free_all();
    tg_pinned_put(g->qs.h_ctr);
    g->qs = QueryScratch{};
    for (auto &q : g->qsl) {
        q.arena.free_all();
        tg_pinned_put(q.h_ctr);
        q = QueryScratch{};
    }
    g->rs.arena.free_all();
    tg_pinned_put(g->rs.h_ctr);
    g->rs = ReachScratch{};
    dmark("scratch");
    if (!g->built) return TG_OK;
    // 2./3. incremental re-transformation of each built direction
    uint32_t *ord = nullptr, *mt = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&ord, m_new * 4, s));
    {
        TG_TRY(merged_order(g->d_u, g->d_t, g->max_t, g->n, g->fwd.order, m_old, m_new, ord, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        dmark("merge");
        g->fwd.arena.free_all();
        g->fwd = ChainGraph{};
        TG_TRY(tg_build_direction(g, &g->fwd, m_new, g->d_u, g->d_v, g->d_t, g->d_dur, g->d_w, nullptr, g->max_t, s,
                                  ord));
        dmark("rebuild");
    }
    if (g->mirror_built) {
        // reading A5's mirror with the (possibly larger) C = max(t + lambda)
        TG_TRY_CUDA(tg_malloc_async((void **)&mt, m_new * 4, s));
        k_mirror_times<<<nblocks(m_new), BT, 0, s>>>(g->d_t, g->d_dur, m_new, g->max_arr, mt);
        g_tg_launches++;
        const uint32_t mir_tmax = g->max_arr - g->min_t;
        TG_TRY(merged_order(g->d_v, mt, mir_tmax, g->n, g->mir.order, m_old, m_new, ord, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        g->mir.arena.free_all();
        g->mir = ChainGraph{};
        TG_TRY(tg_build_direction(g, &g->mir, m_new, g->d_v, g->d_u, mt, g->d_dur, g->d_w, nullptr, mir_tmax, s, ord));
        TG_TRY_CUDA(cudaFreeAsync(mt, s));
    }
    TG_TRY_CUDA(cudaFreeAsync(ord, s));
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    if (prev >= 0 && prev != g->device) cudaSetDevice(prev);
    return TG_OK;
}
