// rank.cu -- per-source reductions of query rows: top-K nearest
// neighbours and the closeness-style (reached, sum) summary of all-source batches.
//
// Paper: the motivating workloads of P:L116 / P:L134 (nearest neighbours, centrality
// over temporal paths).  Rows are computed by tg_query into device memory; top-K
// sorts each chunk of rows by (row, value) with the library's stable LSD radix sort
// (payload = vertex id in ascending order, so ties keep the smaller id first) and
// gathers the first K entries of every row; the summary is one reduction per row.
#include <algorithm>
#include <vector>

#include "tg_internal.cuh"

namespace {

// key = row << 32 | value; the source and unreached vertices get value NONE (sort last)
__global__ void k_topk_keys(const uint32_t *__restrict__ rows, uint32_t nr, uint32_t n,
                            const uint32_t *__restrict__ srcs, unsigned long long *__restrict__ keys,
                            uint32_t *__restrict__ vid) {
    const uint64_t total = (uint64_t)nr * n;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t r = (uint32_t)(i / n), v = (uint32_t)(i - (uint64_t)r * n);
        const uint32_t x = (v == srcs[r]) ? TG_NONE : rows[i];
        keys[i] = ((unsigned long long)r << 32) | x;
        vid[i] = v;
    }
}

__global__ void k_topk_gather(const unsigned long long *__restrict__ keys, const uint32_t *__restrict__ vid,
                              uint32_t nr, uint32_t n, uint32_t K, uint32_t *__restrict__ ov,
                              uint32_t *__restrict__ oval) {
    const uint64_t total = (uint64_t)nr * K;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t r = (uint32_t)(i / K), k = (uint32_t)(i - (uint64_t)r * K);
        uint32_t v = TG_NONE, x = TG_NONE;
        if (k < n) {
            const uint64_t j = (uint64_t)r * n + k;  // every row has exactly n entries
            x = (uint32_t)keys[j];
            if (x != TG_NONE) v = vid[j];
        }
        ov[i] = v;
        oval[i] = x;
    }
}

// block per row: number of reached v != source and the sum of their values
__global__ void __launch_bounds__(256) k_row_summary(const uint32_t *__restrict__ rows, uint32_t n,
                                                     const uint32_t *__restrict__ srcs,
                                                     unsigned long long *__restrict__ cnt,
                                                     unsigned long long *__restrict__ sum) {
    const uint32_t r = blockIdx.y;
    const uint32_t *row = rows + (size_t)r * n;
    unsigned long long c = 0, s = 0;
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        const uint32_t x = row[v];
        if (x != TG_NONE && v != srcs[r]) { c++; s += x; }
    }
    for (int o = 16; o; o >>= 1) {
        c += __shfl_xor_sync(0xffffffffu, c, o);
        s += __shfl_xor_sync(0xffffffffu, s, o);
    }
    if ((threadIdx.x & 31) == 0 && c) {
        atomicAdd(cnt + r, c);
        atomicAdd(sum + r, s);
    }
}

}  // namespace

// rows computed per chunk: bounded by ~2 GiB of row buffer (and the sort's 3x)
static uint32_t chunk_rows(const tg_graph *g, uint32_t k) {
    const uint64_t per = (uint64_t)g->n * 4;
    return (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(k, (2ull << 30) / per));
}

static bool is_dev(const void *p) {
    cudaPointerAttributes a;
    if (!p || cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

extern "C" {

tg_status tg_query_topk(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources, tg_window w,
                        uint32_t K, uint32_t *out_vertex, uint32_t *out_value, void *cuda_stream) {
    if (!g || !sources || !out_vertex || !out_value || n_sources == 0 || K == 0) {
        tg_set_error("tg_query_topk: NULL argument, n_sources == 0 or K == 0");
        return TG_ERR_INVALID;
    }
    if (!(p == TG_EAT || p == TG_FASTEST || p == TG_SHORTEST)) {
        tg_set_error("tg_query_topk: nearest = smallest value: TG_EAT, TG_FASTEST or TG_SHORTEST");
        return TG_ERR_INVALID;
    }
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const uint32_t C = chunk_rows(g, n_sources);
    const uint64_t n = g->n;
    uint32_t *rows = nullptr, *vid = nullptr, *srcs = nullptr, *ov = nullptr, *oval = nullptr;
    unsigned long long *keys = nullptr;
    const bool dev_out = is_dev(out_vertex) && is_dev(out_value);
    tg_status st = TG_OK;
    auto done = [&](tg_status r) {
        cudaFreeAsync(rows, s); cudaFreeAsync(vid, s); cudaFreeAsync(srcs, s); cudaFreeAsync(keys, s);
        if (!dev_out) { cudaFreeAsync(ov, s); cudaFreeAsync(oval, s); }
        cudaStreamSynchronize(s);
        return r;
    };
    if (tg_malloc_async((void **)&rows, C * n * 4, s) != cudaSuccess ||
        tg_malloc_async((void **)&vid, C * n * 4, s) != cudaSuccess ||
        tg_malloc_async((void **)&keys, C * n * 8, s) != cudaSuccess ||
        tg_malloc_async((void **)&srcs, C * 4, s) != cudaSuccess ||
        (!dev_out && (tg_malloc_async((void **)&ov, (uint64_t)C * K * 4, s) != cudaSuccess ||
                      tg_malloc_async((void **)&oval, (uint64_t)C * K * 4, s) != cudaSuccess))) {
        cudaGetLastError();
        tg_set_error("tg_query_topk: device allocation failed");
        return done(TG_ERR_NOMEM);
    }
    int rbits = 1;
    while ((1u << rbits) < C) rbits++;
    for (uint32_t b0 = 0; b0 < n_sources; b0 += C) {
        const uint32_t nr = std::min(C, n_sources - b0);
        if ((st = tg_query(g, p, sources + b0, nr, w, rows, nullptr, s)) != TG_OK) return done(st);
        if (cudaMemcpyAsync(srcs, sources + b0, nr * 4, cudaMemcpyHostToDevice, s) != cudaSuccess)
            return done(TG_ERR_CUDA);
        const unsigned grid = (unsigned)std::min<uint64_t>((nr * n + 255) / 256, 148ull * 16);
        k_topk_keys<<<grid, 256, 0, s>>>(rows, nr, (uint32_t)n, srcs, keys, vid);
        g_tg_launches++;
        unsigned long long *sk;
        uint32_t *sv;
        if ((st = tg_radix_sort_pairs(keys, vid, (uint64_t)nr * n, 32 + rbits, &sk, &sv, s)) != TG_OK) return done(st);
        uint32_t *dv = dev_out ? out_vertex + (size_t)b0 * K : ov, *dx = dev_out ? out_value + (size_t)b0 * K : oval;
        const unsigned g2 = (unsigned)std::min<uint64_t>(((uint64_t)nr * K + 255) / 256, 148ull * 16);
        k_topk_gather<<<g2, 256, 0, s>>>(sk, sv, nr, (uint32_t)n, K, dv, dx);
        g_tg_launches++;
        if (cudaGetLastError() != cudaSuccess) { tg_set_error("tg_query_topk: launch failed"); return done(TG_ERR_CUDA); }
        if (!dev_out) {
            if (cudaMemcpyAsync(out_vertex + (size_t)b0 * K, ov, (size_t)nr * K * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
                cudaMemcpyAsync(out_value + (size_t)b0 * K, oval, (size_t)nr * K * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess)
                return done(TG_ERR_CUDA);
        }
    }
    return done(TG_OK);
}

tg_status tg_query_summary(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources, tg_window w,
                           uint64_t *out_count, uint64_t *out_sum, void *cuda_stream) {
    if (!g || !sources || !out_count || !out_sum || n_sources == 0) {
        tg_set_error("tg_query_summary: NULL argument or n_sources == 0");
        return TG_ERR_INVALID;
    }
    if (!(p == TG_EAT || p == TG_FASTEST || p == TG_SHORTEST || p == TG_LD || p == TG_LD_SOURCE)) {
        tg_set_error("tg_query_summary: problem has no value row (TG_REACH: use TG_EAT)");
        return TG_ERR_INVALID;
    }
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const uint32_t C = chunk_rows(g, n_sources);
    const uint64_t n = g->n;
    uint32_t *rows = nullptr, *srcs = nullptr;
    unsigned long long *acc = nullptr;
    auto done = [&](tg_status r) {
        cudaFreeAsync(rows, s); cudaFreeAsync(srcs, s); cudaFreeAsync(acc, s);
        cudaStreamSynchronize(s);
        return r;
    };
    if (tg_malloc_async((void **)&rows, C * n * 4, s) != cudaSuccess ||
        tg_malloc_async((void **)&srcs, C * 4, s) != cudaSuccess ||
        tg_malloc_async((void **)&acc, (uint64_t)C * 16, s) != cudaSuccess) {
        cudaGetLastError();
        tg_set_error("tg_query_summary: device allocation failed");
        return done(TG_ERR_NOMEM);
    }
    std::vector<unsigned long long> h((size_t)C * 2);
    for (uint32_t b0 = 0; b0 < n_sources; b0 += C) {
        const uint32_t nr = std::min(C, n_sources - b0);
        tg_status st = tg_query(g, p, sources + b0, nr, w, rows, nullptr, s);
        if (st != TG_OK) return done(st);
        if (cudaMemcpyAsync(srcs, sources + b0, nr * 4, cudaMemcpyHostToDevice, s) != cudaSuccess ||
            cudaMemsetAsync(acc, 0, (size_t)nr * 16, s) != cudaSuccess)
            return done(TG_ERR_CUDA);
        dim3 grid((unsigned)std::min<uint64_t>((n + 255) / 256, 64), nr);
        k_row_summary<<<grid, 256, 0, s>>>(rows, (uint32_t)n, srcs, acc, acc + nr);
        g_tg_launches++;
        if (cudaGetLastError() != cudaSuccess ||
            cudaMemcpyAsync(h.data(), acc, (size_t)nr * 16, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess) {
            tg_set_error("tg_query_summary: CUDA error");
            return done(TG_ERR_CUDA);
        }
        for (uint32_t r = 0; r < nr; r++) { out_count[b0 + r] = h[r]; out_sum[b0 + r] = h[nr + r]; }
    }
    return done(TG_OK);
}

}  // extern "C"
