// primitives.cu -- device-wide exclusive scan and stable LSD radix sort (sm_100a).
//
// Used by the transformer (tg_build_chains): the sort of edges by (u, t, id) that
// exposes the departure nodes (v, tau) of the transformed DAG,
// and the scans that number nodes, chains and slots.
#include <cooperative_groups.h>

#include "tg_internal.cuh"

namespace {

#ifndef TG_RS_V2
#define TG_RS_V2 1  // radix scatter with warp-private ranking
#endif

constexpr int SCAN_THREADS = 256;
constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

template <typename T>
__device__ __forceinline__ T block_excl_scan(T v, T *sh, T &total) {
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    constexpr int NW = SCAN_THREADS / 32;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) sh[wid] = x;
    __syncthreads();
    if (wid == 0) {
        T w = (lane < NW) ? sh[lane] : T(0);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        if (lane < NW) sh[lane] = w;
    }
    __syncthreads();
    T wp = wid ? sh[wid - 1] : T(0);
    total = sh[NW - 1];
    __syncthreads();
    return wp + x - v;
}

// Each thread owns SCAN_ITEMS consecutive elements (two 16-byte loads when the tile is
// full), so a tile needs one block-wide scan of the thread totals.
__device__ __forceinline__ void scan_load8(const uint32_t *in, uint64_t idx, uint64_t count, uint32_t (&x)[SCAN_ITEMS]) {
    if (idx + SCAN_ITEMS <= count) {
        const uint4 a = *(const uint4 *)(in + idx), b = *(const uint4 *)(in + idx + 4);
        x[0] = a.x; x[1] = a.y; x[2] = a.z; x[3] = a.w; x[4] = b.x; x[5] = b.y; x[6] = b.z; x[7] = b.w;
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_ITEMS; i++) x[i] = (idx + i < count) ? in[idx + i] : 0u;
    }
}

__global__ void k_scan_reduce(const uint32_t *__restrict__ in, uint64_t count, uint32_t *__restrict__ sums) {
    __shared__ uint32_t sh[32];
    const uint64_t idx = (uint64_t)blockIdx.x * SCAN_TILE + (uint64_t)threadIdx.x * SCAN_ITEMS;
    uint32_t x[SCAN_ITEMS];
    scan_load8(in, idx, count, x);
    uint32_t acc = 0;
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; i++) acc += x[i];
    uint32_t total;
    block_excl_scan<uint32_t>(acc, sh, total);
    if (threadIdx.x == 0) sums[blockIdx.x] = total;
}

// in == out is allowed: every thread reads its own elements before writing them.
__global__ void k_scan_apply(const uint32_t *in, uint32_t *out, uint64_t count,
                             const uint32_t *__restrict__ tile_off, uint32_t *d_total) {
    __shared__ uint32_t sh[32];
    const uint64_t idx = (uint64_t)blockIdx.x * SCAN_TILE + (uint64_t)threadIdx.x * SCAN_ITEMS;
    uint32_t x[SCAN_ITEMS];
    scan_load8(in, idx, count, x);
    uint32_t acc = 0;
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; i++) acc += x[i];
    uint32_t total;
    uint32_t run = block_excl_scan<uint32_t>(acc, sh, total) + (tile_off ? tile_off[blockIdx.x] : 0u);
#pragma unroll
    for (int i = 0; i < SCAN_ITEMS; i++) {
        const uint32_t v = x[i];
        x[i] = run;
        run += v;
    }
    if (idx + SCAN_ITEMS <= count) {
        *(uint4 *)(out + idx) = make_uint4(x[0], x[1], x[2], x[3]);
        *(uint4 *)(out + idx + 4) = make_uint4(x[4], x[5], x[6], x[7]);
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_ITEMS; i++)
            if (idx + i < count) out[idx + i] = x[i];
    }
    if (d_total && blockIdx.x == gridDim.x - 1 && threadIdx.x == SCAN_THREADS - 1) *d_total = run;
}

}  // namespace

tg_status tg_exclusive_scan_u32(const uint32_t *in, uint32_t *out, uint64_t count, uint32_t *d_total,
                                cudaStream_t s, DevArena *) {
    if (count == 0) {
        if (d_total) TG_TRY_CUDA(cudaMemsetAsync(d_total, 0, 4, s));
        return TG_OK;
    }
    uint64_t tiles = (count + SCAN_TILE - 1) / SCAN_TILE;
    if (tiles == 1) {
        TG_LAUNCH(k_scan_apply, 1, SCAN_THREADS, 0, s, in, out, count, (const uint32_t *)nullptr, d_total);
        return TG_OK;
    }
    uint32_t *sums = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&sums, tiles * sizeof(uint32_t), s));
    TG_LAUNCH(k_scan_reduce, (unsigned)tiles, SCAN_THREADS, 0, s, in, count, sums);
    tg_status st = tg_exclusive_scan_u32(sums, sums, tiles, nullptr, s, nullptr);
    if (st != TG_OK) { cudaFreeAsync(sums, s); return st; }
    TG_LAUNCH(k_scan_apply, (unsigned)tiles, SCAN_THREADS, 0, s, in, out, count, sums, d_total);
    TG_TRY_CUDA(cudaFreeAsync(sums, s));
    return TG_OK;
}

// ============================================================================ radix sort
namespace {

constexpr int RS_THREADS = 256;
constexpr int RS_ITEMS = 16;
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;  // 4096 keys per tile
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr size_t RS_SMEM = (size_t)RS_TILE * (8 + 4) + 2 * RS_WARPS * 256 * 4 + 256 * 4 * 2;

__global__ void __launch_bounds__(RS_THREADS) k_radix_hist(const unsigned long long *__restrict__ keys, uint64_t m,
                                                           int shift, uint32_t *__restrict__ counts,
                                                           uint32_t ntiles) {
    __shared__ uint32_t hist[256];
    hist[threadIdx.x] = 0;
    __syncthreads();
    uint64_t base = (uint64_t)blockIdx.x * RS_TILE;
#pragma unroll 4
    for (int i = 0; i < RS_ITEMS; i++) {
        uint64_t idx = base + (uint64_t)i * RS_THREADS + threadIdx.x;
        if (idx < m) atomicAdd(&hist[(uint32_t)(keys[idx] >> shift) & 255u], 1u);
    }
    __syncthreads();
    counts[(uint64_t)threadIdx.x * ntiles + blockIdx.x] = hist[threadIdx.x];
}

// Stable scatter of one tile: ranks are computed in element order (round, warp,
// lane), the tile is staged in shared memory grouped by digit, then written out
// so that consecutive threads write consecutive global positions.
__global__ void __launch_bounds__(RS_THREADS) k_radix_scatter(const unsigned long long *__restrict__ kin,
                                                              const uint32_t *__restrict__ vin,
                                                              unsigned long long *__restrict__ kout,
                                                              uint32_t *__restrict__ vout, uint64_t m, int shift,
                                                              const uint32_t *__restrict__ offs, uint32_t ntiles) {
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned long long *skey = (unsigned long long *)smem;
    uint32_t *sval = (uint32_t *)(skey + RS_TILE);
    uint32_t *wcnt = sval + RS_TILE;                 // [2][RS_WARPS][256]
    uint32_t *tstart = wcnt + 2 * RS_WARPS * 256;    // [256]
    uint32_t *gofs = tstart + 256;                   // [256]
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE;

    gofs[tid] = offs[(uint64_t)tid * ntiles + blockIdx.x];
    for (int w = 0; w < 2 * RS_WARPS; w++) wcnt[w * 256 + tid] = 0;
    __syncthreads();

    uint32_t lr[RS_ITEMS];
    unsigned long long kk[RS_ITEMS];
    uint32_t vv[RS_ITEMS];
    uint32_t running = 0;  // thread tid owns digit tid
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        uint32_t *A = wcnt + (r & 1) * RS_WARPS * 256;
        uint32_t *B = wcnt + ((r + 1) & 1) * RS_WARPS * 256;
        uint64_t idx = base + (uint64_t)r * RS_THREADS + tid;
        bool valid = idx < m;
        kk[r] = valid ? kin[idx] : 0ull;
        vv[r] = valid ? vin[idx] : 0u;
        uint32_t d = valid ? ((uint32_t)(kk[r] >> shift) & 255u) : 0x100u;
        uint32_t peers = __match_any_sync(0xffffffffu, d);
        uint32_t rank = __popc(peers & lt_mask);
        if (valid && rank == 0) A[warp * 256 + d] = __popc(peers);
        __syncthreads();
        {
            uint32_t run = running;
#pragma unroll
            for (int w = 0; w < RS_WARPS; w++) {
                uint32_t c = A[w * 256 + tid];
                A[w * 256 + tid] = run;
                run += c;
            }
            running = run;
#pragma unroll
            for (int w = 0; w < RS_WARPS; w++) B[w * 256 + tid] = 0;
        }
        __syncthreads();
        lr[r] = valid ? (A[warp * 256 + d] + rank) : 0u;
    }
    // exclusive scan of the tile's digit totals -> tile-local digit starts
    {
        uint32_t x = running;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= o) x += y;
        }
        __syncthreads();
        if (lane == 31) wcnt[warp] = x;
        __syncthreads();
        uint32_t wp = 0;
        for (int w = 0; w < warp; w++) wp += wcnt[w];
        tstart[tid] = wp + x - running;
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        uint64_t idx = base + (uint64_t)r * RS_THREADS + tid;
        if (idx < m) {
            uint32_t d = (uint32_t)(kk[r] >> shift) & 255u;
            uint32_t p = tstart[d] + lr[r];
            skey[p] = kk[r];
            sval[p] = vv[r];
        }
    }
    __syncthreads();
    uint32_t nvalid = (uint32_t)min((uint64_t)RS_TILE, m - base);
    for (uint32_t i = tid; i < nvalid; i += RS_THREADS) {
        unsigned long long k = skey[i];
        uint32_t d = (uint32_t)(k >> shift) & 255u;
        uint32_t pos = gofs[d] + (i - tstart[d]);
        kout[pos] = k;
        vout[pos] = sval[i];
    }
}

#if TG_RS_V2
// Stable scatter of one tile with warp-private ranking: warp w owns the contiguous
// keys [w * 512, w * 512 + 512) of the tile (16 rounds of 32 coalesced keys); a key's
// rank among equal digits of its warp is its peers below it in the round
// (__match_any_sync) plus the warp's running count of that digit, which only warp w
// touches -- no block barrier inside the ranking.  Then one block-level pass turns the
// per-warp digit counts into tile positions ((warp, round, lane) = index order, so
// the scatter is stable), the tile is staged in shared memory grouped by digit and
// written out so that consecutive threads write consecutive global positions.
constexpr size_t RS2_SMEM = (size_t)RS_TILE * (8 + 4) + RS_WARPS * 256 * 4 + 256 * 4 * 2 + 32 * 4;

__global__ void __launch_bounds__(RS_THREADS) k_radix_scatter2(const unsigned long long *__restrict__ kin,
                                                               const uint32_t *__restrict__ vin,
                                                               unsigned long long *__restrict__ kout,
                                                               uint32_t *__restrict__ vout, uint64_t m, int shift,
                                                               const uint32_t *__restrict__ offs, uint32_t ntiles) {
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned long long *skey = (unsigned long long *)smem;
    uint32_t *sval = (uint32_t *)(skey + RS_TILE);
    uint32_t *wcnt = sval + RS_TILE;                 // [RS_WARPS][256]
    uint32_t *tstart = wcnt + RS_WARPS * 256;        // [256]
    uint32_t *gofs = tstart + 256;                   // [256]
    uint32_t *wsum = gofs + 256;                     // [32]
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE;
    constexpr int PER_WARP = RS_TILE / RS_WARPS;

    gofs[tid] = offs[(uint64_t)tid * ntiles + blockIdx.x];
#pragma unroll
    for (int w = 0; w < RS_WARPS; w++) wcnt[w * 256 + tid] = 0;
    __syncthreads();

    uint32_t *mycnt = wcnt + warp * 256;
    unsigned long long kk[RS_ITEMS];
    uint32_t vv[RS_ITEMS], lr[RS_ITEMS];
    const uint64_t wbase = base + (uint64_t)warp * PER_WARP;
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        const uint64_t idx = wbase + (uint64_t)r * 32 + lane;
        const bool valid = idx < m;
        kk[r] = valid ? kin[idx] : ~0ull;
        vv[r] = valid ? vin[idx] : 0u;
    }
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        const uint64_t idx = wbase + (uint64_t)r * 32 + lane;
        const bool valid = idx < m;
        const uint32_t d = valid ? ((uint32_t)(kk[r] >> shift) & 255u) : 0x100u;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        const uint32_t below = __popc(peers & lt_mask);
        const uint32_t c = valid ? mycnt[d] : 0u;
        __syncwarp();
        if (valid && below == 0) mycnt[d] = c + __popc(peers);
        __syncwarp();
        lr[r] = c + below;
    }
    __syncthreads();
    // thread tid owns digit tid: per-warp exclusive prefixes and the tile total
    uint32_t tot = 0;
#pragma unroll
    for (int w = 0; w < RS_WARPS; w++) {
        const uint32_t c = wcnt[w * 256 + tid];
        wcnt[w * 256 + tid] = tot;
        tot += c;
    }
    // exclusive scan of the digit totals -> tile-local digit starts
    uint32_t x = tot;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t wp = 0;
#pragma unroll
    for (int w = 0; w < RS_WARPS; w++) wp += (w < warp) ? wsum[w] : 0u;
    tstart[tid] = wp + x - tot;
    __syncthreads();
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        const uint64_t idx = wbase + (uint64_t)r * 32 + lane;
        if (idx < m) {
            const uint32_t d = (uint32_t)(kk[r] >> shift) & 255u;
            const uint32_t p = tstart[d] + mycnt[d] + lr[r];
            skey[p] = kk[r];
            sval[p] = vv[r];
        }
    }
    __syncthreads();
    const uint32_t nvalid = (uint32_t)min((uint64_t)RS_TILE, m - base);
    for (uint32_t i = tid; i < nvalid; i += RS_THREADS) {
        const unsigned long long k = skey[i];
        const uint32_t d = (uint32_t)(k >> shift) & 255u;
        const uint32_t pos = gofs[d] + (i - tstart[d]);
        kout[pos] = k;
        vout[pos] = sval[i];
    }
}
#endif

}  // namespace

tg_status tg_radix_sort_pairs(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                              unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s) {
    return tg_radix_sort_pairs_snap(keys, vals, m, key_bits, sorted_keys, sorted_vals, s, 0, nullptr);
}

// As above; additionally, after the first `snap_bits` key bits have been sorted
// (snap_bits a multiple of 8), the payload order of that intermediate state (stable
// by the low snap_bits bits) is copied to snap_vals.
tg_status tg_radix_sort_pairs_snap(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                                   unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s,
                                   int snap_bits, uint32_t *snap_vals) {
    if (snap_vals && m >= 1 && (snap_bits <= 0 || m == 1 || key_bits <= 0))
        TG_TRY_CUDA(cudaMemcpyAsync(snap_vals, vals, m * 4, cudaMemcpyDeviceToDevice, s));
    *sorted_keys = keys;
    *sorted_vals = vals;
    if (m <= 1 || key_bits <= 0) return TG_OK;
    uint64_t ntiles = (m + RS_TILE - 1) / RS_TILE;
    if (ntiles * 256 >= 0xFFFFFFFFull) {
        tg_set_error("radix sort: too many tiles");
        return TG_ERR_RANGE;
    }
    unsigned long long *k2 = nullptr;
    uint32_t *v2 = nullptr, *counts = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&k2, m * 8, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&v2, m * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&counts, ntiles * 256 * 4, s));
#if TG_RS_V2
    TG_TRY_CUDA(cudaFuncSetAttribute(k_radix_scatter2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)RS2_SMEM));
#else
    TG_TRY_CUDA(cudaFuncSetAttribute(k_radix_scatter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)RS_SMEM));
#endif
    unsigned long long *ka = keys, *kb = k2;
    uint32_t *va = vals, *vb = v2;
    for (int shift = 0; shift < key_bits; shift += 8) {
        TG_LAUNCH(k_radix_hist, (unsigned)ntiles, RS_THREADS, 0, s, ka, m, shift, counts, (uint32_t)ntiles);
        TG_TRY(tg_exclusive_scan_u32(counts, counts, ntiles * 256, nullptr, s, nullptr));
#if TG_RS_V2
        TG_LAUNCH(k_radix_scatter2, (unsigned)ntiles, RS_THREADS, RS2_SMEM, s, ka, va, kb, vb, m, shift, counts,
                  (uint32_t)ntiles);
#else
        TG_LAUNCH(k_radix_scatter, (unsigned)ntiles, RS_THREADS, RS_SMEM, s, ka, va, kb, vb, m, shift, counts,
                  (uint32_t)ntiles);
#endif
        std::swap(ka, kb);
        std::swap(va, vb);
        if (snap_vals && snap_bits > 0 && shift + 8 == snap_bits)
            TG_TRY_CUDA(cudaMemcpyAsync(snap_vals, va, m * 4, cudaMemcpyDeviceToDevice, s));
    }
    TG_TRY_CUDA(cudaFreeAsync(counts, s));
    if (ka != keys) {
        // result lives in the scratch buffers: copy back so the caller's buffers hold it
        TG_TRY_CUDA(cudaMemcpyAsync(keys, ka, m * 8, cudaMemcpyDeviceToDevice, s));
        TG_TRY_CUDA(cudaMemcpyAsync(vals, va, m * 4, cudaMemcpyDeviceToDevice, s));
    }
    TG_TRY_CUDA(cudaFreeAsync(k2, s));
    TG_TRY_CUDA(cudaFreeAsync(v2, s));
    return TG_OK;
}
