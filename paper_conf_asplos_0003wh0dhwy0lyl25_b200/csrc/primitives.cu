// primitives.cu -- device-wide exclusive scan and stable LSD radix sort (sm_100a).
//
// Used by the transformer (tg_build_chains): the sort of edges by (u, t, id) that
// exposes the departure nodes (v, tau) of the transformed DAG,
// and the scans that number nodes, chains and slots.
#include <cooperative_groups.h>

#include "tg_internal.cuh"

namespace {

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

// Digit width DB (8..10 bits): 2^DB buckets, DPT = 2^DB / 256 consecutive digits per
// thread in the block-level passes.
template <int DB>
__global__ void __launch_bounds__(RS_THREADS) k_radix_hist(const unsigned long long *__restrict__ keys, uint64_t m,
                                                           int shift, uint32_t *__restrict__ counts,
                                                           uint32_t ntiles) {
    constexpr int ND = 1 << DB, DPT = ND / RS_THREADS;
    __shared__ uint32_t hist[ND];
#pragma unroll
    for (int k = 0; k < DPT; k++) hist[threadIdx.x * DPT + k] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE;
#pragma unroll 4
    for (int i = 0; i < RS_ITEMS; i++) {
        const uint64_t idx = base + (uint64_t)i * RS_THREADS + threadIdx.x;
        if (idx < m) atomicAdd(&hist[(uint32_t)(keys[idx] >> shift) & (ND - 1)], 1u);
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < DPT; k++) {
        const uint32_t d = threadIdx.x * DPT + k;
        counts[(uint64_t)d * ntiles + blockIdx.x] = hist[d];
    }
}

// Stable scatter of one tile with warp-private ranking: warp w owns the contiguous
// keys [w * 512, w * 512 + 512) of the tile (16 rounds of 32 coalesced keys); a key's
// rank among equal digits of its warp is its peers below it in the round
// (__match_any_sync) plus the warp's running count of that digit, which only warp w
// touches -- no block barrier inside the ranking.  Then one block-level pass turns the
// per-warp digit counts into tile positions ((warp, round, lane) = index order, so
// the scatter is stable), the tile is staged in shared memory grouped by digit and
// written out so that consecutive threads write consecutive global positions.
template <int DB>
constexpr size_t rs_smem() {
    return (size_t)RS_TILE * (8 + 4) + (size_t)RS_WARPS * (1 << DB) * 4 + (size_t)(1 << DB) * 4 * 2 + 32 * 4;
}

template <int DB>
__global__ void __launch_bounds__(RS_THREADS) k_radix_scatter(const unsigned long long *__restrict__ kin,
                                                              const uint32_t *__restrict__ vin,
                                                              unsigned long long *__restrict__ kout,
                                                              uint32_t *__restrict__ vout, uint64_t m, int shift,
                                                              const uint32_t *__restrict__ offs, uint32_t ntiles) {
    constexpr int ND = 1 << DB, DPT = ND / RS_THREADS;
    extern __shared__ __align__(16) unsigned char smem[];
    unsigned long long *skey = (unsigned long long *)smem;
    uint32_t *sval = (uint32_t *)(skey + RS_TILE);
    uint32_t *wcnt = sval + RS_TILE;                 // [RS_WARPS][ND]
    uint32_t *tstart = wcnt + RS_WARPS * ND;         // [ND]
    uint32_t *gofs = tstart + ND;                    // [ND]
    uint32_t *wsum = gofs + ND;                      // [32]
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE;
    constexpr int PER_WARP = RS_TILE / RS_WARPS;
    const uint32_t d0 = tid * DPT;  // this thread's digits in the block-level passes

#pragma unroll
    for (int k = 0; k < DPT; k++) gofs[d0 + k] = offs[(uint64_t)(d0 + k) * ntiles + blockIdx.x];
    for (int i = tid; i < RS_WARPS * ND; i += RS_THREADS) wcnt[i] = 0;
    __syncthreads();

    uint32_t *mycnt = wcnt + warp * ND;
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
        const uint32_t d = valid ? ((uint32_t)(kk[r] >> shift) & (ND - 1)) : (uint32_t)ND;
        const uint32_t peers = __match_any_sync(0xffffffffu, d);
        const uint32_t below = __popc(peers & lt_mask);
        const uint32_t c = valid ? mycnt[d] : 0u;
        __syncwarp();
        if (valid && below == 0) mycnt[d] = c + __popc(peers);
        __syncwarp();
        lr[r] = c + below;
    }
    __syncthreads();
    // per-warp exclusive prefixes of this thread's digits, and their tile totals
    uint32_t tot[DPT], tsum = 0;
#pragma unroll
    for (int k = 0; k < DPT; k++) {
        uint32_t t = 0;
#pragma unroll
        for (int w = 0; w < RS_WARPS; w++) {
            const uint32_t c = wcnt[w * ND + d0 + k];
            wcnt[w * ND + d0 + k] = t;
            t += c;
        }
        tot[k] = t;
        tsum += t;
    }
    // exclusive scan of the digit totals (thread order = digit order) -> tile-local digit starts
    uint32_t x = tsum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) wsum[warp] = x;
    __syncthreads();
    uint32_t run = x - tsum;
#pragma unroll
    for (int w = 0; w < RS_WARPS; w++) run += (w < warp) ? wsum[w] : 0u;
#pragma unroll
    for (int k = 0; k < DPT; k++) {
        tstart[d0 + k] = run;
        run += tot[k];
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < RS_ITEMS; r++) {
        const uint64_t idx = wbase + (uint64_t)r * 32 + lane;
        if (idx < m) {
            const uint32_t d = (uint32_t)(kk[r] >> shift) & (ND - 1);
            const uint32_t p = tstart[d] + mycnt[d] + lr[r];
            skey[p] = kk[r];
            sval[p] = vv[r];
        }
    }
    __syncthreads();
    const uint32_t nvalid = (uint32_t)min((uint64_t)RS_TILE, m - base);
    for (uint32_t i = tid; i < nvalid; i += RS_THREADS) {
        const unsigned long long k = skey[i];
        const uint32_t d = (uint32_t)(k >> shift) & (ND - 1);
        const uint32_t pos = gofs[d] + (i - tstart[d]);
        kout[pos] = k;
        vout[pos] = sval[i];
    }
}

template <int DB>
tg_status radix_passes(unsigned long long *&ka, uint32_t *&va, unsigned long long *&kb, uint32_t *&vb, uint64_t m,
                       int key_bits, uint64_t ntiles, uint32_t *counts, cudaStream_t s, int snap_bits,
                       uint32_t *snap_vals, int begin_bit = 0) {
    TG_TRY_CUDA(cudaFuncSetAttribute(k_radix_scatter<DB>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)rs_smem<DB>()));
    for (int shift = begin_bit; shift < begin_bit + key_bits; shift += DB) {
        TG_LAUNCH(k_radix_hist<DB>, (unsigned)ntiles, RS_THREADS, 0, s, ka, m, shift, counts, (uint32_t)ntiles);
        TG_TRY(tg_exclusive_scan_u32(counts, counts, ntiles << DB, nullptr, s, nullptr));
        TG_LAUNCH(k_radix_scatter<DB>, (unsigned)ntiles, RS_THREADS, rs_smem<DB>(), s, ka, va, kb, vb, m, shift,
                  counts, (uint32_t)ntiles);
        std::swap(ka, kb);
        std::swap(va, vb);
        if (snap_vals && snap_bits > 0 && shift + DB == snap_bits)
            TG_TRY_CUDA(cudaMemcpyAsync(snap_vals, va, m * 4, cudaMemcpyDeviceToDevice, s));
    }
    return TG_OK;
}

}  // namespace

tg_status tg_radix_sort_pairs(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                              unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s) {
    return tg_radix_sort_pairs_snap(keys, vals, m, key_bits, sorted_keys, sorted_vals, s, 0, nullptr);
}

// As above; additionally, after the first `snap_bits` key bits have been sorted
// (snap_bits a multiple of 8), the payload order of that intermediate state (stable
// by the low snap_bits bits) is copied to snap_vals.
static tg_status radix_sort_impl(unsigned long long *keys, uint32_t *vals, uint64_t m, int begin_bit, int key_bits,
                                 unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s,
                                 int snap_bits, uint32_t *snap_vals);

tg_status tg_radix_sort_pairs_bits(unsigned long long *keys, uint32_t *vals, uint64_t m, int begin_bit, int key_bits,
                                   cudaStream_t s) {
    unsigned long long *sk;
    uint32_t *sv;
    return radix_sort_impl(keys, vals, m, begin_bit, key_bits, &sk, &sv, s, 0, nullptr);
}

tg_status tg_radix_sort_pairs_snap(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                                   unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s,
                                   int snap_bits, uint32_t *snap_vals) {
    return radix_sort_impl(keys, vals, m, 0, key_bits, sorted_keys, sorted_vals, s, snap_bits, snap_vals);
}

static tg_status radix_sort_impl(unsigned long long *keys, uint32_t *vals, uint64_t m, int begin_bit, int key_bits,
                                 unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s,
                                 int snap_bits, uint32_t *snap_vals) {
    if (snap_vals && m >= 1 && (snap_bits <= 0 || m == 1 || key_bits <= 0))
        TG_TRY_CUDA(cudaMemcpyAsync(snap_vals, vals, m * 4, cudaMemcpyDeviceToDevice, s));
    *sorted_keys = keys;
    *sorted_vals = vals;
    if (m <= 1 || key_bits <= 0) return TG_OK;
    uint64_t ntiles = (m + RS_TILE - 1) / RS_TILE;
    if ((ntiles << 10) >= 0xFFFFFFFFull) {
        tg_set_error("radix sort: too many tiles");
        return TG_ERR_RANGE;
    }
    // digit width: the fewest passes over the key bits (ties: the narrower digit); an
    // intermediate snapshot (sweep time order) needs whole 8-bit digits
    int db = 8;
    if (!(snap_vals && snap_bits > 0)) {
        const int p8 = (key_bits + 7) / 8, p9 = (key_bits + 8) / 9, p10 = (key_bits + 9) / 10;
        db = (p10 < p9 && p10 < p8) ? 10 : (p9 < p8 ? 9 : 8);
#ifdef TG_RS_DB_FORCE
        db = TG_RS_DB_FORCE;  // tuning experiments
#endif
    }
    unsigned long long *k2 = nullptr;
    uint32_t *v2 = nullptr, *counts = nullptr;
    TG_TRY_CUDA(tg_malloc_async((void **)&k2, m * 8, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&v2, m * 4, s));
    TG_TRY_CUDA(tg_malloc_async((void **)&counts, (ntiles << db) * 4, s));
    unsigned long long *ka = keys, *kb = k2;
    uint32_t *va = vals, *vb = v2;
    if (db == 10) TG_TRY((radix_passes<10>(ka, va, kb, vb, m, key_bits, ntiles, counts, s, snap_bits, snap_vals, begin_bit)));
    else if (db == 9) TG_TRY((radix_passes<9>(ka, va, kb, vb, m, key_bits, ntiles, counts, s, snap_bits, snap_vals, begin_bit)));
    else TG_TRY((radix_passes<8>(ka, va, kb, vb, m, key_bits, ntiles, counts, s, snap_bits, snap_vals, begin_bit)));
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
