// query_sweep.cu -- EAT / LD / REACH by a time-partitioned sweep of the expanded DAG (sm_100a).
//
// Paper: §4.3 divides the skeleton graph "into a series of partitions according
// to their topological order" and processes the partitions along that order; the time
// of a departure is a topological order of the time-expanded DAG (every edge departs
// strictly before its successors: duration >= 1, reading A2).  Here the partitions are
// taken down to the edge level (DESIGN.md §5 "sweep schedule"):
//
//   edges sorted by departure time, te[i] = {u, v, t, t + duration} (built with the
//   (u, t) sort, build.cu), are cut into partitions [T_b, T_e) of ~part_edges edges at
//   distinct-time boundaries.  A partition is processed in two steps:
//     dense   every edge e = (u, v, t) of the partition, for all S queries of the
//             sub-batch at once (lanes = queries): usable for query q iff
//             EAT(u, q) <= t (window: t >= alpha, t + duration <= omega); then
//             atomicMin(state(v, q), arrival [| id]).  States of arrivals < T_b are
//             final (all earlier partitions are complete), so this decides every edge
//             whose tail was reached before T_b.
//     fixup   an improvement of (v, q) to an arrival a < T_e may enable edges of v that
//             depart in [a, T_e) and were already checked: the unit (v, query group) is
//             pushed to a frontier (bitmap + queue, deduplicated), and the next round
//             re-relaxes v's edges departing in [a, min(last activation, T_e)) through the
//             occurrence index (the GAC activation of query_eat.cu restricted to the
//             partition; `lat` keeps concurrent activations disjoint).  Rounds repeat
//             until no improvement lands inside the partition.
// One cooperative kernel runs all partitions and rounds of a sub-batch (grid-wide
// barriers between phases), so there is no host round trip.  The result is the
// unique fixpoint (EAT, and with packed words the minimum optimal edge id, reading
// A9), identical to the one-pass oracle; tests compare bit for bit.
#include <cooperative_groups.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "tg_internal.cuh"

namespace cg = cooperative_groups;

namespace {

constexpr int SW_T = 256;            // threads per block
constexpr uint32_t FIX_CHUNK = 64;   // occurrences per fixup chunk

struct SweepCtl {
    uint32_t qcnt[3];     // frontier unit queue counts, ring by round
    uint32_t ccnt[3];     // fixup chunk counts, ring by round
    uint32_t rcnt[3];     // chunk record counts, ring by round
    uint32_t rounds;      // fixup rounds run (stats)
    uint32_t parts;       // partitions run (stats)
    uint32_t fix_units;   // frontier units processed (stats)
    uint32_t claim[2];    // dense-step chunk claim counters, by partition parity
    unsigned long long ns[4];  // stats: leader's globaltimer time in dense / fixup A / fixup B / other
};

struct SwP {
    const int4 *te;
    const uint32_t *te_id;
    uint32_t e_begin, e_end;  // window-clipped time-sorted edge range
    uint32_t part_edges;
    const uint32_t *vnode_off, *node_t, *node_eoff, *occ_slot;
    const int4 *slots;
    void *st;       // [v * R + q] packed u64 (PK) or u32 arrival
    uint32_t *lat;  // [v * R + q] departure time up to which v's edges were (re)activated for q
    uint32_t *hb;   // [v * R + q] exclusive departure bound of the edges a fixup must re-check
    uint32_t n, R, G;
    uint32_t alpha, omega;
    uint32_t *fb[2];  // frontier bitmaps [v * G + g] by round parity
    uint32_t *fq[2];  // frontier unit queues by round parity (capacity n * G: bitmap dedupe)
    uint2 *recs;      // fixup chunk records: 32 per-query edge ranges
    uint4 *chq;       // fixup chunks {record, begin, end, unit}
    uint32_t chcap, reccap;
    SweepCtl *ctl;
    int exp;  // diagnostics (results invalid when != 0): 1 = no fixup rounds
};

template <bool PK> struct StW;
template <> struct StW<true> {
    using T = unsigned long long;
    static __device__ __forceinline__ T make(uint32_t arr, uint32_t id) { return ((T)arr << 32) | id; }
    static __device__ __forceinline__ uint32_t time(T w) { return (uint32_t)(w >> 32); }
};
template <> struct StW<false> {
    using T = uint32_t;
    static __device__ __forceinline__ T make(uint32_t arr, uint32_t) { return arr; }
    static __device__ __forceinline__ uint32_t time(T w) { return w; }
};

// QPL consecutive state words of one row (one vector load per lane; the warp reads the
// row [base, base + 32 * QPL) in one coalesced request)
template <bool PK, int QPL>
__device__ __forceinline__ void row_load(const void *st, size_t base, typename StW<PK>::T (&x)[QPL]) {
    using T = typename StW<PK>::T;
    const T *p = (const T *)st + base;
    if constexpr (QPL == 1) {
        x[0] = __ldcg(p);
    } else if constexpr (!PK && QPL == 2) {
        const uint2 r = __ldcg((const uint2 *)p);
        x[0] = r.x; x[1] = r.y;
    } else if constexpr (!PK && QPL == 4) {
        const uint4 r = __ldcg((const uint4 *)p);
        x[0] = r.x; x[1] = r.y; x[2] = r.z; x[3] = r.w;
    } else {  // PK: 16-byte loads of two packed words
#pragma unroll
        for (int j = 0; j < QPL; j += 2) {
            const ulonglong2 r = __ldcg((const ulonglong2 *)(p + j));
            x[j] = r.x; x[j + 1] = r.y;
        }
    }
}

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ uint32_t lower_bound_t(const int4 *te, uint32_t lo, uint32_t hi, uint32_t key) {
    while (lo < hi) {
        const uint32_t mid = lo + ((hi - lo) >> 1);
        if ((uint32_t)__ldg(&te[mid].z) < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

// Frontier push of unit (v, g) with query bits; the thread whose atomicOr turns the
// word non-zero appends the unit to the queue (the bitmap deduplicates).
__device__ __forceinline__ void push_unit(const SwP &P, int par, uint32_t unit, uint32_t bits, uint32_t *qcnt) {
    const uint32_t old = atomicOr(P.fb[par] + unit, bits);
    if (old == 0u) P.fq[par][atomicAdd(qcnt, 1u)] = unit;
}

// ---------------------------------------------------------------------------- dense step
// Warps claim 32-edge chunks of the partition in time order (dynamic counter); lane i
// loads edge i (one coalesced 512 B request), then edges are taken UNR at a time: their
// tail rows (all queries, QPL per lane) are read together, and for the edges usable by
// some query the head rows, then the improving atomics.
//
// Window bound (which already-checked edges can have missed an improvement): an
// improvement of (v, q) to arrival a can only have been missed by edges claimed before
// it became visible.  The improver fences and reads the claim counter h: chunks >= h are
// claimed later and their row reads see the improvement (claim -> fence -> read; write ->
// fence -> read: one of the two sees the other).  Chunks < h hold departures <= t_H (the
// first departure of chunk h), so the fixup of v is bounded to departures in [a, t_H]
// -- and is not needed at all when a > t_H.
template <bool PK, int QPL>
__device__ __forceinline__ void dense_part(const SwP &P, uint32_t b0, uint32_t b1, uint32_t Te, int par_out,
                                           uint32_t *qcnt_out, uint32_t *claim) {
    using T = typename StW<PK>::T;
    constexpr int UNR = 4;
    constexpr int LPG = 32 / QPL;  // lanes per query group of 32
    const int lane = threadIdx.x & 31;
    const uint32_t q0 = lane * QPL;
    const uint32_t nchunks = (b1 - b0 + 31) / 32;
    for (;;) {
        uint32_t c = 0;
        if (lane == 0) {
            c = atomicAdd(claim, 1u);
            if (P.exp != 2) __threadfence();
        }
        c = __shfl_sync(0xffffffffu, c, 0);
        if (c >= nchunks) break;
        const uint32_t base = b0 + c * 32;
        const uint32_t i = base + lane;
        int4 e = make_int4(0, 0, 0, 0);
        uint32_t id = TG_NONE;
        bool ok = false;
        if (i < b1) {
            e = __ldg(P.te + i);
            if (PK) id = __ldg(P.te_id + i);
            ok = (uint32_t)e.w <= P.omega;  // t >= alpha by the range; arrival within the window
        }
        uint32_t todo = __ballot_sync(0xffffffffu, ok);
        while (todo) {
            int src[UNR];
#pragma unroll
            for (int j = 0; j < UNR; j++) {
                src[j] = todo ? __ffs(todo) - 1 : -1;
                if (todo) todo &= todo - 1;
            }
            uint32_t eu[UNR], ev[UNR], et[UNR], ea[UNR], eid[UNR];
#pragma unroll
            for (int j = 0; j < UNR; j++) {
                const int sl = src[j] < 0 ? 0 : src[j];
                eu[j] = __shfl_sync(0xffffffffu, (uint32_t)e.x, sl);
                ev[j] = __shfl_sync(0xffffffffu, (uint32_t)e.y, sl);
                et[j] = __shfl_sync(0xffffffffu, (uint32_t)e.z, sl);
                ea[j] = __shfl_sync(0xffffffffu, (uint32_t)e.w, sl);
                eid[j] = __shfl_sync(0xffffffffu, id, sl);
            }
            T ur[UNR][QPL];
#pragma unroll
            for (int j = 0; j < UNR; j++)
                if (src[j] >= 0) row_load<PK, QPL>(P.st, (size_t)eu[j] * P.R + q0, ur[j]);
            bool use[UNR][QPL];
            bool any[UNR];
#pragma unroll
            for (int j = 0; j < UNR; j++) {
                bool a = false;
#pragma unroll
                for (int k = 0; k < QPL; k++) {
                    use[j][k] = src[j] >= 0 && StW<PK>::time(ur[j][k]) <= et[j];
                    a |= use[j][k];
                }
                any[j] = __any_sync(0xffffffffu, a);
            }
            T vr[UNR][QPL];
#pragma unroll
            for (int j = 0; j < UNR; j++)
                if (any[j]) row_load<PK, QPL>(P.st, (size_t)ev[j] * P.R + q0, vr[j]);
            uint32_t ib[UNR];
            uint32_t ot[UNR][QPL];  // arrival before the improvement: edges departing at >= it
                                    // were usable before (relaxed, or pending in a fixup)
#pragma unroll
            for (int j = 0; j < UNR; j++) {
                ib[j] = 0;
                if (!any[j]) continue;
                const T cand = StW<PK>::make(ea[j], eid[j]);
#pragma unroll
                for (int k = 0; k < QPL; k++) {
                    ot[j][k] = 0;
                    if (use[j][k] && cand < vr[j][k]) {
                        const T old = atomicMin((T *)P.st + (size_t)ev[j] * P.R + q0 + k, cand);
                        ot[j][k] = StW<PK>::time(old);
                        if (ea[j] < ot[j][k] && ea[j] < Te) ib[j] |= 1u << k;
                    }
                }
            }
            bool need = false;
#pragma unroll
            for (int j = 0; j < UNR; j++) need |= ib[j] != 0;
            if (P.exp == 3 || !__any_sync(0xffffffffu, need)) continue;
            // some improvement lands inside the partition: bound it by the claim window
            uint32_t h = 0;
            if (lane == 0) {
                if (P.exp != 2) __threadfence();
                h = *(volatile uint32_t *)claim;
            }
            h = __shfl_sync(0xffffffffu, h, 0);
            const uint64_t hx = (uint64_t)b0 + (uint64_t)h * 32;
            const uint32_t tH = hx < b1 ? (uint32_t)__ldg(&P.te[hx].z) : Te;
#pragma unroll
            for (int j = 0; j < UNR; j++) {
                uint32_t bits = 0;
                if (ib[j] && ea[j] <= tH) {
#pragma unroll
                    for (int k = 0; k < QPL; k++)
                        if ((ib[j] >> k) & 1u) {
                            atomicMax(P.hb + (size_t)ev[j] * P.R + q0 + k, min(ot[j][k], tH + 1));
                            bits |= 1u << ((q0 + k) & 31);
                        }
                }
#pragma unroll
                for (int o = LPG / 2; o; o >>= 1) bits |= __shfl_xor_sync(0xffffffffu, bits, o);
                if ((lane % LPG) == 0 && bits) push_unit(P, par_out, ev[j] * P.G + lane / LPG, bits, qcnt_out);
            }
        }
    }
}

// ---------------------------------------------------------------------------- fixup step
// Per-warp staging of one 32-edge block: (edge, query) pairs as 16-bit entries and slots.
struct WarpStage {
    uint16_t pairs[1024];
    int4 slot[32];
};

// Relax occurrences [pbeg, pend) for the queries of group g whose range [lo, hi) holds
// them (lane = query).  The pairs of a 32-edge block are expanded edge-major so that the
// queries of one edge read adjacent state words; improvements inside the partition are
// pushed with an unbounded window (the dense step of the partition is over).
template <bool PK>
__device__ __forceinline__ void fix_chunk(const SwP &P, uint32_t g, uint32_t lo, uint32_t hi, uint32_t pbeg,
                                          uint32_t pend, uint32_t Te, int par_out, uint32_t *qcnt_out,
                                          WarpStage &ws) {
    using T = typename StW<PK>::T;
    constexpr int MLP = 4;
    const int lane = threadIdx.x & 31;
    for (uint32_t pb = pbeg; pb < pend; pb += 32) {
        const uint32_t p = pb + lane;
        int4 sl = make_int4(0, -1, 0, 0);
        if (p < pend) sl = __ldg(P.slots + __ldg(P.occ_slot + p));
        uint32_t mask = tg_warp_transpose32(lo < hi ? tg_block_bits(lo, hi, pb) : 0u);
        if (p >= pend || (uint32_t)sl.y > P.omega) mask = 0;
        const uint32_t cnt = __popc(mask);
        uint32_t incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        if (total == 0) continue;
        ws.slot[lane] = sl;
        uint32_t pos = incl - cnt, mm = mask;
        while (mm) {
            const uint32_t bq = __ffs(mm) - 1;
            mm &= mm - 1;
            ws.pairs[pos++] = (uint16_t)((lane << 5) | bq);
        }
        __syncwarp();
        for (uint32_t t0 = 0; t0 < total; t0 += 32 * MLP) {
            T cur[MLP];
#pragma unroll
            for (int j = 0; j < MLP; j++) {
                const uint32_t t = t0 + j * 32 + lane;
                if (t < total) {
                    const uint32_t e = ws.pairs[t];
                    cur[j] = __ldcg((const T *)P.st + (size_t)(uint32_t)ws.slot[e >> 5].x * P.R + g * 32 + (e & 31));
                }
            }
#pragma unroll
            for (int j = 0; j < MLP; j++) {
                const uint32_t t = t0 + j * 32 + lane;
                if (t >= total) continue;
                const uint32_t e = ws.pairs[t];
                const int4 s = ws.slot[e >> 5];
                const uint32_t q = g * 32 + (e & 31), v = (uint32_t)s.x, a = (uint32_t)s.y;
                const T cand = StW<PK>::make(a, (uint32_t)s.z);
                if (cand < cur[j]) {
                    const size_t si = (size_t)v * P.R + q;
                    const T old = atomicMin((T *)P.st + si, cand);
                    const uint32_t ot = StW<PK>::time(old);
                    if (a < ot && a < Te) {
                        // departures >= the previous arrival were usable before (relaxed, or
                        // pending in an earlier push): only [a, ot) can be new
                        atomicMax(P.hb + si, ot);
                        push_unit(P, par_out, v * P.G + g, 1u << (q & 31), qcnt_out);
                    }
                }
            }
        }
        __syncwarp();
    }
}

template <bool PK, int QPL>
__global__ void __launch_bounds__(SW_T) k_sweep(SwP P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ uint32_t s_b1, s_Te;
    __shared__ WarpStage stage[SW_T / 32];
    WarpStage &ws = stage[threadIdx.x >> 5];
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    const bool leader = blockIdx.x == 0 && threadIdx.x == 0;
    uint32_t r = 0;      // global round index (dense steps and fixup rounds)
    uint32_t part = 0;
    uint32_t b0 = P.e_begin;
    while (b0 < P.e_end) {
        if (threadIdx.x == 0) {
            // partition [b0, b1): about part_edges edges, cut where the time changes
            uint32_t b1;
            if ((uint64_t)b0 + P.part_edges >= P.e_end) {
                b1 = P.e_end;
            } else {
                const uint32_t tgt = b0 + P.part_edges;
                const uint32_t tt = (uint32_t)__ldg(&P.te[tgt].z);
                b1 = lower_bound_t(P.te, b0 + 1, tgt, tt);
                if (b1 <= b0 + 1 && (uint32_t)__ldg(&P.te[b0].z) == tt)
                    b1 = lower_bound_t(P.te, tgt, P.e_end, tt + 1);  // one time value fills the partition
            }
            s_b1 = b1;
            s_Te = (b1 < P.e_end) ? (uint32_t)__ldg(&P.te[b1].z) : P.omega;
        }
        __syncthreads();
        const uint32_t b1 = s_b1, Te = s_Te;
        __syncthreads();
        // dense step = round r: writes frontier r+1
        if (leader) {
            P.ctl->qcnt[(r + 2) % 3] = 0;
            P.ctl->ccnt[(r + 2) % 3] = 0;
            P.ctl->rcnt[(r + 2) % 3] = 0;
            P.ctl->claim[(part + 1) & 1] = 0;  // the next partition's claim counter (unused now)
            P.ctl->parts++;
        }
        unsigned long long t0 = leader ? gtimer() : 0;
        dense_part<PK, QPL>(P, b0, b1, Te, (r + 1) & 1, &P.ctl->qcnt[(r + 1) % 3], &P.ctl->claim[part & 1]);
        grid.sync();
        if (leader) { const unsigned long long t1 = gtimer(); P.ctl->ns[0] += t1 - t0; t0 = t1; }
        r++;
        // fixup rounds until nothing lands inside the partition:
        //   A: per frontier unit, the queries' ranges [now, min(last activation, window, T_e))
        //      -> a record of 32 ranges + chunks of FIX_CHUNK occurrences;  B: the chunks.
        for (;;) {
            const uint32_t cnt = *(volatile uint32_t *)&P.ctl->qcnt[r % 3];
            if (cnt == 0 || P.exp != 0) break;
            if (leader) {
                P.ctl->qcnt[(r + 2) % 3] = 0;
                P.ctl->ccnt[(r + 2) % 3] = 0;
                P.ctl->rcnt[(r + 2) % 3] = 0;
                P.ctl->rounds++;
                P.ctl->fix_units += cnt;
            }
            const int pin = r & 1, pout = (r + 1) & 1;
            uint32_t *qout = &P.ctl->qcnt[(r + 1) % 3];
            for (uint32_t it = gw; it < cnt; it += nw) {
                const uint32_t unit = P.fq[pin][it];
                const uint32_t word = P.fb[pin][unit];  // nobody writes fb[pin] this round
                __syncwarp();
                if (lane == 0) P.fb[pin][unit] = 0u;   // consumed
                const uint32_t v = unit / P.G, g = unit - v * P.G;
                const uint32_t q = g * 32 + lane;
                uint32_t lo = 0, hi = 0;
                if ((word >> lane) & 1u) {
                    const size_t si = (size_t)v * P.R + q;
                    const uint32_t now = StW<PK>::time(__ldcg((const typename StW<PK>::T *)P.st + si));
                    const uint32_t hb = __ldcg(P.hb + si);
                    const uint32_t prev = atomicMin(P.lat + si, now);
                    const uint32_t tend = min(min(prev, Te), hb);
                    if (now < tend) {
                        const uint32_t a = __ldg(P.vnode_off + v), b = __ldg(P.vnode_off + v + 1);
                        const uint32_t j0 = tg_lower_bound(P.node_t, a, b, now);
                        const uint32_t j1 = tg_lower_bound(P.node_t, j0, b, tend);
                        lo = __ldg(P.node_eoff + j0);
                        hi = __ldg(P.node_eoff + j1);
                    }
                }
                uint32_t ulo = (lo < hi) ? lo : 0xFFFFFFFFu, uhi = hi;
#pragma unroll
                for (int o = 16; o; o >>= 1) {
                    ulo = min(ulo, __shfl_xor_sync(0xffffffffu, ulo, o));
                    uhi = max(uhi, __shfl_xor_sync(0xffffffffu, uhi, o));
                }
                if (ulo >= uhi) continue;
                uint32_t rec = 0, k0 = 0;
                const uint32_t nch = (uhi - ulo + FIX_CHUNK - 1) / FIX_CHUNK;
                if (lane == 0) {
                    rec = atomicAdd(&P.ctl->rcnt[r % 3], 1u);
                    k0 = atomicAdd(&P.ctl->ccnt[r % 3], nch);
                }
                rec = __shfl_sync(0xffffffffu, rec, 0);
                k0 = __shfl_sync(0xffffffffu, k0, 0);
                if (rec < P.reccap && (uint64_t)k0 + nch <= P.chcap) {
                    P.recs[(size_t)rec * 32 + lane] = make_uint2(lo, hi);
                    for (uint32_t c = lane; c < nch; c += 32) {
                        const uint32_t c0 = ulo + c * FIX_CHUNK;
                        P.chq[k0 + c] = make_uint4(rec, c0, min(uhi, c0 + FIX_CHUNK), g);
                    }
                    continue;
                }
                // queue full: do it here (entries below capacity are left empty)
                if (k0 < P.chcap)
                    for (uint32_t c = lane; c < min(nch, P.chcap - k0); c += 32) P.chq[k0 + c] = make_uint4(0, 0, 0, g);
                fix_chunk<PK>(P, g, lo, hi, ulo, uhi, Te, pout, qout, ws);
            }
            grid.sync();
            if (leader) { const unsigned long long t1 = gtimer(); P.ctl->ns[1] += t1 - t0; t0 = t1; }
            const uint32_t nc = min(*(volatile uint32_t *)&P.ctl->ccnt[r % 3], P.chcap);
            for (uint32_t it = gw; it < nc; it += nw) {
                const uint4 c = P.chq[it];
                if (c.y >= c.z) continue;
                const uint2 rg = P.recs[(size_t)c.x * 32 + lane];
                fix_chunk<PK>(P, c.w, rg.x, rg.y, c.y, c.z, Te, pout, qout, ws);
            }
            grid.sync();
            if (leader) {
                const unsigned long long t1 = gtimer();
                P.ctl->ns[2] += t1 - t0;
                t0 = t1;
                P.ctl->ns[3] += nc;  // chunks
            }
            r++;
        }
        b0 = b1;
        part++;
    }
}

// VInitial (Table 1): rows INF (memset), the source word = (alpha, no pred)
template <bool PK>
__global__ void k_sweep_init(void *st, uint32_t R, const uint32_t *srcs, uint32_t S, uint32_t alpha, SweepCtl *ctl) {
    for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q < S; q += gridDim.x * blockDim.x)
        ((typename StW<PK>::T *)st)[(size_t)srcs[q] * R + q] = StW<PK>::make(alpha, TG_NONE);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        for (int i = 0; i < 3; i++) ctl->qcnt[i] = ctl->ccnt[i] = ctl->rcnt[i] = 0;
        ctl->rounds = ctl->parts = ctl->fix_units = 0;
        ctl->claim[0] = ctl->claim[1] = 0;
        ctl->ns[0] = ctl->ns[1] = ctl->ns[2] = ctl->ns[3] = 0;
    }
}

// Extract rows [q][v] from [v][R]; mode 0 EAT, 1 LD (mirror: C - time; the target = omega), 2 REACH.
template <bool PK>
__global__ void __launch_bounds__(256) k_sweep_extract(const void *__restrict__ st_, uint32_t n, uint32_t R,
                                                       uint32_t S, const uint32_t *__restrict__ srcs, int mode,
                                                       uint32_t C, uint32_t omega, uint32_t *__restrict__ out,
                                                       uint32_t *__restrict__ pred,
                                                       const uint32_t *__restrict__ perm) {
    using T = typename StW<PK>::T;
    __shared__ unsigned long long tile[32 * 65];
    const T *st = (const T *)st_;
    const T INF = (T)~0ull;
    const uint32_t nt = (n + 31) / 32;
    for (uint32_t tb = blockIdx.x; tb < nt; tb += gridDim.x) {
        const uint32_t v0 = tb * 32;
        for (uint32_t q0 = 0; q0 < S; q0 += 64) {
            const uint32_t qs = min(64u, S - q0);
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < 32 * qs; i += blockDim.x) {
                const uint32_t dv = i / qs, dq = i - dv * qs;
                const uint32_t v = v0 + dv;
                tile[dv * 65 + dq] = (v < n) ? st[(size_t)(perm ? perm[v] : v) * R + q0 + dq] : INF;
            }
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < 32 * qs; i += blockDim.x) {
                const uint32_t dq = i / 32, dv = i - dq * 32;
                const uint32_t v = v0 + dv, q = q0 + dq;
                if (v >= n) continue;
                const T pk = (T)tile[dv * 65 + dq];
                const bool reached = pk != INF;
                const uint32_t t = StW<PK>::time(pk);
                uint32_t pr = (reached && PK) ? (uint32_t)pk : TG_NONE;
                uint32_t val;
                const uint32_t src = srcs[q];
                if (mode == 0) {
                    val = reached ? t : TG_UNREACHED;
                } else if (mode == 1) {
                    val = (v == src) ? omega : (reached ? C - t : TG_UNREACHED);
                    if (v == src) pr = TG_NONE;
                } else {
                    val = reached ? 1u : 0u;
                }
                out[(size_t)q * n + v] = val;
                if (pred) pred[(size_t)q * n + v] = pr;
            }
        }
    }
}

// Work count (stats): W_q = #{valid e : EAT(u, q) <= t} -- exactly the edges the one-pass
// scan relaxes -- and W_union = #{valid e : some q}, from the
// final states.  Warp per edge, lanes over queries.
template <bool PK, int QPL>
__global__ void k_sweep_work(const int4 *__restrict__ te, uint32_t e0, uint32_t e1, uint32_t omega,
                             const void *__restrict__ st, uint32_t R, uint32_t S,
                             unsigned long long *__restrict__ wq, unsigned long long *__restrict__ wu) {
    using T = typename StW<PK>::T;
    const int lane = threadIdx.x & 31;
    const uint32_t gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    uint32_t c[QPL] = {};
    uint32_t cu = 0;
    for (uint32_t i = e0 + gw; i < e1; i += nw) {
        const int4 e = __ldg(te + i);
        if ((uint32_t)e.w > omega) continue;
        T x[QPL];
        row_load<PK, QPL>(st, (size_t)(uint32_t)e.x * R + lane * QPL, x);
        bool a = false;
#pragma unroll
        for (int k = 0; k < QPL; k++) {
            const bool u = lane * QPL + k < S && StW<PK>::time(x[k]) <= (uint32_t)e.z;
            c[k] += u;
            a |= u;
        }
        cu += __any_sync(0xffffffffu, a) ? 1u : 0u;
    }
#pragma unroll
    for (int k = 0; k < QPL; k++)
        if (lane * QPL + k < S && c[k]) atomicAdd(wq + lane * QPL + k, (unsigned long long)c[k]);
    if (lane == 0 && cu) atomicAdd(wu, (unsigned long long)cu);
}

__global__ void k_lower_bound_te(const int4 *te, uint32_t m, uint32_t key, uint32_t *out) {
    if (threadIdx.x == 0 && blockIdx.x == 0) *out = lower_bound_t(te, 0, m, key);
}

}  // namespace

// ============================================================================ host
struct SweepScratch {
    uint32_t R = 0, n = 0;
    void *st = nullptr;
    uint32_t *lat = nullptr, *hb = nullptr;
    uint32_t *fb[2] = {nullptr, nullptr}, *fq[2] = {nullptr, nullptr};
    uint2 *recs = nullptr;
    uint4 *chq = nullptr;
    uint32_t chcap = 0, reccap = 0;
    SweepCtl *ctl = nullptr;
    uint32_t *bounds = nullptr;
    unsigned long long *wcnt = nullptr;
    DevArena arena;
};

static SweepScratch *scratch_of(tg_graph *g) { return (SweepScratch *)g->sweep; }

void tg_sweep_free(tg_graph *g) {
    SweepScratch *W = scratch_of(g);
    if (!W) return;
    W->arena.free_all();
    delete W;
    g->sweep = nullptr;
}

static tg_status sweep_scratch(tg_graph *g, uint32_t R) {
    SweepScratch *W = scratch_of(g);
    if (W && W->R >= R && W->n == g->n) return TG_OK;
    TG_TRY_CUDA(cudaDeviceSynchronize());
    tg_sweep_free(g);
    W = new SweepScratch();
    g->sweep = W;
    const uint64_t n = g->n, m = g->m;
    const uint32_t G = R / 32;
    W->R = R;
    W->n = g->n;
    DevArena &A = W->arena;
    TG_TRY(A.alloc(&W->st, n * R * 8));  // sized for packed words
    TG_TRY(A.alloc((void **)&W->lat, n * R * 4));
    TG_TRY(A.alloc((void **)&W->hb, n * R * 4));
    for (int i = 0; i < 2; i++) {
        TG_TRY(A.alloc((void **)&W->fb[i], n * G * 4));
        TG_TRY(A.alloc((void **)&W->fq[i], n * G * 4));
        TG_TRY_CUDA(cudaMemset(W->fb[i], 0, n * G * 4));
    }
    W->chcap = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(m / FIX_CHUNK * 4, 1u << 16), 1u << 24);
    W->reccap = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(n * G, 1u << 12), 1u << 22);
    TG_TRY(A.alloc((void **)&W->chq, (uint64_t)W->chcap * 16));
    TG_TRY(A.alloc((void **)&W->recs, (uint64_t)W->reccap * 32 * 8));
    TG_TRY(A.alloc((void **)&W->ctl, sizeof(SweepCtl)));
    TG_TRY(A.alloc((void **)&W->bounds, 16));
    TG_TRY(A.alloc((void **)&W->wcnt, (R + 2) * 8));
    return TG_OK;
}

template <bool PK, int QPL>
static tg_status sweep_launch(tg_graph *g, const ChainGraph &cgr, SwP &P, cudaStream_t s) {
    static int per_sm = -1;
    if (per_sm < 0) {
        TG_TRY_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_sweep<PK, QPL>, SW_T, 0));
        per_sm = std::max(1, std::min(per_sm, 8));
    }
    int dev = 0, sms = 148;
    TG_TRY_CUDA(cudaGetDevice(&dev));
    TG_TRY_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    void *args[] = {&P};
    cudaEvent_t ev0 = g_tg_profile ? tg_prof_begin(s) : nullptr;
    TG_TRY_CUDA(cudaLaunchCooperativeKernel((void *)k_sweep<PK, QPL>, dim3((unsigned)(sms * per_sm)), dim3(SW_T),
                                            args, 0, s));
    g_tg_launches++;
    if (ev0) tg_prof_end("k_sweep", s, ev0);
    (void)cgr;
    return TG_OK;
}

template <bool PK, int QPL>
static tg_status sweep_batch(tg_graph *g, const ChainGraph &cgr, uint32_t Sb, uint32_t alpha, uint32_t omega,
                             bool work, int mode, uint32_t C, tg_window w, uint32_t *o, uint32_t *pr,
                             cudaStream_t s, uint64_t *wq_out, uint64_t *wu_out) {
    SweepScratch &W = *scratch_of(g);
    QueryScratch &Q = g->qs;
    const uint32_t R = 32 * QPL, G = QPL;
    const uint64_t n = g->n;
    TG_TRY_CUDA(cudaMemsetAsync(W.st, 0xFF, n * R * (PK ? 8 : 4), s));
    TG_LAUNCH(k_sweep_init<PK>, 1, 64, 0, s, W.st, R, Q.srcs_int, Sb, alpha, W.ctl);
    if (work) {
        TG_TRY_CUDA(cudaMemsetAsync(W.lat, 0xFF, n * R * 4, s));
        TG_TRY_CUDA(cudaMemsetAsync(W.hb, 0, n * R * 4, s));
        // window: edges with t in [alpha, omega) (t + duration <= omega needs t < omega)
        TG_LAUNCH(k_lower_bound_te, 1, 32, 0, s, cgr.te, (uint32_t)g->m, alpha, W.bounds);
        TG_LAUNCH(k_lower_bound_te, 1, 32, 0, s, cgr.te, (uint32_t)g->m, omega, W.bounds + 1);
        uint32_t hb[2];
        TG_TRY_CUDA(cudaMemcpyAsync(hb, W.bounds, 8, cudaMemcpyDeviceToHost, s));
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        if (hb[0] < hb[1]) {
            SwP P{};
            P.te = cgr.te; P.te_id = cgr.te_id;
            P.e_begin = hb[0]; P.e_end = hb[1];
            P.part_edges = (uint32_t)(g->opt_sweep_part > 0 ? g->opt_sweep_part : (1u << 20));
            P.vnode_off = cgr.vnode_off; P.node_t = cgr.node_t; P.node_eoff = cgr.node_eoff;
            P.occ_slot = cgr.occ_slot; P.slots = cgr.slots;
            P.st = W.st; P.lat = W.lat; P.hb = W.hb;
            P.n = g->n; P.R = R; P.G = G; P.alpha = alpha; P.omega = omega;
            P.fb[0] = W.fb[0]; P.fb[1] = W.fb[1]; P.fq[0] = W.fq[0]; P.fq[1] = W.fq[1];
            P.recs = W.recs; P.chq = W.chq; P.chcap = W.chcap; P.reccap = W.reccap;
            P.ctl = W.ctl;
            P.exp = (int)g->opt_exp;
            TG_TRY((sweep_launch<PK, QPL>(g, cgr, P, s)));
            if (wq_out) {
                TG_TRY_CUDA(cudaMemsetAsync(W.wcnt, 0, (R + 2) * 8, s));
                TG_LAUNCH((k_sweep_work<PK, QPL>), 148 * 8, 256, 0, s, cgr.te, hb[0], hb[1], omega, W.st, R, Sb,
                          W.wcnt, W.wcnt + R);
                std::vector<unsigned long long> h(R + 1);
                TG_TRY_CUDA(cudaMemcpyAsync(h.data(), W.wcnt, (R + 1) * 8, cudaMemcpyDeviceToHost, s));
                SweepCtl hc;
                TG_TRY_CUDA(cudaMemcpyAsync(&hc, W.ctl, sizeof(hc), cudaMemcpyDeviceToHost, s));
                TG_TRY_CUDA(cudaStreamSynchronize(s));
                for (uint32_t q = 0; q < Sb; q++) wq_out[q] = h[q];
                *wu_out = h[R];
                static const bool trace = getenv("TG_TRACE") != nullptr;
                if (trace)
                    fprintf(stderr, "[tg] sweep S=%u: partitions %u, fixup rounds %u, fixup units %u, chunks %llu; "
                            "dense %.3f ms, fixup A %.3f ms, fixup B %.3f ms\n", Sb, hc.parts, hc.rounds, hc.fix_units,
                            hc.ns[3], hc.ns[0] * 1e-6, hc.ns[1] * 1e-6, hc.ns[2] * 1e-6);
            }
        }
    }
    const unsigned xgrid = (unsigned)std::min<uint64_t>((n + 31) / 32, 148ull * 16);
    TG_LAUNCH(k_sweep_extract<PK>, xgrid, 256, 0, s, W.st, g->n, R, Sb, Q.srcs, mode, C, w.t_omega, o, pr,
              g->relabeled ? g->perm : (const uint32_t *)nullptr);
    return TG_OK;
}

bool tg_sweep_available(const tg_graph *g, tg_problem p) {
    const ChainGraph &c = (p == TG_LD) ? g->mir : g->fwd;
    return g->nparts == 0 && c.te != nullptr && g->m < 0xFFFFFFFFull;
}

tg_status tg_run_sweep(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                       uint32_t *pred, bool out_dev, bool pred_dev, cudaStream_t s) {
    const bool ld = (p == TG_LD);
    const ChainGraph &cgr = ld ? g->mir : g->fwd;
    uint32_t alpha = w.t_alpha, omega = w.t_omega;
    bool any_work = true;
    const uint32_t C = g->max_arr;
    if (ld) {  // reading A5: LD(G,x,[a,o]) = C - EAT(G^R, x, [max(0, C-o), C-a]); a > C -> only the target
        if (alpha > C) { any_work = false; alpha = 0; omega = 0; }
        else { uint32_t a2 = (omega >= C) ? 0u : C - omega; omega = C - alpha; alpha = a2; }
    }
    // sub-batch: up to 64 queries share one pass over the edges (rows of 32 * QPL words)
    const uint32_t S = (uint32_t)std::min<int64_t>(g->opt_sub_batch > 0 ? std::min<int64_t>(g->opt_sub_batch, 64) : 64, k);
    const int QPL = S > 32 ? 2 : 1;
    TG_TRY(tg_ensure_scratch_srcs(g, S));
    TG_TRY(sweep_scratch(g, 64));
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
    const bool pk = pred != nullptr || g->opt_packed_state;
    const bool work = any_work && g->m > 0 && alpha < omega;
    for (uint32_t b0 = 0; b0 < k; b0 += S) {
        const uint32_t Sb = std::min(S, k - b0);
        TG_TRY(tg_load_sources(g, sources + b0, Sb, s));
        uint32_t *o = out_dev ? out + (size_t)b0 * n : Q.out_stage;
        uint32_t *pr = pred ? (pred_dev ? pred + (size_t)b0 * n : Q.pred_stage) : nullptr;
        uint64_t *wq = g->opt_stats ? g->last_relax + b0 : nullptr;
        uint64_t wu = 0;
        if (g->opt_stats) for (uint32_t q = 0; q < Sb; q++) wq[q] = 0;
        if (pk) {
            if (QPL == 1) TG_TRY((sweep_batch<true, 1>(g, cgr, Sb, alpha, omega, work, mode, C, w, o, pr, s, wq, &wu)));
            else TG_TRY((sweep_batch<true, 2>(g, cgr, Sb, alpha, omega, work, mode, C, w, o, pr, s, wq, &wu)));
        } else {
            if (QPL == 1) TG_TRY((sweep_batch<false, 1>(g, cgr, Sb, alpha, omega, work, mode, C, w, o, pr, s, wq, &wu)));
            else TG_TRY((sweep_batch<false, 2>(g, cgr, Sb, alpha, omega, work, mode, C, w, o, pr, s, wq, &wu)));
        }
        if (g->opt_stats) {
            for (uint32_t q = 0; q < Sb; q++) g->last.slots_relaxed += wq[q];
            g->last.slots_union += wu;
            SweepCtl hc;
            TG_TRY_CUDA(cudaMemcpyAsync(&hc, scratch_of(g)->ctl, sizeof(hc), cudaMemcpyDeviceToHost, s));
            TG_TRY_CUDA(cudaStreamSynchronize(s));
            g->last.rounds = std::max<uint32_t>(g->last.rounds, hc.parts + hc.rounds);
        }
        g->last.sub_batches++;
        if (!out_dev) TG_TRY_CUDA(cudaMemcpyAsync(out + (size_t)b0 * n, Q.out_stage, (size_t)Sb * n * 4, cudaMemcpyDeviceToHost, s));
        if (pred && !pred_dev) TG_TRY_CUDA(cudaMemcpyAsync(pred + (size_t)b0 * n, Q.pred_stage, (size_t)Sb * n * 4, cudaMemcpyDeviceToHost, s));
    }
    TG_TRY_CUDA(cudaStreamSynchronize(s));
    g->last.kernel_launches = g_tg_launches - launches0;
    return TG_OK;
}
