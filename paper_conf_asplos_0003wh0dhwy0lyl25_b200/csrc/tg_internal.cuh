// tg_internal.cuh -- shared definitions of the CUDA path (product code).
// Nothing here is shared with oracle/ (test infrastructure).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/tg.h"

#define TG_NONE 0xFFFFFFFFu
#define TG_SINGLE 0xFFFFFFFFu  // slot.w for a one-edge chain (no long-chain index)

// ----------------------------------------------------------------------------- errors
void tg_set_error(const std::string &msg);
extern uint64_t g_tg_launches;  // kernels launched by this library (process-wide)

#define TG_TRY_CUDA(expr)                                                                      \
    do {                                                                                       \
        cudaError_t _e = (expr);                                                               \
        if (_e != cudaSuccess) {                                                               \
            tg_set_error(std::string(#expr) + ": " + cudaGetErrorString(_e) + " @" __FILE__); \
            return (_e == cudaErrorMemoryAllocation) ? TG_ERR_NOMEM : TG_ERR_CUDA;             \
        }                                                                                      \
    } while (0)

#define TG_TRY(expr)                   \
    do {                               \
        tg_status _s = (expr);         \
        if (_s != TG_OK) return _s;    \
    } while (0)

// Launch bookkeeping: every kernel launch goes through this macro so that the
// bench can report how many of OUR kernels ran inside its timed region.
// With profiling enabled (tg_profile_enable) a CUDA event pair is recorded around
// every launch on the launching stream; tg_profile_report sums them per kernel.
extern int g_tg_profile;
cudaEvent_t tg_prof_begin(cudaStream_t s);
void tg_prof_end(const char *name, cudaStream_t s, cudaEvent_t ev0);
#define TG_LAUNCH_LVL(lvl, kernel, grid, block, smem, stream, ...)                    \
    do {                                                                              \
        cudaEvent_t _ev0 = (g_tg_profile && g_tg_profile <= (lvl)) ? tg_prof_begin(stream) \
                                                                    : nullptr;          \
        kernel<<<(grid), (block), (smem), (stream)>>>(__VA_ARGS__);                   \
        g_tg_launches++;                                                              \
        if (_ev0) tg_prof_end(#kernel, stream, _ev0);                                 \
        TG_TRY_CUDA(cudaGetLastError());                                              \
    } while (0)
// every kernel (profiled at level 1); the relaxation kernels (profiled at levels 1 and 2)
#define TG_LAUNCH(kernel, grid, block, smem, stream, ...) \
    TG_LAUNCH_LVL(1, kernel, grid, block, smem, stream, __VA_ARGS__)
#define TG_LAUNCH_RELAX(kernel, grid, block, smem, stream, ...) \
    TG_LAUNCH_LVL(2, kernel, grid, block, smem, stream, __VA_ARGS__)

// ----------------------------------------------------------------------------- device memory
// Simple owning device buffer list for a graph handle.
struct DevArena {
    struct Blk { void *p; size_t bytes; };
    std::vector<Blk> blks;
    size_t total = 0;
    uint32_t slack_pct = 0;  // fresh blocks get this much extra room (dynamic graphs: the next,
                             // slightly larger, re-transformation reuses them from the cache)
    cudaStream_t pool_stream = nullptr;  // set: stream-ordered pool blocks (cudaMallocAsync on this
    bool use_pool = false;               // stream, no retry; free_all = cudaFreeAsync) -- query lanes
    tg_status alloc(void **p, size_t bytes);
    void free_all();
};

// One direction of the transformed graph (forward, or the LD mirror).
// Layout in HBM:
//   departure nodes (v, tau) in (v, tau) order:   vnode_off[n+1], node_t[N], node_u[N], node_eoff[N+1]
//   sorted edges (by (u, t, id)), "occurrences": occ_slot[m] -> slot index, occ_node[m] -> node,
//       occ_rec uint2[m] = {v, arrival | walked-chain flag} (the activation's coalesced edge read)
//   slots in chain-major order (chains ordered by head (u, t, first id)):
//       slots int4[m] = {v, arr = t + duration, edge id, long-chain index of a walked chain | TG_SINGLE}
//       slot_w[m], slot_tn[m] (tail departure node or TG_NONE)   -- SP/FP only
//   long chains (>= 2 edges): lc uint2[L] = {first slot, length}
//                             sc int4[L]  = {tail v, tail arrival, tail edge id, head node}
//                             sc_sumw uint64[L], sc_elapsed uint32[L]  (Alg. 2 shortcut weights)
//   chain_first[nchains+1]: first slot of every chain (export / parity)
struct ChainGraph {
    uint32_t n = 0;
    uint64_t m = 0;
    uint64_t nnodes = 0, nchains = 0, nlong = 0;
    uint32_t maxlen = 0;
    uint32_t *vnode_off = nullptr, *node_t = nullptr, *node_u = nullptr, *node_eoff = nullptr;
    uint32_t *occ_slot = nullptr;
    uint32_t *occ_node = nullptr;  // sorted-edge position -> departure node (SP/FP entry state)
    uint2 *occ_rec = nullptr;      // sorted-edge position -> {head v, arrival | 1 << 31 if on a walked chain}
    uint4 *occ_rch = nullptr;      // bit-lane reach (built on first use): {v, arrival | walked flag, tail node, tail tau}
    uint4 *occ_spr = nullptr;      // SP/FP/LDS (built on first use): {v, arrival | walked flag, tail node, w}
    int4 *slots = nullptr;
    uint32_t *slot_w = nullptr, *slot_tn = nullptr;
    uint2 *lc = nullptr;
    int4 *sc = nullptr;
    unsigned long long *sc_sumw = nullptr;
    uint32_t *sc_elapsed = nullptr;
    uint32_t *chain_first = nullptr;
    uint32_t *order = nullptr;  // option "dynamic": the edge ids in (u, t, id) order, kept for insertions
    DevArena arena;             // every array of this direction
};

// Device-side round control of one GAC loop (no host round trip per round): a ring
// of per-round counters, round r at cnt[r % TG_RING]; the first kernel of a round
// clears a later round's slot.  The ring is deeper than the host's round group, so
// after a group the host sees every round of it (the first round whose frontier was
// empty is the round count).
#define TG_RING 16
struct RoundCtl {
    uint32_t round;
    uint32_t stamp;
    uint32_t done_blocks;
    uint32_t last;  // graph loop: the round that ended it (its frontier was empty, or the limit)
    uint32_t cnt[TG_RING][4];
};

struct QueryScratch {
    uint32_t S = 0;          // sources per sub-batch this scratch was sized for
    uint32_t n = 0;
    uint64_t nlong = 0;
    uint64_t nnodes = 0;
    bool nodes_state = false;  // SP/FP node-state arrays present
    void *st = nullptr;  // [n][S] packed u64 (time << 32 | pred), or u32 time when no pred is requested
    uint32_t st_copies = 1;  // option "exchange" with logical partitions: one private state copy each
    uint32_t st_w = 8;       // bytes per state entry allocated (8: packed states fit)
    uint32_t *act = nullptr;           // [S][n] last activated time
    unsigned long long *ub = nullptr;  // [n] arrival-bound codes per 8 queries (query_eat.cu, TG_UB)
    uint32_t stamp = 0;                // SP/FP frontier dedupe stamps handed out (host counter; marks start at 0)
    uint32_t *mark = nullptr;          // [S][n] (EAT) or [S][nnodes] (SP/FP) frontier dedupe stamp
    uint32_t *bits = nullptr;          // [S][ceil(m/32)] "slot relaxed" bits (interior slots of long chains)
    uint64_t bit_words = 0;            // words per query
    uint32_t *dnode = nullptr;         // [S][nnodes] SP/FP node state
    uint32_t *vout = nullptr;          // [S][n] SP/FP per-vertex output
    unsigned long long *fr[2] = {nullptr, nullptr};  // SP/FP frontier items (q << 32 | node)
    uint32_t *fb[2] = {nullptr, nullptr};            // EAT-family frontier masks [n][G]
    uint32_t vwords = 0;                             // G = query groups of 32 (allocation)
    uint2 *recs = nullptr;                           // big-unit records (32 ranges each)
    uint64_t reccap = 0;
    uint64_t fcap = 0;
    uint4 *bigq = nullptr;   // big activation chunks {q, e_begin, e_end, -}
    uint64_t bigcap = 0;
    uint4 *chq = nullptr;    // long chain walks {q, s_begin, s_end, -}
    uint64_t chcap = 0;
    uint32_t *ctr = nullptr;   // counters [2][4] (SP/FP host-driven loop)
    struct RoundCtl *ctl = nullptr;  // device-side round control (EAT family), [TG_MAXP]
    uint32_t *lat = nullptr;         // partitioned mode: last activated arrival [v][q]
    uint32_t *defer = nullptr;       // TG_DEFER experiment: units deferred once
    uint32_t *pcount = nullptr;      // partitioned mode: frontier bits of the next round
    uint32_t *h_ctr = nullptr; // pinned host mirror
    uint32_t *srcs = nullptr;  // [S] sources of the sub-batch (caller's vertex ids)
    uint32_t *srcs_int = nullptr;  // [S] the same in the engine's internal vertex order
    uint32_t *rows = nullptr;      // [S] the caller's output row of each query of the sub-batch
    unsigned long long *relax_cnt = nullptr;  // [S] + distinct-slot count
    uint32_t *touched = nullptr;              // stats: slots relaxed by any query of the sub-batch
    uint32_t *out_stage[2] = {nullptr, nullptr}, *pred_stage[2] = {nullptr, nullptr};  // [S][n] x 2 for host outputs
    DevArena arena;
};

// Out-of-memory graphs (stream.cu; §4.5): the edges are cut
// into blocks of consecutive departure times (a topological order of the transformed
// DAG); each block's chain structure lives in pinned host memory and is streamed to one
// of two device slots while the previous block is being computed.
struct HostBlock {
    uint64_t m = 0, nn = 0, L = 0;
    uint32_t t_lo = 0, t_hi = 0;  // departure times [t_lo, t_hi)
    uint32_t *vnode_off = nullptr, *node_t = nullptr, *node_eoff = nullptr, *occ_slot = nullptr;
    uint2 *occ_rec = nullptr;
    int4 *slots = nullptr;
    uint2 *lc = nullptr;
    int4 *sc = nullptr;
    void *pinned = nullptr;
    uint64_t bytes = 0;
};
struct StreamGraph {
    uint64_t block_edges = 0;
    std::vector<HostBlock> blocks;
    // the input, organised by block (pinned): u, v, t, dur, w, id per block
    std::vector<uint32_t *> bedges;
    std::vector<void *> bedges_pinned;
    bool weighted = false;
    uint64_t max_m = 0, max_nn = 0, max_L = 0;
    ChainGraph slot[2];
    DevArena slot_arena;
    cudaStream_t cs = nullptr;
    cudaEvent_t ready[2] = {nullptr, nullptr}, freed[2] = {nullptr, nullptr};
    uint64_t h2d_bytes = 0;  // streamed by the last query
};

// Bit-lane reachability scratch (query_reach.cu): one u64 word per departure node and
// per vertex for a sub-batch of up to 64 sources.
struct ReachScratch {
    uint64_t nn = 0, n = 0;
    unsigned long long *R = nullptr, *VR = nullptr;
    uint32_t *D[2] = {nullptr, nullptr}, *dmin[2] = {nullptr, nullptr}, *dmax[2] = {nullptr, nullptr};
    uint32_t *vf[2] = {nullptr, nullptr};
    uint4 *bigq = nullptr;
    uint64_t bigcap = 0;
    struct RoundCtl *ctl = nullptr;
    unsigned long long *cnt = nullptr;
    uint32_t *srcs = nullptr, *srcs_int = nullptr;
    uint32_t *stage[1] = {nullptr};
    uint32_t *h_ctr = nullptr;
    DevArena arena;
};

#define TG_LANES 4  // query lanes at most (option "lanes")
#define TG_MAXP 16  // logical vertex-range partitions per process (tests / one rank's share)

struct tg_comm;  // comm.cu: NCCL communicator (loaded with dlopen)

struct tg_graph {
    int device = 0;
    uint32_t n = 0;
    uint64_t m = 0;
    uint32_t *d_u = nullptr, *d_v = nullptr, *d_t = nullptr, *d_dur = nullptr, *d_w = nullptr;
    uint32_t max_t = 0, max_arr = 0, min_t = 0, max_w = 0;
    bool sp_ok = true;
    bool built = false;
    double build_ms = 0;
    ChainGraph fwd, mir;
    // internal vertex order (descending in-degree) for state locality; queries map
    // sources in and results out.  perm[original] = internal, iperm[internal] = original.
    int opt_relabel = 0;  // measured: no gain on R-MAT C2 (12.9 vs 12.5 ms EAT), off by default
    bool relabeled = false;
    uint32_t *perm = nullptr, *iperm = nullptr;
    uint32_t *d_ru = nullptr, *d_rv = nullptr;  // relabeled endpoints
    // vertex-range partitions (multi-GPU mode 1, or logical partitions on one GPU):
    // partition p owns vertices [part_vb[p], part_vb[p+1]); pf/pm hold its chains
    int nparts = 0;                 // 0 = not partitioned
    int opt_partitions = 1;         // logical partitions requested via tg_set_option
    uint32_t part_vb[TG_MAXP + 1] = {0};
    ChainGraph pf[TG_MAXP], pm[TG_MAXP];
    tg_comm *comm = nullptr;
    int comm_mode = 0;              // 0 replicated (source sharding), 1 vertex range
    DevArena arena;        // input copies + chain structures
    QueryScratch qs;
    // query lanes 1 .. TG_LANES-1 (EAT family, device outputs): scratch, stream, join event
    QueryScratch qsl[TG_LANES - 1];
    cudaStream_t lane_stream[TG_LANES - 1] = {};
    cudaEvent_t lane_fork = nullptr, lane_join[TG_LANES - 1] = {};
    ReachScratch rs;
    StreamGraph *stream = nullptr;  // out-of-memory graph (tg_graph_create_streamed)
    uint32_t qs_epoch = 0;  // frontier-dedupe stamp (monotone across rounds and queries)
    // options
    int64_t opt_sub_batch = 0;
    int64_t opt_stats = 0;
    int64_t opt_shortcuts = 1;
    int64_t opt_round_group = 8;  // GAC rounds launched per host convergence check
    int opt_mirror = 1;
    int64_t opt_exchange = 0;  // 1 = vertex-range partitions exchange states every round (cross-rank algorithm)
    int64_t opt_ub = 1;  // arrival bounds per (vertex, 8 queries) prune pairs: 0 off, 1 auto, 2 on (query_eat.cu)
    int64_t opt_graph_loop = 1;  // 0 host-driven rounds, 1 graph loop for graphs >= TG_GRAPH_LOOP_MIN_M edges, 2 always
    int64_t opt_lanes = 4;  // sub-batches in flight (EAT family, device outputs, graph loop): 1 .. TG_LANES  // 1 = GAC rounds run in a device-driven CUDA-graph WHILE loop (query_eat.cu)
    int64_t opt_packed_state = 0;  // 1 = packed (arrival|pred) u64 EAT-family state even without pred (tests)
    int64_t opt_order_sources = 1;  // schedule a call's sources by first departure time (query_eat.cu)
    int64_t opt_reach_bits = 0;  // 1 = TG_REACH without pred on the bit-lane engine (query_reach.cu)
    int64_t opt_dynamic = 0;   // 1 = keep each direction's sorted edge order for tg_graph_insert_edges
    int64_t opt_walk_min = 6;  // chains with fewer edges are not walked (RemoveChain threshold, build time)
    bool mirror_built = false;
    // host-memory outputs: copy stream and per-staging-buffer events (host_out.cu)
    cudaStream_t cstream = nullptr;
    cudaEvent_t ev_x[2] = {nullptr, nullptr}, ev_c[2] = {nullptr, nullptr};
    // last query statistics
    tg_query_stats last{};
    uint64_t *last_relax = nullptr;  // host, per query
    uint32_t last_relax_len = 0;
};

// Stream-ordered temporary allocation; on failure the block cache is returned to
// the driver, the pool trimmed, and the allocation retried once.
cudaError_t tg_malloc_async(void **p, size_t bytes, cudaStream_t s);
// 4 KB pinned host blocks for round-control readback, cached process-wide (a new
// graph per step would otherwise pay cudaMallocHost / cudaFreeHost every step)
cudaError_t tg_pinned_get(void **p);
void tg_pinned_put(void *p);

// ----------------------------------------------------------------------------- primitives
// Exclusive prefix sum of in[0..count) into out (may alias), total -> *d_total (device, may be null).
tg_status tg_exclusive_scan_u32(const uint32_t *in, uint32_t *out, uint64_t count, uint32_t *d_total,
                                cudaStream_t s, DevArena *tmp_owner);
// Stable LSD radix sort of (key, val) pairs on the low `key_bits` bits.
tg_status tg_radix_sort_pairs(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                              unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s);
// Stable LSD radix sort in place on key bits [begin_bit, begin_bit + key_bits).
tg_status tg_radix_sort_pairs_bits(unsigned long long *keys, uint32_t *vals, uint64_t m, int begin_bit, int key_bits,
                                   cudaStream_t s);
// ... and after the first snap_bits (multiple of 8) bits, a copy of the payload order to snap_vals.
tg_status tg_radix_sort_pairs_snap(unsigned long long *keys, uint32_t *vals, uint64_t m, int key_bits,
                                   unsigned long long **sorted_keys, uint32_t **sorted_vals, cudaStream_t s,
                                   int snap_bits, uint32_t *snap_vals);

// presorted: NULL, or the m edge ids already in (u, t, id) order (an insertion's merge)
tg_status tg_build_direction(tg_graph *g, ChainGraph *cg, uint64_t m, const uint32_t *u, const uint32_t *v,
                             const uint32_t *t, const uint32_t *dur, const uint32_t *w, const uint32_t *id_map,
                             uint32_t tmax, cudaStream_t s, const uint32_t *presorted = nullptr);
uint64_t tg_graph_bytes(const tg_graph *g);
tg_status tg_relabel(tg_graph *g, cudaStream_t s);
// sources of a sub-batch: copy (host) and map to the internal vertex order
tg_status tg_load_sources(tg_graph *g, const uint32_t *sources, uint32_t k, cudaStream_t s);
tg_status tg_load_sources_to(tg_graph *g, const uint32_t *sources, uint32_t k, uint32_t *d_srcs, uint32_t *d_int,
                             cudaStream_t s);
tg_status tg_validate_launch(const uint32_t *u, const uint32_t *v, const uint32_t *t, const uint32_t *dur,
                             const uint32_t *w, uint64_t m, uint32_t n, uint32_t *res, cudaStream_t s);
tg_status tg_validate_finish(tg_graph *g, const uint32_t *h);  // h: the 5 accumulated words
tg_status tg_build_streamed(tg_graph *g);
void tg_stream_free(tg_graph *g);
bool tg_graph_loop_allowed();           // query_eat.cu: no kernel profiler attached, TG_GRAPH_LOOP != 0
#ifndef TG_GRAPH_LOOP_MIN_M
#define TG_GRAPH_LOOP_MIN_M (1ull << 23)  // edges: smaller graphs keep host-driven round loops
#endif
struct tg_graph;
bool tg_graph_loop_worth(const tg_graph *g);  // query_eat.cu
// Process-wide cache of instantiated round-loop graphs (query_eat.cu), keyed by the bytes of
// their launch parameters and the device: a new handle whose buffers come back from the
// block cache at the same addresses reuses the instantiation.
cudaGraphExec_t tg_rg_find(const unsigned char *key, size_t len);
// Takes ownership; false (the caller destroys them after use) when the cache is full.
bool tg_rg_add(const unsigned char *key, size_t len, cudaGraph_t graph, cudaGraphExec_t exec);
tg_status tg_run_eat_streamed(tg_graph *g, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                              uint32_t *pred, bool out_dev, bool pred_dev, int mode, cudaStream_t s);
tg_status tg_build_partition(tg_graph *g, ChainGraph *fwd, ChainGraph *mir, uint32_t vb, uint32_t ve, cudaStream_t s,
                             int dirs);  // dirs: bit 0 forward, bit 1 mirror

// Host-memory outputs (host_out.cu).  Sub-batch b is extracted into staging buffer
// b & 1 on the query stream and copied to the host on a copy stream, so the copy of
// sub-batch b overlaps the rounds of sub-batch b + 1.  tg_sink_target waits (on the
// query stream) until buffer b & 1's previous copy has finished; tg_sink_flush issues
// the copy; tg_sink_end waits for the last copies before tg_query returns.
tg_status tg_sink_begin(tg_graph *g, bool out_host, bool pred_host);
tg_status tg_sink_target(tg_graph *g, uint32_t b, bool out_host, bool pred_host, uint32_t **o, uint32_t **pr,
                         cudaStream_t s);
tg_status tg_sink_flush(tg_graph *g, uint32_t b, uint32_t *host_out, uint32_t *host_pred, size_t bytes, cudaStream_t s);
tg_status tg_sink_flush_rows(tg_graph *g, uint32_t b, uint32_t *host_out, uint32_t *host_pred, const uint32_t *rows,
                             uint32_t nrows, uint64_t n, cudaStream_t s);
tg_status tg_sink_end(tg_graph *g);
tg_status tg_schedule_sources(tg_graph *g, const ChainGraph &cgr, const uint32_t *sources, uint32_t k, uint32_t alpha,
                              bool on, std::vector<uint32_t> &order, cudaStream_t s);
void tg_sink_destroy(tg_graph *g);

// ----------------------------------------------------------------------------- device helpers
__device__ __forceinline__ uint32_t tg_lower_bound(const uint32_t *__restrict__ a, uint32_t lo, uint32_t hi,
                                                   uint32_t key) {
    while (lo < hi) {
        uint32_t mid = lo + ((hi - lo) >> 1);
        if (__ldg(a + mid) < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ int4 tg_ld_slot(const int4 *p) {
    int4 r;
    asm volatile("ld.global.nc.v4.s32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// Lower bound of `key` (first index with a[i] >= key) in the sorted a[lo, hi), for
// every lane of a warp searching the SAME range with its own key (all lanes call).
// Up to 32 elements: one coalesced load, then a branchless search over registers by
// shuffles.  Longer ranges: 32 evenly spaced samples locate a bucket of < stride
// elements, searched per lane (its lines are shared by the warp, so mostly L1 hits).
__device__ __forceinline__ uint32_t tg_warp_lower_bound(const uint32_t *__restrict__ a, uint32_t lo, uint32_t hi,
                                                        uint32_t key) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t n = hi - lo;
    const uint32_t stride = n <= 32 ? 1u : (n + 31) / 32;
    const uint32_t idx = lane * stride;
    const uint32_t x = idx < n ? __ldg(a + lo + idx) : 0xFFFFFFFFu;
    uint32_t c = 0;  // samples < key (the samples are sorted; padding is above every key)
#pragma unroll
    for (uint32_t st = 16; st; st >>= 1) {
        const uint32_t y = __shfl_sync(0xffffffffu, x, c + st - 1);
        if (y < key) c += st;
    }
    if (__shfl_sync(0xffffffffu, x, c & 31) < key && c == 31) c = 32;
    if (stride == 1) return lo + min(c, n);
    const uint32_t blo = c == 0 ? lo : lo + (c - 1) * stride + 1;
    const uint32_t bhi = min(hi, lo + c * stride);
    return tg_lower_bound(a, blo, bhi, key);
}

// Bits [a, b) of the 32-edge block starting at pb covered by the edge range [lo, hi).
__device__ __forceinline__ uint32_t tg_block_bits(uint32_t lo, uint32_t hi, uint32_t pb) {
    const uint32_t a = lo <= pb ? 0u : min(lo - pb, 32u);
    const uint32_t b = hi <= pb ? 0u : min(hi - pb, 32u);
    return (uint32_t)(((1ull << b) - 1ull) & ~((1ull << a) - 1ull));
}

// 32 x 32 bit-matrix transpose across a warp: on entry lane L holds row L (bit k =
// element (L, k)); on exit lane L holds column L (bit q = element (q, L)).  Five
// butterfly stages swap the off-diagonal j x j blocks (j = 16, 8, 4, 2, 1).
__device__ __forceinline__ uint32_t tg_warp_transpose32(uint32_t x) {
    const uint32_t lane = threadIdx.x & 31;
#pragma unroll
    for (int j = 16, i = 0; j; j >>= 1, i++) {
        constexpr uint32_t M[5] = {0x0000FFFFu, 0x00FF00FFu, 0x0F0F0F0Fu, 0x33333333u, 0x55555555u};
        const uint32_t m = M[i];
        const uint32_t y = __shfl_xor_sync(0xffffffffu, x, j);
        x = (lane & j) ? ((x & ~m) | ((y & ~m) >> j)) : ((x & m) | ((y & m) << j));
    }
    return x;
}

static inline uint32_t tg_grid_persistent(int blocks_per_sm = 8) {
    return 148u * (uint32_t)blocks_per_sm;
}
