// stream.cu -- graphs larger than the device memory.
//
// Paper §4.5: partitions of the transformed graph are streamed from CPU
// memory to the GPU in topological order, with the transfer of the next partitions
// overlapped with the computation of the current one (multiple streams).  B200 form:
//   * the topological order of the transformed DAG is departure time (every edge of
//     the DAG goes strictly forward in time, lambda >= 1), so a partition is a block
//     of edges with departure times in [t_lo, t_hi) -- cut from a 2^16-bin time
//     histogram so that each block holds at most `block_edges` edges (a single bin
//     larger than that becomes one block of its own);
//   * tg_graph_create_streamed validates the host edge arrays chunk by chunk on the
//     device and scatters them into per-block pinned host arrays (chunk-wise stable
//     radix sort by block id); nothing of size m stays on the device;
//   * tg_build_chains transforms each block on the device (Alg. 1 + Alg. 2 +
//     occurrence index, tg_build_direction with the original edge ids) and keeps the
//     arrays the EAT engine reads in pinned host memory;
//   * tg_query (EAT, REACH) runs the GAC rounds block after block in time order
//     (query_eat.cu tg_run_eat_streamed): an edge of block b can only be enabled by
//     arrivals of edges departing earlier (blocks <= b), and nothing of a later block
//     can improve it, so block b's fixpoint from the arrivals of blocks < b is final.
//     Block b+1 is copied into the other device slot on a copy stream meanwhile.
#include <algorithm>
#include <cstring>

#include "tg_internal.cuh"

namespace {

constexpr int BT = 256;
constexpr uint64_t CHUNK = 1ull << 25;  // edges per host->device chunk

inline unsigned nblocks(uint64_t n) {
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + BT - 1) / BT, 148ull * 32));
}

__global__ void k_time_hist(const uint32_t *__restrict__ t, uint64_t m, int sh, uint32_t *__restrict__ hist) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x)
        atomicAdd(hist + (t[i] >> sh), 1u);
}

// block of every edge of the chunk (cuts: B + 1 ascending time bounds) as a sort key
__global__ void k_block_keys(const uint32_t *__restrict__ t, uint64_t m, const uint32_t *__restrict__ cuts, uint32_t B,
                             unsigned long long *__restrict__ key, uint32_t *__restrict__ idx) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t x = t[i];
        uint32_t lo = 0, hi = B;  // last b with cuts[b] <= x
        while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (cuts[mid] <= x) lo = mid; else hi = mid;
        }
        key[i] = lo;
        idx[i] = (uint32_t)i;
    }
}

// edges per block of the chunk (warp-aggregated: lanes with the same block add once)
__global__ void k_block_count(const unsigned long long *__restrict__ key, uint64_t m, uint32_t *__restrict__ cnt) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i0 = (uint64_t)blockIdx.x * blockDim.x; i0 < m; i0 += stride) {
        const uint64_t i = i0 + threadIdx.x;
        const bool on = i < m;
        const uint32_t k = on ? (uint32_t)key[i] : 0xFFFFFFFFu;
        const uint32_t peers = __match_any_sync(0xffffffffu, k);
        if (on && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(cnt + k, (uint32_t)__popc(peers));
    }
}

// gather the chunk's five arrays (+ global edge id) in block order into out[6][m]
__global__ void k_block_gather(const uint32_t *__restrict__ idx, uint64_t m, uint64_t base,
                               const uint32_t *__restrict__ u, const uint32_t *__restrict__ v,
                               const uint32_t *__restrict__ t, const uint32_t *__restrict__ d,
                               const uint32_t *__restrict__ w, uint32_t *__restrict__ out) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t j = idx[i];
        out[i] = u[j];
        out[m + i] = v[j];
        out[2 * m + i] = t[j];
        out[3 * m + i] = d[j];
        out[4 * m + i] = w ? w[j] : d[j];
        out[5 * m + i] = (uint32_t)(base + j);
    }
}

int bits_of(uint64_t x) {
    int b = 0;
    while (b < 64 && (x >> b) != 0) b++;
    return std::max(b, 1);
}

}  // namespace

// pinned host memory (NOMEM on failure)
static tg_status host_alloc(void **p, size_t bytes) {
    if (cudaHostAlloc(p, std::max<size_t>(bytes, 16), cudaHostAllocDefault) != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        tg_set_error("cudaHostAlloc(" + std::to_string(bytes) + ") failed");
        return TG_ERR_NOMEM;
    }
    return TG_OK;
}

void tg_stream_free(tg_graph *g) {
    StreamGraph *S = g->stream;
    if (!S) return;
    if (S->cs) cudaStreamSynchronize(S->cs);
    for (auto &b : S->blocks) cudaFreeHost(b.pinned);
    for (void *p : S->bedges_pinned) cudaFreeHost(p);
    S->slot_arena.free_all();
    for (int i = 0; i < 2; i++) {
        if (S->ready[i]) cudaEventDestroy(S->ready[i]);
        if (S->freed[i]) cudaEventDestroy(S->freed[i]);
    }
    if (S->cs) cudaStreamDestroy(S->cs);
    delete S;
    g->stream = nullptr;
}

extern "C" tg_status tg_graph_create_streamed(uint32_t n_vertices, uint64_t n_edges, const uint32_t *u,
                                              const uint32_t *v, const uint32_t *t_start, const uint32_t *duration,
                                              const uint32_t *weight, int device, uint64_t block_edges,
                                              tg_graph **out_graph) {
    if (!out_graph) { tg_set_error("out_graph is NULL"); return TG_ERR_INVALID; }
    *out_graph = nullptr;
    if (n_vertices == 0) { tg_set_error("n_vertices must be >= 1"); return TG_ERR_INVALID; }
    if (n_edges >= 0xFFFFFFFFull) { tg_set_error("n_edges must be < 2^32 - 1"); return TG_ERR_RANGE; }
    if (n_edges > 0 && (!u || !v || !t_start || !duration)) { tg_set_error("edge array is NULL"); return TG_ERR_INVALID; }
    if (block_edges == 0) { tg_set_error("block_edges must be >= 1"); return TG_ERR_INVALID; }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
        cudaGetLastError();
        tg_set_error("bad device ordinal / no CUDA device");
        return TG_ERR_INVALID;
    }
    int prev = -1;
    cudaGetDevice(&prev);
    cudaSetDevice(device);
    tg_graph *g = new tg_graph();
    g->device = device;
    g->n = n_vertices;
    g->m = n_edges;
    g->stream = new StreamGraph();
    StreamGraph &SG = *g->stream;
    SG.block_edges = block_edges;
    SG.weighted = weight != nullptr;
    cudaStream_t s = 0;
    auto fail = [&](tg_status st) {
        tg_stream_free(g);
        g->arena.free_all();
        delete g;
        if (prev >= 0) cudaSetDevice(prev);
        return st;
    };
    const uint64_t m = n_edges, ch = std::min<uint64_t>(CHUNK, std::max<uint64_t>(m, 1));
    // device staging for one chunk: 5 input arrays + sort scratch + gathered 6 arrays
    uint32_t *dch = nullptr, *res = nullptr, *hist = nullptr, *cuts = nullptr, *idx = nullptr, *gat = nullptr;
    unsigned long long *key = nullptr;
    auto free_dev = [&]() {
        for (void *p : {(void *)dch, (void *)res, (void *)hist, (void *)cuts, (void *)idx, (void *)gat, (void *)key})
            if (p) cudaFreeAsync(p, s);
        cudaStreamSynchronize(s);
    };
    if (tg_malloc_async((void **)&dch, ch * 5 * 4, s) != cudaSuccess || tg_malloc_async((void **)&res, 32, s) != cudaSuccess ||
        tg_malloc_async((void **)&hist, 65537 * 4, s) != cudaSuccess) {
        cudaGetLastError();
        free_dev();
        tg_set_error("device staging allocation failed");
        return fail(TG_ERR_NOMEM);
    }
    const uint32_t *src[5] = {u, v, t_start, duration, weight};
    auto upload = [&](uint64_t b0, uint64_t c) -> tg_status {
        for (int i = 0; i < 5; i++)
            if (src[i]) TG_TRY_CUDA(cudaMemcpyAsync(dch + i * ch, src[i] + b0, c * 4, cudaMemcpyDefault, s));
        return TG_OK;
    };
    // pass 1: validation (max t / arrival / weight, the SP bound)
    {
        const uint32_t init[5] = {0, 0, 0, 0, 0xFFFFFFFFu};
        if (cudaMemcpyAsync(res, init, 20, cudaMemcpyHostToDevice, s) != cudaSuccess) { free_dev(); return fail(TG_ERR_CUDA); }
        for (uint64_t b0 = 0; b0 < m; b0 += ch) {
            const uint64_t c = std::min(ch, m - b0);
            tg_status st = upload(b0, c);
            if (st == TG_OK)
                st = tg_validate_launch(dch, dch + ch, dch + 2 * ch, dch + 3 * ch, weight ? dch + 4 * ch : nullptr, c,
                                        n_vertices, res, s);
            if (st != TG_OK) { free_dev(); return fail(st); }
        }
        uint32_t h[5];
        if (cudaMemcpyAsync(h, res, 20, cudaMemcpyDeviceToHost, s) != cudaSuccess || cudaStreamSynchronize(s) != cudaSuccess) {
            free_dev();
            return fail(TG_ERR_CUDA);
        }
        tg_status st = tg_validate_finish(g, h);
        if (st != TG_OK) { free_dev(); return fail(st); }
    }
    // pass 2: time histogram -> blocks of consecutive departure times
    const int sh = std::max(0, bits_of(g->max_t) - 16);
    std::vector<uint32_t> hh(65536, 0);
    if (m) {
        cudaMemsetAsync(hist, 0, 65536 * 4, s);
        for (uint64_t b0 = 0; b0 < m; b0 += ch) {
            const uint64_t c = std::min(ch, m - b0);
            if (cudaMemcpyAsync(dch, t_start + b0, c * 4, cudaMemcpyDefault, s) != cudaSuccess) { free_dev(); return fail(TG_ERR_CUDA); }
            k_time_hist<<<nblocks(c), BT, 0, s>>>(dch, c, sh, hist);
            g_tg_launches++;
        }
        if (cudaMemcpyAsync(hh.data(), hist, 65536 * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess) {
            free_dev();
            return fail(TG_ERR_CUDA);
        }
    }
    std::vector<uint32_t> cut;  // block b = times [cut[b], cut[b+1])
    std::vector<uint64_t> bm;
    {
        uint64_t acc = 0;
        cut.push_back(0);
        for (uint32_t bin = 0; bin < 65536; bin++) {
            if (acc > 0 && acc + hh[bin] > block_edges) {
                bm.push_back(acc);
                cut.push_back(bin << sh);
                acc = 0;
            }
            acc += hh[bin];
        }
        bm.push_back(acc);
        cut.push_back(0xFFFFFFFFu);
    }
    const uint32_t B = (uint32_t)bm.size();
    SG.blocks.resize(B);
    for (uint32_t b = 0; b < B; b++) {
        SG.blocks[b].t_lo = cut[b];
        SG.blocks[b].t_hi = cut[b + 1];
        SG.blocks[b].m = bm[b];
        void *p = nullptr;
        tg_status st = host_alloc(&p, bm[b] * 6 * 4);
        if (st != TG_OK) { free_dev(); return fail(st); }
        SG.bedges_pinned.push_back(p);
        SG.bedges.push_back((uint32_t *)p);
    }
    // pass 3: scatter every chunk into the blocks' pinned arrays (stable within a chunk)
    if (m) {
        if (tg_malloc_async((void **)&cuts, (B + 1) * 4, s) != cudaSuccess ||
            tg_malloc_async((void **)&idx, ch * 4, s) != cudaSuccess ||
            tg_malloc_async((void **)&key, ch * 8, s) != cudaSuccess ||
            tg_malloc_async((void **)&gat, ch * 6 * 4, s) != cudaSuccess) {
            cudaGetLastError();
            free_dev();
            tg_set_error("device staging allocation failed");
            return fail(TG_ERR_NOMEM);
        }
        cudaMemcpyAsync(cuts, cut.data(), (B + 1) * 4, cudaMemcpyHostToDevice, s);
        std::vector<uint64_t> fill(B, 0);
        std::vector<uint32_t> ccount(B);
        for (uint64_t b0 = 0; b0 < m; b0 += ch) {
            const uint64_t c = std::min(ch, m - b0);
            tg_status st = upload(b0, c);
            if (st != TG_OK) { free_dev(); return fail(st); }
            k_block_keys<<<nblocks(c), BT, 0, s>>>(dch + 2 * ch, c, cuts, B, key, idx);
            g_tg_launches++;
            unsigned long long *sk;
            uint32_t *sv;
            if ((st = tg_radix_sort_pairs(key, idx, c, bits_of(B), &sk, &sv, s)) != TG_OK) { free_dev(); return fail(st); }
            k_block_gather<<<nblocks(c), BT, 0, s>>>(idx, c, b0, dch, dch + ch, dch + 2 * ch, dch + 3 * ch,
                                                     weight ? dch + 4 * ch : nullptr, gat);
            g_tg_launches++;
            // per-block counts of this chunk (the segments of the sorted chunk)
            cudaMemsetAsync(hist, 0, B * 4, s);
            k_block_count<<<nblocks(c), BT, 0, s>>>(key, c, hist);
            g_tg_launches++;
            if (cudaMemcpyAsync(ccount.data(), hist, B * 4, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
                cudaStreamSynchronize(s) != cudaSuccess) {
                free_dev();
                return fail(TG_ERR_CUDA);
            }
            uint64_t off = 0;
            for (uint32_t b = 0; b < B; b++) {
                const uint64_t k = ccount[b];
                if (k) {
                    const uint64_t M = bm[b];
                    for (int a = 0; a < 6; a++)
                        if (cudaMemcpyAsync(SG.bedges[b] + a * M + fill[b], gat + a * c + off, k * 4, cudaMemcpyDeviceToHost,
                                            s) != cudaSuccess) {
                            free_dev();
                            return fail(TG_ERR_CUDA);
                        }
                }
                fill[b] += k;
                off += k;
            }
            if (cudaStreamSynchronize(s) != cudaSuccess) { free_dev(); return fail(TG_ERR_CUDA); }
        }
    }
    free_dev();
    *out_graph = g;
    if (prev >= 0) cudaSetDevice(prev);
    return TG_OK;
}

// Transform every block on the device and keep its engine arrays in pinned host memory.
tg_status tg_build_streamed(tg_graph *g) {
    StreamGraph &SG = *g->stream;
    cudaStream_t s = 0;
    const uint64_t n = g->n;
    for (size_t b = 0; b < SG.blocks.size(); b++) {
        HostBlock &H = SG.blocks[b];
        const uint64_t M = H.m;
        uint32_t *d = nullptr;
        TG_TRY_CUDA(tg_malloc_async((void **)&d, std::max<uint64_t>(M, 1) * 6 * 4, s));
        if (M) TG_TRY_CUDA(cudaMemcpyAsync(d, SG.bedges[b], M * 6 * 4, cudaMemcpyHostToDevice, s));
        ChainGraph cg;
        tg_status st = tg_build_direction(g, &cg, M, d, d + M, d + 2 * M, d + 3 * M, d + 4 * M, d + 5 * M, g->max_t, s);
        if (st != TG_OK) { cg.arena.free_all(); cudaFreeAsync(d, s); return st; }
        H.nn = cg.nnodes;
        H.L = M ? cg.nlong : 0;
        // the arrays the EAT engine reads, packed into one pinned block
        const uint64_t L1 = std::max<uint64_t>(H.L, 1);
        const uint64_t sz[8] = {(n + 1) * 4, H.nn * 4, (H.nn + 1) * 4, M * 4, M * 8, M * 16, L1 * 8, L1 * 16};
        uint64_t tot = 0;
        for (uint64_t x : sz) tot += (x + 255) & ~255ull;
        TG_TRY(host_alloc(&H.pinned, tot));
        H.bytes = tot;
        char *p = (char *)H.pinned;
        void **dst[8] = {(void **)&H.vnode_off, (void **)&H.node_t, (void **)&H.node_eoff, (void **)&H.occ_slot,
                         (void **)&H.occ_rec, (void **)&H.slots, (void **)&H.lc, (void **)&H.sc};
        const void *srcp[8] = {cg.vnode_off, cg.node_t, cg.node_eoff, cg.occ_slot, cg.occ_rec, cg.slots, cg.lc, cg.sc};
        for (int i = 0; i < 8; i++) {
            *dst[i] = p;
            const uint64_t bytes = (i == 0) ? sz[0] : (M ? sz[i] : 0);
            if (bytes && srcp[i]) TG_TRY_CUDA(cudaMemcpyAsync(p, srcp[i], bytes, cudaMemcpyDeviceToHost, s));
            p += (sz[i] + 255) & ~255ull;
        }
        TG_TRY_CUDA(cudaStreamSynchronize(s));
        cg.arena.free_all();
        TG_TRY_CUDA(cudaFreeAsync(d, s));
        SG.max_m = std::max(SG.max_m, M);
        SG.max_nn = std::max(SG.max_nn, H.nn);
        SG.max_L = std::max(SG.max_L, H.L);
    }
    // the input copies are no longer needed
    for (void *p : SG.bedges_pinned) cudaFreeHost(p);
    SG.bedges_pinned.clear();
    SG.bedges.clear();
    // two device slots sized for the largest block
    for (int i = 0; i < 2; i++) {
        ChainGraph &c = SG.slot[i];
        DevArena &A = SG.slot_arena;
        c.n = g->n;
        TG_TRY(A.alloc((void **)&c.vnode_off, (n + 1) * 4));
        TG_TRY(A.alloc((void **)&c.node_t, std::max<uint64_t>(SG.max_nn, 1) * 4));
        TG_TRY(A.alloc((void **)&c.node_eoff, (SG.max_nn + 1) * 4));
        TG_TRY(A.alloc((void **)&c.occ_slot, std::max<uint64_t>(SG.max_m, 1) * 4));
        TG_TRY(A.alloc((void **)&c.occ_rec, std::max<uint64_t>(SG.max_m, 1) * 8));
        TG_TRY(A.alloc((void **)&c.slots, std::max<uint64_t>(SG.max_m, 1) * 16));
        TG_TRY(A.alloc((void **)&c.lc, std::max<uint64_t>(SG.max_L, 1) * 8));
        TG_TRY(A.alloc((void **)&c.sc, std::max<uint64_t>(SG.max_L, 1) * 16));
    }
    TG_TRY_CUDA(cudaStreamCreateWithFlags(&SG.cs, cudaStreamNonBlocking));
    for (int i = 0; i < 2; i++) {
        TG_TRY_CUDA(cudaEventCreateWithFlags(&SG.ready[i], cudaEventDisableTiming));
        TG_TRY_CUDA(cudaEventCreateWithFlags(&SG.freed[i], cudaEventDisableTiming));
    }
    return TG_OK;
}

// Copy block b into device slot i on the copy stream once the slot's previous block is
// done (event freed[i], recorded by the query stream), then record ready[i].
tg_status tg_stream_load(tg_graph *g, uint32_t b, int i) {
    StreamGraph &SG = *g->stream;
    const HostBlock &H = SG.blocks[b];
    ChainGraph &c = SG.slot[i];
    const uint64_t n = g->n, M = H.m;
    TG_TRY_CUDA(cudaStreamWaitEvent(SG.cs, SG.freed[i], 0));
    const uint64_t L = H.L;
    struct { void *d; const void *h; uint64_t bytes; } cp[8] = {
        {c.vnode_off, H.vnode_off, (n + 1) * 4}, {c.node_t, H.node_t, H.nn * 4}, {c.node_eoff, H.node_eoff, (H.nn + 1) * 4},
        {c.occ_slot, H.occ_slot, M * 4}, {c.occ_rec, H.occ_rec, M * 8}, {c.slots, H.slots, M * 16},
        {c.lc, H.lc, L * 8}, {c.sc, H.sc, L * 16}};
    for (auto &x : cp) {
        if (!x.bytes) continue;
        TG_TRY_CUDA(cudaMemcpyAsync(x.d, x.h, x.bytes, cudaMemcpyHostToDevice, SG.cs));
        SG.h2d_bytes += x.bytes;
    }
    c.m = M;
    c.nnodes = H.nn;
    c.nlong = L;
    TG_TRY_CUDA(cudaEventRecord(SG.ready[i], SG.cs));
    return TG_OK;
}
