// api.cu -- the C-ABI entry points of include/tg.h.
#include <algorithm>
#include <mutex>
#include <chrono>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "tg_internal.cuh"

uint64_t g_tg_launches = 0;
static thread_local std::string t_err;

// ----------------------------------------------------------------------------- profiling
int g_tg_profile = 0;
namespace {
struct ProfRec { const char *name; cudaEvent_t e0, e1; };
std::vector<ProfRec> g_prof;
std::vector<cudaEvent_t> g_ev_pool;
cudaEvent_t ev_get() {
    if (!g_ev_pool.empty()) { cudaEvent_t e = g_ev_pool.back(); g_ev_pool.pop_back(); return e; }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
}
}  // namespace

cudaEvent_t tg_prof_begin(cudaStream_t s) {
    cudaEvent_t e = ev_get();
    cudaEventRecord(e, s);
    return e;
}

void tg_prof_end(const char *name, cudaStream_t s, cudaEvent_t ev0) {
    cudaEvent_t e = ev_get();
    cudaEventRecord(e, s);
    if (name[0] == '(') name++;  // TG_LAUNCH((k<A, B>), ...): parenthesised template launches
    g_prof.push_back({name, ev0, e});
}

void tg_set_error(const std::string &msg) { t_err = msg; }

// ----------------------------------------------------------------------------- caching allocator
// Device blocks released by a graph / query scratch are kept in a per-device free
// list and handed out again for requests of a similar size (<= 2x), so repeated
// create/build/query cycles do not pay cudaMalloc/cudaFree (which synchronises).
namespace {
struct CachedBlk { void *p; size_t bytes; int dev; };
std::vector<CachedBlk> g_cache;
std::mutex g_cache_mu;
size_t round_bytes(size_t b) { return (b + 511) & ~size_t(511); }
}  // namespace

static void *cache_take(size_t bytes, int dev, size_t *got) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    size_t best = (size_t)-1;
    int bi = -1;
    for (size_t i = 0; i < g_cache.size(); i++) {
        const CachedBlk &c = g_cache[i];
        if (c.dev == dev && c.bytes >= bytes && c.bytes <= 2 * bytes + (1u << 20) && c.bytes < best) {
            best = c.bytes;
            bi = (int)i;
        }
    }
    if (bi < 0) return nullptr;
    void *p = g_cache[bi].p;
    *got = g_cache[bi].bytes;
    g_cache.erase(g_cache.begin() + bi);
    return p;
}

static void cache_release_all(int dev) {
    std::lock_guard<std::mutex> lk(g_cache_mu);
    for (size_t i = 0; i < g_cache.size();) {
        if (dev < 0 || g_cache[i].dev == dev) {
            cudaFree(g_cache[i].p);
            g_cache.erase(g_cache.begin() + i);
        } else {
            i++;
        }
    }
}

cudaError_t tg_malloc_async(void **p, size_t bytes, cudaStream_t s) {
    cudaError_t e = cudaMallocAsync(p, bytes, s);
    if (e == cudaErrorMemoryAllocation) {
        cudaGetLastError();
        int dev = 0;
        cudaGetDevice(&dev);
        cudaStreamSynchronize(s);
        cache_release_all(dev);
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
        e = cudaMallocAsync(p, bytes, s);
    }
    return e;
}

namespace {
std::vector<void *> g_pinned;
std::mutex g_pinned_mu;
}  // namespace

cudaError_t tg_pinned_get(void **p) {
    {
        std::lock_guard<std::mutex> lk(g_pinned_mu);
        if (!g_pinned.empty()) {
            *p = g_pinned.back();
            g_pinned.pop_back();
            return cudaSuccess;
        }
    }
    return cudaMallocHost(p, 8192);  // >= TG_MAXP RoundCtl records
}

void tg_pinned_put(void *p) {
    if (!p) return;
    std::lock_guard<std::mutex> lk(g_pinned_mu);
    g_pinned.push_back(p);
}

tg_status DevArena::alloc(void **p, size_t bytes) {
    *p = nullptr;
    bytes = round_bytes(bytes ? bytes : 16);
    if (use_pool) {  // no retry: a query lane that does not fit is simply not used
        void *q = nullptr;
        if (cudaMallocAsync(&q, bytes, pool_stream) != cudaSuccess) {
            cudaGetLastError();
            tg_set_error("query lane scratch does not fit");
            return TG_ERR_NOMEM;
        }
        *p = q;
        blks.push_back({q, bytes});
        total += bytes;
        return TG_OK;
    }
    int dev = 0;
    cudaGetDevice(&dev);
    size_t got = bytes;
    void *q = cache_take(bytes, dev, &got);
    if (!q) {
        if (slack_pct) bytes = round_bytes(bytes + bytes / 100 * slack_pct);
        got = bytes;
        cudaError_t e = cudaMalloc(&q, bytes);
        if (e != cudaSuccess) {
            cudaGetLastError();
            // return cached blocks and the stream-ordered pool's free memory to the driver, retry once
            cudaDeviceSynchronize();
            cache_release_all(dev);
            cudaMemPool_t pool;
            if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
            e = cudaMalloc(&q, bytes);
        }
        if (e != cudaSuccess) {
            cudaGetLastError();
            tg_set_error(std::string("cudaMalloc(") + std::to_string(bytes) + "): " + cudaGetErrorString(e));
            return TG_ERR_NOMEM;
        }
    }
    *p = q;
    blks.push_back({q, got});
    total += got;
    return TG_OK;
}

void DevArena::free_all() {
    if (use_pool) {  // stream-ordered: after the lane's queued work
        for (const Blk &b : blks) cudaFreeAsync(b.p, pool_stream);
        blks.clear();
        total = 0;
        return;
    }
    // callers synchronise before releasing (blocks may be reused by the next owner at once)
    int dev = 0;
    cudaGetDevice(&dev);
    std::lock_guard<std::mutex> lk(g_cache_mu);
    for (const Blk &b : blks) g_cache.push_back({b.p, b.bytes, dev});
    blks.clear();
    total = 0;
}

tg_status tg_validate_edges(tg_graph *g, cudaStream_t s);
tg_status tg_build_mirror(tg_graph *g, cudaStream_t s);
tg_status tg_run_eat_family(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w,
                            uint32_t *out, uint32_t *pred, bool out_dev, bool pred_dev, cudaStream_t s);
tg_status tg_run_reach_bits(tg_graph *g, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                            bool out_dev, cudaStream_t s);
tg_status tg_run_spfp(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w, uint32_t *out,
                      bool out_dev, cudaStream_t s);
tg_status tg_run_eat_partitioned(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t k, tg_window w,
                                 uint32_t *out, uint32_t *pred, bool out_dev, bool pred_dev, cudaStream_t s);
int tg_comm_rank(const tg_comm *c);
int tg_comm_world(const tg_comm *c);

static bool is_device_ptr(const void *p) {
    if (!p) return false;
    cudaPointerAttributes a;
    cudaError_t e = cudaPointerGetAttributes(&a, p);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

namespace {
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};
}  // namespace

uint64_t tg_graph_bytes(const tg_graph *g) {
    uint64_t b = g->arena.total + g->qs.arena.total + g->qsl[0].arena.total + g->qsl[1].arena.total + g->qsl[2].arena.total + g->rs.arena.total + g->fwd.arena.total + g->mir.arena.total;
    for (int p = 0; p < TG_MAXP; p++) b += g->pf[p].arena.total + g->pm[p].arena.total;
    if (g->stream) b += g->stream->slot_arena.total;
    return b;
}

extern "C" {

const char *tg_status_string(tg_status s) {
    switch (s) {
        case TG_OK: return "TG_OK";
        case TG_ERR_INVALID: return "TG_ERR_INVALID";
        case TG_ERR_RANGE: return "TG_ERR_RANGE";
        case TG_ERR_NOMEM: return "TG_ERR_NOMEM";
        case TG_ERR_CUDA: return "TG_ERR_CUDA";
        case TG_ERR_STATE: return "TG_ERR_STATE";
        case TG_ERR_NCCL: return "TG_ERR_NCCL";
    }
    return "TG_ERR_UNKNOWN";
}

const char *tg_last_error(void) { return t_err.c_str(); }

uint64_t tg_kernel_launch_count(void) { return g_tg_launches; }

void tg_release_cached_memory(void) {
    cudaDeviceSynchronize();
    cache_release_all(-1);
    int dev = 0;
    cudaGetDevice(&dev);
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) cudaMemPoolTrimTo(pool, 0);
    cudaGetLastError();
}

void tg_profile_enable(int on) { g_tg_profile = (on < 0 || on > 2) ? 1 : on; }

int tg_profile_report(char *buf, uint64_t buf_len) {
    // {"kernel": [launches, total_ms], ...}.  Recorded launches are folded into a
    // running table; a call with a buffer writes the table and clears it, a call
    // with buf == NULL only returns the size needed.
    struct Acc { std::string name; uint64_t n = 0; double ms = 0; };
    static std::vector<Acc> acc;
    // graph round loops of concurrent query lanes overlap in time: their union as well
    // ("k_eat_rounds_union": the wall time some lane's round loop was running)
    {
        const char *pre = "k_eat_rounds";
        cudaEvent_t ref = nullptr;
        std::vector<std::pair<double, double>> iv;
        for (auto &r : g_prof) {
            if (std::strncmp(r.name, pre, std::strlen(pre)) != 0) continue;
            cudaEventSynchronize(r.e1);
            if (!ref) ref = r.e0;
            float a = 0, b = 0;
            cudaEventElapsedTime(&a, ref, r.e0);
            cudaEventElapsedTime(&b, ref, r.e1);
            iv.push_back({a, b});
        }
        if (!iv.empty()) {
            std::sort(iv.begin(), iv.end());
            double tot = 0, lo = iv[0].first, hi = iv[0].second;
            for (auto &x : iv) {
                if (x.first > hi) { tot += hi - lo; lo = x.first; hi = x.second; }
                else hi = std::max(hi, x.second);
            }
            tot += hi - lo;
            const std::string nm = "k_eat_rounds_union";
            auto it = std::find_if(acc.begin(), acc.end(), [&](const Acc &p) { return p.name == nm; });
            if (it == acc.end()) { acc.push_back(Acc{nm}); it = acc.end() - 1; }
            it->n += iv.size();
            it->ms += tot;
        }
    }
    for (auto &r : g_prof) {
        cudaEventSynchronize(r.e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, r.e0, r.e1);
        std::string nm(r.name);
        if (!nm.empty() && nm.back() == ')') nm.pop_back();  // "(k<A, B>)" launches
        auto it = std::find_if(acc.begin(), acc.end(), [&](const Acc &p) { return p.name == nm; });
        if (it == acc.end()) { acc.push_back(Acc{nm}); it = acc.end() - 1; }
        it->n++;
        it->ms += ms;
        g_ev_pool.push_back(r.e0);
        g_ev_pool.push_back(r.e1);
    }
    g_prof.clear();
    std::string js = "{";
    for (size_t i = 0; i < acc.size(); i++) {
        char tmp[320];
        snprintf(tmp, sizeof(tmp), "%s\"%s\": [%llu, %.6f]", i ? ", " : "", acc[i].name.c_str(),
                 (unsigned long long)acc[i].n, acc[i].ms);
        js += tmp;
    }
    js += "}";
    if (!buf || buf_len == 0) return (int)js.size() + 1;
    snprintf(buf, buf_len, "%s", js.c_str());
    acc.clear();
    return (int)js.size() + 1;
}

tg_status tg_graph_create(uint32_t n_vertices, uint64_t n_edges, const uint32_t *u, const uint32_t *v,
                          const uint32_t *t_start, const uint32_t *duration, const uint32_t *weight, int device,
                          tg_graph **out_graph) {
    t_err.clear();
    if (!out_graph) { tg_set_error("out_graph is NULL"); return TG_ERR_INVALID; }
    *out_graph = nullptr;
    if (n_vertices == 0) { tg_set_error("n_vertices must be >= 1"); return TG_ERR_INVALID; }
    if (n_edges >= 0xFFFFFFFFull) { tg_set_error("n_edges must be < 2^32 - 1"); return TG_ERR_RANGE; }
    if (n_edges > 0 && (!u || !v || !t_start || !duration)) { tg_set_error("edge array is NULL"); return TG_ERR_INVALID; }
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
        cudaGetLastError();
        tg_set_error("no CUDA device");
        return TG_ERR_CUDA;
    }
    if (device < 0 || device >= ndev) { tg_set_error("bad device ordinal"); return TG_ERR_INVALID; }
    DeviceGuard dg(device);
    {
        // keep the stream-ordered pool's memory between builds (the default release
        // threshold of 0 returns it to the driver at every synchronisation, and the
        // next cudaMallocAsync has to map it again)
        static bool pool_set[64] = {false};
        if (device < 64 && !pool_set[device]) {
            cudaMemPool_t pool;
            if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
                uint64_t thr = UINT64_MAX;
                cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
            }
            cudaGetLastError();
            pool_set[device] = true;
        }
    }
    tg_graph *g = new tg_graph();
    g->device = device;
    g->n = n_vertices;
    g->m = n_edges;
    const size_t bytes = n_edges * 4;
    tg_status st = TG_OK;
    auto fail = [&](tg_status s) { g->arena.free_all(); delete g; return s; };
    uint32_t **dst[5] = {&g->d_u, &g->d_v, &g->d_t, &g->d_dur, &g->d_w};
    const uint32_t *src[5] = {u, v, t_start, duration, weight};
    for (int i = 0; i < 5; i++) {
        if (i == 4 && !weight) { g->d_w = g->d_dur; break; }  // reading A7: w = duration
        if ((st = g->arena.alloc((void **)dst[i], bytes)) != TG_OK) return fail(st);
        if (n_edges) {
            cudaError_t e = cudaMemcpy(*dst[i], src[i], bytes, cudaMemcpyDefault);
            if (e != cudaSuccess) { tg_set_error(cudaGetErrorString(e)); cudaGetLastError(); return fail(TG_ERR_CUDA); }
        }
    }
    if ((st = tg_validate_edges(g, 0)) != TG_OK) return fail(st);
    *out_graph = g;
    return TG_OK;
}

tg_status tg_build_chains(tg_graph *g) {
    t_err.clear();
    if (!g) { tg_set_error("graph is NULL"); return TG_ERR_INVALID; }
    if (g->built) return TG_OK;
    DeviceGuard dg(g->device);
    auto t0 = std::chrono::steady_clock::now();
    if (g->stream) {
        // out-of-memory graph: every time block transformed on the device, kept in host memory
        TG_TRY(tg_build_streamed(g));
    } else if (g->comm && g->comm_mode == 1) {
        // this rank's vertex range of a single partitioned query batch
        const int r = tg_comm_rank(g->comm), P = tg_comm_world(g->comm);
        g->nparts = 1;
        g->part_vb[0] = (uint32_t)((uint64_t)g->n * r / P);
        g->part_vb[1] = (uint32_t)((uint64_t)g->n * (r + 1) / P);
        TG_TRY(tg_build_partition(g, &g->pf[0], &g->pm[0], g->part_vb[0], g->part_vb[1], 0, g->opt_mirror ? 3 : 1));
        g->mirror_built = g->opt_mirror != 0;
    } else if (g->opt_partitions > 1) {
        // logical vertex-range partitions on one GPU (same algorithm, shared state)
        const int P = g->opt_partitions;
        g->nparts = P;
        for (int p = 0; p <= P; p++) g->part_vb[p] = (uint32_t)((uint64_t)g->n * p / P);
        for (int p = 0; p < P; p++)
            TG_TRY(tg_build_partition(g, &g->pf[p], &g->pm[p], g->part_vb[p], g->part_vb[p + 1], 0, g->opt_mirror ? 3 : 1));
        g->mirror_built = g->opt_mirror != 0;
    } else {
        if (g->opt_relabel) TG_TRY(tg_relabel(g, 0));
        const uint32_t *U = g->relabeled ? g->d_ru : g->d_u, *V = g->relabeled ? g->d_rv : g->d_v;
        TG_TRY(tg_build_direction(g, &g->fwd, g->m, U, V, g->d_t, g->d_dur, g->d_w, nullptr, g->max_t, 0));
        if (g->opt_mirror) {
            TG_TRY(tg_build_mirror(g, 0));
            g->mirror_built = true;
        }
    }
    TG_TRY_CUDA(cudaDeviceSynchronize());
    g->build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    g->built = true;
    return TG_OK;
}

tg_status tg_query(tg_graph *g, tg_problem p, const uint32_t *sources, uint32_t n_sources, tg_window w, uint32_t *out,
                   uint32_t *pred, void *cuda_stream) {
    t_err.clear();
    if (!g) { tg_set_error("graph is NULL"); return TG_ERR_INVALID; }
    if (!g->built) { tg_set_error("tg_query before tg_build_chains"); return TG_ERR_STATE; }
    if (!sources || !out || n_sources == 0) { tg_set_error("sources/out NULL or n_sources == 0"); return TG_ERR_INVALID; }
    if ((int)p < 0 || (int)p > TG_LD_SOURCE) { tg_set_error("unknown problem"); return TG_ERR_INVALID; }
    if (pred && !(p == TG_EAT || p == TG_LD || p == TG_REACH)) {
        tg_set_error("pred is only defined for TG_EAT / TG_LD / TG_REACH");
        return TG_ERR_INVALID;
    }
    if (w.t_alpha > w.t_omega) { tg_set_error("t_alpha > t_omega"); return TG_ERR_INVALID; }
    if (is_device_ptr(sources)) { tg_set_error("sources must be a host pointer"); return TG_ERR_INVALID; }
    for (uint32_t i = 0; i < n_sources; i++)
        if (sources[i] >= g->n) { tg_set_error("source >= n_vertices"); return TG_ERR_RANGE; }
    if (p == TG_SHORTEST && !g->sp_ok) {
        tg_set_error("shortest-path distances could overflow uint32 for this graph's weights");
        return TG_ERR_RANGE;
    }
    DeviceGuard dg(g->device);
    cudaStream_t s = (cudaStream_t)cuda_stream;
    const bool out_dev = is_device_ptr(out);
    const bool pred_dev = is_device_ptr(pred);
    if (g->stream) {
        if (!(p == TG_EAT || p == TG_REACH)) {
            tg_set_error("streamed (out-of-memory) graphs answer TG_EAT / TG_REACH");
            return TG_ERR_STATE;
        }
        return tg_run_eat_streamed(g, sources, n_sources, w, out, pred, out_dev, pred_dev, p == TG_REACH ? 2 : 0, s);
    }
    if (p == TG_LD && !g->mirror_built) {  // lazily built mirror (option "mirror" = 0)
        if (g->nparts > 0) {
            for (int pi = 0; pi < g->nparts; pi++)
                TG_TRY(tg_build_partition(g, &g->pf[pi], &g->pm[pi], g->part_vb[pi], g->part_vb[pi + 1], 0, 2));
        } else {
            TG_TRY(tg_build_mirror(g, 0));
        }
        g->mirror_built = true;
    }
    if (g->nparts > 0) {
        if (!(p == TG_EAT || p == TG_LD || p == TG_REACH)) {
            tg_set_error("vertex-range partitioned graphs answer TG_EAT / TG_LD / TG_REACH only");
            return TG_ERR_STATE;
        }
        return tg_run_eat_partitioned(g, p, sources, n_sources, w, out, pred, out_dev, pred_dev, s);
    }
    if (p == TG_REACH && !pred && g->opt_reach_bits) return tg_run_reach_bits(g, sources, n_sources, w, out, out_dev, s);
    if (p == TG_EAT || p == TG_LD || p == TG_REACH) {
        return tg_run_eat_family(g, p, sources, n_sources, w, out, pred, out_dev, pred_dev, s);
    }
    return tg_run_spfp(g, p, sources, n_sources, w, out, out_dev, s);
}

void tg_graph_destroy(tg_graph *g) {
    if (!g) return;
    DeviceGuard dg(g->device);
    cudaDeviceSynchronize();
    tg_sink_destroy(g);
    tg_stream_free(g);
    g->qs.arena.free_all();
    tg_pinned_put(g->qs.h_ctr);
    for (auto &q : g->qsl) {
        q.arena.free_all();
        tg_pinned_put(q.h_ctr);
    }
    for (auto &x : g->lane_stream)
        if (x) cudaStreamDestroy(x);
    for (auto &e : g->lane_join)
        if (e) cudaEventDestroy(e);
    if (g->lane_fork) cudaEventDestroy(g->lane_fork);
    g->rs.arena.free_all();
    tg_pinned_put(g->rs.h_ctr);
    g->fwd.arena.free_all();
    g->mir.arena.free_all();
    for (int p = 0; p < TG_MAXP; p++) { g->pf[p].arena.free_all(); g->pm[p].arena.free_all(); }
    g->arena.free_all();
    delete[] g->last_relax;
    delete g;
}

tg_status tg_graph_info(const tg_graph *g, tg_info *info) {
    if (!g || !info) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    std::memset(info, 0, sizeof(*info));
    info->n_vertices = g->n;
    info->n_edges = g->m;
    info->n_nodes = g->fwd.nnodes;
    info->n_chains = g->fwd.nchains;
    info->n_long_chains = g->fwd.nlong;
    info->max_chain_len = g->fwd.maxlen;
    if (g->stream)
        for (const HostBlock &b : g->stream->blocks) {  // streamed: totals over the time blocks
            info->n_nodes += b.nn;
            info->n_long_chains += b.L;
        }
    for (int p = 0; p < g->nparts; p++) {  // partitioned: totals over this process's partitions
        info->n_nodes += g->pf[p].nnodes;
        info->n_chains += g->pf[p].nchains;
        info->n_long_chains += g->pf[p].nlong;
        info->max_chain_len = std::max(info->max_chain_len, g->pf[p].maxlen);
    }
    info->c_mirror = g->max_arr;
    info->device_bytes = tg_graph_bytes(g);
    info->build_ms = g->build_ms;
    info->built = g->built ? 1 : 0;
    info->n_chains_mirror = g->mir.nchains;
    if (g->stream) {
        info->n_blocks = (uint32_t)g->stream->blocks.size();
        for (const HostBlock &b : g->stream->blocks) info->host_bytes += b.bytes;
    }
    return TG_OK;
}

tg_status tg_export_chains(const tg_graph *g, int mirrored, uint64_t *chain_off, uint32_t *chain_edges,
                           uint32_t *sc_tail_v, uint32_t *sc_arr, uint64_t *sc_sum_w, uint32_t *sc_elapsed) {
    if (!g || !chain_off || !chain_edges) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    if (!g->built) { tg_set_error("graph not built"); return TG_ERR_STATE; }
    if (g->nparts > 0 || g->stream) { tg_set_error("chain export is for unpartitioned, device-resident graphs"); return TG_ERR_STATE; }
    if (mirrored && !g->mirror_built) { tg_set_error("the mirror graph has not been built"); return TG_ERR_STATE; }
    DeviceGuard dg(g->device);
    const ChainGraph &c = mirrored ? g->mir : g->fwd;
    const uint64_t m = g->m, nc = c.nchains;
    std::vector<uint32_t> first(nc + 1);
    std::vector<int4> slots(m);
    TG_TRY_CUDA(cudaMemcpy(first.data(), c.chain_first, (nc + 1) * 4, cudaMemcpyDeviceToHost));
    if (m) TG_TRY_CUDA(cudaMemcpy(slots.data(), c.slots, m * 16, cudaMemcpyDeviceToHost));
    // chain order: when the engine relabelled vertices its chains are ordered by the
    // internal head vertex; export them in the paper's (original head u, t, first id) order
    std::vector<uint64_t> order(nc);
    for (uint64_t i = 0; i < nc; i++) order[i] = i;
    std::vector<uint32_t> hu, ht, iperm;
    if (g->relabeled && nc) {
        hu.resize(m);
        ht.resize(m);
        iperm.resize(g->n);
        TG_TRY_CUDA(cudaMemcpy(hu.data(), mirrored ? g->d_v : g->d_u, m * 4, cudaMemcpyDeviceToHost));
        TG_TRY_CUDA(cudaMemcpy(iperm.data(), g->iperm, (size_t)g->n * 4, cudaMemcpyDeviceToHost));
        std::vector<uint32_t> dur(m);
        TG_TRY_CUDA(cudaMemcpy(dur.data(), g->d_dur, m * 4, cudaMemcpyDeviceToHost));
        for (uint64_t i = 0; i < m; i++) ht[i] = (uint32_t)slots[i].y - dur[(uint32_t)slots[i].z];  // per slot
        std::sort(order.begin(), order.end(), [&](uint64_t a, uint64_t b) {
            const int4 &sa = slots[first[a]], &sb = slots[first[b]];
            const uint32_t ua = hu[(uint32_t)sa.z], ub = hu[(uint32_t)sb.z];
            if (ua != ub) return ua < ub;
            const uint32_t ta = ht[first[a]], tb = ht[first[b]];
            if (ta != tb) return ta < tb;
            return (uint32_t)sa.z < (uint32_t)sb.z;
        });
    }
    {
        uint64_t pos = 0;
        for (uint64_t i = 0; i < nc; i++) {
            chain_off[i] = pos;
            for (uint32_t sl = first[order[i]]; sl < first[order[i] + 1]; sl++) chain_edges[pos++] = (uint32_t)slots[sl].z;
        }
        chain_off[nc] = pos;
    }
    if (sc_tail_v || sc_arr || sc_sum_w || sc_elapsed) {
        std::vector<int4> sc(c.nlong);
        std::vector<unsigned long long> sumw(c.nlong);
        std::vector<uint32_t> el(c.nlong), w(m), slot_w(m), t(m);
        if (c.nlong) {
            TG_TRY_CUDA(cudaMemcpy(sc.data(), c.sc, c.nlong * 16, cudaMemcpyDeviceToHost));
            TG_TRY_CUDA(cudaMemcpy(sumw.data(), c.sc_sumw, c.nlong * 8, cudaMemcpyDeviceToHost));
            TG_TRY_CUDA(cudaMemcpy(el.data(), c.sc_elapsed, c.nlong * 4, cudaMemcpyDeviceToHost));
        }
        if (m) {
            TG_TRY_CUDA(cudaMemcpy(slot_w.data(), c.slot_w, m * 4, cudaMemcpyDeviceToHost));
            // departure time of a one-edge chain = arrival - duration of its edge
            std::vector<uint32_t> dur(m);
            TG_TRY_CUDA(cudaMemcpy(dur.data(), g->d_dur, m * 4, cudaMemcpyDeviceToHost));
            for (uint64_t s = 0; s < m; s++) t[s] = (uint32_t)slots[s].y - dur[(uint32_t)slots[s].z];
        }
        // long-chain index: chains with >= 2 edges numbered in internal chain order
        std::vector<uint32_t> lidx(nc, 0);
        for (uint64_t ch = 0, l = 0; ch < nc; ch++)
            if (first[ch + 1] - first[ch] >= 2) lidx[ch] = (uint32_t)l++;
        auto vout = [&](uint32_t v) { return g->relabeled ? iperm[v] : v; };
        for (uint64_t oi = 0; oi < nc; oi++) {
            const uint64_t ch = order[oi];
            uint32_t b = first[ch], e = first[ch + 1];
            int4 sl = slots[b];
            const uint64_t ochn = oi;  // output position
            if (e - b >= 2) {
                const uint32_t l = lidx[ch];
                if (sc_tail_v) sc_tail_v[ochn] = vout((uint32_t)sc[l].x);
                if (sc_arr) sc_arr[ochn] = (uint32_t)sc[l].y;
                if (sc_sum_w) sc_sum_w[ochn] = sumw[l];
                if (sc_elapsed) sc_elapsed[ochn] = el[l];
            } else {  // Alg. 2 line 8: a one-edge chain is its own shortcut
                if (sc_tail_v) sc_tail_v[ochn] = vout((uint32_t)sl.x);
                if (sc_arr) sc_arr[ochn] = (uint32_t)sl.y;
                if (sc_sum_w) sc_sum_w[ochn] = slot_w[b];
                if (sc_elapsed) sc_elapsed[ochn] = (uint32_t)sl.y - t[b];
            }
        }
    }
    return TG_OK;
}

tg_status tg_last_query_stats(const tg_graph *g, tg_query_stats *st, uint64_t *per_query_relax) {
    if (!g || !st) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    *st = g->last;
    if (per_query_relax && g->last_relax)
        std::memcpy(per_query_relax, g->last_relax, (size_t)g->last_relax_len * 8);
    return TG_OK;
}

tg_status tg_set_option(tg_graph *g, const char *key, int64_t value) {
    if (!g || !key) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    std::string k(key);
    if (k == "sub_batch") g->opt_sub_batch = value;
    else if (k == "stats") g->opt_stats = value;
    else if (k == "shortcuts") g->opt_shortcuts = value;
    else if (k == "round_group") g->opt_round_group = value;
    else if (k == "mirror") g->opt_mirror = value ? 1 : 0;
    else if (k == "relabel") {
        if (g->built) { tg_set_error("set relabel before tg_build_chains"); return TG_ERR_STATE; }
        g->opt_relabel = value ? 1 : 0;
    }
    else if (k == "exchange") g->opt_exchange = value ? 1 : 0;
    else if (k == "packed_state") g->opt_packed_state = value ? 1 : 0;
    else if (k == "graph_loop") g->opt_graph_loop = value < 0 ? 0 : (value > 2 ? 2 : value);
    else if (k == "lanes") g->opt_lanes = value < 1 ? 1 : (value > TG_LANES ? TG_LANES : value);
    else if (k == "ub_filter") g->opt_ub = value < 0 ? 0 : (value > 2 ? 2 : value);
    else if (k == "reach_bits") g->opt_reach_bits = value ? 1 : 0;
    else if (k == "order_sources") g->opt_order_sources = value ? 1 : 0;
    else if (k == "dynamic") {
        if (g->built) { tg_set_error("set dynamic before tg_build_chains"); return TG_ERR_STATE; }
        g->opt_dynamic = value ? 1 : 0;
    }
    else if (k == "walk_min") {
        if (g->built) { tg_set_error("set walk_min before tg_build_chains"); return TG_ERR_STATE; }
        g->opt_walk_min = value < 2 ? 2 : value;
    }
    else if (k == "partitions") {
        if (g->built) { tg_set_error("set partitions before tg_build_chains"); return TG_ERR_STATE; }
        if (value < 1 || value > TG_MAXP) { tg_set_error("partitions must be in [1, 16]"); return TG_ERR_RANGE; }
        g->opt_partitions = (int)value;
    }
    else { tg_set_error("unknown option " + k); return TG_ERR_INVALID; }
    return TG_OK;
}

}  // extern "C"
