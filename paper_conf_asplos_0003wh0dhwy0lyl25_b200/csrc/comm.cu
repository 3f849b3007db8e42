// comm.cu -- NCCL communicator for the vertex-range multi-GPU mode.
//
// A single huge query is partitioned by vertex range: rank r owns the chains of
// the edges leaving its vertices and, after each GAC round, the packed
// (arrival << 32 | pred) states of all ranks are combined with an
// ncclAllReduce(min) over NVLink / NVSwitch.  Min of packed words is
// order-independent, so results are identical for every rank count.
//
// NCCL is loaded with dlopen("libnccl.so.2") at first use, so the library links no
// NCCL at build time and shares the copy the process already has (e.g. the one
// PyTorch loaded) instead of bringing a second one.
#include <dlfcn.h>

#include <cstring>
#include <string>

#include "tg_internal.cuh"

namespace {

struct NcclUid { char internal[128]; };
typedef void *ncclComm_p;
// enums from nccl.h (stable across 2.x): ncclSum = 0, ncclMin = 3; ncclUint32 = 3, ncclUint64 = 5
constexpr int kNcclSum = 0, kNcclMin = 3, kNcclUint32 = 3, kNcclUint64 = 5;

struct NcclApi {
    bool ok = false;
    std::string err;
    int (*GetUniqueId)(NcclUid *) = nullptr;
    int (*CommInitRank)(ncclComm_p *, int, NcclUid, int) = nullptr;
    int (*CommDestroy)(ncclComm_p) = nullptr;
    int (*AllReduce)(const void *, void *, size_t, int, int, ncclComm_p, cudaStream_t) = nullptr;
    const char *(*GetErrorString)(int) = nullptr;
};

NcclApi &nccl() {
    static NcclApi api;
    static bool tried = false;
    if (tried) return api;
    tried = true;
    void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
    if (!h) {
        api.err = std::string("dlopen libnccl.so.2 failed: ") + dlerror();
        return api;
    }
    api.GetUniqueId = (int (*)(NcclUid *))dlsym(h, "ncclGetUniqueId");
    api.CommInitRank = (int (*)(ncclComm_p *, int, NcclUid, int))dlsym(h, "ncclCommInitRank");
    api.CommDestroy = (int (*)(ncclComm_p))dlsym(h, "ncclCommDestroy");
    api.AllReduce = (int (*)(const void *, void *, size_t, int, int, ncclComm_p, cudaStream_t))dlsym(h, "ncclAllReduce");
    api.GetErrorString = (const char *(*)(int))dlsym(h, "ncclGetErrorString");
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllReduce && api.GetErrorString;
    if (!api.ok) api.err = "libnccl.so.2 lacks a required symbol";
    return api;
}

}  // namespace

struct tg_comm {
    ncclComm_p comm = nullptr;
    int rank = 0, world = 1, device = 0;
};

#define TG_TRY_NCCL(expr)                                                                  \
    do {                                                                                   \
        int _r = (expr);                                                                   \
        if (_r != 0) {                                                                     \
            tg_set_error(std::string(#expr) + ": " + nccl().GetErrorString(_r));           \
            return TG_ERR_NCCL;                                                            \
        }                                                                                  \
    } while (0)

tg_status tg_comm_allreduce_min_u64(tg_comm *c, unsigned long long *buf, uint64_t count, cudaStream_t s) {
    if (!c->comm) return TG_OK;  // world 1 without NCCL
    TG_TRY_NCCL(nccl().AllReduce(buf, buf, count, kNcclUint64, kNcclMin, c->comm, s));
    return TG_OK;
}

tg_status tg_comm_allreduce_min_u32(tg_comm *c, uint32_t *buf, uint64_t count, cudaStream_t s) {
    if (!c->comm) return TG_OK;
    TG_TRY_NCCL(nccl().AllReduce(buf, buf, count, kNcclUint32, kNcclMin, c->comm, s));
    return TG_OK;
}

tg_status tg_comm_allreduce_sum_u32(tg_comm *c, uint32_t *buf, uint64_t count, cudaStream_t s) {
    if (!c->comm) return TG_OK;
    TG_TRY_NCCL(nccl().AllReduce(buf, buf, count, kNcclUint32, kNcclSum, c->comm, s));
    return TG_OK;
}

int tg_comm_rank(const tg_comm *c) { return c->rank; }
int tg_comm_world(const tg_comm *c) { return c->world; }

extern "C" {

tg_status tg_nccl_unique_id(void *out_id) {
    if (!out_id) { tg_set_error("out_id is NULL"); return TG_ERR_INVALID; }
    NcclApi &api = nccl();
    if (!api.ok) { tg_set_error(api.err); return TG_ERR_NCCL; }
    NcclUid id;
    TG_TRY_NCCL(api.GetUniqueId(&id));
    std::memcpy(out_id, &id, sizeof(id));
    return TG_OK;
}

tg_status tg_comm_create(const void *nccl_unique_id, int rank, int world, int device, tg_comm **out) {
    if (!out || !nccl_unique_id) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    *out = nullptr;
    if (world < 1 || rank < 0 || rank >= world) { tg_set_error("bad rank / world"); return TG_ERR_INVALID; }
    tg_comm *c = new tg_comm();
    c->rank = rank;
    c->world = world;
    c->device = device;
    NcclApi &api = nccl();
    if (world > 1 && !api.ok) { tg_set_error(api.err); delete c; return TG_ERR_NCCL; }
    if (api.ok) {  // world 1 also goes through NCCL when it is available (exercises the path)
        int prev = 0;
        cudaGetDevice(&prev);
        cudaSetDevice(device);
        NcclUid id;
        std::memcpy(&id, nccl_unique_id, sizeof(id));
        int r = api.CommInitRank(&c->comm, world, id, rank);
        cudaSetDevice(prev);
        if (r != 0) {
            tg_set_error(std::string("ncclCommInitRank: ") + api.GetErrorString(r));
            delete c;
            return TG_ERR_NCCL;
        }
    }
    *out = c;
    return TG_OK;
}

void tg_comm_destroy(tg_comm *c) {
    if (!c) return;
    if (c->comm && nccl().ok) nccl().CommDestroy(c->comm);
    delete c;
}

tg_status tg_graph_attach_comm(tg_graph *g, tg_comm *c, int mode) {
    if (!g || !c) { tg_set_error("NULL argument"); return TG_ERR_INVALID; }
    if (mode != 0 && mode != 1) { tg_set_error("mode must be 0 (replicate) or 1 (vertex range)"); return TG_ERR_INVALID; }
    if (g->built) { tg_set_error("attach the communicator before tg_build_chains"); return TG_ERR_STATE; }
    if (c->device != g->device) { tg_set_error("communicator and graph live on different devices"); return TG_ERR_INVALID; }
    g->comm = c;
    g->comm_mode = mode;
    return TG_OK;
}

}  // extern "C"
