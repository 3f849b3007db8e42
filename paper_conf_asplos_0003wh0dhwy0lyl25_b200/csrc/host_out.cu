// host_out.cu -- host-memory outputs of tg_query: double-buffered device staging
// with the device->host copies on their own stream (overlapping the next sub-batch).
#include "tg_internal.cuh"

tg_status tg_sink_begin(tg_graph *g, bool out_host, bool pred_host) {
    if (!out_host && !pred_host) return TG_OK;
    QueryScratch &Q = g->qs;
    const uint64_t bytes = (uint64_t)Q.S * g->n * 4;
    for (int i = 0; i < 2; i++) {
        if (out_host && !Q.out_stage[i]) TG_TRY(Q.arena.alloc((void **)&Q.out_stage[i], bytes));
        if (pred_host && !Q.pred_stage[i]) TG_TRY(Q.arena.alloc((void **)&Q.pred_stage[i], bytes));
    }
    if (!g->cstream) {
        TG_TRY_CUDA(cudaStreamCreateWithFlags(&g->cstream, cudaStreamNonBlocking));
        for (int i = 0; i < 2; i++) {
            TG_TRY_CUDA(cudaEventCreateWithFlags(&g->ev_x[i], cudaEventDisableTiming));
            TG_TRY_CUDA(cudaEventCreateWithFlags(&g->ev_c[i], cudaEventDisableTiming));
            TG_TRY_CUDA(cudaEventRecord(g->ev_c[i], g->cstream));  // "copy done" for the first use
        }
    }
    return TG_OK;
}

tg_status tg_sink_target(tg_graph *g, uint32_t b, bool out_host, bool pred_host, uint32_t **o, uint32_t **pr,
                         cudaStream_t s) {
    if (!out_host && !pred_host) return TG_OK;
    const int i = (int)(b & 1);
    TG_TRY_CUDA(cudaStreamWaitEvent(s, g->ev_c[i], 0));  // buffer i's previous copy has left
    if (out_host) *o = g->qs.out_stage[i];
    if (pred_host && *pr) *pr = g->qs.pred_stage[i];
    return TG_OK;
}

tg_status tg_sink_flush(tg_graph *g, uint32_t b, uint32_t *host_out, uint32_t *host_pred, size_t bytes, cudaStream_t s) {
    if (!host_out && !host_pred) return TG_OK;
    const int i = (int)(b & 1);
    TG_TRY_CUDA(cudaEventRecord(g->ev_x[i], s));
    TG_TRY_CUDA(cudaStreamWaitEvent(g->cstream, g->ev_x[i], 0));
    if (host_out)
        TG_TRY_CUDA(cudaMemcpyAsync(host_out, g->qs.out_stage[i], bytes, cudaMemcpyDeviceToHost, g->cstream));
    if (host_pred)
        TG_TRY_CUDA(cudaMemcpyAsync(host_pred, g->qs.pred_stage[i], bytes, cudaMemcpyDeviceToHost, g->cstream));
    TG_TRY_CUDA(cudaEventRecord(g->ev_c[i], g->cstream));
    return TG_OK;
}

// as tg_sink_flush, with the staging buffer's row q going to the caller's row rows[q]
tg_status tg_sink_flush_rows(tg_graph *g, uint32_t b, uint32_t *host_out, uint32_t *host_pred, const uint32_t *rows,
                             uint32_t nrows, uint64_t n, cudaStream_t s) {
    if (!host_out && !host_pred) return TG_OK;
    const int i = (int)(b & 1);
    TG_TRY_CUDA(cudaEventRecord(g->ev_x[i], s));
    TG_TRY_CUDA(cudaStreamWaitEvent(g->cstream, g->ev_x[i], 0));
    for (uint32_t q = 0; q < nrows; q++) {
        if (host_out)
            TG_TRY_CUDA(cudaMemcpyAsync(host_out + (size_t)rows[q] * n, g->qs.out_stage[i] + (size_t)q * n, n * 4,
                                        cudaMemcpyDeviceToHost, g->cstream));
        if (host_pred)
            TG_TRY_CUDA(cudaMemcpyAsync(host_pred + (size_t)rows[q] * n, g->qs.pred_stage[i] + (size_t)q * n, n * 4,
                                        cudaMemcpyDeviceToHost, g->cstream));
    }
    TG_TRY_CUDA(cudaEventRecord(g->ev_c[i], g->cstream));
    return TG_OK;
}

tg_status tg_sink_end(tg_graph *g) {
    if (g->cstream) TG_TRY_CUDA(cudaStreamSynchronize(g->cstream));
    return TG_OK;
}

void tg_sink_destroy(tg_graph *g) {
    if (!g->cstream) return;
    cudaStreamSynchronize(g->cstream);
    for (int i = 0; i < 2; i++) {
        cudaEventDestroy(g->ev_x[i]);
        cudaEventDestroy(g->ev_c[i]);
    }
    cudaStreamDestroy(g->cstream);
    g->cstream = nullptr;
}
