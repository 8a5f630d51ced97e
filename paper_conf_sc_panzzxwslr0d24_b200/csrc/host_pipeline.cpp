// host_pipeline.cpp -- recflex_forward_host_batches: the end-to-end serving
// loop over host-resident batches.  Three streams overlap the three stages of
// consecutive batches -- H2D of batch i+1's KJT, the forward of batch i, D2H of
// batch i-1's pooled output -- through two staging slots on the device, so a
// step costs max(H2D, forward, D2H) instead of their sum (the PCIe directions
// are independent copy engines).  Same results as recflex_forward_host per batch.
#include <cuda_runtime.h>

#include <algorithm>

#include "plan_internal.h"

using namespace recflex;

struct HostPipe {
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev_h2d[2] = {}, ev_comp[2] = {}, ev_d2h[2] = {};
    int32_t *idx[2] = {}, *off[2] = {};
    float *out[2] = {};
    int64_t idx_cap[2] = {}, off_cap[2] = {}, out_cap[2] = {};
};

namespace recflex {
void host_pipe_free(recflex_plan_s *p) {
    HostPipe *h = p->pipe;
    if (!h) return;
    for (int s = 0; s < 2; ++s) {
        cudaFree(h->idx[s]);
        cudaFree(h->off[s]);
        cudaFree(h->out[s]);
        if (h->ev_h2d[s]) cudaEventDestroy(h->ev_h2d[s]);
        if (h->ev_comp[s]) cudaEventDestroy(h->ev_comp[s]);
        if (h->ev_d2h[s]) cudaEventDestroy(h->ev_d2h[s]);
    }
    if (h->h2d) cudaStreamDestroy(h->h2d);
    if (h->d2h) cudaStreamDestroy(h->d2h);
    delete h;
    p->pipe = nullptr;
}
}  // namespace recflex

template <typename T>
static cudaError_t ensure(T *&ptr, int64_t &cap, int64_t n) {
    if (n <= cap && ptr) return cudaSuccess;
    cudaFree(ptr);
    ptr = nullptr;
    cap = 0;
    cudaError_t e = cudaMalloc(&ptr, sizeof(T) * std::max<int64_t>(n, 1));
    if (e == cudaSuccess) cap = std::max<int64_t>(n, 1);
    return e;
}

extern "C" recflex_status_t recflex_forward_host_batches(recflex_plan_t p, int32_t num_batches,
                                                         const int32_t *const *h_indices, const int64_t *nnz,
                                                         const int32_t *const *h_offsets, const int32_t *batch_sizes,
                                                         const void *const *tables, float *const *h_out,
                                                         void *stream_) {
    if (!p || num_batches < 0 || !tables || (num_batches > 0 && (!h_indices || !nnz || !h_offsets || !batch_sizes ||
                                                                 !h_out)))
        return RECFLEX_ERR_INVALID_ARG;
    for (int i = 0; i < num_batches; ++i) {
        const int B = batch_sizes[i];
        if (B < 0 || B > p->max_batch || nnz[i] < 0 || (B > 0 && (!h_offsets[i] || !h_out[i])) ||
            (nnz[i] > 0 && !h_indices[i]))
            return RECFLEX_ERR_INVALID_ARG;
    }
    if (num_batches == 0) return RECFLEX_OK;
    cudaStream_t stream = (cudaStream_t)stream_;
    cudaError_t e = cudaSetDevice(p->device);
    if (e != cudaSuccess) return cuda_status(e);
    if (!p->pipe) {
        HostPipe *h = new HostPipe;
        p->pipe = h;
        e = cudaStreamCreateWithFlags(&h->h2d, cudaStreamNonBlocking);
        if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->d2h, cudaStreamNonBlocking);
        for (int s = 0; s < 2 && e == cudaSuccess; ++s) {
            e = cudaEventCreateWithFlags(&h->ev_h2d[s], cudaEventDisableTiming);
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_comp[s], cudaEventDisableTiming);
            if (e == cudaSuccess) e = cudaEventCreateWithFlags(&h->ev_d2h[s], cudaEventDisableTiming);
        }
        if (e != cudaSuccess) {
            host_pipe_free(p);
            return cuda_status_at(e, "recflex_forward_host_batches: streams/events");
        }
    }
    HostPipe *h = p->pipe;
    // the previous call's copies may still be in flight on the pipe streams
    e = cudaStreamSynchronize(h->d2h);
    if (e == cudaSuccess) e = cudaStreamSynchronize(h->h2d);
    if (e != cudaSuccess) return cuda_status(e);
    for (int i = 0; i < num_batches; ++i) {
        const int s = i & 1;
        const int B = batch_sizes[i];
        if (B == 0) continue;
        const int64_t n_off = (int64_t)p->F * B + 1, n_out = (int64_t)B * p->d_tot;
        // slot s is free once batch i-2's forward has read its inputs and its
        // D2H has drained its output (buffer growth must not race them)
        if (i >= 2 && (nnz[i] > h->idx_cap[s] || n_off > h->off_cap[s] || n_out > h->out_cap[s])) {
            e = cudaEventSynchronize(h->ev_d2h[s]);
            if (e != cudaSuccess) return cuda_status(e);
        }
        e = ensure(h->idx[s], h->idx_cap[s], nnz[i]);
        if (e == cudaSuccess) e = ensure(h->off[s], h->off_cap[s], n_off);
        if (e == cudaSuccess) e = ensure(h->out[s], h->out_cap[s], n_out);
        if (e != cudaSuccess) return cuda_status_at(e, "recflex_forward_host_batches: staging");
        if (i >= 2) e = cudaStreamWaitEvent(h->h2d, h->ev_comp[s], 0);
        if (e == cudaSuccess && nnz[i] > 0)
            e = cudaMemcpyAsync(h->idx[s], h_indices[i], sizeof(int32_t) * nnz[i], cudaMemcpyHostToDevice, h->h2d);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(h->off[s], h_offsets[i], sizeof(int32_t) * n_off, cudaMemcpyHostToDevice, h->h2d);
        if (e == cudaSuccess) e = cudaEventRecord(h->ev_h2d[s], h->h2d);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(stream, h->ev_h2d[s], 0);
        if (e == cudaSuccess && i >= 2) e = cudaStreamWaitEvent(stream, h->ev_d2h[s], 0);
        if (e != cudaSuccess) return cuda_status(e);
        recflex_status_t st = recflex_forward(p, h->idx[s], h->off[s], B, tables, h->out[s], stream);
        if (st != RECFLEX_OK) return st;
        e = cudaEventRecord(h->ev_comp[s], stream);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(h->d2h, h->ev_comp[s], 0);
        if (e == cudaSuccess)
            e = cudaMemcpyAsync(h_out[i], h->out[s], sizeof(float) * n_out, cudaMemcpyDeviceToHost, h->d2h);
        if (e == cudaSuccess) e = cudaEventRecord(h->ev_d2h[s], h->d2h);
        if (e != cudaSuccess) return cuda_status(e);
    }
    e = cudaStreamSynchronize(h->d2h);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    return cuda_status(e);
}
