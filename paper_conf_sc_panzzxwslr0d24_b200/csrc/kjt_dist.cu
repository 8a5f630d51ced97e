// kjt_dist.cu -- table-wise input distribution (SURVEY §8e "Input distribution
// (the KJT all-to-all)", §8f NEXT #4; PAPER.md P:350 places whole tables on
// GPUs).  Rank j arrives with a data-parallel KJT (all F features, its Bl local
// samples); after the exchange rank r must hold all B = W*Bl samples of the
// features it owns, feature-major in global sample order -- the input of its
// recflex_forward.  The collective itself is the caller's (NCCL alltoallv);
// this file holds the two HBM-bound regrouping passes around it:
//
//   pack   : local KJT -> destination-major send buffers (lengths, IDs) and the
//            per-destination ID counts (the alltoallv split sizes);
//   unpack : source-major receive buffers -> the owned features' KJT (offsets
//            by a segmented scan, IDs by contiguous (source, feature) segment
//            copies).
//
// Both passes are one small scan kernel (1 CTA: per-segment lengths and their
// exclusive scans, F or W*F_r entries) plus one persistent copy kernel whose
// CTAs stride over fixed-size chunks of the segment list, so a feature with
// 40x the average IDs is spread over many SMs (load balance independent of
// the heterogeneity that motivates RecFlex).  No host round trip, no
// allocation per call; graph-capturable.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "plan_internal.h"

namespace recflex {
namespace {

constexpr int kScanThreads = 1024;
constexpr int kCopyThreads = 256;
constexpr int kChunk = 4096;  // IDs per copy chunk (16 per thread)

// Block-wide exclusive scan of one int64 value per thread; returns the
// exclusive prefix and writes the block total to *total.
__device__ int64_t block_exclusive_scan(int64_t v, int64_t *total) {
    __shared__ int64_t warp_sums[32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    int64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int64_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[warp] = x;
    __syncthreads();
    if (warp == 0) {
        int64_t w = lane < nw ? warp_sums[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t y = __shfl_up_sync(0xffffffffu, w, o);
            if (lane >= o) w += y;
        }
        warp_sums[lane] = w;  // inclusive warp prefix
    }
    __syncthreads();
    const int64_t before = (warp > 0 ? warp_sums[warp - 1] : 0) + x - v;
    *total = warp_sums[nw - 1];
    __syncthreads();  // warp_sums reused by the next call
    return before;
}

// Segment list shared by both passes: segment i copies len[i] IDs from
// src + a[i] to dst + b[i]; chunk_pfx[i] = first chunk of segment i.
struct Segs {
    const int64_t *a, *b, *len, *chunk_pfx;
    int n;
};

// Chunk c -> its segment by binary search over chunk_pfx[0..n].
__device__ __forceinline__ int seg_of_chunk(const int64_t *pfx, int n, int64_t c) {
    int lo = 0, hi = n;  // pfx[lo] <= c < pfx[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (__ldg(pfx + mid) <= c) lo = mid; else hi = mid;
    }
    return lo;
}

__device__ void copy_chunks(Segs s, const int32_t *__restrict__ src, int32_t *__restrict__ dst) {
    const int64_t nchunks = s.chunk_pfx[s.n];
    for (int64_t c = blockIdx.x; c < nchunks; c += gridDim.x) {
        const int i = seg_of_chunk(s.chunk_pfx, s.n, c);
        const int64_t off = (c - s.chunk_pfx[i]) * kChunk;
        const int64_t n = min((int64_t)kChunk, s.len[i] - off);
        const int32_t *p = src + s.a[i] + off;
        int32_t *q = dst + s.b[i] + off;
        constexpr int kPer = kChunk / kCopyThreads;
        int32_t v[kPer];
#pragma unroll
        for (int u = 0; u < kPer; ++u) {
            const int64_t e = (int64_t)u * kCopyThreads + threadIdx.x;
            if (e < n) v[u] = __ldcs(p + e);  // streamed once
        }
#pragma unroll
        for (int u = 0; u < kPer; ++u) {
            const int64_t e = (int64_t)u * kCopyThreads + threadIdx.x;
            if (e < n) q[e] = v[u];
        }
    }
}

// ---- pack ------------------------------------------------------------------

// One CTA.  Segment k = send_order[k] (features grouped by owner): its IDs are
// the contiguous local range [off[f*Bl], off[(f+1)*Bl]); destination offset =
// exclusive scan in send order.  dest_counts[r] = IDs sent to rank r.
__global__ void __launch_bounds__(kScanThreads) kjt_pack_scan_kernel(
    const int32_t *__restrict__ offsets, int Bl, int F, const int32_t *__restrict__ send_order,
    const int32_t *__restrict__ dest_first, int W, int64_t *seg_a, int64_t *seg_b, int64_t *seg_len,
    int64_t *chunk_pfx, int32_t *dest_counts) {
    int64_t carry_ids = 0, carry_chunks = 0;
    for (int base = 0; base < F; base += kScanThreads) {
        const int k = base + threadIdx.x;
        int64_t len = 0, a = 0;
        if (k < F) {
            const int f = send_order[k];
            a = offsets[(int64_t)f * Bl];
            len = (int64_t)offsets[(int64_t)(f + 1) * Bl] - a;
        }
        const int64_t ch = (len + kChunk - 1) / kChunk;
        int64_t tot_ids, tot_ch;
        const int64_t pos = block_exclusive_scan(len, &tot_ids);
        const int64_t cpos = block_exclusive_scan(ch, &tot_ch);
        if (k < F) {
            seg_a[k] = a;
            seg_b[k] = carry_ids + pos;
            seg_len[k] = len;
            chunk_pfx[k] = carry_chunks + cpos;
        }
        carry_ids += tot_ids;
        carry_chunks += tot_ch;
    }
    if (threadIdx.x == 0) chunk_pfx[F] = carry_chunks;
    __syncthreads();
    for (int r = threadIdx.x; r < W; r += blockDim.x) {
        const int k0 = dest_first[r], k1 = dest_first[r + 1];
        const int64_t end = k1 < F ? seg_b[k1] : carry_ids;
        dest_counts[r] = (int32_t)(k1 > k0 ? end - seg_b[k0] : 0);
    }
}

__global__ void __launch_bounds__(kCopyThreads) kjt_pack_copy_kernel(
    const int32_t *__restrict__ indices, const int32_t *__restrict__ offsets, int Bl, int F,
    const int32_t *__restrict__ send_order, Segs segs, int32_t *__restrict__ send_lengths,
    int32_t *__restrict__ send_indices) {
    // lengths, destination-major: send_lengths[k*Bl + s] = L(send_order[k], s)
    const int64_t nl = (int64_t)F * Bl;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nl; e += (int64_t)gridDim.x * blockDim.x) {
        const int k = (int)(e / Bl), s = (int)(e - (int64_t)k * Bl);
        const int64_t o = (int64_t)__ldg(send_order + k) * Bl + s;
        send_lengths[e] = __ldg(offsets + o + 1) - __ldg(offsets + o);
    }
    copy_chunks(segs, indices, send_indices);
}

// ---- unpack ------------------------------------------------------------------

// One CTA per received segment (j, k): its ID count.
__global__ void __launch_bounds__(kCopyThreads) kjt_unpack_reduce_kernel(const int32_t *__restrict__ recv_lengths,
                                                                         int Bl, int64_t *seg_len) {
    const int64_t base = (int64_t)blockIdx.x * Bl;
    int64_t v = 0;
    for (int s = threadIdx.x; s < Bl; s += blockDim.x) v += __ldg(recv_lengths + base + s);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    __shared__ int64_t ws[kCopyThreads / 32];
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
        int64_t t = 0;
        for (int w = 0; w < kCopyThreads / 32; ++w) t += ws[w];
        seg_len[blockIdx.x] = t;
    }
}

// One CTA.  Segment i = j*Fr + k (source-major, as received).  Source offset =
// exclusive scan in (j, k) order; destination offset = exclusive scan in
// (k, j) order (feature-major, then source rank = global sample block).
__global__ void __launch_bounds__(kScanThreads) kjt_unpack_scan_kernel(int W, int Fr, int B, int64_t *seg_a,
                                                                       int64_t *seg_b, const int64_t *seg_len,
                                                                       int64_t *chunk_pfx, int32_t *offsets_out) {
    const int n = W * Fr;
    int64_t carry = 0, carry_ch = 0, tot, tot_ch;
    for (int base = 0; base < n; base += kScanThreads) {  // source order
        const int i = base + threadIdx.x;
        const int64_t len = i < n ? seg_len[i] : 0;
        const int64_t ch = (len + kChunk - 1) / kChunk;
        const int64_t pos = block_exclusive_scan(len, &tot);
        const int64_t cpos = block_exclusive_scan(ch, &tot_ch);
        if (i < n) {
            seg_a[i] = carry + pos;
            chunk_pfx[i] = carry_ch + cpos;
        }
        carry += tot;
        carry_ch += tot_ch;
    }
    if (threadIdx.x == 0) {
        chunk_pfx[n] = carry_ch;
        offsets_out[(int64_t)Fr * B] = (int32_t)carry;
    }
    carry = 0;
    for (int base = 0; base < n; base += kScanThreads) {  // destination order q = k*W + j
        const int q = base + threadIdx.x;
        int i = 0;
        int64_t len = 0;
        if (q < n) {
            const int k = q / W, j = q - k * W;
            i = j * Fr + k;
            len = seg_len[i];
        }
        const int64_t pos = block_exclusive_scan(len, &tot);
        if (q < n) seg_b[i] = carry + pos;
        carry += tot;
    }
}

// Offsets: CTA-strided over segments (block scan of Bl lengths + the segment's
// destination start); then the ID chunks.
__global__ void __launch_bounds__(kCopyThreads) kjt_unpack_main_kernel(
    const int32_t *__restrict__ recv_lengths, const int32_t *__restrict__ recv_indices, int W, int Fr, int Bl,
    Segs segs, int32_t *__restrict__ indices_out, int32_t *__restrict__ offsets_out) {
    const int B = W * Bl;
    for (int i = blockIdx.x; i < segs.n; i += gridDim.x) {
        const int j = i / Fr, k = i - j * Fr;
        const int32_t *len = recv_lengths + (int64_t)i * Bl;
        int32_t *o = offsets_out + (int64_t)k * B + (int64_t)j * Bl;
        int64_t carry = segs.b[i];
        for (int base = 0; base < Bl; base += kCopyThreads) {
            const int s = base + threadIdx.x;
            const int64_t v = s < Bl ? __ldg(len + s) : 0;
            int64_t tot;
            const int64_t pos = block_exclusive_scan(v, &tot);
            if (s < Bl) o[s] = (int32_t)(carry + pos);
            carry += tot;
        }
    }
    copy_chunks(segs, recv_indices, indices_out);
}

int copy_grid(int device) {
    static int sms = 0;
    if (!sms && cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) sms = 148;
    return sms * 8;  // 8 CTAs of 256 threads per SM (2048 threads)
}

}  // namespace
}  // namespace recflex

using namespace recflex;

struct recflex_kjt_dist_s {
    int F = 0, W = 0, rank = 0, Bl = 0, device = 0, Fr = 0;
    std::vector<int32_t> owner, send_counts_len, recv_counts_len;
    int32_t *d_send_order = nullptr, *d_dest_first = nullptr;
    int64_t *d_seg = nullptr;  // 4 arrays of nseg(+1) int64: a, b, len, chunk_pfx
    int nseg_max = 0;
};

extern "C" {

recflex_status_t recflex_kjt_dist_create(int32_t F, const int32_t *feature_owner, int32_t W, int32_t rank,
                                         int32_t Bl, int32_t device, recflex_kjt_dist_t *out) {
    if (!out || !feature_owner || F <= 0 || W <= 0 || rank < 0 || rank >= W || Bl < 0) {
        set_last_error("recflex_kjt_dist_create: invalid argument");
        return RECFLEX_ERR_INVALID_ARG;
    }
    if ((int64_t)F * Bl >= (int64_t)1 << 31 || (int64_t)W * Bl >= (int64_t)1 << 31) {
        set_last_error("recflex_kjt_dist_create: F*Bl and W*Bl must be < 2^31 (int32 offsets, reading C4)");
        return RECFLEX_ERR_INVALID_ARG;
    }
    *out = nullptr;
    auto *h = new recflex_kjt_dist_s;
    h->F = F, h->W = W, h->rank = rank, h->Bl = Bl, h->device = device;
    h->owner.assign(feature_owner, feature_owner + F);
    std::vector<int32_t> order;
    std::vector<int32_t> first(W + 1, 0);
    for (int r = 0; r < W; ++r) {
        first[r] = (int32_t)order.size();
        for (int f = 0; f < F; ++f) {
            if (h->owner[f] < 0 || h->owner[f] >= W) {
                delete h;
                set_last_error("recflex_kjt_dist_create: feature_owner out of [0, W)");
                return RECFLEX_ERR_INVALID_ARG;
            }
            if (h->owner[f] == r) order.push_back(f);
        }
    }
    first[W] = F;
    h->Fr = first[rank + 1] - first[rank];
    h->send_counts_len.resize(W);
    h->recv_counts_len.assign(W, h->Fr * Bl);
    for (int r = 0; r < W; ++r) h->send_counts_len[r] = (first[r + 1] - first[r]) * Bl;
    h->nseg_max = std::max(F, W * h->Fr);
    cudaError_t e = cudaSetDevice(device);
    if (e == cudaSuccess) e = cudaMalloc(&h->d_send_order, sizeof(int32_t) * (F + W + 1));
    if (e == cudaSuccess) e = cudaMalloc(&h->d_seg, sizeof(int64_t) * 4 * (h->nseg_max + 1));
    if (e == cudaSuccess) {
        h->d_dest_first = h->d_send_order + F;
        e = cudaMemcpy(h->d_send_order, order.data(), sizeof(int32_t) * F, cudaMemcpyHostToDevice);
    }
    if (e == cudaSuccess)
        e = cudaMemcpy(h->d_dest_first, first.data(), sizeof(int32_t) * (W + 1), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
        recflex_kjt_dist_destroy(h);
        return cuda_status_at(e, "recflex_kjt_dist_create");
    }
    *out = h;
    return RECFLEX_OK;
}

void recflex_kjt_dist_destroy(recflex_kjt_dist_t h) {
    if (!h) return;
    if (h->d_send_order) cudaFree(h->d_send_order);
    if (h->d_seg) cudaFree(h->d_seg);
    delete h;
}

recflex_status_t recflex_kjt_dist_sizes(recflex_kjt_dist_t h, int32_t *send_length_counts,
                                        int32_t *recv_length_counts, int32_t *num_owned) {
    if (!h) return RECFLEX_ERR_INVALID_ARG;
    for (int r = 0; r < h->W; ++r) {
        if (send_length_counts) send_length_counts[r] = h->send_counts_len[r];
        if (recv_length_counts) recv_length_counts[r] = h->recv_counts_len[r];
    }
    if (num_owned) *num_owned = h->Fr;
    return RECFLEX_OK;
}

recflex_status_t recflex_kjt_pack(recflex_kjt_dist_t h, const int32_t *indices, const int32_t *offsets,
                                  int32_t *send_lengths, int32_t *send_indices, int32_t *dest_counts,
                                  void *stream_) {
    if (!h || !offsets || !dest_counts || (h->Bl > 0 && !send_lengths)) {
        set_last_error("recflex_kjt_pack: invalid argument");
        return RECFLEX_ERR_INVALID_ARG;
    }
    cudaStream_t stream = (cudaStream_t)stream_;
    const int n = h->F;
    int64_t *a = h->d_seg, *b = a + (n + 1), *len = b + (n + 1), *pfx = len + (n + 1);
    kjt_pack_scan_kernel<<<1, kScanThreads, 0, stream>>>(offsets, h->Bl, h->F, h->d_send_order, h->d_dest_first,
                                                         h->W, a, b, len, pfx, dest_counts);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_status_at(e, "kjt pack scan launch");
    Segs s{a, b, len, pfx, n};
    kjt_pack_copy_kernel<<<copy_grid(h->device), kCopyThreads, 0, stream>>>(indices, offsets, h->Bl, h->F,
                                                                            h->d_send_order, s, send_lengths,
                                                                            send_indices);
    return cuda_status_at(cudaGetLastError(), "kjt pack copy launch");
}

recflex_status_t recflex_kjt_unpack(recflex_kjt_dist_t h, const int32_t *recv_lengths, const int32_t *recv_indices,
                                    int32_t *indices_out, int32_t *offsets_out, void *stream_) {
    if (!h || !offsets_out || (h->Fr > 0 && h->Bl > 0 && !recv_lengths)) {
        set_last_error("recflex_kjt_unpack: invalid argument");
        return RECFLEX_ERR_INVALID_ARG;
    }
    cudaStream_t stream = (cudaStream_t)stream_;
    const int n = h->W * h->Fr;
    int64_t *a = h->d_seg, *b = a + (n + 1), *len = b + (n + 1), *pfx = len + (n + 1);
    if (n > 0) {
        if (h->Bl > 0) {
            kjt_unpack_reduce_kernel<<<n, kCopyThreads, 0, stream>>>(recv_lengths, h->Bl, len);
        } else {
            cudaError_t e = cudaMemsetAsync(len, 0, sizeof(int64_t) * n, stream);
            if (e != cudaSuccess) return cuda_status_at(e, "kjt unpack memset");
        }
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_status_at(e, "kjt unpack reduce launch");
    }
    kjt_unpack_scan_kernel<<<1, kScanThreads, 0, stream>>>(h->W, h->Fr, h->W * h->Bl, a, b, len, pfx, offsets_out);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_status_at(e, "kjt unpack scan launch");
    if (n == 0) return RECFLEX_OK;
    Segs s{a, b, len, pfx, n};
    kjt_unpack_main_kernel<<<copy_grid(h->device), kCopyThreads, 0, stream>>>(recv_lengths, recv_indices, h->W, h->Fr,
                                                                              h->Bl, s, indices_out, offsets_out);
    return cuda_status_at(cudaGetLastError(), "kjt unpack main launch");
}

}  // extern "C"
