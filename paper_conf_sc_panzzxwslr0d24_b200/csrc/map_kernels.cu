// map_kernels.cu -- runtime thread mapping on the device (Fig. 8
// d_task_map / d_blocks_map) plus small helper kernels.
//
// The paper computes the map on the host ("host-side workload analysis",
// P:170); here one CTA reads the batch's offsets and scans, so the forward has
// no host round trip (reading C13).  Same integers as the oracle's formula:
//   part 0 (sample-partitioned): need_f = ceil(B / per_block)
//   part 1 (lookup-partitioned): npb = max(per_block, ceil(nnz_f/(slots-2)))
//                                need_f = floor(nnz_f / npb) + 1
//   feature_blocks = need_f, or nalloc_f under a static mapping
//   cap > 0: feature_blocks = min(feature_blocks, cap)
//   block_start = exclusive scan of feature_blocks in feature order.
#include <cuda_runtime.h>

#include <algorithm>

#include "recflex_internal.h"

namespace recflex {

int fused_launch_k1(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k2(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k3(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k4(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k5(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k6(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k7(const FusedArgs &, const LaunchCfg &, void *);
int fused_launch_k8(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k1(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k2(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k3(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k4(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k5(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k6(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k7(const FusedArgs &, const LaunchCfg &, void *);
int backward_launch_k8(const FusedArgs &, const LaunchCfg &, void *);
int fused_prepare_k1(int, int);
int fused_prepare_k2(int, int);
int fused_prepare_k3(int, int);
int fused_prepare_k4(int, int);
int fused_prepare_k5(int, int);
int fused_prepare_k6(int, int);
int fused_prepare_k7(int, int);
int fused_prepare_k8(int, int);
int fused_occupancy_k1(int, int *, int *, int *);
int fused_occupancy_k2(int, int *, int *, int *);
int fused_occupancy_k3(int, int *, int *, int *);
int fused_occupancy_k4(int, int *, int *, int *);
int fused_occupancy_k5(int, int *, int *, int *);
int fused_occupancy_k6(int, int *, int *, int *);
int fused_occupancy_k7(int, int *, int *, int *);
int fused_occupancy_k8(int, int *, int *, int *);

int fused_launch(int k, const FusedArgs &a, const LaunchCfg &cfg, void *stream) {
    switch (k) {
        case 1: return fused_launch_k1(a, cfg, stream);
        case 2: return fused_launch_k2(a, cfg, stream);
        case 3: return fused_launch_k3(a, cfg, stream);
        case 4: return fused_launch_k4(a, cfg, stream);
        case 5: return fused_launch_k5(a, cfg, stream);
        case 6: return fused_launch_k6(a, cfg, stream);
        case 7: return fused_launch_k7(a, cfg, stream);
        case 8: return fused_launch_k8(a, cfg, stream);
        default: return (int)cudaErrorInvalidValue;
    }
}

int backward_launch(int k, const FusedArgs &a, const LaunchCfg &cfg, void *stream) {
    switch (k) {
        case 1: return backward_launch_k1(a, cfg, stream);
        case 2: return backward_launch_k2(a, cfg, stream);
        case 3: return backward_launch_k3(a, cfg, stream);
        case 4: return backward_launch_k4(a, cfg, stream);
        case 5: return backward_launch_k5(a, cfg, stream);
        case 6: return backward_launch_k6(a, cfg, stream);
        case 7: return backward_launch_k7(a, cfg, stream);
        case 8: return backward_launch_k8(a, cfg, stream);
        default: return (int)cudaErrorInvalidValue;
    }
}

int fused_prepare(int k, int device, int smem, int carveout) {
    cudaError_t e = cudaSetDevice(device);
    if (e != cudaSuccess) return (int)e;
    switch (k) {
        case 1: return fused_prepare_k1(smem, carveout);
        case 2: return fused_prepare_k2(smem, carveout);
        case 3: return fused_prepare_k3(smem, carveout);
        case 4: return fused_prepare_k4(smem, carveout);
        case 5: return fused_prepare_k5(smem, carveout);
        case 6: return fused_prepare_k6(smem, carveout);
        case 7: return fused_prepare_k7(smem, carveout);
        case 8: return fused_prepare_k8(smem, carveout);
        default: return (int)cudaErrorInvalidValue;
    }
}

int fused_occupancy(int k, int smem, int *blocks, int *regs, int *spill) {
    switch (k) {
        case 1: return fused_occupancy_k1(smem, blocks, regs, spill);
        case 2: return fused_occupancy_k2(smem, blocks, regs, spill);
        case 3: return fused_occupancy_k3(smem, blocks, regs, spill);
        case 4: return fused_occupancy_k4(smem, blocks, regs, spill);
        case 5: return fused_occupancy_k5(smem, blocks, regs, spill);
        case 6: return fused_occupancy_k6(smem, blocks, regs, spill);
        case 7: return fused_occupancy_k7(smem, blocks, regs, spill);
        case 8: return fused_occupancy_k8(smem, blocks, regs, spill);
        default: return (int)cudaErrorInvalidValue;
    }
}

// ---------------------------------------------------------------------------
// Map kernel: one CTA of 1024 threads, features in chunks of 1024 with a carry.
// ---------------------------------------------------------------------------
constexpr int kMapThreads = 1024;

__global__ void __launch_bounds__(kMapThreads) recflex_map_kernel(MapArgs a) {
    __shared__ int warp_tot[kMapThreads / 32];
    __shared__ int s_carry;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        s_carry = 0;
        *a.counter = 0;  // the fused kernel's task counter
    }
    __syncthreads();
    for (int base = 0; base < a.F; base += kMapThreads) {
        const int f = base + tid;
        int blocks = 0;
        if (f < a.F && a.B > 0) {
            const FeatureDesc &fd = a.desc[f];
            if (fd.part == 0) {
                blocks = (a.B + fd.per_block - 1) / fd.per_block;
            } else {
                const int64_t fi = fd.in_feature;
                const int nnz = a.offsets[(fi + 1) * a.B] - a.offsets[fi * a.B];
                int npb = fd.per_block;
                const int room = fd.slots - 2;  // slots hold blocks+1 entries (sentinel)
                const int need = (nnz + room - 1) / room;
                if (need > npb) npb = need;
                a.npb_eff[f] = npb;
                blocks = nnz / npb + 1;
            }
            a.need[f] = blocks;
            // static thread mapping: a fixed number of allocated
            // tasks whatever the batch; they fold the needed ones (fused kernel)
            if (fd.nalloc > 0) blocks = fd.nalloc;
            if (fd.cap > 0 && blocks > fd.cap) blocks = fd.cap;
        }
        // block-wide exclusive scan
        int incl = blocks;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int v = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += v;
        }
        if (lane == 31) warp_tot[warp] = incl;
        __syncthreads();
        if (warp == 0) {
            int w = warp_tot[lane];
            int wi = w;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int v = __shfl_up_sync(0xffffffffu, wi, o);
                if (lane >= o) wi += v;
            }
            warp_tot[lane] = wi - w;  // exclusive warp prefix
        }
        __syncthreads();
        const int excl = s_carry + warp_tot[warp] + incl - blocks;
        if (f < a.F) a.block_start[f] = excl;
        __syncthreads();
        if (tid == kMapThreads - 1) s_carry = excl + blocks;
        __syncthreads();
    }
    if (tid == 0) a.block_start[a.F] = s_carry;
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

int map_launch(const MapArgs &a, void *stream) {
    recflex_map_kernel<<<1, kMapThreads, 0, (cudaStream_t)stream>>>(a);
    return (int)cudaGetLastError();
}

// ---------------------------------------------------------------------------
// Fill kernel (only for lookup-partitioned features): task_start[q] = first
// sample whose bag starts in lookup window q (Fig. 8's d_task_map payload for
// adaptive tasks).  CTA (chunk, k): part-1 feature k, samples [chunk * kFillSpan,
// +kFillSpan), kFillPer per thread with independent coalesced offset loads (one
// wave instead of a thread per sample -- the per-sample form was a chain of
// dependent loads repeated over ~10 waves: 29 us on sharded1000).  Disjoint writes.
// ---------------------------------------------------------------------------
constexpr int kFillPer = 16;
constexpr int kFillSpan = 256 * kFillPer;

__global__ void __launch_bounds__(256) recflex_fill_kernel(FillArgs a) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const int f = a.part1_features[blockIdx.y];
    const FeatureDesc &fd = a.desc[f];
    const int32_t *offs = a.offsets + (size_t)fd.in_feature * a.B;
    const int base = offs[0];
    const int npb = a.npb_eff[f];
    const int blocks = a.need[f];  // needed tasks (a static feature allocates a different count)
    int32_t *ts = a.task_start + fd.slot_base;
    const int s0 = blockIdx.x * kFillSpan + threadIdx.x;
    int cur[kFillPer], prev[kFillPer];
#pragma unroll
    for (int i = 0; i < kFillPer; ++i) {
        const int s = s0 + i * 256;
        cur[i] = s < a.B ? offs[s] : 0;
        prev[i] = (s < a.B && s > 0) ? offs[s - 1] : base;
    }
#pragma unroll
    for (int i = 0; i < kFillPer; ++i) {
        const int s = s0 + i * 256;
        if (s >= a.B) break;
        const int q_hi = (cur[i] - base) / npb;
        const int q_lo = (s == 0) ? -1 : (prev[i] - base) / npb;
        for (int q = q_lo + 1; q <= q_hi && q <= blocks; ++q) ts[q] = s;
        if (s == a.B - 1)
            for (int q = q_hi + 1; q <= blocks; ++q) ts[q] = a.B;
    }
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

int fill_launch(const FillArgs &a, int B, bool pdl, void *stream) {
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3((B + kFillSpan - 1) / kFillSpan, a.num_part1);
    lc.blockDim = dim3(256);
    lc.stream = (cudaStream_t)stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = pdl ? 1 : 0;
    lc.attrs = attr;
    lc.numAttrs = 1;
    return (int)cudaLaunchKernelEx(&lc, recflex_fill_kernel, a);
}

// ---------------------------------------------------------------------------
// Validation: flag bit 1 = bad offsets, bit 2 = index out of range.
// ---------------------------------------------------------------------------
__global__ void recflex_validate_kernel(const FeatureDesc *desc, int F, int in_F, const int32_t *indices,
                                        const int32_t *offsets, int B, int32_t *flag) {
    const int64_t n_off = (int64_t)in_F * B;
    const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    if (blockIdx.y == 0) {
        for (int64_t k = gtid; k < n_off; k += stride)
            if (offsets[k + 1] < offsets[k]) atomicOr(flag, 1);
        if (gtid == 0 && offsets[0] != 0) atomicOr(flag, 1);
        return;
    }
    const int f = blockIdx.y - 1;
    if (f >= F) return;
    const FeatureDesc &fd = desc[f];
    const int64_t a = offsets[(int64_t)fd.in_feature * B], b = offsets[(int64_t)(fd.in_feature + 1) * B];
    for (int64_t j = a + gtid; j < b; j += stride) {
        const int v = indices[j];
        if (v < 0 || (int64_t)v >= fd.rows) atomicOr(flag, 2);
    }
}

int validate_launch(const FeatureDesc *desc, int F, int in_F, const int32_t *indices, const int32_t *offsets, int B,
                    int32_t *flag, void *stream) {
    dim3 grid(64, F + 1);
    recflex_validate_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(desc, F, in_F, indices, offsets, B, flag);
    return (int)cudaGetLastError();
}

// dst[i] = (src[i] + shift) mod rows  -- the tuner's duplicated input (reading C17)
__global__ void recflex_remap_kernel(const int32_t *src, int32_t *dst, int64_t n, int64_t shift, int64_t rows) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        dst[i] = (int32_t)(((int64_t)src[i] + shift) % rows);
}

int remap_launch(const int32_t *src, int32_t *dst, int64_t n, int64_t shift, int64_t rows, void *stream) {
    if (n <= 0) return 0;
    int grid = (int)((n + 255) / 256);
    if (grid > 4096) grid = 4096;
    recflex_remap_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>(src, dst, n, shift, rows);
    return (int)cudaGetLastError();
}

// Relayout after the pooled-output all-to-all: received chunk i is rank i's
// [rows][dims[i]] block (chunks contiguous in rank order); it goes to columns
// [cols[i], cols[i] + dims[i]) of out [rows][d_tot].  blockIdx.y = chunk (no
// per-element rank search); 16-byte copies when the chunk and the layout are
// 4-float aligned (every config), else scalar.  Dims travel by value.
__global__ void __launch_bounds__(256) recflex_concat_kernel(const float *__restrict__ recv, float *__restrict__ out,
                                                             ConcatArgs a) {
    const int i = blockIdx.y;
    const int d = a.dims[i];
    const int64_t n = (int64_t)a.rows * d;
    const float *src = recv + (int64_t)a.rows * a.cols[i];
    float *dst = out + a.cols[i];
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (((d | a.cols[i] | a.d_tot) & 3) == 0) {
        const int d4 = d >> 2;
        const int64_t n4 = n >> 2;
        for (int64_t e = t0; e < n4; e += stride) {
            const int64_t r = e / d4;
            const int c = (int)(e - r * d4);
            const float4 v = __ldg(reinterpret_cast<const float4 *>(src) + e);
            *reinterpret_cast<float4 *>(dst + r * a.d_tot + 4 * c) = v;
        }
    } else {
        for (int64_t e = t0; e < n; e += stride) {
            const int64_t r = e / d;
            const int c = (int)(e - r * d);
            dst[r * a.d_tot + c] = src[e];
        }
    }
}

int concat_launch(const float *recv, const ConcatArgs &a, float *out, void *stream) {
    if (a.W <= 0 || a.rows <= 0 || a.d_tot <= 0) return 0;
    int64_t max_n = 0;
    for (int i = 0; i < a.W; ++i) max_n = std::max<int64_t>(max_n, (int64_t)a.rows * a.dims[i]);
    int gx = (int)std::min<int64_t>((max_n / 4 + 255) / 256, 148 * 8 / std::max(1, a.W) + 1);
    gx = std::max(gx, 1);
    recflex_concat_kernel<<<dim3(gx, a.W), 256, 0, (cudaStream_t)stream>>>(recv, out, a);
    return (int)cudaGetLastError();
}

// Exchange completion (recflex_forward_exchange), one warp launched right
// after the fused kernel on the same stream: stream order puts every pooled
// row the fused kernel stored (into local, NVLink-peer or IPC-mapped buffers)
// before this kernel; lane 0 bumps the epoch, fences at system scope and
// publishes it into every destination's flag array (slot `rank`) with a
// system-scope release; then lane j spins until writer j has published this
// step (acquire at system scope), so work ordered after this kernel sees every
// peer's rows.  A writer that never arrives (a dead peer) traps after ~60 s.
// (The signal lives in its own kernel, not in the fused kernel's epilogue: a
// CTA barrier after the fused kernel's task loop changed how the compiler
// reconverged the warp-decoupled loop and deadlocked warps on B200.)
__global__ void recflex_route_signal_wait_kernel(uint32_t *const *flags, const uint32_t *local, int32_t *epoch,
                                                 int rank, int world) {
    __shared__ unsigned s_target;
    const int j = threadIdx.x;
    if (j == 0) {
        const unsigned e = (unsigned)*reinterpret_cast<volatile int32_t *>(epoch) + 1u;
        *reinterpret_cast<volatile int32_t *>(epoch) = (int32_t)e;
        __threadfence_system();
        for (int r = 0; r < world; ++r)
            asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flags[r] + rank), "r"(e) : "memory");
        s_target = e;
    }
    __syncthreads();
    if (j >= world) return;
    const unsigned target = s_target;
    unsigned long long t0 = 0, now;
    while (true) {
        unsigned v;
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(local + j) : "memory");
        if ((int)(v - target) >= 0) break;
        __nanosleep(200);
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
        if (t0 == 0) t0 = now;
        else if (now - t0 > 60ull * 1000000000ull) asm volatile("trap;");
    }
}

int route_signal_wait_launch(uint32_t *const *flags, const uint32_t *local_flags, int32_t *epoch, int rank, int world,
                             void *stream) {
    recflex_route_signal_wait_kernel<<<1, 32 * ((world + 31) / 32), 0, (cudaStream_t)stream>>>(flags, local_flags,
                                                                                              epoch, rank, world);
    return (int)cudaGetLastError();
}

__global__ void recflex_flush_kernel(float4 *buf, int64_t n4, float v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x)
        buf[i] = make_float4(v, v, v, v);
}

int flush_launch(void *buf, size_t bytes, void *stream) {
    const int64_t n4 = (int64_t)(bytes / 16);
    if (n4 == 0) return 0;
    recflex_flush_kernel<<<148 * 8, 256, 0, (cudaStream_t)stream>>>((float4 *)buf, n4, 0.f);
    return (int)cudaGetLastError();
}

}  // namespace recflex
