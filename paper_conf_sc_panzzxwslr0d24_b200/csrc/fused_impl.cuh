// fused_impl.cuh -- the fused heterogeneous-schedule kernel (Fig. 8),
// B200 form: persistent CTAs (#SM x k) pull tasks from a device counter, so the
// grid never depends on host-side knowledge of the batch (the device-side map
// kernel produced block_start); launched with PDL behind the map kernel.
//
// Per task t (the paper's blockIdx.x):
//   feature_idx = the f with block_start[f] <= t < block_start[f+1]
//                 (d_task_map[t].x, Fig. 8 line 9)
//   rel_bidx    = t - block_start[f]                        (d_task_map[t].y)
//   feature_blocks = block_start[f+1] - block_start[f]      (d_blocks_map[f])
//   schedule_id = desc[f].sched                             (schedule_map[f])
//   if-else dispatch to the inlined schedule (no function pointers).
// Shared memory is one union for all schedules (Fig. 8 lines 12-15): the
// BLOCK-family reduction scratch plus the block_start cache, inside the
// dynamic allocation that also pads the CTA to exactly k per SM.
#pragma once
#include "schedules.cuh"

namespace recflex {

template <int I>
__device__ __forceinline__ void dispatch_schedule(int id, const TaskCtx &x, float *red) {
    if constexpr (I < kCatalogSize) {
        if (id == I) {
            constexpr CatalogEntry e = kCatalog[I];
            if constexpr (e.family == RECFLEX_FAMILY_GROUP)
                sched_group<e.G, e.VEC, e.C, e.U>(x.table, x.offs, x.idx, x.out, x.dim, x.pool, x.out_stride, x.s0, x.s1);
            else
                sched_block<e.G, e.VEC, e.C, e.U>(x.table, x.offs, x.idx, x.out, x.dim, x.pool, x.out_stride, x.s0,
                                                  x.s1, red);
        } else {
            dispatch_schedule<I + 1>(id, x, red);
        }
    }
}

constexpr int kRedFloats = 8 * 256;  // BLOCK family: [8 warps][SPAN <= 256]

template <int KOCC>
__global__ void __launch_bounds__(kBlockThreads, KOCC) recflex_fused_kernel(FusedArgs a) {
    extern __shared__ __align__(16) unsigned char dyn_smem[];
    __shared__ int s_task[2];
    float *red = reinterpret_cast<float *>(dyn_smem);                       // union member 1
    int *bs_s = reinterpret_cast<int *>(dyn_smem + kRedFloats * sizeof(float));  // union member 2
    const int tid = threadIdx.x;
    const int F = a.F;
    const bool bs_in_smem = (F + 1) <= kSmemBlockStartCap;

    // PDL: everything above overlapped the map kernel; wait for its results.
    asm volatile("griddepcontrol.wait;" ::: "memory");

    const int total = a.block_start[F];
    if (bs_in_smem)
        for (int i = tid; i <= F; i += kBlockThreads) bs_s[i] = a.block_start[i];
    const int *bs = bs_in_smem ? bs_s : a.block_start;
    if (tid == 0) s_task[0] = atomicAdd(a.counter, 1);
    __syncthreads();

    int buf = 0;
    while (true) {
        const int t = s_task[buf];
        if (t >= total) break;
        long long t0 = 0;
        if (tid == 0) {
            s_task[buf ^ 1] = atomicAdd(a.counter, 1);  // prefetch the next task id
            if (a.timers) t0 = clock64();
        }
        // feature_idx: upper_bound(block_start, t) - 1
        int lo = 0, hi = F;
        while (hi - lo > 1) {
            const int mid = (lo + hi) >> 1;
            if (bs[mid] <= t) lo = mid;
            else hi = mid;
        }
        const int f = lo;
        const int rel = t - bs[f];
        const FeatureDesc fd = a.desc[f];
        int s0, s1;
        if (fd.part == 0) {
            s0 = rel * fd.per_block;
            s1 = min(a.B, s0 + fd.per_block);
        } else {
            const int32_t *ts = a.task_start + fd.slot_base;
            s0 = ts[rel];
            s1 = ts[rel + 1];
        }
        TaskCtx x;
        x.table = fd.table;
        x.offs = a.offsets + (size_t)fd.in_feature * a.B;
        x.idx = a.indices;
        x.out = a.out + fd.col;
        x.dim = fd.dim;
        x.pool = fd.pool;
        x.out_stride = a.out_stride;
        x.s0 = s0;
        x.s1 = s1;
        dispatch_schedule<0>(fd.sched, x, red);
        __syncthreads();
        if (tid == 0 && a.timers && t < a.timers_cap) a.timers[t] = clock64() - t0;
        buf ^= 1;
    }
}

template <int KOCC>
int fused_launch_impl(const FusedArgs &a, const LaunchCfg &cfg, void *stream) {
    cudaLaunchConfig_t lc = {};
    lc.gridDim = dim3(cfg.grid);
    lc.blockDim = dim3(kBlockThreads);
    lc.dynamicSmemBytes = cfg.smem;
    lc.stream = (cudaStream_t)stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = cfg.pdl ? 1 : 0;
    lc.attrs = attr;
    lc.numAttrs = 1;
    return (int)cudaLaunchKernelEx(&lc, recflex_fused_kernel<KOCC>, a);
}

template <int KOCC>
int fused_prepare_impl(int smem) {
    cudaError_t e = cudaFuncSetAttribute(recflex_fused_kernel<KOCC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(recflex_fused_kernel<KOCC>, cudaFuncAttributePreferredSharedMemoryCarveout,
                             cudaSharedmemCarveoutMaxShared);
    return (int)e;
}

template <int KOCC>
int fused_occupancy_impl(int smem, int *blocks, int *regs, int *spill) {
    cudaFuncAttributes fa;
    cudaError_t e = cudaFuncGetAttributes(&fa, recflex_fused_kernel<KOCC>);
    if (e != cudaSuccess) return (int)e;
    if (regs) *regs = fa.numRegs;
    if (spill) *spill = (int)fa.localSizeBytes;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, recflex_fused_kernel<KOCC>, kBlockThreads, smem);
    return (int)e;
}

}  // namespace recflex

#define RECFLEX_INSTANTIATE_FUSED(K)                                                                          \
    namespace recflex {                                                                                       \
    int fused_launch_k##K(const FusedArgs &a, const LaunchCfg &cfg, void *stream) {                           \
        return fused_launch_impl<K>(a, cfg, stream);                                                          \
    }                                                                                                         \
    int fused_prepare_k##K(int smem) { return fused_prepare_impl<K>(smem); }                                  \
    int fused_occupancy_k##K(int smem, int *b, int *r, int *s) { return fused_occupancy_impl<K>(smem, b, r, s); } \
    }
