// fused_impl.cuh -- the fused heterogeneous-schedule kernel (Fig. 8),
// B200 form: persistent CTAs (#SM x k) pull tasks from a device counter, so the
// grid never depends on host-side knowledge of the batch (the device-side map
// kernel produced block_start); launched with PDL behind the map kernel.  The
// task is still the CTA-sized mapping unit of the paper, but warps of a
// CTA advance through the task sequence independently (ring of task slots):
// GROUP-family tasks never wait on a CTA barrier.
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

#ifndef RECFLEX_JIT
template <int I, int END>
__device__ __forceinline__ void dispatch_chain(int id, const TaskCtx &x, float *red, int *bag_ctr) {
    if constexpr (I < END && I < kCatalogSize) {
        if (id == I) {
            constexpr CatalogEntry e = kCatalog[I];
            // fp32 entries: G compiled in (the tuned path); reduced-precision
            // entries share one instantiation per (family, ET, VEC, C, U) with
            // G passed at run time -- ptxas time grows superlinearly with the
            // number of functions in the kernel's call graph.
            constexpr int GT = (e.ET == RECFLEX_DTYPE_F32) ? e.G : 0;
            if constexpr (e.family == RECFLEX_FAMILY_GROUP)
                sched_group<e.ET, GT, e.VEC, e.C, e.U>(x.table, x.rowb, e.G, x.offs, x.idx, x.out, x.dim, x.pool, x.ro,
                                                        x.s0, x.s1, bag_ctr);
            else if constexpr (e.family == RECFLEX_FAMILY_WARP)
                sched_warp<e.ET, GT, e.VEC, e.C, e.U>(x.table, x.rowb, e.G, x.offs, x.idx, x.out, x.dim, x.pool, x.ro,
                                                       x.s0, x.s1, bag_ctr);
            else if constexpr (e.family == RECFLEX_FAMILY_FLAT)
                sched_flat<e.ET, GT, e.VEC, e.U>(x.table, x.rowb, e.G, x.offs, x.idx, x.out, x.dim, x.pool, x.ro, x.s0,
                                                  x.s1, bag_ctr);
            else
                sched_block<e.ET, GT, e.VEC, e.C, e.U>(x.table, x.rowb, e.G, x.offs, x.idx, x.out, x.dim, x.pool, x.ro,
                                                        x.s0, x.s1, red);
        } else {
            dispatch_chain<I + 1, END>(id, x, red, bag_ctr);
        }
    }
}

// The if-else chain over the catalog, cut into runs of 64 entries so
// the template recursion stays shallow (fp32 entries keep their place in the
// first run).
__device__ __forceinline__ void dispatch_schedule(int id, const TaskCtx &x, float *red, int *bag_ctr) {
    static_assert(kCatalogSize <= 256, "extend dispatch_schedule");
    if (id < 64) dispatch_chain<0, 64>(id, x, red, bag_ctr);
    else if (id < 128) dispatch_chain<64, 128>(id, x, red, bag_ctr);
    else if (id < 192) dispatch_chain<128, 192>(id, x, red, bag_ctr);
    else dispatch_chain<192, 256>(id, x, red, bag_ctr);
}

// Single call site for the whole catalog: the kernel calls this once per task
// (few live values cross the call), and it branches to the schedule.
static __device__ __noinline__ void dispatch_task(int id, const char *T, unsigned rowb, const int32_t *offs,
                                                  const int32_t *idx, float *out, int d, int pool, const OutRoute ro,
                                                  int s0, int s1, float *red, int *bag) {
    TaskCtx x;
    x.table = T;
    x.rowb = rowb;
    x.offs = offs;
    x.idx = idx;
    x.out = out;
    x.dim = d;
    x.pool = pool;
    x.ro = ro;
    x.s0 = s0;
    x.s1 = s1;
    dispatch_schedule(id, x, red, bag);
}

#endif  // !RECFLEX_JIT

constexpr int kRedFloats = 8 * 256;  // BLOCK family: [8 warps][SPAN <= 256]
constexpr int kWarps = kBlockThreads / 32;
constexpr int kRing = 8;             // task slots in flight per CTA

#define RECFLEX_FAMILY_OF(fam, et, g, v, c, u) fam,
__constant__ signed char kFamilyDev[kCatalogSize] = {RECFLEX_CATALOG(RECFLEX_FAMILY_OF)};
#undef RECFLEX_FAMILY_OF

// One task in flight inside a CTA.  Warps walk the same task sequence
// n = 0, 1, 2, ... independently; slot n % kRing holds task n.
struct TaskSlot {
    int t;       // global task id (>= total: end of work)
    int f;       // feature_idx
    int s0, s1;  // samples of the task
    int bag;     // GROUP family: next bag to claim (relative to s0)
    int left;    // warps that finished this task
    int state;   // 0 free, 1 being filled, 2 ready
    int seq;     // task sequence number held
    unsigned long long wtime;  // tuning: sum over warps of cycles spent on the task
};

__device__ __forceinline__ int vld(const int *p) { return *reinterpret_cast<const volatile int *>(p); }
__device__ __forceinline__ void vst(int *p, int v) { *reinterpret_cast<volatile int *>(p) = v; }
// Slot hand-off flags: release store by the filling / last-leaving warp,
// acquire load by the waiting warps (CTA scope, shared memory).
__device__ __forceinline__ int ld_acquire(const int *p) {
    int v;
    asm volatile("ld.acquire.cta.shared::cta.b32 %0, [%1];"
                 : "=r"(v)
                 : "r"((unsigned)__cvta_generic_to_shared(p))
                 : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int *p, int v) {
    asm volatile("st.release.cta.shared::cta.b32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(p)), "r"(v)
                 : "memory");
}
__device__ __forceinline__ unsigned long long vld64(const unsigned long long *p) {
    return *reinterpret_cast<const volatile unsigned long long *>(p);
}

__device__ __forceinline__ int find_feature(const int *bs, int F, int t) {
    int lo = 0, hi = F;  // upper_bound(block_start, t) - 1
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (bs[mid] <= t) lo = mid;
        else hi = mid;
    }
    return lo;
}

// Samples [s0, s1) of needed task q of feature f (the runtime thread map's
// task, Fig. 8): sample-partitioned -> per_block consecutive samples;
// lookup-partitioned -> the range the fill kernel wrote.
__device__ __forceinline__ void task_range(const FeatureDesc &fd, int q, const FusedArgs &a, int &s0, int &s1) {
    if (fd.part == 0) {
        s0 = min(a.B, q * fd.per_block);
        s1 = min(a.B, s0 + fd.per_block);
    } else {
        const int32_t *ts = a.task_start + fd.slot_base;
        s0 = ts[q];
        s1 = ts[q + 1];
    }
}

// Claim the next task from the device counter and decode it into slot S
// (called by one lane that won the slot's 0 -> 1 CAS); publishes with a
// release store of state = 2.
__device__ __forceinline__ void fill_slot(TaskSlot &S, int n, const FusedArgs &a, const int *bs, int F, int total) {
    const int t = atomicAdd(a.counter, 1);
    S.t = t;
    S.seq = n;
    S.bag = 0;
    S.left = 0;
    S.wtime = 0;
    if (t < total) {
        const int f = find_feature(bs, F, t);
        const int rel = t - bs[f];
        const FeatureDesc &fd = a.desc[f];
        int s0 = 0, s1 = 0;
        if (fd.nalloc == 0) task_range(fd, rel, a, s0, s1);  // static tasks resolve their ranges in the loop
        S.f = f;
        S.s0 = s0;
        S.s1 = s1;
        st_release(&S.state, 2);  // publish first: waiting warps need not wait for the prefetch below
#ifndef RECFLEX_NO_L2PF
        if (s1 > s0) {
            // stage the task's contiguous lookup-ID range into L2 with one bulk
            // prefetch (TMA engine); its two offset loads are off the slot's
            // publish path
            const int32_t *offs = a.offsets + (size_t)fd.in_feature * a.B;
            const int32_t j0 = __ldg(offs + s0), j1 = __ldg(offs + s1);
            const uintptr_t b = reinterpret_cast<uintptr_t>(a.indices + j0) & ~uintptr_t(15);
            const uintptr_t e = (reinterpret_cast<uintptr_t>(a.indices + j1) + 15) & ~uintptr_t(15);
            if (e > b)
                asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(b), "r"((unsigned)(e - b)) : "memory");
        }
#endif
        return;
    }
    st_release(&S.state, 2);
}

// BWD = false: the forward (gather + pool, catalog dispatch).  BWD = true: the
// backward scatter (sched_backward) over the SAME task map and task ring.
template <int KOCC, bool BWD>
__device__ __forceinline__ void fused_body(const FusedArgs &a) {
    extern __shared__ __align__(16) unsigned char dyn_smem[];
    __shared__ TaskSlot ring[kRing];
    float *red = reinterpret_cast<float *>(dyn_smem);                            // union member 1
    int *bs_s = reinterpret_cast<int *>(dyn_smem + kRedFloats * sizeof(float));  // union member 2
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const int F = a.F;
    // block_start cached in shared memory when it fits in the launch's dynamic
    // smem (tuning launches run more -- virtual -- features than the plan sized for)
    const bool bs_in_smem = (F + 1) <= kSmemBlockStartCap && kRedFloats * 4 + 4 * (F + 1) <= a.smem_bytes;

    // PDL: everything above overlapped the map kernel; wait for its results.
    asm volatile("griddepcontrol.wait;" ::: "memory");

    const int total = a.block_start[F];
    // exchange mode: this step's destination buffers (double-buffered by epoch parity)
    float *const *optrs = a.out_ptrs;
    if (!BWD && a.route_epoch) optrs += (size_t)(vld(a.route_epoch) & 1) * a.route_world;
    if (bs_in_smem)
        for (int i = tid; i <= F; i += kBlockThreads) bs_s[i] = a.block_start[i];
    const int *bs = bs_in_smem ? bs_s : a.block_start;
    if (tid < kRing) {
        ring[tid].state = 0;
        ring[tid].seq = -1;
        ring[tid].left = 0;
    }
    __syncthreads();

    // Warp-decoupled task loop: a warp that runs out of bags in task n moves
    // on to task n+1 without waiting for the CTA's other warps (no per-task
    // __syncthreads for GROUP schedules); BLOCK schedules synchronise the CTA
    // on entry and exit.  The first warp to reach a free slot fills it.
    for (int n = 0;; ++n) {
        TaskSlot &S = ring[n % kRing];
        if (lane == 0) {
            long long spin0 = 0;
            while (true) {
                const int st = ld_acquire(&S.state);
                if (st == 2) {
                    if (vld(&S.seq) == n) break;
                } else if (st == 0 && atomicCAS(&S.state, 0, 1) == 0) {
                    fill_slot(S, n, a, bs, F, total);
                    break;
                }
                __nanosleep(32);
                // watchdog: a slot that never becomes ready is a protocol bug;
                // fail the launch (cudaErrorIllegalInstruction) instead of
                // hanging the device (~10 s at 2 GHz)
                const long long now = clock64();
                if (spin0 == 0) spin0 = now;
                else if (now - spin0 > 20000000000LL) asm volatile("trap;");
            }
        }
        __syncwarp();
        __threadfence_block();
        const int t = vld(&S.t);
        if (t >= total) break;
        // Tuning timer ("block execution time"): warps of one CTA can be
        // on different tasks, so a task's cost is the warp-cycles spent on it
        // (sum over warps of enter->leave) / 8 -- for a CTA-synchronous task
        // this is exactly its span; for a warp-decoupled task it does not
        // count the time its warps spent on neighbouring tasks.
        const long long w0 = a.timers ? clock64() : 0;
        const int f = vld(&S.f);
        const FeatureDesc fd = a.desc[f];
#ifdef RECFLEX_JIT
        const int jv = a.jit_var[f];
        const bool block_family = jit_is_block(jv);
#else
        const bool block_family = kFamilyDev[fd.sched] == RECFLEX_FAMILY_BLOCK;
#endif
        // static thread mapping runs its needed tasks CTA-synchronously;
        // compiled only into plan-specialised kernels of plans that use it
        // (its loop state would cost registers in every other kernel)
#if defined(RECFLEX_JIT) && RECFLEX_JIT_STATIC
        const bool stat = !BWD && fd.nalloc > 0;
#else
        constexpr bool stat = false;
#endif
        const bool cta_wide = !BWD && (block_family || stat);
        if (cta_wide) __syncthreads();  // every warp reaches task n (they walk the same sequence)
        OutRoute ro;
        ro.ptrs = optrs;
        ro.rows = a.route_rows;
        ro.colofs = a.col_base + fd.col;
        ro.stride = a.out_stride;
#if defined(RECFLEX_JIT) && RECFLEX_JIT_STATIC
        // Static thread mapping (the paper's ablation straw man):
        // allocated task rel performs the needed tasks rel, rel + nalloc,
        // rel + 2*nalloc, ... one after another (reading C31); an allocated
        // task beyond the batch's need idles.  Runtime mapping: one pass.
        // (One call site for the dispatch: the schedules are inlined once.)
        int q = stat ? t - bs[f] : 0;
        const int need = stat ? a.need[f] : 1;
        while (q < need) {
            int s0, s1;
            if (stat) {
                task_range(fd, q, a, s0, s1);
            } else {
                s0 = vld(&S.s0);
                s1 = vld(&S.s1);
            }
            TaskCtx x;
            x.table = static_cast<const char *>(fd.table);
            x.offs = a.offsets + (size_t)fd.in_feature * a.B;
            x.idx = a.indices;
            x.out = a.out + fd.col;
            x.ro = ro;
            x.s0 = s0;
            x.s1 = s1;
            jit_dispatch(jv, x, red, &S.bag);
            if (!stat) break;
            __syncthreads();           // every warp is done with needed task q
            if (tid == 0) S.bag = 0;   // fresh bag counter for the next one
            __syncthreads();
            q += fd.nalloc;
        }
#else
        if constexpr (BWD) {
            sched_backward(a.grad + fd.col, a.out_stride, a.targets[f], a.offsets + (size_t)fd.in_feature * a.B,
                           a.indices, fd.dim, fd.pool, a.bscale, vld(&S.s0), vld(&S.s1), &S.bag, a.bvec != 0);
        } else {
#ifdef RECFLEX_JIT
            TaskCtx x;
            x.table = static_cast<const char *>(fd.table);
            x.offs = a.offsets + (size_t)fd.in_feature * a.B;
            x.idx = a.indices;
            x.out = a.out + fd.col;
            x.ro = ro;
            x.s0 = vld(&S.s0);
            x.s1 = vld(&S.s1);
            jit_dispatch(jv, x, red, &S.bag);
#else
            dispatch_task(fd.sched, static_cast<const char *>(fd.table), (unsigned)fd.row_bytes,
                          a.offsets + (size_t)fd.in_feature * a.B, a.indices, a.out + fd.col, fd.dim, fd.pool, ro,
                          vld(&S.s0), vld(&S.s1), red, &S.bag);
#endif
        }
#endif
        if (cta_wide) __syncthreads();
        __syncwarp();
        if (lane == 0) {
            if (a.timers) atomicAdd(&S.wtime, (unsigned long long)(clock64() - w0));
            __threadfence_block();
            if (atomicAdd(&S.left, 1) == kWarps - 1) {
                if (a.timers && t < a.timers_cap) a.timers[t] = (long long)(vld64(&S.wtime) / kWarps);
                S.seq = -1;
                st_release(&S.state, 0);
            }
        }
    }
}

template <int KOCC>
__global__ void __launch_bounds__(kBlockThreads, KOCC) recflex_fused_kernel(FusedArgs a) {
    fused_body<KOCC, false>(a);
}

template <int KOCC>
__global__ void __launch_bounds__(kBlockThreads, KOCC) recflex_backward_kernel(FusedArgs a) {
    fused_body<KOCC, true>(a);
}

#ifndef __CUDACC_RTC__
template <int KOCC, bool BWD>
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
    if constexpr (BWD) return (int)cudaLaunchKernelEx(&lc, recflex_backward_kernel<KOCC>, a);
    else return (int)cudaLaunchKernelEx(&lc, recflex_fused_kernel<KOCC>, a);
}

template <int KOCC>
int fused_prepare_impl(int smem, int carveout) {
    cudaError_t e = cudaFuncSetAttribute(recflex_fused_kernel<KOCC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(recflex_fused_kernel<KOCC>, cudaFuncAttributePreferredSharedMemoryCarveout,
                             carveout);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(recflex_backward_kernel<KOCC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return (int)e;
    e = cudaFuncSetAttribute(recflex_backward_kernel<KOCC>, cudaFuncAttributePreferredSharedMemoryCarveout,
                             carveout);
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

#endif  // !__CUDACC_RTC__

}  // namespace recflex

#define RECFLEX_INSTANTIATE_FUSED(K)                                                                          \
    namespace recflex {                                                                                       \
    int fused_launch_k##K(const FusedArgs &a, const LaunchCfg &cfg, void *stream) {                           \
        return fused_launch_impl<K, false>(a, cfg, stream);                                                   \
    }                                                                                                         \
    int backward_launch_k##K(const FusedArgs &a, const LaunchCfg &cfg, void *stream) {                        \
        return fused_launch_impl<K, true>(a, cfg, stream);                                                    \
    }                                                                                                         \
    int fused_prepare_k##K(int smem, int cv) { return fused_prepare_impl<K>(smem, cv); }                      \
    int fused_occupancy_k##K(int smem, int *b, int *r, int *s) { return fused_occupancy_impl<K>(smem, b, r, s); } \
    }
