// plan_internal.h -- host-side plan state shared by plan.cpp and tuner.cpp.
#pragma once
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <string>
#include <vector>

#include "recflex_internal.h"

namespace recflex {

// NVTX range for the host-side timeline of an API call (header-only NVTX3: a
// no-op unless a profiler injects itself, e.g. nsys / ncu --nvtx).
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

// Device-side state one pipeline launch (map -> fill -> fused) reads.
struct Exec {
    int F = 0;                      // descriptors
    int in_F = 0;                   // KJT features in offsets
    FeatureDesc *d_desc = nullptr;
    int32_t *d_block_start = nullptr;
    int32_t *d_npb_eff = nullptr;
    int32_t *d_need = nullptr;      // [F] needed tasks per feature (map kernel)
    int32_t *d_counter = nullptr;
    int32_t *d_task_start = nullptr;
    int32_t *d_part1 = nullptr;
    int num_part1 = 0;
    long long *d_timers = nullptr;
    int timers_cap = 0;
    float *const *out_ptrs = nullptr;  // routed mode: device array of destination buffers
    int route_rows = 0;                // 0 = local output
    int col_base = 0;
    // exchange mode (recflex_forward_exchange): double-buffered destinations
    int32_t *route_epoch = nullptr;
    int route_world = 0;
    // backward (NEXT #4)
    bool backward = false;
    const float *grad = nullptr;
    float *const *d_targets = nullptr;
    float bscale = 1.f;
    int bvec = 0;
};

struct EventTriple {
    cudaEvent_t e0, e1, e2;
};

// Pinned host staging for the plan's small async uploads (descriptors, pointer
// tables): a pageable source would make cudaMemcpyAsync synchronous and is not
// graph-capturable.  Slots rotate; a slot is reused only after its copy ran.
struct StageSlot {
    void *h = nullptr;
    size_t cap = 0;
    cudaEvent_t ev = nullptr;
    bool pending = false;
};
constexpr int kStageSlots = 4;

// A plan-specialised fused kernel (jit.cpp) compiled for one occupancy k.
struct JitKernel {
    void *module = nullptr;    // CUmodule
    void *function = nullptr;  // CUfunction
    uint64_t sig = 0;          // schedule signature it was generated from (jit_plan_sig)
    int32_t *d_var = nullptr;  // device: variant id per task-order position (this kernel's numbering)
    std::vector<int32_t> h_var;  // host: variant id per feature (feature order)
    int variants = 0;
    int smem = 0, occ = 0, carveout = 0;
    int regs = 0, local_bytes = 0;
    bool cache_hit = false;
    double compile_ms = 0;
};

}  // namespace recflex

struct recflex_plan_s {
    int device = 0;
    int F = 0;
    int max_batch = 0;
    int num_sms = 148;
    int64_t d_tot = 0;
    std::vector<recflex_feature_spec_t> specs;
    std::vector<recflex::FeatureDesc> desc;  // host mirror, feature order
    // Task order (reading C35): the device descriptor array -- and with it the
    // task map, every per-feature device array (need, npb_eff, block_start,
    // variant ids, backward targets) and the order in which the persistent
    // CTAs claim tasks -- lists the features in this order: position e holds
    // feature order[e].  Empty = feature order (the paper's).
    std::vector<int32_t> order;
    // Output layout (C35): false = features concatenated in feature order (the
    // paper's), true = concatenated in task order (recflex_get_columns).
    bool columns_follow_order = false;
    // L2 eviction priority of every feature's row loads in the plan-specialised
    // kernel (C36): 0 default, 1 evict_first, 2 evict_last.  Empty = all 0.
    std::vector<int8_t> l2;
    std::vector<int32_t> part1;              // task-order positions with part == 1
    std::vector<const void *> tables;        // cached table pointers
    int k = 4;
    int task_lookups = 4096;  // lookups per task targeted by the default schedules
    bool small_batch = false; // the expected batch is < 8 waves of 512-lookup tasks (latency-bound)
    bool desc_dirty = true;
    bool pdl = true;
    bool force_smem_pad = false;  // RECFLEX_SMEM_PAD=1: always pad shared memory to k CTAs/SM (A/B)
    int64_t slots_total = 0;

    recflex::Exec ex;  // plan-owned device scratch

    // per-occupancy launch configuration (index k = 1..8)
    int smem[recflex::kMaxOcc + 1] = {0};
    int occ[recflex::kMaxOcc + 1] = {0};
    bool prepared[recflex::kMaxOcc + 1] = {false};
    int carveout[recflex::kMaxOcc + 1] = {0};  // shared-memory carveout (percent) chosen for k

    // profiling
    bool profiling = false;
    std::vector<recflex::EventTriple> ev_pending;
    std::vector<recflex::EventTriple> ev_free;
    double map_ms = 0, fused_ms = 0;
    int64_t forwards = 0;

    // host-buffer entry point staging
    // routed forward: destination pointer table (device) and its host copy
    float **d_route = nullptr;
    std::vector<float *> route_cache;
    // backward: target pointer table (device) and its host copy
    float **d_targets = nullptr;
    std::vector<float *> targets_cache;
    int32_t *d_stage_idx = nullptr;
    int64_t stage_idx_cap = 0;
    int32_t *d_stage_off = nullptr;
    int64_t stage_off_cap = 0;
    float *d_stage_out = nullptr;
    int64_t stage_out_cap = 0;
    // recflex_forward_host_batches: double-buffered staging + copy streams
    struct HostPipe *pipe = nullptr;

    recflex_tune_stats_t last_stats = {};

    recflex::StageSlot stage[recflex::kStageSlots];
    int stage_next = 0;

    // recflex_forward_exchange state (device scratch + host caches)
    float **d_xroute = nullptr;       // 2 x W destination pointers
    uint32_t **d_xflags = nullptr;    // W flag-array pointers
    int32_t *d_xcount = nullptr;      // [0] epoch (completed exchange steps)
    std::vector<void *> xroute_cache;
    int64_t x_steps = 0;              // host mirror of the epoch (eager calls)

    // plan-specialised fused kernels (jit.cpp): used by forwards at occupancy k
    // while jit[k].version == sched_version (any schedule change bumps it)
    recflex::JitKernel jit[recflex::kMaxOcc + 1];
    int64_t sched_version = 0;
    int64_t sig_version = -1;    // sched_version the cached signature belongs to
    uint64_t sig_cached = 0;
    int num_static = 0;          // features with a static thread mapping (P:338 ablation)
    bool use_jit = true;
};

namespace recflex {

recflex_status_t cuda_status(cudaError_t e);
recflex_status_t cuda_status_at(cudaError_t e, const char *where);
void set_last_error(const char *msg);
recflex_status_t prepare_occupancy(recflex_plan_s *p, int k);
void host_pipe_free(recflex_plan_s *p);
int min_dyn_smem(int F);
// Launch map (+fill) + fused for an Exec.  Events (optional) bracket map and fused.
recflex_status_t run_pipeline(recflex_plan_s *p, const Exec &ex, const int32_t *indices, const int32_t *offsets, int B,
                              float *out, int out_stride, int k, cudaStream_t stream, EventTriple *ev);
recflex_status_t upload_desc(recflex_plan_s *p, cudaStream_t stream);
recflex_status_t staged_copy(recflex_plan_s *p, void *d_dst, const void *src, size_t bytes, cudaStream_t stream);
bool schedule_valid_for(const recflex_schedule_t &s, int dim, int dtype, int col, int d_tot);
// feature at task-order position e
inline int feature_at(const recflex_plan_s *p, int e) { return p->order.empty() ? e : p->order[e]; }
// task-order heuristics (RECFLEX_ORDER_*): out = permutation, position -> feature
void task_order_of_kind(const recflex_plan_s *p, int kind, std::vector<int32_t> &out);
recflex_status_t apply_task_order(recflex_plan_s *p, const int32_t *order);
recflex_status_t normalize_order(const recflex_plan_s *p, const int32_t *order, std::vector<int32_t> &o);
recflex_status_t set_layout(recflex_plan_s *p, const std::vector<int32_t> &order, bool follow,
                            const std::vector<recflex_schedule_t> *scheds);
recflex_status_t jit_upload_var(recflex_plan_s *p);
int row_bytes_of(int dim, int dtype);
recflex_schedule_t default_schedule(const recflex_feature_spec_t &spec, int target, bool small_batch);
int find_catalog(int family, int G, int VEC, int C, int U, int ET = 0);
int samples_per_task_default(int sched_id, float mean_len, float coverage, int target);
int slots_for(int max_batch, float max_len);
// plan-specialised fused kernel (jit.cpp)
bool jit_ready(recflex_plan_s *p, int k);
uint64_t jit_plan_sig(recflex_plan_s *p);
int jit_launch(recflex_plan_s *p, int k, const FusedArgs &a, bool pdl, cudaStream_t stream);
recflex_status_t jit_compile_plan(recflex_plan_s *p, const int *ks, int nk);
void jit_release(recflex_plan_s *p);

}  // namespace recflex
