// plan_internal.h -- host-side plan state shared by plan.cpp and tuner.cpp.
#pragma once
#include <cuda_runtime.h>

#include <string>
#include <vector>

#include "recflex_internal.h"

namespace recflex {

// Device-side state one pipeline launch (map -> fill -> fused) reads.
struct Exec {
    int F = 0;                      // descriptors
    int in_F = 0;                   // KJT features in offsets
    FeatureDesc *d_desc = nullptr;
    int32_t *d_block_start = nullptr;
    int32_t *d_npb_eff = nullptr;
    int32_t *d_counter = nullptr;
    int32_t *d_task_start = nullptr;
    int32_t *d_part1 = nullptr;
    int num_part1 = 0;
    long long *d_timers = nullptr;
    int timers_cap = 0;
    float *const *out_ptrs = nullptr;  // routed mode: device array of destination buffers
    int route_rows = 0;                // 0 = local output
    int col_base = 0;
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

}  // namespace recflex

struct recflex_plan_s {
    int device = 0;
    int F = 0;
    int max_batch = 0;
    int num_sms = 148;
    int64_t d_tot = 0;
    std::vector<recflex_feature_spec_t> specs;
    std::vector<recflex::FeatureDesc> desc;  // host mirror
    std::vector<int32_t> part1;              // features with part == 1
    std::vector<const void *> tables;        // cached table pointers
    int k = 4;
    int task_lookups = 4096;  // lookups per task targeted by the default schedules
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
bool schedule_valid_for(const recflex_schedule_t &s, int dim, int dtype, int col, int d_tot);
int row_bytes_of(int dim, int dtype);
recflex_schedule_t default_schedule(const recflex_feature_spec_t &spec, int target);
int find_catalog(int family, int G, int VEC, int C, int U, int ET = 0);
int samples_per_task_default(int sched_id, float mean_len, float coverage, int target);
int slots_for(int max_batch, float max_len);

}  // namespace recflex
