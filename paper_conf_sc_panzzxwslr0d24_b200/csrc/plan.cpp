// plan.cpp -- C ABI: plan lifecycle, forward, schedules, occupancy, validation,
// introspection, persistence.  (Tuner in tuner.cpp.)
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "plan_internal.h"

using namespace recflex;

namespace recflex {

static thread_local char g_last_error[512] = "";

void set_last_error(const char *msg) {
    std::snprintf(g_last_error, sizeof(g_last_error), "%s", msg);
}

recflex_status_t cuda_status_at(cudaError_t e, const char *where) {
    if (e == cudaSuccess) return RECFLEX_OK;
    std::snprintf(g_last_error, sizeof(g_last_error), "%s: %s (%s)", where ? where : "cuda", cudaGetErrorName(e),
                  cudaGetErrorString(e));
    if (e == cudaErrorMemoryAllocation) return RECFLEX_ERR_OOM;
    return RECFLEX_ERR_CUDA;
}

recflex_status_t cuda_status(cudaError_t e) { return cuda_status_at(e, "cuda"); }

static int next_pow2(int v) {
    int p = 1;
    while (p < v) p <<= 1;
    return p;
}

int find_catalog(int family, int G, int VEC, int C, int U, int ET) {
    for (int i = 0; i < kCatalogSize; ++i) {
        const CatalogEntry &e = kCatalog[i];
        if (e.family == family && e.ET == ET && e.G == G && e.VEC == VEC && e.C == C && e.U == U) return i;
    }
    return -1;
}

int row_bytes_of(int dim, int dtype) {
    switch (dtype) {
        case RECFLEX_DTYPE_F16:
        case RECFLEX_DTYPE_BF16: return 2 * dim;
        case RECFLEX_DTYPE_I8: return (int)RECFLEX_I8_ROW_BYTES(dim);
        case RECFLEX_DTYPE_FP8: return dim;
        default: return 4 * dim;
    }
}

// samples per task for sample-partitioned tasks: about `target` expected
// lookups per task (enough work to amortise the task fetch), between 1 and 32
// rounds of the CTA's bag slots.
int samples_per_task_default(int sched_id, float mean_len, float coverage, int target) {
    const CatalogEntry &e = kCatalog[sched_id];
    const int slots = (e.family == RECFLEX_FAMILY_GROUP) ? kBlockThreads / e.G
                      : (e.family == RECFLEX_FAMILY_FLAT) ? (kBlockThreads / e.G) * 8
                      : (e.family == RECFLEX_FAMILY_WARP) ? kBlockThreads / 32
                                                          : 1;
    double el = std::max(0.25, (double)mean_len * std::max(0.05, (double)coverage));
    int R = (int)std::lround((double)target / (slots * el));
    R = std::min(32, std::max(1, R));
    if (e.family == RECFLEX_FAMILY_BLOCK) R = std::min(64, std::max(1, (int)std::lround(0.5 * target / el)));
    return slots * R;
}

// Plan-level lookups per task: ~4096, but small enough that the expected
// batch yields >= 8 waves of #SM x 4 CTAs (Eq. 2 assumes a negligible tail,
// P:116), and never below 256.
int task_lookups_target(const recflex_feature_spec_t *specs, int F, int max_batch, int num_sms) {
    double tot = 0;
    for (int f = 0; f < F; ++f)
        tot += (double)max_batch * std::max(0.25, (double)specs[f].mean_len * std::max(0.05, (double)specs[f].coverage));
    double t = tot / (8.0 * num_sms * 4);
    return (int)std::min(4096.0, std::max(256.0, t));
}

recflex_schedule_t default_schedule(const recflex_feature_spec_t &spec, int target, bool small_batch) {
    recflex_schedule_t s = {0, 0, 1, 0};
    const int d = spec.dim;
    int id = -1;
    if (spec.dtype != RECFLEX_DTYPE_F32) {
        // Reduced-precision rows: the same shapes in BYTES as the fp32 rule
        // below -- 32-byte lanes for short rows (16-bit) / 16-byte lanes
        // (int8), one lane group per row, U = 2 for one-hot bags.
        const int et = spec.dtype;
        const int U = spec.mean_len >= 2.5f ? 4 : 2;
        if (et == RECFLEX_DTYPE_FP8) {
            // 16-byte lanes (16 codes), one lane group per row
            if (d % 16 == 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(32, next_pow2(d / 16)), 16, 1, U, et);
            if (id < 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(16, next_pow2(d / 8)), 8, 1, U, et);
        } else if (et == RECFLEX_DTYPE_I8) {
            if (d % 16 == 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(32, next_pow2(d / 16)), 16, 1, U, et);
            if (id < 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(16, next_pow2(d / 8)), 8, 1, U, et);
        } else {
            if (d % 16 == 0 && d <= 128) id = find_catalog(RECFLEX_FAMILY_GROUP, d / 16, 16, 1, 2, et);
            if (id < 0 && d % 8 == 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(32, next_pow2(d / 8)), 8, 1, U, et);
            if (id < 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(8, next_pow2(d / 4)), 4, 1, 4, et);
        }
        s.sched_id = id;
        s.per_block = id >= 0 ? samples_per_task_default(id, spec.mean_len, spec.coverage, target) : 1;
        return s;
    }
    // Small batches (the whole batch is well under 8 waves of 512-lookup tasks:
    // medium, fig3) are latency-bound: a multi-hot bag pooled by one lane group is
    // a chain of L/U dependent row round trips.  Split such bags across the lane
    // groups of a warp (WARP-SPLIT family, 32/G x U rows of the bag in flight)
    // with 4 bags per warp per task (measured on B200: medium 0.072 -> 0.038 ms
    // fused, tools/latency_probe.py).
    if (small_batch && spec.mean_len >= 8.f && d % 4 == 0 && d >= 8 && d <= 64) {
        id = find_catalog(RECFLEX_FAMILY_WARP, d / 4, 4, 1, d / 4 <= 2 ? 2 : 4);
        if (id >= 0) {
            s.sched_id = id;
            s.part = 0;
            s.per_block = 32;
            return s;
        }
    }
    // Untuned defaults follow what the tuner picks most on B200 (sharded1000 /
    // heavy): rows up to 64 floats -> 256-bit loads with d/8 lanes per bag
    // (more bags in flight per warp), U = 2; wider rows -> a warp (or more
    // passes) of 128-bit lanes, U = 4 for multi-hot bags.
    if (d % 8 == 0 && d <= 64) {
        id = find_catalog(RECFLEX_FAMILY_GROUP, std::max(1, d / 8), 8, 1, 2);
    } else if (d % 4 == 0) {
        int lanes = d / 4;
        int G = std::min(32, next_pow2(lanes));
        int U = spec.mean_len >= 2.5f ? 4 : 2;
        id = find_catalog(RECFLEX_FAMILY_GROUP, G, 4, 1, U);
    }
    if (id < 0) id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(32, next_pow2(d)), 1, 1, 4);
    s.sched_id = id;
    s.part = 0;
    s.per_block = samples_per_task_default(id, spec.mean_len, spec.coverage, target);
    return s;
}

int slots_for(int max_batch, float max_len) {
    // reserved task-range entries for a lookup-partitioned feature: tasks of
    // >= 128 lookups at the planned maximum, + sentinel; the map kernel raises
    // the per-task lookups if a batch would need more (always correct).
    double ml = std::max(1.0, (double)max_len);
    double need = (double)max_batch * ml / 128.0 + 3.0;
    need = std::min(need, (double)(1 << 20));
    return (int)std::max(64.0, need);
}

bool schedule_valid_for(const recflex_schedule_t &s, int dim, int dtype, int col, int d_tot) {
    if (s.sched_id < 0 || s.sched_id >= kCatalogSize) return false;
    if (s.part < 0 || s.part > 1) return false;
    if (s.per_block < 1 || s.static_blocks < 0) return false;
    const CatalogEntry &e = kCatalog[s.sched_id];
    if (!catalog_valid(e, dim, dtype)) return false;
    // vector stores need 16-byte aligned output columns
    if (e.VEC > 1 && ((col % 4) != 0 || (d_tot % 4) != 0)) return false;
    return true;
}

int min_dyn_smem(int F) {
    int m = 8 * 256 * 4;  // BLOCK-family reduction scratch
    if (F + 1 <= kSmemBlockStartCap) m += 4 * (F + 1);
    return (m + 127) / 128 * 128;
}

// Occupancy control (C15): exactly k CTAs per SM.  The register cap of
// __launch_bounds__(256, k) alone enforces k whenever the kernel uses its full
// cap (the fused kernel does at every k); then the CTA keeps only the dynamic
// shared memory it needs and the carveout leaves the rest of the SM's 256 KB
// to L1 -- padding shared memory as well (the paper's second knob) shrank L1
// to ~30 KB at k = 4, so the per-bag register spills of the schedule
// functions went to L2 (1.2 GB of local-memory traffic per heavy batch).
// Shared-memory padding is used only when registers do not already limit the
// kernel to k (or when RECFLEX_SMEM_PAD=1 forces the old behaviour).
recflex_status_t prepare_occupancy(recflex_plan_s *p, int k) {
    if (k < 1 || k > kMaxOcc) return RECFLEX_ERR_INVALID_ARG;
    if (p->prepared[k]) return RECFLEX_OK;
    cudaError_t e = cudaSetDevice(p->device);
    if (e != cudaSuccess) return cuda_status(e);
    const int sm_total = 233472;  // 228 KB per SM
    const int mind = min_dyn_smem(p->F);
    int rc = fused_prepare(k, p->device, 232448 - 1024, (int)cudaSharedmemCarveoutMaxShared);
    if (rc) return cuda_status((cudaError_t)rc);
    int blocks = 0, regs = 0, spill = 0;
    rc = fused_occupancy(k, mind, &blocks, &regs, &spill);
    if (rc) return cuda_status((cudaError_t)rc);
    int dyn = mind;
    if (p->force_smem_pad || blocks > k) {
        dyn = ((sm_total / k - 1152) / 128) * 128;
        dyn = std::max(dyn, mind);
        dyn = std::min(dyn, 232448 - 1024);  // 227 KB opt-in max minus static smem (<= 1 KB)
        // walk the padding until the occupancy API reports exactly k (or as close as possible)
        for (int it = 0; it < 64; ++it) {
            rc = fused_occupancy(k, dyn, &blocks, &regs, &spill);
            if (rc) return cuda_status((cudaError_t)rc);
            if (blocks > k) {
                dyn += 128;
            } else if (blocks < k && dyn - 128 >= mind) {
                int b2 = 0;
                fused_occupancy(k, dyn - 128, &b2, &regs, &spill);
                if (b2 <= k) dyn -= 128;
                else break;
                if (b2 == k) break;
            } else {
                break;
            }
        }
        p->carveout[k] = 100;
    } else {
        // smallest carveout (percent of 228 KB) that holds k CTAs' shared memory
        // (dynamic + <= 1 KB static + 1 KB per-CTA reservation)
        const int need = k * (dyn + 2048);
        p->carveout[k] = std::min(100, (need * 100 + sm_total - 1) / sm_total);
        rc = fused_prepare(k, p->device, 232448 - 1024, p->carveout[k]);
        if (rc) return cuda_status((cudaError_t)rc);
    }
    rc = fused_occupancy(k, dyn, &blocks, &regs, &spill);
    if (rc) return cuda_status((cudaError_t)rc);
    p->smem[k] = dyn;
    p->occ[k] = std::max(1, std::min(blocks, k));
    p->prepared[k] = true;
    return RECFLEX_OK;
}

// Async host -> device copy of a small plan array through pinned staging (so
// it is truly asynchronous and never reads pageable memory).  Refuses to run
// inside a stream capture: the captured copy would read the staging slot at
// every replay, after later uploads reused it (run one forward before capturing).
recflex_status_t staged_copy(recflex_plan_s *p, void *d_dst, const void *src, size_t bytes, cudaStream_t stream) {
    if (bytes == 0) return RECFLEX_OK;
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(stream, &cs);
    if (cs != cudaStreamCaptureStatusNone) {
        set_last_error("plan descriptors / pointer tables changed inside a CUDA graph capture: run one forward "
                       "with these tables and destinations before capturing");
        return RECFLEX_ERR_INVALID_ARG;
    }
    StageSlot &sl = p->stage[p->stage_next];
    p->stage_next = (p->stage_next + 1) % kStageSlots;
    cudaError_t e = cudaSuccess;
    if (!sl.ev) e = cudaEventCreateWithFlags(&sl.ev, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_status(e);
    if (sl.pending) {
        e = cudaEventSynchronize(sl.ev);  // the copy that last used this slot has run (normally long ago)
        if (e != cudaSuccess) return cuda_status(e);
        sl.pending = false;
    }
    if (sl.cap < bytes) {
        cudaFreeHost(sl.h);
        sl.h = nullptr;
        sl.cap = 0;
        e = cudaMallocHost(&sl.h, bytes);
        if (e != cudaSuccess) return cuda_status(e);
        sl.cap = bytes;
    }
    std::memcpy(sl.h, src, bytes);
    e = cudaMemcpyAsync(d_dst, sl.h, bytes, cudaMemcpyHostToDevice, stream);
    if (e != cudaSuccess) return cuda_status(e);
    e = cudaEventRecord(sl.ev, stream);
    if (e != cudaSuccess) return cuda_status(e);
    sl.pending = true;
    return RECFLEX_OK;
}

// The device descriptor array lists the features in task order (C35).
recflex_status_t upload_desc(recflex_plan_s *p, cudaStream_t stream) {
    for (int f = 0; f < p->F; ++f) p->desc[f].table = p->tables[f];
    p->part1.clear();
    std::vector<FeatureDesc> dv(p->F);
    for (int e = 0; e < p->F; ++e) {
        dv[e] = p->desc[feature_at(p, e)];
        if (dv[e].part == 1) p->part1.push_back(e);
    }
    recflex_status_t st = staged_copy(p, p->ex.d_desc, dv.data(), sizeof(FeatureDesc) * p->F, stream);
    if (st != RECFLEX_OK) return st;
    if (!p->part1.empty()) {
        st = staged_copy(p, p->ex.d_part1, p->part1.data(), sizeof(int32_t) * p->part1.size(), stream);
        if (st != RECFLEX_OK) return st;
    }
    p->ex.num_part1 = (int)p->part1.size();
    p->desc_dirty = false;
    return RECFLEX_OK;
}

recflex_status_t run_pipeline(recflex_plan_s *p, const Exec &ex, const int32_t *indices, const int32_t *offsets,
                              int B, float *out, int out_stride, int k, cudaStream_t stream, EventTriple *ev) {
    recflex_status_t st = prepare_occupancy(p, k);
    if (st != RECFLEX_OK) return st;
    if (ev) cudaEventRecord(ev->e0, stream);
    NvtxRange nvtx_map("recflex pipeline (map, fill, fused)");
    MapArgs ma;
    ma.desc = ex.d_desc;
    ma.offsets = offsets;
    ma.F = ex.F;
    ma.B = B;
    ma.in_F = ex.in_F;
    ma.block_start = ex.d_block_start;
    ma.npb_eff = ex.d_npb_eff;
    ma.need = ex.d_need;
    ma.counter = ex.d_counter;
    int rc = map_launch(ma, stream);
    if (rc) return cuda_status_at((cudaError_t)rc, "map kernel launch");
    if (ex.num_part1 > 0) {
        FillArgs fa;
        fa.desc = ex.d_desc;
        fa.offsets = offsets;
        fa.block_start = ex.d_block_start;
        fa.npb_eff = ex.d_npb_eff;
        fa.need = ex.d_need;
        fa.part1_features = ex.d_part1;
        fa.num_part1 = ex.num_part1;
        fa.B = B;
        fa.task_start = ex.d_task_start;
        rc = fill_launch(fa, B, p->pdl, stream);
        if (rc) return cuda_status_at((cudaError_t)rc, "fill kernel launch");
    }
    if (ev) cudaEventRecord(ev->e1, stream);
    FusedArgs a;
    a.desc = ex.d_desc;
    a.block_start = ex.d_block_start;
    a.task_start = ex.d_task_start;
    a.need = ex.d_need;
    a.indices = indices;
    a.offsets = offsets;
    a.out = out;
    a.counter = ex.d_counter;
    a.timers = ex.d_timers;
    a.timers_cap = ex.timers_cap;
    a.F = ex.F;
    a.B = B;
    a.out_stride = out_stride;
    a.smem_bytes = p->smem[k];
    a.out_ptrs = ex.out_ptrs;
    a.route_rows = ex.route_rows;
    a.col_base = ex.col_base;
    a.route_epoch = ex.route_epoch;
    a.route_world = ex.route_world;
    a.grad = ex.grad;
    a.targets = ex.d_targets;
    a.bscale = ex.bscale;
    a.bvec = ex.bvec;
    LaunchCfg cfg;
    cfg.grid = p->num_sms * p->occ[k];
    cfg.smem = p->smem[k];
    // With events between the kernels, PDL overlap is disabled (the event is a
    // stream dependency point anyway).
    cfg.pdl = p->pdl && ev == nullptr;
    a.jit_var = nullptr;
    if (ex.d_desc == p->ex.d_desc && p->num_static > 0 && (ex.backward || !jit_ready(p, k))) {
        set_last_error("a static thread mapping (static_blocks > 0) runs only in the plan-specialised kernel: "
                       "call recflex_plan_compile (forward only)");
        return RECFLEX_ERR_NOT_SUPPORTED;
    }
    if (!ex.backward && ex.d_desc == p->ex.d_desc && jit_ready(p, k))
        rc = jit_launch(p, k, a, cfg.pdl, stream);  // the plan-specialised kernel (jit.cpp)
    else
        rc = ex.backward ? backward_launch(k, a, cfg, stream) : fused_launch(k, a, cfg, stream);
    if (rc) return cuda_status_at((cudaError_t)rc, ex.backward ? "backward kernel launch" : "fused kernel launch");
    if (ev) cudaEventRecord(ev->e2, stream);
    return RECFLEX_OK;
}

// Estimated bytes one task of feature f moves under its schedule (hotness
// stats only): sample-partitioned tasks hold per_block bags of mean length
// coverage * mean_len, lookup-partitioned tasks per_block lookups.
static double task_bytes_estimate(const recflex_plan_s *p, int f) {
    const FeatureDesc &d = p->desc[f];
    const recflex_feature_spec_t &sp = p->specs[f];
    const double rb = (double)d.row_bytes;
    if (d.part == 1) return (double)d.per_block * rb;
    const double L = std::max(0.05, (double)sp.mean_len * (double)sp.coverage);
    return (double)d.per_block * L * rb;
}

void task_order_of_kind(const recflex_plan_s *p, int kind, std::vector<int32_t> &out) {
    out.resize(p->F);
    for (int f = 0; f < p->F; ++f) out[f] = f;
    if (kind == RECFLEX_ORDER_FEATURE) return;
    std::vector<double> est(p->F);
    for (int f = 0; f < p->F; ++f) est[f] = task_bytes_estimate(p, f);
    if (kind == RECFLEX_ORDER_LPT)
        std::stable_sort(out.begin(), out.end(), [&](int a, int b) { return est[a] > est[b]; });
    else
        std::stable_sort(out.begin(), out.end(), [&](int a, int b) { return est[a] < est[b]; });
}

// Installs a task order (empty = feature order), the column mode and --
// optionally -- new schedules as one change: every schedule is validated at
// the output column it would get first (vector stores need col % 4 == 0), and
// on error nothing changes.  Setup call: waits for the device (no forward of
// the old layout still reads the plan's arrays), re-uploads the order-
// dependent arrays of compiled kernels, marks the descriptors dirty.
recflex_status_t set_layout(recflex_plan_s *p, const std::vector<int32_t> &order, bool follow,
                            const std::vector<recflex_schedule_t> *scheds) {
    std::vector<int32_t> col(p->F);
    int64_t c = 0;
    for (int e = 0; e < p->F; ++e) {
        const int f = (follow && !order.empty()) ? order[e] : e;
        col[f] = (int32_t)c;
        c += p->desc[f].dim;
    }
    for (int f = 0; f < p->F; ++f) {
        const FeatureDesc &d = p->desc[f];
        const recflex_schedule_t s = scheds ? (*scheds)[f] : recflex_schedule_t{d.sched, d.part, d.per_block, d.nalloc};
        if (!schedule_valid_for(s, d.dim, d.dtype, col[f], (int)p->d_tot)) {
            if (scheds) return RECFLEX_ERR_INVALID_ARG;
            set_last_error("column order: a feature's schedule needs a 16-byte aligned output column");
            return RECFLEX_ERR_NOT_SUPPORTED;
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_status(e);
    if (scheds)
        for (int f = 0; f < p->F; ++f) {
            const recflex_schedule_t &s = (*scheds)[f];
            FeatureDesc &d = p->desc[f];
            if (d.sched != s.sched_id || (d.nalloc > 0) != (s.static_blocks > 0)) ++p->sched_version;
            p->num_static += (s.static_blocks > 0 ? 1 : 0) - (d.nalloc > 0 ? 1 : 0);
            d.sched = s.sched_id;
            d.part = s.part;
            d.per_block = s.per_block;
            d.nalloc = s.static_blocks;
        }
    for (int f = 0; f < p->F; ++f) p->desc[f].col = col[f];
    const bool order_changed = order != p->order;
    p->order = order;
    p->columns_follow_order = follow;
    p->desc_dirty = true;
    p->targets_cache.clear();
    // the device descriptors (columns, schedules, order) and the compiled
    // kernels' variant ids change together, now: a CUDA graph captured earlier
    // replays on these arrays without an eager forward to upload them
    recflex_status_t st = upload_desc(p, nullptr);
    if (st == RECFLEX_OK) {
        e = cudaStreamSynchronize(nullptr);
        if (e != cudaSuccess) st = cuda_status(e);
    }
    if (st != RECFLEX_OK) return st;
    return order_changed ? jit_upload_var(p) : RECFLEX_OK;
}

// order: permutation of 0..F-1 (position -> feature) or nullptr = feature order.
recflex_status_t normalize_order(const recflex_plan_s *p, const int32_t *order, std::vector<int32_t> &o) {
    o.clear();
    if (!order) return RECFLEX_OK;
    std::vector<char> seen(p->F, 0);
    bool identity = true;
    for (int e = 0; e < p->F; ++e) {
        const int32_t f = order[e];
        if (f < 0 || f >= p->F || seen[f]) return RECFLEX_ERR_INVALID_ARG;
        seen[f] = 1;
        identity = identity && f == e;
    }
    if (!identity) o.assign(order, order + p->F);
    return RECFLEX_OK;
}

recflex_status_t apply_task_order(recflex_plan_s *p, const int32_t *order) {
    std::vector<int32_t> o;
    recflex_status_t st = normalize_order(p, order, o);
    if (st != RECFLEX_OK) return st;
    if (o == p->order) return RECFLEX_OK;
    return set_layout(p, o, p->columns_follow_order, nullptr);
}

}  // namespace recflex

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" {

const char *recflex_last_error(void) { return g_last_error; }

const char *recflex_status_string(recflex_status_t s) {
    switch (s) {
        case RECFLEX_OK: return "ok";
        case RECFLEX_ERR_INVALID_ARG: return "invalid argument";
        case RECFLEX_ERR_CUDA: return "CUDA error";
        case RECFLEX_ERR_OOM: return "out of device memory";
        case RECFLEX_ERR_NOT_SUPPORTED: return "not supported";
        case RECFLEX_ERR_INDEX_OOB: return "lookup ID out of range";
    }
    return "unknown status";
}

int32_t recflex_catalog_size(void) { return kCatalogSize; }

recflex_status_t recflex_catalog_info(int32_t id, recflex_catalog_info_t *info) {
    if (id < 0 || id >= kCatalogSize || !info) return RECFLEX_ERR_INVALID_ARG;
    const CatalogEntry &e = kCatalog[id];
    info->family = e.family;
    info->group = e.G;
    info->vec = e.VEC;
    info->cols = e.C;
    info->unroll = e.U;
    info->dtype = e.ET;
    return RECFLEX_OK;
}

int32_t recflex_catalog_valid(int32_t id, int32_t dim) {
    if (id < 0 || id >= kCatalogSize) return 0;
    return catalog_valid(kCatalog[id], dim) ? 1 : 0;
}

int32_t recflex_catalog_valid_dtype(int32_t id, int32_t dim, int32_t dtype) {
    if (id < 0 || id >= kCatalogSize) return 0;
    return catalog_valid(kCatalog[id], dim, dtype) ? 1 : 0;
}

static void plan_free_device(recflex_plan_s *p) {
    jit_release(p);
    for (auto &sl : p->stage) {
        if (sl.pending) cudaEventSynchronize(sl.ev);
        if (sl.ev) cudaEventDestroy(sl.ev);
        cudaFreeHost(sl.h);
        sl = StageSlot();
    }
    cudaFree(p->d_xroute);
    cudaFree(p->d_xflags);
    cudaFree(p->d_xcount);
    cudaFree(p->d_route);
    cudaFree(p->d_targets);
    cudaFree(p->ex.d_desc);
    cudaFree(p->ex.d_block_start);
    cudaFree(p->ex.d_npb_eff);
    cudaFree(p->ex.d_need);
    cudaFree(p->ex.d_counter);
    cudaFree(p->ex.d_task_start);
    cudaFree(p->ex.d_part1);
    cudaFree(p->d_stage_idx);
    cudaFree(p->d_stage_off);
    cudaFree(p->d_stage_out);
    host_pipe_free(p);
    for (auto &t : p->ev_pending) {
        cudaEventDestroy(t.e0);
        cudaEventDestroy(t.e1);
        cudaEventDestroy(t.e2);
    }
    for (auto &t : p->ev_free) {
        cudaEventDestroy(t.e0);
        cudaEventDestroy(t.e1);
        cudaEventDestroy(t.e2);
    }
}

recflex_status_t recflex_plan_create(const recflex_feature_spec_t *specs, int32_t F, int32_t max_batch, int32_t device,
                                     recflex_plan_t *out) {
    if (!specs || !out || F <= 0 || max_batch <= 0) return RECFLEX_ERR_INVALID_ARG;
    *out = nullptr;
    int64_t d_tot = 0;
    for (int f = 0; f < F; ++f) {
        const recflex_feature_spec_t &s = specs[f];
        if (s.num_rows <= 0 || s.num_rows >= (int64_t(1) << 31)) return RECFLEX_ERR_INVALID_ARG;
        if (s.dim <= 0 || s.dim > 65536) return RECFLEX_ERR_INVALID_ARG;
        if (s.pool != RECFLEX_POOL_SUM && s.pool != RECFLEX_POOL_MEAN) return RECFLEX_ERR_INVALID_ARG;
        if (!(s.mean_len >= 0.f) || !(s.max_len >= 0.f) || !(s.coverage >= 0.f) || s.coverage > 1.f)
            return RECFLEX_ERR_INVALID_ARG;
        if (s.dtype < RECFLEX_DTYPE_F32 || s.dtype > RECFLEX_DTYPE_FP8) return RECFLEX_ERR_INVALID_ARG;
        if ((s.dtype == RECFLEX_DTYPE_F16 || s.dtype == RECFLEX_DTYPE_BF16) && s.dim % 4 != 0)
            return RECFLEX_ERR_INVALID_ARG;
        if ((s.dtype == RECFLEX_DTYPE_I8 || s.dtype == RECFLEX_DTYPE_FP8) && s.dim % 8 != 0)
            return RECFLEX_ERR_INVALID_ARG;
        d_tot += s.dim;
    }
    if (d_tot >= (int64_t(1) << 31) || (int64_t)max_batch * d_tot >= (int64_t(1) << 40)) return RECFLEX_ERR_INVALID_ARG;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) return RECFLEX_ERR_INVALID_ARG;
    if (cudaSetDevice(device) != cudaSuccess) return RECFLEX_ERR_CUDA;

    recflex_plan_s *p = new recflex_plan_s();
    p->device = device;
    p->F = F;
    p->max_batch = max_batch;
    p->d_tot = d_tot;
    p->specs.assign(specs, specs + F);
    cudaDeviceGetAttribute(&p->num_sms, cudaDevAttrMultiProcessorCount, device);
    p->desc.resize(F);
    p->tables.assign(F, nullptr);
    int64_t col = 0, slot = 0;
    for (int f = 0; f < F; ++f) {
        FeatureDesc &d = p->desc[f];
        std::memset(&d, 0, sizeof(d));
        d.rows = (int32_t)specs[f].num_rows;
        d.dim = specs[f].dim;
        d.col = (int32_t)col;
        d.pool = specs[f].pool;
        d.in_feature = f;
        d.dtype = specs[f].dtype;
        d.row_bytes = row_bytes_of(specs[f].dim, specs[f].dtype);
        d.cap = 0;
        d.slots = slots_for(max_batch, specs[f].max_len);
        d.slot_base = (int32_t)slot;
        slot += d.slots;
        col += specs[f].dim;
    }
    if (slot >= (int64_t(1) << 31)) {
        delete p;
        return RECFLEX_ERR_INVALID_ARG;
    }
    p->slots_total = slot;
    p->task_lookups = task_lookups_target(specs, F, max_batch, p->num_sms);
    {
        double tot = 0;
        for (int f = 0; f < F; ++f)
            tot += (double)max_batch * std::max(0.25, (double)specs[f].mean_len * std::max(0.05, (double)specs[f].coverage));
        p->small_batch = tot < 8.0 * p->num_sms * 4 * 512;
    }
    for (int f = 0; f < F; ++f) {
        recflex_schedule_t s = default_schedule(specs[f], p->task_lookups, p->small_batch);
        if (!schedule_valid_for(s, p->desc[f].dim, p->desc[f].dtype, p->desc[f].col, (int)d_tot)) {
            if (specs[f].dtype != RECFLEX_DTYPE_F32) {
                // reduced-precision entries need a 16-byte-aligned output column
                delete p;
                return RECFLEX_ERR_NOT_SUPPORTED;
            }
            s.sched_id = find_catalog(RECFLEX_FAMILY_GROUP, std::min(32, next_pow2(specs[f].dim)), 1, 1, 4);
            s.per_block = samples_per_task_default(s.sched_id, specs[f].mean_len, specs[f].coverage, p->task_lookups);
        }
        p->desc[f].sched = s.sched_id;
        p->desc[f].part = s.part;
        p->desc[f].per_block = s.per_block;
    }
    cudaError_t e = cudaSuccess;
    p->ex.F = F;
    p->ex.in_F = F;
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_desc, sizeof(FeatureDesc) * F);
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_block_start, sizeof(int32_t) * (F + 1));
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_npb_eff, sizeof(int32_t) * F);
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_need, sizeof(int32_t) * F);
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_counter, sizeof(int32_t) * 4);
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_task_start, sizeof(int32_t) * std::max<int64_t>(1, slot));
    if (e == cudaSuccess) e = cudaMalloc(&p->ex.d_part1, sizeof(int32_t) * F);
    if (e == cudaSuccess) e = cudaMemset(p->ex.d_npb_eff, 0, sizeof(int32_t) * F);
    if (e != cudaSuccess) {
        plan_free_device(p);
        delete p;
        return cuda_status(e);
    }
    {
        // default L2 policy (C36): the heuristic's evict_last part (recurring rows of
        // small tables); evict_first is left to the measured selection
        int l2 = 0;
        cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, device);
        std::vector<int32_t> pol(F);
        if (l2 > 0 && recflex_l2_policy_heuristic(p, l2, pol.data()) == RECFLEX_OK) {
            for (int32_t &v : pol)
                if (v != RECFLEX_L2_EVICT_LAST) v = RECFLEX_L2_DEFAULT;
            recflex_set_l2_policy(p, pol.data());
        }
    }
    if (const char *env = std::getenv("RECFLEX_OCCUPANCY")) {
        int k = std::atoi(env);
        if (k >= 1 && k <= kMaxOcc) p->k = k;
    }
    if (const char *env = std::getenv("RECFLEX_NO_PDL")) p->pdl = !(env[0] == '1');
    if (const char *env = std::getenv("RECFLEX_SMEM_PAD")) p->force_smem_pad = (env[0] == '1');
    *out = p;
    return RECFLEX_OK;
}

namespace {
// Makes the plan's device current for the call and restores the caller's.
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};
}  // namespace

void recflex_destroy(recflex_plan_t p) {
    if (!p) return;
    DeviceGuard guard(p->device);
    plan_free_device(p);
    delete p;
}

static recflex_status_t sync_tables(recflex_plan_s *p, const void *const *tables, cudaStream_t stream) {
    bool changed = false;
    for (int f = 0; f < p->F; ++f) {
        const void *t = tables[f];
        if (!t) return RECFLEX_ERR_INVALID_ARG;
        if (t != p->tables[f]) {
            const CatalogEntry &e = kCatalog[p->desc[f].sched];
            (void)e;
            if (((uintptr_t)t) % 32 != 0) return RECFLEX_ERR_INVALID_ARG;
            p->tables[f] = t;
            changed = true;
        }
    }
    if (changed || p->desc_dirty) return upload_desc(p, stream);
    return RECFLEX_OK;
}


recflex_status_t recflex_forward(recflex_plan_t p, const int32_t *indices, const int32_t *offsets, int32_t B,
                                 const void *const *tables, float *out, void *stream_) {
    NvtxRange nvtx("recflex_forward");
    if (!p || !tables) return RECFLEX_ERR_INVALID_ARG;
    if (B < 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    if (B == 0) return RECFLEX_OK;
    if (!indices || !offsets || !out) return RECFLEX_ERR_INVALID_ARG;
    if (((uintptr_t)out) % 16 != 0) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    recflex_status_t st = sync_tables(p, tables, stream);
    if (st != RECFLEX_OK) return st;
    EventTriple *ev = nullptr;
    EventTriple trip;
    if (p->profiling) {
        if (!p->ev_free.empty()) {
            trip = p->ev_free.back();
            p->ev_free.pop_back();
        } else {
            cudaEventCreate(&trip.e0);
            cudaEventCreate(&trip.e1);
            cudaEventCreate(&trip.e2);
        }
        ev = &trip;
    }
    st = run_pipeline(p, p->ex, indices, offsets, B, out, (int)p->d_tot, p->k, stream, ev);
    if (ev) p->ev_pending.push_back(trip);
    return st;
}

recflex_status_t recflex_forward_routed(recflex_plan_t p, const int32_t *indices, const int32_t *offsets, int32_t B,
                                        const void *const *tables, float *const *host_dst, int32_t num_dst,
                                        int32_t rows_per_dst, int32_t dst_stride, int32_t col_base, void *stream_) {
    NvtxRange nvtx("recflex_forward_routed");
    if (!p || !tables || !host_dst || num_dst <= 0 || num_dst > 1024 || rows_per_dst <= 0 || dst_stride <= 0 ||
        col_base < 0 || col_base + p->d_tot > dst_stride)
        return RECFLEX_ERR_INVALID_ARG;
    if (B < 0 || B > p->max_batch || (int64_t)num_dst * rows_per_dst != B) return RECFLEX_ERR_INVALID_ARG;
    if (B == 0) return RECFLEX_OK;
    if (!indices || !offsets) return RECFLEX_ERR_INVALID_ARG;
    // vector stores need 16-byte aligned rows / columns
    if ((dst_stride % 4) || (col_base % 4)) return RECFLEX_ERR_INVALID_ARG;
    for (int j = 0; j < num_dst; ++j)
        if (!host_dst[j] || ((uintptr_t)host_dst[j]) % 16) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    recflex_status_t st = sync_tables(p, tables, stream);
    if (st != RECFLEX_OK) return st;
    bool same = (int)p->route_cache.size() == num_dst;
    for (int j = 0; same && j < num_dst; ++j) same = p->route_cache[j] == host_dst[j];
    if (!same) {
        if ((int)p->route_cache.size() < num_dst) {
            cudaFree(p->d_route);
            p->d_route = nullptr;
            cudaError_t e = cudaMalloc(&p->d_route, sizeof(float *) * num_dst);
            if (e != cudaSuccess) return cuda_status(e);
        }
        p->route_cache.assign(host_dst, host_dst + num_dst);
        st = staged_copy(p, p->d_route, p->route_cache.data(), sizeof(float *) * num_dst, stream);
        if (st != RECFLEX_OK) return st;
    }
    Exec ex = p->ex;
    ex.out_ptrs = p->d_route;
    ex.route_rows = rows_per_dst;
    ex.col_base = col_base;
    return run_pipeline(p, ex, indices, offsets, B, host_dst[0], dst_stride, p->k, stream, nullptr);
}

recflex_status_t recflex_forward_exchange(recflex_plan_t p, const int32_t *indices, const int32_t *offsets, int32_t B,
                                          const void *const *tables, const recflex_exchange_t *x,
                                          int32_t *buffer_index, void *stream_) {
    NvtxRange nvtx("recflex_forward_exchange");
    if (!p || !tables || !x) return RECFLEX_ERR_INVALID_ARG;
    const int W = x->world;
    if (W <= 0 || W > 1024 || x->rank < 0 || x->rank >= W || x->rows_per_dst <= 0 || x->dst_stride <= 0 ||
        x->col_base < 0 || x->col_base + p->d_tot > x->dst_stride || !x->dst[0] || !x->dst[1] || !x->flags ||
        !x->local_flags)
        return RECFLEX_ERR_INVALID_ARG;
    if (B != (int64_t)W * x->rows_per_dst || B > p->max_batch || B <= 0) return RECFLEX_ERR_INVALID_ARG;
    if (!indices || !offsets) return RECFLEX_ERR_INVALID_ARG;
    if ((x->dst_stride % 4) || (x->col_base % 4)) return RECFLEX_ERR_INVALID_ARG;
    for (int b = 0; b < 2; ++b)
        for (int j = 0; j < W; ++j)
            if (!x->dst[b][j] || ((uintptr_t)x->dst[b][j]) % 16) return RECFLEX_ERR_INVALID_ARG;
    for (int j = 0; j < W; ++j)
        if (!x->flags[j]) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    recflex_status_t st = sync_tables(p, tables, stream);
    if (st != RECFLEX_OK) return st;
    // pointer tables: [2W] destinations then [W] flag arrays, cached
    std::vector<void *> want;
    for (int b = 0; b < 2; ++b)
        for (int j = 0; j < W; ++j) want.push_back(x->dst[b][j]);
    for (int j = 0; j < W; ++j) want.push_back(x->flags[j]);
    if (want != p->xroute_cache) {
        if (p->xroute_cache.size() != want.size()) {
            cudaFree(p->d_xroute);
            cudaFree(p->d_xflags);
            p->d_xroute = nullptr;
            p->d_xflags = nullptr;
            cudaError_t e = cudaMalloc(&p->d_xroute, sizeof(float *) * 2 * W);
            if (e == cudaSuccess) e = cudaMalloc(&p->d_xflags, sizeof(uint32_t *) * W);
            if (e != cudaSuccess) return cuda_status(e);
        }
        if (!p->d_xcount) {
            cudaError_t e = cudaMalloc(&p->d_xcount, sizeof(int32_t) * 4);
            if (e == cudaSuccess) e = cudaMemsetAsync(p->d_xcount, 0, sizeof(int32_t) * 4, stream);
            if (e != cudaSuccess) return cuda_status(e);
            p->x_steps = 0;
        }
        st = staged_copy(p, p->d_xroute, want.data(), sizeof(void *) * 2 * W, stream);
        if (st == RECFLEX_OK) st = staged_copy(p, p->d_xflags, want.data() + 2 * W, sizeof(void *) * W, stream);
        if (st != RECFLEX_OK) return st;
        p->xroute_cache = want;
    }
    Exec ex = p->ex;
    ex.out_ptrs = p->d_xroute;
    ex.route_rows = x->rows_per_dst;
    ex.col_base = x->col_base;
    ex.route_epoch = p->d_xcount;
    ex.route_world = W;
    st = run_pipeline(p, ex, indices, offsets, B, x->dst[0][0], x->dst_stride, p->k, stream, nullptr);
    if (st != RECFLEX_OK) return st;
    int rc = route_signal_wait_launch(p->d_xflags, x->local_flags, p->d_xcount, x->rank, W, stream);
    if (rc) return cuda_status_at((cudaError_t)rc, "exchange signal/wait kernel launch");
    if (buffer_index) *buffer_index = (int32_t)(p->x_steps & 1);
    ++p->x_steps;
    return RECFLEX_OK;
}

recflex_status_t recflex_backward(recflex_plan_t p, const int32_t *indices, const int32_t *offsets, int32_t B,
                                  const float *grad, float *const *targets, float scale, void *stream_) {
    NvtxRange nvtx("recflex_backward");
    if (!p || !targets || B < 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    if (B == 0) return RECFLEX_OK;
    if (!indices || !offsets || !grad || ((uintptr_t)grad) % 16) return RECFLEX_ERR_INVALID_ARG;
    for (int f = 0; f < p->F; ++f)
        if (!targets[f] || ((uintptr_t)targets[f]) % 16) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    // the task map reads the descriptors (schedules, part); tables are not read
    if (p->desc_dirty) {
        recflex_status_t st = upload_desc(p, stream);
        if (st != RECFLEX_OK) return st;
    }
    bool same = (int)p->targets_cache.size() == p->F;
    for (int f = 0; same && f < p->F; ++f) same = p->targets_cache[f] == targets[f];
    if (!same) {
        if (!p->d_targets) {
            cudaError_t e = cudaMalloc(&p->d_targets, sizeof(float *) * p->F);
            if (e != cudaSuccess) return cuda_status(e);
        }
        p->targets_cache.assign(targets, targets + p->F);
        std::vector<float *> tv(p->F);  // device table in task order (C35)
        for (int e = 0; e < p->F; ++e) tv[e] = p->targets_cache[feature_at(p, e)];
        recflex_status_t st = staged_copy(p, p->d_targets, tv.data(), sizeof(float *) * p->F, stream);
        if (st != RECFLEX_OK) return st;
    }
    Exec ex = p->ex;
    ex.backward = true;
    ex.grad = grad;
    ex.d_targets = p->d_targets;
    ex.bscale = scale;
    int vec_ok = (p->d_tot % 4) == 0;
    for (int f = 0; f < p->F && vec_ok; ++f)
        if (p->desc[f].dim % 4 == 0 && p->desc[f].col % 4 != 0) vec_ok = 0;
    ex.bvec = vec_ok;
    return run_pipeline(p, ex, indices, offsets, B, nullptr, (int)p->d_tot, p->k, stream, nullptr);
}

recflex_status_t recflex_ipc_get_handle(const void *d_ptr, void *handle64) {
    if (!d_ptr || !handle64) return RECFLEX_ERR_INVALID_ARG;
    cudaIpcMemHandle_t h;
    cudaError_t e = cudaIpcGetMemHandle(&h, const_cast<void *>(d_ptr));
    if (e != cudaSuccess) return cuda_status_at(e, "cudaIpcGetMemHandle");
    static_assert(sizeof(h) == 64, "IPC handle size");
    std::memcpy(handle64, &h, 64);
    return RECFLEX_OK;
}

recflex_status_t recflex_ipc_open_handle(const void *handle64, void **d_ptr) {
    if (!handle64 || !d_ptr) return RECFLEX_ERR_INVALID_ARG;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle64, 64);
    cudaError_t e = cudaIpcOpenMemHandle(d_ptr, h, cudaIpcMemLazyEnablePeerAccess);
    return cuda_status_at(e, "cudaIpcOpenMemHandle");
}

recflex_status_t recflex_device_alloc(size_t bytes, int32_t device, void **d_ptr) {
    if (!d_ptr || bytes == 0) return RECFLEX_ERR_INVALID_ARG;
    cudaError_t e = cudaSetDevice(device);
    if (e == cudaSuccess) e = cudaMalloc(d_ptr, bytes);
    return cuda_status_at(e, "cudaMalloc");
}

recflex_status_t recflex_device_free(void *d_ptr) {
    if (!d_ptr) return RECFLEX_ERR_INVALID_ARG;
    return cuda_status_at(cudaFree(d_ptr), "cudaFree");
}

recflex_status_t recflex_ipc_close(void *d_ptr) {
    if (!d_ptr) return RECFLEX_ERR_INVALID_ARG;
    return cuda_status_at(cudaIpcCloseMemHandle(d_ptr), "cudaIpcCloseMemHandle");
}

recflex_status_t recflex_forward_host(recflex_plan_t p, const int32_t *h_indices, int64_t nnz, const int32_t *h_offsets,
                                      int32_t B, const void *const *tables, float *h_out, void *stream_) {
    if (!p || !tables || B < 0 || B > p->max_batch || nnz < 0) return RECFLEX_ERR_INVALID_ARG;
    if (B == 0) return RECFLEX_OK;
    if (!h_offsets || !h_out || (nnz > 0 && !h_indices)) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    const int64_t n_off = (int64_t)p->F * B + 1;
    const int64_t n_out = (int64_t)B * p->d_tot;
    cudaError_t e = cudaSuccess;
    if (nnz > p->stage_idx_cap) {
        cudaFree(p->d_stage_idx);
        p->d_stage_idx = nullptr;
        e = cudaMalloc(&p->d_stage_idx, sizeof(int32_t) * std::max<int64_t>(nnz, 1));
        if (e != cudaSuccess) return cuda_status(e);
        p->stage_idx_cap = nnz;
    }
    if (!p->d_stage_idx) {
        e = cudaMalloc(&p->d_stage_idx, sizeof(int32_t));
        if (e != cudaSuccess) return cuda_status(e);
    }
    if (n_off > p->stage_off_cap) {
        cudaFree(p->d_stage_off);
        e = cudaMalloc(&p->d_stage_off, sizeof(int32_t) * n_off);
        if (e != cudaSuccess) return cuda_status(e);
        p->stage_off_cap = n_off;
    }
    if (n_out > p->stage_out_cap) {
        cudaFree(p->d_stage_out);
        e = cudaMalloc(&p->d_stage_out, sizeof(float) * n_out);
        if (e != cudaSuccess) return cuda_status(e);
        p->stage_out_cap = n_out;
    }
    if (nnz > 0) e = cudaMemcpyAsync(p->d_stage_idx, h_indices, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice, stream);
    if (e == cudaSuccess)
        e = cudaMemcpyAsync(p->d_stage_off, h_offsets, sizeof(int32_t) * n_off, cudaMemcpyHostToDevice, stream);
    if (e != cudaSuccess) return cuda_status(e);
    recflex_status_t st = recflex_forward(p, p->d_stage_idx, p->d_stage_off, B, tables, p->d_stage_out, stream);
    if (st != RECFLEX_OK) return st;
    e = cudaMemcpyAsync(h_out, p->d_stage_out, sizeof(float) * n_out, cudaMemcpyDeviceToHost, stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    return cuda_status(e);
}

recflex_status_t recflex_get_schedule(recflex_plan_t p, int32_t f, recflex_schedule_t *s, int32_t *blocks_per_sm) {
    if (!p || f < 0 || f >= p->F) return RECFLEX_ERR_INVALID_ARG;
    if (s) {
        s->sched_id = p->desc[f].sched;
        s->part = p->desc[f].part;
        s->per_block = p->desc[f].per_block;
        s->static_blocks = p->desc[f].nalloc;
    }
    if (blocks_per_sm) *blocks_per_sm = p->k;
    return RECFLEX_OK;
}

recflex_status_t recflex_set_schedule(recflex_plan_t p, int32_t f, const recflex_schedule_t *s) {
    if (!p || !s || f < 0 || f >= p->F) return RECFLEX_ERR_INVALID_ARG;
    if (!schedule_valid_for(*s, p->desc[f].dim, p->desc[f].dtype, p->desc[f].col, (int)p->d_tot))
        return RECFLEX_ERR_INVALID_ARG;
    // a compiled JIT kernel no longer matches if the entry or the presence of a
    // static mapping (compiled in only when used) changes
    if (p->desc[f].sched != s->sched_id || (p->desc[f].nalloc > 0) != (s->static_blocks > 0)) ++p->sched_version;
    p->num_static += (s->static_blocks > 0 ? 1 : 0) - (p->desc[f].nalloc > 0 ? 1 : 0);
    p->desc[f].sched = s->sched_id;
    p->desc[f].part = s->part;
    p->desc[f].per_block = s->per_block;
    p->desc[f].nalloc = s->static_blocks;
    p->desc_dirty = true;
    return RECFLEX_OK;
}

recflex_status_t recflex_set_occupancy(recflex_plan_t p, int32_t k) {
    if (!p || k < 1 || k > kMaxOcc) return RECFLEX_ERR_INVALID_ARG;
    p->k = k;
    return RECFLEX_OK;
}

recflex_status_t recflex_get_occupancy(recflex_plan_t p, int32_t *k) {
    if (!p || !k) return RECFLEX_ERR_INVALID_ARG;
    *k = p->k;
    return RECFLEX_OK;
}

recflex_status_t recflex_occupancy_check(int32_t device, int32_t k, int32_t *active, int32_t *regs, int32_t *spill) {
    if (k < 1 || k > kMaxOcc) return RECFLEX_ERR_INVALID_ARG;
    recflex_feature_spec_t spec = {1000, 16, 0, 1.f, 1.f, 1.f, 0};
    recflex_plan_t p = nullptr;
    recflex_status_t st = recflex_plan_create(&spec, 1, 1, device, &p);
    if (st != RECFLEX_OK) return st;
    st = prepare_occupancy(p, k);
    if (st == RECFLEX_OK) {
        int b = 0, r = 0, s = 0;
        int rc = fused_occupancy(k, p->smem[k], &b, &r, &s);
        if (rc) st = cuda_status((cudaError_t)rc);
        if (active) *active = b;
        if (regs) *regs = r;
        if (spill) *spill = s;
    }
    recflex_destroy(p);
    return st;
}

recflex_status_t recflex_debug_task_map(recflex_plan_t p, const int32_t *offsets, int32_t B, int32_t *h_bs,
                                        int32_t *h_ranges, int64_t cap, void *stream_) {
    if (!p || !offsets || !h_bs || B < 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    if (p->desc_dirty || p->ex.num_part1 != 0 || true) {
        // descriptors may be stale if no forward ran yet (tables not known): upload with null tables
        for (int f = 0; f < p->F; ++f) p->desc[f].table = p->tables[f];
        recflex_status_t st = upload_desc(p, stream);
        if (st != RECFLEX_OK) return st;
    }
    MapArgs ma;
    ma.desc = p->ex.d_desc;
    ma.offsets = offsets;
    ma.F = p->F;
    ma.B = B;
    ma.in_F = p->F;
    ma.block_start = p->ex.d_block_start;
    ma.npb_eff = p->ex.d_npb_eff;
    ma.need = p->ex.d_need;
    ma.counter = p->ex.d_counter;
    int rc = map_launch(ma, stream);
    if (rc) return cuda_status((cudaError_t)rc);
    if (p->ex.num_part1 > 0 && B > 0) {
        FillArgs fa;
        fa.desc = p->ex.d_desc;
        fa.offsets = offsets;
        fa.block_start = p->ex.d_block_start;
        fa.npb_eff = p->ex.d_npb_eff;
        fa.need = p->ex.d_need;
        fa.part1_features = p->ex.d_part1;
        fa.num_part1 = p->ex.num_part1;
        fa.B = B;
        fa.task_start = p->ex.d_task_start;
        rc = fill_launch(fa, B, false, stream);
        if (rc) return cuda_status((cudaError_t)rc);
    }
    cudaError_t e = cudaMemcpyAsync(h_bs, p->ex.d_block_start, sizeof(int32_t) * (p->F + 1), cudaMemcpyDeviceToHost,
                                    stream);
    if (e == cudaSuccess) e = cudaStreamSynchronize(stream);
    if (e != cudaSuccess) return cuda_status(e);
    if (h_ranges) {
        const int64_t total = h_bs[p->F];
        if (cap < 2 * total) return RECFLEX_ERR_INVALID_ARG;
        std::vector<int32_t> ts;
        if (p->slots_total > 0) {
            ts.resize(p->slots_total);
            e = cudaMemcpy(ts.data(), p->ex.d_task_start, sizeof(int32_t) * p->slots_total, cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) return cuda_status(e);
        }
        for (int e = 0; e < p->F; ++e) {
            const int f = feature_at(p, e);  // block_start lists task-order positions (C35)
            for (int64_t t = h_bs[e]; t < h_bs[e + 1]; ++t) {
                const int rel = (int)(t - h_bs[e]);
                if (p->desc[f].part == 1 && p->desc[f].nalloc == 0) {
                    h_ranges[2 * t] = ts[p->desc[f].slot_base + rel];
                    h_ranges[2 * t + 1] = ts[p->desc[f].slot_base + rel + 1];
                } else {
                    h_ranges[2 * t] = -1;
                    h_ranges[2 * t + 1] = -1;
                }
            }
        }
    }
    return RECFLEX_OK;
}

recflex_status_t recflex_get_task_slots(recflex_plan_t p, int32_t f, int32_t *slots) {
    if (!p || !slots || f < 0 || f >= p->F) return RECFLEX_ERR_INVALID_ARG;
    *slots = p->desc[f].slots;
    return RECFLEX_OK;
}

recflex_status_t recflex_debug_task_need(recflex_plan_t p, int32_t *host_need) {
    if (!p || !host_need) return RECFLEX_ERR_INVALID_ARG;
    DeviceGuard guard(p->device);
    std::vector<int32_t> need(p->F);
    cudaError_t e = cudaMemcpy(need.data(), p->ex.d_need, sizeof(int32_t) * p->F, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return cuda_status(e);
    for (int i = 0; i < p->F; ++i) host_need[feature_at(p, i)] = need[i];  // back to feature order
    return RECFLEX_OK;
}

recflex_status_t recflex_set_task_order(recflex_plan_t p, const int32_t *order) {
    if (!p) return RECFLEX_ERR_INVALID_ARG;
    DeviceGuard guard(p->device);
    return apply_task_order(p, order);
}

recflex_status_t recflex_set_column_order(recflex_plan_t p, int32_t follow_task_order) {
    if (!p || follow_task_order < 0 || follow_task_order > 1) return RECFLEX_ERR_INVALID_ARG;
    DeviceGuard guard(p->device);
    if ((follow_task_order != 0) == p->columns_follow_order) return RECFLEX_OK;
    return set_layout(p, p->order, follow_task_order != 0, nullptr);
}

recflex_status_t recflex_set_l2_policy(recflex_plan_t p, const int32_t *policy) {
    if (!p) return RECFLEX_ERR_INVALID_ARG;
    std::vector<int8_t> l2;
    if (policy) {
        bool any = false;
        for (int f = 0; f < p->F; ++f) {
            if (policy[f] < RECFLEX_L2_DEFAULT || policy[f] > RECFLEX_L2_KEEP_L1) return RECFLEX_ERR_INVALID_ARG;
            any = any || policy[f] != RECFLEX_L2_DEFAULT;
        }
        if (any) l2.assign(policy, policy + p->F);
    }
    if (l2 != p->l2) {
        p->l2.swap(l2);
        ++p->sched_version;  // the plan-specialised kernel compiles the policies in
    }
    return RECFLEX_OK;
}

recflex_status_t recflex_get_l2_policy(recflex_plan_t p, int32_t *policy) {
    if (!p || !policy) return RECFLEX_ERR_INVALID_ARG;
    for (int f = 0; f < p->F; ++f) policy[f] = p->l2.empty() ? 0 : p->l2[f];
    return RECFLEX_OK;
}

recflex_status_t recflex_l2_policy_heuristic(recflex_plan_t p, int64_t l2_bytes, int32_t *policy) {
    if (!p || !policy || l2_bytes <= 0) return RECFLEX_ERR_INVALID_ARG;
    for (int f = 0; f < p->F; ++f) {
        const recflex_feature_spec_t &sp = p->specs[f];
        const double table = (double)sp.num_rows * (double)p->desc[f].row_bytes;
        const double lookups = (double)p->max_batch * (double)sp.mean_len * (double)sp.coverage;
        const double reuse = lookups / std::max(1.0, (double)sp.num_rows);  // lookups per row per batch
        int pol = RECFLEX_L2_DEFAULT;
        if (table <= 0.25 * (double)l2_bytes && reuse >= 1.0) pol = RECFLEX_L2_EVICT_LAST;
        else if (table >= (double)l2_bytes || reuse < 0.5) pol = RECFLEX_L2_EVICT_FIRST;
        policy[f] = pol;
    }
    return RECFLEX_OK;
}

recflex_status_t recflex_get_columns(recflex_plan_t p, int64_t *col) {
    if (!p || !col) return RECFLEX_ERR_INVALID_ARG;
    for (int f = 0; f < p->F; ++f) col[f] = p->desc[f].col;
    return RECFLEX_OK;
}

recflex_status_t recflex_get_task_order(recflex_plan_t p, int32_t *order) {
    if (!p || !order) return RECFLEX_ERR_INVALID_ARG;
    for (int e = 0; e < p->F; ++e) order[e] = feature_at(p, e);
    return RECFLEX_OK;
}

recflex_status_t recflex_task_order_heuristic(recflex_plan_t p, int32_t kind, int32_t *order) {
    if (!p || !order || kind < 0 || kind >= RECFLEX_NUM_ORDERS) return RECFLEX_ERR_INVALID_ARG;
    std::vector<int32_t> o;
    task_order_of_kind(p, kind, o);
    std::copy(o.begin(), o.end(), order);
    return RECFLEX_OK;
}

// Measured task granularity (C37): every feature's tasks scaled by 1, 1/2 or 2
// (samples per task for sample-partitioned schedules, lookups per task for
// lookup-partitioned ones, at least 16), the task order re-derived if it is a
// heuristic's; the fastest scale is kept (ties: 1, then 1/2, then 2).
recflex_status_t recflex_select_task_size(recflex_plan_t p, const int32_t *indices, const int32_t *offsets,
                                          int32_t B, const void *const *tables, int32_t reps, int32_t *chosen,
                                          float *ms_out, void *stream_) {
    if (!p || !indices || !offsets || !tables || B <= 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    NvtxRange nvtx("recflex_select_task_size");
    DeviceGuard guard(p->device);
    cudaStream_t stream = (cudaStream_t)stream_;
    // which heuristic (if any) the current order is, to re-derive it per candidate
    int kind = -1;
    for (int k = 0; k < RECFLEX_NUM_ORDERS && kind < 0; ++k) {
        std::vector<int32_t> o;
        task_order_of_kind(p, k, o);
        std::vector<int32_t> cur(p->F);
        for (int e = 0; e < p->F; ++e) cur[e] = feature_at(p, e);
        if (o == cur) kind = k;
    }
    const std::vector<int32_t> keep_order = p->order;
    std::vector<recflex_schedule_t> base(p->F);
    for (int f = 0; f < p->F; ++f) base[f] = {p->desc[f].sched, p->desc[f].part, p->desc[f].per_block, p->desc[f].nalloc};
    const int num = 2, den[3] = {2, 4, 1};  // scale = num / den: 1, 1/2, 2
    auto scaled = [&](int c) {
        std::vector<recflex_schedule_t> ss = base;
        for (auto &x : ss) {
            const int64_t v = (int64_t)x.per_block * num / den[c];
            x.per_block = (int32_t)std::max<int64_t>(x.part == 1 ? 16 : 1, std::min<int64_t>(v, 1 << 30));
        }
        return ss;
    };
    auto apply = [&](int c) -> recflex_status_t {
        std::vector<int32_t> o = keep_order;
        std::vector<recflex_schedule_t> ss = scaled(c);
        // schedules first (columns unchanged), then the re-derived order
        recflex_status_t st = set_layout(p, p->order, p->columns_follow_order, &ss);
        if (st != RECFLEX_OK || kind < 0) return st;
        task_order_of_kind(p, kind, o);
        return apply_task_order(p, o.data());
    };
    float *out = nullptr, *flush = nullptr;
    const size_t flush_bytes = size_t(256) << 20;  // 2x L2
    cudaError_t e = cudaMalloc(&out, sizeof(float) * (size_t)B * p->d_tot);
    if (e == cudaSuccess) e = cudaMalloc(&flush, flush_bytes);
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    recflex_status_t st = e == cudaSuccess ? RECFLEX_OK : cuda_status(e);
    if (st == RECFLEX_OK && p->use_jit && !jit_ready(p, p->k)) {
        int k = p->k;
        st = jit_compile_plan(p, &k, 1);  // per-task sizes are not compiled in: one kernel serves all scales
    }
    float med[3] = {0.f, 0.f, 0.f};
    for (int c = 0; c < 3 && st == RECFLEX_OK; ++c) {
        st = apply(c);
        std::vector<float> ms;
        for (int r = 0; r < std::max(3, reps) + 1 && st == RECFLEX_OK; ++r) {
            flush_launch(flush, flush_bytes, stream);
            cudaEventRecord(e0, stream);
            st = recflex_forward(p, indices, offsets, B, tables, out, stream);
            cudaEventRecord(e1, stream);
            e = cudaEventSynchronize(e1);
            if (e != cudaSuccess) st = cuda_status(e);
            float t = 0;
            cudaEventElapsedTime(&t, e0, e1);
            if (r > 0) ms.push_back(t);
        }
        if (!ms.empty()) {
            std::sort(ms.begin(), ms.end());
            med[c] = ms[ms.size() / 2];
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(out);
    cudaFree(flush);
    int best = 0;
    if (st == RECFLEX_OK)
        for (int c = 1; c < 3; ++c)
            if (med[c] < med[best]) best = c;
    if (st != RECFLEX_OK) {
        set_layout(p, keep_order, p->columns_follow_order, &base);
        return st;
    }
    st = apply(best);
    if (st != RECFLEX_OK) return st;
    if (chosen) *chosen = best;
    if (ms_out)
        for (int c = 0; c < 3; ++c) ms_out[c] = med[c];
    return RECFLEX_OK;
}

// Measured choice among the task-order heuristics (C35): time the plan's
// current kernel under each order on the caller's batch (median of reps
// forwards, L2 flushed before each), keep the fastest (ties: the lower kind).
recflex_status_t recflex_select_task_order(recflex_plan_t p, const int32_t *indices, const int32_t *offsets,
                                           int32_t B, const void *const *tables, int32_t reps, int32_t *chosen,
                                           float *ms_out, void *stream_) {
    if (!p || !indices || !offsets || !tables || B <= 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    NvtxRange nvtx("recflex_select_task_order");
    DeviceGuard guard(p->device);
    cudaStream_t stream = (cudaStream_t)stream_;
    if (p->use_jit && !jit_ready(p, p->k)) {
        int k = p->k;
        recflex_status_t st = jit_compile_plan(p, &k, 1);
        if (st != RECFLEX_OK) return st;
    }
    float *out = nullptr, *flush = nullptr;
    const size_t flush_bytes = size_t(256) << 20;  // 2x L2
    cudaError_t e = cudaMalloc(&out, sizeof(float) * (size_t)B * p->d_tot);
    if (e == cudaSuccess) e = cudaMalloc(&flush, flush_bytes);
    cudaEvent_t e0 = nullptr, e1 = nullptr;
    if (e == cudaSuccess) e = cudaEventCreate(&e0);
    if (e == cudaSuccess) e = cudaEventCreate(&e1);
    recflex_status_t st = e == cudaSuccess ? RECFLEX_OK : cuda_status(e);
    const std::vector<int32_t> keep = p->order;
    float med[RECFLEX_NUM_ORDERS] = {0.f};
    std::vector<std::vector<int32_t>> orders(RECFLEX_NUM_ORDERS);
    for (int kind = 0; kind < RECFLEX_NUM_ORDERS && st == RECFLEX_OK; ++kind) {
        task_order_of_kind(p, kind, orders[kind]);
        st = apply_task_order(p, orders[kind].data());
        std::vector<float> ms;
        for (int r = 0; r < std::max(3, reps) + 1 && st == RECFLEX_OK; ++r) {
            flush_launch(flush, flush_bytes, stream);
            cudaEventRecord(e0, stream);
            st = recflex_forward(p, indices, offsets, B, tables, out, stream);
            cudaEventRecord(e1, stream);
            e = cudaEventSynchronize(e1);
            if (e != cudaSuccess) st = cuda_status(e);
            float t = 0;
            cudaEventElapsedTime(&t, e0, e1);
            if (r > 0) ms.push_back(t);
        }
        if (!ms.empty()) {
            std::sort(ms.begin(), ms.end());
            med[kind] = ms[ms.size() / 2];
        }
    }
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(out);
    cudaFree(flush);
    if (st != RECFLEX_OK) {
        apply_task_order(p, keep.empty() ? nullptr : keep.data());
        return st;
    }
    int best = 0;
    for (int kind = 1; kind < RECFLEX_NUM_ORDERS; ++kind)
        if (med[kind] < med[best]) best = kind;
    st = apply_task_order(p, orders[best].data());
    if (st != RECFLEX_OK) return st;
    if (chosen) *chosen = best;
    if (ms_out)
        for (int kind = 0; kind < RECFLEX_NUM_ORDERS; ++kind) ms_out[kind] = med[kind];
    return RECFLEX_OK;
}

recflex_status_t recflex_validate(recflex_plan_t p, const int32_t *indices, const int32_t *offsets, int32_t B,
                                  void *stream_) {
    if (!p || !offsets || B < 0 || B > p->max_batch) return RECFLEX_ERR_INVALID_ARG;
    if (B == 0) return RECFLEX_OK;
    cudaStream_t stream = (cudaStream_t)stream_;
    DeviceGuard guard(p->device);
    recflex_status_t st = upload_desc(p, stream);
    if (st != RECFLEX_OK) return st;
    int32_t *d_flag = nullptr;
    cudaError_t e = cudaMalloc(&d_flag, sizeof(int32_t));
    if (e != cudaSuccess) return cuda_status(e);
    cudaMemsetAsync(d_flag, 0, sizeof(int32_t), stream);
    // offsets first (a broken CSR would make the index ranges meaningless)
    int rc = validate_launch(p->ex.d_desc, 0, p->F, indices, offsets, B, d_flag, stream);
    int32_t flag = 0;
    if (!rc) e = cudaMemcpyAsync(&flag, d_flag, sizeof(int32_t), cudaMemcpyDeviceToHost, stream);
    if (!rc && e == cudaSuccess) e = cudaStreamSynchronize(stream);
    if (rc || e != cudaSuccess) {
        cudaFree(d_flag);
        return rc ? cuda_status((cudaError_t)rc) : cuda_status(e);
    }
    if (flag & 1) {
        cudaFree(d_flag);
        return RECFLEX_ERR_INVALID_ARG;
    }
    if (!indices) {
        cudaFree(d_flag);
        return RECFLEX_ERR_INVALID_ARG;
    }
    rc = validate_launch(p->ex.d_desc, p->F, p->F, indices, offsets, B, d_flag, stream);
    if (!rc) e = cudaMemcpyAsync(&flag, d_flag, sizeof(int32_t), cudaMemcpyDeviceToHost, stream);
    if (!rc && e == cudaSuccess) e = cudaStreamSynchronize(stream);
    cudaFree(d_flag);
    if (rc) return cuda_status((cudaError_t)rc);
    if (e != cudaSuccess) return cuda_status(e);
    if (flag & 1) return RECFLEX_ERR_INVALID_ARG;
    if (flag & 2) return RECFLEX_ERR_INDEX_OOB;
    return RECFLEX_OK;
}

recflex_status_t recflex_set_profiling(recflex_plan_t p, int32_t enable) {
    if (!p) return RECFLEX_ERR_INVALID_ARG;
    p->profiling = enable != 0;
    return RECFLEX_OK;
}

recflex_status_t recflex_get_kernel_times(recflex_plan_t p, double *map_ms, double *fused_ms, int64_t *forwards,
                                          int32_t reset) {
    if (!p) return RECFLEX_ERR_INVALID_ARG;
    for (auto &t : p->ev_pending) {
        cudaError_t e = cudaEventSynchronize(t.e2);
        if (e != cudaSuccess) return cuda_status(e);
        float a = 0, b = 0;
        cudaEventElapsedTime(&a, t.e0, t.e1);
        cudaEventElapsedTime(&b, t.e1, t.e2);
        p->map_ms += a;
        p->fused_ms += b;
        p->forwards += 1;
        p->ev_free.push_back(t);
    }
    p->ev_pending.clear();
    if (map_ms) *map_ms = p->map_ms;
    if (fused_ms) *fused_ms = p->fused_ms;
    if (forwards) *forwards = p->forwards;
    if (reset) {
        p->map_ms = p->fused_ms = 0;
        p->forwards = 0;
    }
    return RECFLEX_OK;
}

// Fingerprint of the first n catalog entries (family, ET, G, VEC, C, U): a plan
// names schedules by catalog id, so an import must see the same entries.
static uint64_t catalog_fingerprint(int n) {
    uint64_t h = 1469598103934665603ull;
    for (int i = 0; i < n && i < kCatalogSize; ++i) {
        const CatalogEntry &e = kCatalog[i];
        const int v[6] = {e.family, e.ET, e.G, e.VEC, e.C, e.U};
        for (int x : v) {
            h ^= (uint64_t)(uint32_t)x;
            h *= 1099511628211ull;
        }
    }
    return h & 0xffffffffffffull;  // 48 bits: exact in a JSON number
}

recflex_status_t recflex_plan_export(recflex_plan_t p, char *buf, size_t cap, size_t *len) {
    if (!p) return RECFLEX_ERR_INVALID_ARG;
    std::string s = "{\"abi\": " + std::to_string(RECFLEX_ABI_VERSION) + ", \"catalog_size\": " +
                    std::to_string(kCatalogSize) + ", \"catalog_fingerprint\": " +
                    std::to_string(catalog_fingerprint(kCatalogSize)) + ", \"num_features\": " +
                    std::to_string(p->F) + ", \"occupancy\": " + std::to_string(p->k) + ", \"schedules\": [";
    for (int f = 0; f < p->F; ++f) {
        if (f) s += ", ";
        s += "[" + std::to_string(p->desc[f].sched) + ", " + std::to_string(p->desc[f].part) + ", " +
             std::to_string(p->desc[f].per_block);
        if (p->desc[f].nalloc > 0) s += ", " + std::to_string(p->desc[f].nalloc);
        s += "]";
    }
    s += "]";
    if (!p->order.empty()) {
        s += ", \"order\": [";
        for (int e = 0; e < p->F; ++e) s += (e ? ", " : "") + std::to_string(p->order[e]);
        s += "]";
    }
    if (p->columns_follow_order) s += ", \"columns\": \"task-order\"";
    if (!p->l2.empty()) {
        s += ", \"l2\": [";
        for (int f = 0; f < p->F; ++f) s += (f ? ", " : "") + std::to_string((int)p->l2[f]);
        s += "]";
    }
    s += ", \"kernel\": \"";
    s += p->use_jit ? "plan-specialised" : "catalog";
    s += "\"}";
    if (len) *len = s.size() + 1;
    if (buf && cap > 0) {
        size_t n = std::min(cap - 1, s.size());
        std::memcpy(buf, s.data(), n);
        buf[n] = '\0';
        if (cap < s.size() + 1) return RECFLEX_ERR_INVALID_ARG;
    }
    return RECFLEX_OK;
}

static bool parse_int_after(const char *&c, long *v) {
    while (*c && !(*c == '-' || (*c >= '0' && *c <= '9'))) {
        if (*c == ']' || *c == '}') return false;
        ++c;
    }
    if (!*c) return false;
    char *end = nullptr;
    *v = std::strtol(c, &end, 10);
    c = end;
    return true;
}

recflex_status_t recflex_plan_import(recflex_plan_t p, const char *json) {
    if (!p || !json) return RECFLEX_ERR_INVALID_ARG;
    const char *c = std::strstr(json, "\"catalog_size\"");
    long v = 0;
    if (!c) return RECFLEX_ERR_INVALID_ARG;
    c += 14;
    // the catalog is append-only: a plan exported with a smaller catalog names
    // the same entries
    if (!parse_int_after(c, &v) || v < 1 || v > kCatalogSize) return RECFLEX_ERR_NOT_SUPPORTED;
    const int exported_catalog = (int)v;
    if (const char *fp = std::strstr(json, "\"catalog_fingerprint\"")) {
        fp += 21;
        while (*fp && (*fp < '0' || *fp > '9')) ++fp;
        const unsigned long long got = std::strtoull(fp, nullptr, 10);
        if (got != catalog_fingerprint(exported_catalog)) {
            set_last_error("plan import: catalog fingerprint mismatch (the plan names other schedules)");
            return RECFLEX_ERR_NOT_SUPPORTED;
        }
    }
    c = std::strstr(json, "\"num_features\"");
    if (!c) return RECFLEX_ERR_INVALID_ARG;
    c += 14;
    if (!parse_int_after(c, &v) || v != p->F) return RECFLEX_ERR_INVALID_ARG;
    c = std::strstr(json, "\"occupancy\"");
    if (!c) return RECFLEX_ERR_INVALID_ARG;
    c += 11;
    if (!parse_int_after(c, &v) || v < 1 || v > kMaxOcc) return RECFLEX_ERR_INVALID_ARG;
    const int k = (int)v;
    c = std::strstr(json, "\"schedules\"");
    if (!c) return RECFLEX_ERR_INVALID_ARG;
    c = std::strchr(c, '[');
    if (!c) return RECFLEX_ERR_INVALID_ARG;
    ++c;
    std::vector<recflex_schedule_t> ss(p->F);
    for (int f = 0; f < p->F; ++f) {
        c = std::strchr(c, '[');
        if (!c) return RECFLEX_ERR_INVALID_ARG;
        ++c;
        long a = 0, b = 0, d = 0, st = 0;
        if (!parse_int_after(c, &a) || !parse_int_after(c, &b) || !parse_int_after(c, &d))
            return RECFLEX_ERR_INVALID_ARG;
        const char *save = c;
        if (!parse_int_after(c, &st)) {  // optional 4th entry: static_blocks
            st = 0;
            c = save;
        }
        ss[f] = {(int32_t)a, (int32_t)b, (int32_t)d, (int32_t)st};
    }
    // optional: the task order and column layout (C35); absent = feature order
    std::vector<int32_t> order;
    if (const char *oc = std::strstr(json, "\"order\"")) {
        oc = std::strchr(oc, '[');
        if (!oc) return RECFLEX_ERR_INVALID_ARG;
        ++oc;
        std::vector<int32_t> raw(p->F);
        for (int e = 0; e < p->F; ++e) {
            long f = 0;
            if (!parse_int_after(oc, &f) || f < 0 || f >= p->F) return RECFLEX_ERR_INVALID_ARG;
            raw[e] = (int32_t)f;
        }
        if (normalize_order(p, raw.data(), order) != RECFLEX_OK) return RECFLEX_ERR_INVALID_ARG;
    }
    // optional: L2 eviction priorities (C36); absent = default everywhere
    std::vector<int32_t> l2;
    if (const char *lc = std::strstr(json, "\"l2\"")) {
        lc = std::strchr(lc, '[');
        if (!lc) return RECFLEX_ERR_INVALID_ARG;
        ++lc;
        l2.resize(p->F);
        for (int f = 0; f < p->F; ++f) {
            long v = 0;
            if (!parse_int_after(lc, &v) || v < 0 || v > RECFLEX_L2_KEEP_L1) return RECFLEX_ERR_INVALID_ARG;
            l2[f] = (int32_t)v;
        }
    }
    bool follow = false;
    if (const char *cc = std::strstr(json, "\"columns\"")) {
        const char *v = std::strchr(cc + 9, '"');
        follow = v && !std::strncmp(v, "\"task-order\"", 12);
    }
    {
        DeviceGuard guard(p->device);
        recflex_status_t st = set_layout(p, order, follow, &ss);  // validates every schedule at its column
        if (st != RECFLEX_OK) return st;
    }
    recflex_set_l2_policy(p, l2.empty() ? nullptr : l2.data());
    p->k = k;
    // optional: which kernel the plan runs (recflex_select_kernel's choice)
    if (const char *kc = std::strstr(json, "\"kernel\"")) {
        const char *v = std::strchr(kc + 8, '"');  // opening quote of the value
        if (v && !std::strncmp(v, "\"catalog\"", 9)) p->use_jit = false;
        else if (v && !std::strncmp(v, "\"plan-specialised\"", 18)) p->use_jit = true;
    }
    return RECFLEX_OK;
}

recflex_status_t recflex_shard_concat(const float *recv, int32_t W, int32_t rows, const int32_t *host_dims, float *out,
                                      void *stream_) {
    if (!recv || !out || !host_dims || W <= 0 || W > kMaxConcatRanks || rows < 0) return RECFLEX_ERR_INVALID_ARG;
    ConcatArgs a;
    a.W = W;
    a.rows = rows;
    int64_t tot = 0;
    for (int i = 0; i < W; ++i) {
        if (host_dims[i] < 0) return RECFLEX_ERR_INVALID_ARG;
        a.dims[i] = host_dims[i];
        a.cols[i] = (int32_t)tot;
        tot += host_dims[i];
    }
    if (tot >= (int64_t(1) << 31)) return RECFLEX_ERR_INVALID_ARG;
    a.d_tot = (int32_t)tot;
    int rc = concat_launch(recv, a, out, stream_);
    if (rc) return cuda_status((cudaError_t)rc);
    return RECFLEX_OK;
}

recflex_status_t recflex_l2_flush(void *buf, size_t bytes, void *stream_) {
    if (!buf) return RECFLEX_ERR_INVALID_ARG;
    int rc = flush_launch(buf, bytes, stream_);
    return rc ? cuda_status((cudaError_t)rc) : RECFLEX_OK;
}

}  // extern "C"
