/*
 * recflex.h -- C ABI of the B200-native RecFlex hot path (librecflex.so).
 *
 * The operation (PAPER.md "P:n" = line n of the paper text):
 *   For every feature field f and sample s, gather the rows of table T_f named
 *   by the lookup IDs of bag (f, s) and pool them by elementwise reduction
 *   (§II-A, Fig. 1); per-feature results are concatenated.
 *   Each field runs its own schedule inside ONE fused kernel (§IV-B, Fig. 8,
 *   P:168-234); schedules are chosen by the two-stage interference-simulated
 *   tuner (§IV-A, Eq. 1-5); the block-to-feature map is computed
 *   per batch from the offsets -- here by a device-side scan, with
 *   no host round trip.
 *
 * Conventions for every entry point:
 *   - Pointers named d_* / documented "device" are CUDA device pointers on the
 *     plan's device; "host" pointers are ordinary (ideally pinned) host memory.
 *   - A stream argument is a cudaStream_t passed as void* (NULL = legacy
 *     default stream).
 *   - Every call returns a recflex_status_t.  Host-checkable misuse returns
 *     RECFLEX_ERR_INVALID_ARG before any launch; launch failures return
 *     RECFLEX_ERR_CUDA.  Device-data errors (out-of-range IDs, non-monotone
 *     offsets) are undefined behaviour in recflex_forward; recflex_validate
 *     detects them (reading C3).
 *   - The caller owns tables, indices, offsets, out and streams.  The plan
 *     owns its descriptors and scratch.
 *   - A plan is not thread-safe; one plan must not have two forwards in
 *     flight on different streams (they share scratch).
 *
 * Data layout (readings C4, C6, C7 in DESIGN.md):
 *   indices : int32 [nnz]          lookup IDs, feature-major KJT
 *   offsets : int32 [F*B + 1]      bag (f,s) = indices[offsets[f*B+s] .. offsets[f*B+s+1])
 *                                  offsets[0] == 0, non-decreasing, nnz < 2^31
 *   tables  : F row-major tables, 32-byte aligned base, in the feature's
 *             storage type (recflex_dtype_t; the paper is
 *             silent on precision, reading C5):
 *               F32  float32  [rows_f][d_f]                      (default)
 *               F16  binary16 [rows_f][d_f]
 *               BF16 bfloat16 [rows_f][d_f]
 *               FP8  OCP E4M3 codes [rows_f][d_f] (1 byte each)
 *               I8   rowwise-quantised: row r is RECFLEX_I8_ROW_BYTES(d_f)
 *                    bytes = d_f int8 codes q, then float32 scale, float32
 *                    bias, zero padding to a multiple of 16 bytes; the row's
 *                    value in column c is scale * q[c] + bias
 *             Rows are always accumulated in fp32; the output is fp32.
 *   out     : float32 row-major [B][D_tot], D_tot = sum d_f, feature f at
 *             columns [col_f, col_f + d_f), col_f = sum_{g<f} d_g; 16-byte
 *             aligned base
 */
#ifndef RECFLEX_H_
#define RECFLEX_H_

#ifdef __CUDACC_RTC__
/* device-side compilation of the plan-specialised fused kernel (NVRTC, no libc headers) */
typedef signed char int8_t;
typedef int int32_t;
typedef unsigned int uint32_t;
typedef long long int64_t;
typedef unsigned long long uint64_t;
typedef unsigned long long uintptr_t;
#else
#include <stddef.h>
#include <stdint.h>
#endif

#ifdef __cplusplus
extern "C" {
#endif

#define RECFLEX_ABI_VERSION 4
#define RECFLEX_MAX_OCCUPANCY 8          /* CTAs of 256 threads per SM: K = 8 (reading C14) */

typedef struct recflex_plan_s *recflex_plan_t; /* opaque, library-owned */

typedef enum { RECFLEX_POOL_SUM = 0, RECFLEX_POOL_MEAN = 1 } recflex_pool_t;

/* Storage type of a feature's table rows. */
typedef enum {
    RECFLEX_DTYPE_F32 = 0,  /* float32                                                   */
    RECFLEX_DTYPE_F16 = 1,  /* IEEE binary16; needs d_f % 4 == 0                         */
    RECFLEX_DTYPE_BF16 = 2, /* bfloat16 (upper half of a float32); needs d_f % 4 == 0    */
    RECFLEX_DTYPE_I8 = 3,   /* int8 codes + per-row float32 scale and bias; d_f % 8 == 0 */
    RECFLEX_DTYPE_FP8 = 4   /* OCP FP8 E4M3 ("e4m3fn") codes, d_f bytes per row, no
                               scale (a per-table scale is linear in the pooled output
                               and folds into its consumer); d_f % 8 == 0             */
} recflex_dtype_t;

/* Bytes per row of an I8 table: d codes + 8 bytes scale/bias, padded to 16. */
#define RECFLEX_I8_ROW_BYTES(d) ((((int64_t)(d)) + 8 + 15) / 16 * 16)

typedef enum {
    RECFLEX_OK = 0,
    RECFLEX_ERR_INVALID_ARG = 1,
    RECFLEX_ERR_CUDA = 2,
    RECFLEX_ERR_OOM = 3,
    RECFLEX_ERR_NOT_SUPPORTED = 4,
    RECFLEX_ERR_INDEX_OOB = 5
} recflex_status_t;

/* Per-feature table spec plus hotness statistics from historical data
 * ("embedding table specifications"; P:160 historical inputs). */
typedef struct {
    int64_t num_rows; /* rows_f, 1 <= rows_f < 2^31                              */
    int32_t dim;      /* d_f >= 1; vector paths need d_f % 4 == 0 (else scalar)   */
    int32_t pool;     /* recflex_pool_t; MEAN of an empty bag is 0 (reading C1)   */
    float mean_len;   /* E[L | L > 0]   (pooling factor)                    */
    float max_len;    /* observed max L (sizes scratch for nnz-partitioned tasks) */
    float coverage;   /* P(L > 0)                                    */
    int32_t dtype;    /* recflex_dtype_t of the table rows (0 = F32)              */
} recflex_feature_spec_t;

/* A feature's schedule: catalog entry + its runtime thread-mapping parameters
 * ("tunable parameters").  part 0: a task (CTA work unit) covers
 * per_block consecutive samples; part 1: a task covers the bags whose first
 * lookup falls in a window of per_block lookups (adaptive to the batch).
 * Either way the batch NEEDS blocks_f = ceil(B/per_block) (part 0) or
 * floor(nnz_f/npb)+1 (part 1) tasks, computed on the device per batch: the
 * runtime thread mapping of §IV-B.
 * static_blocks > 0 replaces it by the paper's STATIC thread mapping (the
 * ablation straw man): exactly static_blocks tasks are allocated
 * whatever the batch, and allocated task a performs the needed tasks
 * a, a + static_blocks, a + 2*static_blocks, ... one after another ("if we
 * allocate two blocks ... while the input workload requires three blocks at
 * runtime, the first block will perform the computation of two blocks
 * sequentially"; reading C31); allocated tasks with nothing to do idle.
 * Never chosen by the tuner; for experiments. */
typedef struct {
    int32_t sched_id;      /* index into the catalog (recflex_catalog_info)         */
    int32_t part;          /* 0 sample-, 1 lookup(nnz)-partitioned                   */
    int32_t per_block;     /* samples per task (part 0), lookups per task (part 1)   */
    int32_t static_blocks; /* 0: runtime thread mapping; > 0: static, that many tasks */
} recflex_schedule_t;

/* Catalog entry description (hand-written sm_100a schedule templates). */
typedef enum {
    RECFLEX_FAMILY_GROUP = 0, /* G lanes per bag; 256/G bags in flight per CTA (G=32: warp per sample) */
    RECFLEX_FAMILY_BLOCK = 1, /* all 256 threads on one bag; smem partials + fixed-order reduction    */
    RECFLEX_FAMILY_FLAT = 2,  /* G lanes walk a run of 8 consecutive bags as one lookup range       */
    RECFLEX_FAMILY_WARP = 3   /* the 32/G lane groups of a warp share one bag (strided lookups,
                                 xor-butterfly reduction): 32/G x U rows of a bag in flight        */
} recflex_family_t;

typedef struct {
    int32_t family; /* recflex_family_t                                        */
    int32_t group;  /* G: lanes cooperating on one row (power of two, 1..32)   */
    int32_t vec;    /* floats per lane per load: 1, 4 (128-bit) or 8 (256-bit) */
    int32_t cols;   /* C: column chunks per lane (row span = G*vec*C floats)   */
    int32_t unroll; /* U: rows in flight per lane                              */
    int32_t dtype;  /* recflex_dtype_t the entry gathers (vec counts elements)  */
} recflex_catalog_info_t;

/* ---- plan lifecycle --------------------------------------------------- */

/* Validates specs (incl. each dtype's dim constraint), computes col_f (prefix sum of dims), picks heuristic
 * default schedules (an untuned plan is valid), allocates plan scratch sized
 * for max_batch on `device`.  No device data is read.  *out receives the plan. */
recflex_status_t recflex_plan_create(const recflex_feature_spec_t *specs, int32_t num_features,
                                     int32_t max_batch, int32_t device, recflex_plan_t *out);

/* Frees all plan-owned memory.  NULL is a no-op. */
void recflex_destroy(recflex_plan_t plan);

const char *recflex_status_string(recflex_status_t status);

/* Human-readable detail of the last CUDA failure seen by this thread
 * ("<where>: <cudaError name> (<text>)"); empty if none.  Not cleared on success. */
const char *recflex_last_error(void);

/* ---- the hot path ----------------------------------------------------- */

/* Fused multi-feature embedding-bag forward (async, stream-ordered, no host
 * synchronisation and no allocation: CUDA-graph capturable).
 *   indices, offsets : device, layout above; batch_size = B (0 <= B <= max_batch;
 *                      B == 0 is a no-op)
 *   tables           : HOST array of F device pointers (cached; re-uploaded
 *                      only when a pointer changes)
 *   out              : device float32 [B][D_tot], fully overwritten
 * Launches: map kernel (device-side workload scan), optional task-range fill
 * kernel (only if some feature is lookup-partitioned), fused kernel (PDL). */
recflex_status_t recflex_forward(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                 int32_t batch_size, const void *const *tables, float *out,
                                 void *stream);

/* Same operation from HOST buffers (end-to-end path): copies h_indices[nnz] and
 * h_offsets[F*B+1] to plan-owned device staging, runs recflex_forward, copies
 * the pooled output back to h_out [B][D_tot]; blocks until h_out is written.
 * Staging grows on demand (this entry point may allocate). */
recflex_status_t recflex_forward_host(recflex_plan_t plan, const int32_t *h_indices, int64_t nnz,
                                      const int32_t *h_offsets, int32_t batch_size,
                                      const void *const *tables, float *h_out, void *stream);

/* The serving loop over host-resident batches (end-to-end path): batch i's
 * KJT (h_indices[i][nnz[i]], h_offsets[i][F*B_i+1], pinned host memory for
 * full copy bandwidth) is copied in, pooled, and its output copied to
 * h_out[i] [B_i][D_tot], exactly as recflex_forward_host does per batch, but
 * pipelined over two plan-owned device staging slots and two copy streams:
 * the H2D of batch i+1 and the D2H of batch i-1 overlap the forward of batch
 * i.  Blocks until every h_out[i] is written.  Host arrays of num_batches
 * entries; staging grows on demand (may allocate); results identical to
 * recflex_forward per batch.  Errors: INVALID_ARG (null/negative/too-large
 * arguments, checked before any copy), CUDA/OOM. */
recflex_status_t recflex_forward_host_batches(recflex_plan_t plan, int32_t num_batches,
                                              const int32_t *const *h_indices, const int64_t *nnz,
                                              const int32_t *const *h_offsets, const int32_t *batch_sizes,
                                              const void *const *tables, float *const *h_out, void *stream);

/* ---- tuner (§IV-A) ------------------------------------------------------ */

typedef struct {
    int32_t num_occupancies; /* how many entries of occupancies[] to try (0 = all 1..8)    */
    int32_t occupancies[RECFLEX_MAX_OCCUPANCY];
    int32_t reps;            /* stage-2 timed forwards per batch (median), default 7       */
    int32_t pad_waves;       /* padding tasks = pad_waves * #SM * k, default 4     */
    int32_t max_candidates;  /* per feature, 0 = all valid catalog candidates              */
    int32_t verbose;         /* 1: print per-stage summaries to stderr                     */
    int32_t skip_guard;      /* 0: also time the incoming schedules at every k and keep
                                them if faster than the two-stage result (K extra evals)   */
    int32_t refine;          /* 1: after selection, try every candidate per cluster of
                                same-dim / same-length-class features in the real fused
                                forward at the chosen k; keep if > 0.5% faster.
                                Outside O(F*K + K); off by default, reported apart        */
    int32_t local_mode;      /* 0: interference-simulated co-execution with padding (the
                                paper's method: all candidates of a feature in one padded
                                launch, cost = their own block times); 1: separate-combine
                                straw man -- each candidate timed alone in a non-padded
                                launch (for the Fig. 11 ablation); 2: isolated
                                co-execution -- one padded launch per candidate, cost = the
                                launch's total block time, i.e. its own blocks plus the
                                slowdown it inflicts on the padding (reading C34)          */
    int32_t stage2_catalog;  /* 0: stage 2 (and guard / refinement) time the plan-
                                specialised kernel each choice compiles to (NVRTC, the
                                kernel forwards run); 1: the precompiled catalog kernel   */
    int32_t no_tail;         /* 0: stage-1 cost = W_c / (#SM*k) + max(0, Lmax_c - T_est)
                                (tail-aware, reading C33; T_est = measured latency of the
                                incoming plan at k, K*N extra timed forwards); 1: the
                                paper's plain sum of block times W_c (Eq. 3)              */
    int32_t keep_order;      /* 0: after kernel selection, recflex_select_task_order on the
                                first batch (3 x reps forwards); 1: keep the plan's order  */
    int32_t keep_l2;         /* 0: then recflex_select_l2_policy (plan-specialised kernel
                                only; <= 3 compiles + 3 x reps forwards); 1: keep it       */
    int32_t keep_task_size;  /* 0: before the order selection, recflex_select_task_size
                                (3 x reps forwards); 1: keep the per-task sizes            */
    float switch_margin;     /* stage 1: a candidate other than the feature's incoming
                                schedule must cost < (1 - margin) x the incoming one to be
                                chosen (reading C38; 0 = the paper's plain argmin)         */
    int32_t position_balance; /* 1: stage-1 launches list a feature's candidates in reverse
                                on every other (batch, k), so no candidate always runs
                                next to the pre- or the post-padding (reading C39)         */
} recflex_tune_options_t;

typedef struct {
    int64_t local_launches;   /* stage 1 co-execution launches  (= F*K*N)           */
    int64_t global_launches;  /* stage 2 timed fused launches    (= K*N*reps)        */
    int64_t local_evals;      /* stage-1 cost evaluations (one per (k, f)) = F*K     */
    int64_t global_evals;     /* stage-2 cost evaluations (one per k)      = K       */
    int64_t guard_evals;      /* guard evaluations of the incoming plan    = K (or 0) */
    int32_t guard_won;        /* 1 if the incoming schedules were kept             */
    int32_t best_occupancy;
    double best_ms;           /* summed median forward time over tuning batches    */
    double tune_seconds;
    int64_t refine_evals;     /* cluster-refinement forwards timed                 */
    double refine_gain;       /* latency before refinement / after (>= 1)          */
    double two_stage_ms;      /* stage-2 latency of the two-stage choice alone     */
    double incoming_ms;       /* best guard latency of the incoming schedules      */
    int64_t jit_compiles;     /* plan-specialised kernels compiled (or cache hits) */
    double compile_seconds;   /* wall time spent compiling them                    */
    double refine_seconds;    /* wall time of the refinement stage                 */
    int32_t task_order;       /* RECFLEX_ORDER_* kept by the order selection, -1 = not run */
    int32_t l2_policy;        /* recflex_select_l2_policy's choice, -1 = not run           */
    int32_t task_size;        /* recflex_select_task_size's choice, -1 = not run           */
} recflex_tune_stats_t;

/* Two-stage interference-simulated tuning over num_batches historical batches
 * (Eq. 5).  indices[i] / offsets[i] are DEVICE pointers of batch i with
 * batch_sizes[i] samples; tables as in recflex_forward.  Blocking; may
 * allocate.  Leaves the plan with the selected occupancy and schedules. */
recflex_status_t recflex_tune(recflex_plan_t plan, int32_t num_batches, const int32_t *const *indices,
                              const int32_t *const *offsets, const int32_t *batch_sizes,
                              const void *const *tables, void *stream);
recflex_status_t recflex_tune_ex(recflex_plan_t plan, int32_t num_batches, const int32_t *const *indices,
                                 const int32_t *const *offsets, const int32_t *batch_sizes,
                                 const void *const *tables, void *stream,
                                 const recflex_tune_options_t *options, recflex_tune_stats_t *stats);

/* The selection logic of the two-stage tuner, on caller-supplied costs
 * (Eq. 3 per-feature local objective, Eq. 4 global objective).
 *   local_cost(user, k_index, f, costs_out[num_candidates[f]]): one call = one
 *     co-execution launch; fills the summed block times of every candidate.
 *   global_cost(user, k_index, choice[F]) -> fused-kernel latency at O_k.
 * Writes choice_out[F] and *best_k_index; tie -> lowest candidate index (local),
 * larger k index (global).  Returns call counts through *local_calls and *global_calls. */
typedef void (*recflex_local_cost_fn)(void *user, int32_t k_index, int32_t f, double *costs_out);
typedef double (*recflex_global_cost_fn)(void *user, int32_t k_index, const int32_t *choice);
recflex_status_t recflex_two_stage_select(int32_t num_features, int32_t num_k, const int32_t *num_candidates,
                                          recflex_local_cost_fn local_cost, recflex_global_cost_fn global_cost,
                                          void *user, int32_t *choice_out, int32_t *best_k_index,
                                          int64_t *local_calls, int64_t *global_calls);

/* ---- schedules / occupancy / catalog ------------------------------------ */

recflex_status_t recflex_get_schedule(recflex_plan_t plan, int32_t f, recflex_schedule_t *sched,
                                      int32_t *blocks_per_sm);
/* Validates the schedule against d_f (vector width divides d_f, ...). */
recflex_status_t recflex_set_schedule(recflex_plan_t plan, int32_t f, const recflex_schedule_t *sched);
/* k CTAs (of 256 threads) per SM, 1..8: register cap __launch_bounds__(256,k)
 * + shared-memory padding (reading C15). */
recflex_status_t recflex_set_occupancy(recflex_plan_t plan, int32_t k);
recflex_status_t recflex_get_occupancy(recflex_plan_t plan, int32_t *k);

int32_t recflex_catalog_size(void);
recflex_status_t recflex_catalog_info(int32_t sched_id, recflex_catalog_info_t *info);
/* 1 if catalog entry sched_id can run a float32 feature of dimension dim. */
int32_t recflex_catalog_valid(int32_t sched_id, int32_t dim);
/* 1 if catalog entry sched_id can run a feature of dimension dim stored as dtype. */
int32_t recflex_catalog_valid_dtype(int32_t sched_id, int32_t dim, int32_t dtype);

/* cudaOccupancyMaxActiveBlocksPerMultiprocessor of the fused-kernel variant
 * for occupancy k with its padded shared memory (should equal k). */
recflex_status_t recflex_occupancy_check(int32_t device, int32_t k, int32_t *active_blocks_per_sm,
                                         int32_t *registers_per_thread, int32_t *spill_bytes);

/* ---- plan-specialised fused kernel (the paper's fusion compiler) --------- */

/* The paper compiles one fused kernel per model with every feature's tuned
 * schedule inlined into the if-else dispatch (§IV-B, Fig. 8; P:178
 * "make all functions inline within the branches").  recflex_plan_compile
 * generates that kernel for the plan's CURRENT schedules -- one branch per
 * distinct (catalog entry, d_f, pool, row pitch), the entry's template called
 * with those values as compile-time literals -- and compiles it for sm_100a
 * with NVRTC (libnvrtc.so.12, loaded at run time), once per occupancy listed
 * (occupancies = NULL / num = 0: the plan's current k).  Blocking; compiles
 * concurrently; cubins are cached on disk (recflex_set_jit_cache_dir, else
 * env RECFLEX_JIT_CACHE, else no cache).  From then on recflex_forward and
 * recflex_forward_routed at occupancy k launch the compiled kernel as long as
 * no feature's sched_id has changed since (recflex_set_schedule, import and
 * tuning invalidate it; forwards then use the precompiled catalog kernel
 * until the next compile -- same results, bit for bit, by construction: the
 * same schedule templates in the same order).  RECFLEX_ERR_NOT_SUPPORTED if
 * NVRTC or the driver entry points are unavailable (recflex_last_error says
 * which). */
recflex_status_t recflex_plan_compile(recflex_plan_t plan, const int32_t *occupancies, int32_t num_occupancies);

typedef struct {
    int32_t compiled;      /* a kernel exists for this k                          */
    int32_t active;        /* it matches the current schedules and is used        */
    int32_t variants;      /* distinct (entry, d, pool, pitch) branches           */
    int32_t registers;     /* per thread (cuFuncGetAttribute)                     */
    int32_t local_bytes;   /* local memory per thread (spills / stack)            */
    int32_t blocks_per_sm; /* occupancy after smem / carveout setup (== k)        */
    int32_t smem_bytes;    /* dynamic shared memory per CTA                       */
    int32_t cache_hit;     /* cubin came from the disk cache                      */
    float compile_ms;      /* NVRTC (or cache read) wall time                      */
} recflex_jit_info_t;
/* k = 0: the plan's current occupancy. */
recflex_status_t recflex_jit_info(recflex_plan_t plan, int32_t k, recflex_jit_info_t *info);
/* enable = 0: forwards ignore compiled kernels (A/B against the catalog kernel).
 * The choice is part of the plan's exported state ("kernel"). */
recflex_status_t recflex_set_jit(recflex_plan_t plan, int32_t enable);
recflex_status_t recflex_get_jit(recflex_plan_t plan, int32_t *enabled);
/* Stage 2 over the plan's two kernels: compiles the plan-specialised kernel
 * for the current schedules and k (if needed), times it and the catalog kernel
 * on one batch (device pointers; median of reps forwards, L2 flushed before
 * each) and keeps the faster for later forwards.  *jit_ms / *catalog_ms
 * (nullable) receive the medians.  Blocking; allocates scratch. */
recflex_status_t recflex_select_kernel(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                       int32_t batch_size, const void *const *tables, int32_t reps, float *jit_ms,
                                       float *catalog_ms, void *stream);
/* Directory for cached cubins (created on first write); NULL or "" = none. */
recflex_status_t recflex_set_jit_cache_dir(const char *dir);
/* The generator alone (no GPU needed): CUDA source of the specialised kernel
 * for num_features features (catalog ids, dims, pools, dtypes -- dtypes NULL =
 * all F32) at occupancy k; buf (nullable) receives up to cap-1 bytes + NUL,
 * *len the full length; variant_of_feature[F] (nullable) the branch each
 * feature takes; *num_variants the branch count.  INVALID_ARG if an entry is
 * not valid for its feature. */
recflex_status_t recflex_jit_generate(const int32_t *sched_ids, const int32_t *dims, const int32_t *pools,
                                      const int32_t *dtypes, int32_t num_features, int32_t k, char *buf,
                                      size_t cap, size_t *len, int32_t *variant_of_feature,
                                      int32_t *num_variants);
/* NVRTC-compile generated source to an sm_100a cubin (no GPU needed).
 * cubin_buf (nullable, cap bytes) receives the cubin if it fits, *cubin_len
 * its size; log_buf (nullable) the NVRTC log (ptxas -v lines included). */
recflex_status_t recflex_jit_compile_source(const char *source, void *cubin_buf, size_t cap, size_t *cubin_len,
                                            char *log_buf, size_t log_cap, int32_t *cache_hit);

/* ---- introspection / validation / persistence ---------------------------- */

/* Runs the map (+ fill) kernels for offsets (device) and copies the task map
 * to the host: host_block_start[F+1] (exclusive scan of feature_blocks taken
 * in the plan's TASK ORDER -- entry e belongs to feature order[e] of
 * recflex_get_task_order; Fig. 8 d_task_map in compressed form);
 * host_task_range (nullable) receives, for
 * lookup-partitioned features, [s0, s1) of every task as 2*total ints
 * (-1 for sample-partitioned tasks).  Blocking. */
recflex_status_t recflex_debug_task_map(recflex_plan_t plan, const int32_t *offsets, int32_t batch_size,
                                        int32_t *host_block_start, int32_t *host_task_range,
                                        int64_t task_range_capacity, void *stream);

/* Task-range slots the plan reserved for feature f (lookup-partitioned
 * schedules): max(64, max_batch * max_len / 128 + 3).  A batch whose
 * floor(nnz_f/npb)+1 tasks would not fit in slots - 1 runs with npb raised to
 * ceil(nnz_f / (slots - 2)) (reading C12). */
recflex_status_t recflex_get_task_slots(recflex_plan_t plan, int32_t f, int32_t *slots);

/* Tasks every feature NEEDED in the plan's last map (forward or
 * recflex_debug_task_map): ceil(B/per_block) or floor(nnz_f/npb)+1 -- equal to
 * the feature's task count unless a static mapping (static_blocks > 0) folds
 * them onto fewer.  host_need[F].  Blocking. */
recflex_status_t recflex_debug_task_need(recflex_plan_t plan, int32_t *host_need);

/* ---- task order (reading C35; a B200 addition, not in the paper) ---------
 * The persistent CTAs claim tasks from one counter in task-map order, and the
 * task map concatenates the features in the plan's task order (the paper:
 * feature order, as blockIdx.x).  The order changes neither what a task
 * computes nor where it stores (outputs are bitwise identical under every
 * order); it changes which work overlaps and how long the kernel's tail is.
 * Heuristics over the estimated bytes per task (per_block bags of
 * coverage * mean_len rows, or per_block lookups, times the row pitch):    */
#define RECFLEX_ORDER_FEATURE 0 /* feature order (the paper's)                    */
#define RECFLEX_ORDER_LPT 1     /* longest estimated task first (stable)          */
#define RECFLEX_ORDER_SPT 2     /* shortest estimated task first (stable)         */
#define RECFLEX_NUM_ORDERS 3
/* order[F]: a permutation of 0..F-1 (position -> feature) or NULL = feature
 * order.  INVALID_ARG if not a permutation.  Setup call: synchronises the
 * device and uploads the plan's device arrays at once, so a CUDA graph captured
 * earlier replays in the new order.  Part of the exported plan ("order"). */
recflex_status_t recflex_set_task_order(recflex_plan_t plan, const int32_t *order);
/* Output layout: follow_task_order = 0 (default) -> out[s][col_f..col_f+d_f)
 * with the features concatenated in feature order (the paper's); 1 -> in the
 * plan's task order, so features whose tasks run back to back write adjacent
 * columns (a later recflex_set_task_order moves the columns with it).
 * NOT_SUPPORTED if a feature's schedule needs a 16-byte aligned column it
 * would not get.  Setup call: synchronises the device.  col[F] of
 * recflex_get_columns receives every feature's first output column. */
recflex_status_t recflex_set_column_order(recflex_plan_t plan, int32_t follow_task_order);
recflex_status_t recflex_get_columns(recflex_plan_t plan, int64_t *col);
/* ---- L2 eviction priority of row loads (reading C36; a B200 addition) ----
 * Within one batch the rows of a small table recur (sharded1000: 62 % of the
 * gathered row bytes are repeats), but the rows of large tables stream
 * through L2 and evict them.  The plan-specialised kernel can tag a feature's
 * row loads with an L2 cache policy (createpolicy + ld...L2::cache_hint):    */
#define RECFLEX_L2_DEFAULT 0
#define RECFLEX_L2_EVICT_FIRST 1  /* stream: rows rarely recur within a batch   */
#define RECFLEX_L2_EVICT_LAST 2   /* keep: small table, rows recur              */
#define RECFLEX_L2_KEEP_L1 3      /* keep, and allocate the rows in L1 as well  */
/* A new plan starts with the heuristic's EVICT_LAST part (below; L2 size from
 * the device) and DEFAULT elsewhere; an imported plan without "l2" has
 * DEFAULT everywhere.
 * policy[F] (values above) or NULL = default for every feature.  (KEEP_L1 was
 * measured no better than EVICT_LAST on sharded1000 / industrial.)  Takes effect
 * in the next compiled plan-specialised kernel (part of its signature; the
 * catalog kernel ignores it).  INVALID_ARG on an unknown value.  Part of the
 * exported plan ("l2"). */
recflex_status_t recflex_set_l2_policy(recflex_plan_t plan, const int32_t *policy);
recflex_status_t recflex_get_l2_policy(recflex_plan_t plan, int32_t *policy);
/* The heuristic policy for an L2 of l2_bytes: evict_last when the table is at
 * most l2_bytes / 4 and a batch looks each row up at least once on average
 * (max_batch * mean_len * coverage >= rows); evict_first when the table is
 * larger than the L2 or a batch looks up fewer than half its rows; else
 * default.  Writes policy[F]; does not apply it. */
recflex_status_t recflex_l2_policy_heuristic(recflex_plan_t plan, int64_t l2_bytes, int32_t *policy);
/* Measured choice (plan-specialised kernel only; NOT_SUPPORTED otherwise):
 * candidate 0 = no hints, 1 = the heuristic policy, 2 = its evict_last part
 * alone; each compiled (NVRTC, disk cache) and timed on one batch (median of
 * reps forwards, L2 flushed before each); the fastest is kept (ties: 0, then
 * 2, then 1).  *chosen / ms[3] (nullable) receive the choice and the medians.
 * Blocking; allocates scratch; the previous policy is kept on error. */
recflex_status_t recflex_select_l2_policy(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                          int32_t batch_size, const void *const *tables, int32_t reps,
                                          int64_t l2_bytes, int32_t *chosen, float *ms, void *stream);
/* ---- task granularity (reading C37) ---------------------------------------
 * The default schedules size tasks for a plan-wide lookup target and the
 * tuner keeps that size; with the task order and L2 policy in place the best
 * size can move.  Times the plan with every feature's per_block scaled by 1,
 * 1/2 and 2 (lookup-partitioned: >= 16 lookups per task; a heuristic task
 * order is re-derived for each), on one batch (median of reps forwards, L2
 * flushed before each), keeps the fastest (ties: 1, 1/2, 2).  *chosen (0, 1, 2
 * = x1, x1/2, x2) and ms[3] (nullable).  Blocking; allocates scratch. */
recflex_status_t recflex_select_task_size(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                          int32_t batch_size, const void *const *tables, int32_t reps,
                                          int32_t *chosen, float *ms, void *stream);
/* order[F] receives the plan's current task order. */
recflex_status_t recflex_get_task_order(recflex_plan_t plan, int32_t *order);
/* order[F] receives heuristic `kind` (RECFLEX_ORDER_*) for the plan's current
 * schedules, without applying it. */
recflex_status_t recflex_task_order_heuristic(recflex_plan_t plan, int32_t kind, int32_t *order);
/* Times the plan's current kernel under every heuristic order on one batch
 * (device pointers; median of reps forwards, L2 flushed before each), keeps
 * the fastest (ties: the lower kind).  *chosen (nullable) receives its kind,
 * ms[RECFLEX_NUM_ORDERS] (nullable) the medians.  Blocking; allocates
 * scratch; the plan keeps its previous order on error. */
recflex_status_t recflex_select_task_order(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                           int32_t batch_size, const void *const *tables, int32_t reps,
                                           int32_t *chosen, float *ms, void *stream);

/* Checks offsets (offsets[0]==0, monotone, F*B+1 entries) and that every ID of
 * feature f is in [0, rows_f).  Blocking.  RECFLEX_ERR_INDEX_OOB / INVALID_ARG. */
recflex_status_t recflex_validate(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                  int32_t batch_size, void *stream);

/* JSON export/import of the tuned state (occupancy + per-feature schedules),
 * P:164 "re-tune periodically".  export: writes up to cap bytes incl. NUL,
 * *len = required size. */
recflex_status_t recflex_plan_export(recflex_plan_t plan, char *buf, size_t cap, size_t *len);
recflex_status_t recflex_plan_import(recflex_plan_t plan, const char *json);

/* Profiling: when enabled, recflex_forward brackets its kernels with CUDA
 * events on the launch stream; recflex_get_kernel_times returns the summed
 * device milliseconds of the map(+fill) and fused kernels since the last reset
 * and the number of forwards.  Blocking (synchronises the events). */
recflex_status_t recflex_set_profiling(recflex_plan_t plan, int32_t enable);
recflex_status_t recflex_get_kernel_times(recflex_plan_t plan, double *map_ms, double *fused_ms,
                                          int64_t *forwards, int32_t reset);

/* ---- fused pooled-output exchange ------------------------ */

/* recflex_forward with the table-wise all-to-all folded into the fused
 * kernel's store epilogue: the pooled row of sample s (of this plan's
 * features) is written straight into destination j = s / rows_per_dst,
 * buffer host_dst[j] (a DEVICE pointer valid on this plan's device: local,
 * NVLink peer-enabled, or CUDA-IPC mapped), at row s - j*rows_per_dst and
 * columns [col_base + col_f, col_base + col_f + d_f) of a [rows][dst_stride]
 * float32 layout.  Requires B == num_dst * rows_per_dst, 16-byte aligned
 * buffers, col_base and dst_stride multiples of 4, col_base + D_tot <= stride.
 * Async on `stream`; the caller orders the destination's reads after every
 * writer's kernel (e.g. a collective barrier on the same streams). */
recflex_status_t recflex_forward_routed(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                        int32_t batch_size, const void *const *tables, float *const *host_dst,
                                        int32_t num_dst, int32_t rows_per_dst, int32_t dst_stride,
                                        int32_t col_base, void *stream);

/* The safe form of the fused exchange for a step loop (P:350 table-wise
 * placement): double-buffered destinations and a
 * device-side completion signal, no host or collective barrier per step.
 *   world, rank   : W ranks, this rank's index
 *   rows_per_dst  : B / W (samples each rank receives)
 *   dst_stride    : columns of the exchanged [rows][stride] float32 layout
 *   col_base      : first column of this rank's features in it
 *   dst[b][j]     : host arrays of W DEVICE pointers -- buffer b (0, 1) of rank
 *                   j (local, NVLink peer-enabled or CUDA-IPC mapped), 16-byte
 *                   aligned
 *   flags[j]      : host array of W DEVICE pointers -- rank j's flag array of W
 *                   uint32 (zero-initialised before the first step, owned by
 *                   rank j, mapped here like the buffers)
 *   local_flags   : this rank's own flag array (flags[rank] as seen locally)
 * Step n of this plan (n = 0, 1, ... counted per plan) writes buffer n & 1 of
 * every destination; *buffer_index receives n & 1 for the caller's own
 * buffer.  A one-warp kernel enqueued right after the fused kernel on
 * `stream` (so after every pooled row of the step is stored) publishes n + 1
 * into every destination's flags[rank] with a system-scope release, then
 * acquires flags[j] >= n + 1 for every writer j.  So work enqueued
 * on `stream` after this call sees the complete exchanged rows of step n.
 * Write-after-read safety: step n + 2 reuses buffer n & 1; a writer starts
 * step n + 2 only after its own wait of step n + 1, i.e. after every rank's
 * kernel of step n + 1 ran -- and each rank launches step n + 1 after the
 * work it enqueued on `stream` before that call.  Hence the returned buffer
 * is valid for work enqueued on `stream` before this plan's next-but-one
 * exchange call (consume it on the same stream, or copy it).  Every rank must
 * call this the same number of times; a writer that never arrives makes the
 * wait kernel trap after ~60 s.  Async; B == world * rows_per_dst. */
typedef struct {
    int32_t world;
    int32_t rank;
    int32_t rows_per_dst;
    int32_t dst_stride;
    int32_t col_base;
    float *const *dst[2];
    uint32_t *const *flags;
    uint32_t *local_flags;
} recflex_exchange_t;
recflex_status_t recflex_forward_exchange(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                          int32_t batch_size, const void *const *tables,
                                          const recflex_exchange_t *exchange, int32_t *buffer_index, void *stream);

/* ---- backward (training) --------------------------------- */

/* The adjoint of recflex_forward (training is "not fundamentally
 * excluded"): for every bag (f, s) of the batch and every lookup j in it,
 *     targets[f][indices[j]][c] += scale * w * grad[s][col_f + c],   c < d_f,
 * w = 1 (SUM) or 1/L (MEAN, L the bag length; empty bags contribute nothing).
 * scale = 1 into zeroed buffers gives the dense table gradients; targets =
 * the (float32) tables and scale = -lr is one fused SGD step.
 *   grad    : DEVICE float32 [B][D_tot], 16-byte aligned (the gradient of out)
 *   targets : HOST array of F DEVICE float32 [rows_f][d_f] buffers, 16-byte
 *             aligned, updated in place (independent of the tables' storage
 *             dtype: fp32 master weights / gradient buffers)
 * Runs the plan's map kernel and a persistent scatter kernel over the same
 * task map as the forward (one CTA-task = the forward task's samples); each
 * bag's gradient row is loaded once and added to its rows with vector
 * reductions in L2 (red.global.add.v4.f32).  Contributions to one row from
 * different bags are added in no fixed order: results are exact when every
 * partial sum is representable (integer data), else within the fp32
 * summation bound.  Async on `stream`, no allocation after the first call. */
recflex_status_t recflex_backward(recflex_plan_t plan, const int32_t *indices, const int32_t *offsets,
                                  int32_t batch_size, const float *grad, float *const *targets, float scale,
                                  void *stream);

/* CUDA IPC helpers for the routed forward across processes: 64-byte handle of
 * a device allocation, map a peer process's handle, unmap. */
recflex_status_t recflex_ipc_get_handle(const void *d_ptr, void *handle64);
recflex_status_t recflex_ipc_open_handle(const void *handle64, void **d_ptr);
recflex_status_t recflex_ipc_close(void *d_ptr);
/* Own cudaMalloc allocation (so its IPC handle maps at offset 0) / free. */
recflex_status_t recflex_device_alloc(size_t bytes, int32_t device, void **d_ptr);
recflex_status_t recflex_device_free(void *d_ptr);

/* ---- multi-GPU exchange helper ------------------------------------------- */

/* Relayout after the table-wise pooled-output all-to-all:
 * recv holds W chunks, chunk i = [rows][dims[i]] (row-major, contiguous, in
 * rank order); out = [rows][sum dims] with chunk i at column offset
 * sum_{j<i} dims[j].  Device pointers, async on stream. */
recflex_status_t recflex_shard_concat(const float *recv, int32_t num_ranks, int32_t rows,
                                      const int32_t *host_dims, float *out, void *stream);

/* ---- table-wise input distribution ----------------- */

/* The KJT all-to-all in front of a table-wise sharded forward (TorchRec's
 * "input dist"; PAPER.md P:350 places whole tables on GPUs).  W ranks; rank j
 * holds a data-parallel KJT over ALL F features and its Bl local samples
 * (global samples j*Bl .. j*Bl+Bl-1): indices int32[nnz_j], offsets
 * int32[F*Bl+1], feature-major as in recflex_forward.  After pack ->
 * alltoallv (caller's, e.g. NCCL) -> unpack, rank r holds the KJT of the
 * features it owns (ascending feature id) over all B = W*Bl samples in global
 * order -- exactly the input recflex_forward of its plan takes.
 *
 * create: feature_owner[F] (host) = owning rank of every feature; the handle
 *   owns small device scratch (O(F + W*F_r)); device = CUDA ordinal.
 *   F*Bl and W*Bl must be < 2^31.  Errors: INVALID_ARG, CUDA/OOM. */
typedef struct recflex_kjt_dist_s *recflex_kjt_dist_t;
recflex_status_t recflex_kjt_dist_create(int32_t num_features, const int32_t *feature_owner, int32_t num_ranks,
                                         int32_t rank, int32_t local_batch, int32_t device,
                                         recflex_kjt_dist_t *out);
void recflex_kjt_dist_destroy(recflex_kjt_dist_t dist);
/* Host-known alltoallv sizes of the LENGTHS exchange (in int32 elements, per
 * peer, arrays of num_ranks) and the number of owned features F_r. */
recflex_status_t recflex_kjt_dist_sizes(recflex_kjt_dist_t dist, int32_t *send_length_counts,
                                        int32_t *recv_length_counts, int32_t *num_owned);
/* Sender side (all DEVICE pointers, async on stream, no allocation):
 *   send_lengths int32[F*Bl]: for every destination r in rank order, for every
 *     feature r owns (ascending id), the Bl bag lengths of this rank's samples;
 *   send_indices int32[nnz_local]: the same (destination, feature) order, each
 *     feature's IDs as one contiguous run (sample order kept);
 *   dest_counts int32[W]: IDs sent to each rank (the IDs alltoallv splits).
 * Offsets must be monotone (undefined otherwise, as in recflex_forward). */
recflex_status_t recflex_kjt_pack(recflex_kjt_dist_t dist, const int32_t *indices, const int32_t *offsets,
                                  int32_t *send_lengths, int32_t *send_indices, int32_t *dest_counts,
                                  void *stream);
/* Receiver side (DEVICE pointers, async on stream, no allocation):
 *   recv_lengths int32[W*F_r*Bl]: what pack sent here, concatenated in source
 *     rank order ([j][k][s]); recv_indices: the received IDs, same order;
 *   indices_out int32[sum of recv IDs], offsets_out int32[F_r*W*Bl+1]: the
 *     owned features' KJT, feature-major, samples in global order. */
recflex_status_t recflex_kjt_unpack(recflex_kjt_dist_t dist, const int32_t *recv_lengths,
                                    const int32_t *recv_indices, int32_t *indices_out, int32_t *offsets_out,
                                    void *stream);

/* Writes `bytes` of a device scratch buffer to evict L2 (timing hygiene). */
recflex_status_t recflex_l2_flush(void *d_scratch, size_t bytes, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* RECFLEX_H_ */
