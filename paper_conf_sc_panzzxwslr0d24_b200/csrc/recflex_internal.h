// recflex_internal.h -- shared between host plan code and device kernels of
// librecflex.so (NOT shared with oracle/).
#pragma once
#ifndef __CUDACC_RTC__
#include <stdint.h>
#endif

#include "../../include/recflex.h"

namespace recflex {

constexpr int kBlockThreads = 256;   // one CTA = the thread-mapping unit
constexpr int kMaxOcc = RECFLEX_MAX_OCCUPANCY;
constexpr int kSmemBlockStartCap = 4096;   // features whose block_start fits in smem (ints)

// Per-feature device descriptor: the paper's `args + arg_offsets[f]` and
// `schedule_map[f]` (Fig. 8) folded into one record.
struct __align__(16) FeatureDesc {
    const void *table;    // T_f, [rows][row_bytes] in the feature's dtype
    int32_t rows;         // < 2^31 (recflex_plan_create)
    int32_t nalloc;       // static thread mapping: allocated tasks, 0 = runtime mapping
    int32_t dim;
    int32_t col;          // col_f
    int32_t pool;         // 0 sum, 1 mean
    int32_t sched;        // catalog id
    int32_t part;         // 0 sample-partitioned, 1 lookup-partitioned
    int32_t per_block;    // spb or npb
    int32_t cap;          // max tasks (tuning padding), 0 = none
    int32_t slots;        // reserved task-range slots (part 1), incl. sentinel
    int32_t slot_base;    // first slot of this feature in task_range scratch (part 1)
    int32_t in_feature;   // which KJT feature slot this descriptor reads (identity for plans)
    int32_t row_bytes;    // bytes per table row (d*4, d*2, or RECFLEX_I8_ROW_BYTES(d))
    int32_t dtype;        // recflex_dtype_t (the schedule's entry has the same ET)
};
static_assert(sizeof(FeatureDesc) == 64, "FeatureDesc layout");

struct MapArgs {
    const FeatureDesc *desc;
    const int32_t *offsets;
    int32_t F;
    int32_t B;
    int32_t in_F;          // number of KJT features in offsets (F_in), offsets has in_F*B+1 entries
    int32_t *block_start;  // [F+1]
    int32_t *npb_eff;      // [F] effective lookups per task (part 1)
    int32_t *need;         // [F] tasks the batch needs (runtime mapping); = block count unless static
    int32_t *counter;      // task counter for the persistent fused kernel
};

struct FillArgs {
    const FeatureDesc *desc;
    const int32_t *offsets;
    const int32_t *block_start;
    const int32_t *npb_eff;
    const int32_t *need;            // [F] needed tasks (static features allocate fewer)
    const int32_t *part1_features;  // list of part-1 feature ids
    int32_t num_part1;
    int32_t B;
    int32_t *task_start;            // slots
};

struct FusedArgs {
    const FeatureDesc *desc;
    const int32_t *block_start;   // [F+1]
    const int32_t *task_start;    // part-1 slots
    const int32_t *need;          // [F] needed tasks (static thread mapping folds them onto nalloc)
    const int32_t *indices;
    const int32_t *offsets;
    float *out;
    int32_t *counter;
    long long *timers;            // per task cycles (tuning), or nullptr
    int32_t F;
    int32_t B;
    int32_t out_stride;           // D_tot
    int32_t timers_cap;
    int32_t smem_bytes;           // dynamic shared memory of the launch
    // fused pooled-output exchange (routed mode): sample s is stored into
    // out_ptrs[s / route_rows] at row s % route_rows, column col_base + col_f
    float *const *out_ptrs;       // device array of destination pointers (peer / IPC-mapped)
    int32_t route_rows;           // 0 = local mode (out + s * out_stride + col_f)
    int32_t col_base;
    // backward (NEXT #4): grad [B][out_stride], targets[f] fp32 [rows_f][d_f]
    const float *grad;
    float *const *targets;        // device array of F target pointers
    float bscale;
    int32_t bvec;                 // 1: 16-byte aligned grad columns (D_tot, col_f multiples of 4)
    // plan-specialised (JIT-compiled) fused kernel: variant id of every feature
    const int32_t *jit_var;
    // exchange mode (recflex_forward_exchange): out_ptrs holds 2 x route_world
    // destination pointers, buffer = *route_epoch & 1 (the exchange kernel that
    // follows the fused kernel bumps the epoch and signals).  nullptr: plain
    // routed mode.
    int32_t *route_epoch;
    int32_t route_world;
};

// ---------------------------------------------------------------------------
// Schedule catalog: X(family, ET, G, VEC, C, U), ET = recflex_dtype_t of the rows.  The id of an entry is its
// position.  Hand-written templates ("schedule templates").
// ---------------------------------------------------------------------------
#define RECFLEX_CATALOG(X)                                                      \
    /* GROUP, 128-bit rows, one column chunk per lane */                        \
    X(0, 0, 1, 4, 1, 2) X(0, 0, 1, 4, 1, 4) X(0, 0, 1, 4, 1, 8)                          \
    X(0, 0, 2, 4, 1, 2) X(0, 0, 2, 4, 1, 4) X(0, 0, 2, 4, 1, 8)                          \
    X(0, 0, 4, 4, 1, 2) X(0, 0, 4, 4, 1, 4) X(0, 0, 4, 4, 1, 8)                          \
    X(0, 0, 8, 4, 1, 2) X(0, 0, 8, 4, 1, 4) X(0, 0, 8, 4, 1, 8)                          \
    X(0, 0, 16, 4, 1, 2) X(0, 0, 16, 4, 1, 4) X(0, 0, 16, 4, 1, 8)                       \
    X(0, 0, 32, 4, 1, 2) X(0, 0, 32, 4, 1, 4) X(0, 0, 32, 4, 1, 8)                       \
    /* GROUP, 128-bit rows, two column chunks per lane */                       \
    X(0, 0, 1, 4, 2, 2) X(0, 0, 1, 4, 2, 4)                                           \
    X(0, 0, 2, 4, 2, 2) X(0, 0, 2, 4, 2, 4)                                           \
    X(0, 0, 4, 4, 2, 2) X(0, 0, 4, 4, 2, 4)                                           \
    X(0, 0, 8, 4, 2, 2) X(0, 0, 8, 4, 2, 4)                                           \
    X(0, 0, 16, 4, 2, 2) X(0, 0, 16, 4, 2, 4)                                         \
    X(0, 0, 32, 4, 2, 2) X(0, 0, 32, 4, 2, 4)                                         \
    /* GROUP, 256-bit rows (LDG.256) */                                         \
    X(0, 0, 1, 8, 1, 2) X(0, 0, 1, 8, 1, 4)                                           \
    X(0, 0, 2, 8, 1, 2) X(0, 0, 2, 8, 1, 4)                                           \
    X(0, 0, 4, 8, 1, 2) X(0, 0, 4, 8, 1, 4)                                           \
    X(0, 0, 8, 8, 1, 2) X(0, 0, 8, 8, 1, 4)                                           \
    X(0, 0, 16, 8, 1, 2) X(0, 0, 16, 8, 1, 4)                                         \
    X(0, 0, 32, 8, 1, 2) X(0, 0, 32, 8, 1, 4)                                         \
    /* GROUP, scalar rows (any dim / alignment) */                              \
    X(0, 0, 1, 1, 1, 4) X(0, 0, 2, 1, 1, 4) X(0, 0, 4, 1, 1, 4)                          \
    X(0, 0, 8, 1, 1, 4) X(0, 0, 16, 1, 1, 4) X(0, 0, 32, 1, 1, 4)                        \
    /* BLOCK: whole CTA on one bag, 128-bit rows */                             \
    X(1, 0, 1, 4, 1, 4) X(1, 0, 2, 4, 1, 4) X(1, 0, 4, 4, 1, 4)                          \
    X(1, 0, 8, 4, 1, 4) X(1, 0, 16, 4, 1, 4) X(1, 0, 32, 4, 1, 2) X(1, 0, 32, 4, 1, 4)     \
    /* BLOCK, 256-bit rows */                                                   \
    X(1, 0, 16, 8, 1, 2) X(1, 0, 16, 8, 1, 4)                                         \
    /* FLAT: runs of bags walked as one lookup range, 128-bit rows */           \
    X(2, 0, 1, 4, 1, 2) X(2, 0, 1, 4, 1, 4) X(2, 0, 2, 4, 1, 2) X(2, 0, 2, 4, 1, 4)         \
    X(2, 0, 4, 4, 1, 2) X(2, 0, 4, 4, 1, 4) X(2, 0, 8, 4, 1, 2) X(2, 0, 8, 4, 1, 4)         \
    X(2, 0, 16, 4, 1, 2) X(2, 0, 16, 4, 1, 4) X(2, 0, 32, 4, 1, 2) X(2, 0, 32, 4, 1, 4)     \
    /* FLAT, 256-bit rows */                                                    \
    X(2, 0, 1, 8, 1, 2) X(2, 0, 1, 8, 1, 4) X(2, 0, 2, 8, 1, 2) X(2, 0, 2, 8, 1, 4)         \
    X(2, 0, 4, 8, 1, 2) X(2, 0, 4, 8, 1, 4) X(2, 0, 8, 8, 1, 2) X(2, 0, 8, 8, 1, 4)         \
    X(2, 0, 16, 8, 1, 2) X(2, 0, 16, 8, 1, 4)                                  \
    RECFLEX_CATALOG_LOWP(X)
#define RECFLEX_CATALOG_LOWP(X) RECFLEX_CATALOG_HALF(X, 1) RECFLEX_CATALOG_HALF(X, 2) RECFLEX_CATALOG_I8(X) \
    RECFLEX_CATALOG_FP8(X) RECFLEX_CATALOG_HALF_U8(X, 1) RECFLEX_CATALOG_HALF_U8(X, 2) RECFLEX_CATALOG_WARP(X)

// Reduced-precision rows, appended so the fp32 ids above
// stay stable.  VEC counts ELEMENTS per lane per load: for 16-bit types
// 4 -> 64-bit, 8 -> 128-bit, 16 -> 256-bit loads; for int8 8 -> 64-bit,
// 16 -> 128-bit.  Accumulation is fp32 as for float32 rows.
#define RECFLEX_CATALOG_HALF(X, T)                                              \
    X(0, T, 1, 8, 1, 2) X(0, T, 1, 8, 1, 4) X(0, T, 2, 8, 1, 2) X(0, T, 2, 8, 1, 4) \
    X(0, T, 4, 8, 1, 2) X(0, T, 4, 8, 1, 4) X(0, T, 8, 8, 1, 2) X(0, T, 8, 8, 1, 4) \
    X(0, T, 16, 8, 1, 2) X(0, T, 16, 8, 1, 4) X(0, T, 32, 8, 1, 2) X(0, T, 32, 8, 1, 4) \
    X(0, T, 1, 16, 1, 2) X(0, T, 1, 16, 1, 4) X(0, T, 2, 16, 1, 2) X(0, T, 2, 16, 1, 4) \
    X(0, T, 4, 16, 1, 2) X(0, T, 4, 16, 1, 4) X(0, T, 8, 16, 1, 2) X(0, T, 8, 16, 1, 4) \
    X(0, T, 16, 16, 1, 2) X(0, T, 16, 16, 1, 4) X(0, T, 32, 16, 1, 2) X(0, T, 32, 16, 1, 4) \
    X(0, T, 1, 4, 1, 4) X(0, T, 2, 4, 1, 4) X(0, T, 4, 4, 1, 4) X(0, T, 8, 4, 1, 4)  \
    X(1, T, 16, 8, 1, 4) X(1, T, 8, 16, 1, 4)                                   \
    X(2, T, 1, 8, 1, 4) X(2, T, 2, 8, 1, 4) X(2, T, 4, 8, 1, 4) X(2, T, 8, 8, 1, 4)
#define RECFLEX_CATALOG_I8(X)                                                   \
    X(0, 3, 1, 8, 1, 2) X(0, 3, 1, 8, 1, 4) X(0, 3, 2, 8, 1, 2) X(0, 3, 2, 8, 1, 4) \
    X(0, 3, 4, 8, 1, 2) X(0, 3, 4, 8, 1, 4) X(0, 3, 8, 8, 1, 2) X(0, 3, 8, 8, 1, 4) \
    X(0, 3, 16, 8, 1, 2) X(0, 3, 16, 8, 1, 4)                                  \
    X(0, 3, 1, 16, 1, 2) X(0, 3, 1, 16, 1, 4) X(0, 3, 2, 16, 1, 2) X(0, 3, 2, 16, 1, 4) \
    X(0, 3, 4, 16, 1, 2) X(0, 3, 4, 16, 1, 4) X(0, 3, 8, 16, 1, 2) X(0, 3, 8, 16, 1, 4) \
    X(0, 3, 16, 16, 1, 2) X(0, 3, 16, 16, 1, 4) X(0, 3, 32, 16, 1, 2) X(0, 3, 32, 16, 1, 4) \
    X(1, 3, 8, 16, 1, 4)                                                        \
    X(2, 3, 1, 16, 1, 4) X(2, 3, 2, 16, 1, 4) X(2, 3, 4, 16, 1, 4) X(2, 3, 8, 16, 1, 4)

// FP8 E4M3 rows (1 byte per element, no scale): VEC 4 -> 32-bit, 8 -> 64-bit,
// 16 -> 128-bit, 32 -> 256-bit loads; widened exactly with cvt.rn.f16x2.e4m3x2.
// (A 128-byte row is one cache line: 32 lanes x 4 codes keeps only 4
// accumulators per lane, so U = 8 rows fit in flight under the k = 6..8 caps.)
#define RECFLEX_CATALOG_FP8(X)                                                  \
    X(0, 4, 1, 8, 1, 2) X(0, 4, 1, 8, 1, 4) X(0, 4, 2, 8, 1, 2) X(0, 4, 2, 8, 1, 4) \
    X(0, 4, 4, 8, 1, 2) X(0, 4, 4, 8, 1, 4) X(0, 4, 8, 8, 1, 2) X(0, 4, 8, 8, 1, 4) \
    X(0, 4, 16, 8, 1, 2) X(0, 4, 16, 8, 1, 4)                                  \
    X(0, 4, 1, 16, 1, 2) X(0, 4, 1, 16, 1, 4) X(0, 4, 2, 16, 1, 2) X(0, 4, 2, 16, 1, 4) \
    X(0, 4, 4, 16, 1, 2) X(0, 4, 4, 16, 1, 4) X(0, 4, 8, 16, 1, 2) X(0, 4, 8, 16, 1, 4) \
    X(0, 4, 16, 16, 1, 2) X(0, 4, 16, 16, 1, 4) X(0, 4, 32, 16, 1, 2) X(0, 4, 32, 16, 1, 4) \
    X(0, 4, 1, 32, 1, 2) X(0, 4, 2, 32, 1, 2) X(0, 4, 4, 32, 1, 2) X(0, 4, 4, 32, 1, 4) \
    X(0, 4, 32, 4, 1, 4) X(0, 4, 32, 4, 1, 8) X(0, 4, 16, 4, 1, 8) X(0, 4, 16, 8, 1, 8) \
    X(1, 4, 8, 16, 1, 4)                                                        \
    X(2, 4, 1, 16, 1, 4) X(2, 4, 2, 16, 1, 4) X(2, 4, 4, 16, 1, 4) X(2, 4, 8, 16, 1, 4)

// 16-bit rows, 8 rows in flight per lane group (appended: ids above stay stable);
// 32 lanes x 4 elements keep 4 accumulators per lane (cf. the FP8 entries).
#define RECFLEX_CATALOG_HALF_U8(X, T) X(0, T, 16, 8, 1, 8) X(0, T, 32, 4, 1, 8) X(0, T, 8, 8, 1, 8)

// WARP-SPLIT family (appended): the lane groups of one warp share a bag; NG*U
// rows in flight per bag, NG = 32/G; R = NG*U divides 32.
#define RECFLEX_CATALOG_WARP(X)                                                 \
    X(3, 0, 1, 4, 1, 1)                                                         \
    X(3, 0, 2, 4, 1, 2) X(3, 0, 2, 8, 1, 2)                                     \
    X(3, 0, 4, 4, 1, 2) X(3, 0, 4, 4, 1, 4) X(3, 0, 4, 8, 1, 2) X(3, 0, 4, 8, 1, 4) \
    X(3, 0, 8, 4, 1, 2) X(3, 0, 8, 4, 1, 4) X(3, 0, 8, 8, 1, 2) X(3, 0, 8, 8, 1, 4) \
    X(3, 0, 16, 4, 1, 2) X(3, 0, 16, 4, 1, 4) X(3, 0, 16, 8, 1, 2) X(3, 0, 16, 8, 1, 4)

struct CatalogEntry {
    int family, ET, G, VEC, C, U;
};

#define RECFLEX_CAT_ENTRY(fam, et, g, v, c, u) {fam, et, g, v, c, u},
static constexpr CatalogEntry kCatalog[] = {RECFLEX_CATALOG(RECFLEX_CAT_ENTRY)};
#undef RECFLEX_CAT_ENTRY
constexpr int kCatalogSize = sizeof(kCatalog) / sizeof(kCatalog[0]);

// Can entry e run a feature of dimension d stored as dtype?  (same element
// type; vector width divides d; at least a quarter of the lanes hold real
// columns; wide rows take several passes)
inline bool catalog_valid(const CatalogEntry &e, int d, int dtype = RECFLEX_DTYPE_F32) {
    if (d <= 0) return false;
    if (e.ET != dtype) return false;
    if (d % e.VEC != 0) return false;
    if (dtype == RECFLEX_DTYPE_I8 && d % 8 != 0) return false;  // scale/bias 8-byte aligned
    if (dtype == RECFLEX_DTYPE_FP8 && d % 8 != 0) return false;  // rows 8-byte aligned
    int span = e.G * e.VEC * e.C;
    if (4 * d < span) return false;
    return true;
}

// ---- kernel launchers (device code in .cu files) ----------------------------
struct LaunchCfg {
    int grid;
    int smem;     // dynamic shared memory bytes (padding for occupancy control)
    bool pdl;
};

int fused_launch(int k, const FusedArgs &a, const LaunchCfg &cfg, void *stream);  // returns cudaError_t
int backward_launch(int k, const FusedArgs &a, const LaunchCfg &cfg, void *stream);
int fused_prepare(int k, int device, int smem_bytes, int carveout);                              // cudaFuncSetAttribute
int fused_occupancy(int k, int smem_bytes, int *blocks, int *regs, int *spill);
int map_launch(const MapArgs &a, void *stream);
int fill_launch(const FillArgs &a, int B, bool pdl, void *stream);
int validate_launch(const FeatureDesc *desc, int F, int in_F, const int32_t *indices, const int32_t *offsets, int B,
                    int32_t *flag, void *stream);
int remap_launch(const int32_t *src, int32_t *dst, int64_t n, int64_t shift, int64_t rows, void *stream);
constexpr int kMaxConcatRanks = 64;
struct ConcatArgs {
    int32_t W, rows, d_tot;
    int32_t dims[kMaxConcatRanks];
    int32_t cols[kMaxConcatRanks];
};
int concat_launch(const float *recv, const ConcatArgs &a, float *out, void *stream);
int flush_launch(void *buf, size_t bytes, void *stream);
int route_signal_wait_launch(uint32_t *const *flags, const uint32_t *local_flags, int32_t *epoch, int rank, int world,
                             void *stream);

}  // namespace recflex
