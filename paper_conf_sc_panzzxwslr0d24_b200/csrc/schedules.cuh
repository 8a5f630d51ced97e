// schedules.cuh -- the hand-written schedule catalog (sm_100a).
//
// The paper's schedule templates are device functions that do
// one feature's gather+pool for the CTA's slice of work ("Schedule1 ..
// ScheduleN", Fig. 8 line 1).  Two families here, each a template over
//   G   lanes cooperating on one table row (power of two, <= 32),
//   VEC floats per lane per load (1: 32-bit, 4: LDG.128, 8: LDG.256),
//   C   column chunks held per lane (row span G*VEC*C floats per pass),
//   U   rows in flight per lane (unroll of the bag loop).
// GROUP: 256/G groups per CTA, each group pools whole bags (G = 32 is the
//        TorchRec-style warp-per-sample mapping, G < 32 packs several samples
//        per warp for small dims / one-hot fields).
// BLOCK: the whole CTA pools one bag (HugeCTR-style block-per-sample),
//        warp-shuffle + shared-memory fixed-order reduction, for long bags.
//
// Accumulation is fp32 in registers in a fixed order per (plan, batch):
// GROUP adds a bag's rows strictly in ascending lookup order, so its result is
// the sequential fp32 sum; BLOCK uses a fixed strided split + fixed tree.  The
// forward uses no floating-point atomics -> bitwise run-to-run determinism
// (C22).  The backward (sched_backward) does: its scatter reduces with
// red.global.add in L2, in an order that is not fixed (exact on integer data,
// within the fp32 summation bound otherwise).
#pragma once
#ifndef __CUDACC_RTC__
#include <cuda_runtime.h>
#endif

#include "recflex_internal.h"

namespace recflex {

#ifndef RECFLEX_SCHED_FN
#define RECFLEX_SCHED_FN __device__ __noinline__
#endif

// ---- loads ---------------------------------------------------------------
// Rows are gathered once and never reused by the CTA: bypass L1 allocation so
// the (reused) index lines stay resident.  `.nc` = read-only path.
//
// L2 eviction priority of a feature's row loads (reading C36), a compile-time
// P of the plan-specialised kernel: 0 = default, 1 = evict_first (rows of
// large tables that rarely recur within a batch: let them stream through L2),
// 2 = evict_last (small tables whose rows recur: keep them across the stream).
// The policy is a 64-bit operand built by createpolicy (a uniform value).
// P = 3 (small tables whose rows recur within a CTA's tasks): evict_last in L2
// and the rows ALLOCATE in L1 (no .L1::no_allocate).
template <int P>
__device__ __forceinline__ uint64_t l2pol() {
    uint64_t pol = 0;
    if constexpr (P == 1) asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    else if constexpr (P == 2 || P == 3) asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

template <int VEC, int P = 0>
__device__ __forceinline__ void ld_row(const float *p, float (&v)[VEC]) {
    static_assert(VEC == 1 || VEC == 4 || VEC == 8, "1, 4 or 8 floats");
    if constexpr (P == 0) {
        if constexpr (VEC == 1)
            asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v[0]) : "l"(p));
        else if constexpr (VEC == 4)
            asm("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
                : "l"(p));
        else
            asm("ld.global.nc.L1::no_allocate.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                : "l"(p));
    } else if constexpr (P == 3) {
        const uint64_t pol = l2pol<P>();
        if constexpr (VEC == 1)
            asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v[0]) : "l"(p), "l"(pol));
        else if constexpr (VEC == 4)
            asm("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
                : "l"(p), "l"(pol));
        else
            asm("ld.global.nc.L2::cache_hint.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8], %9;"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                : "l"(p), "l"(pol));
    } else {
        const uint64_t pol = l2pol<P>();
        if constexpr (VEC == 1)
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v[0]) : "l"(p), "l"(pol));
        else if constexpr (VEC == 4)
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3])
                : "l"(p), "l"(pol));
        else
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8], %9;"
                : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                : "l"(p), "l"(pol));
    }
}

__device__ __forceinline__ int ld_idx(const int32_t *p) { return __ldg(p); }

// ---- typed row loads -------------------------------------
// RowFrag<ET, VEC>: VEC consecutive elements of one table row starting at
// column col, held in registers in their STORED form between the load and
// the accumulation (so U rows in flight cost U * VEC * sizeof(elem) bytes of
// registers, not U * VEC floats), widened to fp32 only in add_to.  `row` is
// the row's first byte (table base + id * row_bytes).  ET = recflex_dtype_t:
//   F32  : 4/16/32-byte loads
//   F16  : 8/16/32-byte loads of binary16, exact widening (cvt.f32.f16)
//   BF16 : same loads, widening = the 16 bits placed in the upper half
//   I8   : 8/16-byte loads of int8 codes plus the row's float32 scale and bias
//          (bytes [d, d+8) of the row); value = fma(scale, q, bias) in fp32.
//          q -> fp32 without I2F: the code byte is placed in the mantissa of
//          2^23 (PRMT) and 2^23 + 128 subtracted (exact).
template <int NW, int P = 0>
__device__ __forceinline__ void ld_words(const void *p, unsigned (&w)[NW]) {
    if constexpr (P == 3) {
        const uint64_t pol = l2pol<P>();
        if constexpr (NW == 1)
            asm("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(w[0]) : "l"(p), "l"(pol));
        else if constexpr (NW == 2)
            asm("ld.global.nc.L2::cache_hint.v2.b32 {%0, %1}, [%2], %3;" : "=r"(w[0]), "=r"(w[1]) : "l"(p), "l"(pol));
        else if constexpr (NW == 4)
            asm("ld.global.nc.L2::cache_hint.v4.b32 {%0, %1, %2, %3}, [%4], %5;"
                : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
                : "l"(p), "l"(pol));
        else
            asm("ld.global.nc.L2::cache_hint.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8], %9;"
                : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
                : "l"(p), "l"(pol));
    } else if constexpr (P != 0) {
        const uint64_t pol = l2pol<P>();
        if constexpr (NW == 1)
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(w[0]) : "l"(p), "l"(pol));
        else if constexpr (NW == 2)
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.b32 {%0, %1}, [%2], %3;"
                : "=r"(w[0]), "=r"(w[1])
                : "l"(p), "l"(pol));
        else if constexpr (NW == 4)
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.b32 {%0, %1, %2, %3}, [%4], %5;"
                : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
                : "l"(p), "l"(pol));
        else
            asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8], %9;"
                : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
                : "l"(p), "l"(pol));
    } else if constexpr (NW == 1) {
        asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(w[0]) : "l"(p));
    } else if constexpr (NW == 2) {
        asm("ld.global.nc.L1::no_allocate.v2.b32 {%0, %1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "l"(p));
    } else if constexpr (NW == 4) {
        asm("ld.global.nc.L1::no_allocate.v4.b32 {%0, %1, %2, %3}, [%4];"
            : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3])
            : "l"(p));
    } else {
        static_assert(NW == 8, "1, 2, 4 or 8 words");
        asm("ld.global.nc.L1::no_allocate.v8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
            : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
            : "l"(p));
    }
}

__device__ __forceinline__ float f16_lo(unsigned w) {
    float f;
    asm("{\n\t.reg .b16 l, h;\n\tmov.b32 {l, h}, %1;\n\tcvt.f32.f16 %0, l;\n\t}" : "=f"(f) : "r"(w));
    return f;
}
__device__ __forceinline__ float f16_hi(unsigned w) {
    float f;
    asm("{\n\t.reg .b16 l, h;\n\tmov.b32 {l, h}, %1;\n\tcvt.f32.f16 %0, h;\n\t}" : "=f"(f) : "r"(w));
    return f;
}
// int8 code (byte k of w) -> fp32, exact: 2^23 + (q + 128) - (2^23 + 128)
template <int K>
__device__ __forceinline__ float i8_at(unsigned w) {
    const unsigned biased = __byte_perm(w ^ 0x80808080u, 0x4B000000u, 0x7640 | K);  // {0x4B,0,0,byte^0x80}
    return __uint_as_float(biased) - 8388736.0f;
}

template <int ET, int VEC>
struct RowFrag;

template <int VEC>
struct RowFrag<RECFLEX_DTYPE_F32, VEC> {
    float x[VEC];
    __device__ __forceinline__ void zero() {
#pragma unroll
        for (int e = 0; e < VEC; ++e) x[e] = 0.f;
    }
    template <int P = 0>
    __device__ __forceinline__ void load(const char *row, int col, int) {
        ld_row<VEC, P>(reinterpret_cast<const float *>(row) + col, x);
    }
    __device__ __forceinline__ void add_to(float (&acc)[VEC]) const {
#pragma unroll
        for (int e = 0; e < VEC; ++e) acc[e] += x[e];
    }
};

template <int VEC>
struct RowFrag<RECFLEX_DTYPE_F16, VEC> {
    unsigned w[VEC / 2];
    __device__ __forceinline__ void zero() {
#pragma unroll
        for (int e = 0; e < VEC / 2; ++e) w[e] = 0u;
    }
    template <int P = 0>
    __device__ __forceinline__ void load(const char *row, int col, int) { ld_words<VEC / 2, P>(row + 2 * col, w); }
    __device__ __forceinline__ void add_to(float (&acc)[VEC]) const {
#pragma unroll
        for (int i = 0; i < VEC / 2; ++i) {
            acc[2 * i] += f16_lo(w[i]);
            acc[2 * i + 1] += f16_hi(w[i]);
        }
    }
};

template <int VEC>
struct RowFrag<RECFLEX_DTYPE_BF16, VEC> {
    unsigned w[VEC / 2];
    __device__ __forceinline__ void zero() {
#pragma unroll
        for (int e = 0; e < VEC / 2; ++e) w[e] = 0u;
    }
    template <int P = 0>
    __device__ __forceinline__ void load(const char *row, int col, int) { ld_words<VEC / 2, P>(row + 2 * col, w); }
    __device__ __forceinline__ void add_to(float (&acc)[VEC]) const {
#pragma unroll
        for (int i = 0; i < VEC / 2; ++i) {
            acc[2 * i] += __uint_as_float(w[i] << 16);
            acc[2 * i + 1] += __uint_as_float(w[i] & 0xffff0000u);
        }
    }
};

// FP8 E4M3: two codes -> f16x2 (exact: E4M3 is a subset of binary16) -> two fp32.
__device__ __forceinline__ void e4m3x4_to_f32(unsigned w, float &a, float &b, float &c, float &d) {
    unsigned lo, hi;
    asm("{\n\t.reg .b16 l, h;\n\tmov.b32 {l, h}, %2;\n\tcvt.rn.f16x2.e4m3x2 %0, l;\n\tcvt.rn.f16x2.e4m3x2 %1, h;\n\t}"
        : "=r"(lo), "=r"(hi)
        : "r"(w));
    a = f16_lo(lo);
    b = f16_hi(lo);
    c = f16_lo(hi);
    d = f16_hi(hi);
}

template <int VEC>
struct RowFrag<RECFLEX_DTYPE_FP8, VEC> {
    static_assert(VEC % 4 == 0, "fp8 rows: 4 codes per word");
    unsigned w[VEC / 4];
    __device__ __forceinline__ void zero() {
#pragma unroll
        for (int e = 0; e < VEC / 4; ++e) w[e] = 0u;
    }
    template <int P = 0>
    __device__ __forceinline__ void load(const char *row, int col, int) { ld_words<VEC / 4, P>(row + col, w); }
    __device__ __forceinline__ void add_to(float (&acc)[VEC]) const {
#pragma unroll
        for (int i = 0; i < VEC / 4; ++i) {
            float a, b, c, d;
            e4m3x4_to_f32(w[i], a, b, c, d);
            acc[4 * i + 0] += a;
            acc[4 * i + 1] += b;
            acc[4 * i + 2] += c;
            acc[4 * i + 3] += d;
        }
    }
};

template <int VEC>
struct RowFrag<RECFLEX_DTYPE_I8, VEC> {
    static_assert(VEC % 4 == 0, "int8 rows: 4 codes per word");
    unsigned w[VEC / 4];
    unsigned sb[2];  // scale, bias
    __device__ __forceinline__ void zero() {
#pragma unroll
        for (int e = 0; e < VEC / 4; ++e) w[e] = 0u;
        sb[0] = sb[1] = 0u;
    }
    template <int P = 0>
    __device__ __forceinline__ void load(const char *row, int col, int d) {
        ld_words<VEC / 4, P>(row + col, w);
        ld_words<2, P>(row + d, sb);  // 8-byte aligned: d % 8 == 0
    }
    __device__ __forceinline__ void add_to(float (&acc)[VEC]) const {
        const float sc = __uint_as_float(sb[0]), bi = __uint_as_float(sb[1]);
#pragma unroll
        for (int i = 0; i < VEC / 4; ++i) {
            acc[4 * i + 0] += fmaf(sc, i8_at<0>(w[i]), bi);
            acc[4 * i + 1] += fmaf(sc, i8_at<1>(w[i]), bi);
            acc[4 * i + 2] += fmaf(sc, i8_at<2>(w[i]), bi);
            acc[4 * i + 3] += fmaf(sc, i8_at<3>(w[i]), bi);
        }
    }
};

// Registers of a U x C row-fragment set start at zero: a fragment that a
// predicated-off load leaves unwritten must not make the compiler keep the
// array in local memory to preserve "old" contents (measured: every ragged
// bag tail stored its just-loaded rows to the stack).
template <int ET, int VEC, int U, int C>
__device__ __forceinline__ void rf_zero(RowFrag<ET, VEC> (&v)[U][C]) {
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
        for (int c = 0; c < C; ++c) v[u][c].zero();
}

template <int VEC>
__device__ __forceinline__ void st_out(float *p, const float (&v)[VEC]) {
    if constexpr (VEC == 1) {
        p[0] = v[0];
    } else if constexpr (VEC == 4) {
        *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
    } else {
#pragma unroll
        for (int i = 0; i < VEC / 4; ++i)
            reinterpret_cast<float4 *>(p)[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
    }
}

// Pool epilogue: MEAN = SUM / L, correctly rounded to fp32; an empty bag stays
// 0 for both pools (readings C1, C21).  The quotient is formed in fp64 with a
// Newton-refined reciprocal (relative error < 2^-51) and rounded once to fp32:
// a/L for a 24-bit-mantissa a and integer 1 <= L < 2^24 is never an fp32
// rounding midpoint and lies >= ~2^-49 (relative) away from one, so this
// equals IEEE div.rn -- without div.rn's out-of-line slow-path CALL, whose
// caller-saved spills would otherwise inflate every inlined schedule.
__device__ __forceinline__ float div_by_len(float a, int L) {
    const double b = (double)L;
    double y;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(b));
#pragma unroll
    for (int it = 0; it < 3; ++it) {
        const double e = fma(-b, y, 1.0);
        y = fma(y, e, y);
    }
    return (float)((double)a * y);
}

template <int VEC>
__device__ __forceinline__ void pool_finish(float (&acc)[VEC], int pool, int L) {
    if (pool == RECFLEX_POOL_MEAN && L > 0) {
#pragma unroll
        for (int e = 0; e < VEC; ++e) acc[e] = div_by_len(acc[e], L);
    }
}

// Where the pooled row of sample s goes.  Local mode (rows == 0): out + s *
// stride (out already offset by col_f).  Routed mode (fused pooled-output
// exchange): sample s belongs to destination rank j = s / rows,
// whose [rows][stride] buffer (a peer / IPC-mapped pointer) receives it at row
// s - j*rows, column colofs (+ the lane's column): the all-to-all happens in
// the store epilogue of the fused kernel itself.
struct OutRoute {
    float *const *ptrs;  // destination buffers (routed mode)
    int rows;            // samples per destination, 0 = local mode
    int colofs;          // col_base of this rank + col_f (routed mode)
    int stride;          // row stride of the output (floats)
};

__device__ __forceinline__ float *out_row(float *out, int s, const OutRoute &r) {
    if (r.rows == 0) return out + (size_t)s * r.stride;
    const int j = s / r.rows;
    return r.ptrs[j] + (size_t)(s - j * r.rows) * r.stride + r.colofs;
}

// Everything a schedule needs for one task, passed by value (registers): the
// paper's `args + arg_offsets[feature_idx]` (Fig. 8 line 17) resolved.
struct TaskCtx {
    const char *table;      // T_f (first byte of row 0)
    unsigned rowb;          // bytes per row
    const int32_t *offs;    // this feature's B+1 offsets
    const int32_t *idx;     // all lookup IDs
    float *out;             // out + col_f
    int dim;
    int pool;
    OutRoute ro;            // output placement (local or routed to peers)
    int s0, s1;             // samples of this task
};

// ---- GROUP family --------------------------------------------------------
// One bag [lo, hi) pooled by the G lanes of a group: lane lg holds columns
// p*SPAN + c*G*VEC + lg*VEC (+0..VEC-1); U rows in flight per lane.
template <int ET, int GT, int VEC, int C, int U, int P = 0>
__device__ __forceinline__ void group_bag(const char *__restrict__ T, unsigned rowb, const int32_t *__restrict__ idx, int d,
                                          int pool, float *__restrict__ orow, int lo, int hi, int lg, int gr) {
    const int G = GT ? GT : gr;  // GT == 0: lane-group size at run time (see kRuntimeG)
    const int SPAN = G * VEC * C;
    const int passes = (d + SPAN - 1) / SPAN;
    {
        for (int p = 0; p < passes; ++p) {
            int colv[C];
            bool ok[C];
#pragma unroll
            for (int c = 0; c < C; ++c) {
                colv[c] = p * SPAN + c * G * VEC + lg * VEC;
                ok[c] = colv[c] < d;
            }
            float acc[C][VEC];
#pragma unroll
            for (int c = 0; c < C; ++c)
#pragma unroll
                for (int e = 0; e < VEC; ++e) acc[c][e] = 0.f;

#ifndef RECFLEX_NO_SHFL_IDX
            if (U <= G && G >= 4) {
                // Lookup IDs through registers: lane lg holds ID cb+lg of the
                // current chunk of G IDs (one coalesced load per chunk) and the
                // next chunk is already in flight; each iteration broadcasts its
                // U IDs with shuffles.  This takes the per-iteration index load
                // (20% of heavy's stall samples as a dependent L1 load) off the
                // row loads' critical path.
                const int lane = threadIdx.x & 31;
                const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
                int cb = lo;
                int cur = (lo + lg < hi) ? ld_idx(idx + lo + lg) : 0;
                int nxt = (lo + G + lg < hi) ? ld_idx(idx + lo + G + lg) : 0;
                int j = lo;
                for (; j + U <= hi; j += U) {
                    if (j - cb >= G) {
                        cb += G;
                        cur = nxt;
                        nxt = (cb + G + lg < hi) ? ld_idx(idx + cb + G + lg) : 0;
                    }
                    unsigned id[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) id[u] = (unsigned)__shfl_sync(gmask, cur, (j - cb) + u, G);
                    RowFrag<ET, VEC> v[U][C];
                    rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                    for (int u = 0; u < U; ++u)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                    for (int u = 0; u < U; ++u)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (ok[c])
                                v[u][c].add_to(acc[c]);
                }
                if (j < hi) {
                    if (j - cb >= G) {
                        cb += G;
                        cur = nxt;
                    }
                    const int n = hi - j;
                    unsigned id[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) id[u] = (unsigned)__shfl_sync(gmask, cur, (j - cb) + u, G);
                    RowFrag<ET, VEC> v[U][C];
                    rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                    for (int u = 0; u < U; ++u)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (u < n && ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                    for (int u = 0; u < U; ++u)
                        if (u < n)
#pragma unroll
                            for (int c = 0; c < C; ++c)
                                if (ok[c])
                                    v[u][c].add_to(acc[c]);
                }
#pragma unroll
                for (int c = 0; c < C; ++c) {
                    if (ok[c]) {
                        pool_finish<VEC>(acc[c], pool, hi - lo);
                        st_out<VEC>(orow + colv[c], acc[c]);
                    }
                }
                continue;
            }
#endif
            // U lookup IDs, then their U rows, then the adds: all U row loads are
            // in flight before the first add consumes one (a one-iteration-ahead
            // index prefetch was measured 2x slower: under the register cap
            // ptxas interleaves the in-order adds with the loads).  Rows are
            // added in ascending lookup order (the sequential fp32 bag sum).
            int j = lo;
            for (; j + U <= hi; j += U) {
                int id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = ld_idx(idx + j + u);
                RowFrag<ET, VEC> v[U][C];
                rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (ok[c])
                            v[u][c].add_to(acc[c]);
            }
            if (j < hi) {  // ragged tail of the bag: n < U rows
                const int n = hi - j;
                int id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = (u < n) ? ld_idx(idx + j + u) : 0;
                RowFrag<ET, VEC> v[U][C];
                rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (u < n && ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (u < n)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (ok[c])
                                v[u][c].add_to(acc[c]);
            }
#pragma unroll
            for (int c = 0; c < C; ++c) {
                if (ok[c]) {
                    pool_finish<VEC>(acc[c], pool, hi - lo);
                    st_out<VEC>(orow + colv[c], acc[c]);
                }
            }
        }
    }
}

// Samples [s0, s1) of the task.  Groups claim bags dynamically from a shared
// counter (*bag_ctr, zeroed before the task), so a long-tail bag delays only
// its own group; the next bag's offsets are loaded while the current bag is
// pooled.  Which group pools a bag does not change the bag's arithmetic (rows
// in ascending lookup order) -> results are independent of the claim order.
template <int ET, int GT, int VEC, int C, int U, int P = 0>
RECFLEX_SCHED_FN void sched_group(const char *__restrict__ T, unsigned rowb, int gr, const int32_t *__restrict__ offs,
                                        const int32_t *__restrict__ idx, float *__restrict__ out, int d, int pool,
                                        const OutRoute ro, int s0, int s1, int *bag_ctr) {
    const int G = GT ? GT : gr;
    const int lane = threadIdx.x & 31;
    const int lg = lane & (G - 1);
    const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
    auto claim = [&]() -> int {
        int v = 0;
        if (lg == 0) v = atomicAdd(bag_ctr, 1);
        return s0 + __shfl_sync(gmask, v, 0, G);
    };
    int s = claim();
    int lo = 0, hi = 0;
    if (s < s1) {
        lo = ld_idx(offs + s);
        hi = ld_idx(offs + s + 1);
    }
    while (s < s1) {
        const int sn = claim();
        int lon = 0, hin = 0;
        if (sn < s1) {
            lon = ld_idx(offs + sn);
            hin = ld_idx(offs + sn + 1);
        }
        group_bag<ET, GT, VEC, C, U, P>(T, rowb, idx, d, pool, out_row(out, s, ro), lo, hi, lg, G);
        s = sn;
        lo = lon;
        hi = hin;
    }
}

// ---- WARP-SPLIT family -------------------------------------------------------
// One bag at a time per WARP: its NG = 32/G lane groups share the bag, group g
// taking lookups lo+g, lo+g+NG, ... (U rows each per iteration, so NG*U rows of
// the bag are in flight at once instead of U), then the groups' partials are
// combined with a fixed xor-butterfly (every lane gets bit-identical sums) and
// group 0 stores.  For long bags in small batches, where the GROUP family's
// per-bag chain of L/U dependent row round trips is the critical path (medium,
// fig3).  IDs come through registers: lane l holds ID cb + l of the current
// 32-ID chunk, the next chunk in flight; an iteration consumes R = NG*U IDs
// (R divides 32 for every catalog entry).  Bags are claimed per warp from the
// task's counter (results do not depend on which warp pools a bag).
template <int ET, int GT, int VEC, int C, int U, int P = 0>
RECFLEX_SCHED_FN void sched_warp(const char *__restrict__ T, unsigned rowb, int gr, const int32_t *__restrict__ offs,
                                 const int32_t *__restrict__ idx, float *__restrict__ out, int d, int pool,
                                 const OutRoute ro, int s0, int s1, int *bag_ctr) {
    const int G = GT ? GT : gr;
    const int NG = 32 / G;
    const int R = NG * U;
    const int lane = threadIdx.x & 31;
    const int g = lane / G, lg = lane % G;
    const int SPAN = G * VEC * C;
    const int passes = (d + SPAN - 1) / SPAN;
    while (true) {
        int v = 0;
        if (lane == 0) v = atomicAdd(bag_ctr, 1);
        const int s = s0 + __shfl_sync(0xffffffffu, v, 0);
        if (s >= s1) break;
        const int lo = ld_idx(offs + s), hi = ld_idx(offs + s + 1);
        float *__restrict__ orow = out_row(out, s, ro);
        for (int p = 0; p < passes; ++p) {
            int colv[C];
            bool ok[C];
#pragma unroll
            for (int c = 0; c < C; ++c) {
                colv[c] = p * SPAN + c * G * VEC + lg * VEC;
                ok[c] = colv[c] < d;
            }
            float acc[C][VEC];
#pragma unroll
            for (int c = 0; c < C; ++c)
#pragma unroll
                for (int e = 0; e < VEC; ++e) acc[c][e] = 0.f;
            int cb = lo;
            int cur = (lo + lane < hi) ? ld_idx(idx + lo + lane) : 0;
            int nxt = (lo + 32 + lane < hi) ? ld_idx(idx + lo + 32 + lane) : 0;
            for (int j = lo; j < hi; j += R) {
                if (j - cb >= 32) {
                    cb += 32;
                    cur = nxt;
                    nxt = (cb + 32 + lane < hi) ? ld_idx(idx + cb + 32 + lane) : 0;
                }
                unsigned id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = (unsigned)__shfl_sync(0xffffffffu, cur, (j - cb) + u * NG + g);
                RowFrag<ET, VEC> rv[U][C];
                rf_zero<ET, VEC, U, C>(rv);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (j + u * NG + g < hi && ok[c]) rv[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (j + u * NG + g < hi)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (ok[c]) rv[u][c].add_to(acc[c]);
            }
            // the NG group partials -> one sum (fixed butterfly order)
            for (int o = G; o < 32; o <<= 1)
#pragma unroll
                for (int c = 0; c < C; ++c)
#pragma unroll
                    for (int e = 0; e < VEC; ++e) acc[c][e] += __shfl_xor_sync(0xffffffffu, acc[c][e], o);
            if (g == 0) {
#pragma unroll
                for (int c = 0; c < C; ++c) {
                    if (ok[c]) {
                        pool_finish<VEC>(acc[c], pool, hi - lo);
                        st_out<VEC>(orow + colv[c], acc[c]);
                    }
                }
            }
        }
    }
}

// ---- FLAT family -----------------------------------------------------------
// A group claims a run of kFlatRun consecutive bags and walks their lookups as
// one contiguous range (the KJT stores a run's bags back to back): every
// iteration keeps U rows in flight whatever the bag lengths, so one-hot and
// short bags no longer pay a dependent offsets -> IDs -> rows chain per bag.
// When a row crosses the current bag's end, the finished bag is pooled and
// stored and its accumulator reset; rows of a bag are still added in
// ascending lookup order (same arithmetic as GROUP).
constexpr int kFlatRun = 8;

template <int ET, int GT, int VEC, int U, int P = 0>
RECFLEX_SCHED_FN void sched_flat(const char *__restrict__ T, unsigned rowb, int gr, const int32_t *__restrict__ offs,
                                       const int32_t *__restrict__ idx, float *__restrict__ out, int d, int pool,
                                       const OutRoute ro, int s0, int s1, int *bag_ctr) {
    const int G = GT ? GT : gr;
    const int lane = threadIdx.x & 31;
    const int lg = lane & (G - 1);
    const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
    const int SPAN = G * VEC;
    const int passes = (d + SPAN - 1) / SPAN;
    while (true) {
        int v = 0;
        if (lg == 0) v = atomicAdd(bag_ctr, kFlatRun);
        const int s = s0 + __shfl_sync(gmask, v, 0, G);
        if (s >= s1) break;
        const int se = min(s1, s + kFlatRun);
        const int A = ld_idx(offs + s);
        const int Z = ld_idx(offs + se);
        for (int p = 0; p < passes; ++p) {
            const int col = p * SPAN + lg * VEC;
            const bool ok = col < d;
            float acc[VEC];
#pragma unroll
            for (int e = 0; e < VEC; ++e) acc[e] = 0.f;
            int b = s;               // bag being accumulated
            int bstart = A;          // its first lookup
            int bend = ld_idx(offs + s + 1);
            auto finish_bag = [&]() {
                if (ok) {
                    pool_finish<VEC>(acc, pool, bend - bstart);
                    st_out<VEC>(out_row(out, b, ro) + col, acc);
                }
#pragma unroll
                for (int e = 0; e < VEC; ++e) acc[e] = 0.f;
                ++b;
                bstart = bend;
                if (b < se) bend = ld_idx(offs + b + 1);
            };
            for (int j = A; j < Z; j += U) {
                unsigned id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = (j + u < Z) ? (unsigned)ld_idx(idx + j + u) : 0u;
                RowFrag<ET, VEC> r[U];
                #pragma unroll
                for (int u = 0; u < U; ++u) r[u].zero();
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (j + u < Z && ok) r[u].template load<P>(T + (size_t)id[u] * rowb, col, d);
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    if (j + u < Z) {
                        while (j + u >= bend) finish_bag();
                        r[u].add_to(acc);
                    }
                }
            }
            while (b < se) finish_bag();  // the last bag(s) of the run, incl. trailing empty bags
        }
    }
}

// ---- backward (training) --------------------------------------
// The adjoint of the pooled gather: for every bag (f, s) of the task and every
// lookup j of it, target[idx[j]][c] += scale * w * grad[s][col_f + c] with
// w = 1 (SUM) or 1/L (MEAN, the correctly rounded fp32 quotient).  A group of
// G lanes holds the bag's gradient row in registers (loaded once, 16-byte
// loads) and scatters it to the bag's rows with vector reductions at L2
// (red.global.add.v4.f32, sm_90+): no read-modify-write round trip through the
// SM.  Bags are claimed dynamically as in GROUP; the reduction order across
// bags is not fixed (fp32 adds in L2 commute only up to rounding) -> results
// are exact when every partial sum is exactly representable (integer data)
// and within the summation bound otherwise.
__device__ __forceinline__ void red_add_v4(float *p, float a, float b, float c, float d) {
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(a), "f"(b), "f"(c), "f"(d)
                 : "memory");
}

static __device__ __noinline__ void sched_backward(const float *__restrict__ grad, int gstride, float *__restrict__ target,
                                            const int32_t *__restrict__ offs, const int32_t *__restrict__ idx, int d,
                                            int pool, float scale, int s0, int s1, int *bag_ctr, bool vec_ok) {
    const bool vec = vec_ok && (d % 4) == 0;  // 16-byte aligned grad columns and target rows
    const int per_lane = vec ? 4 : 1;
    int G = 1;
    while (G < 32 && G * per_lane < d) G <<= 1;
    const int lane = threadIdx.x & 31;
    const int lg = lane & (G - 1);
    const unsigned gmask = (G == 32) ? 0xffffffffu : (((1u << G) - 1u) << (lane & ~(G - 1)));
    const int span = G * per_lane;
    while (true) {
        int v = 0;
        if (lg == 0) v = atomicAdd(bag_ctr, 1);
        const int s = s0 + __shfl_sync(gmask, v, 0, G);
        if (s >= s1) break;
        const int lo = ld_idx(offs + s), hi = ld_idx(offs + s + 1);
        const int L = hi - lo;
        if (L == 0) continue;
        const float *gr = grad + (size_t)s * gstride;
        for (int col = lg * per_lane; col < d; col += span) {
            if (vec) {
                const float4 g4 = *reinterpret_cast<const float4 *>(gr + col);
                float g[4] = {g4.x, g4.y, g4.z, g4.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    if (pool == RECFLEX_POOL_MEAN) g[e] = div_by_len(g[e], L);
                    g[e] *= scale;
                }
                int j = lo;
                for (; j + 4 <= hi; j += 4) {  // 4 lookup IDs in flight, then 4 reductions
                    unsigned id[4];
#pragma unroll
                    for (int u = 0; u < 4; ++u) id[u] = (unsigned)ld_idx(idx + j + u);
#pragma unroll
                    for (int u = 0; u < 4; ++u) red_add_v4(target + (size_t)id[u] * (unsigned)d + col, g[0], g[1], g[2], g[3]);
                }
                for (; j < hi; ++j)
                    red_add_v4(target + (size_t)(unsigned)ld_idx(idx + j) * (unsigned)d + col, g[0], g[1], g[2], g[3]);
            } else {
                float g = gr[col];
                if (pool == RECFLEX_POOL_MEAN) g = div_by_len(g, L);
                g *= scale;
                for (int j = lo; j < hi; ++j) atomicAdd(target + (size_t)(unsigned)ld_idx(idx + j) * (unsigned)d + col, g);
            }
        }
    }
}

// ---- BLOCK family ----------------------------------------------------------
// One bag at a time for the whole CTA.  Group g takes lookups lo+g, lo+g+NG, ...
// (adjacent groups read adjacent IDs: coalesced index loads).  Partials:
// xor-butterfly across the groups of a warp (every lane gets bit-identical
// sums), then the 8 warp partials are summed in warp order from shared memory.
template <int ET, int GT, int VEC, int C, int U, int P = 0>
RECFLEX_SCHED_FN void sched_block(const char *__restrict__ T, unsigned rowb, int gr, const int32_t *__restrict__ offs,
                                        const int32_t *__restrict__ idx, float *__restrict__ out, int d, int pool,
                                        const OutRoute ro, int s0, int s1, float *red /* [8][SPAN] */) {
    const int G = GT ? GT : gr;
    const int NG = kBlockThreads / G;
    const int SPAN = G * VEC * C;
    constexpr int NW = kBlockThreads / 32;
    const int tid = threadIdx.x;
    const int gid = tid / G;
    const int lg = tid % G;
    const int warp = tid >> 5;
    const int lane = tid & 31;
    const int passes = (d + SPAN - 1) / SPAN;

    for (int s = s0; s < s1; ++s) {
        const int lo = ld_idx(offs + s);
        const int hi = ld_idx(offs + s + 1);
        float *__restrict__ orow = out_row(out, s, ro);
        for (int p = 0; p < passes; ++p) {
            int colv[C];
            bool ok[C];
#pragma unroll
            for (int c = 0; c < C; ++c) {
                colv[c] = p * SPAN + c * G * VEC + lg * VEC;
                ok[c] = colv[c] < d;
            }
            float acc[C][VEC];
#pragma unroll
            for (int c = 0; c < C; ++c)
#pragma unroll
                for (int e = 0; e < VEC; ++e) acc[c][e] = 0.f;

            // this group's strided share of the bag: lookups lo+gid, lo+gid+NG, ...
            int j = lo + gid;
            for (; j + (U - 1) * NG < hi; j += U * NG) {
                int id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = ld_idx(idx + j + u * NG);
                RowFrag<ET, VEC> v[U][C];
                rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (ok[c])
                            v[u][c].add_to(acc[c]);
            }
            {
                int id[U];
#pragma unroll
                for (int u = 0; u < U; ++u) id[u] = (j + u * NG < hi) ? ld_idx(idx + j + u * NG) : 0;
                RowFrag<ET, VEC> v[U][C];
                rf_zero<ET, VEC, U, C>(v);
#pragma unroll
                for (int u = 0; u < U; ++u)
#pragma unroll
                    for (int c = 0; c < C; ++c)
                        if (j + u * NG < hi && ok[c]) v[u][c].template load<P>(T + (size_t)id[u] * rowb, colv[c], d);
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (j + u * NG < hi)
#pragma unroll
                        for (int c = 0; c < C; ++c)
                            if (ok[c])
                                v[u][c].add_to(acc[c]);
            }
            // groups of one warp -> one partial (butterfly: identical on all lanes)
#pragma unroll
            for (int o = G; o < 32; o <<= 1)
#pragma unroll
                for (int c = 0; c < C; ++c)
#pragma unroll
                    for (int e = 0; e < VEC; ++e) acc[c][e] += __shfl_xor_sync(0xffffffffu, acc[c][e], o);
            if (lane < G) {
#pragma unroll
                for (int c = 0; c < C; ++c)
#pragma unroll
                    for (int e = 0; e < VEC; ++e) red[warp * SPAN + c * G * VEC + lg * VEC + e] = acc[c][e];
            }
            __syncthreads();
            const int L = hi - lo;
            for (int q = tid; q < SPAN; q += kBlockThreads) {
                const int col = p * SPAN + q;
                if (col < d) {
                    float v[1] = {0.f};
#pragma unroll
                    for (int w = 0; w < NW; ++w) v[0] += red[w * SPAN + q];
                    pool_finish<1>(v, pool, L);
                    orow[col] = v[0];
                }
            }
            __syncthreads();
        }
    }
}

}  // namespace recflex
