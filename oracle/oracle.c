/*
 * oracle.c -- CPU oracle for the RecFlex hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (paper_conf_sc_panzzxwslr0d24_b200/) never links,
 * imports or calls it, and shares no code, header or constant with it.
 *
 * Plain, slow, obviously correct: fp64 accumulation, loops in the order the
 * definition states, no blocking, no fusion, no reordering.
 *
 * Functions and the passages they follow (PAPER.md line numbers, "P:n"):
 *
 *   oracle_embedding_bag  -- the embedding-bag operation, P:41 (§II-A, Fig. 1)
 *       and P:51: "An input sample of the operation consists of single or
 *       multiple lookup IDs, which are used to retrieve corresponding rows in
 *       the embedding table.  Then, the retrieved embedding vectors of the
 *       same sample will be applied by a pooling operation (i.e., elementwise
 *       reduction)"; per-feature outputs "are then concatenated".
 *       Readings: C1 pool = SUM or MEAN, empty bag -> 0;
 *       C2 duplicate IDs counted with multiplicity; C6 output row-major
 *       [B][D_tot], feature f at column col_f = sum_{g<f} d_g.
 *       Pinned by tests/test_oracle.py (worked example in tests/golden,
 *       torch.nn.functional.embedding_bag, brute force, closed-form invariants).
 *
 *   oracle_decode         -- the value of element c of a stored table row, per
 *       storage type (the paper is silent on precision,
 *       reading C5): F32 = the float; F16 = IEEE 754 binary16 written out
 *       from its fields (sign, 5-bit exponent with bias 15, 10-bit fraction,
 *       subnormals, inf/nan); BF16 = the 16 bits as the upper half of an IEEE
 *       binary32; I8 = scale * q + bias with q the signed code and scale, bias
 *       the row's two float32 after its d codes (rowwise-quantised row: d
 *       codes, scale, bias, zero padding to a multiple of 16 bytes),
 *       evaluated in fp64; FP8 = OCP E4M3 ("e4m3fn": 4-bit exponent with
 *       bias 7, 3-bit fraction, subnormals, S.1111.111 = NaN, no infinities)
 *       written out from its fields, one byte per element.
 *       Pinned by tests/test_oracle.py: exhaustive over all 2^16 patterns
 *       against numpy float16 and torch bfloat16, all 256 FP8 codes against
 *       torch float8_e4m3fn, hand-decoded I8 and FP8 rows.
 *
 *   oracle_embedding_bag_backward -- the adjoint of oracle_embedding_bag
 *       (training; "there is no fundamental reason
 *       limiting RecFlex from optimizing the training process"): with the
 *       upstream gradient G = dLoss/d out [B][D_tot], row r of table f
 *       receives  sum over bags (f,s) and positions j with indices[j] == r of
 *       w_{f,s} * G[s][col_f + c],  w = 1 (SUM) or 1/L_{f,s} (MEAN), i.e.
 *       the derivative of the definition above.  Written as the update
 *       target_f[r][c] += scale * w * G[s][col_f + c] (scale = 1 into zeroed
 *       buffers: the dense gradient; scale = -lr into the table: one SGD
 *       step).  fp64, in ascending (f, s, j) order; also returns per element
 *       the number of terms and the sum of their magnitudes (for the
 *       floating-point error bound of a GPU result accumulated in any order).
 *       Pinned by tests/test_oracle.py: hand-worked example, torch autograd
 *       of embedding_bag in fp64, the adjoint identity <G, A T> = <A^T G, T>.
 *
 *   oracle_task_map       -- the runtime thread map of Fig. 8:
 *       d_blocks_map[f] = feature_blocks, and d_task_map[b] = (feature_idx,
 *       rel_bidx) enumerating, feature by feature, rel = 0..feature_blocks-1.
 *       The blocks a batch NEEDS follow reading C12 (blocks "adaptive" to the
 *       batch's workload): sample-partitioned schedules take
 *       ceil(B/spb); nnz-partitioned schedules take floor(nnz_f/npb) + 1, where
 *       npb is raised to ceil(nnz_f/(slots_f - 2)) when the feature's reserved
 *       task slots would not hold the batch (reading C12).
 *       Under a static thread mapping the feature instead gets a
 *       fixed number of allocated blocks whatever the batch.  An optional cap
 *       (tuning padding) limits the count.  Pinned by hand-worked
 *       goldens (tests/golden/worked_example.json) and brute-force
 *       enumeration in tests/test_oracle.py.
 *
 *   oracle_static_assignment -- the static thread mapping of P:338: "if we
 *       allocate two blocks to a specific feature at compile time while the
 *       input workload requires three blocks at runtime, the first block will
 *       perform the computation of two blocks sequentially".  Needed block q
 *       (0 <= q < need) is performed by allocated block q mod nalloc as its
 *       (q div nalloc)-th step (reading C31: round robin).  Pinned by the
 *       P:338 golden.
 *
 *   oracle_nnz_task_ranges -- for an nnz-partitioned feature, the samples a
 *       task owns: {s : floor((off[s]-off[0]) / npb) == rel}, written out by
 *       brute force over s for every task (reading C12).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_OK 0
#define ORACLE_ERR_INDEX -1
#define ORACLE_ERR_OFFSETS -2
#define ORACLE_ERR_ARG -3

#define POOL_SUM 0
#define POOL_MEAN 1

#define DT_F32 0
#define DT_F16 1
#define DT_BF16 2
#define DT_I8 3
#define DT_FP8 4

/* bytes per stored row of dimension d */
int64_t oracle_row_bytes(int dtype, int d) {
    switch (dtype) {
        case DT_F16:
        case DT_BF16: return 2 * (int64_t)d;
        case DT_I8: return ((int64_t)d + 8 + 15) / 16 * 16;
        case DT_FP8: return (int64_t)d;
        default: return 4 * (int64_t)d;
    }
}

/* value of element c of the stored row at `row` (d elements) */
double oracle_decode(int dtype, const unsigned char *row, int c, int d) {
    if (dtype == DT_F16) {
        unsigned h = (unsigned)row[2 * c] | ((unsigned)row[2 * c + 1] << 8);
        int sign = (h >> 15) & 1, e = (h >> 10) & 31, m = h & 1023;
        double v;
        if (e == 0) v = ldexp((double)m, -24);                 /* subnormal: m * 2^-24 */
        else if (e == 31) v = m ? NAN : INFINITY;
        else v = ldexp((double)(1024 + m), e - 25);            /* (1 + m/1024) * 2^(e-15) */
        return sign ? -v : v;
    }
    if (dtype == DT_BF16) {
        uint32_t u = ((uint32_t)row[2 * c] | ((uint32_t)row[2 * c + 1] << 8)) << 16;
        float f;
        memcpy(&f, &u, 4);
        return (double)f;
    }
    if (dtype == DT_FP8) {
        /* OCP FP8 E4M3 ("fn"): sign, 4-bit exponent with bias 7, 3-bit
         * fraction; exponent 0 = subnormal m * 2^-9; S.1111.111 = NaN; no inf */
        unsigned b = row[c];
        int sign = (b >> 7) & 1, e = (b >> 3) & 15, m = b & 7;
        double v;
        if (e == 0) v = ldexp((double)m, -9);
        else if (e == 15 && m == 7) v = NAN;
        else v = ldexp((double)(8 + m), e - 10);               /* (1 + m/8) * 2^(e-7) */
        return sign ? -v : v;
    }
    if (dtype == DT_I8) {
        int q = (int)(signed char)row[c];
        float scale, bias;
        memcpy(&scale, row + d, 4);
        memcpy(&bias, row + d + 4, 4);
        return (double)scale * (double)q + (double)bias;
    }
    {
        float f;
        memcpy(&f, row + 4 * (int64_t)c, 4);
        return (double)f;
    }
}

/* decode n stored rows into out[n][d] (for pinning the decode) */
int oracle_decode_rows(int dtype, const void *rows, int64_t n, int d, double *out) {
    const int64_t rb = oracle_row_bytes(dtype, d);
    for (int64_t r = 0; r < n; ++r)
        for (int c = 0; c < d; ++c) out[r * d + c] = oracle_decode(dtype, (const unsigned char *)rows + r * rb, c, d);
    return ORACLE_OK;
}

int oracle_version(void) { return 1; }

int oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/*
 * F features, batch B.
 * dims[f], pools[f], rows[f]; dtypes[f] (NULL = all float32); tables[f] ->
 * [rows[f]] stored rows of oracle_row_bytes(dtypes[f], dims[f]) bytes.
 * indices int32[nnz], offsets int32[F*B+1] (feature-major KJT CSR).
 * out -> double [B][sum(dims)].
 * nthreads <= 0: library default.
 */
int oracle_embedding_bag_typed(int F, int B, const int *dims, const int *pools, const int *dtypes,
                               const void *const *tables, const int64_t *rows,
                               const int32_t *indices, const int32_t *offsets,
                               double *out, int nthreads) {
    if (F <= 0 || B < 0) return ORACLE_ERR_ARG;
    int64_t d_tot = 0;
    int64_t *col = (int64_t *)malloc(sizeof(int64_t) * (size_t)F);
    if (!col) return ORACLE_ERR_ARG;
    for (int f = 0; f < F; ++f) {          /* col_f = sum_{g<f} d_g  (P:41 concatenation) */
        col[f] = d_tot;
        d_tot += dims[f];
    }
    /* validate the CSR once, sequentially (reading C3: precondition) */
    if (offsets[0] != 0) { free(col); return ORACLE_ERR_OFFSETS; }
    for (int64_t k = 0; k < (int64_t)F * B; ++k)
        if (offsets[k + 1] < offsets[k]) { free(col); return ORACLE_ERR_OFFSETS; }
    for (int f = 0; f < F; ++f) {
        int64_t a = offsets[(int64_t)f * B], b = offsets[(int64_t)(f + 1) * B];
        for (int64_t j = a; j < b; ++j)
            if (indices[j] < 0 || (int64_t)indices[j] >= rows[f]) { free(col); return ORACLE_ERR_INDEX; }
    }
#ifdef _OPENMP
    if (nthreads > 0) omp_set_num_threads(nthreads);
#else
    (void)nthreads;
#endif
    /* features write disjoint output columns -> identical result for any thread count */
#pragma omp parallel for schedule(dynamic)
    for (int f = 0; f < F; ++f) {
        const int d = dims[f];
        const int dt = dtypes ? dtypes[f] : DT_F32;
        const int64_t rb = oracle_row_bytes(dt, d);
        const unsigned char *T = (const unsigned char *)tables[f];
        double *acc = (double *)malloc(sizeof(double) * (size_t)(d > 0 ? d : 1));
        for (int s = 0; s < B; ++s) {
            const int64_t lo = offsets[(int64_t)f * B + s];
            const int64_t hi = offsets[(int64_t)f * B + s + 1];
            const int64_t L = hi - lo;
            for (int c = 0; c < d; ++c) acc[c] = 0.0;
            for (int64_t j = lo; j < hi; ++j) {             /* ascending j */
                const unsigned char *row = T + (int64_t)indices[j] * rb;
                for (int c = 0; c < d; ++c) acc[c] += oracle_decode(dt, row, c, d);
            }
            double *o = out + (int64_t)s * d_tot + col[f];
            for (int c = 0; c < d; ++c) {
                if (pools[f] == POOL_MEAN)
                    o[c] = (L > 0) ? acc[c] / (double)L : 0.0;   /* reading C1: empty -> 0 */
                else
                    o[c] = acc[c];
            }
        }
        free(acc);
    }
    free(col);
    return ORACLE_OK;
}

int oracle_embedding_bag(int F, int B, const int *dims, const int *pools,
                         const float *const *tables, const int64_t *rows,
                         const int32_t *indices, const int32_t *offsets,
                         double *out, int nthreads) {
    return oracle_embedding_bag_typed(F, B, dims, pools, NULL, (const void *const *)tables, rows, indices, offsets,
                                      out, nthreads);
}

/*
 * Backward of the embedding bag (the adjoint), fp64.
 * targets[f] -> double [rows[f]][dims[f]] (accumulated into, caller-initialised);
 * grad -> double [B][sum(dims)]; counts[f] (nullable) -> int64 [rows[f]] terms per
 * row; abssum[f] (nullable) -> double [rows[f]][dims[f]] sum of |term| (accumulated).
 */
int oracle_embedding_bag_backward(int F, int B, const int *dims, const int *pools, const int64_t *rows,
                                  const int32_t *indices, const int32_t *offsets, const double *grad, double scale,
                                  double *const *targets, int64_t *const *counts, double *const *abssum) {
    if (F <= 0 || B < 0) return ORACLE_ERR_ARG;
    int64_t d_tot = 0;
    for (int f = 0; f < F; ++f) d_tot += dims[f];
    if (offsets[0] != 0) return ORACLE_ERR_OFFSETS;
    for (int64_t k = 0; k < (int64_t)F * B; ++k)
        if (offsets[k + 1] < offsets[k]) return ORACLE_ERR_OFFSETS;
    int64_t col = 0;
    for (int f = 0; f < F; ++f) {
        const int d = dims[f];
        for (int s = 0; s < B; ++s) {
            const int64_t lo = offsets[(int64_t)f * B + s];
            const int64_t hi = offsets[(int64_t)f * B + s + 1];
            const int64_t L = hi - lo;
            /* MEAN: the term is G / L (a division, as the forward divides the sum
             * by L): exact whenever G is a multiple of L, unlike G * fl(1/L) */
            const int mean = pools[f] == POOL_MEAN && L > 0;
            const double *g = grad + (int64_t)s * d_tot + col;
            for (int64_t j = lo; j < hi; ++j) {
                const int64_t r = indices[j];
                if (r < 0 || r >= rows[f]) return ORACLE_ERR_INDEX;
                for (int c = 0; c < d; ++c) {
                    const double term = scale * (mean ? g[c] / (double)L : g[c]);
                    targets[f][r * d + c] += term;
                    if (abssum) abssum[f][r * d + c] += term < 0 ? -term : term;
                }
                if (counts) counts[f][r] += 1;
            }
        }
        col += d;
    }
    return ORACLE_OK;
}

/*
 * Task map of Fig. 8.
 *   mode[f]:  0 = sample-partitioned (per_block[f] = samples per block)
 *             1 = nnz-partitioned    (per_block[f] = lookups per block)
 *   slots[f]: nnz-partitioned only: task slots reserved for the feature (0 =
 *             unlimited); npb_eff = max(per_block, ceil(nnz_f / (slots - 2)))
 *   static_blocks[f]: 0 = runtime mapping, > 0 = static mapping with that
 *             many allocated blocks
 *   cap[f]:   0 = none, else feature_blocks = min(feature_blocks, cap[f])
 * Any of slots / static_blocks / cap may be NULL (all zero).
 * Outputs need_map[F] (blocks the batch needs), npb_map[F] (effective lookups
 * per block; per_block for mode 0), blocks_map[F] (d_blocks_map),
 * task_feature/task_rel[max_tasks] (d_task_map .x/.y), *num_tasks.
 * Returns ORACLE_ERR_ARG if max_tasks is short or a parameter is invalid.
 */
int oracle_task_map(int F, int B, const int *mode, const int *per_block, const int *slots, const int *static_blocks,
                    const int *cap, const int32_t *offsets, int *need_map, int *npb_map, int *blocks_map,
                    int *task_feature, int *task_rel, int64_t max_tasks, int64_t *num_tasks) {
    int64_t n = 0;
    for (int f = 0; f < F; ++f) {
        int64_t need, npb = per_block[f];
        if (per_block[f] < 1) return ORACLE_ERR_ARG;
        if (mode[f] == 0) {
            need = ((int64_t)B + per_block[f] - 1) / per_block[f];
        } else if (mode[f] == 1) {
            int64_t nnz_f = (int64_t)offsets[(int64_t)(f + 1) * B] - offsets[(int64_t)f * B];
            if (slots && slots[f] > 0) {
                int64_t room = slots[f] - 2;
                if (room < 1) return ORACLE_ERR_ARG;
                int64_t lo = (nnz_f + room - 1) / room;
                if (lo > npb) npb = lo;
            }
            need = nnz_f / npb + 1;
        } else {
            return ORACLE_ERR_ARG;
        }
        if (B == 0) need = 0;
        int64_t blocks = need;
        if (static_blocks && static_blocks[f] > 0 && B > 0) blocks = static_blocks[f];
        if (cap && cap[f] > 0 && blocks > cap[f]) blocks = cap[f];
        if (need_map) need_map[f] = (int)need;
        if (npb_map) npb_map[f] = (int)npb;
        blocks_map[f] = (int)blocks;
        for (int64_t rel = 0; rel < blocks; ++rel) {
            if (n >= max_tasks) return ORACLE_ERR_ARG;
            task_feature[n] = f;
            task_rel[n] = (int)rel;
            ++n;
        }
    }
    *num_tasks = n;
    return ORACLE_OK;
}

/*
 * Static thread mapping: needed block q runs on allocated block
 * alloc_of[q] = q mod nalloc as its seq_of[q] = q div nalloc -th sequential
 * step (reading C31).  Allocated blocks a >= need run nothing.
 */
int oracle_static_assignment(int need, int nalloc, int *alloc_of, int *seq_of) {
    if (need < 0 || nalloc < 1) return ORACLE_ERR_ARG;
    for (int q = 0; q < need; ++q) {
        alloc_of[q] = q % nalloc;
        seq_of[q] = q / nalloc;
    }
    return ORACLE_OK;
}

/*
 * Sample range owned by each task of one nnz-partitioned feature:
 * off -> the feature's B+1 offsets (absolute), npb lookups per block.
 * For task q in [0, blocks): s0[q] = min{s : floor((off[s]-off[0])/npb) >= q}
 * (B if none) and s1[q] = s0[q+1]-style end, computed by brute force as
 * the first and one-past-last s whose floor equals q (empty range -> s0=s1).
 */
int oracle_nnz_task_ranges(int B, int npb, const int32_t *off, int blocks, int *s0, int *s1) {
    for (int q = 0; q < blocks; ++q) {
        int first = -1, last = -1;
        for (int s = 0; s < B; ++s) {
            int64_t t = ((int64_t)off[s] - off[0]) / npb;
            if (t == q) {
                if (first < 0) first = s;
                last = s;
            }
        }
        if (first < 0) {
            /* no bag starts in this task: empty range positioned at the first later bag */
            int pos = B;
            for (int s = 0; s < B; ++s)
                if (((int64_t)off[s] - off[0]) / npb > q) { pos = s; break; }
            s0[q] = pos;
            s1[q] = pos;
        } else {
            s0[q] = first;
            s1[q] = last + 1;
        }
    }
    return ORACLE_OK;
}
