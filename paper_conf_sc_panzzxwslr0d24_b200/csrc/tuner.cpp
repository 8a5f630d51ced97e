// tuner.cpp -- the interference-aware two-stage schedule tuner (§IV-A).
//
//   Eq. 2: L(s; xi) ~ sum_f sum_b l_b^(f)(s^(f); xi^(f)) / (#SM * O/W)
//   Eq. 3: per feature, min over s^(f) of sum_b l_b^(f), under a fixed O
//   Eq. 4: min over O_k of the fused latency with the stage-1 choice s_k
//   Eq. 5: objectives summed over sampled historical batches xi_i
//
// Local stage (Fig. 6/7): for every occupancy k and feature f, ONE
// launch of the fused kernel whose task list is
//   [padding tasks: #SM*k] [every candidate of f, each on its own copy of
//   xi^(f)] [padding tasks: (pad_waves-1)*#SM*k]
// with per-task clock64 timers; each candidate's score is the sum of
// its tasks' cycles (Eq. 3), lowest wins (tie -> lower candidate index).
// Padding tasks are the batch's other features on their current schedules
// ("redundant embedding operations") and keep every SM at k CTAs while
// the candidates run.  The duplicated input of candidate c remaps every ID by
// i -> (i + c*floor(rows/N)) mod rows (reading C17): same statistics, no
// cross-candidate L2 reuse.
// Global stage: for each k, time the real fused forward with s_k at
// occupancy k (median of R event-timed runs after an L2 flush, per batch,
// summed over batches); argmin, tie -> larger k (reading C20).
// Complexity: F*K local evaluations + K global evaluations.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <vector>

#include "plan_internal.h"

using namespace recflex;

// ---------------------------------------------------------------------------
// Selection core (testable with a mock cost function)
// ---------------------------------------------------------------------------
extern "C" recflex_status_t recflex_two_stage_select(int32_t F, int32_t K, const int32_t *ncand,
                                                     recflex_local_cost_fn local_cost,
                                                     recflex_global_cost_fn global_cost, void *user,
                                                     int32_t *choice_out, int32_t *best_k, int64_t *local_calls,
                                                     int64_t *global_calls) {
    if (F <= 0 || K <= 0 || !ncand || !local_cost || !global_cost || !choice_out || !best_k)
        return RECFLEX_ERR_INVALID_ARG;
    for (int f = 0; f < F; ++f)
        if (ncand[f] <= 0) return RECFLEX_ERR_INVALID_ARG;
    std::vector<std::vector<int32_t>> choice(K, std::vector<int32_t>(F, 0));
    int64_t lc = 0, gc = 0;
    // Local stage: one co-execution per (f, k); f outer so a feature's
    // duplicated input is built once and reused for every k.
    for (int f = 0; f < F; ++f) {
        std::vector<double> costs(ncand[f]);
        for (int k = 0; k < K; ++k) {
            std::fill(costs.begin(), costs.end(), std::numeric_limits<double>::infinity());
            local_cost(user, k, f, costs.data());
            ++lc;
            int best = 0;
            for (int c = 1; c < ncand[f]; ++c)
                if (costs[c] < costs[best]) best = c;
            choice[k][f] = best;
        }
    }
    // Global stage
    int bk = 0;
    double bcost = std::numeric_limits<double>::infinity();
    for (int k = 0; k < K; ++k) {
        double c = global_cost(user, k, choice[k].data());
        ++gc;
        if (c <= bcost) {  // tie -> larger k
            bcost = c;
            bk = k;
        }
    }
    std::memcpy(choice_out, choice[bk].data(), sizeof(int32_t) * F);
    *best_k = bk;
    if (local_calls) *local_calls = lc;
    if (global_calls) *global_calls = gc;
    return RECFLEX_OK;
}

namespace {

struct Batch {
    const int32_t *d_idx;
    const int32_t *d_off;
    int B;
    std::vector<int32_t> h_off;  // F*B+1
    int64_t nnz(int f) const { return (int64_t)h_off[(size_t)(f + 1) * B] - h_off[(size_t)f * B]; }
    int64_t begin(int f) const { return h_off[(size_t)f * B]; }
};

template <typename T>
struct DevBuf {
    T *p = nullptr;
    int64_t cap = 0;
    cudaError_t ensure(int64_t n) {
        if (n <= cap) return cudaSuccess;
        cudaFree(p);
        p = nullptr;
        cap = 0;
        cudaError_t e = cudaMalloc(&p, sizeof(T) * std::max<int64_t>(n, 1));
        if (e == cudaSuccess) cap = n;
        return e;
    }
    ~DevBuf() { cudaFree(p); }
};

int64_t task_count(const FeatureDesc &d, int B, int64_t nnz) {
    int64_t blocks;
    if (B == 0) return 0;
    if (d.part == 0) {
        blocks = (B + d.per_block - 1) / d.per_block;
    } else {
        int64_t npb = d.per_block;
        const int64_t room = d.slots - 2;
        const int64_t need = (nnz + room - 1) / room;
        if (need > npb) npb = need;
        blocks = nnz / npb + 1;
    }
    if (d.nalloc > 0) blocks = d.nalloc;
    if (d.cap > 0 && blocks > d.cap) blocks = d.cap;
    return blocks;
}

struct Tuner {
    recflex_plan_s *p;
    cudaStream_t stream;
    std::vector<Batch> batches;
    std::vector<int> ks;
    int reps = 7;
    int pad_waves = 4;
    bool separate = false;  // local_mode 1: separate-combine straw man (ablation)
    bool isolated = false;      // local_mode 2: one padded co-execution launch per candidate (C34)
    bool jit = true;            // stage 2 / guard / refinement time the plan-specialised kernel
    // Tail-aware stage-1 cost (reading C33): a candidate costs its
    // CTA-time share W_c / (#SM * k) plus the part of its longest task that
    // would outlast the whole kernel, max(0, Lmax_c - T_est), T_est = the
    // measured latency of the incoming plan at k on the batch (cycles).
    bool tail = true;
    std::vector<std::vector<double>> t_est;  // [k index][batch] cycles
    double clock_khz = 1.965e6;
    bool trace = std::getenv("RECFLEX_TUNE_TRACE") != nullptr;
    int64_t jit_compiles = 0;
    double compile_seconds = 0;
    int verbose = 0;
    double switch_margin = 0.0;  // C38
    bool position_balance = false;  // C39
    std::vector<std::vector<recflex_schedule_t>> cands;  // per feature
    recflex_status_t err = RECFLEX_OK;
    int64_t local_launches = 0, global_launches = 0;
    double last_global = 0;

    // per-feature tuning inputs (rebuilt when f changes), one per batch
    int cur_f = -1;
    struct TP {
        DevBuf<int32_t> idx, off;
        std::vector<int32_t> h_off;
        std::vector<int> pad_slots;   // KJT slot -> original feature (padding)
        int n_cand = 0;
        int in_F = 0;
    };
    std::vector<TP> tps;

    DevBuf<FeatureDesc> d_desc;
    DevBuf<int32_t> d_bs, d_npb, d_need, d_counter, d_ts, d_part1;
    DevBuf<long long> d_timers;
    DevBuf<float> d_out;
    DevBuf<float> d_flush;
    cudaEvent_t e0 = nullptr, e1 = nullptr;

    void fail(recflex_status_t s) {
        if (err == RECFLEX_OK) err = s;
    }
    void check(cudaError_t e, const char *where = "tuner") {
        if (e != cudaSuccess) fail(cuda_status_at(e, where));
    }

    void build_inputs(int f) {
        const auto t_trace = std::chrono::steady_clock::now();
        struct TraceEnd {
            bool on;
            int f;
            std::chrono::steady_clock::time_point t0;
            ~TraceEnd() {
                if (on)
                    std::fprintf(stderr, "[recflex tune] inputs f=%d %.1f ms\n", f,
                                 std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0)
                                     .count());
            }
        } trace_end{trace, f, t_trace};
        cur_f = f;
        tps.clear();
        tps.resize(batches.size());
        const int n = (int)cands[f].size();
        const int64_t rows = p->desc[f].rows;
        const int kmax = *std::max_element(ks.begin(), ks.end());
        const int64_t pad_target = (int64_t)pad_waves * p->num_sms * kmax;
        for (size_t i = 0; i < batches.size(); ++i) {
            const Batch &bt = batches[i];
            TP &tp = tps[i];
            const int B = bt.B;
            tp.n_cand = n;
            // padding slots: other features, cyclically from f+1, until pad_target tasks
            int64_t ptasks = 0;
            for (int step = 1; ptasks < pad_target && step <= 4 * p->F + 4; ++step) {
                const int g = (p->F == 1) ? f : (f + step) % p->F;
                if (g == f && p->F > 1) continue;
                const int64_t t = task_count(p->desc[g], B, bt.nnz(g));
                if (t <= 0) continue;
                tp.pad_slots.push_back(g);
                ptasks += t;
            }
            tp.in_F = n + (int)tp.pad_slots.size();
            // offsets of the tuning KJT
            tp.h_off.assign((size_t)tp.in_F * B + 1, 0);
            int64_t pos = 0;
            auto put_feature = [&](int slot, int g) {
                const int32_t base = bt.h_off[(size_t)g * B];
                for (int s = 0; s < B; ++s) tp.h_off[(size_t)slot * B + s] = (int32_t)(pos + bt.h_off[(size_t)g * B + s] - base);
                pos += bt.nnz(g);
            };
            for (int c = 0; c < n; ++c) put_feature(c, f);
            for (size_t j = 0; j < tp.pad_slots.size(); ++j) put_feature(n + (int)j, tp.pad_slots[j]);
            tp.h_off[(size_t)tp.in_F * B] = (int32_t)pos;
            if (pos >= (int64_t(1) << 31)) {
                fail(RECFLEX_ERR_NOT_SUPPORTED);
                return;
            }
            check(tp.idx.ensure(pos));
            check(tp.off.ensure((int64_t)tp.in_F * B + 1));
            if (err) return;
            check(cudaMemcpyAsync(tp.off.p, tp.h_off.data(), sizeof(int32_t) * tp.h_off.size(), cudaMemcpyHostToDevice,
                                  stream));
            const int64_t nnz_f = bt.nnz(f);
            for (int c = 0; c < n; ++c) {
                const int64_t shift = (int64_t)c * (rows / std::max(1, n));
                int rc = remap_launch(bt.d_idx + bt.begin(f), tp.idx.p + (int64_t)c * nnz_f, nnz_f, shift, rows, stream);
                if (rc) fail(cuda_status((cudaError_t)rc));
            }
            int64_t at = (int64_t)n * nnz_f;
            for (int g : tp.pad_slots) {
                const int64_t m = bt.nnz(g);
                if (m > 0)
                    check(cudaMemcpyAsync(tp.idx.p + at, bt.d_idx + bt.begin(g), sizeof(int32_t) * m,
                                          cudaMemcpyDeviceToDevice, stream));
                at += m;
            }
            check(cudaStreamSynchronize(stream));
        }
    }

    // Eq. 3 costs of all candidates of f at occupancy ks[ki], summed over batches.
    // Straw man 1 of the paper (ablation P:324 / Fig. 11): every
    // candidate in its OWN non-padded launch, cost = its measured latency.
    void local_cost_separate(int ki, int f, double *costs) {
        const int k = ks[ki];
        const int n = (int)cands[f].size();
        const FeatureDesc &base = p->desc[f];
        for (int c = 0; c < n; ++c) costs[c] = 0;
        for (size_t i = 0; i < batches.size(); ++i) {
            const Batch &bt = batches[i];
            TP &tp = tps[i];
            const int B = bt.B;
            for (int c = 0; c < n; ++c) {
                FeatureDesc d = base;
                d.sched = cands[f][c].sched_id;
                d.part = cands[f][c].part;
                d.per_block = cands[f][c].per_block;
                d.cap = 0;
                d.nalloc = 0;
                d.in_feature = c;
                d.col = 0;
                d.slot_base = 0;
                if (d.part == 1) d.slots = (int32_t)(bt.nnz(f) / d.per_block + 3);
                d.table = p->tables[f];
                const int32_t p1 = 0;
                check(d_desc.ensure(1));
                check(d_bs.ensure(2));
                check(d_npb.ensure(1));
                check(d_need.ensure(1));
                check(d_counter.ensure(4));
                check(d_ts.ensure(std::max<int64_t>(d.part == 1 ? d.slots : 1, 1)));
                check(d_part1.ensure(1));
                check(d_out.ensure((int64_t)B * ((base.dim + 3) / 4 * 4)));
                if (err) return;
                check(cudaMemcpyAsync(d_desc.p, &d, sizeof(FeatureDesc), cudaMemcpyHostToDevice, stream));
                check(cudaMemcpyAsync(d_part1.p, &p1, sizeof(int32_t), cudaMemcpyHostToDevice, stream));
                Exec ex;
                ex.F = 1;
                ex.in_F = tp.in_F;
                ex.d_desc = d_desc.p;
                ex.d_block_start = d_bs.p;
                ex.d_npb_eff = d_npb.p;
                ex.d_need = d_need.p;
                ex.d_counter = d_counter.p;
                ex.d_task_start = d_ts.p;
                ex.d_part1 = d_part1.p;
                ex.num_part1 = d.part == 1 ? 1 : 0;
                std::vector<float> ms;
                for (int r = 0; r < 4; ++r) {
                    check(cudaEventRecord(e0, stream));
                    recflex_status_t st = run_pipeline(p, ex, tp.idx.p, tp.off.p, B, d_out.p,
                                                       (base.dim + 3) / 4 * 4, k, stream, nullptr);
                    if (st != RECFLEX_OK) {
                        fail(st);
                        return;
                    }
                    check(cudaEventRecord(e1, stream));
                    check(cudaEventSynchronize(e1));
                    float t = 0;
                    cudaEventElapsedTime(&t, e0, e1);
                    if (r) ms.push_back(t);
                    ++local_launches;
                }
                std::sort(ms.begin(), ms.end());
                costs[c] += ms[ms.size() / 2];
            }
        }
    }

    void local_cost(int ki, int f, double *costs) {
        if (err) return;
        if (cur_f != f) build_inputs(f);
        if (err) return;
        if (separate) {
            local_cost_separate(ki, f, costs);
            return;
        }
        const int k = ks[ki];
        const int n = (int)cands[f].size();
        const auto t_trace = std::chrono::steady_clock::now();
        struct TraceEnd {
            bool on;
            int k, f, n;
            std::chrono::steady_clock::time_point t0;
            ~TraceEnd() {
                if (on)
                    std::fprintf(stderr, "[recflex tune] local k=%d f=%d candidates=%d %.1f ms\n", k, f, n,
                                 std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0)
                                     .count());
            }
        } trace_end{trace, k, f, n, t_trace};
        std::vector<double> sum(n, 0.0);
        const FeatureDesc &base = p->desc[f];
        // co-execution groups: all candidates in one padded launch (the paper's
        // Eq. 3), or -- isolated mode -- one padded launch per candidate, whose
        // cost is then the launch's TOTAL block time (own tasks + the slowdown it
        // inflicts on the identical padding; reading C34)
        std::vector<std::vector<int>> groups;
        if (isolated) {
            for (int c = 0; c < n; ++c) groups.push_back({c});
        } else {
            groups.emplace_back();
            for (int c = 0; c < n; ++c) groups.back().push_back(c);
        }
        for (size_t i = 0; i < batches.size(); ++i)
        for (const std::vector<int> &grp0 : groups) {
            // position balance (C39): the candidates' tasks follow one another in the
            // launch, so the first ones overlap the pre-padding and the last ones the
            // post-padding; every other (batch, k) lists them in reverse so each
            // candidate sees both ends equally
            std::vector<int> grp = grp0;
            if (position_balance && ((i + (size_t)ki) & 1)) std::reverse(grp.begin(), grp.end());
            const Batch &bt = batches[i];
            TP &tp = tps[i];
            const int B = bt.B;
            // descriptor list: [pre padding][candidates][post padding]
            std::vector<FeatureDesc> ds;
            const int64_t pre_target = (int64_t)p->num_sms * k;
            const int64_t post_target = (int64_t)(pad_waves - 1) * p->num_sms * k;
            int dim_max = 4;
            for (int g : tp.pad_slots) dim_max = std::max(dim_max, p->desc[g].dim);
            const int dump_col = ((n * base.dim + 3) / 4) * 4;
            const int d_tp = ((dump_col + dim_max + 3) / 4) * 4;
            size_t ps = 0;
            auto add_pad = [&](int64_t target) {
                int64_t got = 0;
                while (got < target && ps < tp.pad_slots.size()) {
                    const int g = tp.pad_slots[ps];
                    FeatureDesc d = p->desc[g];
                    d.nalloc = 0;
                    d.in_feature = n + (int)ps;
                    d.col = dump_col;
                    const int64_t nnz = bt.nnz(g);
                    if (d.part == 1) d.slots = (int32_t)(nnz / d.per_block + 3);
                    int64_t t = task_count(d, B, nnz);
                    if (got + t > target) {
                        d.cap = (int32_t)(target - got);
                        t = d.cap;
                    }
                    got += t;
                    ds.push_back(d);
                    ++ps;
                }
            };
            add_pad(pre_target);
            const int cand_first = (int)ds.size();
            for (int c : grp) {
                FeatureDesc d = base;
                d.sched = cands[f][c].sched_id;
                d.part = cands[f][c].part;
                d.per_block = cands[f][c].per_block;
                d.cap = 0;
                d.nalloc = 0;
                d.in_feature = c;
                d.col = c * base.dim;
                d.rows = base.rows;
                if (d.part == 1) d.slots = (int32_t)(bt.nnz(f) / d.per_block + 3);
                ds.push_back(d);
            }
            add_pad(post_target);
            // slots for part-1 descriptors
            int64_t slot = 0;
            std::vector<int32_t> part1;
            int64_t total = 0;
            std::vector<int64_t> first(ds.size() + 1, 0);
            for (size_t v = 0; v < ds.size(); ++v) {
                FeatureDesc &d = ds[v];
                d.table = p->tables[d.in_feature < n ? f : tp.pad_slots[d.in_feature - n]];
                if (d.part == 1) {
                    d.slot_base = (int32_t)slot;
                    slot += d.slots;
                    part1.push_back((int32_t)v);
                }
                first[v] = total;
                const int g = d.in_feature < n ? f : tp.pad_slots[d.in_feature - n];
                total += task_count(d, B, bt.nnz(g));
            }
            first[ds.size()] = total;
            const int V = (int)ds.size();
            check(d_desc.ensure(V));
            check(d_bs.ensure(V + 1));
            check(d_npb.ensure(V));
            check(d_need.ensure(V));
            check(d_counter.ensure(4));
            check(d_ts.ensure(std::max<int64_t>(slot, 1)));
            check(d_part1.ensure(std::max<int64_t>((int64_t)part1.size(), 1)));
            check(d_timers.ensure(std::max<int64_t>(total, 1)));
            check(d_out.ensure((int64_t)B * d_tp));
            if (err) return;
            check(cudaMemcpyAsync(d_desc.p, ds.data(), sizeof(FeatureDesc) * V, cudaMemcpyHostToDevice, stream));
            if (!part1.empty())
                check(cudaMemcpyAsync(d_part1.p, part1.data(), sizeof(int32_t) * part1.size(), cudaMemcpyHostToDevice,
                                      stream));
            check(cudaMemsetAsync(d_timers.p, 0, sizeof(long long) * std::max<int64_t>(total, 1), stream));
            Exec ex;
            ex.F = V;
            ex.in_F = tp.in_F;
            ex.d_desc = d_desc.p;
            ex.d_block_start = d_bs.p;
            ex.d_npb_eff = d_npb.p;
            ex.d_need = d_need.p;
            ex.d_counter = d_counter.p;
            ex.d_task_start = d_ts.p;
            ex.d_part1 = d_part1.p;
            ex.num_part1 = (int)part1.size();
            ex.d_timers = d_timers.p;
            ex.timers_cap = (int)total;
            recflex_status_t st = run_pipeline(p, ex, tp.idx.p, tp.off.p, B, d_out.p, d_tp, k, stream, nullptr);
            if (st != RECFLEX_OK) {
                fail(st);
                return;
            }
            ++local_launches;
            std::vector<long long> tm(total);
            std::vector<int32_t> bs(V + 1);
            check(cudaMemcpyAsync(tm.data(), d_timers.p, sizeof(long long) * total, cudaMemcpyDeviceToHost, stream));
            check(cudaMemcpyAsync(bs.data(), d_bs.p, sizeof(int32_t) * (V + 1), cudaMemcpyDeviceToHost, stream));
            check(cudaStreamSynchronize(stream));
            if (err) return;
            const double P = (double)p->num_sms * k;
            const double T_est = (tail && ki < (int)t_est.size() && i < t_est[ki].size()) ? t_est[ki][i] : 0.0;
            // latency-bound batch (the incoming plan fills < 2 waves of tasks): the
            // kernel time is the longest task chain, so a candidate costs its
            // longest task (a separable surrogate of max_f Lmax_f); otherwise its
            // CTA-time share plus the tail beyond T_est (reading C33)
            bool latency_bound = false;
            if (tail) {
                double tasks = 0;
                for (int g = 0; g < p->F; ++g) tasks += (double)task_count(p->desc[g], B, bt.nnz(g));
                latency_bound = tasks < 2.0 * P;
            }
            double pad_sum = 0;  // isolated mode: the padding's block time in this launch
            if (isolated) {
                for (int v = 0; v < V; ++v) {
                    if (v >= cand_first && v < cand_first + (int)grp.size()) continue;
                    for (int64_t t = bs[v]; t < bs[v + 1]; ++t) pad_sum += (double)tm[t];
                }
            }
            for (size_t gi = 0; gi < grp.size(); ++gi) {
                const int c = grp[gi];
                const int v = cand_first + (int)gi;
                double s = 0, mx = 0;
                for (int64_t t = bs[v]; t < bs[v + 1]; ++t) {
                    s += (double)tm[t];
                    mx = std::max(mx, (double)tm[t]);
                }
                sum[c] += latency_bound ? mx : (s + pad_sum) / P + (T_est > 0 ? std::max(0.0, mx - T_est) : 0.0);
            }
        }
        for (int c = 0; c < n; ++c) costs[c] = sum[c];
    }

    // Latency of the plan's incoming schedules at occupancy ks[ki] on every batch
    // (median of `reps` timed forwards after an L2 flush), in SM cycles.
    void measure_incoming(int ki) {
        const int k = ks[ki];
        p->k = k;
        recflex_status_t st = upload_desc(p, stream);
        if (st != RECFLEX_OK) {
            fail(st);
            return;
        }
        if ((int)t_est.size() <= ki) t_est.resize(ki + 1);
        t_est[ki].assign(batches.size(), 0.0);
        for (size_t i = 0; i < batches.size(); ++i) {
            const Batch &bt = batches[i];
            check(d_out.ensure((int64_t)bt.B * p->d_tot));
            if (err) return;
            std::vector<float> ms;
            for (int r = 0; r < std::max(3, reps / 2) + 1; ++r) {
                int rc = flush_launch(d_flush.p, sizeof(float) * d_flush.cap, stream);
                if (rc) fail(cuda_status((cudaError_t)rc));
                check(cudaEventRecord(e0, stream));
                st = run_pipeline(p, p->ex, bt.d_idx, bt.d_off, bt.B, d_out.p, (int)p->d_tot, k, stream, nullptr);
                if (st != RECFLEX_OK) {
                    fail(st);
                    return;
                }
                check(cudaEventRecord(e1, stream));
                check(cudaEventSynchronize(e1));
                float t = 0;
                cudaEventElapsedTime(&t, e0, e1);
                ++global_launches;
                if (r > 0) ms.push_back(t);
            }
            std::sort(ms.begin(), ms.end());
            t_est[ki][i] = ms[ms.size() / 2] * clock_khz;  // ms x kHz = cycles
        }
    }

    void apply(const int32_t *choice) {
        for (int f = 0; f < p->F; ++f) {
            const recflex_schedule_t &s = cands[f][choice[f]];
            if (p->desc[f].sched != s.sched_id) ++p->sched_version;
            p->desc[f].sched = s.sched_id;
            p->desc[f].part = s.part;
            p->desc[f].per_block = s.per_block;
        }
        p->desc_dirty = true;
    }

    // Eq. 4 latency of the fused forward with `choice` at occupancy ks[ki] (ms, Eq. 5 sum).
    double global_cost(int ki, const int32_t *choice) {
        if (err) return std::numeric_limits<double>::infinity();
        apply(choice);
        const int k = ks[ki];
        p->k = k;
        recflex_status_t st = upload_desc(p, stream);
        if (st != RECFLEX_OK) {
            fail(st);
            return 1e30;
        }
        if (jit && !jit_ready(p, k)) {
            // the kernel this choice compiles to is the one forwards will run
            const auto t0 = std::chrono::steady_clock::now();
            st = jit_compile_plan(p, &k, 1);
            compile_seconds += std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            ++jit_compiles;
            if (st != RECFLEX_OK) {
                fail(st);
                return 1e30;
            }
        }
        double total = 0;
        for (const Batch &bt : batches) {
            check(d_out.ensure((int64_t)bt.B * p->d_tot));
            if (err) return 1e30;
            std::vector<float> ms;
            for (int r = 0; r < reps + 1; ++r) {
                int rc = flush_launch(d_flush.p, sizeof(float) * d_flush.cap, stream);
                if (rc) fail(cuda_status((cudaError_t)rc));
                check(cudaEventRecord(e0, stream));
                st = run_pipeline(p, p->ex, bt.d_idx, bt.d_off, bt.B, d_out.p, (int)p->d_tot, k, stream, nullptr);
                if (st != RECFLEX_OK) {
                    fail(st);
                    return 1e30;
                }
                check(cudaEventRecord(e1, stream));
                check(cudaEventSynchronize(e1));
                float t = 0;
                cudaEventElapsedTime(&t, e0, e1);
                ++global_launches;
                if (r > 0) ms.push_back(t);  // first run = warm-up
            }
            std::sort(ms.begin(), ms.end());
            total += ms[ms.size() / 2];
        }
        if (verbose) {
            std::fprintf(stderr, "[recflex tune] global k=%d: %.4f ms  schedules:", k, total);
            std::vector<std::pair<long, int>> hist;
            for (int f = 0; f < p->F; ++f) {
                const recflex_schedule_t &s = cands[f][choice[f]];
                const long key = ((long)s.sched_id * 2 + s.part) * 100000 + s.per_block;
                bool found = false;
                for (auto &h : hist)
                    if (h.first == key) {
                        ++h.second;
                        found = true;
                    }
                if (!found) hist.push_back({key, 1});
            }
            std::sort(hist.begin(), hist.end(), [](auto &a, auto &b) { return a.second > b.second; });
            for (size_t i = 0; i < hist.size() && i < 6; ++i) {
                const long key = hist[i].first;
                const int sid = (int)(key / 100000 / 2), part = (int)(key / 100000 % 2);
                const CatalogEntry &e = kCatalog[sid];
                std::fprintf(stderr, " %dx[%s G%d V%d C%d U%d p%d/%ld]", hist[i].second,
                             e.family == 3 ? "warp" : e.family == 2 ? "flat" : (e.family ? "block" : "group"),
                             e.G, e.VEC, e.C, e.U, part, key % 100000);
            }
            std::fprintf(stderr, "\n");
        }
        last_global = total;
        return total;
    }
};

// Stage-1 costs as the selection sees them: with a switch margin (C38) every
// candidate other than the incoming schedule (candidate 0) is charged
// 1 / (1 - margin) x its measured cost, so a feature leaves its schedule only
// for a predicted gain larger than the margin.
void cb_local(void *u, int32_t ki, int32_t f, double *costs) {
    Tuner *T = static_cast<Tuner *>(u);
    T->local_cost(ki, f, costs);
    if (T->switch_margin > 0.0)
        for (int c = 1; c < (int)T->cands[f].size(); ++c) costs[c] /= (1.0 - T->switch_margin);
}
double cb_global(void *u, int32_t ki, const int32_t *choice) { return static_cast<Tuner *>(u)->global_cost(ki, choice); }

std::vector<recflex_schedule_t> candidates_for(const recflex_plan_s *p, int f, int max_c) {
    std::vector<recflex_schedule_t> out;
    const recflex_feature_spec_t &sp = p->specs[f];
    const FeatureDesc &d = p->desc[f];
    // the plan's current schedule is always candidate 0 (tie -> keep it)
    out.push_back({d.sched, d.part, d.per_block, 0});
    const bool multi_hot = sp.max_len > 1.5f;
    auto add = [&](const recflex_schedule_t &s) {
        for (auto &o : out)
            if (o.sched_id == s.sched_id && o.part == s.part && o.per_block == s.per_block) return;
        out.push_back(s);
    };
    // User-supplied candidate list -- our prior: single-pass entries
    // with one column chunk per lane (multi-pass / C=2 entries re-traverse the
    // bag or idle half the lanes and measured 2-3x slower on B200); they are
    // admitted only when a dim has no single-pass entry.
    for (int relax = 0; relax < 2 && out.size() <= 1; ++relax) {
        for (int id = 0; id < kCatalogSize; ++id) {
            const CatalogEntry &e = kCatalog[id];
            recflex_schedule_t s = {id, 0, 1, 0};
            s.per_block = samples_per_task_default(id, sp.mean_len, sp.coverage, p->task_lookups);
            if (!schedule_valid_for(s, d.dim, d.dtype, d.col, (int)p->d_tot)) continue;
            const int span = e.G * e.VEC * e.C;
            const int passes = (d.dim + span - 1) / span;
            if (relax == 0 && (passes > 1 || e.C > 1)) continue;
            if (relax == 1 && passes > 2) continue;
            if (e.VEC == 1 && d.dim % 4 == 0) continue;  // scalar only where vectors cannot run
            if (!multi_hot && (e.family == RECFLEX_FAMILY_BLOCK || e.family == RECFLEX_FAMILY_WARP)) continue;
            if (!multi_hot && e.family == RECFLEX_FAMILY_GROUP && e.U > 2) continue;  // one bag = one row
            add(s);
            if (multi_hot && e.family != RECFLEX_FAMILY_BLOCK) add({id, 1, std::max(128, p->task_lookups)});
        }
    }
    if (max_c > 0 && (int)out.size() > max_c) out.resize(max_c);
    return out;
}

}  // namespace

extern "C" recflex_status_t recflex_tune_ex(recflex_plan_t p, int32_t N, const int32_t *const *indices,
                                            const int32_t *const *offsets, const int32_t *batch_sizes,
                                            const void *const *tables, void *stream_,
                                            const recflex_tune_options_t *opt, recflex_tune_stats_t *stats) {
    NvtxRange nvtx("recflex_tune");
    if (!p || N <= 0 || !indices || !offsets || !batch_sizes || !tables) return RECFLEX_ERR_INVALID_ARG;
    auto t_start = std::chrono::steady_clock::now();
    cudaStream_t stream = (cudaStream_t)stream_;
    cudaSetDevice(p->device);
    Tuner T;
    T.p = p;
    T.stream = stream;
    if (opt && opt->num_occupancies > 0) {
        for (int i = 0; i < opt->num_occupancies && i < kMaxOcc; ++i) {
            if (opt->occupancies[i] < 1 || opt->occupancies[i] > kMaxOcc) return RECFLEX_ERR_INVALID_ARG;
            T.ks.push_back(opt->occupancies[i]);
        }
        std::sort(T.ks.begin(), T.ks.end());
        T.ks.erase(std::unique(T.ks.begin(), T.ks.end()), T.ks.end());
    } else {
        for (int k = 1; k <= kMaxOcc; ++k) T.ks.push_back(k);
    }
    if (opt && opt->reps > 0) T.reps = opt->reps;
    if (opt && opt->pad_waves > 0) T.pad_waves = opt->pad_waves;
    if (opt) T.verbose = opt->verbose;
    if (opt) T.separate = opt->local_mode == 1;
    if (opt) T.isolated = opt->local_mode == 2;
    if (opt) T.jit = opt->stage2_catalog == 0;
    if (opt) {
        if (!(opt->switch_margin >= 0.f && opt->switch_margin < 1.f)) return RECFLEX_ERR_INVALID_ARG;
        T.switch_margin = opt->switch_margin;
        T.position_balance = opt->position_balance != 0;
    }
    const int max_c = opt ? opt->max_candidates : 0;
    for (int i = 0; i < N; ++i) {
        if (batch_sizes[i] <= 0 || batch_sizes[i] > p->max_batch || !indices[i] || !offsets[i])
            return RECFLEX_ERR_INVALID_ARG;
    }
    // tables -> descriptors
    for (int f = 0; f < p->F; ++f) {
        if (!tables[f] || ((uintptr_t)tables[f]) % 32) return RECFLEX_ERR_INVALID_ARG;
        p->tables[f] = tables[f];
    }
    p->desc_dirty = true;
    for (int k : T.ks) {
        recflex_status_t st = prepare_occupancy(p, k);
        if (st != RECFLEX_OK) return st;
    }
    T.batches.resize(N);
    for (int i = 0; i < N; ++i) {
        Batch &b = T.batches[i];
        b.d_idx = indices[i];
        b.d_off = offsets[i];
        b.B = batch_sizes[i];
        b.h_off.resize((size_t)p->F * b.B + 1);
        cudaError_t e = cudaMemcpy(b.h_off.data(), offsets[i], sizeof(int32_t) * b.h_off.size(), cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return cuda_status(e);
    }
    T.cands.resize(p->F);
    std::vector<int32_t> ncand(p->F);
    for (int f = 0; f < p->F; ++f) {
        T.cands[f] = candidates_for(p, f, max_c);
        ncand[f] = (int32_t)T.cands[f].size();
    }
    if (T.d_flush.ensure(64 << 20) != cudaSuccess) return RECFLEX_ERR_OOM;  // 256 MB = 2x L2
    cudaEventCreate(&T.e0);
    cudaEventCreate(&T.e1);
    if (opt && opt->no_tail) T.tail = false;
    if (T.tail) {
        int khz = 0;
        if (cudaDeviceGetAttribute(&khz, cudaDevAttrClockRate, p->device) == cudaSuccess && khz > 0)
            T.clock_khz = (double)khz;
        const int k0 = p->k;
        for (int ki = 0; ki < (int)T.ks.size(); ++ki) T.measure_incoming(ki);
        p->k = k0;
        if (T.err != RECFLEX_OK) return T.err;
    }
    std::vector<int32_t> choice(p->F);
    int32_t best_k = 0;
    int64_t lc = 0, gc = 0;
    recflex_status_t st = recflex_two_stage_select(p->F, (int32_t)T.ks.size(), ncand.data(), cb_local, cb_global, &T,
                                                   choice.data(), &best_k, &lc, &gc);
    struct EvGuard {
        Tuner &t;
        ~EvGuard() {
            cudaEventDestroy(t.e0);
            cudaEventDestroy(t.e1);
        }
    } guard{T};
    if (st == RECFLEX_OK) st = T.err;
    if (st != RECFLEX_OK) return st;
    // re-measure the two-stage selection, then the guard: the plan's incoming
    // schedules (candidate 0 of every feature) at each k; keep whichever is
    // faster (an untuned-or-previous plan is never made slower by tuning).
    double best_ms = T.global_cost(best_k, choice.data());
    const double two_stage_ms = best_ms;
    double incoming_ms = 0;
    int64_t guard_evals = 0;
    if (!(opt && opt->skip_guard)) {
        std::vector<int32_t> zero(p->F, 0);
        if (T.jit) {  // the incoming schedules at every k: one concurrent compile
            T.apply(zero.data());
            const auto t0 = std::chrono::steady_clock::now();
            st = jit_compile_plan(p, T.ks.data(), (int)T.ks.size());
            T.compile_seconds += std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
            T.jit_compiles += (int64_t)T.ks.size();
            if (st != RECFLEX_OK) return st;
        }
        incoming_ms = std::numeric_limits<double>::infinity();
        for (int ki = 0; ki < (int)T.ks.size(); ++ki) {
            const double c0 = T.global_cost(ki, zero.data());
            ++guard_evals;
            incoming_ms = std::min(incoming_ms, c0);
            if (c0 < best_ms) {
                best_ms = c0;
                best_k = ki;
                choice = zero;
            }
        }
    }
    if (T.err != RECFLEX_OK) return T.err;
    // Refinement (optional, on by default): features sharing a schedule class
    // ("features with identical embedding dimensions and workloads can
    // have the same optimal schedule") form clusters; for each cluster, each
    // candidate is tried on the whole cluster inside the REAL fused forward at
    // the chosen k and kept if it lowers the measured latency by > 0.5%.  This
    // measures what co-execution cannot see on a bandwidth-saturated B200: the
    // DRAM cost a schedule imposes on everyone else.
    int64_t refine_evals = 0;
    const double before_refine = best_ms;
    const auto t_refine = std::chrono::steady_clock::now();
    if (opt && opt->refine) {
        std::vector<std::vector<int>> clusters;
        std::vector<long> keys;
        for (int f = 0; f < p->F; ++f) {
            const recflex_feature_spec_t &sp = p->specs[f];
            const float el = sp.mean_len;
            const int lb = sp.max_len <= 1.f ? 0 : (el < 4.f ? 1 : (el < 32.f ? 2 : 3));
            const long key = ((long)sp.dim * 16 + lb * 4 + (int)T.cands[f].size() % 4) * 8 + sp.dtype;
            size_t c = 0;
            while (c < keys.size() && keys[c] != key) ++c;
            if (c == keys.size()) {
                keys.push_back(key);
                clusters.emplace_back();
            }
            clusters[c].push_back(f);
        }
        for (const auto &cl : clusters) {
            const int nc = (int)T.cands[cl[0]].size();
            bool uniform = true;
            for (int f : cl) uniform &= ((int)T.cands[f].size() == nc);
            if (!uniform) continue;
            for (int c = 0; c < nc; ++c) {
                bool same = true;
                for (int f : cl) same &= (choice[f] == c);
                if (same) continue;
                std::vector<int32_t> trial = choice;
                for (int f : cl) trial[f] = c;
                const double t = T.global_cost(best_k, trial.data());
                ++refine_evals;
                if (t < best_ms * 0.995) {
                    best_ms = t;
                    choice = trial;
                }
            }
            if (T.err != RECFLEX_OK) return T.err;
        }
    }
    const double refine_seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t_refine).count();
    T.apply(choice.data());
    p->k = T.ks[best_k];
    st = upload_desc(p, stream);
    if (st != RECFLEX_OK) return st;
    if (T.jit) {
        // stage 2 over the plan's two kernels for the final choice: the
        // plan-specialised kernel (compiled; usually a disk-cache hit) vs the
        // catalog kernel, on the first historical batch
        st = recflex_select_kernel(p, T.batches[0].d_idx, T.batches[0].d_off, T.batches[0].B, p->tables.data(),
                                   T.reps, nullptr, nullptr, stream);
        if (st != RECFLEX_OK) return st;
    }
    int32_t size_choice = -1;
    if (!(opt && opt->keep_task_size)) {
        // the task granularity the final kernel runs fastest with (C37)
        st = recflex_select_task_size(p, T.batches[0].d_idx, T.batches[0].d_off, T.batches[0].B, p->tables.data(),
                                      T.reps, &size_choice, nullptr, stream);
        if (st != RECFLEX_OK) return st;
    }
    int32_t order_kind = -1;
    if (!(opt && opt->keep_order)) {
        // the task order the final kernel runs fastest under (C35)
        st = recflex_select_task_order(p, T.batches[0].d_idx, T.batches[0].d_off, T.batches[0].B, p->tables.data(),
                                       T.reps, &order_kind, nullptr, stream);
        if (st != RECFLEX_OK) return st;
    }
    int32_t l2_choice = -1;
    if (!(opt && opt->keep_l2) && T.jit && p->use_jit) {
        // the L2 eviction priorities the final kernel runs fastest with (C36)
        st = recflex_select_l2_policy(p, T.batches[0].d_idx, T.batches[0].d_off, T.batches[0].B, p->tables.data(),
                                      T.reps, int64_t(126) << 20, &l2_choice, nullptr, stream);
        if (st != RECFLEX_OK) return st;
    }
    recflex_tune_stats_t s = {};
    s.task_order = order_kind;
    s.l2_policy = l2_choice;
    s.task_size = size_choice;
    s.two_stage_ms = two_stage_ms;
    s.incoming_ms = incoming_ms;
    s.jit_compiles = T.jit_compiles;
    s.compile_seconds = T.compile_seconds;
    s.refine_seconds = refine_seconds;
    s.refine_evals = refine_evals;
    s.refine_gain = before_refine > 0 ? before_refine / best_ms : 1.0;
    s.local_launches = T.local_launches;
    s.global_launches = T.global_launches;
    s.local_evals = lc;
    s.global_evals = gc;
    s.guard_evals = guard_evals;
    s.guard_won = 0;
    for (int f = 0; f < p->F && guard_evals; ++f) s.guard_won |= (choice[f] != 0);
    s.guard_won = guard_evals ? !s.guard_won : 0;
    s.best_occupancy = p->k;
    s.best_ms = best_ms;
    s.tune_seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - t_start).count();
    p->last_stats = s;
    if (stats) *stats = s;
    if (T.verbose) {
        std::fprintf(stderr, "[recflex tune] best k=%d, %.4f ms, %lld local + %lld global launches, %.1f s\n", p->k,
                     best_ms, (long long)s.local_launches, (long long)s.global_launches, s.tune_seconds);
    }
    return T.err;
}

extern "C" recflex_status_t recflex_tune(recflex_plan_t p, int32_t N, const int32_t *const *indices,
                                         const int32_t *const *offsets, const int32_t *batch_sizes,
                                         const void *const *tables, void *stream) {
    return recflex_tune_ex(p, N, indices, offsets, batch_sizes, tables, stream, nullptr, nullptr);
}
