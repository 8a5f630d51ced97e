// tma_gather_probe.cu -- can the TMA engine gather random embedding rows faster than
// per-thread loads?  (B200 probe for DESIGN.md §11; not part of the library.)
//
// Random row gathers over a large table by `cp.async.bulk.tensor.2d ... tile::gather4`
// (4 rows named by 4 row coordinates per instruction) into a shared-memory ring,
// completion through mbarrier transaction counts; every thread then sums its part of the
// landed rows (so nothing is elided).  One elected thread per CTA issues a whole batch
// of stages, the CTA consumes them, repeat.  Reports rows/s and GB/s per row size; the
// per-thread-load ceiling of tools/gather_probe.cu is ~40 G rows/s for rows <= 128 B.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_gather_probe tma_gather_probe.cu \
//        -L/usr/local/cuda/lib64/stubs -lcuda
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x)                                                                                  \
    do {                                                                                       \
        cudaError_t e = (x);                                                                   \
        if (e != cudaSuccess) {                                                                \
            printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e));                   \
            exit(1);                                                                           \
        }                                                                                      \
    } while (0)

constexpr int kRowsPerStage = 32;    // 8 gather4 per stage
// stages in flight per CTA: up to 16, at most 96 KB of ring (two CTAs fit an SM)
template <int ROWB>
__host__ __device__ constexpr int stages_for() {
    return (98304 / (kRowsPerStage * ROWB)) < 16 ? (98304 / (kRowsPerStage * ROWB)) : 16;
}

__device__ __forceinline__ void mbar_init(unsigned mb, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(mb), "r"(count));
}
__device__ __forceinline__ void mbar_expect(unsigned mb, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(bytes) : "memory");
}
// watchdog: trap instead of hanging the GPU if a transfer never completes
__device__ __forceinline__ void mbar_wait(unsigned mb, unsigned parity) {
    const long long t0 = clock64();
    while (true) {
        unsigned ok = 0;
        asm volatile(
            "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(mb), "r"(parity)
            : "memory");
        if (ok) return;
        if (clock64() - t0 > 4000000000LL) asm volatile("trap;");
    }
}

template <int ROWB>
__global__ void __launch_bounds__(256) tma_gather(const __grid_constant__ CUtensorMap tmap, const int *__restrict__ idx,
                                                 long long n_total, float *out) {
    constexpr int kStages = stages_for<ROWB>();
    extern __shared__ __align__(128) unsigned char smem[];
    __shared__ __align__(8) uint64_t bar[kStages];
    constexpr int kStageBytes = kRowsPerStage * ROWB;
    const long long per_iter = (long long)kStages * kRowsPerStage;
    float acc = 0.f;
    if (threadIdx.x == 0)
        for (int s = 0; s < kStages; ++s) mbar_init((unsigned)__cvta_generic_to_shared(&bar[s]), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncthreads();
    unsigned parity = 0;
    for (long long base = (long long)blockIdx.x * per_iter; base < n_total; base += (long long)gridDim.x * per_iter) {
        // thread 0 arms every stage's barrier with its byte count; then one thread per
        // gather4 (4 rows) loads its 4 IDs (one 16-byte load) and issues the transfer
        if (threadIdx.x == 0)
            for (int s = 0; s < kStages; ++s) mbar_expect((unsigned)__cvta_generic_to_shared(&bar[s]), kStageBytes);
        __syncthreads();
        if (threadIdx.x < kStages * (kRowsPerStage / 4)) {
            const int s = threadIdx.x / (kRowsPerStage / 4), g = threadIdx.x % (kRowsPerStage / 4);
            const long long j = base + (long long)s * kRowsPerStage + g * 4;
            int4 r = make_int4(0, 0, 0, 0);
            if (j + 3 < n_total) r = __ldg(reinterpret_cast<const int4 *>(idx + j));
            const unsigned mb = (unsigned)__cvta_generic_to_shared(&bar[s]);
            const unsigned dst = (unsigned)__cvta_generic_to_shared(smem + (size_t)s * kStageBytes + (size_t)g * 4 * ROWB);
            asm volatile(
                "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
                "l"(&tmap), "r"(0), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w), "r"(mb)
                : "memory");
        }
        for (int s = 0; s < kStages; ++s) {
            mbar_wait((unsigned)__cvta_generic_to_shared(&bar[s]), parity);
            const float4 *st = reinterpret_cast<const float4 *>(smem + (size_t)s * kStageBytes);
            for (int e = threadIdx.x; e < kStageBytes / 16; e += blockDim.x) {
                const float4 v = st[e];
                acc += v.x + v.y + v.z + v.w;
            }
        }
        parity ^= 1u;
        __syncthreads();  // every thread is done with the ring before it is refilled
    }
    if (acc == 123.456f) out[0] = acc;
}


template <int ROWB>
void run(void *table, long long rows, const int *idx, long long n, float *out, int ctas_per_sm, int sms) {
    CUtensorMap tm;
    const cuuint64_t dims[2] = {(cuuint64_t)(ROWB / 4), (cuuint64_t)rows};
    const cuuint64_t strides[1] = {(cuuint64_t)ROWB};
    const cuuint32_t box[2] = {(cuuint32_t)(ROWB / 4), 1};
    const cuuint32_t estr[2] = {1, 1};
    CUresult r = cuTensorMapEncodeTiled(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, table, dims, strides, box, estr,
                                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                        CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        printf("row %4d B: cuTensorMapEncodeTiled failed (%d)\n", ROWB, (int)r);
        return;
    }
    constexpr int kStages = stages_for<ROWB>();
    const int smem = kStages * kRowsPerStage * ROWB;
    CK(cudaFuncSetAttribute(tma_gather<ROWB>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    int occ = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, tma_gather<ROWB>, 256, smem));
    if (occ < ctas_per_sm) ctas_per_sm = occ;
    const int grid = sms * ctas_per_sm;
    tma_gather<ROWB><<<grid, 256, smem>>>(tm, idx, n, out);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int rep = 0; rep < 5; ++rep) {
        cudaEventRecord(e0);
        tma_gather<ROWB><<<grid, 256, smem>>>(tm, idx, n, out);
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    printf("TMA gather4  row %4d B  ctas/SM=%d  rows in flight/SM=%d : %8.3f ms  %6.1f G rows/s  %7.0f GB/s\n", ROWB,
           ctas_per_sm, ctas_per_sm * kStages * kRowsPerStage, best, n / best / 1e6, n * (double)ROWB / best / 1e6);
}

__global__ void fill_idx(int *idx, long long n, long long rows, unsigned seed) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned long long x = (unsigned long long)i * 0x9E3779B97F4A7C15ull + seed;
        x ^= x >> 31;
        x *= 0xBF58476D1CE4E5B9ull;
        x ^= x >> 29;
        idx[i] = (int)(x % (unsigned long long)rows);
    }
}

int main() {
    cudaFree(nullptr);
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t table_bytes = size_t(8) << 30;  // 8 GB: far beyond L2
    void *table = nullptr;
    CK(cudaMalloc(&table, table_bytes));
    CK(cudaMemset(table, 0, table_bytes));
    const long long n = 64ll << 20;  // 64 M random rows per launch (a multiple of every stage batch)
    int *idx = nullptr;
    float *out = nullptr;
    CK(cudaMalloc(&idx, sizeof(int) * n));
    CK(cudaMalloc(&out, 16));
    for (int ctas : {1, 2}) {
#define ROW(RB)                                                                             \
    {                                                                                       \
        const long long rows = (long long)(table_bytes / RB);                               \
        fill_idx<<<sms * 8, 256>>>(idx, n, rows < (1ll << 31) ? rows : (1ll << 31) - 1, 7u); \
        CK(cudaDeviceSynchronize());                                                        \
        run<RB>(table, rows < (1ll << 31) ? rows : (1ll << 31) - 1, idx, n, out, ctas, sms); \
    }
        ROW(32)
        ROW(64)
        ROW(128)
        ROW(256)
        ROW(512)
    }
    return 0;
}
