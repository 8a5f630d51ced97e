// gather_probe.cu -- B200 ceiling for random row gathers (calibration for the
// roofline discussion in DESIGN.md; not part of the library).
//
// Each warp reads rows named by a random index array (uniform over a table of
// `rows` x `bytes_per_row`), U rows in flight per lane-group, sums them and
// writes one float per warp (so the loads cannot be elided).  Reports the
// achieved read bandwidth for several row sizes, unrolls and CTAs/SM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_probe gather_probe.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

// G lanes per row, 16 B per lane -> row = 16*G bytes
template <int G, int U>
__global__ void probe(const float4 *__restrict__ table, const int *__restrict__ idx, long long n_rows_total,
                      float *out) {
    const int lane = threadIdx.x & 31;
    const int lg = lane % G;
    const long long group = ((long long)blockIdx.x * blockDim.x + threadIdx.x) / G;
    const long long ngroups = ((long long)gridDim.x * blockDim.x) / G;
    float acc = 0.f;
    for (long long j = group * U; j < n_rows_total; j += ngroups * U) {
        float4 v[U];
        int id[U];
#pragma unroll
        for (int u = 0; u < U; ++u) id[u] = (j + u < n_rows_total) ? __ldg(idx + j + u) : 0;
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const float4 *p = table + (long long)id[u] * G + lg;
            asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                         : "=f"(v[u].x), "=f"(v[u].y), "=f"(v[u].z), "=f"(v[u].w) : "l"(p));
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc += v[u].x + v[u].y + v[u].z + v[u].w;
    }
    if (acc == 123.456f) out[0] = acc;
}

// Bag mode (512 B rows only): warp-per-bag over fixed-length bags of L lookups,
// warps claim bags from a global counter, pooled row stored per bag.
template <int U>
__global__ void probe_bags(const float4 *__restrict__ table, const int *__restrict__ idx, int nbags, int L,
                           float4 *out, int *counter) {
    const int lane = threadIdx.x & 31;
    while (true) {
        int b = 0;
        if (lane == 0) b = atomicAdd(counter, 1);
        b = __shfl_sync(0xffffffffu, b, 0);
        if (b >= nbags) break;
        float4 acc = make_float4(0, 0, 0, 0);
        const int lo = b * L, hi = lo + L;
        for (int j = lo; j < hi; j += U) {
            float4 v[U];
            int id[U];
#pragma unroll
            for (int u = 0; u < U; ++u) id[u] = __ldg(idx + j + u);
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const float4 *p = table + (long long)id[u] * 32 + lane;
                asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                             : "=f"(v[u].x), "=f"(v[u].y), "=f"(v[u].z), "=f"(v[u].w) : "l"(p));
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w;
            }
        }
        out[(long long)b * 32 + lane] = acc;
    }
}

template <int U>
void run_bags(const float4 *table, const int *idx, long long n, int L, float4 *out, int *counter, int ctas, int sms) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int nbags = (int)(n / L);
    float best = 1e9;
    for (int r = 0; r < 6; ++r) {
        cudaMemset(counter, 0, 4);
        cudaEventRecord(a);
        probe_bags<U><<<sms * ctas, 256>>>(table, idx, nbags, L, out, counter);
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r && ms < best) best = ms;
    }
    double bytes = (double)nbags * L * 516 + (double)nbags * 512;
    printf("bags L=%4d U=%d ctas/SM=%d : %8.3f ms  %7.0f GB/s (rows+idx+out)\n", L, U, ctas, best, bytes / best / 1e6);
}

template <int G, int U>
void run(const float4 *table, long long table_rows, const int *idx, long long n, float *out, int ctas_per_sm, int sms) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    int grid = sms * ctas_per_sm;
    probe<G, U><<<grid, 256>>>(table, idx, n, out);
    CK(cudaDeviceSynchronize());
    float best = 1e9;
    for (int r = 0; r < 5; ++r) {
        cudaEventRecord(a);
        probe<G, U><<<grid, 256>>>(table, idx, n, out);
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    double bytes = (double)n * 16 * G + (double)n * 4;
    printf("row %4d B  U=%d  ctas/SM=%d : %8.3f ms  %7.0f GB/s (rows+idx)\n", 16 * G, U, ctas_per_sm, best,
           bytes / best / 1e6);
}

__global__ void init_idx(int *idx, long long n, long long rows, unsigned long long seed) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned long long z = (i + seed) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        idx[i] = (int)(z % (unsigned long long)(rows < 2147483647ll ? rows : 2147483647ll));
    }
}

int main(int argc, char **argv) {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long long table_gib = argc > 1 ? atoll(argv[1]) : 40;
    const int only512 = argc > 2 ? atoi(argv[2]) : 0;
    const long long table_bytes = table_gib << 30;  // table (>> L2)
    printf("table %lld GiB\n", table_gib);
    float4 *table;
    CK(cudaMalloc(&table, table_bytes));
    CK(cudaMemset(table, 0, table_bytes));
    const long long total_row_bytes = 16ll << 30;  // 16 GiB gathered per launch
    float *out;
    CK(cudaMalloc(&out, 4));
    // row sizes 16..512 B
    auto go = [&](auto gtag, int ctas) {
        constexpr int G = decltype(gtag)::value;
        long long rows = table_bytes / (16 * G);
        long long n = total_row_bytes / (16 * G);
        int *idx;
        CK(cudaMalloc(&idx, n * 4));
        init_idx<<<4096, 256>>>(idx, n, rows, 12345);
        CK(cudaDeviceSynchronize());
        run<G, 2>(table, rows, idx, n, out, ctas, sms);
        run<G, 4>(table, rows, idx, n, out, ctas, sms);
        run<G, 8>(table, rows, idx, n, out, ctas, sms);
        cudaFree(idx);
    };
    if (only512 == 2) {  // bag mode
        long long rows = table_bytes / 512;
        long long n = total_row_bytes / 512;
        int *idx, *counter;
        float4 *outb;
        CK(cudaMalloc(&idx, n * 4));
        CK(cudaMalloc(&counter, 4));
        CK(cudaMalloc(&outb, (n / 1) * 16 * 32 / 50 + 4096));
        init_idx<<<4096, 256>>>(idx, n, rows, 12345);
        CK(cudaDeviceSynchronize());
        for (int ctas : {4, 6})
            for (int L : {100, 1000}) {
                run_bags<2>(table, idx, n, L, outb, counter, ctas, sms);
                run_bags<4>(table, idx, n, L, outb, counter, ctas, sms);
            }
        return 0;
    }
    for (int ctas : {4, 6, 8}) {
        go(std::integral_constant<int, 32>{}, ctas);
        if (only512) continue;
        go(std::integral_constant<int, 16>{}, ctas);
        go(std::integral_constant<int, 8>{}, ctas);
        go(std::integral_constant<int, 4>{}, ctas);
        go(std::integral_constant<int, 2>{}, ctas);
        go(std::integral_constant<int, 1>{}, ctas);
    }
    // sequential copy reference
    {
        long long n = (16ll << 30) / 4;
        float *a, *b;
        CK(cudaMalloc(&a, n * 4));
        CK(cudaMalloc(&b, n * 4));
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        CK(cudaMemcpy(b, a, n * 4, cudaMemcpyDeviceToDevice));
        float best = 1e9;
        for (int r = 0; r < 5; ++r) {
            cudaEventRecord(e0);
            cudaMemcpy(b, a, n * 4, cudaMemcpyDeviceToDevice);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (ms < best) best = ms;
        }
        printf("memcpy D2D 16 GiB: %.3f ms  %.0f GB/s (read+write)\n", best, 2.0 * n * 4 / best / 1e6);
    }
    return 0;
}
