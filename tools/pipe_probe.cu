// pipe_probe.cu -- does issuing iteration i+1's row loads before iteration i's
// adds help a warp-per-bag gather on B200, and does it matter how the lookup
// IDs reach the lanes (broadcast L1 loads vs shuffles from a coalesced chunk)?
// Development probe for DESIGN.md §6 (not part of the library).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pipe_probe pipe_probe.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ float4 ldrow(const float4 *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ void add(float4 &a, const float4 &b) { a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w; }

// MODE 0: ids by broadcast __ldg, no pipelining (probe_bags)
// MODE 1: ids by broadcast __ldg, rows of the next iteration issued before the adds
// MODE 2: ids by shuffle from a 32-ID register chunk, no pipelining (library style)
// MODE 3: ids by shuffle, pipelined
template <int MODE, int U>
__global__ void __launch_bounds__(256) bags(const float4 *__restrict__ table, const int *__restrict__ idx, int nbags,
                                            int L, float4 *out, int *counter, int scatter_out) {
    const int lane = threadIdx.x & 31;
    while (true) {
        int b = 0;
        if (lane == 0) b = atomicAdd(counter, 1);
        b = __shfl_sync(0xffffffffu, b, 0);
        if (b >= nbags) break;
        float4 acc = make_float4(0, 0, 0, 0);
        const int lo = b * L, hi = lo + L;  // L % (2U) == 0, L % 32 == 0 for the shuffle modes
        if (MODE == 0) {
            for (int j = lo; j < hi; j += U) {
                float4 v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) v[u] = ldrow(table + (long long)__ldg(idx + j + u) * 32 + lane);
#pragma unroll
                for (int u = 0; u < U; ++u) add(acc, v[u]);
            }
        } else if (MODE == 1) {
            float4 va[U], vb[U];
#pragma unroll
            for (int u = 0; u < U; ++u) va[u] = ldrow(table + (long long)__ldg(idx + lo + u) * 32 + lane);
            for (int j = lo; j < hi; j += 2 * U) {
#pragma unroll
                for (int u = 0; u < U; ++u) vb[u] = ldrow(table + (long long)__ldg(idx + j + U + u) * 32 + lane);
#pragma unroll
                for (int u = 0; u < U; ++u) add(acc, va[u]);
                if (j + 2 * U < hi) {
#pragma unroll
                    for (int u = 0; u < U; ++u) va[u] = ldrow(table + (long long)__ldg(idx + j + 2 * U + u) * 32 + lane);
                }
#pragma unroll
                for (int u = 0; u < U; ++u) add(acc, vb[u]);
            }
        } else if (MODE == 2) {
            for (int c = lo; c < hi; c += 32) {
                const int chunk = __ldg(idx + c + lane);
                for (int j = 0; j < 32; j += U) {
                    float4 v[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) v[u] = ldrow(table + (long long)__shfl_sync(0xffffffffu, chunk, j + u) * 32 + lane);
#pragma unroll
                    for (int u = 0; u < U; ++u) add(acc, v[u]);
                }
            }
        } else {
            for (int c = lo; c < hi; c += 32) {
                const int chunk = __ldg(idx + c + lane);
                float4 va[U], vb[U];
#pragma unroll
                for (int u = 0; u < U; ++u) va[u] = ldrow(table + (long long)__shfl_sync(0xffffffffu, chunk, u) * 32 + lane);
                for (int j = 0; j < 32; j += 2 * U) {
#pragma unroll
                    for (int u = 0; u < U; ++u) vb[u] = ldrow(table + (long long)__shfl_sync(0xffffffffu, chunk, j + U + u) * 32 + lane);
#pragma unroll
                    for (int u = 0; u < U; ++u) add(acc, va[u]);
                    if (j + 2 * U < 32) {
#pragma unroll
                        for (int u = 0; u < U; ++u) va[u] = ldrow(table + (long long)__shfl_sync(0xffffffffu, chunk, j + 2 * U + u) * 32 + lane);
                    }
#pragma unroll
                    for (int u = 0; u < U; ++u) add(acc, vb[u]);
                }
            }
        }
        if (scatter_out) out[((long long)(b % 8192) * 3200 + (b / 8192) * 32) % (1ll << 24) + lane] = acc;
        else out[(long long)b * 32 + lane] = acc;
    }
}

__global__ void fill_random(float *t, long long n) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned z = (unsigned)(i * 2654435761ull) ^ (unsigned)(i >> 29);
        z ^= z >> 15; z *= 0x2c1b3c6dU; z ^= z >> 12;
        t[i] = (float)(z & 0xffff) * (1.0f / 65536.0f) - 0.5f;
    }
}

__global__ void init_idx(int *idx, long long n, long long rows, unsigned long long seed) {
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
        unsigned long long z = (i + seed) * 0x9E3779B97F4A7C15ull;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        z ^= z >> 31;
        idx[i] = (int)(z % (unsigned long long)rows);
    }
}

template <int MODE, int U>
void run(const float4 *table, const int *idx, long long n, int L, float4 *out, int *counter, int ctas, int sms, int scatter = 0) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const int nbags = (int)(n / L);
    float best = 1e9;
    for (int r = 0; r < 6; ++r) {
        cudaMemset(counter, 0, 4);
        cudaEventRecord(a);
        bags<MODE, U><<<sms * ctas, 256>>>(table, idx, nbags, L, out, counter, scatter);
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r && ms < best) best = ms;
    }
    const double bytes = (double)nbags * L * 516 + (double)nbags * 512;
    printf("mode %d U=%d L=%d ctas/SM=%d scatter=%d : %7.3f ms %6.0f GB/s\n", MODE, U, L, ctas, scatter, best, bytes / best / 1e6);
}

int main() {
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const long long table_bytes = 40ll << 30;
    float4 *table;
    CK(cudaMalloc(&table, table_bytes));
    CK(cudaMemset(table, 0, table_bytes));
    const long long rows = table_bytes / 512, n = (16ll << 30) / 512;
    int *idx, *counter;
    float4 *out;
    CK(cudaMalloc(&idx, n * 4));
    CK(cudaMalloc(&counter, 4));
    CK(cudaMalloc(&out, (n / 32 + 1) * 512));
    init_idx<<<4096, 256>>>(idx, n, rows, 12345);
    CK(cudaDeviceSynchronize());
    const int L = 96;
    CK(cudaMalloc(&out, (1ll << 24) * 16 + 4096));
    for (int ctas : {4}) {
        run<2, 2>(table, idx, n, L, out, counter, ctas, sms, 0);
        run<2, 2>(table, idx, n, L, out, counter, ctas, sms, 1);
    }
    fill_random<<<4096, 256>>>((float *)table, table_bytes / 4);
    CK(cudaDeviceSynchronize());
    printf("random table contents:\n");
    for (int ctas : {4, 6}) {
        run<2, 2>(table, idx, n, L, out, counter, ctas, sms, 0);
        run<2, 2>(table, idx, n, L, out, counter, ctas, sms, 1);
        run<0, 2>(table, idx, n, L, out, counter, ctas, sms, 0);
    }
    return 0;
}
