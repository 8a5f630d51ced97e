// kjt_probe.cu -- the minimal warp-per-bag gather (pipe_probe mode 2) run on a
// REAL heavy batch (KJT dumped by tools/kjt_probe.py): separates "the data's
// access pattern" from "the library's task machinery" in the heavy gap
// (DESIGN.md §6).  Development probe, not part of the library.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o kjt_probe kjt_probe.cu
//   ./kjt_probe <indices.bin> <offsets.bin> F B rows_per_table ntables
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ float4 ldrow(const float4 *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}

// ORDER 0: bags claimed feature-major (f, s) like the library's task order;
// ORDER 1: sample-major (s, f).
template <int U, int ORDER>
__global__ void __launch_bounds__(256) kjt_bags(const float4 *__restrict__ table, long long rows_per_table, int ntables,
                                                const int *__restrict__ idx, const int *__restrict__ off, int F, int B,
                                                float4 *out, int *counter) {
    const int lane = threadIdx.x & 31;
    const int nb = F * B;
    while (true) {
        int b = 0;
        if (lane == 0) b = atomicAdd(counter, 1);
        b = __shfl_sync(0xffffffffu, b, 0);
        if (b >= nb) break;
        const int f = ORDER == 0 ? b / B : b % F;
        const int s = ORDER == 0 ? b % B : b / F;
        const int lo = __ldg(off + f * B + s), hi = __ldg(off + f * B + s + 1);
        const float4 *T = table + (long long)(f % ntables) * rows_per_table * 32;
        float4 acc = make_float4(0, 0, 0, 0);
        for (int c = lo; c < hi; c += 32) {
            const int n = min(32, hi - c);
            const int chunk = lane < n ? __ldg(idx + c + lane) : 0;
            int j = 0;
            for (; j + U <= n; j += U) {
                float4 v[U];
#pragma unroll
                for (int u = 0; u < U; ++u) v[u] = ldrow(T + (long long)__shfl_sync(0xffffffffu, chunk, j + u) * 32 + lane);
#pragma unroll
                for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
            }
            for (; j < n; ++j) {
                const float4 v = ldrow(T + (long long)__shfl_sync(0xffffffffu, chunk, j) * 32 + lane);
                acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
            }
        }
        out[((long long)s * F + f) * 32 + lane] = acc;
    }
}

template <int U, int ORDER>
void run(const float4 *table, long long rpt, int nt, const int *idx, const int *off, int F, int B, float4 *out,
         int *counter, long long nnz, int ctas, int sms) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e9;
    for (int r = 0; r < 6; ++r) {
        cudaMemset(counter, 0, 4);
        cudaEventRecord(a);
        kjt_bags<U, ORDER><<<sms * ctas, 256>>>(table, rpt, nt, idx, off, F, B, out, counter);
        cudaEventRecord(b);
        CK(cudaEventSynchronize(b));
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r && ms < best) best = ms;
    }
    const double bytes = (double)nnz * 516 + (double)F * B * 512;
    printf("kjt U=%d order=%d ctas/SM=%d : %7.3f ms %6.0f GB/s\n", U, ORDER, ctas, best, bytes / best / 1e6);
}

int main(int argc, char **argv) {
    if (argc < 7) { printf("usage: kjt_probe idx.bin off.bin F B rows_per_table ntables\n"); return 1; }
    const int F = atoi(argv[3]), B = atoi(argv[4]);
    const long long rpt = atoll(argv[5]);
    const int nt = atoi(argv[6]);
    std::vector<int> off((size_t)F * B + 1);
    FILE *fo = fopen(argv[2], "rb");
    if (fread(off.data(), 4, off.size(), fo) != off.size()) { printf("short offsets\n"); return 1; }
    fclose(fo);
    const long long nnz = off.back();
    std::vector<int> idx(nnz);
    FILE *fi = fopen(argv[1], "rb");
    if ((long long)fread(idx.data(), 4, nnz, fi) != nnz) { printf("short indices\n"); return 1; }
    fclose(fi);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float4 *table, *out;
    int *d_idx, *d_off, *counter;
    CK(cudaMalloc(&table, (size_t)nt * rpt * 512));
    CK(cudaMemset(table, 0, (size_t)nt * rpt * 512));
    CK(cudaMalloc(&d_idx, nnz * 4));
    CK(cudaMalloc(&d_off, off.size() * 4));
    CK(cudaMalloc(&out, (size_t)F * B * 512));
    CK(cudaMalloc(&counter, 4));
    CK(cudaMemcpy(d_idx, idx.data(), nnz * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(d_off, off.data(), off.size() * 4, cudaMemcpyHostToDevice));
    printf("F=%d B=%d nnz=%lld\n", F, B, nnz);
    for (int ctas : {3, 4, 6}) {
        run<2, 0>(table, rpt, nt, d_idx, d_off, F, B, out, counter, nnz, ctas, sms);
        run<4, 0>(table, rpt, nt, d_idx, d_off, F, B, out, counter, nnz, ctas, sms);
        run<2, 1>(table, rpt, nt, d_idx, d_off, F, B, out, counter, nnz, ctas, sms);
    }
    return 0;
}
