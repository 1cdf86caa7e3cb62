// ubench_rowread.cu -- what limits GESUMMV's read stream (2 x 64 MiB) on B200?  Three read-only
// access patterns over the same two 4096 x 4096 fp32 matrices, each summed so nothing is dead:
//   rows   : one warp per row, ascending 512-byte column blocks, 4 blocks of 16-byte loads in
//            flight per lane (RowDotBody's pattern), 128-thread CTAs, one wave
//   rows4  : one warp per 4 consecutive rows, 8 lanes per row, coalesced 128 bytes per row per
//            load instruction (keeps RowDotBody's canonical partition fold reproducible)
//   chunks : contiguous 8 KB per CTA, many short CTAs (the pattern of torch's copy kernel)
// Event-timed after an L2 flush, median of 20.  build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)
constexpr int N = 4096;

__device__ __forceinline__ float4 ldnc(const float *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}

__global__ void __launch_bounds__(128, 7) rows(const float *A, const float *B, float *out) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    const float *pa = A + i * N + 4 * lane, *pb = B + i * N + 4 * lane;
    float s = 0.f;
    for (int k = 0; k < N / 128; k += 4) {
        float4 a[4], b[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) { a[u] = ldnc(pa + (k + u) * 128); b[u] = ldnc(pb + (k + u) * 128); }
#pragma unroll
        for (int u = 0; u < 4; ++u) s += a[u].x + a[u].y + a[u].z + a[u].w + b[u].x + b[u].y + b[u].z + b[u].w;
    }
    if (s == 123.f) out[i] = s;
}

__global__ void __launch_bounds__(128, 4) rows4(const float *A, const float *B, float *out) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 3, l = lane & 7;
    const long long i = (long long)blockIdx.x * 16 + warp * 4 + g;
    const float *pa = A + i * N + 4 * l, *pb = B + i * N + 4 * l;
    float s = 0.f;
    for (int k = 0; k < N / 128; ++k) {
        float4 a[4], b[4];
#pragma unroll
        for (int c = 0; c < 4; ++c) { a[c] = ldnc(pa + k * 128 + c * 32); b[c] = ldnc(pb + k * 128 + c * 32); }
#pragma unroll
        for (int c = 0; c < 4; ++c) s += a[c].x + a[c].y + a[c].z + a[c].w + b[c].x + b[c].y + b[c].z + b[c].w;
    }
    if (s == 123.f) out[i] = s;
}

__global__ void __launch_bounds__(128) chunks(const float *A, const float *B, float *out) {
    // block b < nb/2 reads A, the rest B: 2048 floats (8 KB) per block, 4 x 16 B per thread
    const long long nb = 2ll * N * N / 2048;
    const float *p = (blockIdx.x < nb / 2 ? A + blockIdx.x * 2048ll : B + (blockIdx.x - nb / 2) * 2048ll) + 4 * threadIdx.x;
    float4 v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) v[u] = ldnc(p + u * 512);
    float s = 0.f;
#pragma unroll
    for (int u = 0; u < 4; ++u) s += v[u].x + v[u].y + v[u].z + v[u].w;
    if (s == 123.f) out[blockIdx.x] = s;
}

int main() {
    float *A, *B, *out, *flush;
    CK(cudaMalloc(&A, 4ull * N * N)); CK(cudaMalloc(&B, 4ull * N * N)); CK(cudaMalloc(&out, 1 << 24));
    CK(cudaMalloc(&flush, 512ull << 20));
    CK(cudaMemset(A, 0, 4ull * N * N)); CK(cudaMemset(B, 0, 4ull * N * N));
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    auto run = [&](const char *name, auto launch) {
        std::vector<float> ts;
        for (int r = 0; r < 25; ++r) {
            cudaMemsetAsync(flush, r, 512ull << 20);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 5) ts.push_back(ms * 1e3f);
        }
        std::sort(ts.begin(), ts.end());
        const float us = ts[ts.size() / 2];
        printf("%-8s %8.2f us  %7.1f GB/s\n", name, us, 2.0 * 4 * N * N / (us * 1e-6) / 1e9);
    };
    for (int rep = 0; rep < 2; ++rep) {
        run("rows", [&] { rows<<<N / 4, 128>>>(A, B, out); });
        run("rows4", [&] { rows4<<<N / 16, 128>>>(A, B, out); });
        run("chunks", [&] { chunks<<<2 * N * N / 2048, 128>>>(A, B, out); });
    }
    return 0;
}
