// ubench_ffma2.cu -- can packed FFMA2 (fma.rn.f32x2, sm_100a) lift an issue-bound 8x8 register
// outer product (the GemmBody inner loop: per k, 8 A and 8 B values from shared memory, 64 fmas)?
//   ffma  : 64 scalar fmaf per k
//   ffma2 : 32 fma.rn.f32x2 per k, A broadcast as a pair {a, a}
// Both compute the same IEEE fp32 fmas in the same per-output order (bit-identical outputs).
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/uf scripts/ubench_ffma2.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstring>
#include <vector>

constexpr int KT = 16, BM = 128;

__device__ __forceinline__ float2 f2fma(float2 a, float2 b, float2 c) {
    unsigned long long r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r)
        : "l"(*reinterpret_cast<unsigned long long *>(&a)), "l"(*reinterpret_cast<unsigned long long *>(&b)),
          "l"(*reinterpret_cast<unsigned long long *>(&c)));
    return *reinterpret_cast<float2 *>(&r);
}

template <int MODE, int MINB>
__global__ void __launch_bounds__(256, MINB) op(const float *g, float *out, int iters) {
    __shared__ __align__(16) float sA[KT][BM + 4], sB[KT][BM + 4];
    for (int q = threadIdx.x; q < KT * BM; q += 256) {
        sA[q / BM][q % BM] = g[q];
        sB[q / BM][q % BM] = g[q + KT * BM];
    }
    __syncthreads();
    const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
    float acc[8][8];
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll 2
        for (int k = 0; k < KT; ++k) {
            const float4 a0 = *reinterpret_cast<const float4 *>(&sA[k][ty * 4]);
            const float4 a1 = *reinterpret_cast<const float4 *>(&sA[k][64 + ty * 4]);
            const float4 b0 = *reinterpret_cast<const float4 *>(&sB[k][tx * 4]);
            const float4 b1 = *reinterpret_cast<const float4 *>(&sB[k][64 + tx * 4]);
            const float a[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
            const float b[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
            if (MODE == 0) {
#pragma unroll
                for (int i = 0; i < 8; ++i)
#pragma unroll
                    for (int j = 0; j < 8; ++j) acc[i][j] = __fmaf_rn(a[i], b[j], acc[i][j]);
            } else {
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    const float2 ai = make_float2(a[i], a[i]);
#pragma unroll
                    for (int j = 0; j < 8; j += 2) {
                        float2 c = make_float2(acc[i][j], acc[i][j + 1]);
                        c = f2fma(ai, make_float2(b[j], b[j + 1]), c);
                        acc[i][j] = c.x; acc[i][j + 1] = c.y;
                    }
                }
            }
        }
    }
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) s += acc[i][j];
    out[blockIdx.x * 256 + threadIdx.x] = s;
}

template <int MB>
void run(float *g, float *out, cudaEvent_t e0, cudaEvent_t e1, int iters) {
    printf("min blocks %d\n", MB);
    for (int grid : {296, 592}) {
        std::vector<float> r0, r1;
        for (int mode = 0; mode < 2; ++mode) {
            for (int rep = 0; rep < 3; ++rep) {
                cudaEventRecord(e0);
                if (mode == 0) op<0, MB><<<grid, 256>>>(g, out, iters); else op<1, MB><<<grid, 256>>>(g, out, iters);
                cudaEventRecord(e1); cudaEventSynchronize(e1);
                float ms; cudaEventElapsedTime(&ms, e0, e1);
                const double fl = 2.0 * 64 * KT * (double)iters * 256 * grid;
                if (rep == 2) printf("grid %d %-6s %8.3f ms  %6.1f TFLOP/s  %s\n", grid, mode ? "ffma2" : "ffma", ms, fl / ms / 1e9,
                                     cudaGetErrorString(cudaGetLastError()));
            }
            std::vector<float> o(grid * 256);
            cudaMemcpy(o.data(), out, o.size() * 4, cudaMemcpyDeviceToHost);
            (mode ? r1 : r0) = o;
        }
        printf("bits equal: %d\n", memcmp(r0.data(), r1.data(), r0.size() * 4) == 0);
    }
}

int main() {
    float *g, *out;
    cudaMalloc(&g, 2 * KT * BM * 4); cudaMalloc(&out, 148 * 2 * 256 * 4 * 4);
    std::vector<float> h(2 * KT * BM);
    for (size_t i = 0; i < h.size(); ++i) h[i] = 1.0f + 1e-3f * (float)(i % 97);
    cudaMemcpy(g, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int iters = 2000;
    run<1>(g, out, e0, e1, iters);
    run<2>(g, out, e0, e1, iters);
    return 0;
}
