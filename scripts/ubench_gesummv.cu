// ubench_gesummv.cu -- read pipelines for GESUMMV's two 4096 x 4096 fp32 row streams (134 MB),
// all with RowDotBody's canonical arithmetic (lane l: partials 4l..4l+3 over ascending 128-column
// blocks, fold ((p0+p1)+p2)+p3, xor butterfly 16..1), so every variant's y is bit-identical.
//   rows_u4  : RowDotBody as shipped (one warp per row, 4 blocks of 16-B loads in flight, 7 CTA/SM)
//   rows_u8  : 8 blocks in flight per lane
//   bulk<S>  : per-warp TMA bulk-copy ring (cp.async.bulk + mbarrier), S stages of 2 x 2 KB
//   read     : grid-stride pure read, 8 x 16 B per thread in flight (the read ceiling, no dot)
// L2 flushed like bench.py (256 MiB write + 256 MiB read sweep), event-timed, median of 30.
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/ug scripts/ubench_gesummv.cu
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <vector>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s: %s\n", #x, cudaGetErrorString(e_)); return 1; } } while (0)
constexpr int N = 4096;

__device__ __forceinline__ float4 ldnc(const float *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float fold(float p0, float p1, float p2, float p3) {
    float v = __fadd_rn(__fadd_rn(__fadd_rn(p0, p1), p2), p3);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

template <int U, int MINB>
__global__ void __launch_bounds__(128, MINB) rows(const float *A, const float *B, const float *x, float *tmp, float *y, float alpha, float beta) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    const float *pa = A + i * N + 4 * lane, *pb = B + i * N + 4 * lane, *px = x + 4 * lane;
    float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
    for (int k = 0; k < N / 128; k += U, pa += U * 128, pb += U * 128, px += U * 128) {
        float4 av[U], bv[U], xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { av[u] = ldnc(pa + u * 128); bv[u] = ldnc(pb + u * 128); }
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = __ldg(reinterpret_cast<const float4 *>(px + u * 128));
#pragma unroll
        for (int u = 0; u < U; ++u) {
            a0 = __fmaf_rn(av[u].x, xv[u].x, a0); a1 = __fmaf_rn(av[u].y, xv[u].y, a1);
            a2 = __fmaf_rn(av[u].z, xv[u].z, a2); a3 = __fmaf_rn(av[u].w, xv[u].w, a3);
            b0 = __fmaf_rn(bv[u].x, xv[u].x, b0); b1 = __fmaf_rn(bv[u].y, xv[u].y, b1);
            b2 = __fmaf_rn(bv[u].z, xv[u].z, b2); b3 = __fmaf_rn(bv[u].w, xv[u].w, b3);
        }
    }
    const float va = fold(a0, a1, a2, a3), vb = fold(b0, b1, b2, b3);
    if (lane == 0) { tmp[i] = va; y[i] = __fadd_rn(__fmul_rn(alpha, va), __fmul_rn(beta, vb)); }
}

// rows_u4 with the row length a runtime argument (as in the library body)
template <int U, int MINB>
__global__ void __launch_bounds__(128, MINB) rows_rt(const float *A, const float *B, const float *x, float *tmp, float *y, float alpha, float beta, long long ncols) {
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    const float *pa = A + i * ncols + 4 * lane, *pb = B + i * ncols + 4 * lane, *px = x + 4 * lane;
    float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
    const long long nfull = ncols / 128;
    for (long long k = 0; k + U <= nfull; k += U, pa += U * 128, pb += U * 128, px += U * 128) {
        float4 av[U], bv[U], xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { av[u] = ldnc(pa + u * 128); bv[u] = ldnc(pb + u * 128); }
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = __ldg(reinterpret_cast<const float4 *>(px + u * 128));
#pragma unroll
        for (int u = 0; u < U; ++u) {
            a0 = __fmaf_rn(av[u].x, xv[u].x, a0); a1 = __fmaf_rn(av[u].y, xv[u].y, a1);
            a2 = __fmaf_rn(av[u].z, xv[u].z, a2); a3 = __fmaf_rn(av[u].w, xv[u].w, a3);
            b0 = __fmaf_rn(bv[u].x, xv[u].x, b0); b1 = __fmaf_rn(bv[u].y, xv[u].y, b1);
            b2 = __fmaf_rn(bv[u].z, xv[u].z, b2); b3 = __fmaf_rn(bv[u].w, xv[u].w, b3);
        }
    }
    const float va = fold(a0, a1, a2, a3), vb = fold(b0, b1, b2, b3);
    if (lane == 0) { tmp[i] = va; y[i] = __fadd_rn(__fmul_rn(alpha, va), __fmul_rn(beta, vb)); }
}

__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long *b, unsigned cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect(unsigned long long *b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, unsigned long long *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *b, unsigned parity) {
    asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W;\n}"
                 ::"r"(smem_u32(b)), "r"(parity) : "memory");
}

// per-warp ring: stage = SB floats of A + SB floats of B (SB = 128 * BLK)
template <int S, int BLK, int MINB>
__global__ void __launch_bounds__(128, MINB) bulk(const float *A, const float *B, const float *x, float *tmp, float *y, float alpha, float beta) {
    constexpr int SB = 128 * BLK;
    constexpr int NST = N / SB;   // stages per row
    extern __shared__ __align__(128) float sm[];
    __shared__ __align__(8) unsigned long long bar[4][S];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    float *ring = sm + warp * S * 2 * SB;
    const long long i = (long long)blockIdx.x * 4 + warp;
    const float *Ar = A + i * N, *Br = B + i * N;
    if (lane == 0) {
        for (int s = 0; s < S; ++s) mbar_init(&bar[warp][s], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        for (int s = 0; s < S && s < NST; ++s) {
            mbar_expect(&bar[warp][s], 2 * SB * 4);
            bulk_g2s(ring + s * 2 * SB, Ar + s * SB, SB * 4, &bar[warp][s]);
            bulk_g2s(ring + s * 2 * SB + SB, Br + s * SB, SB * 4, &bar[warp][s]);
        }
    }
    __syncwarp();
    float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
    const float *px = x + 4 * lane;
    for (int st = 0; st < NST; ++st) {
        const int s = st % S;
        float4 xv[BLK];
#pragma unroll
        for (int u = 0; u < BLK; ++u) xv[u] = __ldg(reinterpret_cast<const float4 *>(px + st * SB + u * 128));
        mbar_wait(&bar[warp][s], (st / S) & 1);
        const float *ra = ring + s * 2 * SB + 4 * lane, *rb = ra + SB;
#pragma unroll
        for (int u = 0; u < BLK; ++u) {
            const float4 av = *reinterpret_cast<const float4 *>(ra + u * 128);
            const float4 bv = *reinterpret_cast<const float4 *>(rb + u * 128);
            a0 = __fmaf_rn(av.x, xv[u].x, a0); a1 = __fmaf_rn(av.y, xv[u].y, a1);
            a2 = __fmaf_rn(av.z, xv[u].z, a2); a3 = __fmaf_rn(av.w, xv[u].w, a3);
            b0 = __fmaf_rn(bv.x, xv[u].x, b0); b1 = __fmaf_rn(bv.y, xv[u].y, b1);
            b2 = __fmaf_rn(bv.z, xv[u].z, b2); b3 = __fmaf_rn(bv.w, xv[u].w, b3);
        }
        __syncwarp();
        if (lane == 0 && st + S < NST) {
            mbar_expect(&bar[warp][s], 2 * SB * 4);
            bulk_g2s(ring + s * 2 * SB, Ar + (st + S) * SB, SB * 4, &bar[warp][s]);
            bulk_g2s(ring + s * 2 * SB + SB, Br + (st + S) * SB, SB * 4, &bar[warp][s]);
        }
    }
    const float va = fold(a0, a1, a2, a3), vb = fold(b0, b1, b2, b3);
    if (lane == 0) { tmp[i] = va; y[i] = __fadd_rn(__fmul_rn(alpha, va), __fmul_rn(beta, vb)); }
}

__global__ void __launch_bounds__(256) readall(const float *A, const float *B, float *out, long long n4) {
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x, nth = (long long)gridDim.x * blockDim.x;
    float s = 0.f;
    for (long long v = tid; v < 2 * n4; v += 8 * nth) {
        float4 r[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const long long w = v + u * nth;
            r[u] = w < 2 * n4 ? ldnc((w < n4 ? A : B - 4 * n4) + 4 * w) : make_float4(0, 0, 0, 0);
        }
#pragma unroll
        for (int u = 0; u < 8; ++u) s += r[u].x + r[u].y + r[u].z + r[u].w;
    }
    if (s == 123.f) out[tid & 1023] = s;
}

int main() {
    float *A, *B, *x, *tmp, *y, *tmp0, *y0, *flush, *out;
    const size_t mb = 4ull * N * N;
    CK(cudaMalloc(&A, mb)); CK(cudaMalloc(&B, mb)); CK(cudaMalloc(&x, 4 * N));
    CK(cudaMalloc(&tmp, 4 * N)); CK(cudaMalloc(&y, 4 * N)); CK(cudaMalloc(&tmp0, 4 * N)); CK(cudaMalloc(&y0, 4 * N));
    CK(cudaMalloc(&out, 1 << 16)); CK(cudaMalloc(&flush, 256ull << 20));
    {
        std::vector<float> h(size_t(N) * N);
        unsigned s = 12345;
        for (auto &v : h) { s = s * 1664525u + 1013904223u; v = (float)((s >> 8) & 0xFFFF) / 65536.f - 0.5f; }
        CK(cudaMemcpy(A, h.data(), mb, cudaMemcpyHostToDevice));
        for (auto &v : h) { s = s * 1664525u + 1013904223u; v = (float)((s >> 8) & 0xFFFF) / 65536.f - 0.5f; }
        CK(cudaMemcpy(B, h.data(), mb, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(x, h.data(), 4 * N, cudaMemcpyHostToDevice));
    }
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    const float alpha = 1.5f, beta = 1.2f;
    auto run = [&](const char *name, auto launch, bool check) {
        std::vector<float> ts;
        for (int r = 0; r < 35; ++r) {
            cudaMemsetAsync(flush, r, 256ull << 20);
            readall<<<148 * 8, 256>>>(flush, flush, out, (256ll << 20) / 32);
            cudaEventRecord(e0);
            launch();
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 5) ts.push_back(ms * 1e3f);
        }
        cudaError_t e = cudaGetLastError();
        std::sort(ts.begin(), ts.end());
        const float us = ts[ts.size() / 2];
        int same = -1;
        if (check) {
            std::vector<float> a(2 * N), b(2 * N);
            cudaMemcpy(a.data(), tmp, 4 * N, cudaMemcpyDeviceToHost); cudaMemcpy(a.data() + N, y, 4 * N, cudaMemcpyDeviceToHost);
            cudaMemcpy(b.data(), tmp0, 4 * N, cudaMemcpyDeviceToHost); cudaMemcpy(b.data() + N, y0, 4 * N, cudaMemcpyDeviceToHost);
            same = memcmp(a.data(), b.data(), 8 * N) == 0;
        }
        printf("%-16s %8.2f us (min %7.2f)  %7.1f GB/s  bits=%d %s\n", name, us, ts[0], 2.0 * mb / (us * 1e-6) / 1e9, same,
               e == cudaSuccess ? "" : cudaGetErrorString(e));
    };
    rows<4, 7><<<N / 4, 128>>>(A, B, x, tmp0, y0, alpha, beta);
    CK(cudaDeviceSynchronize());
    auto bset = [&](auto kern, int smem) { cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem); };
    bset(bulk<2, 4, 6>, 4 * 2 * 2 * 512 * 4);
    bset(bulk<3, 4, 4>, 4 * 3 * 2 * 512 * 4);
    bset(bulk<4, 2, 6>, 4 * 4 * 2 * 256 * 4);
    bset(bulk<6, 2, 4>, 4 * 6 * 2 * 256 * 4);
    bset(bulk<4, 4, 3>, 4 * 4 * 2 * 512 * 4);
    bset(bulk<8, 1, 6>, 4 * 8 * 2 * 128 * 4);
    for (int rep = 0; rep < 2; ++rep) {
        run("rows_u4", [&] { rows<4, 7><<<N / 4, 128>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("rows_u8", [&] { rows<8, 4><<<N / 4, 128>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("rows_rt_u4", [&] { rows_rt<4, 7><<<N / 4, 128>>>(A, B, x, tmp, y, alpha, beta, (long long)N); }, true);
        run("rows_rt_u8m6", [&] { rows_rt<8, 6><<<N / 4, 128>>>(A, B, x, tmp, y, alpha, beta, (long long)N); }, true);
        run("bulk_s2_b4", [&] { bulk<2, 4, 6><<<N / 4, 128, 4 * 2 * 2 * 512 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("bulk_s3_b4", [&] { bulk<3, 4, 4><<<N / 4, 128, 4 * 3 * 2 * 512 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("bulk_s4_b2", [&] { bulk<4, 2, 6><<<N / 4, 128, 4 * 4 * 2 * 256 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("bulk_s6_b2", [&] { bulk<6, 2, 4><<<N / 4, 128, 4 * 6 * 2 * 256 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("bulk_s4_b4", [&] { bulk<4, 4, 3><<<N / 4, 128, 4 * 4 * 2 * 512 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("bulk_s8_b1", [&] { bulk<8, 1, 6><<<N / 4, 128, 4 * 8 * 2 * 128 * 4>>>(A, B, x, tmp, y, alpha, beta); }, true);
        run("read_1184x256", [&] { readall<<<148 * 8, 256>>>(A, B, out, (long long)N * N / 4); }, false);
        run("read_2368x256", [&] { readall<<<148 * 16, 256>>>(A, B, out, (long long)N * N / 4); }, false);
        run("empty", [&] { readall<<<1, 32>>>(A, B, out, 0); }, false);
    }
    return 0;
}
