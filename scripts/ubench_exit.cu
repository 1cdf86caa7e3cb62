// ubench_exit.cu -- cost of the GPU-exit signal of a lite (single-wave, plain-grid) cooperative
// launch, on the GESUMMV row-dot read pattern (N = 4096 fp32, 2 matrices, 1024 CTAs x 128).
// Epilogue variants:
//   0 none (the GPU-only grid)
//   1 hierarchical arrival (16 leaf counters + root, atomicAdd) -> last CTA st.relaxed.sys
//   2 flat arrival (one atomicAdd counter) -> last CTA st.relaxed.sys
//   3 per-CTA flag: every CTA st.relaxed.sys its epoch into a mapped host array (no atomics)
//   4 fire-and-forget red.add per CTA; CTA 0 waits for the count, then st.relaxed.sys
//   5 per-SM flag: the CTA st.relaxed.sys into flags[smid] (host checks 148 words)
//   6 variant 1 plus the block-0 counter reset at grid start (the current runtime)
// Prints: single-kernel time (L2 flushed, events), 3-kernel PDL chain time, and the host-side
// latency from the end-of-chain event to the host seeing the last exit word.
//
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o ubench_exit ubench_exit.cu -lcuda
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <algorithm>
#include <chrono>
#include <cstdint>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e_)); exit(1);} } while (0)

__device__ __forceinline__ float4 ld_stream4(const float *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float fold4(float p0, float p1, float p2, float p3) {
    float v = __fadd_rn(__fadd_rn(__fadd_rn(p0, p1), p2), p3);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }

struct P {
    const float *A, *B, *x; float *o0, *o1; int n; float alpha, beta;
    unsigned *ctr;                  // 17 device counters (+ one for variant 4)
    unsigned long long *exit_word;  // mapped host
    unsigned *flags;                // mapped host, per CTA / per SM
    unsigned epoch;
    int pdl_wait;
};

template <int V>
__global__ void __launch_bounds__(128, 8) rowdot(const __grid_constant__ P p) {
    if (p.pdl_wait) asm volatile("griddepcontrol.wait;" ::: "memory");
    if (V == 6 && blockIdx.x == 0) {
        if (threadIdx.x == 0) { for (int q = 0; q < 17; ++q) p.ctr[32 + q] = 0u; __threadfence(); }
        __syncthreads();
    }
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    if (i < p.n) {
        const float *pa = p.A + i * p.n + 4 * lane, *pb = p.B + i * p.n + 4 * lane, *px = p.x + 4 * lane;
        float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
        const int nfull = p.n / 128;
        constexpr int U = 4;
        for (int k = 0; k < nfull; k += U, pa += U * 128, pb += U * 128, px += U * 128) {
            float4 av[U], bv[U], xv[U];
#pragma unroll
            for (int u = 0; u < U; ++u) { av[u] = ld_stream4(pa + u * 128); bv[u] = ld_stream4(pb + u * 128); }
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
        const float va = fold4(a0, a1, a2, a3), vb = fold4(b0, b1, b2, b3);
        if (lane == 0) { p.o0[i] = va; p.o1[i] = __fadd_rn(__fmul_rn(p.alpha, va), __fmul_rn(p.beta, vb)); }
    }
    if (V == 0) return;
    __syncthreads();
    if (threadIdx.x != 0) return;
    const unsigned long long ep = p.epoch;
    if (V == 1 || V == 6) {
        const unsigned leaf = blockIdx.x & 15u, nleaf = gridDim.x > 16u ? 16u : gridDim.x;
        const unsigned leaf_size = (gridDim.x - leaf + 15u) / 16u;
        unsigned *c = p.ctr + (V == 6 ? 32 : 0);
        if (atomicAdd(c + 1 + leaf, 1u) == leaf_size - 1 && atomicAdd(c, 1u) == nleaf - 1)
            asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p.exit_word), "l"(ep) : "memory");
    } else if (V == 2) {
        if (atomicAdd(p.ctr + 20, 1u) == gridDim.x - 1)
            asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p.exit_word), "l"(ep) : "memory");
    } else if (V == 3) {
        asm volatile("st.relaxed.sys.global.b32 [%0], %1;" ::"l"(p.flags + blockIdx.x), "r"((unsigned)ep) : "memory");
    } else if (V == 4) {
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(p.ctr + 24) : "memory");
        if (blockIdx.x == 0) {
            unsigned v;
            do { asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p.ctr + 24) : "memory"); }
            while (v < gridDim.x);
            asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p.exit_word), "l"(ep) : "memory");
        }
    } else if (V == 5) {
        asm volatile("st.relaxed.sys.global.b32 [%0], %1;" ::"l"(p.flags + smid()), "r"((unsigned)ep) : "memory");
    }
}

__global__ void sweep_kernel(const float4 *p, size_t n, float *sink) {
    float acc = 0;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) { float4 v = __ldcs(p + i); acc += v.x; }
    if (acc == 12345.0f) *sink = acc;
}
static float *g_flush, *g_sink;
static void flush_l2() {
    CK(cudaMemsetAsync(g_flush, 1, 256u << 20));
    sweep_kernel<<<148 * 8, 256>>>((const float4 *)g_flush, (256u << 20) / 16, g_sink);
}
template <int V>
static void launch(const P &p, bool pdl) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((p.n + 3) / 4); cfg.blockDim = dim3(128); cfg.stream = 0;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at; cfg.numAttrs = pdl ? 1 : 0;
    P q = p; q.pdl_wait = 0;
    CK(cudaLaunchKernelEx(&cfg, rowdot<V>, q));
}

int main(int argc, char **argv) {
    const int n = 4096;
    const size_t nn = (size_t)n * n;
    float *A[3], *B[3], *x, *o0, *o1;
    for (int k = 0; k < 3; ++k) { CK(cudaMalloc(&A[k], nn * 4)); CK(cudaMalloc(&B[k], nn * 4)); CK(cudaMemset(A[k], 0, nn * 4)); CK(cudaMemset(B[k], 0, nn * 4)); }
    CK(cudaMalloc(&x, n * 4)); CK(cudaMalloc(&o0, n * 4)); CK(cudaMalloc(&o1, n * 4)); CK(cudaMemset(x, 0, n * 4));
    CK(cudaMalloc(&g_flush, 256u << 20)); CK(cudaMalloc(&g_sink, 64));
    unsigned *ctr; CK(cudaMalloc(&ctr, 4096)); CK(cudaMemset(ctr, 0, 4096));
    unsigned long long *exit_h, *exit_d; unsigned *flags_h, *flags_d;
    CK(cudaHostAlloc(&exit_h, 64, cudaHostAllocMapped)); CK(cudaHostGetDevicePointer(&exit_d, exit_h, 0));
    CK(cudaHostAlloc(&flags_h, 8192, cudaHostAllocMapped)); CK(cudaHostGetDevicePointer(&flags_d, flags_h, 0));
    memset(exit_h, 0, 64); memset(flags_h, 0, 8192);
    const double bytes = 2.0 * nn * 4 + 3.0 * n * 4;
    unsigned epoch = 0;
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    auto run = [&](int V, int nk, bool host_wait, double *t_host_after_event) -> float {
        std::vector<float> ts; std::vector<double> lat;
        for (int r = 0; r < 43; ++r) {
            flush_l2();
            CK(cudaMemsetAsync(ctr, 0, 4096));
            CK(cudaDeviceSynchronize());
            ++epoch;
            CK(cudaEventRecord(e0));
            for (int k = 0; k < nk; ++k) {
                P p{A[k], B[k], x, o0, o1, n, 1.5f, 1.2f, ctr + 64 * k, exit_d + k, flags_d + 2048 * k, epoch, 0};
                const bool pdl = k > 0;
                switch (V) {
                case 0: launch<0>(p, pdl); break; case 1: launch<1>(p, pdl); break; case 2: launch<2>(p, pdl); break;
                case 3: launch<3>(p, pdl); break; case 4: launch<4>(p, pdl); break; case 5: launch<5>(p, pdl); break;
                case 6: launch<6>(p, pdl); break;
                }
            }
            CK(cudaEventRecord(e1));
            if (host_wait && V != 0) {
                // host sees the last kernel's exit signal
                const int k = nk - 1;
                volatile unsigned long long *w = exit_h + k;
                volatile unsigned *f = flags_h + 2048 * k;
                const unsigned g = (n + 3) / 4;
                for (;;) {
                    bool done;
                    if (V == 3) { done = true; for (unsigned c = 0; c < g; ++c) if (f[c] < epoch) { done = false; break; } }
                    else if (V == 5) { done = true; for (unsigned c = 0; c < 148; ++c) if (f[c] < epoch) { done = false; break; } }
                    else done = *w >= epoch;
                    if (done) break;
                }
                auto th = std::chrono::steady_clock::now();
                CK(cudaEventSynchronize(e1));
                auto te = std::chrono::steady_clock::now();
                lat.push_back(std::chrono::duration<double, std::micro>(te - th).count());
            }
            CK(cudaEventSynchronize(e1));
            float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
            if (r >= 3) ts.push_back(ms);
        }
        CK(cudaGetLastError());
        std::sort(ts.begin(), ts.end());
        if (t_host_after_event) { std::sort(lat.begin(), lat.end()); *t_host_after_event = lat.empty() ? 0 : lat[lat.size() / 2]; }
        return ts[ts.size() / 2];
    };
    // V5 needs all flags of SMs that ran a CTA: with 1024 CTAs on 148 SMs every SM runs one
    for (int V = 0; V <= 6; ++V) {
        const float t1 = run(V, 1, false, nullptr);
        const float t3 = run(V, 3, false, nullptr);
        double lat = 0;
        const float t3h = run(V, 3, true, &lat);
        printf("V%d  1 kernel %7.2f us (%6.1f GB/s)   3-kernel PDL chain %7.2f us   chain with host poll %7.2f us, event done %6.2f us after host saw exit\n",
               V, t1 * 1e3, bytes / (t1 * 1e-3) / 1e9, t3 * 1e3, t3h * 1e3, lat);
    }
    return 0;
}
