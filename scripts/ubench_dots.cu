// ubench_dots.cu -- standalone microbenchmark of row-dot / col-dot body variants (N = 4096 fp32),
// the HBM-bound kernels of the bench step (GESUMMV, BICG q = A p, BICG s = A^T r).
// Every variant must reproduce the canonical operation order bit-exactly (checked against
// variant 0, the body in csrc/kernels.cu at the time of writing); it prints median kernel time
// (CUDA events, L2 flushed before every rep) and algorithmic GB/s.
//
// build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -o ubench_dots ubench_dots.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <algorithm>
#include <cstdint>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e_)); exit(1);} } while (0)

__device__ __forceinline__ float4 ld_stream4(const float *p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float4 ld_cached4(const float *p) { return __ldg(reinterpret_cast<const float4 *>(p)); }
__device__ __forceinline__ void prefetch_l2_bulk(const void *p, unsigned bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
__device__ __forceinline__ float fold4(float p0, float p1, float p2, float p3) {
    float v = __fadd_rn(__fadd_rn(__fadd_rn(p0, p1), p2), p3);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

struct RP { const float *A, *B, *x; float *o0, *o1; int n; float alpha, beta; };

// ---- row-dot: one warp per row, 4 rows per 128-thread CTA; PF: 0 none, 1 whole-row L2 bulk
// prefetch at start, 2 windowed bulk prefetch (PD blocks ahead)
template <int NMAT, int U, int PF, int MINB>
__global__ void __launch_bounds__(128, MINB) rowdot(const __grid_constant__ RP p) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    if (i >= p.n) return;
    const float *Ar = p.A + i * p.n, *Br = NMAT == 2 ? p.B + i * p.n : nullptr;
    const int nfull = p.n / 128;
    constexpr int PD = 8;   // window, in 128-column blocks (2 KB per matrix)
    if (PF == 1 && lane == 0) {
        prefetch_l2_bulk(Ar, p.n * 4);
        if (NMAT == 2) prefetch_l2_bulk(Br, p.n * 4);
    }
    if (PF == 2 && lane == 0) {
        prefetch_l2_bulk(Ar, PD * 512);
        if (NMAT == 2) prefetch_l2_bulk(Br, PD * 512);
    }
    float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
    const float *pa = Ar + 4 * lane, *pb = NMAT == 2 ? Br + 4 * lane : nullptr, *px = p.x + 4 * lane;
    for (int k = 0; k < nfull; k += U, pa += U * 128, px += U * 128) {
        if (PF == 2 && lane == 0 && (k % PD) == 0 && k + PD < nfull) {
            prefetch_l2_bulk(Ar + (k + PD) * 128, PD * 512);
            if (NMAT == 2) prefetch_l2_bulk(Br + (k + PD) * 128, PD * 512);
        }
        float4 av[U], bv[U], xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            av[u] = ld_stream4(pa + u * 128);
            if (NMAT == 2) bv[u] = ld_stream4(pb + u * 128);
        }
        if (NMAT == 2) pb += U * 128;
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = ld_cached4(px + u * 128);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            a0 = __fmaf_rn(av[u].x, xv[u].x, a0); a1 = __fmaf_rn(av[u].y, xv[u].y, a1);
            a2 = __fmaf_rn(av[u].z, xv[u].z, a2); a3 = __fmaf_rn(av[u].w, xv[u].w, a3);
            if (NMAT == 2) {
                b0 = __fmaf_rn(bv[u].x, xv[u].x, b0); b1 = __fmaf_rn(bv[u].y, xv[u].y, b1);
                b2 = __fmaf_rn(bv[u].z, xv[u].z, b2); b3 = __fmaf_rn(bv[u].w, xv[u].w, b3);
            }
        }
    }
    const float va = fold4(a0, a1, a2, a3);
    if (NMAT == 1) { if (lane == 0) p.o0[i] = va; }
    else {
        const float vb = fold4(b0, b1, b2, b3);
        if (lane == 0) { p.o0[i] = va; p.o1[i] = __fadd_rn(__fmul_rn(p.alpha, va), __fmul_rn(p.beta, vb)); }
    }
}

// ---- row-dot with register double buffering: the next U blocks' loads are issued before the
// current ones are consumed (continuous loads per warp); RW rows per warp interleaved (RW
// independent streams per warp).  Same canonical order as rowdot.
template <int NMAT, int U, int RW, int MINB>
__global__ void __launch_bounds__(128, MINB) rowdot_db(const __grid_constant__ RP p) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i0 = ((long long)blockIdx.x * 4 + warp) * RW;
    if (i0 >= p.n) return;
    const int nfull = p.n / 128;
    float acc[RW][2][4];
#pragma unroll
    for (int r = 0; r < RW; ++r)
#pragma unroll
        for (int m = 0; m < 2; ++m)
#pragma unroll
            for (int q = 0; q < 4; ++q) acc[r][m][q] = 0.f;
    const float *pa[RW], *pb[RW];
#pragma unroll
    for (int r = 0; r < RW; ++r) { pa[r] = p.A + (i0 + r) * p.n + 4 * lane; pb[r] = p.B + (i0 + r) * p.n + 4 * lane; }
    const float *px = p.x + 4 * lane;
    float4 cur[RW][2][U], nxt[RW][2][U];
#pragma unroll
    for (int r = 0; r < RW; ++r)
#pragma unroll
        for (int u = 0; u < U; ++u) { cur[r][0][u] = ld_stream4(pa[r] + u * 128); if (NMAT == 2) cur[r][1][u] = ld_stream4(pb[r] + u * 128); }
    for (int k = 0; k < nfull; k += U) {
        const bool more = k + U < nfull;
        if (more) {
#pragma unroll
            for (int r = 0; r < RW; ++r)
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    nxt[r][0][u] = ld_stream4(pa[r] + (k + U + u) * 128);
                    if (NMAT == 2) nxt[r][1][u] = ld_stream4(pb[r] + (k + U + u) * 128);
                }
        }
        float4 xv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) xv[u] = ld_cached4(px + (k + u) * 128);
#pragma unroll
        for (int r = 0; r < RW; ++r)
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
                for (int m = 0; m < NMAT; ++m) {
                    acc[r][m][0] = __fmaf_rn(cur[r][m][u].x, xv[u].x, acc[r][m][0]);
                    acc[r][m][1] = __fmaf_rn(cur[r][m][u].y, xv[u].y, acc[r][m][1]);
                    acc[r][m][2] = __fmaf_rn(cur[r][m][u].z, xv[u].z, acc[r][m][2]);
                    acc[r][m][3] = __fmaf_rn(cur[r][m][u].w, xv[u].w, acc[r][m][3]);
                }
        if (more) {
#pragma unroll
            for (int r = 0; r < RW; ++r)
#pragma unroll
                for (int m = 0; m < 2; ++m)
#pragma unroll
                    for (int u = 0; u < U; ++u) cur[r][m][u] = nxt[r][m][u];
        }
    }
#pragma unroll
    for (int r = 0; r < RW; ++r) {
        const float va = fold4(acc[r][0][0], acc[r][0][1], acc[r][0][2], acc[r][0][3]);
        if (NMAT == 1) { if (lane == 0) p.o0[i0 + r] = va; }
        else {
            const float vb = fold4(acc[r][1][0], acc[r][1][1], acc[r][1][2], acc[r][1][3]);
            if (lane == 0) { p.o0[i0 + r] = va; p.o1[i0 + r] = __fadd_rn(__fmul_rn(p.alpha, va), __fmul_rn(p.beta, vb)); }
        }
    }
}

// plain copy (read + write) of the same byte count: 8 independent 16-byte loads per thread
__global__ void __launch_bounds__(256) copy8_kernel(const float4 *__restrict__ s, float4 *__restrict__ d, size_t n) {
    const size_t st = (size_t)gridDim.x * blockDim.x * 8;
    for (size_t i = (size_t)blockIdx.x * blockDim.x * 8 + threadIdx.x; i < n; i += st) {
        float4 v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) if (i + q * blockDim.x < n) v[q] = __ldcs(s + i + q * blockDim.x);
#pragma unroll
        for (int q = 0; q < 8; ++q) if (i + q * blockDim.x < n) __stcs(d + i + q * blockDim.x, v[q]);
    }
}
// read-only, 8 independent 16-byte loads per thread in flight
__global__ void __launch_bounds__(256) read8_kernel(const float4 *__restrict__ s, size_t n, float *sink) {
    const size_t st = (size_t)gridDim.x * blockDim.x * 8;
    float acc = 0.f;
    for (size_t i = (size_t)blockIdx.x * blockDim.x * 8 + threadIdx.x; i < n; i += st) {
        float4 v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) v[q] = (i + q * blockDim.x < n) ? __ldcs(s + i + q * blockDim.x) : make_float4(0, 0, 0, 0);
#pragma unroll
        for (int q = 0; q < 8; ++q) acc += v[q].x;
    }
    if (acc == 12345.0f) *sink = acc;
}

// ---- row-dot through shared memory: TMA bulk copies (cp.async.bulk) of each warp's row
// into a per-CTA ring of NS stages; stage = 4 rows x SB columns x NMAT matrices.
__device__ __forceinline__ void mbar_init(uint64_t *b, unsigned cnt) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, unsigned phase) {
    asm volatile("{\n\t.reg .pred P;\n\tWAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
                 "@!P bra WAIT_%=;\n\t}" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"((unsigned)__cvta_generic_to_shared(dst)), "l"(src), "r"(bytes),
                   "r"((unsigned)__cvta_generic_to_shared(bar)) : "memory");
}

// per warp: its own ring (NS stages x NMAT x SBc columns); lane 0 produces, the warp consumes.
template <int NMAT, int NS, int SBc, int MINB>
__global__ void __launch_bounds__(128, MINB) rowdot_tma(const __grid_constant__ RP p) {
    extern __shared__ __align__(128) float sm[];
    __shared__ __align__(8) uint64_t bars[4][NS];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long i = (long long)blockIdx.x * 4 + warp;
    float *ring = sm + warp * (NS * NMAT * SBc);
    if (lane == 0) for (int s = 0; s < NS; ++s) mbar_init(&bars[warp][s], 1);
    __syncwarp();
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    __syncwarp();
    if (i >= p.n) return;
    const float *Ar = p.A + i * p.n, *Br = NMAT == 2 ? p.B + i * p.n : nullptr;
    const int nst = p.n / SBc;   // stages per row
    if (lane == 0) {
        for (int s = 0; s < NS && s < nst; ++s) {
            mbar_expect_tx(&bars[warp][s], NMAT * SBc * 4);
            bulk_g2s(ring + s * NMAT * SBc, Ar + s * SBc, SBc * 4, &bars[warp][s]);
            if (NMAT == 2) bulk_g2s(ring + s * NMAT * SBc + SBc, Br + s * SBc, SBc * 4, &bars[warp][s]);
        }
    }
    float a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
    for (int st = 0; st < nst; ++st) {
        const int s = st % NS;
        mbar_wait(&bars[warp][s], (st / NS) & 1);
        const float *ra = ring + s * NMAT * SBc, *rb = ra + SBc;
#pragma unroll
        for (int u = 0; u < SBc / 128; ++u) {
            const float4 av = *reinterpret_cast<const float4 *>(ra + u * 128 + 4 * lane);
            const float4 xv = ld_cached4(p.x + st * SBc + u * 128 + 4 * lane);
            a0 = __fmaf_rn(av.x, xv.x, a0); a1 = __fmaf_rn(av.y, xv.y, a1);
            a2 = __fmaf_rn(av.z, xv.z, a2); a3 = __fmaf_rn(av.w, xv.w, a3);
            if (NMAT == 2) {
                const float4 bv = *reinterpret_cast<const float4 *>(rb + u * 128 + 4 * lane);
                b0 = __fmaf_rn(bv.x, xv.x, b0); b1 = __fmaf_rn(bv.y, xv.y, b1);
                b2 = __fmaf_rn(bv.z, xv.z, b2); b3 = __fmaf_rn(bv.w, xv.w, b3);
            }
        }
        __syncwarp();
        if (lane == 0 && st + NS < nst) {
            const int nx = st + NS;
            mbar_expect_tx(&bars[warp][s], NMAT * SBc * 4);
            bulk_g2s(ring + s * NMAT * SBc, Ar + nx * SBc, SBc * 4, &bars[warp][s]);
            if (NMAT == 2) bulk_g2s(ring + s * NMAT * SBc + SBc, Br + nx * SBc, SBc * 4, &bars[warp][s]);
        }
    }
    const float va = fold4(a0, a1, a2, a3);
    if (NMAT == 1) { if (lane == 0) p.o0[i] = va; }
    else {
        const float vb = fold4(b0, b1, b2, b3);
        if (lane == 0) { p.o0[i] = va; p.o1[i] = __fadd_rn(__fmul_rn(p.alpha, va), __fmul_rn(p.beta, vb)); }
    }
}

// ---- col-dot (s[j] = sum_i r[i] A[i][j]); canonical: 32 row partitions q = i % 32, ascending
// fma chains, then sequential sum q = 0..31.
struct CP { const float *A, *v; float *out; int n; };

// C0: current body: CB = 32 columns, 1024 threads (warp = partition, lane = column), unroll 8
__global__ void __launch_bounds__(1024, 1) coldot0(const __grid_constant__ CP p) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    __shared__ float red[32][33];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const long long j = (long long)blockIdx.x * 32 + lane;
    float acc = 0;
    const long long stride = 32ll * p.n;
    const float *pc = p.A + j + (long long)w * p.n;
    long long i = w;
    for (; i + 7 * 32 < p.n; i += 8 * 32) {
        float a[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) { a[u] = __ldcs(pc); pc += stride; }
#pragma unroll
        for (int u = 0; u < 8; ++u) acc = __fmaf_rn(a[u], p.v[i + 32 * u], acc);
    }
    for (; i < p.n; i += 32, pc += stride) acc = __fmaf_rn(__ldcs(pc), p.v[i], acc);
    red[w][lane] = acc;
    __syncthreads();
    if (w == 0) {
        float tot = red[0][lane];
        for (int q = 1; q < 32; ++q) tot = __fadd_rn(tot, red[q][lane]);
        p.out[j] = tot;
    }
}

// C1: CB columns as CB/4 float4 quads x 32 partitions; thread t: quad = t % NQ, q = t / NQ.
// unroll U rows of the chain per batch of loads.
template <int CB, int U, int MINB>
__global__ void __launch_bounds__(CB * 8, MINB) coldot_v4(const __grid_constant__ CP p) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    constexpr int NQ = CB / 4, NT = CB * 8;
    __shared__ float red[32][CB + 1];
    const int t = threadIdx.x, quad = t % NQ, q = t / NQ;
    const long long j = (long long)blockIdx.x * CB + 4 * quad;
    float c0 = 0, c1 = 0, c2 = 0, c3 = 0;
    const long long stride = 32ll * p.n;
    const float *pc = p.A + j + (long long)q * p.n;
    long long i = q;
    for (; i + (U - 1) * 32 < p.n; i += U * 32) {
        float4 a[U]; float r[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { a[u] = ld_stream4(pc); pc += stride; }
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = __ldg(p.v + i + 32 * u);
#pragma unroll
        for (int u = 0; u < U; ++u) {
            c0 = __fmaf_rn(a[u].x, r[u], c0); c1 = __fmaf_rn(a[u].y, r[u], c1);
            c2 = __fmaf_rn(a[u].z, r[u], c2); c3 = __fmaf_rn(a[u].w, r[u], c3);
        }
    }
    for (; i < p.n; i += 32, pc += stride) {
        const float4 a = ld_stream4(pc); const float r = __ldg(p.v + i);
        c0 = __fmaf_rn(a.x, r, c0); c1 = __fmaf_rn(a.y, r, c1);
        c2 = __fmaf_rn(a.z, r, c2); c3 = __fmaf_rn(a.w, r, c3);
    }
    red[q][4 * quad + 0] = c0; red[q][4 * quad + 1] = c1; red[q][4 * quad + 2] = c2; red[q][4 * quad + 3] = c3;
    __syncthreads();
    if (t < CB) {
        float tot = red[0][t];
        for (int qq = 1; qq < 32; ++qq) tot = __fadd_rn(tot, red[qq][t]);
        p.out[(long long)blockIdx.x * CB + t] = tot;
    }
    (void)NT;
}

// ---------------------------------------------------------------------------------------
static float *g_flush, *g_sink;
// read-only sweep of a 256 MiB buffer: L2 ends full of clean unrelated lines
__global__ void sweep_kernel(const float4 *p, size_t n, float *sink) {
    float acc = 0;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        const float4 v = __ldcs(p + i); acc += v.x + v.y + v.z + v.w;
    }
    if (acc == 12345.0f) *sink = acc;
}
// ceiling: pure streaming read of `bytes`, 128-bit loads, 4 in flight per thread
__global__ void read_kernel(const float4 *p, size_t n, float *sink) {
    float acc = 0;
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    const size_t st = (size_t)gridDim.x * blockDim.x;
    for (; i + 3 * st < n; i += 4 * st) {
        float4 v0 = ld_stream4((const float *)(p + i)), v1 = ld_stream4((const float *)(p + i + st));
        float4 v2 = ld_stream4((const float *)(p + i + 2 * st)), v3 = ld_stream4((const float *)(p + i + 3 * st));
        acc += v0.x + v1.y + v2.z + v3.w;
    }
    for (; i < n; i += st) { float4 v = __ldcs(p + i); acc += v.x; }
    if (acc == 12345.0f) *sink = acc;
}
__global__ void empty_kernel() {}
template <class K, class P>
static void launch_pdl(K k, dim3 g, dim3 b, bool pdl, const P &p) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = g; cfg.blockDim = b; cfg.dynamicSmemBytes = 0; cfg.stream = 0;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at; cfg.numAttrs = pdl ? 1 : 0;
    CK(cudaLaunchKernelEx(&cfg, k, p));
}
static void flush_l2() {
    CK(cudaMemsetAsync(g_flush, 1, 256u << 20));
    sweep_kernel<<<148 * 8, 256>>>((const float4 *)g_flush, (256u << 20) / 16, g_sink);
}

template <class F>
static float time_it(F launch, int reps = 30) {
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    std::vector<float> ts;
    for (int r = 0; r < reps + 3; ++r) {
        flush_l2();
        CK(cudaEventRecord(e0));
        launch();
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
        if (r >= 3) ts.push_back(ms);
    }
    CK(cudaGetLastError());
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];
}

int main(int argc, char **argv) {
    const int n = argc > 1 ? atoi(argv[1]) : 4096;
    const size_t nn = (size_t)n * n;
    std::vector<float> hA(nn), hB(nn), hx(n);
    uint64_t s = 12345;
    auto rnd = [&]() { s = s * 6364136223846793005ull + 1442695040888963407ull; return (float)((s >> 40) & 0xFFFFFF) / 16777216.0f; };
    for (auto &v : hA) v = rnd();
    for (auto &v : hB) v = rnd();
    for (auto &v : hx) v = rnd();
    float *A, *B, *x, *o0, *o1, *r0, *r1;
    CK(cudaMalloc(&A, nn * 4)); CK(cudaMalloc(&B, nn * 4)); CK(cudaMalloc(&x, n * 4));
    CK(cudaMalloc(&o0, n * 4)); CK(cudaMalloc(&o1, n * 4)); CK(cudaMalloc(&r0, n * 4)); CK(cudaMalloc(&r1, n * 4));
    CK(cudaMalloc(&g_flush, 256u << 20)); CK(cudaMalloc(&g_sink, 64));
    CK(cudaMemcpy(A, hA.data(), nn * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(B, hB.data(), nn * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(x, hx.data(), n * 4, cudaMemcpyHostToDevice));
    const double peak = argc > 2 ? atof(argv[2]) : 6553.0;
    auto same = [&](float *a, float *b) {
        std::vector<uint32_t> ha(n), hb(n);
        CK(cudaMemcpy(ha.data(), a, n * 4, cudaMemcpyDeviceToHost)); CK(cudaMemcpy(hb.data(), b, n * 4, cudaMemcpyDeviceToHost));
        return memcmp(ha.data(), hb.data(), n * 4) == 0;
    };
    auto report = [&](const char *name, float ms, double bytes, bool ok) {
        printf("%-44s %8.2f us  %7.1f GB/s  frac %.3f  %s\n", name, ms * 1e3, bytes / (ms * 1e-3) / 1e9,
               bytes / (ms * 1e-3) / 1e9 / peak, ok ? "bit-exact" : "MISMATCH");
    };
    const double b2 = 2.0 * nn * 4 + 3.0 * n * 4, b1 = 1.0 * nn * 4 + 2.0 * n * 4;
    const int g4 = (n + 3) / 4;
    for (int bpsm : {4, 8, 16}) {
        char nm[64]; snprintf(nm, 64, "read ceiling 2 x N^2 floats, %d CTA/SM", bpsm);
        float ms = time_it([&] { read_kernel<<<148 * bpsm, 256>>>((const float4 *)A, nn / 4, g_sink); read_kernel<<<148 * bpsm, 256>>>((const float4 *)B, nn / 4, g_sink); });
        report(nm, ms, 2.0 * nn * 4, true);
        snprintf(nm, 64, "read ceiling N^2 floats, %d CTA/SM", bpsm);
        ms = time_it([&] { read_kernel<<<148 * bpsm, 256>>>((const float4 *)A, nn / 4, g_sink); });
        report(nm, ms, 1.0 * nn * 4, true);
    }
    // ---- GESUMMV (NMAT = 2)
    RP ref{A, B, x, r0, r1, n, 1.5f, 1.2f};
    RP pp{A, B, x, o0, o1, n, 1.5f, 1.2f};
    {
        float ms = time_it([&] { rowdot<2, 2, 0, 8><<<g4, 128>>>(ref); });
        report("gesummv R0 U2 (current)", ms, b2, true);
    }
#define ROWV(NAME, ...) { CK(cudaMemset(o0, 0, n * 4)); CK(cudaMemset(o1, 0, n * 4)); \
        float ms = time_it([&] { __VA_ARGS__<<<g4, 128>>>(pp); }); report(NAME, ms, b2, same(o0, r0) && same(o1, r1)); }
    ROWV("gesummv R1 U2 whole-row L2 prefetch", rowdot<2, 2, 1, 8>)
    ROWV("gesummv R2 U2 windowed L2 prefetch", rowdot<2, 2, 2, 8>)
    ROWV("gesummv U4 minb7", rowdot<2, 4, 0, 7>)
    {   // ceilings for 134 MB at this size
        for (int bpsm : {2, 4, 8}) {
            char nm[64]; snprintf(nm, 64, "copy 64 MiB (134 MB moved), %d CTA/SM", bpsm);
            float ms = time_it([&] { copy8_kernel<<<148 * bpsm, 256>>>((const float4 *)A, (float4 *)B, nn / 4); });
            report(nm, ms, 2.0 * nn * 4, true);
            snprintf(nm, 64, "read 2 x 64 MiB, 8 loads in flight, %d CTA/SM", bpsm);
            ms = time_it([&] { read8_kernel<<<148 * bpsm, 256>>>((const float4 *)A, nn / 4, g_sink); read8_kernel<<<148 * bpsm, 256>>>((const float4 *)B, nn / 4, g_sink); });
            report(nm, ms, 2.0 * nn * 4, true);
        }
        CK(cudaMemcpy(B, hB.data(), nn * 4, cudaMemcpyHostToDevice));
    }
    ROWV("gesummv double-buffered U2 RW1", (rowdot_db<2, 2, 1, 7>))
    ROWV("gesummv double-buffered U2 RW1 minb4", (rowdot_db<2, 2, 1, 4>))
    ROWV("gesummv double-buffered U1 RW2", (rowdot_db<2, 1, 2, 4>))
    ROWV("gesummv double-buffered U4 RW1 minb4", (rowdot_db<2, 4, 1, 4>))
    ROWV("gesummv U4 minb7 whole-row prefetch", rowdot<2, 4, 1, 7>)
    ROWV("gesummv U1 whole-row prefetch", rowdot<2, 1, 1, 8>)
#define ROWT(NAME, NMAT_, NS, SBc, MINB) { CK(cudaMemset(o0, 0, n * 4)); CK(cudaMemset(o1, 0, n * 4)); \
        const int smb = 4 * NS * NMAT_ * SBc * 4; \
        CK(cudaFuncSetAttribute(rowdot_tma<NMAT_, NS, SBc, MINB>, cudaFuncAttributeMaxDynamicSharedMemorySize, smb)); \
        float ms = time_it([&] { rowdot_tma<NMAT_, NS, SBc, MINB><<<g4, 128, smb>>>(pp); }); \
        report(NAME, ms, NMAT_ == 2 ? b2 : b1, NMAT_ == 2 ? (same(o0, r0) && same(o1, r1)) : same(o0, r0)); }
    ROWT("gesummv TMA ring NS2 x 512 cols", 2, 2, 512, 1)
    ROWT("gesummv TMA ring NS3 x 256 cols", 2, 3, 256, 1)
    ROWT("gesummv TMA ring NS2 x 256 cols", 2, 2, 256, 1)
    ROWT("gesummv TMA ring NS4 x 128 cols", 2, 4, 128, 1)
    // ---- BICG q (NMAT = 1)
    {
        RP r{A, nullptr, x, r0, nullptr, n, 0, 0};
        float ms = time_it([&] { rowdot<1, 4, 0, 8><<<g4, 128>>>(r); });
        report("bicg_q R0 U4 (current)", ms, b1, true);
        RP q{A, nullptr, x, o0, nullptr, n, 0, 0};
#define ROWQ(NAME, ...) { CK(cudaMemset(o0, 0, n * 4)); float ms = time_it([&] { __VA_ARGS__<<<g4, 128>>>(q); }); report(NAME, ms, b1, same(o0, r0)); }
        ROWQ("bicg_q U4 whole-row prefetch", rowdot<1, 4, 1, 8>)
        ROWQ("bicg_q U4 windowed prefetch", rowdot<1, 4, 2, 8>)
        ROWQ("bicg_q U8 minb7", rowdot<1, 8, 0, 7>)
        ROWQ("bicg_q U2 whole-row prefetch", rowdot<1, 2, 1, 8>)
        pp = RP{A, nullptr, x, o0, nullptr, n, 0, 0};
        ROWT("bicg_q TMA ring NS4 x 256 cols", 1, 4, 256, 1)
        ROWT("bicg_q TMA ring NS2 x 512 cols", 1, 2, 512, 1)
    }
    // ---- BICG s (col-dot)
    {
        CP r{A, x, r0, n};
        float ms = time_it([&] { coldot0<<<n / 32, 1024>>>(r); });
        report("bicg_s C0 CB32 1024thr (current)", ms, b1, true);
        CP c{A, x, o0, n};
#define COLV(NAME, CB, U, MINB) { CK(cudaMemset(o0, 0, n * 4)); \
        float ms = time_it([&] { coldot_v4<CB, U, MINB><<<n / CB, CB * 8>>>(c); }); report(NAME, ms, b1, same(o0, r0)); }
        COLV("bicg_s CB16 U8", 16, 8, 1)
        COLV("bicg_s CB16 U16", 16, 16, 1)
        COLV("bicg_s CB32 U8", 32, 8, 1)
        COLV("bicg_s CB32 U16", 32, 16, 1)
        COLV("bicg_s CB8 U16", 8, 16, 1)
        COLV("bicg_s CB8 U32", 8, 32, 1)
        COLV("bicg_s CB16 U32", 16, 32, 1)
    }
    // ---- fixed costs: empty kernel; streaming read at several sizes
    {
        float ms = time_it([&] { empty_kernel<<<148, 128>>>(); });
        printf("%-44s %8.2f us\n", "empty kernel (event to event)", ms * 1e3);
        float *big; const size_t nb = 1ull << 30; CK(cudaMalloc(&big, nb)); CK(cudaMemset(big, 0, nb));
        for (size_t mb : {16, 32, 64, 128, 256, 512, 1024}) {
            char nm[64]; snprintf(nm, 64, "read ceiling %zu MiB", mb);
            ms = time_it([&] { read_kernel<<<148 * 8, 256>>>((const float4 *)big, (mb << 20) / 16, g_sink); });
            report(nm, ms, (double)(mb << 20), true);
        }
        CK(cudaFree(big));
    }
    // ---- the bench step's three kernels back to back, plain stream order vs PDL (independent)
    {
        RP g2{A, B, x, o0, o1, n, 1.5f, 1.2f};
        RP q1{A, nullptr, x, r0, nullptr, n, 0, 0};
        CP c1{A, x, r1, n};
        for (int pdl = 0; pdl < 2; ++pdl) {
            float ms = time_it([&] {
                launch_pdl(rowdot<2, 2, 0, 8>, dim3(g4), dim3(128), false, g2);
                launch_pdl(coldot0, dim3(n / 32), dim3(1024), pdl, c1);
                launch_pdl(rowdot<1, 4, 0, 8>, dim3(g4), dim3(128), pdl, q1);
            });
            report(pdl ? "step: 3 current kernels, PDL" : "step: 3 current kernels, stream order", ms, b2 + 2 * b1, true);
            ms = time_it([&] {
                launch_pdl(rowdot<2, 4, 0, 7>, dim3(g4), dim3(128), false, g2);
                launch_pdl(coldot_v4<32, 16, 1>, dim3(n / 32), dim3(256), pdl, c1);
                launch_pdl(rowdot<1, 4, 0, 8>, dim3(g4), dim3(128), pdl, q1);
            });
            report(pdl ? "step: 3 best kernels, PDL" : "step: 3 best kernels, stream order", ms, b2 + 2 * b1, true);
            // as the runtime queues them: an event after each kernel, a side stream waiting on it
            // with a small D2H copy
            static cudaStream_t side = nullptr; static cudaEvent_t ev[3]; static float *hbuf = nullptr;
            if (!side) {
                CK(cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking));
                for (auto &e : ev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
                CK(cudaMallocHost(&hbuf, 3 * n * 4));
            }
            cudaEvent_t se0, se1; CK(cudaEventCreate(&se0)); CK(cudaEventCreate(&se1));
            ms = time_it([&] {
                launch_pdl(rowdot<2, 4, 0, 7>, dim3(g4), dim3(128), false, g2);
                CK(cudaEventRecord(ev[0], 0)); CK(cudaStreamWaitEvent(side, ev[0], 0));
                CK(cudaMemcpyAsync(hbuf, o0, n * 4, cudaMemcpyDeviceToHost, side));
                launch_pdl(coldot_v4<32, 16, 1>, dim3(n / 32), dim3(256), pdl, c1);
                CK(cudaEventRecord(ev[1], 0)); CK(cudaStreamWaitEvent(side, ev[1], 0));
                CK(cudaMemcpyAsync(hbuf + n, r1, n * 4, cudaMemcpyDeviceToHost, side));
                launch_pdl(rowdot<1, 4, 0, 8>, dim3(g4), dim3(128), pdl, q1);
                CK(cudaEventRecord(ev[2], 0)); CK(cudaStreamWaitEvent(side, ev[2], 0));
                CK(cudaMemcpyAsync(hbuf + 2 * n, r0, n * 4, cudaMemcpyDeviceToHost, side));
                CK(cudaEventRecord(se1, side)); CK(cudaStreamWaitEvent(0, se1, 0));
            });
            report(pdl ? "step: 3 best + events + D2H, PDL" : "step: 3 best + events + D2H, stream order", ms, b2 + 2 * b1, true);
            {
                static cudaEvent_t tev[3];
                static bool made = false;
                if (!made) { for (auto &e : tev) CK(cudaEventCreate(&e)); made = true; }
                ms = time_it([&] {
                    launch_pdl(rowdot<2, 4, 0, 7>, dim3(g4), dim3(128), false, g2);
                    CK(cudaEventRecord(tev[0], 0));
                    launch_pdl(coldot_v4<32, 16, 1>, dim3(n / 32), dim3(256), pdl, c1);
                    CK(cudaEventRecord(tev[1], 0));
                    launch_pdl(rowdot<1, 4, 0, 8>, dim3(g4), dim3(128), pdl, q1);
                    CK(cudaEventRecord(tev[2], 0));
                });
                report(pdl ? "step: 3 best, TIMING events only, PDL" : "step: 3 best, TIMING events only, stream order", ms, b2 + 2 * b1, true);
            }
            for (int variant = 0; variant < 4; ++variant) {
                ms = time_it([&] {
                    launch_pdl(rowdot<2, 4, 0, 7>, dim3(g4), dim3(128), false, g2);
                    CK(cudaEventRecord(ev[0], 0));
                    if (variant >= 1) CK(cudaStreamWaitEvent(side, ev[0], 0));
                    if (variant == 2) CK(cudaMemcpyAsync(hbuf, o0, n * 4, cudaMemcpyDeviceToHost, side));
                    launch_pdl(coldot_v4<32, 16, 1>, dim3(n / 32), dim3(256), pdl, c1);
                    CK(cudaEventRecord(ev[1], 0));
                    if (variant >= 1) CK(cudaStreamWaitEvent(side, ev[1], 0));
                    if (variant == 2) CK(cudaMemcpyAsync(hbuf + n, r1, n * 4, cudaMemcpyDeviceToHost, side));
                    launch_pdl(rowdot<1, 4, 0, 8>, dim3(g4), dim3(128), pdl, q1);
                    CK(cudaEventRecord(ev[2], 0));
                    if (variant >= 1) CK(cudaStreamWaitEvent(side, ev[2], 0));
                    if (variant >= 2) CK(cudaMemcpyAsync(hbuf + 2 * n, r0, n * 4, cudaMemcpyDeviceToHost, side));
                    if (variant == 3) {   // all three returns after the last kernel
                        CK(cudaMemcpyAsync(hbuf, o0, n * 4, cudaMemcpyDeviceToHost, side));
                        CK(cudaMemcpyAsync(hbuf + n, r1, n * 4, cudaMemcpyDeviceToHost, side));
                    }
                    if (variant >= 1) { CK(cudaEventRecord(se1, side)); CK(cudaStreamWaitEvent(0, se1, 0)); }
                });
                static const char *vn[4] = {"events only", "events + side waits", "events + per-kernel D2H", "events + D2H at end"};
                char nm[80]; snprintf(nm, 80, "step: 3 best, %s, %s", vn[variant], pdl ? "PDL" : "stream order");
                report(nm, ms, b2 + 2 * b1, true);
            }
        }
    }
    return 0;
}
