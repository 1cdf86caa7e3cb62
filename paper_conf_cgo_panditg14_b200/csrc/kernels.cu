// kernels.cu -- sm_100a kernels of the B200 FluidiCL hot path.
//
//  * coop_kernel<Body>: the persistent work-group dispatcher (C8, Fig 8, L16.s12/s.26-27,
//    Figs 11-12 / L22.s1-4).  CTAs claim GPU tasks in ascending key order (key = lowest
//    flattened work-group id a task covers, so the GPU "starts executing from the other end",
//    L16.s8) and read the host's watermark word {epoch, W} with an ld.relaxed.sys load.  A task
//    runs iff epoch matches and key < W; otherwise the CTA exits -- every later task is covered
//    too because W only decreases and keys only increase.  Long tasks poll the word again every
//    `abort_period` inner iterations (C24/C25, L20.s44-51) and abort before storing (write-once).
//  * plain_kernel<Body>: the same bodies as an ordinary grid with no status reads (GPU-only).
//  * merge_kernel<ES>: the Fig 9 diff-merge (L18.s1-5), 128-bit vectorised, bitwise compare at
//    element granularity (L16.s32-35), predicated stores, warp ballot to skip unchanged runs.
//
// A "task" is the GPU's unit of claiming: a sub-range of one work-group (row/col dot kernels)
// or a tile of several work-groups (GEMM-like, stencil and elementwise kernels).  Work-group
// independence (L14.s22-23) makes both legal; the merge absorbs any duplicated work.
//
// Arithmetic follows the canonical operation order shared with host_bodies.cpp (see
// fcl_internal.h): __fmaf_rn / __fadd_rn / __fmul_rn / __fdiv_rn / __fsqrt_rn only.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <type_traits>

#include "fcl_internal.h"

namespace fcl {

// ------------------------------------------------------------------------------------------
// Arithmetic (canonical IEEE operations; integer variants wrap mod 2^32)
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ float op_fma(float a, float b, float c) { return __fmaf_rn(a, b, c); }
__device__ __forceinline__ int32_t op_fma(int32_t a, int32_t b, int32_t c) {
    return (int32_t)((uint32_t)a * (uint32_t)b + (uint32_t)c);
}
__device__ __forceinline__ float op_add(float a, float b) { return __fadd_rn(a, b); }
__device__ __forceinline__ int32_t op_add(int32_t a, int32_t b) { return (int32_t)((uint32_t)a + (uint32_t)b); }
__device__ __forceinline__ float op_mul(float a, float b) { return __fmul_rn(a, b); }
__device__ __forceinline__ int32_t op_mul(int32_t a, int32_t b) { return (int32_t)((uint32_t)a * (uint32_t)b); }

// Packed fp32 fma (sm_100a FFMA2, PTX fma.rn.f32x2): two independent IEEE fp32 fmas with
// round-to-nearest in one instruction -- each lane's result is bit-identical to op_fma's.  Used
// by the GEMM bodies' register outer product, which is issue-bound with scalar FFMA.
__device__ __forceinline__ float2 op_fma2(float2 a, float2 b, float2 c) {
    unsigned long long r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;"
        : "=l"(r)
        : "l"(*reinterpret_cast<const unsigned long long *>(&a)), "l"(*reinterpret_cast<const unsigned long long *>(&b)),
          "l"(*reinterpret_cast<const unsigned long long *>(&c)));
    return *reinterpret_cast<const float2 *>(&r);
}

// acc[r][c] = fma(a[r], b[c], acc[r][c]) for every r < 8, c < TN (one k step of a register tile;
// every output one fma, so the per-output k-chain is unchanged)
#ifndef FCL_GEMM_FFMA2
#define FCL_GEMM_FFMA2 1
#endif
template <int TN>
__device__ __forceinline__ void outer(float (&acc)[8][TN], const float *a, const float *b) {
    if (FCL_GEMM_FFMA2) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const float2 ar = make_float2(a[r], a[r]);
#pragma unroll
            for (int c = 0; c < TN; c += 2) {
                const float2 v = op_fma2(ar, make_float2(b[c], b[c + 1]), make_float2(acc[r][c], acc[r][c + 1]));
                acc[r][c] = v.x; acc[r][c + 1] = v.y;
            }
        }
    } else {
#pragma unroll
        for (int r = 0; r < 8; ++r)
#pragma unroll
            for (int c = 0; c < TN; ++c) acc[r][c] = op_fma(a[r], b[c], acc[r][c]);
    }
}
template <int TN>
__device__ __forceinline__ void outer(int32_t (&acc)[8][TN], const int32_t *a, const int32_t *b) {
#pragma unroll
    for (int r = 0; r < 8; ++r)
#pragma unroll
        for (int c = 0; c < TN; ++c) acc[r][c] = op_fma(a[r], b[c], acc[r][c]);
}

template <typename T> struct V4;
template <> struct V4<float> { typedef float4 type; };
template <> struct V4<int32_t> { typedef int4 type; };

// Streaming 128-bit load that does not allocate in L1 (data read exactly once).
template <typename T>
__device__ __forceinline__ typename V4<T>::type ld_stream4(const T *p) {
    typename V4<T>::type v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(*reinterpret_cast<uint32_t *>(&v.x)), "=r"(*reinterpret_cast<uint32_t *>(&v.y)),
                   "=r"(*reinterpret_cast<uint32_t *>(&v.z)), "=r"(*reinterpret_cast<uint32_t *>(&v.w))
                 : "l"(p));
    return v;
}
// 128-bit load through L2 only (.cg): for input rows that H2D copies may still be writing while
// the kernel runs (streamed inputs) -- never served from a stale L1 line or the
// non-coherent path.
template <typename T>
__device__ __forceinline__ typename V4<T>::type ld_cg4(const T *p) {
    return __ldcg(reinterpret_cast<const typename V4<T>::type *>(p));
}
template <typename T>
__device__ __forceinline__ typename V4<T>::type ld_cached4(const T *p) {
    return __ldg(reinterpret_cast<const typename V4<T>::type *>(p));
}

// ------------------------------------------------------------------------------------------
// Watermark access (D1/D2, Fig 8)
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ unsigned long long ld_status(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
// System-scope acquire: data published before the word (H2D pieces ahead of the arrival-front
// memop on the same stream) is visible to this thread's later loads, and -- through the CTA
// barrier that follows -- to the CTA's.
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ unsigned int decode_w(unsigned long long st, const CoopCtl &c) {
    // A status word from another kernel (stale epoch) means "nothing covered" (C14, L20.s9).
    return ((unsigned int)(st >> 32) == c.epoch) ? (unsigned int)st : c.w_default;
}

// Status prefetch without a register: thread 0 copies the 16-byte aligned pair holding the
// status word into shared memory with cp.async.cg (L2, never a stale L1 line; the publication
// memop lands in L2) and collects it at the next check.  Status in mapped host memory is read
// synchronously instead (system-scope load, no caching assumptions).
__device__ __forceinline__ void status_prefetch(const CoopCtl &c, unsigned long long *s_st) {
    if (c.status_mapped) return;
    const unsigned long long *src = (const unsigned long long *)((uintptr_t)c.status & ~(uintptr_t)15);
    const unsigned int dst = (unsigned int)__cvta_generic_to_shared(s_st);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n\tcp.async.commit_group;\n" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ unsigned long long status_take(const CoopCtl &c, const unsigned long long *s_st) {
    if (c.status_mapped) return ld_status(c.status);
    asm volatile("cp.async.wait_all;\n" ::: "memory");
    return *(volatile const unsigned long long *)(s_st + (((uintptr_t)c.status >> 3) & 1));
}

// Per-task view of the status for in-task polling (abort checks in loops, Fig 12).  Nothing
// of it lives in registers across the body: the prefetched status, the task key and the abort
// verdict are all in shared memory, so a polling body keeps its whole register budget.
struct TaskCtx {
    const CoopCtl *c;            // nullptr for plain launches (parameter space, no register copy)
    unsigned long long *s_st;    // shared, 16-byte aligned: status pair prefetched by thread 0
    long long *s_key;            // shared: key of the running task
    int *s_flag;                 // shared, 2 slots (D2: the local 'completedatcpu'); w + 1 after an abort
    int polls;                   // polls so far (uniform): slot polls & 1 is the next one's
    // The watermark this task was checked against: work-groups with flattened id >= wmask are
    // the host's, so a task spanning several work-groups (tiles) stores none of their outputs --
    // at a fixed split every output word is then written by exactly one device (north_star's
    // invariant, L16.s9 "non-overlapping parts").  0xFFFFFFFF: no mask (plain grids, first tasks).
    unsigned int wmask;

    // In-task poll period in body iterations (a huge value when there is none).
    __device__ __forceinline__ long long period() const {
        return (c != nullptr && c->abort_period > 0) ? (long long)c->abort_period : (1ll << 62);
    }
    // A poll in two halves around a barrier the body executes anyway (no barrier of its own):
    // post() -- thread 0 takes the prefetched status and writes the verdict into this poll's
    // slot -- before the barrier, verdict() after it (all threads).  Consecutive polls use
    // alternate slots, so a poll never overwrites a verdict a slow thread has yet to read.
    __device__ __forceinline__ void post() {
        if (threadIdx.x == 0) {
            const unsigned int w = decode_w(status_take(*c, s_st), *c);
            status_prefetch(*c, s_st);   // consumed at the next poll
            s_flag[polls & 1] = ((unsigned long long)*s_key >= (unsigned long long)w) ? (int)(w + 1u) : 0;
        }
    }
    __device__ __forceinline__ bool verdict() {
        const int f = ((volatile int *)s_flag)[polls & 1];
        ++polls;
        return f != 0;
    }
    // A complete poll (called by ALL threads at a CTA-uniform point).
    __device__ __forceinline__ bool check() {
        if (c == nullptr || c->abort_period <= 0) return false;
        post();
        __syncthreads();
        return verdict();
    }
    __device__ __forceinline__ unsigned int abort_w() const { return (unsigned int)(s_flag[(polls - 1) & 1] - 1); }
};

// ------------------------------------------------------------------------------------------
// Diff-merge (Fig 9): gpu[e] = (cpu[e] != twin[e]) ? cpu[e] : gpu[e], bitwise, per element.
// cpu/twin are streamed once with 128-bit no-L1-allocate loads (4 vectors in flight per
// thread); changed elements are stored with predicated element stores (a fully changed vector
// with one 128-bit store), so the GPU copy is never read: traffic = 8 B/word read + 4 B per
// changed word written.  Byte/half-word element sizes blend within the 32-bit lane.
// ------------------------------------------------------------------------------------------
template <int ES>
__device__ __forceinline__ void merge_vec(uint8_t *g, const uint4 c, const uint4 t) {
    const uint32_t cw[4] = {c.x, c.y, c.z, c.w}, tw[4] = {t.x, t.y, t.z, t.w};
    if (ES == 4) {
        const bool ch0 = cw[0] != tw[0], ch1 = cw[1] != tw[1], ch2 = cw[2] != tw[2], ch3 = cw[3] != tw[3];
        if (ch0 && ch1 && ch2 && ch3) { *reinterpret_cast<uint4 *>(g) = c; return; }
        uint32_t *gw = reinterpret_cast<uint32_t *>(g);
        if (ch0) gw[0] = cw[0];
        if (ch1) gw[1] = cw[1];
        if (ch2) gw[2] = cw[2];
        if (ch3) gw[3] = cw[3];
    } else if (ES == 8) {
        const bool ch0 = (cw[0] != tw[0]) || (cw[1] != tw[1]);
        const bool ch1 = (cw[2] != tw[2]) || (cw[3] != tw[3]);
        if (ch0 && ch1) { *reinterpret_cast<uint4 *>(g) = c; return; }
        unsigned long long *gd = reinterpret_cast<unsigned long long *>(g);
        if (ch0) gd[0] = ((unsigned long long)cw[1] << 32) | cw[0];
        if (ch1) gd[1] = ((unsigned long long)cw[3] << 32) | cw[2];
    } else {
        uint32_t m[4];
        bool all = true, any = false;
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            if (ES == 1) m[q] = __vcmpne4(cw[q], tw[q]);
            else m[q] = __vcmpne2(cw[q], tw[q]);
            all &= (m[q] == 0xFFFFFFFFu);
            any |= (m[q] != 0u);
        }
        if (all) { *reinterpret_cast<uint4 *>(g) = c; return; }
        if (!any) return;
        uint32_t *gw = reinterpret_cast<uint32_t *>(g);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            if (m[q] == 0xFFFFFFFFu) gw[q] = cw[q];
            else if (m[q]) gw[q] = (cw[q] & m[q]) | (gw[q] & ~m[q]);
        }
    }
}

template <int ES>
__device__ __forceinline__ void merge_scalar(uint8_t *g, const uint8_t *c, const uint8_t *t, size_t nbytes) {
    for (size_t e = 0; e + ES <= nbytes; e += ES) {
        bool ch = false;
#pragma unroll
        for (int b = 0; b < ES; ++b) ch |= (c[e + b] != t[e + b]);
        if (ch) {
#pragma unroll
            for (int b = 0; b < ES; ++b) g[e + b] = c[e + b];
        }
    }
}

// The twin stream may alias the destination (twin := device copy for exact spans), so it is
// read through the coherent path.
__device__ __forceinline__ uint4 ld_na_v4(const uint8_t *p) {
    uint4 v;
    asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

__device__ __forceinline__ uint4 ld_nc_v4(const uint8_t *p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

// Merge [0, nbytes) of one buffer with all threads of the grid (head/tail bytes scalar).
template <int ES>
__device__ __forceinline__ void merge_range(uint8_t *gpu, const uint8_t *cpu, const uint8_t *twin, size_t nbytes,
                                            size_t tid, size_t nthreads) {
    size_t head = 0, nvec = 0, tail = nbytes;
    const uintptr_t ag = reinterpret_cast<uintptr_t>(gpu) & 15u;
    if (ag == (reinterpret_cast<uintptr_t>(cpu) & 15u) && ag == (reinterpret_cast<uintptr_t>(twin) & 15u)) {
        head = ag ? 16 - ag : 0;
        if (head > nbytes) head = nbytes;
        nvec = (nbytes - head) / 16;
        tail = nbytes - head - 16 * nvec;
    }
    if (tid == 0 && head) merge_scalar<ES>(gpu, cpu, twin, head);
    if (tid == (nthreads > 1 ? 1 : 0) && tail) {
        const size_t off = head + 16 * nvec;
        merge_scalar<ES>(gpu + off, cpu + off, twin + off, tail);
    }
    uint8_t *g = gpu + head;
    const uint8_t *c = cpu + head, *t = twin + head;
    constexpr int U = 4;
    size_t v = tid;
    for (; v + (U - 1) * nthreads < nvec; v += U * nthreads) {
        uint4 cv[U], tv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) { cv[u] = ld_nc_v4(c + 16 * (v + u * nthreads)); tv[u] = ld_na_v4(t + 16 * (v + u * nthreads)); }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const bool diff = (cv[u].x != tv[u].x) | (cv[u].y != tv[u].y) | (cv[u].z != tv[u].z) | (cv[u].w != tv[u].w);
            // warp vote: a warp whose 512-byte segment is unchanged skips the store path
            if (__ballot_sync(__activemask(), diff) && diff) merge_vec<ES>(g + 16 * (v + u * nthreads), cv[u], tv[u]);
        }
    }
    for (; v < nvec; v += nthreads) {
        const uint4 cv = ld_nc_v4(c + 16 * v), tv = ld_na_v4(t + 16 * v);
        if ((cv.x != tv.x) | (cv.y != tv.y) | (cv.z != tv.z) | (cv.w != tv.w)) merge_vec<ES>(g + 16 * v, cv, tv);
    }
}

template <int ES>
__global__ void __launch_bounds__(256)
merge_kernel(uint8_t *gpu, const uint8_t *cpu, const uint8_t *twin, size_t nbytes) {
    merge_range<ES>(gpu, cpu, twin, nbytes, (size_t)blockIdx.x * blockDim.x + threadIdx.x,
                    (size_t)gridDim.x * blockDim.x);
}

// Merge of every OUT/INOUT buffer of a cooperative launch, queued behind the dispatcher.
// The domain [span_lo(wm), span_hi(hi)) of each buffer comes from the watermark the
// dispatcher acted on (it skipped only work-groups >= wm, whose host results were staged
// before the watermark was published, L16.s15); nothing is merged if it never skipped.
__device__ __forceinline__ void merge_dev_body(const DevMergeList &L, unsigned long long r, size_t tid, size_t nth) {
    const unsigned int w32 = decode_wm_word(r, L.epoch);
    const long long wm = (long long)w32;
    if (w32 == 0xFFFFFFFFu || wm >= L.hi) return;
    for (int b = 0; b < L.n; ++b) {
        long long b0 = 0, b1 = L.total[b];
        if (L.unit_wgs[b] > 0) {
            b0 = (wm / L.unit_wgs[b]) * L.unit_bytes[b];
            b1 = ((L.hi + L.unit_wgs[b] - 1) / L.unit_wgs[b]) * L.unit_bytes[b];
            if (b0 > L.total[b]) b0 = L.total[b];
            if (b1 > L.total[b]) b1 = L.total[b];
        }
        if (b1 <= b0) continue;
        switch (L.es[b]) {
        case 1: merge_range<1>(L.gpu[b] + b0, L.cpu[b] + b0, L.twin[b] + b0, (size_t)(b1 - b0), tid, nth); break;
        case 2: merge_range<2>(L.gpu[b] + b0, L.cpu[b] + b0, L.twin[b] + b0, (size_t)(b1 - b0), tid, nth); break;
        case 4: merge_range<4>(L.gpu[b] + b0, L.cpu[b] + b0, L.twin[b] + b0, (size_t)(b1 - b0), tid, nth); break;
        default: merge_range<8>(L.gpu[b] + b0, L.cpu[b] + b0, L.twin[b] + b0, (size_t)(b1 - b0), tid, nth); break;
        }
    }
}

// The same merge shared out dynamically: 64 KB chunks of the concatenated domains are claimed
// from `ctr` by whole CTAs (any number of CTAs may take part).
__device__ void merge_dev_chunks(const DevMergeList &L, long long wm, unsigned long long *ctr) {
    constexpr long long CH = 64 * 1024;
    long long b0[6], b1[6], nch[6];
    long long total = 0;
    for (int b = 0; b < L.n; ++b) {
        b0[b] = 0; b1[b] = L.total[b];
        if (L.unit_wgs[b] > 0) {
            b0[b] = (wm / L.unit_wgs[b]) * L.unit_bytes[b];
            b1[b] = ((L.hi + L.unit_wgs[b] - 1) / L.unit_wgs[b]) * L.unit_bytes[b];
            if (b0[b] > L.total[b]) b0[b] = L.total[b];
            if (b1[b] > L.total[b]) b1[b] = L.total[b];
        }
        nch[b] = b1[b] > b0[b] ? (b1[b] - b0[b] + CH - 1) / CH : 0;
        total += nch[b];
    }
    __shared__ long long s_chunk;
    for (;;) {
        if (threadIdx.x == 0) s_chunk = (long long)atomicAdd(ctr, 1ull);
        __syncthreads();
        long long k = s_chunk;
        __syncthreads();
        if (k >= total) return;
        int b = 0;
        while (k >= nch[b]) { k -= nch[b]; ++b; }
        const long long off = b0[b] + k * CH;
        const size_t len = (size_t)((off + CH < b1[b]) ? CH : b1[b] - off);
        switch (L.es[b]) {
        case 1: merge_range<1>(L.gpu[b] + off, L.cpu[b] + off, L.twin[b] + off, len, threadIdx.x, blockDim.x); break;
        case 2: merge_range<2>(L.gpu[b] + off, L.cpu[b] + off, L.twin[b] + off, len, threadIdx.x, blockDim.x); break;
        case 4: merge_range<4>(L.gpu[b] + off, L.cpu[b] + off, L.twin[b] + off, len, threadIdx.x, blockDim.x); break;
        default: merge_range<8>(L.gpu[b] + off, L.cpu[b] + off, L.twin[b] + off, len, threadIdx.x, blockDim.x); break;
        }
    }
}

__global__ void __launch_bounds__(256) merge_dev_kernel(const DevMergeList L) {
    __shared__ unsigned long long s_wm;
    if (threadIdx.x == 0) s_wm = ld_status(L.wm_word);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        // the dispatcher has finished (stream order): tell the host executor (L18.s19)
        if (L.exit_word)
            asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(L.exit_word), "l"((unsigned long long)L.epoch) : "memory");
        if (L.tstamp) L.tstamp[0] = globaltimer();
    }
    __syncthreads();
    struct StampEnd {
        unsigned long long *p;
        __device__ ~StampEnd() { if (p && threadIdx.x == 0) atomicMax(p + 1, globaltimer()); }
    } stamp_end{L.tstamp};
    merge_dev_body(L, s_wm, (size_t)blockIdx.x * blockDim.x + threadIdx.x, (size_t)gridDim.x * blockDim.x);
}

// ------------------------------------------------------------------------------------------
// Dispatcher (persistent, ascending claim) and plain grid
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ void record_wm(const CoopCtl &c, unsigned int w) {
    // epoch-tagged: a later launch's word always wins, within a launch the smallest watermark
    atomicMax(c.wm_out, ((unsigned long long)c.epoch << 32) | (unsigned long long)(0xFFFFFFFFu - w));
}

// (a body may ask for a lower occupancy target in the dispatcher, whose loop state costs registers)
template <class Body> struct CoopMinBlocks { static constexpr int value = Body::kMinBlocks; };

// A body's shared memory: static (the default), or dynamic for a body whose stages exceed the
// 48 KB of static shared memory (Body::kDynSmem; the launch passes sizeof(Smem) and the kernels
// get the attribute once, ensure_smem).
template <class Body, class = void> struct DynSmem { static constexpr bool value = false; };
template <class Body> struct DynSmem<Body, std::void_t<decltype(Body::kDynSmem)>> { static constexpr bool value = Body::kDynSmem; };
template <class Body> struct SmemHolder {
    typedef typename std::conditional<DynSmem<Body>::value, int, typename Body::Smem>::type type;
};
extern __shared__ __align__(16) unsigned char fcl_dyn_smem[];
template <class Body>
__device__ __forceinline__ typename Body::Smem &body_smem(typename SmemHolder<Body>::type &st) {
    if constexpr (DynSmem<Body>::value) return *reinterpret_cast<typename Body::Smem *>(fcl_dyn_smem);
    else return st;
}

// Masked bodies get a second, unmasked copy in the dispatcher (A/B knob)
#ifndef FCL_UNMASKED_COPY
#define FCL_UNMASKED_COPY 1
#endif
// Tasks claimed per atomic on the claim counter by bodies that claim ahead (A/B knob; 1 = the
// paper's one work-group claim at a time, Fig 8)
#ifndef FCL_CLAIM_BATCH
#define FCL_CLAIM_BATCH 1
#endif
template <class Body>
__global__ void __launch_bounds__(Body::kThreads, CoopMinBlocks<Body>::value)
coop_kernel(const __grid_constant__ CoopCtl c, const __grid_constant__ typename Body::Params bp) {
    __shared__ long long s_task, s_key;
    __shared__ __align__(16) unsigned long long s_st[2];
    __shared__ unsigned int s_w;
    __shared__ int s_flag[2];
    __shared__ __align__(16) typename SmemHolder<Body>::type smem_st;
    typename Body::Smem &smem = body_smem<Body>(smem_st);

    if (blockIdx.x == 0 && threadIdx.x == 0) {   // counters of the next launch (stream-ordered)
        *c.claim_next = 0ull;
        if (c.barrier_next)
            for (int q = 0; q < 17; ++q) c.barrier_next[q] = 0u;
        if (c.merge_ctr_next) *c.merge_ctr_next = 0ull;
        if (c.tasks_next) *c.tasks_next = 0ull;
        if (c.tstamp) {   // stats mode: start stamp, reset this launch's merge end and the next end
            c.tstamp[0] = globaltimer();
            c.tstamp[3] = 0ull;
            c.tstamp_next[1] = 0ull;
        }
    }
    // The first task of every CTA is blockIdx.x: no claim and no status wait before it starts.
    // Running a work-group the host already covers is never wrong (the merge keeps the host's
    // words), and long tasks still poll the status inside their loops; the status load issued
    // here is consumed at that first poll.  Later tasks are claimed from the device counter
    // and checked against the watermark (Fig 8) with the load prefetched during the previous
    // task, so neither the claim nor the check is on the critical path.  Only the claimed index
    // and one status word stay live across a task (thread 0's); everything else is in shared
    // memory or the parameter bank, so the dispatcher does not take registers from the body.
    long long t = c.task_lo + (long long)blockIdx.x;
    unsigned int w = c.w_default;
    bool checked = false;
    if (c.check_first) {   // deterministic mode (forced split): check before the first task too
        if (threadIdx.x == 0) s_w = decode_w(ld_status(c.status), c);
        __syncthreads();
        w = s_w;
        checked = true;
        __syncthreads();
    }
    const bool claims = c.task_lo + (long long)gridDim.x < c.task_hi;
    TaskCtx tc;
    tc.c = &c; tc.s_flag = s_flag; tc.s_key = &s_key; tc.s_st = s_st; tc.wmask = 0xFFFFFFFFu; tc.polls = 0;
    // the status is needed only by in-task polls and by the check before a claimed task
    const bool need_status = claims || c.abort_period > 0;
    if (threadIdx.x == 0 && need_status) status_prefetch(c, s_st);
    long long b_next = 0, b_end = 0;   // thread 0: claimed batch (FCL_CLAIM_BATCH > 1)
    bool marked = false;   // thread 0: this CTA recorded a watermark (skip or abort)
    unsigned int rec_w = c.w_default;   // thread 0: lowest mask watermark recorded so far
    for (;;) {
        if (t >= c.task_hi) break;
        const long long key = Body::key(bp, t);
        if (c.task_delay_ns) {
            // fault injection (opts.gpu_delay_us): the GPU reaches this task late -- and, as a
            // work-group that starts late (Fig 8), checks the status when it does
            if (threadIdx.x == 0) {
                const unsigned long long t0 = globaltimer();
                while (globaltimer() - t0 < c.task_delay_ns) __nanosleep(1000);
                s_w = decode_w(ld_status(c.status), c);
            }
            __syncthreads();
            w = s_w;
            checked = true;
            __syncthreads();
        }
        if (checked && (unsigned long long)key >= (unsigned long long)w) {   // covered by the host
            if (threadIdx.x == 0) { record_wm(c, w); marked = true; }
            break;
        }
        if (c.arrival) {
            // streamed inputs: wait until this task's rows arrived, or the host covers it (then
            // every later task is covered too); a stalled stream is a bug -- trap, never hang
            if (threadIdx.x == 0) {
                int covered = 0;
                const unsigned long long t0 = globaltimer();
                unsigned int ns = 128;
                for (;;) {
                    const unsigned long long a = ld_acquire_sys(c.arrival);
                    const unsigned int front = ((unsigned int)(a >> 32) == c.epoch) ? (unsigned int)a : 0u;
                    if ((unsigned long long)key < (unsigned long long)front) break;
                    const unsigned int wv = decode_w(ld_status(c.status), c);
                    if ((unsigned long long)key >= (unsigned long long)wv) { record_wm(c, wv); marked = true; covered = 1; break; }
                    if (globaltimer() - t0 > 5000000000ull) __trap();
                    __nanosleep(ns);
                    if (ns < 2048) ns *= 2;
                }
                s_flag[0] = covered;
            }
            __syncthreads();
            const int covered = s_flag[0];
            __syncthreads();
            if (covered) break;
        }
        if (threadIdx.x == 0) s_key = key;   // read back by thread 0 only
        // claim the next task while this one runs (no claim at all when the grid already
        // covers every task: no contention on the counter)
        long long t_next = c.task_hi;
        if (!Body::kLateClaim && threadIdx.x == 0 && claims) {
            if (FCL_CLAIM_BATCH == 1) {
                t_next = c.task_lo + (long long)gridDim.x + (long long)atomicAdd(c.claim, 1ull);
            } else {   // B ascending tasks per atomic (thread 0's batch: [b_next, b_end))
                if (b_next >= b_end) {
                    b_next = c.task_lo + (long long)gridDim.x + (long long)atomicAdd(c.claim, (unsigned long long)FCL_CLAIM_BATCH);
                    b_end = b_next + FCL_CLAIM_BATCH;
                }
                t_next = b_next++;
            }
        }
        // a task that may span work-groups the host covers stores only those below w (the
        // watermark acted on: the merge domain starts at or below it)
        // (w == the range end: nothing covered, no mask -- the stores then skip the per-row work-group test)
        tc.wmask = (Body::kMasks && checked && w < c.w_default) ? w : 0xFFFFFFFFu;
        if (Body::kMasks && checked && w < rec_w && threadIdx.x == 0) {
            record_wm(c, w);
            rec_w = w;
            marked = true;
        }
        // (a task with nothing covered -- the common case -- runs a copy of the body in which the
        // mask is the constant "keep everything": no per-row work-group tests or their branches)
        bool aborted;
        if (FCL_UNMASKED_COPY && Body::kMasks && tc.wmask == 0xFFFFFFFFu) {
            TaskCtx t2 = tc;
            t2.wmask = 0xFFFFFFFFu;
            aborted = Body::run(bp, t, t2, smem);
            tc.polls = t2.polls;
        } else {
            aborted = Body::run(bp, t, tc, smem);
        }
        if (aborted) {
            if (threadIdx.x == 0) { record_wm(c, tc.abort_w()); marked = true; }
            break;
        }
        if (threadIdx.x == 0) {
            if (c.tasks) atomicAdd(c.tasks, 1ull);
            if (c.exec_cnt) {   // test hook (opts.record_exec_counts): completed tasks and their mask
                atomicAdd(c.exec_cnt + (t - c.task_lo), 1u);
                c.exec_w[t - c.task_lo] = tc.wmask;
            }
            // long tasks claim after they finish: nothing of the dispatcher stays in a register
            if (Body::kLateClaim && claims) t_next = c.task_lo + (long long)gridDim.x + (long long)atomicAdd(c.claim, 1ull);
            s_task = t_next;
            if (need_status) {
                s_w = decode_w(status_take(c, s_st), c);
                status_prefetch(c, s_st);   // for the next task's polls / check
            } else {
                s_w = c.w_default;
            }
        }
        __syncthreads();
        t = s_task;
        w = s_w;
        checked = true;
        __syncthreads();
    }
    if (threadIdx.x == 0 && need_status && !c.status_mapped) asm volatile("cp.async.wait_all;\n" ::: "memory");
    if (c.tstamp && threadIdx.x == 0) atomicMax(c.tstamp + 1, globaltimer());
    if (!c.fused) return;
    // Fused tail.  Every CTA registers its arrival; the LAST one to arrive publishes the
    // GPU-exit signal (L18.s19).  The diff-merge (Fig 9) then runs over the domain given by the
    // lowest watermark any CTA acted on, shared out in 64 KB chunks from a counter, by the CTAs
    // still present: the last one, plus those that had already seen a skip when they arrived
    // (they wait for the last arrival, since a merge is certain).  With nothing to merge -- the
    // GPU-favoured case -- no CTA waits at all.
    __syncthreads();
    if (threadIdx.x == 0) {
        // Only a CTA that recorded a watermark must make that record (and the partial writes
        // of an aborted task) visible before it arrives; complete work-groups are bit-identical
        // to the host's, so when their writes land does not matter.  The merge-role probe is
        // issued before the arrival atomics so the two round trips overlap.
        const unsigned long long wm_probe = ld_status(c.mg.wm_word);
        if (marked) __threadfence();
        // hierarchical arrival count: 16 leaf counters, the CTA completing a leaf bumps the
        // root, the CTA completing the root is the last one (no 1000-way contention on a word)
        const unsigned int leaf = blockIdx.x & 15u;
        const unsigned int nleaf = (gridDim.x > 16u) ? 16u : gridDim.x;
        const unsigned int leaf_size = (gridDim.x - leaf + 15u) / 16u;
        bool last = false;
        if (atomicAdd(c.barrier + 1 + leaf, 1u) == leaf_size - 1) {
            __threadfence();
            last = atomicAdd(c.barrier, 1u) == nleaf - 1;
        }
        const bool skip_seen = decode_wm_word(wm_probe, c.epoch) != 0xFFFFFFFFu;
        int role = last ? 2 : (skip_seen && c.mg.n > 0 ? 1 : 0);
        if (role == 1) {   // wait for the last arrival (the kernel is cooperative: all resident)
            unsigned int v;
            unsigned int ns = 256;
            for (;;) {
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(c.barrier) : "memory");
                if (v >= nleaf) break;
                __nanosleep(ns);
                if (ns < 4096) ns *= 2;
            }
        }
        if (last) {
            __threadfence();
            asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(c.exit_word), "l"((unsigned long long)c.epoch) : "memory");
            if (c.mg.tstamp) c.mg.tstamp[0] = globaltimer();
        }
        s_task = role ? (long long)ld_status(c.mg.wm_word) : 0;
        s_w = (unsigned int)role;
    }
    __syncthreads();
    if (s_w == 0u || c.mg.n == 0) return;
    const unsigned int w32 = decode_wm_word((unsigned long long)s_task, c.epoch);
    if (w32 == 0xFFFFFFFFu || (long long)w32 >= c.mg.hi) return;
    merge_dev_chunks(c.mg, (long long)w32, c.merge_ctr);
    if (c.mg.tstamp && threadIdx.x == 0) atomicMax(c.mg.tstamp + 1, globaltimer());
}

// Programmatic dependent launch (PDL).  Plain grids are launched with programmatic stream
// serialization, so the next plain grid on the stream may start while this one drains (its
// launch latency and ramp hide under our tail).  Every CTA signals launch_dependents at its
// start -- after griddepcontrol.wait when the runtime found a dependency on a grid still in
// flight (pdl_wait), and after block 0 has reset the next slot's counters (fenced), which the
// next grid may use at once.
__device__ __forceinline__ void pdl_wait_prior() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

template <class Body>
__global__ void __launch_bounds__(Body::kThreads, Body::kMinBlocks)
plain_kernel(const __grid_constant__ typename Body::Params bp, long long task_lo, const SlotReset r, int pdl_wait) {
    __shared__ int s_flag[2];
    if (pdl_wait) pdl_wait_prior();
    if (r.tstamp && blockIdx.x == 0 && threadIdx.x == 0) r.tstamp[0] = globaltimer();
    if (blockIdx.x == 0) {
        if (r.claim && threadIdx.x == 0) {   // next slot's dispatcher counters
            *r.claim = 0ull;
            for (int q = 0; q < 17; ++q) r.barrier[q] = 0u;
            *r.merge_ctr = 0ull;
            if (r.tasks) *r.tasks = 0ull;
            __threadfence();
        }
        __syncthreads();
    }
    pdl_trigger();
    if (r.delay_ns && blockIdx.x == 0) {   // test hook: a slow GPU (tests/test_gpu_select.py)
        const unsigned long long t0 = globaltimer();
        while (globaltimer() - t0 < r.delay_ns) __nanosleep(1000);
    }
    __shared__ __align__(16) typename SmemHolder<Body>::type smem_st;
    typename Body::Smem &smem = body_smem<Body>(smem_st);
    __shared__ long long s_key;
    TaskCtx tc;
    tc.c = nullptr; tc.s_st = nullptr; tc.s_flag = s_flag; tc.s_key = &s_key; tc.wmask = 0xFFFFFFFFu; tc.polls = 0;
    Body::run(bp, task_lo + (long long)blockIdx.x, tc, smem);
    if (r.exec_cnt && threadIdx.x == 0) atomicAdd(r.exec_cnt + blockIdx.x, 1u);   // test hook
    if (r.tstamp) {
        __syncthreads();
        if (threadIdx.x == 0) atomicMax(r.tstamp + 1, globaltimer());
    }
    if (r.exit_word) {   // lite cooperative launch: GPU-exit signal for the host (L18.s19)
        __syncthreads();
        if (threadIdx.x == 0) {
            // hierarchical arrival (16 leaves + root); no fence: the word publishes no data,
            // the outputs' return copies are ordered behind the grid on the streams
            const unsigned int leaf = blockIdx.x & 15u;
            const unsigned int nleaf = (gridDim.x > 16u) ? 16u : gridDim.x;
            const unsigned int leaf_size = (gridDim.x - leaf + 15u) / 16u;
            if (atomicAdd(r.arrive + 1 + leaf, 1u) == leaf_size - 1 && atomicAdd(r.arrive, 1u) == nleaf - 1)
                asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(r.exit_word), "l"((unsigned long long)r.epoch) : "memory");
        }
    }
}

// Twin capture (C5, L16.s2-3): copy every OUT/INOUT buffer to its twin in ONE launch.
struct CopyList { uint8_t *dst[6]; const uint8_t *src[6]; size_t bytes[6]; int n; };

__global__ void __launch_bounds__(256) copies_kernel(const CopyList L, int pdl_wait) {
    // (launched behind plain grids with programmatic serialization: wait until they have
    // completed and their stores are visible -- griddepcontrol.wait covers every earlier grid)
    if (pdl_wait) asm volatile("griddepcontrol.wait;" ::: "memory");
    const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    const size_t nth = (size_t)gridDim.x * blockDim.x;
    for (int b = 0; b < L.n; ++b) {
        const size_t nv = L.bytes[b] / 16;
        const uint4 *s = reinterpret_cast<const uint4 *>(L.src[b]);
        uint4 *d = reinterpret_cast<uint4 *>(L.dst[b]);
        for (size_t v = tid; v < nv; v += nth) d[v] = __ldcs(s + v);
        const size_t tail = L.bytes[b] - 16 * nv;
        if (tid < tail) L.dst[b][16 * nv + tid] = L.src[b][16 * nv + tid];
    }
}

__global__ void store64_kernel(unsigned long long *addr, unsigned long long v, unsigned long long *stamp) {
    asm volatile("st.release.sys.global.b64 [%0], %1;" ::"l"(addr), "l"(v) : "memory");
    if (stamp) *stamp = globaltimer();   // (measurement: when the store became visible)
}

// ------------------------------------------------------------------------------------------
// Row-dot bodies: ATAX kernel 1 (tmp = A x), BICG kernel 2 (q = A p), GESUMMV.
// A work-group is lws consecutive rows; a task is R <= 8 of them, one warp per row.
// Canonical order: partial q (q = j % 128) accumulates A[i][j]*x[j] for ascending j; lane l
// owns partials 4l..4l+3, folds them ((p0+p1)+p2)+p3, then a xor-butterfly over lanes
// (offsets 16, 8, 4, 2, 1) -- host_bodies.cpp replays exactly this.
// ------------------------------------------------------------------------------------------
struct EmptySmem { int dummy; };

template <typename T, int NMAT>
struct RowDotBody {
    // 4 warps, one row each: 64 registers allow 8 CTAs (32 warps) per SM, so a 4096-row
    // launch (1024 tasks) is resident in a single wave with 2 KB of loads in flight per warp.
    // GESUMMV: 4 blocks of loads in flight at 72 registers = 7 CTAs per SM (1036 >= 1024 tasks,
    // still one wave at N = 4096; 0.74 vs 0.71 of HBM with 2 blocks, scripts/ubench_dots.cu).
    static constexpr int kThreads = 128;
#ifndef FCL_ROWDOT_MINB2
#define FCL_ROWDOT_MINB2 7
#endif
#ifndef FCL_ROWDOT_MINB1
#define FCL_ROWDOT_MINB1 8
#endif
    static constexpr int kMinBlocks = (NMAT == 2) ? FCL_ROWDOT_MINB2 : FCL_ROWDOT_MINB1;
    static constexpr bool kMasks = false;   // a task is part of one work-group
    static constexpr bool kLateClaim = false;
    static constexpr int kWarps = kThreads / 32;
    static constexpr int U = 4;   // 128-column blocks whose loads are issued together
    struct Params {
        const T *A; const T *B; const T *x; T *out0; T *out1;
        long long nrows, ncols, lws; int R; T alpha, beta; int vec4;
        int streamed;   // A/B rows arrive by H2D pieces during the kernel: loads through L2 only
    };
    typedef EmptySmem Smem;

    __device__ static long long key(const Params &p, long long t) { return (t * p.R) / p.lws; }
    template <bool CG>
    __device__ static typename V4<T>::type ldm4(const T *q) { return CG ? ld_cg4(q) : ld_stream4(q); }
    template <bool CG>
    __device__ static T ldm(const T *q) { return CG ? __ldcg(q) : *q; }

    __device__ static T warp_fold(T p0, T p1, T p2, T p3) {
        T v = op_add(op_add(op_add(p0, p1), p2), p3);
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) v = op_add(v, __shfl_xor_sync(0xffffffffu, v, off));
        return v;
    }

    __device__ static bool run(const Params &p, long long t, TaskCtx &tc, Smem &sm) {
        return p.streamed ? run_t<true>(p, t, tc, sm) : run_t<false>(p, t, tc, sm);
    }
    template <bool CG>
    __device__ static bool run_t(const Params &p, long long t, TaskCtx &, Smem &) {
        const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
        for (int r = warp; r < p.R; r += kWarps) {
            const long long i = t * p.R + r;
            if (i >= p.nrows) return false;
            const T *Ar = p.A + i * p.ncols;
            const T *Br = (NMAT == 2) ? p.B + i * p.ncols : nullptr;
            T a0 = 0, a1 = 0, a2 = 0, a3 = 0, b0 = 0, b1 = 0, b2 = 0, b3 = 0;
            const long long nfull = p.ncols / 128;
            long long k = 0;
            if (p.vec4) {
                // explicit pointer walk (no per-load index arithmetic, whatever the register
                // budget of the kernel the body is compiled into)
                const T *pa = Ar + 4 * lane, *pb = (NMAT == 2) ? Br + 4 * lane : nullptr, *px = p.x + 4 * lane;
                for (; k + U <= nfull; k += U, pa += U * 128, px += U * 128) {
                    typename V4<T>::type av[U], bv[U], xv[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        av[u] = ldm4<CG>(pa + u * 128);
                        if (NMAT == 2) bv[u] = ldm4<CG>(pb + u * 128);
                    }
                    if (NMAT == 2) pb += U * 128;
#pragma unroll
                    for (int u = 0; u < U; ++u) xv[u] = ld_cached4(px + u * 128);
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        a0 = op_fma(av[u].x, xv[u].x, a0); a1 = op_fma(av[u].y, xv[u].y, a1);
                        a2 = op_fma(av[u].z, xv[u].z, a2); a3 = op_fma(av[u].w, xv[u].w, a3);
                        if (NMAT == 2) {
                            b0 = op_fma(bv[u].x, xv[u].x, b0); b1 = op_fma(bv[u].y, xv[u].y, b1);
                            b2 = op_fma(bv[u].z, xv[u].z, b2); b3 = op_fma(bv[u].w, xv[u].w, b3);
                        }
                    }
                }
                for (; k < nfull; ++k) {
                    const long long j = k * 128 + 4 * lane;
                    typename V4<T>::type av = ldm4<CG>(Ar + j), xv = ld_cached4(p.x + j);
                    a0 = op_fma(av.x, xv.x, a0); a1 = op_fma(av.y, xv.y, a1);
                    a2 = op_fma(av.z, xv.z, a2); a3 = op_fma(av.w, xv.w, a3);
                    if (NMAT == 2) {
                        typename V4<T>::type bv = ldm4<CG>(Br + j);
                        b0 = op_fma(bv.x, xv.x, b0); b1 = op_fma(bv.y, xv.y, b1);
                        b2 = op_fma(bv.z, xv.z, b2); b3 = op_fma(bv.w, xv.w, b3);
                    }
                }
            }
            // scalar path (unaligned rows) and the ragged tail, same partition order
            for (; k * 128 < p.ncols; ++k) {
                const long long j = k * 128 + 4 * lane;
#define FCL_ROWDOT_TAIL(C, AC, BC)                                             \
                if (j + C < p.ncols) {                                         \
                    const T xv = p.x[j + C];                                   \
                    AC = op_fma(ldm<CG>(Ar + j + C), xv, AC);                  \
                    if (NMAT == 2) BC = op_fma(ldm<CG>(Br + j + C), xv, BC);   \
                }
                FCL_ROWDOT_TAIL(0, a0, b0)
                FCL_ROWDOT_TAIL(1, a1, b1)
                FCL_ROWDOT_TAIL(2, a2, b2)
                FCL_ROWDOT_TAIL(3, a3, b3)
#undef FCL_ROWDOT_TAIL
            }
            const T va = warp_fold(a0, a1, a2, a3);
            if (NMAT == 1) {
                if (lane == 0) p.out0[i] = va;
            } else {
                const T vb = warp_fold(b0, b1, b2, b3);
                if (lane == 0) {
                    p.out0[i] = va;                                              // tmp[i]
                    p.out1[i] = op_add(op_mul(p.alpha, va), op_mul(p.beta, vb)); // y[i]
                }
            }
        }
        return false;
    }
};

// ------------------------------------------------------------------------------------------
// Column-dot bodies: ATAX kernel 2 (y = A^T tmp), BICG kernel 1 (s = A^T r), CORR mean / std.
// A work-group is lws consecutive columns; a task is CB <= 32 of them, all rows.
// Canonical order: partial q (q = i % 32) accumulates rows i = q, q+32, ... ascending; the 32
// partials are then added sequentially q = 0..31.
// Thread t owns partial q = t / 8 of the 4 columns 4*(t % 8) .. +3 of the task, so a warp
// reads 4 rows x 128 contiguous bytes per load and each thread keeps U = 16 row loads (16 B
// each) in flight: 256 threads, 16 KB in flight per CTA (the 1024-thread scalar layout kept
// only 4 B per thread in flight and reached 0.50 of HBM at N = 4096; this one 0.60,
// scripts/ubench_dots.cu).
// ------------------------------------------------------------------------------------------
enum { COL_DOT = 0, COL_SUM = 1, COL_SQDEV = 2 };

template <typename T, int MODE>
struct ColDotBody {
    static constexpr int kThreads = 256;
#ifndef FCL_COLDOT_MINB
#define FCL_COLDOT_MINB 2
#endif
    static constexpr int kMinBlocks = FCL_COLDOT_MINB;
    static constexpr bool kMasks = false;   // a task is part of one work-group
    static constexpr bool kLateClaim = false;
    static constexpr int U = 16;
    struct Params {
        const T *A; const T *v; const T *mean; T *out;
        long long nrows, ncols, lws; int CB; float nf, eps; int vec4;
    };
    struct Smem { T red[32][33]; };

    __device__ static long long key(const Params &p, long long t) { return (t * p.CB) / p.lws; }

    __device__ static T term(const Params &p, T a, T vi, T mj, T acc) {
        if (MODE == COL_DOT) return op_fma(a, vi, acc);
        if (MODE == COL_SUM) return op_add(acc, a);
        const T c = op_add(a, -mj);   // a - mean (exact negation, then one rounding)
        return op_fma(c, c, acc);
    }

    __device__ static bool run(const Params &p, long long t, TaskCtx &, Smem &sm) {
        const int quad = threadIdx.x & 7, q = threadIdx.x >> 3;
        const long long j0 = t * p.CB + 4 * quad;          // first of this thread's 4 columns
        // columns of this thread inside the task and the matrix (CB < 4 only for tiny lws)
        const int ncol = (int)max(0ll, min(min(4ll, (long long)p.CB - 4 * quad), p.ncols - j0));
        T c0 = 0, c1 = 0, c2 = 0, c3 = 0;
        if (ncol > 0) {
            T m[4] = {0, 0, 0, 0};
            if (MODE == COL_SQDEV)
                for (int c = 0; c < ncol; ++c) m[c] = p.mean[j0 + c];
            const long long stride = 32 * p.ncols;
            const T *pc = p.A + j0 + (long long)q * p.ncols;   // explicit pointer walk down the rows
            long long i = q;
            if (p.vec4 && ncol == 4) {
                for (; i + (U - 1) * 32 < p.nrows; i += U * 32) {
                    typename V4<T>::type a[U];
                    T vi[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) { a[u] = ld_stream4(pc); pc += stride; }
#pragma unroll
                    for (int u = 0; u < U; ++u) vi[u] = (MODE == COL_DOT) ? __ldg(p.v + i + 32 * u) : T(0);
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        c0 = term(p, a[u].x, vi[u], m[0], c0); c1 = term(p, a[u].y, vi[u], m[1], c1);
                        c2 = term(p, a[u].z, vi[u], m[2], c2); c3 = term(p, a[u].w, vi[u], m[3], c3);
                    }
                }
                for (; i < p.nrows; i += 32, pc += stride) {
                    const typename V4<T>::type a = ld_stream4(pc);
                    const T vi = (MODE == COL_DOT) ? __ldg(p.v + i) : T(0);
                    c0 = term(p, a.x, vi, m[0], c0); c1 = term(p, a.y, vi, m[1], c1);
                    c2 = term(p, a.z, vi, m[2], c2); c3 = term(p, a.w, vi, m[3], c3);
                }
            } else {   // unaligned rows or the ragged last columns: scalar loads, same order
                for (; i < p.nrows; i += 32, pc += stride) {
                    const T vi = (MODE == COL_DOT) ? p.v[i] : T(0);
                    c0 = term(p, __ldcs(pc), vi, m[0], c0);
                    if (ncol > 1) c1 = term(p, __ldcs(pc + 1), vi, m[1], c1);
                    if (ncol > 2) c2 = term(p, __ldcs(pc + 2), vi, m[2], c2);
                    if (ncol > 3) c3 = term(p, __ldcs(pc + 3), vi, m[3], c3);
                }
            }
        }
        sm.red[q][4 * quad + 0] = c0; sm.red[q][4 * quad + 1] = c1;
        sm.red[q][4 * quad + 2] = c2; sm.red[q][4 * quad + 3] = c3;
        __syncthreads();
        const long long j = t * p.CB + threadIdx.x;
        if (threadIdx.x < p.CB && j < p.ncols) {
            T tot = sm.red[0][threadIdx.x];
#pragma unroll 8
            for (int qq = 1; qq < 32; ++qq) tot = op_add(tot, sm.red[qq][threadIdx.x]);
            T o;
            if (MODE == COL_DOT) {
                o = tot;
            } else if (MODE == COL_SUM) {
                o = (T)__fdiv_rn((float)tot, p.nf);
            } else {
                float s = __fsqrt_rn(__fdiv_rn((float)tot, p.nf));
                o = (T)((s <= p.eps) ? 1.0f : s);
            }
            p.out[j] = o;
        }
        __syncthreads();
        return false;
    }
};

// ------------------------------------------------------------------------------------------
// 2-D tiled bodies over a row-major output: a task is a tile of th x tw work-groups, tiles
// enumerated row-major so that keys ascend.  key = gx0 + ngx * gy0.
// ------------------------------------------------------------------------------------------
struct Tile2D {
    long long nrows, ncols;  // output extent
    long long ngx, lws0, lws1;
    int tw, th;              // tile size in work-groups
    long long ntx;           // tiles per tile-row
    // task t -> (tile column, tile row).  FCL_TASK_DIV32=1 divides in 32 bits (task ids are below
    // the flattened work-group count, < 2^32, checked at launch) instead of calling the 64-bit
    // division subroutine -- measured: the 2DCONV dispatcher then runs at 0.44 instead of 0.78 of
    // the copy peak, the plain grid unchanged (profiles/r02_ab_task_div32.txt); off.
#ifndef FCL_TASK_DIV32
#define FCL_TASK_DIV32 0
#endif
    __device__ __host__ void split(long long t, long long &tx, long long &ty) const {
        if (FCL_TASK_DIV32) {
            const unsigned int ut = (unsigned int)t, un = (unsigned int)ntx;
            tx = (long long)(ut % un);
            ty = (long long)(ut / un);
        } else {
            tx = t % ntx;
            ty = t / ntx;
        }
    }
    __device__ __host__ long long key(long long t) const {
        long long tx, ty;
        split(t, tx, ty);
        return tx * tw + ngx * (ty * th);
    }
    // work-group of output element (i, j), Fig 5 flattening
    // (32-bit arithmetic: extents and flattened ids are < 2^32, checked at launch)
    __device__ unsigned int fgid(long long i, long long j) const {
        return (unsigned int)j / (unsigned int)lws0 + (unsigned int)ngx * ((unsigned int)i / (unsigned int)lws1);
    }
    // is output (i, j) below the mask watermark (0xFFFFFFFF: no mask)?
    __device__ bool keep(unsigned int wm, long long i, long long j) const {
        return wm == 0xFFFFFFFFu || fgid(i, j) < wm;
    }
};

// CORR reduce (in place): d[i][j] = (d[i][j] - mean[j]) / (sqrt(n) * std[j]).
struct CorrReduceBody {
    static constexpr int kThreads = 256;
    static constexpr int kMinBlocks = 4;
    static constexpr bool kMasks = true;   // a task may span work-groups: stores masked by TaskCtx::wmask
    static constexpr bool kLateClaim = false;
    struct Params { float *data; const float *mean; const float *std_; Tile2D tl; float sqrtn; };
    typedef EmptySmem Smem;
    __device__ static long long key(const Params &p, long long t) { return p.tl.key(t); }
    __device__ static bool run(const Params &p, long long t, TaskCtx &tc, Smem &) {
        const Tile2D &tl = p.tl;
        long long tx, ty;
        tl.split(t, tx, ty);
        const long long c0 = tx * tl.tw * tl.lws0, r0 = ty * tl.th * tl.lws1;
        const int tcols = (int)(tl.tw * tl.lws0), trows = (int)(tl.th * tl.lws1);
        const unsigned int wm = tc.wmask;
        for (int e = threadIdx.x; e < tcols * trows; e += kThreads) {
            const long long i = r0 + e / tcols, j = c0 + e % tcols;
            if (i < tl.nrows && j < tl.ncols && tl.keep(wm, i, j)) {
                float *q = p.data + i * tl.ncols + j;
                const float den = __fmul_rn(p.sqrtn, p.std_[j]);
                *q = __fdiv_rn(__fadd_rn(*q, -p.mean[j]), den);
            }
        }
        return false;
    }
};

// 2DCONV (PolyBench/GPU): interior B[i][j] = sum of 9 taps, canonical PolyBench term order
// (column j-1 rows i-1..i+1, then column j, then column j+1): first tap a product, the other
// eight fused multiply-adds.  Border untouched.
// Thread mapping (vector path): a tile is 256 columns x 32 rows; a thread owns 4 consecutive
// columns (float4) of 8 rows; its 10 input rows are loaded up front (memory-level parallelism),
// the left/right halo columns come from the neighbouring lanes by shuffle (edge lanes load
// them), and each output row is one 16-byte store (masked at the image border).
// The 2DCONV task tile: FCL_CONV_TILE_COLS x FCL_CONV_TILE_ROWS outputs, one warp per 128 x 8
// block.  Default 128 x 8 -- one warp per CTA: the body has no barrier, so a warp-sized CTA lets
// the persistent dispatcher hand out tasks without a CTA barrier between them (256 x 32 tiles
// with 8 warps spent 1.25 barrier stalls per issue waiting for the slowest warp of each task).
#ifndef FCL_CONV_TILE_COLS
#define FCL_CONV_TILE_COLS 128
#endif
#ifndef FCL_CONV_TILE_ROWS
#define FCL_CONV_TILE_ROWS 8
#endif
template <typename T>
struct Conv2DBody {
    static constexpr int kWarpsX = FCL_CONV_TILE_COLS / 128;   // 128-column warp blocks across a tile
    static constexpr int kThreads = 32 * kWarpsX * (FCL_CONV_TILE_ROWS / 8);
    // 10 x 16 B of loads in flight per thread needs the registers: 2 CTAs of 8 warps, or 16 of one
    // plain grid: 20 warps per SM at 96 registers (0.337 -> 0.316 ms at 16384^2); the dispatcher
    // keeps 16 (its loop state does not fit 96 registers without spilling: 0.74 ms with the
    // 256 x 32 tiles; with 128 x 8 tiles 17-20 warps spill 38-70 bytes and run within 2 %,
    // profiles/r02_ab_conv2d_coop_warps.txt)
    static constexpr int kMinBlocks = 20 * 32 / kThreads;
#ifndef FCL_CONV_COOP_WARPS
#define FCL_CONV_COOP_WARPS 16
#endif
    static constexpr int kMinBlocksCoop = FCL_CONV_COOP_WARPS * 32 / kThreads;
    static constexpr bool kMasks = true;   // a task may span work-groups: stores masked by TaskCtx::wmask
    static constexpr bool kLateClaim = false;
    struct Params { const T *A; T *B; Tile2D tl; T c[9]; int vec4; };   // c[a*3+b]: row offset a-1, col offset b-1
    typedef EmptySmem Smem;
    __device__ static long long key(const Params &p, long long t) { return p.tl.key(t); }

    __device__ static T tap9(const Params &p, T l0, T l1, T l2, T m0, T m1, T m2, T r0, T r1, T r2) {
        T s = op_mul(p.c[0], l0);
        s = op_fma(p.c[3], l1, s);
        s = op_fma(p.c[6], l2, s);
        s = op_fma(p.c[1], m0, s);
        s = op_fma(p.c[4], m1, s);
        s = op_fma(p.c[7], m2, s);
        s = op_fma(p.c[2], r0, s);
        s = op_fma(p.c[5], r1, s);
        s = op_fma(p.c[8], r2, s);
        return s;
    }

    // A warp's 128 x 8 block away from every border (input rows ib-1 .. ib+8 and columns
    // j-1 .. j+4 exist for all lanes, no output on the border): no per-row or per-column
    // checks, one pointer walking the rows, and the halo columns loaded by the two edge lanes
    // for every row up front, so that no shuffle sits under a divergent branch.
    __device__ static void run_interior(const Params &p, long long ib, long long j, int lane, unsigned int wm) {
        typedef typename V4<T>::type T4;
        const long long nj = p.tl.ncols;
        const T *src = p.A + (ib - 1) * nj + j;
        const bool l0 = lane == 0, l31 = lane == 31;
        const T *edge = src + (l0 ? -1 : 4);
        T4 v[10];
        T lh[10], rh[10];
#pragma unroll
        for (int q = 0; q < 10; ++q) v[q] = ld_cached4(src + q * nj);
#pragma unroll
        for (int q = 0; q < 10; ++q) lh[q] = (l0 || l31) ? __ldg(edge + q * nj) : T(0);
#pragma unroll
        for (int q = 0; q < 10; ++q) {
            const T up = __shfl_up_sync(0xffffffffu, v[q].w, 1);
            const T dn = __shfl_down_sync(0xffffffffu, v[q].x, 1);
            rh[q] = l31 ? lh[q] : dn;
            lh[q] = l0 ? lh[q] : up;
        }
        T *dst = p.B + ib * nj + j;
#pragma unroll
        for (int q = 1; q <= 8; ++q) {
            T4 o;
            o.x = tap9(p, lh[q - 1], lh[q], lh[q + 1], v[q - 1].x, v[q].x, v[q + 1].x, v[q - 1].y, v[q].y, v[q + 1].y);
            o.y = tap9(p, v[q - 1].x, v[q].x, v[q + 1].x, v[q - 1].y, v[q].y, v[q + 1].y, v[q - 1].z, v[q].z, v[q + 1].z);
            o.z = tap9(p, v[q - 1].y, v[q].y, v[q + 1].y, v[q - 1].z, v[q].z, v[q + 1].z, v[q - 1].w, v[q].w, v[q + 1].w);
            o.w = tap9(p, v[q - 1].z, v[q].z, v[q + 1].z, v[q - 1].w, v[q].w, v[q + 1].w, rh[q - 1], rh[q], rh[q + 1]);
            if (wm == 0xFFFFFFFFu || p.tl.keep(wm, ib + q - 1, j + 3)) {   // (fgid grows with j)
                __stcs(reinterpret_cast<T4 *>(dst + (q - 1) * nj), o);
            } else {
                T *d = dst + (q - 1) * nj;
                if (p.tl.keep(wm, ib + q - 1, j)) __stcs(d, o.x);
                if (p.tl.keep(wm, ib + q - 1, j + 1)) __stcs(d + 1, o.y);
                if (p.tl.keep(wm, ib + q - 1, j + 2)) __stcs(d + 2, o.z);
            }
        }
    }

    __device__ static bool run(const Params &p, long long t, TaskCtx &tc, Smem &) {
        const Tile2D &tl = p.tl;
        long long tx, ty;
        tl.split(t, tx, ty);
        const long long c0 = tx * tl.tw * tl.lws0, r0 = ty * tl.th * tl.lws1;
        const int tcols = (int)(tl.tw * tl.lws0), trows = (int)(tl.th * tl.lws1);
        const long long ni = tl.nrows, nj = tl.ncols;
        const unsigned int wm = tc.wmask;
        if (p.vec4 && tcols == FCL_CONV_TILE_COLS && trows == FCL_CONV_TILE_ROWS) {
            const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
            const int cg = warp % kWarpsX;           // which 128-column block of the tile
            const int rg = warp / kWarpsX;           // which 8-row group
            const long long j = c0 + cg * 128 + lane * 4;   // first of this thread's 4 columns
            const long long ib = r0 + rg * 8;        // first output row of the group
            const long long wj0 = c0 + cg * 128;     // the warp's first column (warp-uniform test)
            if (ib >= 1 && ib + 8 <= ni - 1 && wj0 >= 1 && wj0 + 128 <= nj - 1) {
                run_interior(p, ib, j, lane, wm);
                return false;
            }
            if (ib >= ni) return false;
            const bool colok = j < nj;               // nj % 4 == 0 on this path
            typename V4<T>::type v[10];
            T lh[10], rh[10];
#pragma unroll
            for (int q = 0; q < 10; ++q) {
                const long long r = ib - 1 + q;
                if (colok && r >= 0 && r < ni) v[q] = ld_cached4(p.A + r * nj + j);
                else { v[q].x = v[q].y = v[q].z = v[q].w = T(0); }
            }
#pragma unroll
            for (int q = 0; q < 10; ++q) {
                T left = __shfl_up_sync(0xffffffffu, v[q].w, 1);
                T right = __shfl_down_sync(0xffffffffu, v[q].x, 1);
                const long long r = ib - 1 + q;
                if (lane == 0) left = (colok && j >= 1 && r >= 0 && r < ni) ? __ldg(p.A + r * nj + j - 1) : T(0);
                if (lane == 31) right = (j + 4 < nj && r >= 0 && r < ni) ? __ldg(p.A + r * nj + j + 4) : T(0);
                lh[q] = left; rh[q] = right;
            }
            if (!colok) return false;
#pragma unroll
            for (int q = 1; q <= 8; ++q) {
                const long long i = ib + q - 1;
                if (i < 1 || i >= ni - 1) continue;
                typename V4<T>::type o;
                o.x = tap9(p, lh[q - 1], lh[q], lh[q + 1], v[q - 1].x, v[q].x, v[q + 1].x, v[q - 1].y, v[q].y, v[q + 1].y);
                o.y = tap9(p, v[q - 1].x, v[q].x, v[q + 1].x, v[q - 1].y, v[q].y, v[q + 1].y, v[q - 1].z, v[q].z, v[q + 1].z);
                o.z = tap9(p, v[q - 1].y, v[q].y, v[q + 1].y, v[q - 1].z, v[q].z, v[q + 1].z, v[q - 1].w, v[q].w, v[q + 1].w);
                o.w = tap9(p, v[q - 1].z, v[q].z, v[q + 1].z, v[q - 1].w, v[q].w, v[q + 1].w, rh[q - 1], rh[q], rh[q + 1]);
                T *dst = p.B + i * nj + j;
                if (j >= 1 && j + 4 <= nj - 1 && tl.keep(wm, i, j + 3)) {
                    __stcs(reinterpret_cast<typename V4<T>::type *>(dst), o);
                } else {   // a border column inside this vector stays untouched (and masked ones)
                    if (j >= 1 && j < nj - 1 && tl.keep(wm, i, j)) __stcs(dst, o.x);
                    if (j + 1 >= 1 && j + 1 < nj - 1 && tl.keep(wm, i, j + 1)) __stcs(dst + 1, o.y);
                    if (j + 2 >= 1 && j + 2 < nj - 1 && tl.keep(wm, i, j + 2)) __stcs(dst + 2, o.z);
                    if (j + 3 >= 1 && j + 3 < nj - 1 && tl.keep(wm, i, j + 3)) __stcs(dst + 3, o.w);
                }
            }
            return false;
        }
        // generic path (any tile shape / alignment): one column per thread, sliding window
        for (int cc = threadIdx.x; cc < tcols; cc += kThreads) {
            const long long j = c0 + cc;
            if (j < 1 || j >= nj - 1) continue;
            long long i = r0 < 1 ? 1 : r0;
            const long long iend = (r0 + trows < ni - 1) ? r0 + trows : ni - 1;
            if (i >= iend) continue;
            const T *a = p.A + j;
            T w0[3], w1[3], w2[3];
#pragma unroll
            for (int b = 0; b < 3; ++b) { w0[b] = __ldg(a + (i - 1) * nj + b - 1); w1[b] = __ldg(a + i * nj + b - 1); }
            for (; i < iend; ++i) {
#pragma unroll
                for (int b = 0; b < 3; ++b) w2[b] = __ldg(a + (i + 1) * nj + b - 1);
                if (tl.keep(wm, i, j))
                    __stcs(p.B + i * nj + j, tap9(p, w0[0], w1[0], w2[0], w0[1], w1[1], w2[1], w0[2], w1[2], w2[2]));
#pragma unroll
                for (int b = 0; b < 3; ++b) { w0[b] = w1[b]; w1[b] = w2[b]; }
            }
        }
        return false;
    }
};
template <typename T> struct CoopMinBlocks<Conv2DBody<T>> { static constexpr int value = Conv2DBody<T>::kMinBlocksCoop; };

// ------------------------------------------------------------------------------------------
// GEMM-like bodies on CUDA cores (fp32 FFMA / int32 IMAD; no tensor cores: fp32 parity, see
// DESIGN.md §6): SYRK, SYR2K and CORR's symmat.  Output tile 128 x 128, 256 threads, 8 x 8
// outputs per thread, k-tile 16, double-buffered shared memory plus register double-buffered
// fragments.  Every output accumulates its k-chain in ascending k with one fma per term.
// SYR2K is one GEMM over the interleaved K' = 2M: k' = 2k holds (A_i[k], B_j[k]) and
// k' = 2k+1 holds (B_i[k], A_j[k]) -- exactly the canonical "A_i*B_j then B_i*A_j" per-k order.
// ------------------------------------------------------------------------------------------
enum { G_SYRK = 0, G_SYR2K = 1, G_CORR = 2 };
constexpr int GBM = 128, GBK = 16, GPAD = 4;

// TN: outputs per thread along the tile's columns.  TN = 8: 256 threads, 8 x 8 outputs each,
// two CTAs per SM.  TN = 4: 512 threads, 8 x 4 each, one CTA per SM -- for the SYRK / SYR2K
// upper-triangle grids (136 tiles at N = 2048, one per SM), where 16 warps hide the k'-tile
// loads that 8 cannot.
//
// SYR2K's canonical per-k order is symmetric: output (i, j) with i <= j
// accumulates A_i[k]*B_j[k] then B_i[k]*A_j[k]; an output below the diagonal takes its mirror's
// chain, B_i[k]*A_j[k] then A_i[k]*B_j[k].  So acc(i, j) == acc(j, i) bit for bit, and like SYRK
// the kernel can run the upper-triangle tiles only and write each one's mirror block; a tile
// below the diagonal (slices) is the same GEMM with A and B exchanged, and a diagonal tile
// stores its upper half and that half's mirror.
template <typename T, int OP, int TN = 8>
struct GemmBody {
    static_assert(TN == 8 || TN == 4, "TN = 4: the upper-triangle grids, CORR symmat");
    static constexpr int kThreads = TN == 8 ? 256 : 512;
    // k'-tile (k' rows per barrier) of the upper-triangle grids.  SYR2K: 64 (its 135 KB of stages
    // in dynamic shared memory, one CTA per SM), 0.449 -> 0.415 ms at 2048 against 32 with the FFMA2
    // loop and swizzled stages; SYRK keeps 16 (64: 0.229, 32: 0.215, 16: 0.216 ms)
    // (profiles/r02_ab_gemm_gbk64.txt; before FFMA2: profiles/r02_ab_gemm_gbk.txt).
#ifndef FCL_GEMM_GBK_SYR2K
#define FCL_GEMM_GBK_SYR2K 64
#endif
#ifndef FCL_GEMM_GBK_SYRK
#define FCL_GEMM_GBK_SYRK 16
#endif
    static constexpr int GBK = TN != 4 ? ::fcl::GBK
                               : (OP == G_SYR2K ? FCL_GEMM_GBK_SYR2K : OP == G_SYRK ? FCL_GEMM_GBK_SYRK : ::fcl::GBK);
#ifndef FCL_GEMM_MINB
#define FCL_GEMM_MINB 2
#endif
    static constexpr int kMinBlocks = TN == 8 ? FCL_GEMM_MINB : 1;
    static constexpr int TXN = GBM / TN;                 // threads along the columns
    static constexpr int NB = TN / 4;                    // float4 column groups per thread
    static constexpr int LD = GBM * GBK / kThreads;      // elements of each operand a thread loads per k'-tile
    static_assert(LD % 4 == 0 && GBK % LD == 0, "gload / sstore: whole float4 loads, whole k-row groups");
    static constexpr bool kMasks = true;   // a task may span work-groups: stores masked by TaskCtx::wmask
    static constexpr bool kLateClaim = true;   // tasks of ~0.1-1 ms: an exposed claim costs nothing
    typedef typename V4<T>::type T4;
    struct Params {
        const T *A; const T *B; T *C;
        long long n;      // output is n x n (CORR: M x M)
        long long m;      // contraction length (CORR: number of data rows N)
        long long ld;     // row length of the operand matrix (SYRK/SYR2K: m; CORR: n)
        T alpha, beta;
        long long ntile;  // tiles per dimension
        long long ngx, lws0, lws1, lws;  // work-group geometry for keys
        int vec4;
        int sym;          // SYRK: upper-triangle tiles, each also writes its mirror (KArgs::sym)
    };
    // CORR's operand is K-major already (data[k][col]): interior tiles stream it with cp.async
    // straight into shared memory, NSA stages of GBKA k-rows (NSA - 1 tiles in flight, no register
    // staging), sharing the bytes of the register-staged path's stages.  16 k-rows x 2 stages:
    // half the barriers of 8 x 4 (1.448 against 1.565 ms at 4096, scripts/ab_corr.sh; 8 x 3,
    // 8 x 5 and unpadded rows no better; in dynamic shared memory 32 x 2 ran 1.444, 16 x 3 1.516,
    // 32 x 3 1.481, 64 x 2 1.665 ms -- not worth leaving static shared memory).
#ifndef FCL_CORR_GBKA
#define FCL_CORR_GBKA 16
#endif
#ifndef FCL_CORR_NSA
#define FCL_CORR_NSA 2
#endif
#ifndef FCL_CORR_APAD
#define FCL_CORR_APAD 4
#endif
    static constexpr int GBKA = FCL_CORR_GBKA, NSA = FCL_CORR_NSA, APAD = FCL_CORR_APAD;
    struct SmemBase { T s[2][2][GBK][GBM + GPAD]; };   // [stage][A|B][k'][m]
    struct SmemCorr {
        union {
            T s[2][2][GBK][GBM + GPAD];
            T a[NSA][2][GBKA][GBM + APAD];   // mainloop_async's stages
        };
    };
    typedef typename std::conditional<OP == G_CORR && TN == 8, SmemCorr, SmemBase>::type Smem;
    static constexpr bool kDynSmem = sizeof(Smem) > 40960;

    __device__ static void tile_of(const Params &p, long long t, long long &bi, long long &bj) {
        if (OP == G_CORR || p.sym) {  // upper triangle, row-major over (b1 <= b2)
            long long b1 = 0, rem = t;
            while (rem >= p.ntile - b1) { rem -= p.ntile - b1; ++b1; }
            bi = b1; bj = b1 + rem;
        } else {
            bi = t / p.ntile; bj = t % p.ntile;
        }
    }
    __device__ static long long key(const Params &p, long long t) {
        long long bi, bj;
        tile_of(p, t, bi, bj);
        if (OP == G_CORR) return (bi * GBM) / p.lws;
        return (bj * GBM) / p.lws0 + p.ngx * ((bi * GBM) / p.lws1);
    }

    // 4 consecutive k of row `row` of X (K-contiguous operands), zero outside the matrix
    __device__ static void load4_k(const Params &p, const T *X, long long row, long long k, T *r) {
        if (row < p.n && p.vec4 && k + 3 < p.m) {
            const T4 v = ld_cached4(X + row * p.ld + k);
            r[0] = v.x; r[1] = v.y; r[2] = v.z; r[3] = v.w;
        } else {
#pragma unroll
            for (int q = 0; q < 4; ++q) r[q] = (row < p.n && k + q < p.m) ? X[row * p.ld + k + q] : T(0);
        }
    }
    // 4 consecutive columns of data row k (CORR: MN-contiguous operand)
    __device__ static void load4_row(const Params &p, const T *X, long long k, long long col, T *r) {
        if (k < p.m && p.vec4 && col + 3 < p.n) {
            const T4 v = ld_cached4(X + k * p.ld + col);
            r[0] = v.x; r[1] = v.y; r[2] = v.z; r[3] = v.w;
        } else {
#pragma unroll
            for (int q = 0; q < 4; ++q) r[q] = (k < p.m && col + q < p.n) ? X[k * p.ld + col + q] : T(0);
        }
    }

    // 4 consecutive elements, no bounds checks (interior tiles: every index in range, vec4)
    __device__ static void ld4(const T *q, T *r) {
        const T4 v = ld_cached4(q);
        r[0] = v.x; r[1] = v.y; r[2] = v.z; r[3] = v.w;
    }
    // KP consecutive k of row `row` of X (SYR2K operands): IN without bounds checks
    template <bool IN, int KP>
    __device__ static void loadk(const Params &p, const T *X, long long row, long long k, T *r) {
        if (KP % 4 == 0) {   // (k a multiple of KP: 16-byte aligned when IN)
#pragma unroll
            for (int u = 0; u < KP / 4; ++u) {
                if (IN) ld4(X + row * p.ld + k + 4 * u, r + 4 * u);
                else load4_k(p, X, row, k + 4 * u, r + 4 * u);
            }
        } else if (IN) {   // (k even, ld % 4 == 0: 8-byte aligned)
            typedef typename std::conditional<sizeof(T) == 4 && std::is_same<T, float>::value, float2, int2>::type T2;
            const T2 v = __ldg(reinterpret_cast<const T2 *>(X + row * p.ld + k));
            r[0] = v.x; r[1] = v.y;
        } else {
#pragma unroll
            for (int q = 0; q < KP; ++q) r[q] = (row < p.n && k + q < p.m) ? X[row * p.ld + k + q] : T(0);
        }
    }
    // One k'-tile into registers: 8 elements of each operand tile per thread.  IN: the tile and
    // the k'-range are interior (no bounds checks).
    template <bool IN>
    __device__ static void gload(const Params &p, long long i0, long long j0, long long kt, T ra[LD], T rb[LD], bool sw) {
        const int tid = threadIdx.x;
        if (OP == G_SYR2K) {   // this k'-tile covers k in [kt*GBK/2, (kt+1)*GBK/2), KP of them per thread
            constexpr int KP = LD / 2, TPR = (GBK / 2) / KP;
            const int row = tid / TPR;
            const long long k = kt * (GBK / 2) + (tid % TPR) * KP;
            const T *PA = sw ? p.B : p.A, *PB = sw ? p.A : p.B;   // sw: a tile below the diagonal
            // loaded straight into the staging registers in memory order (the interleave to
            // k' = 2k, 2k + 1 happens in sstore: a register shuffle here would wait for the load)
            loadk<IN, KP>(p, PA, i0 + row, k, ra); loadk<IN, KP>(p, PB, i0 + row, k, ra + KP);   // A_i[k..], B_i[k..]
            loadk<IN, KP>(p, PB, j0 + row, k, rb); loadk<IN, KP>(p, PA, j0 + row, k, rb + KP);   // B_j[k..], A_j[k..]
            return;
        }
        if (IN) {
            if (OP == G_CORR) {
                const int kk = tid / (GBM / LD), c = (tid % (GBM / LD)) * LD;
                const T *row = p.A + (kt * GBK + kk) * p.ld;
                ld4(row + i0 + c, ra); ld4(row + j0 + c, rb);
                if (LD == 8) { ld4(row + i0 + c + 4, ra + 4); ld4(row + j0 + c + 4, rb + 4); }
            } else if (OP == G_SYRK) {
                const int row = tid / (GBK / LD);
                const long long k = kt * GBK + (tid % (GBK / LD)) * LD;
                const T *xa = p.A + (i0 + row) * p.ld + k, *xb = p.A + (j0 + row) * p.ld + k;
#pragma unroll
                for (int u = 0; u < LD / 4; ++u) { ld4(xa + 4 * u, ra + 4 * u); ld4(xb + 4 * u, rb + 4 * u); }
            }
            return;
        }
        if (OP == G_CORR) {
            const int kk = tid / (GBM / LD), c = (tid % (GBM / LD)) * LD;
            const long long k = kt * GBK + kk;
            load4_row(p, p.A, k, i0 + c, ra); load4_row(p, p.A, k, j0 + c, rb);
            if (LD == 8) { load4_row(p, p.A, k, i0 + c + 4, ra + 4); load4_row(p, p.A, k, j0 + c + 4, rb + 4); }
        } else {   // SYRK
            const int row = tid / (GBK / LD);
            const long long k = kt * GBK + (tid % (GBK / LD)) * LD;
#pragma unroll
            for (int u = 0; u < LD / 4; ++u) {
                load4_k(p, p.A, i0 + row, k + 4 * u, ra + 4 * u); load4_k(p, p.A, j0 + row, k + 4 * u, rb + 4 * u);
            }
        }
    }
    __device__ static T4 mk4(T a, T b, T c, T d) { T4 v; v.x = a; v.y = b; v.z = c; v.w = d; return v; }
    // Shared-memory column swizzle of the K-major stages (SYRK / SYR2K): sstore transposes, a warp
    // writing RW = 32 / G consecutive rows at G k-offsets LD apart -- which, with rows of GBM + GPAD
    // = 132 floats (4 banks per k), fall on the same banks (2- to 4-way conflicts; ncu r02h: 13.4 M
    // for SYR2K 2048).  Column c of k-row k lives at c ^ swz(k): each k-group moves to its own RW
    // banks, and the xor (a multiple of 4 below 32) keeps every float4 of frag() contiguous.
#ifndef FCL_GEMM_SWIZZLE
#define FCL_GEMM_SWIZZLE 1
#endif
    static constexpr int SG = GBK / LD;   // threads per k-row group in sstore
    __device__ static int swz(int k) {
        return (FCL_GEMM_SWIZZLE && OP != G_CORR) ? ((k / LD) % SG) * (32 / SG) : 0;
    }
    __device__ static void sstore(Smem &sm, int st, const T ra[LD], const T rb[LD]) {
        const int tid = threadIdx.x;
        if (OP == G_CORR) {
            const int kk = tid / (GBM / LD), c = (tid % (GBM / LD)) * LD;
            *reinterpret_cast<T4 *>(&sm.s[st][0][kk][c]) = mk4(ra[0], ra[1], ra[2], ra[3]);
            *reinterpret_cast<T4 *>(&sm.s[st][1][kk][c]) = mk4(rb[0], rb[1], rb[2], rb[3]);
            if (LD == 8) {
                *reinterpret_cast<T4 *>(&sm.s[st][0][kk][c + 4]) = mk4(ra[4], ra[5], ra[6], ra[7]);
                *reinterpret_cast<T4 *>(&sm.s[st][1][kk][c + 4]) = mk4(rb[4], rb[5], rb[6], rb[7]);
            }
        } else if (OP == G_SYR2K) {   // ra = [A_i k.., B_i k..] -> k' = 2q: A_i[k+q], 2q + 1: B_i[k+q]
            constexpr int KP = LD / 2;
            const int row = tid / (GBK / LD), kq = (tid % (GBK / LD)) * LD;
#pragma unroll
            for (int q = 0; q < KP; ++q) {   // (k' = kq .. kq + LD - 1: one swizzle for the thread)
                const int c = row ^ swz(kq);
                sm.s[st][0][kq + 2 * q][c] = ra[q]; sm.s[st][0][kq + 2 * q + 1][c] = ra[KP + q];
                sm.s[st][1][kq + 2 * q][c] = rb[q]; sm.s[st][1][kq + 2 * q + 1][c] = rb[KP + q];
            }
        } else {
            const int row = tid / (GBK / LD), kq = (tid % (GBK / LD)) * LD;
            const int c = row ^ swz(kq);
#pragma unroll
            for (int q = 0; q < LD; ++q) { sm.s[st][0][kq + q][c] = ra[q]; sm.s[st][1][kq + q][c] = rb[q]; }
        }
    }
    __device__ static void frag(const Smem &sm, int st, int kk, int tx, int ty, T a[8], T b[TN]) {
        const int x = swz(kk);
        const T4 a0 = *reinterpret_cast<const T4 *>(&sm.s[st][0][kk][(ty * 4) ^ x]);
        const T4 a1 = *reinterpret_cast<const T4 *>(&sm.s[st][0][kk][(64 + ty * 4) ^ x]);
        a[0] = a0.x; a[1] = a0.y; a[2] = a0.z; a[3] = a0.w; a[4] = a1.x; a[5] = a1.y; a[6] = a1.z; a[7] = a1.w;
#pragma unroll
        for (int h = 0; h < NB; ++h) {
            const T4 bv = *reinterpret_cast<const T4 *>(&sm.s[st][1][kk][(h * 64 + tx * 4) ^ x]);
            b[4 * h] = bv.x; b[4 * h + 1] = bv.y; b[4 * h + 2] = bv.z; b[4 * h + 3] = bv.w;
        }
    }

    __device__ static void cp_async16(void *dst, const void *src) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"((unsigned)__cvta_generic_to_shared(dst)), "l"(src) : "memory");
    }
    __device__ static bool mainloop_async(const Params &p, long long i0, long long j0, TaskCtx &tc, Smem &sm, T (&acc)[8][TN]) {
        static_assert(kThreads == 256 && TN == 8 && GBKA % 8 == 0, "GBKA / 8 16-byte copies per operand and thread");
        const int tid = threadIdx.x, tx = tid % TXN, ty = tid / TXN;
        const int lr = tid >> 5, lc = (tid & 31) * 4;
        const long long nkt = p.m / GBKA;
        auto issue = [&](long long kt) {
            if (kt < nkt) {
                const int st = (int)(kt % NSA);
#pragma unroll
                for (int q = 0; q < GBKA / 8; ++q) {
                    const T *row = p.A + (kt * GBKA + lr + 8 * q) * p.ld;
                    cp_async16(&sm.a[st][0][lr + 8 * q][lc], row + i0 + lc);
                    cp_async16(&sm.a[st][1][lr + 8 * q][lc], row + j0 + lc);
                }
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
        };
#pragma unroll
        for (int q = 0; q < NSA - 1; ++q) issue(q);
        // polls every `per` GBKA-tiles (= period GBK-tiles): a countdown, no division per tile
        const bool polling = tc.c != nullptr && tc.c->abort_period > 0;
        const long long per = polling ? ((long long)tc.c->abort_period * GBK + GBKA - 1) / GBKA : 1;
        long long left = per;
        bool poll = false;   // a poll posted at the end of the previous tile, decided after the barrier
        for (long long kt = 0; kt < nkt; ++kt) {
            asm volatile("cp.async.wait_group %0;" ::"n"(NSA - 2) : "memory");
            __syncthreads();   // tile kt landed for every thread; stage (kt-1) % NSA is free
            if (poll && tc.verdict()) {   // abort check (Fig 12)
                asm volatile("cp.async.wait_all;" ::: "memory");
                return true;
            }
            issue(kt + NSA - 1);
            const int st = (int)(kt % NSA);
            T a[2][8], b[2][TN];
            auto fr = [&](int kk, T *fa, T *fb) {
                const T4 a0 = *reinterpret_cast<const T4 *>(&sm.a[st][0][kk][ty * 4]);
                const T4 a1 = *reinterpret_cast<const T4 *>(&sm.a[st][0][kk][64 + ty * 4]);
                const T4 b0 = *reinterpret_cast<const T4 *>(&sm.a[st][1][kk][tx * 4]);
                const T4 b1 = *reinterpret_cast<const T4 *>(&sm.a[st][1][kk][64 + tx * 4]);
                fa[0] = a0.x; fa[1] = a0.y; fa[2] = a0.z; fa[3] = a0.w; fa[4] = a1.x; fa[5] = a1.y; fa[6] = a1.z; fa[7] = a1.w;
                fb[0] = b0.x; fb[1] = b0.y; fb[2] = b0.z; fb[3] = b0.w; fb[4] = b1.x; fb[5] = b1.y; fb[6] = b1.z; fb[7] = b1.w;
            };
            fr(0, a[0], b[0]);
#pragma unroll
            for (int kk = 0; kk < GBKA; ++kk) {
                if (kk + 1 < GBKA) fr(kk + 1, a[(kk + 1) & 1], b[(kk + 1) & 1]);
                outer<TN>(acc, a[kk & 1], b[kk & 1]);
            }
            poll = false;
            if (polling && --left == 0) {
                left = per;
                poll = kt + 1 < nkt;
                if (poll) tc.post();
            }
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
        return false;
    }

    // The k'-loop (ascending k' per output, one fma per term).  Returns true on an abort.
    template <bool IN>
    __device__ static bool mainloop(const Params &p, long long i0, long long j0, TaskCtx &tc, Smem &sm, T (&acc)[8][TN],
                                    bool sw) {
        const int tx = threadIdx.x % TXN, ty = threadIdx.x / TXN;
        const long long kdim = (OP == G_SYR2K) ? 2 * p.m : p.m;   // K'
        const long long nkt = (kdim + GBK - 1) / GBK;
        T ra[LD], rb[LD];
        gload<IN>(p, i0, j0, 0, ra, rb, sw);
        sstore(sm, 0, ra, rb);
        __syncthreads();
        // abort check every abort_period k'-tiles (Fig 12), folded into the k'-tile's own barrier:
        // one loop, no extra barrier (a plain grid has no polls at all: period() is constant)
        const long long per = tc.period();
        const bool polling = per < nkt;
        long long left = per;
#ifndef FCL_GEMM_UNROLL2
#define FCL_GEMM_UNROLL2 1
#endif
        if (FCL_GEMM_UNROLL2 && TN == 4) {   // (TN = 8: 128 registers already, unrolling spills)
            // two k'-tiles per iteration: the shared-memory stage of each is a compile-time
            // constant (no per-tile stage arithmetic on the fragment addresses)
            long long kt = 0;
            for (; kt + 1 < nkt; kt += 2) {
                if (ktile<IN, 0>(p, i0, j0, kt, nkt, tx, ty, sm, acc, ra, rb, sw, tc, polling, per, left)) return true;
                if (ktile<IN, 1>(p, i0, j0, kt + 1, nkt, tx, ty, sm, acc, ra, rb, sw, tc, polling, per, left)) return true;
            }
            if (kt < nkt && ktile<IN, 0>(p, i0, j0, kt, nkt, tx, ty, sm, acc, ra, rb, sw, tc, polling, per, left)) return true;
            return false;
        }
        for (long long kt = 0; kt < nkt; ++kt) {
            const int st = (int)(kt & 1);
            if (kt + 1 < nkt) gload<IN>(p, i0, j0, kt + 1, ra, rb, sw);   // next k'-tile in flight
            T a[2][8], b[2][TN];
            frag(sm, st, 0, tx, ty, a[0], b[0]);
#pragma unroll
            for (int kk = 0; kk < GBK; ++kk) {
                if (kk + 1 < GBK) frag(sm, st, kk + 1, tx, ty, a[(kk + 1) & 1], b[(kk + 1) & 1]);
                outer<TN>(acc, a[kk & 1], b[kk & 1]);
            }
            bool poll = false;
            if (polling && --left == 0) {
                left = per;
                poll = kt + 1 < nkt;
                if (poll) tc.post();
            }
            if (kt + 1 < nkt) sstore(sm, st ^ 1, ra, rb);
            __syncthreads();
            if (poll && tc.verdict()) return true;
        }
        return false;
    }

    // One k'-tile out of shared-memory stage ST (the next one's loads in flight, stored to the
    // other stage before the barrier; a poll folded into that barrier).  Returns true on an abort.
    template <bool IN, int ST>
    __device__ __forceinline__ static bool ktile(const Params &p, long long i0, long long j0, long long kt, long long nkt,
                                                 int tx, int ty, Smem &sm, T (&acc)[8][TN], T (&ra)[LD], T (&rb)[LD],
                                                 bool sw, TaskCtx &tc, bool polling, long long per, long long &left) {
        const bool more = kt + 1 < nkt;
        if (more) gload<IN>(p, i0, j0, kt + 1, ra, rb, sw);   // next k'-tile in flight
        T a[2][8], b[2][TN];
        frag(sm, ST, 0, tx, ty, a[0], b[0]);
#pragma unroll
        for (int kk = 0; kk < GBK; ++kk) {
            if (kk + 1 < GBK) frag(sm, ST, kk + 1, tx, ty, a[(kk + 1) & 1], b[(kk + 1) & 1]);
            outer<TN>(acc, a[kk & 1], b[kk & 1]);
        }
        bool poll = false;
        if (polling && --left == 0) {
            left = per;
            poll = more;
            if (poll) tc.post();
        }
        if (more) sstore(sm, ST ^ 1, ra, rb);
        __syncthreads();
        return poll && tc.verdict();
    }

    __device__ static bool run(const Params &p, long long t, TaskCtx &tc, Smem &sm) {
        long long bi, bj;
        tile_of(p, t, bi, bj);
        const long long i0 = bi * GBM, j0 = bj * GBM;
        const int tx = threadIdx.x % TXN, ty = threadIdx.x / TXN;
        T acc[8][TN];
#pragma unroll
        for (int r = 0; r < 8; ++r)
#pragma unroll
            for (int c = 0; c < TN; ++c) acc[r][c] = 0;
        const long long kdim = (OP == G_SYR2K) ? 2 * p.m : p.m;
        const bool interior = p.vec4 && i0 + GBM <= p.n && j0 + GBM <= p.n && kdim % GBK == 0 &&
                              (OP != G_SYR2K || p.m % 4 == 0);
#ifndef FCL_CORR_ASYNC
#define FCL_CORR_ASYNC 1
#endif
        bool done_async = false;
        if constexpr (OP == G_CORR && TN == 8 && FCL_CORR_ASYNC) {
            if (interior && p.m % GBKA == 0) {
                if (mainloop_async(p, i0, j0, tc, sm, acc)) return true;
                done_async = true;
            }
        }
        const bool sw = OP == G_SYR2K && bi > bj;   // below the diagonal: the mirror's chain
        if (!done_async && (interior ? mainloop<true>(p, i0, j0, tc, sm, acc, sw) : mainloop<false>(p, i0, j0, tc, sm, acc, sw)))
            return true;
        // epilogue: write-once stores, only of outputs whose work-group is below the mask
        const unsigned int wm = tc.wmask;
        auto keep = [&](long long i, long long j) -> bool {   // output (i, j): its work-group's id < wm
            if (wm == 0xFFFFFFFFu) return true;
            const unsigned int ui = (unsigned int)i, uj = (unsigned int)j;
            const unsigned int f = (OP == G_CORR) ? ui / (unsigned int)p.lws
                                                  : uj / (unsigned int)p.lws0 + (unsigned int)p.ngx * (ui / (unsigned int)p.lws1);
            return f < wm;
        };
        // SYR2K diagonal tile: only its upper half (i <= j) is in the canonical order; the lower
        // half is that half's mirror
        const bool diag2 = OP == G_SYR2K && bi == bj;
        if (OP != G_CORR && ((p.sym && bi != bj) || diag2)) {
            // mirror block: C[j][i] from acc(i, j) (bit-identical to acc(j, i)); the four rows
            // r of a thread's half are four consecutive columns of the mirror row
#pragma unroll
            for (int c = 0; c < TN; ++c) {
                const long long j = j0 + (c / 4) * 64 + tx * 4 + (c % 4);
                if (j >= p.n) continue;
                T *crow = p.C + j * p.n;
#pragma unroll
                for (int half = 0; half < 2; ++half) {
                    const long long ib = i0 + half * 64 + ty * 4;
                    if (p.vec4 && ib + 3 < p.n && keep(j, ib + 3) && (!diag2 || ib + 3 < j)) {
                        T4 cv = *reinterpret_cast<T4 *>(crow + ib);
                        cv.x = op_fma(p.alpha, acc[half * 4 + 0][c], op_mul(p.beta, cv.x));
                        cv.y = op_fma(p.alpha, acc[half * 4 + 1][c], op_mul(p.beta, cv.y));
                        cv.z = op_fma(p.alpha, acc[half * 4 + 2][c], op_mul(p.beta, cv.z));
                        cv.w = op_fma(p.alpha, acc[half * 4 + 3][c], op_mul(p.beta, cv.w));
                        *reinterpret_cast<T4 *>(crow + ib) = cv;
                    } else {
#pragma unroll
                        for (int r = 0; r < 4; ++r) {
                            const long long i = ib + r;
                            if (i < p.n && keep(j, i) && (!diag2 || i < j))
                                crow[i] = op_fma(p.alpha, acc[half * 4 + r][c], op_mul(p.beta, crow[i]));
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const long long i = i0 + ((r < 4) ? ty * 4 + r : 64 + ty * 4 + (r - 4));
#pragma unroll
            for (int half = 0; half < NB; ++half) {
                const long long jb = j0 + half * 64 + tx * 4;
                if (OP == G_CORR) {
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        const long long j = jb + c;
                        if (i < p.n && j < p.n && keep(i, j)) {   // (row i's work-group writes both)
                            if (j > i) { p.C[i * p.n + j] = acc[r][half * 4 + c]; p.C[j * p.n + i] = acc[r][half * 4 + c]; }
                            else if (j == i) p.C[i * p.n + i] = T(1);
                        }
                    }
                } else {
                    if (i >= p.n) continue;
                    T *crow = p.C + i * p.n;
                    if (p.vec4 && jb + 3 < p.n && keep(i, jb + 3) && (!diag2 || jb >= i)) {
                        T4 cv = *reinterpret_cast<T4 *>(crow + jb);
                        cv.x = op_fma(p.alpha, acc[r][half * 4 + 0], op_mul(p.beta, cv.x));
                        cv.y = op_fma(p.alpha, acc[r][half * 4 + 1], op_mul(p.beta, cv.y));
                        cv.z = op_fma(p.alpha, acc[r][half * 4 + 2], op_mul(p.beta, cv.z));
                        cv.w = op_fma(p.alpha, acc[r][half * 4 + 3], op_mul(p.beta, cv.w));
                        *reinterpret_cast<T4 *>(crow + jb) = cv;
                    } else {
#pragma unroll
                        for (int c = 0; c < 4; ++c) {
                            const long long j = jb + c;
                            if (j < p.n && keep(i, j) && (!diag2 || j >= i))
                                crow[j] = op_fma(p.alpha, acc[r][half * 4 + c], op_mul(p.beta, crow[j]));
                        }
                    }
                }
            }
        }
        return false;
    }
};

// ------------------------------------------------------------------------------------------
// Host-side launch plumbing
// ------------------------------------------------------------------------------------------
static thread_local char g_err[256];
const char *gpu_last_error_string() { return g_err; }
static int seterr(cudaError_t e, const char *what) {
    snprintf(g_err, sizeof g_err, "%s: %s", what, cudaGetErrorString(e));
    return -1;
}

static bool is_aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

static int largest_pow2_divisor_le(long long v, int cap) {
    int r = 1;
    while (r * 2 <= cap && v % (r * 2) == 0) r *= 2;
    return r;
}

template <class Body>
static size_t dyn_smem_bytes() { return DynSmem<Body>::value ? sizeof(typename Body::Smem) : 0; }

// the dynamic shared memory attribute of both kernels of a body, once per process
template <class Body>
static void ensure_smem() {
    static const bool once = [] {
        const size_t b = dyn_smem_bytes<Body>();
        if (b > 0) {
            cudaFuncSetAttribute((const void *)coop_kernel<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)b);
            cudaFuncSetAttribute((const void *)plain_kernel<Body>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)b);
            cudaGetLastError();
        }
        return true;
    }();
    (void)once;
}

template <class Body>
static int occupancy_grid(int num_sms) {
    static int per_sm = 0;   // cached per body type
    if (per_sm == 0) {
        int v = 0;
        ensure_smem<Body>();
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&v, coop_kernel<Body>, Body::kThreads, dyn_smem_bytes<Body>()) != cudaSuccess || v < 1)
            v = 1;
        cudaGetLastError();
        per_sm = v;
    }
    return per_sm * num_sms;
}

template <class Body>
static int launch_body(const typename Body::Params &bp, const CoopCtl *c, long long task_lo, long long task_hi,
                       int num_sms, cudaStream_t s, const SlotReset *reset = nullptr, int pdl = PDL_OFF) {
    const long long n = task_hi - task_lo;
    if (n <= 0) return 0;
    ensure_smem<Body>();
    const size_t smem = dyn_smem_bytes<Body>();
    if (c) {
        long long grid = occupancy_grid<Body>(num_sms);
        if (grid > n) grid = n;
        static const bool coop_api = !(getenv("FCL_COOP_LAUNCH") && atoi(getenv("FCL_COOP_LAUNCH")) == 0);
        if (c->fused && coop_api) {
            // cooperative launch: all CTAs co-resident, required by the fused tail's grid barrier
            CoopCtl cc = *c;
            typename Body::Params pp = bp;
            void *args[] = {(void *)&cc, (void *)&pp};
            cudaError_t e = cudaLaunchCooperativeKernel((const void *)coop_kernel<Body>, dim3((unsigned)grid),
                                                        dim3(Body::kThreads), args, smem, s);
            if (e != cudaSuccess) return seterr(e, "coop_kernel cooperative launch");
            return (int)grid;
        }
        coop_kernel<Body><<<(unsigned)grid, Body::kThreads, smem, s>>>(*c, bp);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return seterr(e, "coop_kernel launch");
        return (int)grid;
    }
    SlotReset r{};
    if (reset) r = *reset;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)n);
    cfg.blockDim = dim3(Body::kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl != PDL_OFF ? 1 : 0;
    cudaError_t e = cudaLaunchKernelEx(&cfg, plain_kernel<Body>, bp, (long long)task_lo, r, pdl == PDL_WAIT ? 1 : 0);
    if (e != cudaSuccess) return seterr(e, "plain_kernel launch");
    return (int)n;
}

// ---- per-kernel parameter construction ----
static Tile2D make_tile(const Geom &g, long long nrows, long long ncols, int tw, int th) {
    Tile2D tl;
    tl.nrows = nrows; tl.ncols = ncols;
    tl.ngx = g.ng[0]; tl.lws0 = g.lws[0]; tl.lws1 = g.lws[1];
    tl.tw = tw; tl.th = th;
    tl.ntx = (g.ng[0] + tw - 1) / tw;
    return tl;
}
static void tile_shape(const Geom &g, int want_cols, int want_rows, int &tw, int &th) {
    tw = (int)(want_cols / g.lws[0]); if (tw < 1) tw = 1;
    th = (int)(want_rows / g.lws[1]); if (th < 1) th = 1;
}
// Task tile (in work-groups) of the 2-D tiled kernels: 2DCONV's warp-sized tile, CORR-reduce's
// 256 x 32.
static void tile_shape_of(const KArgs &a, const Geom &g, int &tw, int &th) {
    if (a.kernel == K_CONV2D) tile_shape(g, FCL_CONV_TILE_COLS, FCL_CONV_TILE_ROWS, tw, th);
    else tile_shape(g, 256, 32, tw, th);
}

template <typename T, int NMAT>
static typename RowDotBody<T, NMAT>::Params rowdot_params(const KArgs &a, const Geom &g) {
    typename RowDotBody<T, NMAT>::Params p;
    p.A = (const T *)a.dev[0];
    if (a.kernel == K_GESUMMV) {
        p.B = (const T *)a.dev[1]; p.x = (const T *)a.dev[2]; p.out0 = (T *)a.dev[3]; p.out1 = (T *)a.dev[4];
        p.nrows = a.n0; p.ncols = a.n0;
    } else {
        p.B = nullptr; p.x = (const T *)a.dev[1]; p.out0 = (T *)a.dev[2]; p.out1 = nullptr;
        p.nrows = a.n0; p.ncols = a.n1;
    }
    p.lws = g.lws[0];
    p.R = largest_pow2_divisor_le(g.lws[0], 4);
    if (a.integer) { p.alpha = (T)a.ialpha; p.beta = (T)a.ibeta; }
    else { p.alpha = (T)a.alpha; p.beta = (T)a.beta; }
    p.vec4 = (p.ncols % 4 == 0) && is_aligned16(p.A) && is_aligned16(p.x) && (NMAT == 1 || is_aligned16(p.B));
    p.streamed = a.streamed ? 1 : 0;
    return p;
}

template <typename T, int MODE>
static typename ColDotBody<T, MODE>::Params coldot_params(const KArgs &a, const Geom &g) {
    typename ColDotBody<T, MODE>::Params p;
    p.A = (const T *)a.dev[0];
    p.v = (MODE == COL_DOT) ? (const T *)a.dev[1] : nullptr;
    p.mean = (MODE == COL_SQDEV) ? (const T *)a.dev[1] : nullptr;
    const int oi = (MODE == COL_SQDEV) ? 2 : (MODE == COL_SUM ? 1 : 2);
    p.out = (T *)a.dev[oi];
    p.nrows = a.n0; p.ncols = a.n1; p.lws = g.lws[0];
    p.CB = largest_pow2_divisor_le(g.lws[0], 32);
    p.nf = (float)a.n0; p.eps = a.eps;
    p.vec4 = (p.ncols % 4 == 0) && is_aligned16(p.A);
    return p;
}

template <typename T, int OP, int TN = 8>
static typename GemmBody<T, OP, TN>::Params gemm_params(const KArgs &a, const Geom &g) {
    typename GemmBody<T, OP, TN>::Params p;
    p.A = (const T *)a.dev[0];
    if (OP == G_SYR2K) { p.B = (const T *)a.dev[1]; p.C = (T *)a.dev[2]; }
    else { p.B = nullptr; p.C = (T *)a.dev[1]; }
    if (OP == G_CORR) { p.n = a.n1; p.m = a.n0; p.ld = a.n1; }
    else { p.n = a.n0; p.m = a.n1; p.ld = a.n1; }
    if (a.integer) { p.alpha = (T)a.ialpha; p.beta = (T)a.ibeta; }
    else { p.alpha = (T)a.alpha; p.beta = (T)a.beta; }
    p.ntile = (p.n + GBM - 1) / GBM;
    p.ngx = g.ng[0]; p.lws0 = g.lws[0]; p.lws1 = g.work_dim > 1 ? g.lws[1] : 1; p.lws = g.lws[0];
    p.vec4 = (p.ld % 4 == 0) && (p.n % 4 == 0) && is_aligned16(p.A) && is_aligned16(p.C) &&
             (OP != G_SYR2K || is_aligned16(p.B));
    p.sym = (OP != G_CORR && a.sym) ? 1 : 0;
    return p;
}

// Dispatch on the kernel id: F is a generic functor called with a Body type and its Params.
template <typename F>
static int with_body(const KArgs &a, const Geom &g, F &&f) {
    switch (a.kernel) {
    case K_ATAX_TMP:
    case K_BICG_Q:
        if (a.integer) return f.template go<RowDotBody<int32_t, 1>>(rowdot_params<int32_t, 1>(a, g));
        return f.template go<RowDotBody<float, 1>>(rowdot_params<float, 1>(a, g));
    case K_GESUMMV:
        if (a.integer) return f.template go<RowDotBody<int32_t, 2>>(rowdot_params<int32_t, 2>(a, g));
        return f.template go<RowDotBody<float, 2>>(rowdot_params<float, 2>(a, g));
    case K_ATAX_Y:
    case K_BICG_S:
        if (a.integer) return f.template go<ColDotBody<int32_t, COL_DOT>>(coldot_params<int32_t, COL_DOT>(a, g));
        return f.template go<ColDotBody<float, COL_DOT>>(coldot_params<float, COL_DOT>(a, g));
    case K_CORR_MEAN: return f.template go<ColDotBody<float, COL_SUM>>(coldot_params<float, COL_SUM>(a, g));
    case K_CORR_STD: return f.template go<ColDotBody<float, COL_SQDEV>>(coldot_params<float, COL_SQDEV>(a, g));
    case K_CORR_REDUCE: {
        CorrReduceBody::Params p;
        p.data = (float *)a.dev[0]; p.mean = (const float *)a.dev[1]; p.std_ = (const float *)a.dev[2];
        int tw, th; tile_shape(g, 256, 32, tw, th);
        p.tl = make_tile(g, a.n0, a.n1, tw, th);
        p.sqrtn = __builtin_sqrtf((float)a.n0);
        return f.template go<CorrReduceBody>(p);
    }
    case K_CONV2D: {
        int tw, th; tile_shape_of(a, g, tw, th);
        if (a.integer) {
            Conv2DBody<int32_t>::Params p;
            p.A = (const int32_t *)a.dev[0]; p.B = (int32_t *)a.dev[1];
            p.tl = make_tile(g, a.n0, a.n1, tw, th);
            p.vec4 = (a.n1 % 4 == 0) && is_aligned16(p.A) && is_aligned16(p.B);
            const int32_t c[9] = {2, 5, -8, -3, 6, -9, 4, 7, 1};
            for (int q = 0; q < 9; ++q) p.c[q] = c[q];
            return f.template go<Conv2DBody<int32_t>>(p);
        }
        Conv2DBody<float>::Params p;
        p.A = (const float *)a.dev[0]; p.B = (float *)a.dev[1];
        p.tl = make_tile(g, a.n0, a.n1, tw, th);
        p.vec4 = (a.n1 % 4 == 0) && is_aligned16(p.A) && is_aligned16(p.B);
        const float c[9] = {0.2f, 0.5f, -0.8f, -0.3f, 0.6f, -0.9f, 0.4f, 0.7f, 0.10f};
        for (int q = 0; q < 9; ++q) p.c[q] = c[q];
        return f.template go<Conv2DBody<float>>(p);
    }
    case K_SYRK:
        if (a.sym) {   // upper-triangle grid: one 512-thread CTA per SM
            if (a.integer) return f.template go<GemmBody<int32_t, G_SYRK, 4>>(gemm_params<int32_t, G_SYRK, 4>(a, g));
            return f.template go<GemmBody<float, G_SYRK, 4>>(gemm_params<float, G_SYRK, 4>(a, g));
        }
        if (a.integer) return f.template go<GemmBody<int32_t, G_SYRK>>(gemm_params<int32_t, G_SYRK>(a, g));
        return f.template go<GemmBody<float, G_SYRK>>(gemm_params<float, G_SYRK>(a, g));
    case K_SYR2K:
        if (a.sym) {   // upper-triangle grid: one 512-thread CTA per SM
            if (a.integer) return f.template go<GemmBody<int32_t, G_SYR2K, 4>>(gemm_params<int32_t, G_SYR2K, 4>(a, g));
            return f.template go<GemmBody<float, G_SYR2K, 4>>(gemm_params<float, G_SYR2K, 4>(a, g));
        }
        if (a.integer) return f.template go<GemmBody<int32_t, G_SYR2K>>(gemm_params<int32_t, G_SYR2K>(a, g));
        return f.template go<GemmBody<float, G_SYR2K>>(gemm_params<float, G_SYR2K>(a, g));
    case K_CORR_CORR:
#ifndef FCL_CORR_TN
#define FCL_CORR_TN 8   // (TN = 4, one 512-thread CTA per SM: 1.62 vs 1.55 ms at M = N = 4096)
#endif
        return f.template go<GemmBody<float, G_CORR, FCL_CORR_TN>>(gemm_params<float, G_CORR, FCL_CORR_TN>(a, g));
    default: return -1;
    }
}

// Host mirror of each body's task enumeration (must match Body::key exactly).
static int64_t host_rowdot_key(const Geom &g, int64_t t) {
    const int R = largest_pow2_divisor_le(g.lws[0], 4);
    return (t * R) / g.lws[0];
}

TaskSpace gpu_task_space(const KArgs &a, const Geom &g) {
    TaskSpace ts{0, 256};
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV: {
        const int R = largest_pow2_divisor_le(g.lws[0], 4);
        ts.ntasks = (g.ng[0] * g.lws[0] + R - 1) / R;   // covers every row of every work-group
        ts.threads = 128; break;
    }
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD: {
        const int CB = largest_pow2_divisor_le(g.lws[0], 32);
        ts.ntasks = (g.ng[0] * g.lws[0] + CB - 1) / CB;
        ts.threads = 256; break;
    }
    case K_CORR_REDUCE: case K_CONV2D: {
        int tw, th; tile_shape_of(a, g, tw, th);
        const long long ntx = (g.ng[0] + tw - 1) / tw, nty = (g.ng[1] + th - 1) / th;
        ts.ntasks = ntx * nty; ts.threads = 256; break;
    }
    case K_SYRK: case K_SYR2K: {
        const long long nt = (a.n0 + GBM - 1) / GBM;
        ts.ntasks = a.sym ? nt * (nt + 1) / 2 : nt * nt;
        ts.threads = a.sym ? 512 : 256; break;
    }
    case K_CORR_CORR: {
        const long long nt = (a.n1 + GBM - 1) / GBM;
        ts.ntasks = nt * (nt + 1) / 2; ts.threads = FCL_CORR_TN == 4 ? 512 : 256; break;
    }
    default: break;
    }
    return ts;
}

int64_t gpu_task_key(const KArgs &a, const Geom &g, int64_t t) {
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV: return host_rowdot_key(g, t);
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD: {
        const int CB = largest_pow2_divisor_le(g.lws[0], 32);
        return (t * CB) / g.lws[0];
    }
    case K_CORR_REDUCE: case K_CONV2D: {
        int tw, th; tile_shape_of(a, g, tw, th);
        const long long ntx = (g.ng[0] + tw - 1) / tw;
        return (t % ntx) * tw + g.ng[0] * ((t / ntx) * th);
    }
    case K_SYRK: case K_SYR2K: {
        const long long nt = (a.n0 + GBM - 1) / GBM;
        long long bi = t / nt, bj = t % nt;
        if (a.sym) {   // upper triangle; the key is the direct block's
            long long rem = t;
            bi = 0;
            while (rem >= nt - bi) { rem -= nt - bi; ++bi; }
            bj = bi + rem;
        }
        return (bj * GBM) / g.lws[0] + g.ng[0] * ((bi * GBM) / g.lws[1]);
    }
    case K_CORR_CORR: {
        const long long nt = (a.n1 + GBM - 1) / GBM;
        long long b1 = 0, rem = t;
        while (rem >= nt - b1) { rem -= nt - b1; ++b1; }
        return (b1 * GBM) / g.lws[0];
    }
    default: return 0;
    }
}

void gpu_task_wgs(const KArgs &a, const Geom &g, int64_t t, std::vector<int64_t> &out) {
    auto rect = [&](int64_t gx0, int64_t gx1, int64_t gy0, int64_t gy1) {
        gx1 = gx1 < g.ng[0] ? gx1 : g.ng[0];
        gy1 = gy1 < g.ng[1] ? gy1 : g.ng[1];
        for (int64_t gy = gy0; gy < gy1; ++gy)
            for (int64_t gx = gx0; gx < gx1; ++gx) out.push_back(gx + g.ng[0] * gy);
    };
    switch (a.kernel) {
    case K_ATAX_TMP: case K_BICG_Q: case K_GESUMMV:
    case K_ATAX_Y: case K_BICG_S: case K_CORR_MEAN: case K_CORR_STD:
        out.push_back(gpu_task_key(a, g, t));   // a task is part of one work-group
        break;
    case K_CORR_REDUCE: case K_CONV2D: {
        int tw, th; tile_shape_of(a, g, tw, th);
        const long long ntx = (g.ng[0] + tw - 1) / tw, tx = t % ntx, ty = t / ntx;
        rect(tx * tw, tx * tw + tw, ty * th, ty * th + th);
        break;
    }
    case K_SYRK: case K_SYR2K: {
        const long long nt = (a.n0 + GBM - 1) / GBM;
        long long bi = t / nt, bj = t % nt;
        const bool sym = a.sym;
        if (sym) {
            long long rem = t;
            bi = 0;
            while (rem >= nt - bi) { rem -= nt - bi; ++bi; }
            bj = bi + rem;
        }
        const long long cx = GBM / g.lws[0], cy = GBM / g.lws[1];
        rect(bj * cx, bj * cx + cx, bi * cy, bi * cy + cy);
        if (sym && bi != bj) rect(bi * cx, bi * cx + cx, bj * cy, bj * cy + cy);   // mirror block
        break;
    }
    case K_CORR_CORR: {
        const long long nt = (a.n1 + GBM - 1) / GBM;
        long long b1 = 0, rem = t;
        while (rem >= nt - b1) { rem -= nt - b1; ++b1; }
        const long long f0 = (b1 * GBM) / g.lws[0];
        long long f1 = ((b1 + 1) * GBM - 1) / g.lws[0] + 1;
        if (f1 > g.ng[0]) f1 = g.ng[0];
        for (long long f = f0; f < f1; ++f) out.push_back(f);
        break;
    }
    default: break;
    }
}

bool gpu_geometry_ok(const KArgs &a, const Geom &g, const char **why) {
    switch (a.kernel) {
    case K_SYRK: case K_SYR2K:
        if (g.work_dim != 2 || GBM % g.lws[0] || GBM % g.lws[1]) { *why = "lws must divide 128 in both dims"; return false; }
        break;
    case K_CORR_CORR:
        if (g.work_dim != 1) { *why = "1-D NDRange expected"; return false; }
        break;
    case K_CORR_REDUCE: case K_CONV2D:
        if (g.work_dim != 2) { *why = "2-D NDRange expected"; return false; }
        break;
    default:
        if (g.work_dim != 1) { *why = "1-D NDRange expected"; return false; }
    }
    return true;
}

int64_t gpu_slice_align(const KArgs &a, const Geom &g) {
    switch (a.kernel) {
    case K_CORR_REDUCE: case K_CONV2D: {
        int tw, th; tile_shape_of(a, g, tw, th);
        return g.ng[0] * th;                       // whole tile rows
    }
    case K_SYRK: case K_SYR2K: return g.ng[0] * (GBM / g.lws[1]);
    case K_CORR_CORR: return g.lws[0] >= GBM ? 1 : GBM / g.lws[0];
    default: return 1;                             // tasks never span work-groups
    }
}

int gpu_default_abort_period(const KArgs &a) {
    switch (a.kernel) {
    case K_SYRK: case K_SYR2K: case K_CORR_CORR: return 8;    // every 8 k'-tiles (128 k')
    default: return 0;
    }
}

struct CoopLauncher {
    const CoopCtl *c; int num_sms; cudaStream_t s;
    template <class Body> int go(const typename Body::Params &bp) {
        return launch_body<Body>(bp, c, c->task_lo, c->task_hi, num_sms, s);
    }
};
struct PlainLauncher {
    long long lo, hi; cudaStream_t s; const SlotReset *reset; int pdl;
    template <class Body> int go(const typename Body::Params &bp) {
        return launch_body<Body>(bp, nullptr, lo, hi, 0, s, reset, pdl);
    }
};
struct CapacityQuery {
    int num_sms;
    template <class Body> int go(const typename Body::Params &) { return occupancy_grid<Body>(num_sms); }
};

int64_t gpu_coop_capacity(const KArgs &a, const Geom &g, int num_sms) {
    CapacityQuery q{num_sms};
    return with_body(a, g, q);
}

int gpu_launch_coop(const KArgs &a, const Geom &g, const CoopCtl &c, int num_sms, void *stream) {
    CoopLauncher L{&c, num_sms, (cudaStream_t)stream};
    return with_body(a, g, L);
}

int gpu_launch_plain(const KArgs &a, const Geom &g, int64_t task_lo, int64_t task_hi, void *stream,
                     const SlotReset *reset, int pdl) {
    PlainLauncher L{task_lo, task_hi, (cudaStream_t)stream, reset, pdl};
    return with_body(a, g, L);
}

int gpu_launch_merge(void *gpu, const void *cpu, const void *twin, size_t bytes, int elem_size, int num_sms,
                     void *stream) {
    if (bytes == 0) return 0;
    uint8_t *g = (uint8_t *)gpu;
    const uint8_t *c = (const uint8_t *)cpu, *t = (const uint8_t *)twin;
    long long grid = (long long)((bytes / 64 + 255) / 256);
    const long long cap = (long long)num_sms * 8;
    if (grid > cap) grid = cap;
    if (grid < 1) grid = 1;
    cudaStream_t s = (cudaStream_t)stream;
    switch (elem_size) {
    case 1: merge_kernel<1><<<(unsigned)grid, 256, 0, s>>>(g, c, t, bytes); break;
    case 2: merge_kernel<2><<<(unsigned)grid, 256, 0, s>>>(g, c, t, bytes); break;
    case 4: merge_kernel<4><<<(unsigned)grid, 256, 0, s>>>(g, c, t, bytes); break;
    case 8: merge_kernel<8><<<(unsigned)grid, 256, 0, s>>>(g, c, t, bytes); break;
    default: return -1;
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return seterr(e, "merge_kernel launch");
    return 1;
}

int gpu_launch_merge_dev(const DevMergeList &L, size_t max_bytes, int num_sms, void *stream) {
    long long grid = (long long)((max_bytes / 64 + 255) / 256);
    const long long cap = (long long)num_sms * 8;
    if (grid > cap) grid = cap;
    if (grid < 1) grid = 1;
    merge_dev_kernel<<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>(L);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return seterr(e, "merge_dev_kernel launch");
    return 1;
}

int gpu_launch_copies(int n, void *const *dst, const void *const *src, const size_t *bytes, int num_sms,
                      void *stream, bool pdl) {
    CopyList L;
    size_t total = 0;
    L.n = n;
    for (int b = 0; b < n && b < 6; ++b) {
        if ((reinterpret_cast<uintptr_t>(dst[b]) | reinterpret_cast<uintptr_t>(src[b])) & 15u) return -2;
        L.dst[b] = (uint8_t *)dst[b]; L.src[b] = (const uint8_t *)src[b]; L.bytes[b] = bytes[b];
        total += bytes[b];
    }
    if (total == 0) return 0;
    long long grid = (long long)((total / 16 + 255) / 256);
    if (grid > (long long)num_sms * 8) grid = (long long)num_sms * 8;
    if (grid < 1) grid = 1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(256);
    cfg.stream = (cudaStream_t)stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    cudaError_t e = cudaLaunchKernelEx(&cfg, copies_kernel, L, pdl ? 1 : 0);
    if (e != cudaSuccess) return seterr(e, "copies_kernel launch");
    return 1;
}

// a[j][i] = a[i][j] for i < j: 32 x 32 tiles of the upper triangle, transposed through shared
// memory so that both the read of row block (bi) and the write of column block (bj) coalesce.
template <typename T>
__global__ void __launch_bounds__(256) mirror_upper_kernel(T *a, long long n) {
    __shared__ T tile[32][33];
    const long long nt = (n + 31) / 32;
    for (long long t = blockIdx.x; t < nt * (nt + 1) / 2; t += gridDim.x) {
        long long bi = 0, rem = t;   // upper-triangle tile (bi <= bj), row-major
        while (rem >= nt - bi) { rem -= nt - bi; ++bi; }
        const long long bj = bi + rem;
        const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
        for (int r = ty; r < 32; r += 8) {
            const long long i = bi * 32 + r, j = bj * 32 + tx;
            if (i < n && j < n) tile[r][tx] = a[i * n + j];
        }
        __syncthreads();
        for (int r = ty; r < 32; r += 8) {
            const long long j = bj * 32 + r, i = bi * 32 + tx;   // destination row j, column i
            if (i < n && j < n && i < j) a[j * n + i] = tile[tx][r];
        }
        __syncthreads();
    }
}

int gpu_launch_mirror_upper(void *a, long long n, int elem_size, int num_sms, void *stream) {
    if (n <= 1) return 0;
    const long long nt = (n + 31) / 32;
    long long grid = nt * (nt + 1) / 2;
    if (grid > (long long)num_sms * 8) grid = (long long)num_sms * 8;
    if (elem_size == 4) mirror_upper_kernel<uint32_t><<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>((uint32_t *)a, n);
    else if (elem_size == 8) mirror_upper_kernel<unsigned long long><<<(unsigned)grid, 256, 0, (cudaStream_t)stream>>>((unsigned long long *)a, n);
    else return -2;
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return seterr(e, "mirror_upper_kernel launch");
    return 1;
}

int gpu_launch_store64(unsigned long long *addr, unsigned long long value, void *stream, unsigned long long *stamp) {
    store64_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(addr, value, stamp);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return seterr(e, "store64_kernel launch");
    return 1;
}

}  // namespace fcl

// ------------------------------------------------------------------------------------------
// Eager loading of every kernel of the library.  With CUDA's lazy module loading a kernel is
// loaded at its first launch, and loading may wait for the device: a first-time launch queued
// while a cooperative grid waits for host-driven copies (streamed inputs) can
// then stall the host thread that issues those copies -- a deadlock.  The context loads
// everything once, at creation.
// ------------------------------------------------------------------------------------------
namespace fcl {
template <class Body>
static int preload_body() {
    cudaFuncAttributes at;
    int bad = 0;
    bad |= cudaFuncGetAttributes(&at, coop_kernel<Body>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, plain_kernel<Body>) != cudaSuccess;
    return bad;
}
int gpu_preload_kernels() {
    int bad = 0;
    bad |= preload_body<RowDotBody<float, 1>>() | preload_body<RowDotBody<int32_t, 1>>();
    bad |= preload_body<RowDotBody<float, 2>>() | preload_body<RowDotBody<int32_t, 2>>();
    bad |= preload_body<ColDotBody<float, COL_DOT>>() | preload_body<ColDotBody<int32_t, COL_DOT>>();
    bad |= preload_body<ColDotBody<float, COL_SUM>>() | preload_body<ColDotBody<float, COL_SQDEV>>();
    bad |= preload_body<CorrReduceBody>();
    bad |= preload_body<Conv2DBody<float>>() | preload_body<Conv2DBody<int32_t>>();
    bad |= preload_body<GemmBody<float, G_SYRK>>() | preload_body<GemmBody<int32_t, G_SYRK>>();
    bad |= preload_body<GemmBody<float, G_SYRK, 4>>() | preload_body<GemmBody<int32_t, G_SYRK, 4>>();
    bad |= preload_body<GemmBody<float, G_SYR2K>>() | preload_body<GemmBody<int32_t, G_SYR2K>>();
    bad |= preload_body<GemmBody<float, G_SYR2K, 4>>() | preload_body<GemmBody<int32_t, G_SYR2K, 4>>();
    bad |= preload_body<GemmBody<float, G_CORR, FCL_CORR_TN>>();
    cudaFuncAttributes at;
    bad |= cudaFuncGetAttributes(&at, merge_kernel<1>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, merge_kernel<2>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, merge_kernel<4>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, merge_kernel<8>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, merge_dev_kernel) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, copies_kernel) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, store64_kernel) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, mirror_upper_kernel<uint32_t>) != cudaSuccess;
    bad |= cudaFuncGetAttributes(&at, mirror_upper_kernel<unsigned long long>) != cudaSuccess;
    if (bad) { cudaGetLastError(); return seterr(cudaErrorInvalidDeviceFunction, "kernel preload"); }
    return 0;
}
}  // namespace fcl
