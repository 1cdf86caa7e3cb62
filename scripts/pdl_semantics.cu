// pdl_semantics.cu -- what programmatic dependent launch (PDL) guarantees on this driver/GPU,
// checked before the runtime relies on it:
//  T1  an event recorded between a PDL primary and its secondary completes only when the
//      primary has completed (a side stream waiting on it copies the primary's final data);
//  T2  griddepcontrol.wait in kernel C covers a primary two launches back (A -> B -> C, where B
//      launched early and did not wait);
//  T3  overlap actually happens (B, independent and non-waiting, starts before A ends).
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o pdl_semantics pdl_semantics.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e_)); exit(1);} } while (0)

__device__ __forceinline__ unsigned long long gt() { unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

// spins `ns`, then every thread writes its slice of X with v; triggers dependents at start
__global__ void kA(int *X, int n, int v, long long ns, unsigned long long *stamp) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const unsigned long long t0 = gt();
    if (blockIdx.x == 0 && threadIdx.x == 0) stamp[0] = t0;
    while ((long long)(gt() - t0) < ns) {}
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) X[i] = v;
    __syncthreads();
    if (threadIdx.x == 0) atomicMax(stamp + 1, gt());
}
// independent short kernel: records its start time
__global__ void kB(unsigned long long *stamp, int wait) {
    if (wait) asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (blockIdx.x == 0 && threadIdx.x == 0) stamp[2] = gt();
}
// waits, then checks X == v everywhere
__global__ void kC(const int *X, int n, int v, int *bad, int wait) {
    if (wait) asm volatile("griddepcontrol.wait;" ::: "memory");
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
        if (X[i] != v) atomicAdd(bad, 1);
}

template <class K, class... A>
static void launch(K k, int grid, int block, cudaStream_t s, bool pdl, A... a) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid); cfg.blockDim = dim3(block); cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at; cfg.numAttrs = pdl ? 1 : 0;
    CK(cudaLaunchKernelEx(&cfg, k, a...));
}

int main() {
    const int n = 1 << 24;
    int *X, *bad, *hX;
    unsigned long long *stamp;
    CK(cudaMalloc(&X, n * 4)); CK(cudaMalloc(&bad, 4)); CK(cudaMallocManaged(&stamp, 64));
    CK(cudaMallocHost(&hX, n * 4));
    cudaStream_t s, side;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking));
    cudaEvent_t e;
    CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    int fails1 = 0, fails2 = 0, fails4 = 0, overlaps = 0, reps = 50;
    cudaEvent_t es;
    CK(cudaEventCreateWithFlags(&es, cudaEventDisableTiming));
    for (int r = 0; r < reps; ++r) {
        const int v = 1000 + r;
        // T1: A ; event ; B(pdl) -- side stream copies X after the event
        CK(cudaMemsetAsync(X, 0, n * 4, s));
        for (int k = 0; k < 4; ++k) stamp[k] = 0;
        CK(cudaDeviceSynchronize());
        launch(kA, 592, 256, s, false, X, n, v, 50000ll, stamp);
        CK(cudaEventRecord(e, s));
        launch(kB, 148, 128, s, true, stamp, 0);
        CK(cudaStreamWaitEvent(side, e, 0));
        CK(cudaMemcpyAsync(hX, X, n * 4, cudaMemcpyDeviceToHost, side));
        CK(cudaStreamSynchronize(side));
        int f = 0;
        for (int i = 0; i < n; i += 4099) f += hX[i] != v;
        f += hX[n - 1] != v;
        fails1 += f != 0;
        CK(cudaStreamSynchronize(s));
        overlaps += (stamp[2] != 0 && stamp[2] < stamp[1]);
        // T2: A ; B(pdl, no wait) ; C(pdl, wait) checks A's data
        CK(cudaMemsetAsync(X, 0, n * 4, s));
        CK(cudaMemsetAsync(bad, 0, 4, s));
        launch(kA, 592, 256, s, false, X, n, v, 50000ll, stamp);
        launch(kB, 148, 128, s, true, stamp, 0);
        launch(kC, 592, 256, s, true, (const int *)X, n, v, bad, 1);
        int hb = 0;
        CK(cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        fails2 += hb != 0;
        // T4: side stream: A writes X (long); event es.  main: B (triggers early) ;
        // wait(es) ; C(pdl, no wait) reads X -- the stream wait must hold C back
        CK(cudaMemsetAsync(X, 0, n * 4, s));
        CK(cudaMemsetAsync(bad, 0, 4, s));
        CK(cudaStreamSynchronize(s));
        launch(kA, 592, 256, side, false, X, n, v, 50000ll, stamp);
        CK(cudaEventRecord(es, side));
        launch(kB, 148, 128, s, false, stamp, 0);
        CK(cudaStreamWaitEvent(s, es, 0));
        launch(kC, 592, 256, s, true, (const int *)X, n, v, bad, 0);
        hb = 0;
        CK(cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        fails4 += hb != 0;
    }
    printf("T1 event-after-PDL-primary completes late enough: %s (%d/%d reps failed)\n", fails1 ? "NO" : "yes", fails1, reps);
    printf("T2 griddepcontrol.wait covers the grid two back: %s (%d/%d reps failed)\n", fails2 ? "NO" : "yes", fails2, reps);
    printf("T4 a stream wait between a triggering grid and a PDL grid holds: %s (%d/%d reps failed)\n", fails4 ? "NO" : "yes", fails4, reps);
    printf("T3 independent secondary started before the primary ended: %d/%d reps\n", overlaps, reps);
    return 0;
}
