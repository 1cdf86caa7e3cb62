// ubench_wt.cu -- returning small outputs to pinned host memory: SM stores through the mapping
// (1..148 CTAs, 16-byte coalesced, system fence) vs copy-engine D2H copies.  Event-timed on one
// stream, each variant after an idle GPU.  Diagnostic for the write-through return.
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o ubench_wt ubench_wt.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d: %s\n", #x, __LINE__, cudaGetErrorString(e_)); exit(1);} } while (0)

__global__ void wt_copy(const uint4 *src, uint4 *dst, size_t nv, int fence) {
    for (size_t v = blockIdx.x * (size_t)blockDim.x + threadIdx.x; v < nv; v += (size_t)gridDim.x * blockDim.x)
        dst[v] = __ldcg(src + v);
    if (fence) __threadfence_system();
}
__global__ void empty_k() {}

template <class F>
static float time_it(F f, int reps = 50) {
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    std::vector<float> ts;
    for (int r = 0; r < reps + 5; ++r) {
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        f();
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
        if (r >= 5) ts.push_back(ms * 1e3f);
    }
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];
}

int main() {
    for (size_t kb : {16, 48, 256, 1024}) {
        const size_t bytes = kb << 10;
        void *d, *h, *hd;
        CK(cudaMalloc(&d, bytes)); CK(cudaMemset(d, 1, bytes));
        CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
        CK(cudaHostGetDevicePointer(&hd, h, 0));
        printf("%zu KiB:\n", kb);
        printf("  empty kernel                      %7.2f us\n", time_it([&] { empty_k<<<1, 32>>>(); }));
        for (int grid : {1, 8, 48, 148, 296})
            for (int fence : {0, 1}) {
                float t = time_it([&] { wt_copy<<<grid, 128>>>((const uint4 *)d, (uint4 *)hd, bytes / 16, fence); });
                printf("  SM stores, %3d CTAs x 128, fence %d %7.2f us\n", grid, fence, t);
            }
        printf("  cudaMemcpyAsync D2H               %7.2f us\n", time_it([&] { CK(cudaMemcpyAsync(h, d, bytes, cudaMemcpyDeviceToHost, 0)); }));
        printf("  3 x cudaMemcpyAsync D2H (1/3 each) %7.2f us\n", time_it([&] {
            for (int k = 0; k < 3; ++k) CK(cudaMemcpyAsync((char *)h + k * bytes / 3, (char *)d + k * bytes / 3, bytes / 3, cudaMemcpyDeviceToHost, 0));
        }));
        CK(cudaFree(d)); CK(cudaFreeHost(h));
    }
    return 0;
}
