// Microbenchmark of the lazy-return gather (copies_kernel's pattern): device buffers -> pinned,
// mapped host memory with 16-byte stores from the SMs, as bench.py's step returns its outputs
// (GESUMMV tmp + y, BICG s, q: 4 x 16 KB at N = 4096).  CUDA-event time per launch (median of
// 200, after a warm-up), for several grid shapes, and cudaMemcpyAsync D2H of the same bytes for
// comparison.
//
// Build + run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubench_gather scripts/ubench_gather.cu && /tmp/ubench_gather
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>

struct CopyList { unsigned char *dst[6]; const unsigned char *src[6]; size_t bytes[6]; int n; };

__global__ void gather(const CopyList L) {
    const size_t tid = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    const size_t nth = (size_t)gridDim.x * blockDim.x;
    for (int b = 0; b < L.n; ++b) {
        const size_t nv = L.bytes[b] / 16;
        const uint4 *s = reinterpret_cast<const uint4 *>(L.src[b]);
        uint4 *d = reinterpret_cast<uint4 *>(L.dst[b]);
        for (size_t v = tid; v < nv; v += nth) d[v] = __ldcs(s + v);
    }
}

int main() {
    const int nb = 4;
    const size_t bytes = 16384;
    CopyList L;
    L.n = nb;
    std::vector<void *> hosts;
    for (int b = 0; b < nb; ++b) {
        void *d, *h, *hd;
        cudaMalloc(&d, bytes);
        cudaMemset(d, b, bytes);
        cudaHostAlloc(&h, bytes, cudaHostAllocMapped);
        cudaHostGetDevicePointer(&hd, h, 0);
        L.src[b] = (const unsigned char *)d;
        L.dst[b] = (unsigned char *)hd;
        L.bytes[b] = bytes;
        hosts.push_back(h);
    }
    cudaStream_t s;
    cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int shapes[][2] = {{16, 256}, {32, 128}, {64, 64}, {128, 32}, {8, 512}, {4, 1024}, {1, 1024}};
    for (auto &sh : shapes) {
        std::vector<float> ts;
        for (int r = 0; r < 230; ++r) {
            cudaEventRecord(e0, s);
            gather<<<sh[0], sh[1], 0, s>>>(L);
            cudaEventRecord(e1, s);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 30) ts.push_back(ms);
        }
        std::sort(ts.begin(), ts.end());
        printf("gather grid %4d x %4d: %.2f us (median), %.2f us (p10)\n", sh[0], sh[1], 1e3 * ts[ts.size() / 2], 1e3 * ts[ts.size() / 10]);
    }
    {
        std::vector<float> ts;
        for (int r = 0; r < 230; ++r) {
            cudaEventRecord(e0, s);
            for (int b = 0; b < nb; ++b) cudaMemcpyAsync(hosts[b], L.src[b], bytes, cudaMemcpyDeviceToHost, s);
            cudaEventRecord(e1, s);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 30) ts.push_back(ms);
        }
        std::sort(ts.begin(), ts.end());
        printf("4 x cudaMemcpyAsync D2H: %.2f us (median)\n", 1e3 * ts[ts.size() / 2]);
    }
    return 0;
}
