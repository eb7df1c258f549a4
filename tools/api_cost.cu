// api_cost.cu -- host cost of the CUDA runtime calls the grid build issues
// (profiling aid, not part of libhdb): stream-ordered alloc/free pairs, memsets,
// tiny kernel launches, D2H readback + stream sync round trips.
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k_empty(int* p) { if (p && threadIdx.x == 1234567) *p = 1; }
int main() {
    cudaStream_t s; cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking);
    cudaMemPool_t pool; cudaDeviceGetDefaultMemPool(&pool, 0);
    uint64_t thr = ~0ull; cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    void* h; cudaHostAlloc(&h, 64, 0);
    int* d; cudaMalloc(&d, 1 << 20);
    auto now = [] { return std::chrono::steady_clock::now(); };
    auto us = [](auto a, auto b) { return std::chrono::duration<double, std::micro>(b - a).count(); };
    const int N = 2000;
    for (int rep = 0; rep < 2; ++rep) {
        void* ps[16];
        auto t0 = now();
        for (int i = 0; i < N; ++i) { for (int j = 0; j < 16; ++j) cudaMallocAsync(&ps[j], (size_t)(j + 1) << 20, s); for (int j = 0; j < 16; ++j) cudaFreeAsync(ps[j], s); }
        auto t1 = now();
        for (int i = 0; i < N * 16; ++i) cudaMemsetAsync(d, 0, 64, s);
        auto t2 = now();
        for (int i = 0; i < N * 16; ++i) k_empty<<<148, 256, 0, s>>>(d);
        auto t3 = now();
        cudaStreamSynchronize(s);
        auto t4 = now();
        for (int i = 0; i < N; ++i) { cudaMemcpyAsync(h, d, 8, cudaMemcpyDeviceToHost, s); cudaStreamSynchronize(s); }
        auto t5 = now();
        for (int i = 0; i < N; ++i) { k_empty<<<148, 256, 0, s>>>(d); cudaStreamSynchronize(s); }
        auto t6 = now();
        if (rep) printf("alloc+free pair %.2f us | memset %.2f us | launch %.2f us | D2H 8B + sync %.2f us | launch + sync %.2f us\n",
                        us(t0, t1) / (N * 16), us(t1, t2) / (N * 16), us(t2, t3) / (N * 16), us(t4, t5) / N, us(t5, t6) / N);
    }
    return 0;
}
