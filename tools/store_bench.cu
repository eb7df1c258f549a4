// store_bench.cu -- calibrates B200 store throughput for the emission pattern
// of the neighbour write kernel (profiling aid, not part of libhdb).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void st128(uint4* p, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = make_uint4(i, i, i, i);
}
__global__ void st32(uint32_t* p, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        p[i] = (uint32_t)i;
}
// each warp-store writes `k` consecutive words starting at a running cursor
// (unaligned), mimicking a ballot-compacted emission of k hits.
__global__ void stk(uint32_t* p, uint64_t n, int k) {
    const int lane = threadIdx.x & 31;
    uint64_t w = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    uint64_t per = n / nw;
    uint64_t cur = w * per, end = cur + per - 32;
    while (cur < end) {
        if (lane < k) p[cur + lane] = (uint32_t)cur;
        cur += k;
    }
}
int main() {
    const uint64_t bytes = 5ull << 30;
    void* buf;
    cudaMalloc(&buf, bytes);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto run = [&](const char* name, auto f) {
        for (int it = 0; it < 2; ++it) f();
        cudaEventRecord(a);
        for (int it = 0; it < 5; ++it) f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("%-28s %8.3f ms/iter  %8.1f GB/s\n", name, ms / 5, bytes / (ms / 5 * 1e-3) / 1e9);
    };
    int g = 148 * 8;
    run("st128 coalesced", [&] { st128<<<g, 256>>>((uint4*)buf, bytes / 16); });
    run("st32 coalesced", [&] { st32<<<g, 256>>>((uint32_t*)buf, bytes / 4); });
    for (int k : {32, 27, 13, 7}) {
        char nm[64];
        snprintf(nm, sizeof nm, "stk k=%d (running cursor)", k);
        run(nm, [&] { stk<<<g, 256>>>((uint32_t*)buf, bytes / 4, k); });
    }
    cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
