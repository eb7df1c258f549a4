// lane_store_bench.cu -- store patterns of a query-per-lane emission (profiling aid,
// not part of libhdb): every lane of a warp owns one output list of L ids; the
// warp's 32 lists are consecutive (one reservation per warp), as in the table.
//   lane_scatter : per iteration every lane stores its next id at its own cursor
//                  (32 different lists per STG)
//   staged       : the warp's lists staged in shared memory, copied out with
//                  coalesced 16-B stores (the whole warp range is contiguous)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void lane_scatter(uint32_t* p, uint64_t n, int L) {
    const int lane = threadIdx.x & 31;
    const uint64_t w = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t span = 32ull * L;
    for (uint64_t base = w * span; base + span <= n; base += nw * span) {
        uint32_t* o = p + base + (uint64_t)lane * L;
        for (int i = 0; i < L; ++i) o[i] = (uint32_t)i;
    }
}
// same, but with a per-lane jitter of the list length (L +- L/4): lanes finish apart
__global__ void lane_scatter_jit(uint32_t* p, uint64_t n, int L) {
    const int lane = threadIdx.x & 31;
    const uint64_t w = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t span = 32ull * L;
    const int myL = L - L / 4 + (int)((lane * 7919u) % (unsigned)(L / 2 + 1));
    for (uint64_t base = w * span; base + span <= n; base += nw * span) {
        uint32_t* o = p + base + (uint64_t)lane * L;
        for (int i = 0; i < myL && i < L; ++i) o[i] = (uint32_t)i;
    }
}
__global__ void staged(uint32_t* p, uint64_t n, int L) {
    __shared__ __align__(16) uint32_t st[8][32 * 32 + 8];
    const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
    const uint64_t w = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const int Ls = L < 32 ? L : 32;
    const uint64_t span = 32ull * L;
    for (uint64_t base = w * span; base + span <= n; base += nw * span) {
        for (int done = 0; done < L; done += Ls) {
            for (int i = 0; i < Ls; ++i) st[wi][lane * Ls + i] = (uint32_t)i;   // per-lane STS
            __syncwarp();
            // copy the 32 runs of Ls words: run r goes to base + r*L + done
            for (int r = 0; r < 32; ++r) {
                uint32_t* o = p + base + (uint64_t)r * L + done;
                const int lim = L - done < Ls ? L - done : Ls;
                for (int j = lane; j < lim; j += 32) o[j] = st[wi][r * Ls + j];
            }
            __syncwarp();
        }
    }
}
int main() {
    const uint64_t bytes = 4ull << 30;
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
        printf("%-34s %8.3f ms/iter  %8.1f GB/s\n", name, ms / 5, bytes / (ms / 5 * 1e-3) / 1e9);
    };
    for (int blocks : {148 * 8, 148 * 16}) {
        for (int L : {12, 36, 128, 393}) {
            char nm[80];
            snprintf(nm, sizeof nm, "lane_scatter L=%d g=%d", L, blocks);
            run(nm, [&] { lane_scatter<<<blocks, 256>>>((uint32_t*)buf, bytes / 4, L); });
            snprintf(nm, sizeof nm, "lane_scatter_jit L=%d g=%d", L, blocks);
            run(nm, [&] { lane_scatter_jit<<<blocks, 256>>>((uint32_t*)buf, bytes / 4, L); });
            snprintf(nm, sizeof nm, "staged L=%d g=%d", L, blocks);
            run(nm, [&] { staged<<<blocks, 256>>>((uint32_t*)buf, bytes / 4, L); });
        }
    }
    cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
}
