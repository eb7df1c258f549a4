// kernels_scan.cu -- device exclusive scans (SURVEY 8(a) a4 cell offsets, a7
// neighbour-list offsets).  Reduce-then-scan over 2048-element tiles; inside a
// tile every thread scans 8 consecutive items serially, the warp combines its
// lanes with __shfl_up_sync and the CTA combines its 8 warp totals.  Block
// sums are scanned recursively, in place.  out[n] receives the total.
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

std::atomic<uint64_t> g_kernel_launches{0};

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int SC_THREADS = 256;
constexpr int SC_ITEMS = 8;
constexpr int SC_TILE = SC_THREADS * SC_ITEMS;

template <typename Tin, typename Tacc>
__global__ void __launch_bounds__(SC_THREADS) k_tile_reduce(const Tin* __restrict__ in, uint64_t n,
                                                            Tacc* __restrict__ sums) {
    __shared__ Tacc ws[SC_THREADS / 32];
    const uint64_t base = (uint64_t)blockIdx.x * SC_TILE;
    Tacc acc = 0;
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        uint64_t idx = base + (uint64_t)i * SC_THREADS + threadIdx.x;
        if (idx < n) acc += (Tacc)in[idx];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        Tacc t = 0;
#pragma unroll
        for (int w = 0; w < SC_THREADS / 32; ++w) t += ws[w];
        sums[blockIdx.x] = t;
    }
}

// Exclusive scan of one tile; thread t owns items [t*ITEMS, (t+1)*ITEMS) of the
// tile (blocked arrangement, loaded through shared memory for coalescing).
template <typename Tin, typename Tout>
__global__ void __launch_bounds__(SC_THREADS) k_tile_scan(const Tin* __restrict__ in, Tout* __restrict__ out,
                                                          uint64_t n, const Tout* __restrict__ offs) {
    __shared__ Tout buf[SC_TILE];
    __shared__ Tout wsum[SC_THREADS / 32];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const uint64_t base = (uint64_t)blockIdx.x * SC_TILE;
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        uint64_t idx = base + (uint64_t)i * SC_THREADS + tid;
        buf[i * SC_THREADS + tid] = idx < n ? (Tout)in[idx] : (Tout)0;
    }
    __syncthreads();
    Tout v[SC_ITEMS];
    Tout run = 0;
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        v[i] = run;
        run += buf[tid * SC_ITEMS + i];
    }
    // warp inclusive scan of per-thread totals
    Tout incl = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        Tout y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    Tout wpre = 0;
    Tout tot = 0;
#pragma unroll
    for (int i = 0; i < SC_THREADS / 32; ++i) {
        Tout t = wsum[i];
        wpre += (i < w) ? t : (Tout)0;
        tot += t;
    }
    const Tout boff = offs ? offs[blockIdx.x] : (Tout)0;
    const Tout pre = boff + wpre + (incl - run);
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) buf[tid * SC_ITEMS + i] = pre + v[i];
    __syncthreads();
#pragma unroll
    for (int i = 0; i < SC_ITEMS; ++i) {
        uint64_t idx = base + (uint64_t)i * SC_THREADS + tid;
        if (idx < n) out[idx] = buf[i * SC_THREADS + tid];
    }
    if (tid == 0 && base + SC_TILE >= n) out[n] = boff + tot;   // last tile writes the total
}

template <typename Tin, typename Tout>
void scan_rec(const Tin* in, Tout* out, uint64_t n, Tout* temp, cudaStream_t s) {
    if (n == 0) {
        cudaMemsetAsync(out, 0, sizeof(Tout), s);
        return;
    }
    uint64_t nb = (n + SC_TILE - 1) / SC_TILE;
    if (nb == 1) {
        k_tile_scan<Tin, Tout><<<1, SC_THREADS, 0, s>>>(in, out, n, nullptr);
        ++g_kernel_launches;
        return;
    }
    Tout* sums = temp;                 // nb + 1 entries
    Tout* next = temp + (nb + 1);
    k_tile_reduce<Tin, Tout><<<(unsigned)nb, SC_THREADS, 0, s>>>(in, n, sums);
    ++g_kernel_launches;
    scan_rec<Tout, Tout>(sums, sums, nb, next, s);   // in place
    k_tile_scan<Tin, Tout><<<(unsigned)nb, SC_THREADS, 0, s>>>(in, out, n, sums);
    ++g_kernel_launches;
}

}  // namespace

size_t scan_temp_bytes(uint64_t n) {
    size_t total = 0;
    while (n > (uint64_t)SC_TILE) {
        uint64_t nb = (n + SC_TILE - 1) / SC_TILE;
        total += (nb + 1) * sizeof(uint64_t);
        n = nb;
    }
    return total + 64;
}

void scan_u32_to_u32(const uint32_t* in, uint32_t* out, uint64_t n, void* temp, cudaStream_t s) {
    scan_rec<uint32_t, uint32_t>(in, out, n, (uint32_t*)temp, s);
}

void scan_u32_to_u64(const uint32_t* in, uint64_t* out, uint64_t n, void* temp, cudaStream_t s) {
    scan_rec<uint32_t, uint64_t>(in, out, n, (uint64_t*)temp, s);
}

}  // namespace hdb
