// kernels_grid.cu -- grid construction on sm_100a.
//
// ConstructIndex (Alg. 4 line 5; Sec. IV, Fig. 1): the paper
// bins D by unit cells, then builds G (one [A_min, A_max] range per cell of
// size eps x eps, linear id h) and the lookup array A of point ids.  Here:
//   a1  bbox      -- min/max reduce (+ finiteness check) of the input points
//   a2  keys      -- h = cy * nx + cx with cx = floor((x - xmin) * fl(1/w)) in FP64,
//                    w = eps_F * (1 + 2^-19) (reading R9: a width of exactly eps
//                    loses true neighbours to rounding)
//   a3  sort      -- stable LSD radix sort of (h, id) -> A (sorted pos -> id) and
//                    the points permuted into cell order (the paper's locality
//                    pre-sort, is subsumed)
//   a4  offsets   -- per-cell counts from run boundaries of the sorted keys, then a
//                    warp-shuffle exclusive scan -> dense half-open G (reading R11)
//   +   groups    -- query groups: <= 32 consecutive sorted queries of one cell,
//                    the unit of work of the search kernels.
#include <cuda_runtime.h>
#include <math.h>
#include <string.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

extern std::atomic<uint64_t> g_kernel_launches;

namespace {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ unsigned long long ord_encode(double v) {
    unsigned long long b = (unsigned long long)__double_as_longlong(v);
    return (b & 0x8000000000000000ull) ? ~b : (b | 0x8000000000000000ull);
}

template <typename T>
struct V2;
template <>
struct V2<double> {
    using type = double2;
};
template <>
struct V2<float> {
    using type = float2;
};

__global__ void k_bbox_init(unsigned long long* bb, unsigned int* bad) {
    bb[0] = ~0ull;  // xmin (ordered min)
    bb[1] = ~0ull;  // ymin
    bb[2] = 0ull;   // xmax (ordered max)
    bb[3] = 0ull;   // ymax
    *bad = 0;
}

template <typename T>
__global__ void __launch_bounds__(256) k_bbox(const typename V2<T>::type* __restrict__ xy, uint64_t n,
                                              unsigned long long* bb, unsigned int* bad) {
    double xmn = INFINITY, ymn = INFINITY, xmx = -INFINITY, ymx = -INFINITY;
    unsigned nb = 0;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        auto p = xy[i];
        double x = (double)p.x, y = (double)p.y;
        if (!isfinite(x) || !isfinite(y)) {
            ++nb;
            continue;
        }
        xmn = fmin(xmn, x);
        ymn = fmin(ymn, y);
        xmx = fmax(xmx, x);
        ymx = fmax(ymx, y);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        xmn = fmin(xmn, __shfl_xor_sync(FULL, xmn, o));
        ymn = fmin(ymn, __shfl_xor_sync(FULL, ymn, o));
        xmx = fmax(xmx, __shfl_xor_sync(FULL, xmx, o));
        ymx = fmax(ymx, __shfl_xor_sync(FULL, ymx, o));
        nb += __shfl_xor_sync(FULL, nb, o);
    }
    if ((threadIdx.x & 31) == 0) {
        if (xmn <= xmx) {
            atomicMin(&bb[0], ord_encode(xmn));
            atomicMin(&bb[1], ord_encode(ymn));
            atomicMax(&bb[2], ord_encode(xmx));
            atomicMax(&bb[3], ord_encode(ymx));
        }
        if (nb) atomicAdd(bad, nb);
    }
}

// a2: cell keys.  FP64 cell arithmetic with explicitly rounded ops (no FMA).
template <typename T>
__global__ void __launch_bounds__(256) k_keys(const typename V2<T>::type* __restrict__ xy, uint64_t n,
                                              double xmin, double ymin, double inv_w, uint32_t nx,
                                              uint32_t ny, uint32_t* __restrict__ keys,
                                              uint32_t* __restrict__ vals) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n;
         i += (uint64_t)gridDim.x * blockDim.x) {
        auto p = xy[i];
        double tx = floor(__dmul_rn(__dsub_rn((double)p.x, xmin), inv_w));
        double ty = floor(__dmul_rn(__dsub_rn((double)p.y, ymin), inv_w));
        uint32_t cx = (uint32_t)fmin(fmax(tx, 0.0), (double)(nx - 1));
        uint32_t cy = (uint32_t)fmin(fmax(ty, 0.0), (double)(ny - 1));
        keys[i] = cy * nx + cx;
        vals[i] = (uint32_t)i;
    }
}

// ---------------------------------------------------------------- radix sort
constexpr int RS_THREADS = 256;
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_ITEMS = 16;                         // per thread
constexpr int RS_TILE = RS_THREADS * RS_ITEMS;       // 4096 keys per CTA
constexpr int RS_BITS = 8;
constexpr int RS_BINS = 1 << RS_BITS;

__global__ void __launch_bounds__(RS_THREADS) k_radix_hist(const uint32_t* __restrict__ keys, uint64_t n,
                                                           int shift, uint32_t* __restrict__ hist,
                                                           uint32_t nblocks) {
    __shared__ uint32_t h[RS_BINS];
    const int tid = threadIdx.x;
    const int lane = tid & 31;
    h[tid] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE;
#pragma unroll 4
    for (int r = 0; r < RS_ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * RS_THREADS + tid;
        bool valid = idx < n;
        uint32_t d = valid ? ((keys[idx] >> shift) & (RS_BINS - 1)) : (0x100u + lane);
        unsigned peers = __match_any_sync(FULL, d);
        if (valid && lane == __ffs(peers) - 1) atomicAdd(&h[d], __popc(peers));
    }
    __syncthreads();
    hist[(uint64_t)tid * nblocks + blockIdx.x] = h[tid];
}

// Stable scatter: warp w owns keys [w*512, (w+1)*512) of the tile, processed in
// 16 rounds of 32 consecutive keys; the rank of a key is the number of earlier
// keys of the same digit in (earlier warps of the tile, earlier rounds of this
// warp, lower lanes of this round) plus the digit's global base for the tile.
__global__ void __launch_bounds__(RS_THREADS) k_radix_scatter(const uint32_t* __restrict__ kin,
                                                              const uint32_t* __restrict__ vin,
                                                              uint32_t* __restrict__ kout,
                                                              uint32_t* __restrict__ vout, uint64_t n,
                                                              int shift, const uint32_t* __restrict__ hscan,
                                                              uint32_t nblocks) {
    __shared__ uint32_t wcnt[RS_WARPS][RS_BINS];
    __shared__ uint32_t gbase[RS_BINS];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) wcnt[i][tid] = 0;
    gbase[tid] = hscan[(uint64_t)tid * nblocks + blockIdx.x];
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * RS_TILE + (uint64_t)w * (RS_ITEMS * 32);
    const unsigned lt = (1u << lane) - 1u;
    uint32_t key[RS_ITEMS], val[RS_ITEMS], rank[RS_ITEMS];
#pragma unroll
    for (int r = 0; r < RS_ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * 32 + lane;
        bool valid = idx < n;
        key[r] = valid ? kin[idx] : 0u;
        val[r] = valid ? vin[idx] : 0u;
        uint32_t d = valid ? ((key[r] >> shift) & (RS_BINS - 1)) : (0x100u + lane);
        unsigned peers = __match_any_sync(FULL, d);
        uint32_t before = valid ? wcnt[w][d] : 0u;
        rank[r] = before + __popc(peers & lt);
        __syncwarp();
        if (valid && lane == __ffs(peers) - 1) wcnt[w][d] = before + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    {
        uint32_t s = 0;
#pragma unroll
        for (int i = 0; i < RS_WARPS; ++i) {
            uint32_t t = wcnt[i][tid];
            wcnt[i][tid] = s;
            s += t;
        }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < RS_ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * 32 + lane;
        if (idx < n) {
            uint32_t d = (key[r] >> shift) & (RS_BINS - 1);
            uint32_t pos = gbase[d] + wcnt[w][d] + rank[r];
            kout[pos] = key[r];
            vout[pos] = val[r];
        }
    }
}

template <typename T>
__global__ void __launch_bounds__(256) k_gather(const typename V2<T>::type* __restrict__ in,
                                                const uint32_t* __restrict__ ids, uint64_t n,
                                                typename V2<T>::type* __restrict__ out) {
    for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < n;
         s += (uint64_t)gridDim.x * blockDim.x)
        out[s] = in[ids[s]];
}

// a4 histogram from run boundaries of the sorted keys: one atomic per
// (warp, run) -- dense cells cost one atomic per 32 points.
__global__ void __launch_bounds__(256) k_cell_counts(const uint32_t* __restrict__ keys, uint64_t n,
                                                     uint32_t* __restrict__ cnt,
                                                     unsigned long long* __restrict__ nonempty) {
    const int lane = threadIdx.x & 31;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    // uniform trip count per warp so that __match_any_sync sees all lanes
    for (uint64_t base = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) - lane; base < n;
         base += stride) {
        uint64_t s = base + lane;
        bool valid = s < n;
        uint32_t k = valid ? keys[s] : 0xffffffffu;
        unsigned peers = __match_any_sync(FULL, k);
        if (valid && lane == __ffs(peers) - 1) atomicAdd(&cnt[k], (uint32_t)__popc(peers));
        bool first = valid && (s == 0 || keys[s - 1] != k);
        unsigned fm = __ballot_sync(FULL, first);
        if (lane == 0 && fm) atomicAdd(nonempty, (unsigned long long)__popc(fm));
    }
}

__global__ void __launch_bounds__(256) k_group_flags(const uint32_t* __restrict__ keys,
                                                     const uint32_t* __restrict__ start, uint64_t n,
                                                     uint32_t* __restrict__ flags) {
    for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < n;
         s += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t c0 = start[keys[s]];
        flags[s] = ((uint32_t)s - c0) % (uint32_t)kGroup == 0 ? 1u : 0u;
    }
}

__global__ void __launch_bounds__(256) k_group_scatter(const uint32_t* __restrict__ flags,
                                                       const uint32_t* __restrict__ pos, uint64_t n,
                                                       uint32_t* __restrict__ gstart) {
    for (uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; s < n;
         s += (uint64_t)gridDim.x * blockDim.x)
        if (flags[s]) gstart[pos[s]] = (uint32_t)s;
    if (blockIdx.x == 0 && threadIdx.x == 0) gstart[pos[n]] = (uint32_t)n;
}

inline unsigned grid_for(uint64_t n, int threads = 256, unsigned cap = 148u * 16u) {
    uint64_t b = (n + threads - 1) / threads;
    if (b < 1) b = 1;
    return (unsigned)(b < cap ? b : cap);
}

}  // namespace

double bbox_decode(unsigned long long v, bool) {
    unsigned long long b = (v & 0x8000000000000000ull) ? (v & ~0x8000000000000000ull) : ~v;
    double d;
    memcpy(&d, &b, sizeof d);
    return d;
}

void launch_bbox_init(unsigned long long* bb, unsigned int* bad, cudaStream_t s) {
    k_bbox_init<<<1, 1, 0, s>>>(bb, bad);
    ++g_kernel_launches;
}

void launch_bbox(const void* xy, uint64_t n, hdb_dtype dt, unsigned long long* bb, unsigned int* bad,
                 cudaStream_t s) {
    if (n == 0) return;
    if (dt == HDB_F64)
        k_bbox<double><<<grid_for(n, 256, 148 * 8), 256, 0, s>>>((const double2*)xy, n, bb, bad);
    else
        k_bbox<float><<<grid_for(n, 256, 148 * 8), 256, 0, s>>>((const float2*)xy, n, bb, bad);
    ++g_kernel_launches;
}

void launch_keys(const void* xy, uint64_t n, hdb_dtype dt, double xmin, double ymin, double inv_w,
                 uint32_t nx, uint32_t ny, uint32_t* keys, uint32_t* vals, cudaStream_t s) {
    if (n == 0) return;
    if (dt == HDB_F64)
        k_keys<double><<<grid_for(n), 256, 0, s>>>((const double2*)xy, n, xmin, ymin, inv_w, nx, ny, keys, vals);
    else
        k_keys<float><<<grid_for(n), 256, 0, s>>>((const float2*)xy, n, xmin, ymin, inv_w, nx, ny, keys, vals);
    ++g_kernel_launches;
}

size_t radix_sort_temp_bytes(uint64_t n) {
    uint64_t nblocks = (n + RS_TILE - 1) / RS_TILE;
    uint64_t m = nblocks * RS_BINS;
    return (m + 1) * sizeof(uint32_t) * 2 + scan_temp_bytes(m) + 256;
}

int radix_sort_pairs(uint32_t* k0, uint32_t* v0, uint32_t* k1, uint32_t* v1, uint64_t n, int bits, void* temp,
                     cudaStream_t s) {
    if (n <= 1 || bits <= 0) return 0;
    uint32_t nblocks = (uint32_t)((n + RS_TILE - 1) / RS_TILE);
    uint64_t m = (uint64_t)nblocks * RS_BINS;
    uint32_t* hist = (uint32_t*)temp;
    uint32_t* hscan = hist + (m + 1);
    void* stemp = (void*)(((uintptr_t)(hscan + m + 1) + 255) & ~(uintptr_t)255);
    int cur = 0;
    for (int shift = 0; shift < bits; shift += RS_BITS) {
        uint32_t* ki = cur ? k1 : k0;
        uint32_t* vi = cur ? v1 : v0;
        uint32_t* ko = cur ? k0 : k1;
        uint32_t* vo = cur ? v0 : v1;
        k_radix_hist<<<nblocks, RS_THREADS, 0, s>>>(ki, n, shift, hist, nblocks);
        ++g_kernel_launches;
        scan_u32_to_u32(hist, hscan, m, stemp, s);
        k_radix_scatter<<<nblocks, RS_THREADS, 0, s>>>(ki, vi, ko, vo, n, shift, hscan, nblocks);
        ++g_kernel_launches;
        cur ^= 1;
    }
    return cur;
}

void launch_gather_points(const void* xy_in, const uint32_t* ids, uint64_t n, hdb_dtype dt, void* xy_s,
                          cudaStream_t s) {
    if (n == 0) return;
    if (dt == HDB_F64)
        k_gather<double><<<grid_for(n), 256, 0, s>>>((const double2*)xy_in, ids, n, (double2*)xy_s);
    else
        k_gather<float><<<grid_for(n), 256, 0, s>>>((const float2*)xy_in, ids, n, (float2*)xy_s);
    ++g_kernel_launches;
}

void launch_cell_counts(const uint32_t* keys_sorted, uint64_t n, uint32_t* cell_cnt,
                        unsigned long long* n_nonempty, cudaStream_t s) {
    if (n == 0) return;
    k_cell_counts<<<grid_for(n), 256, 0, s>>>(keys_sorted, n, cell_cnt, n_nonempty);
    ++g_kernel_launches;
}

void launch_group_flags(const uint32_t* keys_sorted, const uint32_t* start, uint64_t n, uint32_t* flags,
                        cudaStream_t s) {
    if (n == 0) return;
    k_group_flags<<<grid_for(n), 256, 0, s>>>(keys_sorted, start, n, flags);
    ++g_kernel_launches;
}

void launch_group_scatter(const uint32_t* flags, const uint32_t* pos, uint64_t n, uint32_t* gstart,
                          cudaStream_t s) {
    k_group_scatter<<<grid_for(n), 256, 0, s>>>(flags, pos, n, gstart);
    ++g_kernel_launches;
}

}  // namespace hdb
