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
//   a4  offsets   -- run boundaries of the sorted keys + a warp-shuffle exclusive
//                    scan -> G restricted to the NON-EMPTY cells: (key, start) pairs,
//                    half-open (reading R11); sparse extents cost nothing
//   +   spans     -- for every non-empty cell, its 2k+1 stencil row spans (cells of
//                    width eps/k): with row-major keys the cells (cx-k..cx+k, y')
//                    are consecutive in key order, so each stencil row is one
//                    contiguous range of sorted positions (binary search)
//   +   groups    -- query groups: <= 32 consecutive sorted queries of one cell,
//                    the unit of work of the search kernels.
#include <cuda_runtime.h>
#include <math.h>
#include <string.h>
#include <stdint.h>

#include <algorithm>

#include "cellkey.cuh"
#include "internal.h"

namespace hdb {

extern std::atomic<uint64_t> g_kernel_launches;

namespace {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ unsigned long long ord_encode(double v) {
    unsigned long long b = (unsigned long long)__double_as_longlong(v);
    return (b & 0x8000000000000000ull) ? ~b : (b | 0x8000000000000000ull);
}


// One launch initialises the bbox reduction, the zeroed words of the build's misc
// buffer (bb[4..nz): counters, occupancy sums, cost histogram) and the
// occupancy-estimate hash table (it replaced a kernel + six memsets: each stream
// op costs several us at C2 sizes)
__global__ void k_bbox_init(unsigned long long* bb, uint32_t nz, unsigned long long* hkey, unsigned int* hcnt,
                            uint32_t tsize) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i == 0) {
        bb[0] = ~0ull;  // xmin (ordered min)
        bb[1] = ~0ull;  // ymin
        bb[2] = 0ull;   // xmax (ordered max)
        bb[3] = 0ull;   // ymax
    }
    if (i >= 4 && i < nz) bb[i] = 0ull;
    for (uint32_t j = i; j < tsize; j += gridDim.x * blockDim.x) {
        hkey[j] = ~0ull;
        hcnt[j] = 0;
    }
}

template <typename T>
__global__ void __launch_bounds__(256) k_bbox(const typename V2<T>::type* __restrict__ xy, uint64_t n,
                                              unsigned long long* bb, unsigned int* bad) {
    double xmn = INFINITY, ymn = INFINITY, xmx = -INFINITY, ymx = -INFINITY;
    unsigned nb = 0;
    auto take = [&](typename V2<T>::type p) {
        const double x = (double)p.x, y = (double)p.y;
        if (!isfinite(x) || !isfinite(y)) {
            ++nb;
            return;
        }
        xmn = fmin(xmn, x);
        ymn = fmin(ymn, y);
        xmx = fmax(xmx, x);
        ymx = fmax(ymx, y);
    };
    // four independent loads in flight per thread (the reduction streams the whole input)
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    for (; i + 3 * stride < n; i += 4 * stride) {
        const auto p0 = xy[i], p1 = xy[i + stride], p2 = xy[i + 2 * stride], p3 = xy[i + 3 * stride];
        take(p0);
        take(p1);
        take(p2);
        take(p3);
    }
    for (; i < n; i += stride) take(xy[i]);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        xmn = fmin(xmn, __shfl_xor_sync(FULL, xmn, o));
        ymn = fmin(ymn, __shfl_xor_sync(FULL, ymn, o));
        xmx = fmax(xmx, __shfl_xor_sync(FULL, xmx, o));
        ymx = fmax(ymx, __shfl_xor_sync(FULL, ymx, o));
        nb += __shfl_xor_sync(FULL, nb, o);
    }
    // block reduction, then one set of atomics per block (per-warp atomics on the same four
    // words serialised at the L2: 31 us of a 1.86M-point bbox)
    __shared__ double red[5][8];
    const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) {
        red[0][w] = xmn;
        red[1][w] = ymn;
        red[2][w] = xmx;
        red[3][w] = ymx;
        red[4][w] = (double)nb;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int i = 1; i < (int)(blockDim.x >> 5); ++i) {
            xmn = fmin(xmn, red[0][i]);
            ymn = fmin(ymn, red[1][i]);
            xmx = fmax(xmx, red[2][i]);
            ymx = fmax(ymx, red[3][i]);
            nb += (unsigned)red[4][i];
        }
        if (xmn <= xmx) {
            atomicMin(&bb[0], ord_encode(xmn));
            atomicMin(&bb[1], ord_encode(ymn));
            atomicMax(&bb[2], ord_encode(xmx));
            atomicMax(&bb[3], ord_encode(ymx));
        }
        if (nb) atomicAdd(bad, nb);
    }
}

// ---------------------------------------------------------------- radix sort
// Stable LSD radix sort of (key, id), 8-bit digits.  Per pass: a per-tile digit
// histogram, a scan of the (digit, tile) counts, and a scatter that ranks each
// tile's keys stably (warp match_any ranks + warp-ordered prefixes), stages them
// in shared memory in digit order, and writes every digit's run of the tile
// contiguously (coalesced) to its global position.
constexpr int RS_THREADS = 256;
constexpr int RS_WARPS = RS_THREADS / 32;
constexpr int RS_BITS = 8;
constexpr int RS_BINS = 1 << RS_BITS;
template <typename K>
struct RsCfg {
    static constexpr int ITEMS = sizeof(K) == 4 ? 16 : 8;       // per thread
    static constexpr int TILE = RS_THREADS * ITEMS;             // 4096 (u32) / 2048 (u64) keys per CTA
};

template <typename K>
__global__ void __launch_bounds__(RS_THREADS) k_radix_hist(const K* __restrict__ keys, uint64_t n, int shift,
                                                           uint32_t* __restrict__ hist, uint32_t nblocks) {
    constexpr int ITEMS = RsCfg<K>::ITEMS, TILE = RsCfg<K>::TILE;
    __shared__ uint32_t h[RS_WARPS][RS_BINS];   // warp-private counters (no match_any)
    const int tid = threadIdx.x, w = tid >> 5;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) h[i][tid] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * TILE;
#pragma unroll 4
    for (int r = 0; r < ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * RS_THREADS + tid;
        if (idx < n) atomicAdd(&h[w][(uint32_t)((keys[idx] >> shift) & (RS_BINS - 1))], 1u);
    }
    __syncthreads();
    uint32_t t = 0;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) t += h[i][tid];
    hist[(uint64_t)tid * nblocks + blockIdx.x] = t;
}

template <typename K>
__global__ void __launch_bounds__(RS_THREADS) k_radix_scatter(const K* __restrict__ kin,
                                                              const uint32_t* __restrict__ vin,
                                                              K* __restrict__ kout, uint32_t* __restrict__ vout,
                                                              uint64_t n, int shift,
                                                              const uint32_t* __restrict__ hscan, uint32_t nblocks) {
    constexpr int ITEMS = RsCfg<K>::ITEMS, TILE = RsCfg<K>::TILE;
    __shared__ uint32_t wcnt[RS_WARPS][RS_BINS];
    __shared__ uint32_t gbase[RS_BINS];     // global start of each digit's run of this tile
    __shared__ uint32_t dstart[RS_BINS];    // tile-local start of each digit
    __shared__ K skey[TILE];
    __shared__ uint32_t sval[TILE];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) wcnt[i][tid] = 0;
    gbase[tid] = hscan[(uint64_t)tid * nblocks + blockIdx.x];
    __syncthreads();
    const uint64_t tbase = (uint64_t)blockIdx.x * TILE;
    const uint64_t base = tbase + (uint64_t)w * (ITEMS * 32);
    const unsigned lt = (1u << lane) - 1u;
    K key[ITEMS];
    uint32_t val[ITEMS], rank[ITEMS];
#pragma unroll
    for (int r = 0; r < ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * 32 + lane;
        bool valid = idx < n;
        key[r] = valid ? kin[idx] : (K)0;
        val[r] = valid ? vin[idx] : 0u;
        uint32_t d = valid ? (uint32_t)((key[r] >> shift) & (RS_BINS - 1)) : (0x100u + lane);
        unsigned peers = __match_any_sync(FULL, d);
        uint32_t before = valid ? wcnt[w][d] : 0u;
        rank[r] = before + __popc(peers & lt);
        __syncwarp();
        if (valid && lane == __ffs(peers) - 1) wcnt[w][d] = before + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive prefix over the warps, and the digit's tile total
    uint32_t tot = 0;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) {
        uint32_t t = wcnt[i][tid];
        wcnt[i][tid] = tot;
        tot += t;
    }
    // exclusive scan of the 256 digit totals (warp shuffles + the 8 warp sums)
    __shared__ uint32_t wsum[RS_WARPS];
    uint32_t incl = tot;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    uint32_t wpre = 0;
#pragma unroll
    for (int i = 0; i < RS_WARPS; ++i) wpre += i < w ? wsum[i] : 0u;
    dstart[tid] = wpre + incl - tot;
    __syncthreads();
    // stage in digit order
#pragma unroll
    for (int r = 0; r < ITEMS; ++r) {
        uint64_t idx = base + (uint64_t)r * 32 + lane;
        if (idx < n) {
            uint32_t d = (uint32_t)((key[r] >> shift) & (RS_BINS - 1));
            uint32_t lp = dstart[d] + wcnt[w][d] + rank[r];
            skey[lp] = key[r];
            sval[lp] = val[r];
        }
    }
    __syncthreads();
    // write each digit's run contiguously
    const uint32_t cnt = (uint32_t)min((uint64_t)TILE, n - tbase);
    for (uint32_t i = tid; i < cnt; i += RS_THREADS) {
        const K k = skey[i];
        const uint32_t d = (uint32_t)((k >> shift) & (RS_BINS - 1));
        const uint32_t pos = gbase[d] + (i - dstart[d]);
        kout[pos] = k;
        vout[pos] = sval[i];
    }
}

// ---------------------------------------------------------------- process-shard bands (8(e))
// A process shard (torchrun rank r of R) takes a band of cell ROWS [Y_r, Y_{r+1}) of the
// global grid as its queries; it needs the points of those rows plus k halo rows on either
// side as candidates, and sorts only those (the grid build is no longer replicated).  The
// bands balance a load estimate per row: the sum of squared cell occupancies (the work of
// a cell's queries grows with its population), from a dense cell histogram.
// One pass over the input: every point's cell row -> rowid[i] (read again by the band
// selection instead of the coordinates), exact row counts (per-block shared histogram
// when the rows fit, else global atomics), and, for every kRowSample-th point, its cell
// in the sampled cell histogram (the load estimate needs only a sample; one atomic per
// point into tens of MB of counters cost 0.36 ms at C5)
constexpr uint32_t kRowSample = 16;
constexpr uint32_t kRowSmem = 8192;   // rows counted in shared memory (32 KB)
template <typename T>
__global__ void __launch_bounds__(256) k_band_hist(const typename V2<T>::type* __restrict__ xy, uint64_t n,
                                                   KeyParams kp, uint32_t* __restrict__ rowid,
                                                   unsigned long long* __restrict__ row_cnt,
                                                   uint32_t* __restrict__ cell_cnt) {
    __shared__ uint32_t rh[kRowSmem];
    const bool smem = kp.ny <= kRowSmem;
    if (smem)
        for (uint32_t y = threadIdx.x; y < kp.ny; y += blockDim.x) rh[y] = 0;
    __syncthreads();
    // four points per thread and step, loaded before any atomic (latency hiding)
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i0 < n; i0 += 4 * stride) {
        typename V2<T>::type p[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t i = i0 + u * stride;
            if (i < n) p[u] = xy[i];
        }
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const uint64_t i = i0 + u * stride;
            if (i >= n) break;
            uint64_t cx, cy;
            cell_xy<T>(p[u], kp, cx, cy);
            rowid[i] = (uint32_t)cy;
            if (smem) atomicAdd(&rh[cy], 1u);
            else atomicAdd(&row_cnt[cy], 1ull);
            if (cell_cnt && i % kRowSample == 0) atomicAdd(&cell_cnt[cy * kp.nx + cx], 1u);
        }
    }
    if (smem) {
        __syncthreads();
        for (uint32_t y = threadIdx.x; y < kp.ny; y += blockDim.x)
            if (rh[y]) atomicAdd(&row_cnt[y], (unsigned long long)rh[y]);
    }
}

// one warp per row: row_load[y] = sum of the sampled cell counts' squares, with the
// sampling bias removed: E[s^2] = f^2 m^2 + f (1 - f) m for a cell of m points, so
// (s^2 - (1 - f) s) / f^2 estimates m^2 (scaled by 2^8 to keep fractions in integers)
__global__ void __launch_bounds__(256) k_row_load(const uint32_t* __restrict__ cell_cnt, uint32_t nx, uint32_t ny,
                                                  unsigned long long* __restrict__ row_load) {
    const int lane = threadIdx.x & 31;
    const double f = 1.0 / kRowSample;
    for (uint64_t y = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5; y < ny;
         y += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
        double l = 0;
        for (uint32_t x = lane; x < nx; x += 32) {
            const double v = cell_cnt[y * nx + x];
            l += fmax(v * v - (1.0 - f) * v, 0.0) / (f * f);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(FULL, l, o);
        if (lane == 0) row_load[y] = (unsigned long long)(l * 256.0);
    }
}

// the shard's query groups: the cells with keys in [key_lo, key_hi) -> groups
// [gofs[c0], gofs[c1]) (out[0], out[1])
__global__ void k_band_groups(const uint64_t* __restrict__ ckey, uint64_t nne, const uint32_t* __restrict__ gofs,
                              uint64_t key_lo, uint64_t key_hi, unsigned long long* __restrict__ out) {
    auto lb = [&](uint64_t k) {
        uint64_t lo = 0, hi = nne;
        while (lo < hi) {
            const uint64_t mid = (lo + hi) >> 1;
            if (ckey[mid] < k) lo = mid + 1;
            else hi = mid;
        }
        return lo;
    };
    out[0] = gofs[lb(key_lo)];
    out[1] = gofs[lb(key_hi)];
}

// ---------------------------------------------------------------- point sort (a2 + a3 + gather)
// The points sorted by cell key with a stable LSD radix sort (8-bit digits)
// whose passes carry the whole record (key, id, xy): the first pass reads the
// INPUT points in input order and computes their keys (a2) on the fly (id =
// input row), the last pass writes the sorted keys, A (sorted pos -> id), the
// sorted points and their f32 filter copy.  This replaces keys -> (key, id) sort
// -> gather: the gather's random reads of the input points (1.4 ms at C5's 50M
// points) are gone, every pass streams coalesced digit runs.  Per pass: a
// per-tile digit histogram (warp-private shared counters, no match_any), a scan
// of the (digit, tile) counts, and the scatter (stable warp match_any ranks,
// staging in shared memory in digit order, coalesced runs).
constexpr int PS_THREADS = 256;
constexpr int PS_WARPS = PS_THREADS / 32;
#ifndef HDB_PS_ITEMS
#define HDB_PS_ITEMS 8
#endif
constexpr int PS_ITEMS = HDB_PS_ITEMS;
constexpr int PS_TILE = PS_THREADS * PS_ITEMS;   // 2048 records per CTA

template <typename T, typename K, bool FROM_POINTS>
__global__ void __launch_bounds__(PS_THREADS) k_ps_hist(const typename V2<T>::type* __restrict__ xy,
                                                        const K* __restrict__ keys, KeyParams kp, uint64_t n,
                                                        int shift, uint32_t* __restrict__ hist, uint32_t nblocks) {
    __shared__ uint32_t h[PS_WARPS][RS_BINS];
    const int tid = threadIdx.x, w = tid >> 5;
#pragma unroll
    for (int i = 0; i < PS_WARPS; ++i) h[i][tid] = 0;
    __syncthreads();
    const uint64_t base = (uint64_t)blockIdx.x * PS_TILE;
    // all loads first, then the shared atomics (an atomic between two loads would keep
    // the next load from being issued early: one DRAM latency per item)
    K kr[PS_ITEMS];
#pragma unroll
    for (int r = 0; r < PS_ITEMS; ++r) {
        const uint64_t idx = base + (uint64_t)r * PS_THREADS + tid;
        if (FROM_POINTS) {
            typename V2<T>::type p{0, 0};
            if (idx < n) p = xy[idx];
            kr[r] = cell_key<T, K>(p, kp);
        } else {
            kr[r] = idx < n ? keys[idx] : (K)0;
        }
    }
#pragma unroll
    for (int r = 0; r < PS_ITEMS; ++r)
        if (base + (uint64_t)r * PS_THREADS + tid < n) atomicAdd(&h[w][(uint32_t)((kr[r] >> shift) & (RS_BINS - 1))], 1u);
    __syncthreads();
    uint32_t t = 0;
#pragma unroll
    for (int i = 0; i < PS_WARPS; ++i) t += h[i][tid];
    hist[(uint64_t)tid * nblocks + blockIdx.x] = t;
}

template <typename T, typename K>
constexpr size_t ps_smem_bytes() {
    return (size_t)PS_TILE * (sizeof(typename V2<T>::type) + sizeof(K) + 4) + (PS_WARPS + 2) * RS_BINS * 4;
}

template <typename T, typename K, bool FIRST, bool LAST>
#ifndef HDB_PS_MINB
#define HDB_PS_MINB 3   // 3 CTAs per SM (80 registers, small spills): C5 grid build 3.80 -> 3.55 ms
#endif
__global__ void __launch_bounds__(PS_THREADS, HDB_PS_MINB) k_ps_scatter(const typename V2<T>::type* __restrict__ xyin,
                                                           const K* __restrict__ kin, const uint32_t* __restrict__ vin,
                                                           KeyParams kp, K* __restrict__ kout,
                                                           uint32_t* __restrict__ vout,
                                                           typename V2<T>::type* __restrict__ xyout,
                                                           float4* __restrict__ xp, double ox, double oy, uint64_t n,
                                                           int shift, const uint32_t* __restrict__ hscan,
                                                           uint32_t nblocks, unsigned int* __restrict__ counters,
                                                           uint32_t n_counters, const uint32_t* __restrict__ gid) {
    using P2 = typename V2<T>::type;
    extern __shared__ __align__(16) unsigned char ps_smem[];
    P2* sxy = (P2*)ps_smem;
    K* skey = (K*)(sxy + PS_TILE);
    uint32_t* sval = (uint32_t*)(skey + PS_TILE);
    uint32_t(*wcnt)[RS_BINS] = (uint32_t(*)[RS_BINS])(sval + PS_TILE);
    uint32_t* gbase = (uint32_t*)(wcnt + PS_WARPS);   // global start of each digit's run of this tile
    uint32_t* dstart = gbase + RS_BINS;                // tile-local start of each digit
    __shared__ uint32_t wsum[PS_WARPS];
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
#pragma unroll
    for (int i = 0; i < PS_WARPS; ++i) wcnt[i][tid] = 0;
    gbase[tid] = hscan[(uint64_t)tid * nblocks + blockIdx.x];
    if (LAST && blockIdx.x == 0) {
        // padding read by the candidate-pair loads (2 entries past n) and the work counters
        if (tid < 2) {
            xyout[n + tid] = P2{0, 0};
            vout[n + tid] = 0;
        }
        float* xpf = (float*)xp;
        for (uint64_t q = n + tid; q < 2 * (n / 2 + 2); q += PS_THREADS) {
            xpf[4 * (q >> 1) + (q & 1)] = 0.f;
            xpf[4 * (q >> 1) + 2 + (q & 1)] = 0.f;
        }
        for (uint32_t c = tid; c < n_counters; c += PS_THREADS) counters[c] = 0;
    }
    __syncthreads();
    const uint64_t tbase = (uint64_t)blockIdx.x * PS_TILE;
    const uint64_t base = tbase + (uint64_t)w * (PS_ITEMS * 32);
    const unsigned lt = (1u << lane) - 1u;
    K key[PS_ITEMS];
    uint32_t val[PS_ITEMS], rank[PS_ITEMS];
    P2 pt[PS_ITEMS];
#pragma unroll
    for (int r = 0; r < PS_ITEMS; ++r) {
        const uint64_t idx = base + (uint64_t)r * 32 + lane;
        const bool valid = idx < n;
        pt[r] = valid ? xyin[idx] : P2{0, 0};
        if (FIRST) {
            key[r] = valid ? cell_key<T, K>(pt[r], kp) : (K)0;
            val[r] = gid ? (valid ? gid[idx] : 0u) : (uint32_t)idx;   // id = input row (or its global id)
        } else {
            key[r] = valid ? kin[idx] : (K)0;
            val[r] = valid ? vin[idx] : 0u;
        }
    }
#pragma unroll
    for (int r = 0; r < PS_ITEMS; ++r) {
        const bool valid = base + (uint64_t)r * 32 + lane < n;
        const uint32_t d = valid ? (uint32_t)((key[r] >> shift) & (RS_BINS - 1)) : (0x100u + lane);
        const unsigned peers = __match_any_sync(FULL, d);
        const uint32_t before = valid ? wcnt[w][d] : 0u;
        rank[r] = before + __popc(peers & lt);
        __syncwarp();
        if (valid && lane == __ffs(peers) - 1) wcnt[w][d] = before + __popc(peers);
        __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive prefix over the warps, and the digit's tile total
    uint32_t tot = 0;
#pragma unroll
    for (int i = 0; i < PS_WARPS; ++i) {
        const uint32_t t = wcnt[i][tid];
        wcnt[i][tid] = tot;
        tot += t;
    }
    uint32_t incl = tot;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    if (lane == 31) wsum[w] = incl;
    __syncthreads();
    uint32_t wpre = 0;
#pragma unroll
    for (int i = 0; i < PS_WARPS; ++i) wpre += i < w ? wsum[i] : 0u;
    dstart[tid] = wpre + incl - tot;
    __syncthreads();
    // stage in digit order
#pragma unroll
    for (int r = 0; r < PS_ITEMS; ++r) {
        if (base + (uint64_t)r * 32 + lane < n) {
            const uint32_t d = (uint32_t)((key[r] >> shift) & (RS_BINS - 1));
            const uint32_t lp = dstart[d] + wcnt[w][d] + rank[r];
            skey[lp] = key[r];
            sval[lp] = val[r];
            sxy[lp] = pt[r];
        }
    }
    __syncthreads();
    // write each digit's run contiguously
    const uint32_t cnt = (uint32_t)min((uint64_t)PS_TILE, n - tbase);
    float* xpf = (float*)xp;
    for (uint32_t i = tid; i < cnt; i += PS_THREADS) {
        const K k = skey[i];
        const uint32_t d = (uint32_t)((k >> shift) & (RS_BINS - 1));
        const uint64_t pos = gbase[d] + (i - dstart[d]);
        const P2 p = sxy[i];
        kout[pos] = k;
        vout[pos] = sval[i];
        xyout[pos] = p;
        if (LAST) {
            // xp: paired-SoA f32 copy {x_2k, x_2k+1, y_2k, y_2k+1} -- f64 input: filter
            // coordinates fl32(fl64(x - ox)); f32 input: the exact coordinates
            float fx, fy;
            if (sizeof(p.x) == 8) {
                fx = (float)__dsub_rn((double)p.x, ox);
                fy = (float)__dsub_rn((double)p.y, oy);
            } else {
                fx = (float)p.x;
                fy = (float)p.y;
            }
            xpf[4 * (pos >> 1) + (pos & 1)] = fx;
            xpf[4 * (pos >> 1) + 2 + (pos & 1)] = fy;
        }
    }
}

// first index i in [lo, hi) with ckey[i] >= k (hi if none)
__device__ __forceinline__ uint64_t lower_bound_u64(const uint64_t* __restrict__ a, uint64_t lo, uint64_t hi,
                                                    uint64_t k) {
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (__ldg(&a[mid]) < k)
            lo = mid + 1;
        else
            hi = mid;
    }
    return lo;
}

// Stencil row spans of every non-empty cell c (cx, cy): with cells of width
// w = eps_F (1 + 2^-19) / k, a neighbour lies at most k cells away, so for each
// of the 2k+1 rows y' in cy-k..cy+k the span covers the sorted positions of
// cells (max(cx-k,0) .. min(cx+k,nx-1), y') -- consecutive keys, one
// contiguous range, found by two binary searches over the non-empty keys
// (rows below cy precede c, rows above follow it).  Also gcount[c] = number of
// 32-query groups of the cell.
// cnext (optional): the paper's dense G over all cells (Fig. 1) in lookup form,
// cnext[h] = index of the first non-empty cell with key >= h, h <= nx*ny --
// then every span is two lookups instead of two binary searches.
__global__ void __launch_bounds__(256) k_cell_spans(const uint64_t* __restrict__ ckey,
                                                    const uint32_t* __restrict__ cstart, uint64_t nne,
                                                    uint32_t nx, uint32_t ny, uint32_t k, uint2* __restrict__ cspan,
                                                    uint32_t* __restrict__ gcount,
                                                    const uint32_t* __restrict__ cnext) {
    const uint32_t nspan = 2 * k + 1;
    for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < nne;
         c += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t key = ckey[c];
        const uint64_t cy = key / nx, cx = key - cy * nx;
        for (uint32_t r = 0; r < nspan; ++r) {
            // Row dy = r - k of the stencil reaches kx(dy) columns either side: a neighbour in
            // cell (dx, dy) is >= (|dx|-1) w, (|dy|-1) w away in x, y, and (eps / w)^2 =
            // k^2 / (1 + 2^-19)^2 < k^2, so (|dx|-1)^2 + (|dy|-1)^2 <= k^2 holds for every
            // neighbour (the 2^-19 margin covers the rounding of the cell indices).  Trims
            // the outer rows' corner cells for k >= 4 (k = 6: 169 -> 157 cells).
            const uint32_t a = r > k ? r - k : k - r;
            uint32_t kx = k;
            if (a >= 2) {
                const uint32_t rem = k * k - (a - 1) * (a - 1);
                uint32_t m = 0;
                while ((m + 1) * (m + 1) <= rem) ++m;   // isqrt (k <= 6)
                kx = min(k, 1 + m);
            }
            const uint64_t xl = cx >= kx ? cx - kx : 0;
            const uint64_t xh = cx + kx < nx ? cx + kx : nx - 1;
            const int64_t yy = (int64_t)cy + (int64_t)r - (int64_t)k;
            uint2 sp = make_uint2(0, 0);
            if (yy >= 0 && yy < (int64_t)ny) {
                const uint64_t rb = (uint64_t)yy * nx;
                uint64_t i0, i1;
                if (cnext) {
                    i0 = __ldg(&cnext[rb + xl]);
                    i1 = __ldg(&cnext[rb + xh + 1]);
                } else {
                    uint64_t lo = 0, hi = nne;
                    if (yy < (int64_t)cy) hi = c;
                    else if (yy > (int64_t)cy) lo = c + 1;
                    i0 = lower_bound_u64(ckey, lo, hi, rb + xl);
                    i1 = lower_bound_u64(ckey, i0, hi, rb + xh + 1);
                }
                sp = make_uint2(cstart[i0], cstart[i1]);
            }
            cspan[nspan * c + r] = sp;
        }
        gcount[c] = (cstart[c + 1] - cstart[c] + (uint32_t)kGroup - 1) / (uint32_t)kGroup;
    }
}

__global__ void __launch_bounds__(256) k_cell_mark(const uint64_t* __restrict__ ckey, uint64_t nne,
                                                   uint32_t* __restrict__ mark) {
    for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < nne; c += (uint64_t)gridDim.x * blockDim.x)
        mark[ckey[c]] = 1;
}

__global__ void __launch_bounds__(256) k_group_build(const uint32_t* __restrict__ cstart,
                                                     const uint32_t* __restrict__ gofs, uint64_t nne, uint64_t n,
                                                     uint32_t* __restrict__ gstart, uint32_t* __restrict__ gcell) {
    for (uint64_t c = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; c < nne;
         c += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t s0 = cstart[c], s1 = cstart[c + 1];
        uint32_t g = gofs[c];
        for (uint32_t s = s0; s < s1; s += kGroup, ++g) {
            gstart[g] = s;
            gcell[g] = (uint32_t)c;
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) gstart[gofs[nne]] = (uint32_t)n;
}

// ---------------------------------------------------------------- dense / sparse groups (NEXT-1)
__global__ void __launch_bounds__(256) k_group_class(const uint32_t* __restrict__ cstart,
                                                     const uint2* __restrict__ cspan, uint32_t nspan,
                                                     const uint32_t* __restrict__ gstart,
                                                     const uint32_t* __restrict__ gcell,
                                                     const uint32_t* __restrict__ ng_dev, uint64_t n,
                                                     uint32_t max_tests, bool qlanes,
                                                     uint32_t* __restrict__ dflag,
                                                     uint32_t* __restrict__ sqn,
                                                     unsigned long long* __restrict__ n_sparse,
                                                     uint8_t* __restrict__ gbin, uint32_t* __restrict__ ohist,
                                                     uint32_t* __restrict__ words, uint32_t win) {
    __shared__ uint32_t sh[kOrderBins];
    for (int b = threadIdx.x; b < kOrderBins; b += blockDim.x) sh[b] = 0;
    __syncthreads();
    const uint64_t ng = *ng_dev;
    uint32_t tot = 0;
    unsigned long long ttot = 0;   // candidate tests of the thread's groups
    for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < n; g += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t d = 0, sq = 0;
        if (g < ng) {
            const uint32_t qs = gstart[g], c = gcell[g];
            const uint32_t nq = min((uint32_t)kGroup, cstart[c + 1] - qs);
            uint64_t cand = 0;
            uint32_t npairs = 0;   // candidate pairs of the virtual chunk sequence (mask layout)
            uint32_t qw = 0, qlen = 0;   // query-lane hit words, longest row span
            for (uint32_t r = 0; r < nspan; ++r) {
                const uint2 sp = cspan[(uint64_t)nspan * c + r];
                cand += sp.y - sp.x;
                if (sp.y > sp.x) {
                    npairs += ((sp.y + 1) >> 1) - (sp.x >> 1);
                    qw += ((sp.y - sp.x) / 2 + 1 + 15) / 16;
                    qlen = max(qlen, sp.y - sp.x);
                }
            }
            const uint32_t ch = (npairs + 31) / 32;
            words[g] = 2 * nq * win * ((ch + win - 1) / win);
            const uint64_t tests = (uint64_t)nq * cand;
            ttot += tests;
            if (qlanes ? (qw <= (uint32_t)kQW && qlen <= (uint32_t)kQS) : tests <= max_tests) sq = nq;
            else d = 1;
            // cost bin: dense groups first, each class by decreasing log2(tests)
            const uint32_t lg = 63 - __clzll(tests | 1);
            const uint32_t b = (d ? 0u : kOrderBins / 2) + (kOrderBins / 2 - 1 - min(lg, (uint32_t)kOrderBins / 2 - 1));
            gbin[g] = (uint8_t)b;
            atomicAdd(&sh[b], 1u);
        }
        if (g >= ng) words[g] = 0;
        dflag[g] = d;
        sqn[g] = sq;
        tot += sq;
    }
    for (int o = 16; o > 0; o >>= 1) {
        tot += __shfl_xor_sync(0xffffffffu, tot, o);
        ttot += __shfl_xor_sync(0xffffffffu, ttot, o);
    }
    if ((threadIdx.x & 31) == 0 && tot) atomicAdd(n_sparse, (unsigned long long)tot);
    if ((threadIdx.x & 31) == 0 && ttot) atomicAdd(n_sparse + 1, ttot);
    __syncthreads();
    for (int b = threadIdx.x; b < kOrderBins; b += blockDim.x)
        if (sh[b]) atomicAdd(&ohist[b], sh[b]);
}

// Cost order: ord = the groups sorted by gbin (a counting
// sort; order inside a bin is arbitrary -- results do not depend on the visiting
// order, only the tail of the dynamic schedule does).  ohist[0..kOrderBins) are
// the bin sizes, ocur[kOrderBins] zeroed cursors.  Tiles of 256 groups per block
// step: block-local ranks by shared atomics, one global atomic per bin and tile.
__global__ void __launch_bounds__(256) k_order_scatter(const uint8_t* __restrict__ gbin,
                                                       const uint32_t* __restrict__ ng_dev, uint64_t n,
                                                       const uint32_t* __restrict__ ohist,
                                                       uint32_t* __restrict__ ocur, uint32_t* __restrict__ ord) {
    __shared__ uint32_t base[kOrderBins], cnt[kOrderBins], at[kOrderBins];
    const uint64_t ng = *ng_dev;
    if (threadIdx.x == 0) {
        uint32_t acc = 0;
        for (int b = 0; b < kOrderBins; ++b) {
            base[b] = acc;
            acc += ohist[b];
        }
    }
    for (uint64_t t0 = (uint64_t)blockIdx.x * blockDim.x; t0 < ng; t0 += (uint64_t)gridDim.x * blockDim.x) {
        for (int b = threadIdx.x; b < kOrderBins; b += blockDim.x) cnt[b] = 0;
        __syncthreads();
        const uint64_t g = t0 + threadIdx.x;
        uint32_t b = 0, r = 0;
        if (g < ng) {
            b = gbin[g];
            r = atomicAdd(&cnt[b], 1u);
        }
        __syncthreads();
        for (int k = threadIdx.x; k < kOrderBins; k += blockDim.x)
            at[k] = cnt[k] ? atomicAdd(&ocur[k], cnt[k]) : 0;
        __syncthreads();
        if (g < ng) ord[base[b] + at[b] + r] = (uint32_t)g;
        __syncthreads();
    }
}

// dl and sql, thread per group (the tests rule: sparse groups hold 1-2 queries)
__global__ void __launch_bounds__(256) k_group_lists_tpg(const uint32_t* __restrict__ gstart,
                                                         const uint32_t* __restrict__ gcell,
                                                         const uint32_t* __restrict__ ng_dev, uint64_t n,
                                                         const uint32_t* __restrict__ dpre,
                                                         const uint32_t* __restrict__ spre, uint32_t* __restrict__ dl,
                                                         uint2* __restrict__ sql) {
    const uint64_t ng = *ng_dev;
    for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < ng; g += (uint64_t)gridDim.x * blockDim.x) {
        if (dpre[g + 1] != dpre[g]) {
            dl[dpre[g]] = (uint32_t)g;
        } else {
            const uint32_t j = spre[g], m = spre[g + 1] - j, qs = gstart[g], c = gcell[g];
            for (uint32_t i = 0; i < m; ++i) sql[j + i] = make_uint2(qs + i, c);
        }
    }
}

// dl (dense groups) and sql (the sparse / small groups' queries).  A warp takes 32
// consecutive groups: their sql entries form one contiguous range of the list, staged in
// shared memory by the groups' lanes and written out with coalesced stores (a thread
// writing its own group's run of ~11 entries made uncoalesced 88-B runs: 0.33 ms at C5
// under the query-lane rule).
__global__ void __launch_bounds__(128) k_group_lists(const uint32_t* __restrict__ gstart,
                                                     const uint32_t* __restrict__ gcell,
                                                     const uint32_t* __restrict__ ng_dev, uint64_t n,
                                                     const uint32_t* __restrict__ dpre,
                                                     const uint32_t* __restrict__ spre, uint32_t* __restrict__ dl,
                                                     uint2* __restrict__ sql) {
    __shared__ uint2 st[4][32 * kGroup];   // 8 KB per warp
    const uint64_t ng = *ng_dev;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (uint64_t g0 = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) - lane; g0 < ng;
         g0 += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t g = g0 + lane;
        uint32_t j = 0, m = 0, qs = 0, c = 0;
        if (g < ng) {
            j = spre[g];
            m = spre[g + 1] - j;
            if (dpre[g + 1] != dpre[g]) dl[dpre[g]] = (uint32_t)g;
            if (m) {
                qs = gstart[g];
                c = gcell[g];
            }
        }
        const uint32_t J0 = __shfl_sync(0xffffffffu, j, 0);
        const uint32_t Jend = __reduce_max_sync(0xffffffffu, j + m);   // (lanes past ng: j = m = 0)
        for (uint32_t i = 0; i < m; ++i) st[w][j - J0 + i] = make_uint2(qs + i, c);
        __syncwarp();
        for (uint32_t e = lane; e < Jend - J0; e += 32) sql[J0 + e] = st[w][e];
        __syncwarp();
    }
}

// ---------------------------------------------------------------- auto cell split
// Point-weighted cell occupancy at width eps, estimated from a strided sample of
// m points: sample counts s_c per cell go into an open-addressing hash table;
// sum s_c (s_c - 1) / (f sum s_c) (f = m / n) estimates sum n_c (n_c - 1) / n.
__device__ __forceinline__ uint64_t mix_key(uint64_t x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    return x;
}

template <typename T>
__global__ void __launch_bounds__(256) k_occ_sample(const typename V2<T>::type* __restrict__ xy, uint64_t n,
                                                    uint64_t stride, uint64_t m, double inv_w,
                                                    unsigned long long* __restrict__ hkey,
                                                    unsigned int* __restrict__ hcnt, uint32_t tmask) {
    // cells of width eps anchored at the origin (no bbox needed: launched with the bbox
    // reduction, before its host sync); the occupancy statistic does not depend on the anchor
    for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < m; j += (uint64_t)gridDim.x * blockDim.x) {
        auto p = xy[j * stride];
        const double tx = fmin(fmax(floor((double)p.x * inv_w), -0x1p40), 0x1p40);
        const double ty = fmin(fmax(floor((double)p.y * inv_w), -0x1p40), 0x1p40);
        const unsigned long long key =
            ((unsigned long long)(long long)tx << 22) ^ (unsigned long long)(long long)ty * 0x9E3779B97F4A7C15ull;
        // warp-aggregate equal keys (dense cells would serialise the atomics)
        const unsigned act = __activemask();
        const unsigned peers = __match_any_sync(act, key);
        const int lane = threadIdx.x & 31;
        if (lane != __ffs(peers) - 1) continue;
        uint32_t slot = (uint32_t)mix_key(key) & tmask;
        while (true) {
            unsigned long long prev = atomicCAS(&hkey[slot], ~0ull, key);
            if (prev == ~0ull || prev == key) {
                atomicAdd(&hcnt[slot], (unsigned)__popc(peers));
                break;
            }
            slot = (slot + 1) & tmask;
        }
    }
}

__global__ void __launch_bounds__(256) k_occ_reduce(const unsigned int* __restrict__ hcnt, uint32_t tsize,
                                                    unsigned long long* __restrict__ out) {
    unsigned long long a = 0, b = 0;
    for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < tsize; i += gridDim.x * blockDim.x) {
        const unsigned long long c = hcnt[i];
        a += c * (c > 0 ? c - 1 : 0);
        b += c;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        a += __shfl_xor_sync(FULL, a, o);
        b += __shfl_xor_sync(FULL, b, o);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&out[0], a);
        atomicAdd(&out[1], b);
    }
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

void launch_bbox_init(unsigned long long* bb, uint32_t nz, unsigned long long* hkey, unsigned int* hcnt,
                      uint32_t tsize, cudaStream_t s) {
    const uint32_t m = std::max(tsize, nz);
    k_bbox_init<<<(m + 255) / 256, 256, 0, s>>>(bb, nz, hkey, hcnt, tsize);
    ++g_kernel_launches;
}

__global__ void k_readback(unsigned long long* out, const uint32_t* ng, const uint64_t* mw, const uint32_t* dn,
                           const uint32_t* sn, const unsigned long long* sp) {
    out[0] = *ng;
    out[1] = *mw;
    out[2] = dn ? *dn : 0;
    out[3] = sn ? *sn : 0;
    out[4] = sp ? sp[0] : 0;
    out[5] = sp ? sp[1] : 0;
}
void launch_readback(unsigned long long* out, const uint32_t* ng, const uint64_t* mw, const uint32_t* dn,
                     const uint32_t* sn, const unsigned long long* sp, cudaStream_t s) {
    k_readback<<<1, 1, 0, s>>>(out, ng, mw, dn, sn, sp);
    ++g_kernel_launches;
}

void launch_bbox(const void* xy, uint64_t n, hdb_dtype dt, unsigned long long* bb, unsigned int* bad,
                 cudaStream_t s) {
    if (n == 0) return;
    if (dt == HDB_F64)
        k_bbox<double><<<grid_for(n, 256, 148 * 4), 256, 0, s>>>((const double2*)xy, n, bb, bad);
    else
        k_bbox<float><<<grid_for(n, 256, 148 * 4), 256, 0, s>>>((const float2*)xy, n, bb, bad);
    ++g_kernel_launches;
}

size_t radix_sort_temp_bytes(uint64_t n) {
    uint64_t nblocks = (n + RsCfg<uint64_t>::TILE - 1) / RsCfg<uint64_t>::TILE;   // the smaller tile: upper bound
    uint64_t m = nblocks * RS_BINS;
    return (m + 1) * sizeof(uint32_t) * 2 + scan_temp_bytes(m) + 256;
}

template <typename K>
int radix_sort_impl(K* k0, uint32_t* v0, K* k1, uint32_t* v1, uint64_t n, int bits, void* temp, cudaStream_t s,
                    int shift0 = 0) {
    if (n <= 1 || bits <= shift0) return 0;
    constexpr int TILE = RsCfg<K>::TILE;
    uint32_t nblocks = (uint32_t)((n + TILE - 1) / TILE);
    uint64_t m = (uint64_t)nblocks * RS_BINS;
    uint32_t* hist = (uint32_t*)temp;
    uint32_t* hscan = hist + (m + 1);
    void* stemp = (void*)(((uintptr_t)(hscan + m + 1) + 255) & ~(uintptr_t)255);
    int cur = 0;
    for (int shift = shift0; shift < bits; shift += RS_BITS) {
        K* ki = cur ? k1 : k0;
        uint32_t* vi = cur ? v1 : v0;
        K* ko = cur ? k0 : k1;
        uint32_t* vo = cur ? v0 : v1;
        k_radix_hist<K><<<nblocks, RS_THREADS, 0, s>>>(ki, n, shift, hist, nblocks);
        ++g_kernel_launches;
        scan_u32_to_u32(hist, hscan, m, stemp, s);
        k_radix_scatter<K><<<nblocks, RS_THREADS, 0, s>>>(ki, vi, ko, vo, n, shift, hscan, nblocks);
        ++g_kernel_launches;
        cur ^= 1;
    }
    return cur;
}


int radix_sort_pairs(void* k0, uint32_t* v0, void* k1, uint32_t* v1, int key_bytes, uint64_t n, int bits, void* temp,
                     cudaStream_t s) {
    if (key_bytes == 4)
        return radix_sort_impl<uint32_t>((uint32_t*)k0, v0, (uint32_t*)k1, v1, n, bits, temp, s);
    return radix_sort_impl<uint64_t>((uint64_t*)k0, v0, (uint64_t*)k1, v1, n, bits, temp, s);
}

// ---- point sort (a2 + a3 + gather in one record sort)
template <typename T, typename K>
struct PointSort {
    using P2 = typename V2<T>::type;
    static constexpr size_t rec = sizeof(P2) + sizeof(K) + 4;
    template <bool F, bool L>
    static void scatter(const P2* xyin, const K* kin, const uint32_t* vin, const KeyParams& kp, K* kout,
                        uint32_t* vout, P2* xyout, float4* xp, double ox, double oy, uint64_t n, int shift,
                        const uint32_t* hscan, uint32_t nb, unsigned int* counters, uint32_t nc, const uint32_t* gid,
                        cudaStream_t s) {
        static bool attr = [] {
            cudaFuncSetAttribute(k_ps_scatter<T, K, F, L>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)ps_smem_bytes<T, K>());
            return true;
        }();
        (void)attr;
        k_ps_scatter<T, K, F, L><<<nb, PS_THREADS, ps_smem_bytes<T, K>(), s>>>(
            xyin, kin, vin, kp, kout, vout, xyout, xp, ox, oy, n, shift, hscan, nb, counters, nc, gid);
        ++g_kernel_launches;
    }
    static void run(const void* xy_in, uint64_t n, const KeyParams& kp, int bits, void* keys_out, uint32_t* ids_out,
                    void* xy_s, float4* xp, double ox, double oy, unsigned int* counters, uint32_t nc, void* temp,
                    const uint32_t* gid, cudaStream_t s) {
        const uint32_t nb = (uint32_t)((n + PS_TILE - 1) / PS_TILE);
        const int passes = std::max(1, (bits + RS_BITS - 1) / RS_BITS);
        const uint64_t m = (uint64_t)nb * RS_BINS;
        unsigned char* t = (unsigned char*)temp;
        auto carve = [&](size_t bytes) {
            void* p = t;
            t += (bytes + 255) & ~(size_t)255;
            return p;
        };
        uint32_t* hist = (uint32_t*)carve(4 * (m + 1));
        uint32_t* hscan = (uint32_t*)carve(4 * (m + 1));
        void* stemp = carve(scan_temp_bytes(m));
        K* kb[2];
        uint32_t* vb[2];
        P2* xb[2];
        for (int i = 0; i < (passes > 2 ? 2 : passes - 1); ++i) {
            kb[i] = (K*)carve(sizeof(K) * n);
            vb[i] = (uint32_t*)carve(4 * n);
            xb[i] = (P2*)carve(sizeof(P2) * n);
        }
        const P2* xin = (const P2*)xy_in;
        for (int p = 0; p < passes; ++p) {
            const int shift = p * RS_BITS;
            const bool first = p == 0, last = p == passes - 1;
            const K* ki = first ? nullptr : kb[(p - 1) & 1];
            const uint32_t* vi = first ? nullptr : vb[(p - 1) & 1];
            const P2* xi = first ? xin : xb[(p - 1) & 1];
            K* ko = last ? (K*)keys_out : kb[p & 1];
            uint32_t* vo = last ? ids_out : vb[p & 1];
            P2* xo = last ? (P2*)xy_s : xb[p & 1];
            if (first)
                k_ps_hist<T, K, true><<<nb, PS_THREADS, 0, s>>>(xin, nullptr, kp, n, shift, hist, nb);
            else
                k_ps_hist<T, K, false><<<nb, PS_THREADS, 0, s>>>(nullptr, ki, kp, n, shift, hist, nb);
            ++g_kernel_launches;
            scan_u32_to_u32(hist, hscan, m, stemp, s);
            if (first && last)
                scatter<true, true>(xi, ki, vi, kp, ko, vo, xo, xp, ox, oy, n, shift, hscan, nb, counters, nc, gid, s);
            else if (first)
                scatter<true, false>(xi, ki, vi, kp, ko, vo, xo, xp, ox, oy, n, shift, hscan, nb, counters, nc, gid, s);
            else if (last)
                scatter<false, true>(xi, ki, vi, kp, ko, vo, xo, xp, ox, oy, n, shift, hscan, nb, counters, nc, gid, s);
            else
                scatter<false, false>(xi, ki, vi, kp, ko, vo, xo, xp, ox, oy, n, shift, hscan, nb, counters, nc, gid, s);
        }
    }
    static size_t temp_bytes(uint64_t n, int bits) {
        const uint64_t nb = (n + PS_TILE - 1) / PS_TILE, m = nb * RS_BINS;
        const int passes = std::max(1, (bits + RS_BITS - 1) / RS_BITS);
        const int bufs = passes > 2 ? 2 : passes - 1;
        return 2 * (4 * (m + 1) + 256) + scan_temp_bytes(m) + 256 + bufs * (n * rec + 3 * 256);
    }
};

void band_rows_hist(const void* xy, uint64_t n, hdb_dtype dt, double xmin, double ymin, double inv_w, uint32_t nx,
                    uint32_t ny, uint32_t* rowid, uint32_t* cell_cnt, unsigned long long* row_cnt,
                    unsigned long long* row_load, cudaStream_t s) {
    const KeyParams kp{xmin, ymin, inv_w, nx, ny};
    if (n == 0) return;
    if (dt == HDB_F64)
        k_band_hist<double><<<grid_for(n, 256, 148 * 4), 256, 0, s>>>((const double2*)xy, n, kp, rowid, row_cnt, cell_cnt);
    else
        k_band_hist<float><<<grid_for(n, 256, 148 * 4), 256, 0, s>>>((const float2*)xy, n, kp, rowid, row_cnt, cell_cnt);
    ++g_kernel_launches;
    if (cell_cnt) {
        k_row_load<<<grid_for(32ull * ny), 256, 0, s>>>(cell_cnt, nx, ny, row_load);
        ++g_kernel_launches;
    }
}

void launch_band_groups(const uint64_t* ckey, uint64_t nne, const uint32_t* gofs, uint64_t key_lo, uint64_t key_hi,
                        unsigned long long* out, cudaStream_t s) {
    k_band_groups<<<1, 1, 0, s>>>(ckey, nne, gofs, key_lo, key_hi, out);
    ++g_kernel_launches;
}

size_t point_sort_temp_bytes(uint64_t n, hdb_dtype dt, int key_bytes, int bits) {
    if (dt == HDB_F64)
        return key_bytes == 4 ? PointSort<double, uint32_t>::temp_bytes(n, bits)
                              : PointSort<double, uint64_t>::temp_bytes(n, bits);
    return key_bytes == 4 ? PointSort<float, uint32_t>::temp_bytes(n, bits) : PointSort<float, uint64_t>::temp_bytes(n, bits);
}

void sort_points(const void* xy_in, uint64_t n, hdb_dtype dt, double xmin, double ymin, double inv_w, uint32_t nx,
                 uint32_t ny, int key_bytes, int bits, void* keys_out, uint32_t* ids_out, void* xy_s, float4* xp,
                 double ox, double oy, unsigned int* counters, uint32_t n_counters, void* temp, cudaStream_t s,
                 const uint32_t* gid) {
    if (n == 0) return;
    const KeyParams kp{xmin, ymin, inv_w, nx, ny};
    if (dt == HDB_F64) {
        if (key_bytes == 4)
            PointSort<double, uint32_t>::run(xy_in, n, kp, bits, keys_out, ids_out, xy_s, xp, ox, oy, counters,
                                             n_counters, temp, gid, s);
        else
            PointSort<double, uint64_t>::run(xy_in, n, kp, bits, keys_out, ids_out, xy_s, xp, ox, oy, counters,
                                             n_counters, temp, gid, s);
    } else {
        if (key_bytes == 4)
            PointSort<float, uint32_t>::run(xy_in, n, kp, bits, keys_out, ids_out, xy_s, xp, 0, 0, counters,
                                            n_counters, temp, gid, s);
        else
            PointSort<float, uint64_t>::run(xy_in, n, kp, bits, keys_out, ids_out, xy_s, xp, 0, 0, counters,
                                            n_counters, temp, gid, s);
    }
}

void launch_cell_spans(const uint64_t* ckey, const uint32_t* cstart, uint64_t nne, uint32_t nx, uint32_t ny,
                       uint32_t k, uint2* cspan, uint32_t* gcount, const uint32_t* cnext, cudaStream_t s) {
    if (nne == 0) return;
    k_cell_spans<<<grid_for(nne), 256, 0, s>>>(ckey, cstart, nne, nx, ny, k, cspan, gcount, cnext);
    ++g_kernel_launches;
}

void launch_cell_mark(const uint64_t* ckey, uint64_t nne, uint32_t* mark, cudaStream_t s) {
    if (nne == 0) return;
    k_cell_mark<<<grid_for(nne), 256, 0, s>>>(ckey, nne, mark);
    ++g_kernel_launches;
}

void launch_group_build(const uint32_t* cstart, const uint32_t* gofs, uint64_t nne, uint64_t n, uint32_t* gstart,
                        uint32_t* gcell, cudaStream_t s) {
    k_group_build<<<grid_for(nne), 256, 0, s>>>(cstart, gofs, nne, n, gstart, gcell);
    ++g_kernel_launches;
}

void launch_group_class(const uint32_t* cstart, const uint2* cspan, uint32_t nspan, const uint32_t* gstart,
                        const uint32_t* gcell, const uint32_t* ng_dev, uint64_t n, uint32_t max_tests,
                        bool qlanes, uint32_t* dflag, uint32_t* sqn, unsigned long long* n_sparse, uint8_t* gbin,
                        uint32_t* ohist, uint32_t* words, uint32_t win, cudaStream_t s) {
    if (n == 0) return;
    k_group_class<<<grid_for(n), 256, 0, s>>>(cstart, cspan, nspan, gstart, gcell, ng_dev, n, max_tests, qlanes,
                                              dflag, sqn,
                                              n_sparse, gbin, ohist, words, win);
    ++g_kernel_launches;
}

void launch_order_scatter(const uint8_t* gbin, const uint32_t* ng_dev, uint64_t n, uint32_t* ohist, uint32_t* ord,
                          cudaStream_t s) {
    if (n == 0) return;
    k_order_scatter<<<grid_for(n), 256, 0, s>>>(gbin, ng_dev, n, ohist, ohist + kOrderBins, ord);
    ++g_kernel_launches;
}

void launch_group_lists(const uint32_t* gstart, const uint32_t* gcell, const uint32_t* ng_dev, uint64_t n,
                        const uint32_t* dpre, const uint32_t* spre, uint32_t* dl, uint2* sql, bool qlanes,
                        cudaStream_t s) {
    if (n == 0) return;
    // the query-lane rule's small groups hold ~11 queries each: warp-staged coalesced runs;
    // the tests rule's sparse groups 1-2: a thread per group (A/B: C2 eps 0.45 step 2.40 vs 2.52 ms)
    if (qlanes)
        k_group_lists<<<grid_for(n, 128), 128, 0, s>>>(gstart, gcell, ng_dev, n, dpre, spre, dl, sql);
    else
        k_group_lists_tpg<<<grid_for(n), 256, 0, s>>>(gstart, gcell, ng_dev, n, dpre, spre, dl, sql);
    ++g_kernel_launches;
}

void launch_occ_estimate(const void* xy, uint64_t n, hdb_dtype dt, uint64_t stride, uint64_t m, double inv_w,
                         unsigned long long* hkey, unsigned int* hcnt, uint32_t tsize, unsigned long long* out,
                         cudaStream_t s) {
    // hkey / hcnt / out were initialised by launch_bbox_init
    if (m) {
        if (dt == HDB_F64)
            k_occ_sample<double><<<grid_for(m), 256, 0, s>>>((const double2*)xy, n, stride, m, inv_w, hkey, hcnt,
                                                             tsize - 1);
        else
            k_occ_sample<float><<<grid_for(m), 256, 0, s>>>((const float2*)xy, n, stride, m, inv_w, hkey, hcnt,
                                                            tsize - 1);
        ++g_kernel_launches;
    }
    k_occ_reduce<<<grid_for(tsize, 256, 148 * 2), 256, 0, s>>>(hcnt, tsize, out);
    ++g_kernel_launches;
}

}  // namespace hdb
