// kernels_search.cu -- the eps-neighbour search on sm_100a.
//
// Functional role: GPUCalcGlobal (Alg. 2) -- for every query point,
// scan the points of the (at most 9) adjacent cells and emit every
// candidate within eps (calcDistance, line 11).  Design:
//
//  * Row spans.  Keys are row-major (h = cy*nx + cx) and points are sorted by
//    key, so the 3 cells (cx-1..cx+1, y') of one stencil row are ONE contiguous
//    span of sorted positions: [G[h(cx-1,y')], G[h(cx+1,y')+1]).  A query's
//    candidates are 3 contiguous spans (reading R8 of Alg. 2 lines 8-10).
//  * Query groups.  A warp owns <= 32 consecutive queries of one cell (they share
//    the 3 spans); lane j streams candidate j of a 32-wide chunk with one
//    coalesced 16-B (f64) / 8-B (f32) load, and every query of the group is
//    tested against the chunk: hit = pred(q_i, c_j); ballot; popc.
//  * Count -> scan -> write (a6-a8): the count pass stores |N_eps(q)|, an exclusive
//    scan gives each query's offset, and the write pass stores the ballot-
//    compacted hits contiguously into the query's CSR segment (no atomics, no
//    overflow, no key/value sort -- Alg. 4 line 7's Thrust sort is unnecessary).
//  * Exact predicate: fl(fl(dx*dx)+fl(dy*dy)) <= fl(eps^2) with __d*_rn / __f*_rn
//    intrinsics, which nvcc never contracts into FMA (reading R2).
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

extern std::atomic<uint64_t> g_kernel_launches;

namespace {

constexpr unsigned FULL = 0xffffffffu;

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

// O1 predicate, exact: no FMA contraction possible with explicit _rn ops.
__device__ __forceinline__ bool pred(double xp, double yp, double xq, double yq, double e2) {
    double dx = __dsub_rn(xp, xq);
    double dy = __dsub_rn(yp, yq);
    return __dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)) <= e2;
}
__device__ __forceinline__ bool pred(float xp, float yp, float xq, float yq, float e2) {
    float dx = __fsub_rn(xp, xq);
    float dy = __fsub_rn(yp, yq);
    return __fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)) <= e2;
}

__device__ __forceinline__ double far_coord(double) { return 1e300; }
__device__ __forceinline__ float far_coord(float) { return 3e38f; }

// Stencil row spans of cell `key`: span r = [lo[r], hi[r]) (empty if out of grid).
__device__ __forceinline__ void row_spans(const uint32_t* __restrict__ start, uint32_t key, uint32_t nx,
                                          uint32_t ny, uint32_t lo[3], uint32_t hi[3]) {
    uint32_t cy = key / nx, cx = key - cy * nx;
    uint32_t xl = cx > 0 ? cx - 1 : 0;
    uint32_t xh = cx + 1 < nx ? cx + 1 : nx - 1;
#pragma unroll
    for (int r = 0; r < 3; ++r) {
        int yy = (int)cy + r - 1;
        if (yy < 0 || yy >= (int)ny) {
            lo[r] = hi[r] = 0;
        } else {
            uint32_t rowb = (uint32_t)yy * nx;
            lo[r] = __ldg(&start[rowb + xl]);
            hi[r] = __ldg(&start[rowb + xh + 1]);
        }
    }
}

// a5: thread per sampled query (the paper's estimator kernel).
template <typename T>
__global__ void __launch_bounds__(256) k_sample_count(GridArgs<T> g, uint64_t stride, uint64_t ns,
                                                      uint32_t* __restrict__ samp_cnt,
                                                      unsigned long long* __restrict__ sum) {
    using V = typename V2<T>::type;
    const V* __restrict__ xy = (const V*)g.xy;
    uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    uint32_t c = 0;
    if (j < ns) {
        uint64_t s = j * stride;
        V q = xy[s];
        uint32_t lo[3], hi[3];
        row_spans(g.start, g.keys[s], g.nx, g.ny, lo, hi);
        for (int r = 0; r < 3; ++r)
            for (uint32_t k = lo[r]; k < hi[r]; ++k) {
                V p = xy[k];
                c += pred(q.x, q.y, p.x, p.y, g.e2) ? 1u : 0u;
            }
        if (samp_cnt) samp_cnt[j] = c;
    }
    unsigned long long t = c;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(FULL, t, o);
    if ((threadIdx.x & 31) == 0 && t) atomicAdd(sum, t);
}

// a6 / a8: warp per query group, lane per candidate.
template <typename T, bool WRITE>
__global__ void __launch_bounds__(kSearchThreads) k_search(GridArgs<T> g, uint32_t g0, uint32_t g1,
                                                           uint32_t* __restrict__ cnt,
                                                           unsigned long long* __restrict__ tests_out,
                                                           const uint64_t* __restrict__ off, uint64_t out_base,
                                                           uint32_t* __restrict__ out) {
    using V = typename V2<T>::type;
    const V* __restrict__ xy = (const V*)g.xy;
    const int lane = threadIdx.x & 31;
    const unsigned lt = (1u << lane) - 1u;
    const uint32_t wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    unsigned long long tests = 0;
    for (uint32_t gi = g0 + wid; gi < g1; gi += nw) {
        const uint32_t qs = __ldg(&g.gstart[gi]);
        const uint32_t key = __ldg(&g.keys[qs]);
        const uint32_t cend = __ldg(&g.start[key + 1]);
        const uint32_t nq = min((uint32_t)kGroup, cend - qs);
        V q;
        q.x = far_coord(T(0));
        q.y = far_coord(T(0));
        if ((uint32_t)lane < nq) q = xy[qs + lane];
        uint64_t cur = 0;     // write: this lane's query's next output slot
        uint32_t c = 0;       // count: this lane's query's count
        if (WRITE && (uint32_t)lane < nq) cur = off[qs + lane] - out_base;
        uint32_t lo[3], hi[3];
        row_spans(g.start, key, g.nx, g.ny, lo, hi);
#pragma unroll 1
        for (int r = 0; r < 3; ++r) {
#pragma unroll 1
            for (uint32_t c0 = lo[r]; c0 < hi[r]; c0 += 32) {
                const uint32_t j = c0 + lane;
                const bool valid = j < hi[r];
                V p;
                p.x = far_coord(T(0));
                p.y = far_coord(T(0));
                uint32_t id = 0;
                if (valid) {
                    p = xy[j];
                    if (WRITE) id = __ldg(&g.ids[j]);
                }
                if (!WRITE) tests += (unsigned long long)nq * min(32u, hi[r] - c0);
#pragma unroll 4
                for (uint32_t i = 0; i < nq; ++i) {
                    const T qx = __shfl_sync(FULL, q.x, i);
                    const T qy = __shfl_sync(FULL, q.y, i);
                    const bool hit = valid && pred(qx, qy, p.x, p.y, g.e2);
                    const unsigned m = __ballot_sync(FULL, hit);
                    if (WRITE) {
                        const uint64_t b = __shfl_sync(FULL, cur, i);
                        if (hit) out[b + __popc(m & lt)] = id;
                        if ((uint32_t)lane == i) cur += __popc(m);
                    } else {
                        if ((uint32_t)lane == i) c += __popc(m);
                    }
                }
            }
        }
        if (!WRITE && (uint32_t)lane < nq) cnt[qs + lane] = c;
    }
    if (!WRITE && tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

__global__ void k_batch_cuts(const uint32_t* __restrict__ gstart, const uint64_t* __restrict__ off, uint64_t g0,
                             uint64_t g1, uint32_t nb, uint64_t* __restrict__ gcut, uint64_t* __restrict__ pcut) {
    uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
    if (b > nb) return;
    const uint64_t p0 = off[gstart[g0]];
    const uint64_t p1 = off[gstart[g1]];
    uint64_t g;
    if (b == 0) {
        g = g0;
    } else if (b == nb) {
        g = g1;
    } else {
        // target pair offset of cut b (128-bit safe: span < 2^64 / nb for any sane P)
        const uint64_t target = p0 + (uint64_t)(((unsigned __int128)(p1 - p0) * b) / nb);
        uint64_t lo = g0, hi = g1;   // first g in [g0, g1] with off[gstart[g]] >= target
        while (lo < hi) {
            uint64_t mid = (lo + hi) >> 1;
            if (off[gstart[mid]] >= target)
                hi = mid;
            else
                lo = mid + 1;
        }
        g = lo;
    }
    gcut[b] = g;
    pcut[b] = off[gstart[g]];
}

__global__ void k_pos_to_group(const uint32_t* __restrict__ gstart, uint64_t ng, const uint64_t* __restrict__ pos,
                               uint32_t m, uint64_t* __restrict__ grp) {
    uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    uint64_t p = pos[i];
    // first group whose start is >= p  (so a shard boundary never splits a group)
    uint64_t lo = 0, hi = ng;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if ((uint64_t)gstart[mid] >= p)
            hi = mid;
        else
            lo = mid + 1;
    }
    grp[i] = lo;
}

__global__ void __launch_bounds__(256) k_scatter_rows(const uint32_t* __restrict__ ids,
                                                      const uint64_t* __restrict__ off,
                                                      const uint32_t* __restrict__ cnt, uint64_t q0, uint64_t q1,
                                                      uint64_t base, uint64_t* __restrict__ begin,
                                                      uint32_t* __restrict__ count) {
    for (uint64_t q = q0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < q1;
         q += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t id = ids[q];
        begin[id] = off[q] - off[q0] + base;
        count[id] = cnt[q];
    }
}

template <typename T>
GridArgs<T> args_of(const DevGrid& g) {
    GridArgs<T> a;
    a.xy = g.xy_s;
    a.ids = g.ids;
    a.keys = g.keys;
    a.start = g.start;
    a.gstart = g.gstart;
    a.nx = g.nx;
    a.ny = g.ny;
    a.n = (uint32_t)g.n;
    if constexpr (sizeof(T) == 8)
        a.e2 = g.e2_d;
    else
        a.e2 = g.e2_f;
    return a;
}

unsigned search_grid(uint64_t ngroups) {
    const uint64_t warps_per_cta = kSearchThreads / 32;
    uint64_t ctas = (ngroups + warps_per_cta - 1) / warps_per_cta;
    const uint64_t cap = 148ull * 8ull;   // 8 CTAs x 8 warps = 64 warps per SM
    if (ctas > cap) ctas = cap;
    return (unsigned)(ctas ? ctas : 1);
}

}  // namespace

void launch_sample_count(const DevGrid& g, uint64_t stride, uint64_t n_sample, uint32_t* samp_cnt,
                         unsigned long long* sum, cudaStream_t s) {
    if (n_sample == 0) return;
    unsigned blocks = (unsigned)((n_sample + 255) / 256);
    if (g.dtype == HDB_F64)
        k_sample_count<double><<<blocks, 256, 0, s>>>(args_of<double>(g), stride, n_sample, samp_cnt, sum);
    else
        k_sample_count<float><<<blocks, 256, 0, s>>>(args_of<float>(g), stride, n_sample, samp_cnt, sum);
    ++g_kernel_launches;
}

void launch_count(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests, int,
                  cudaStream_t s) {
    if (g1 <= g0) return;
    unsigned grid = search_grid(g1 - g0);
    if (g.dtype == HDB_F64)
        k_search<double, false><<<grid, kSearchThreads, 0, s>>>(args_of<double>(g), (uint32_t)g0, (uint32_t)g1,
                                                                cnt, tests, nullptr, 0, nullptr);
    else
        k_search<float, false><<<grid, kSearchThreads, 0, s>>>(args_of<float>(g), (uint32_t)g0, (uint32_t)g1,
                                                               cnt, tests, nullptr, 0, nullptr);
    ++g_kernel_launches;
}

void launch_write(const DevGrid& g, uint64_t g0, uint64_t g1, const uint64_t* off, uint64_t out_base,
                  uint32_t* out, int, cudaStream_t s) {
    if (g1 <= g0) return;
    unsigned grid = search_grid(g1 - g0);
    if (g.dtype == HDB_F64)
        k_search<double, true><<<grid, kSearchThreads, 0, s>>>(args_of<double>(g), (uint32_t)g0, (uint32_t)g1,
                                                               nullptr, nullptr, off, out_base, out);
    else
        k_search<float, true><<<grid, kSearchThreads, 0, s>>>(args_of<float>(g), (uint32_t)g0, (uint32_t)g1,
                                                              nullptr, nullptr, off, out_base, out);
    ++g_kernel_launches;
}

void launch_batch_cuts(const uint32_t* gstart, const uint64_t* off, uint64_t g0, uint64_t g1, uint32_t nb,
                       uint64_t* gcut, uint64_t* pcut, cudaStream_t s) {
    k_batch_cuts<<<(nb + 1 + 127) / 128, 128, 0, s>>>(gstart, off, g0, g1, nb, gcut, pcut);
    ++g_kernel_launches;
}

void launch_pos_to_group(const uint32_t* gstart, uint64_t n_groups, const uint64_t* pos, uint32_t m,
                         uint64_t* grp, cudaStream_t s) {
    if (m == 0) return;
    k_pos_to_group<<<(m + 127) / 128, 128, 0, s>>>(gstart, n_groups, pos, m, grp);
    ++g_kernel_launches;
}

void launch_scatter_rows(const uint32_t* ids, const uint64_t* off, const uint32_t* cnt, uint64_t q0, uint64_t q1,
                         uint64_t base, uint64_t* begin, uint32_t* count, cudaStream_t s) {
    if (q1 <= q0) return;
    uint64_t n = q1 - q0;
    unsigned blocks = (unsigned)((n + 255) / 256);
    if (blocks > 148 * 16) blocks = 148 * 16;
    k_scatter_rows<<<blocks, 256, 0, s>>>(ids, off, cnt, q0, q1, base, begin, count);
    ++g_kernel_launches;
}

}  // namespace hdb
