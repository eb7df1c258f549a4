// kernels_search.cu -- the eps-neighbour search on sm_100a.
//
// Functional role: GPUCalcGlobal (Alg. 2) -- for every query point,
// scan the points of the (at most 9) adjacent cells and emit every
// candidate within eps (calcDistance, line 11).  Design:
//
//  * Row spans.  Keys are row-major (h = cy*nx + cx) and points are sorted by
//    key, so the 3 cells (cx-1..cx+1, y') of one stencil row are ONE contiguous
//    span of sorted positions (reading R8 of Alg. 2 lines 8-10); the grid
//    stores the 3 spans of every non-empty cell.
//  * Query groups.  A warp owns <= 32 consecutive queries of one cell (they share
//    the 3 spans).  Candidates stream through the warp in chunks of 64: lane j
//    holds candidates j and j+32 as one packed f32x2 pair, and every query of
//    the group is tested against the chunk with FADD2/FFMA2 (two tests per
//    instruction); ballot + popc give counts and the compacted write positions.
//  * Exact predicate, fast.  The paper fixes only dist <= eps; the
//    contract here is the f64 no-FMA predicate of the oracle (reading R1/R2).
//    f64 mode evaluates t = (dx^2 - e2) + dy^2 in f32 on coordinates relative to
//    the bbox centre; whenever |t| > band (a rigorous bound on the f32 error,
//    computed on the host -- DESIGN.md "filter bound") sign(t) IS the exact f64
//    decision; the rare |t| <= band tests are re-done in exact f64 with
//    __dsub_rn/__dmul_rn/__dadd_rn (never contracted to FMA).  f32 mode
//    evaluates the f32 predicate itself exactly (sub/mul/add .rn f32x2).
//  * Count -> scan -> write (a6-a8): the count pass stores |N_eps(q)|, an
//    exclusive scan gives each query's offset, and the write pass stores the
//    ballot-compacted hits contiguously into the query's CSR segment (no
//    atomics, no overflow, no key/value sort -- Alg. 4 line 7 is unnecessary).
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int kWarps = kSearchThreads / 32;

struct SArgs {
    const float2* xf;      // f32 coordinates: filter coords (f64 mode) / exact coords (f32 mode)
    const double2* xd;     // exact f64 coordinates (f64 mode)
    const uint32_t* ids;
    const uint32_t* cstart;
    const uint2* cspan;
    const uint32_t* gstart;
    const uint32_t* gcell;
    float e2f;             // f32 mode: fl32(eps^2); f64 mode: fl32(e2_d)
    float band;            // f64 mode: decide in exact f64 when |t| <= band
    double e2d;            // fl64(eps^2)
};

typedef unsigned long long u64x;

__device__ __forceinline__ u64x pack2(float a, float b) {
    u64x r;
    asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b));
    return r;
}
__device__ __forceinline__ float2 unpack2(u64x v) {
    float2 r;
    asm("mov.b64 {%0,%1}, %2;" : "=f"(r.x), "=f"(r.y) : "l"(v));
    return r;
}
__device__ __forceinline__ u64x sub2(u64x a, u64x b) {
    u64x r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64x mul2(u64x a, u64x b) {
    u64x r;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64x add2(u64x a, u64x b) {
    u64x r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ u64x fma2(u64x a, u64x b, u64x c) {
    u64x r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}

// O1 predicate in exact f64: no FMA contraction possible with explicit _rn ops.
__device__ __forceinline__ bool pred_f64(double xp, double yp, double xq, double yq, double e2) {
    double dx = __dsub_rn(xp, xq);
    double dy = __dsub_rn(yp, yq);
    return __dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)) <= e2;
}
__device__ __forceinline__ bool pred_f32(float xp, float yp, float xq, float yq, float e2) {
    float dx = __fsub_rn(xp, xq);
    float dy = __fsub_rn(yp, yq);
    return __fadd_rn(__fmul_rn(dx, dx), __fmul_rn(dy, dy)) <= e2;
}

constexpr float kFar = 1e30f;   // padding coordinate: never a neighbour (t ~ 1e60 -> inf > band)

// Kernel modes: f32 input (exact f32 predicate), f64 input with the f32
// filter + exact f64 fallback, f64 input tested in exact f64 only (used when
// the filter bound is useless, e.g. extent/eps near 2^30 or huge coordinates).
enum Mode { kF32 = 0, kF64Filter = 1, kF64Exact = 2 };

// Tests of query q (broadcast) against the lane's two candidates (packed).
// Returns the two hit predicates via in0/in1.
template <int MODE>
__device__ __forceinline__ void test_pair(const SArgs& a, float4 q, u64x X, u64x Y, bool v0, bool v1, uint32_t j0,
                                          uint32_t j1, const double2& qd, const double2& c0, const double2& c1,
                                          bool& in0, bool& in1) {
    if (MODE == kF64Exact) {
        in0 = v0 && pred_f64(qd.x, qd.y, c0.x, c0.y, a.e2d);
        in1 = v1 && pred_f64(qd.x, qd.y, c1.x, c1.y, a.e2d);
        return;
    }
    const u64x qx = pack2(q.x, q.y);   // {qx, qx}
    const u64x qy = pack2(q.z, q.w);   // {qy, qy}
    const u64x dx = sub2(qx, X);
    const u64x dy = sub2(qy, Y);
    if (MODE == kF64Filter) {
        const u64x ne2 = pack2(-a.e2f, -a.e2f);
        const float2 t = unpack2(fma2(dy, dy, fma2(dx, dx, ne2)));   // (dx^2 - e2) + dy^2
        in0 = v0 && t.x < 0.f;
        in1 = v1 && t.y < 0.f;
        const bool b0 = v0 && fabsf(t.x) <= a.band;
        const bool b1 = v1 && fabsf(t.y) <= a.band;
        if (__any_sync(FULL, b0 || b1)) {   // rare: decide in exact f64
            if (b0) {
                const double2 p = a.xd[j0];
                in0 = pred_f64(qd.x, qd.y, p.x, p.y, a.e2d);
            }
            if (b1) {
                const double2 p = a.xd[j1];
                in1 = pred_f64(qd.x, qd.y, p.x, p.y, a.e2d);
            }
        }
    } else {
        const float2 d2 = unpack2(add2(mul2(dx, dx), mul2(dy, dy)));  // fl(fl(dx^2) + fl(dy^2))
        in0 = v0 && d2.x <= a.e2f;
        in1 = v1 && d2.y <= a.e2f;
    }
}

// a6 / a8: warp per query group, two candidates per lane per chunk.
template <int MODE, bool WRITE>
__global__ void __launch_bounds__(kSearchThreads) k_search(SArgs a, uint32_t g0, uint32_t g1,
                                                           uint32_t* __restrict__ cnt,
                                                           unsigned long long* __restrict__ tests_out,
                                                           const uint64_t* __restrict__ off, uint64_t out_base,
                                                           uint32_t* __restrict__ out) {
    constexpr bool F64 = MODE != kF32;
    __shared__ float4 sq[kWarps][32];              // {qx, qx, qy, qy}
    __shared__ double2 sqd[F64 ? kWarps : 1][32];  // exact query coordinates (f64 modes)
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    const uint32_t wid = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
    unsigned long long tests = 0;
    for (uint32_t gi = g0 + wid; gi < g1; gi += nw) {
        const uint32_t qs = __ldg(&a.gstart[gi]);
        const uint32_t c = __ldg(&a.gcell[gi]);
        const uint32_t nq = min((uint32_t)kGroup, __ldg(&a.cstart[c + 1]) - qs);
        __syncwarp();
        if ((uint32_t)lane < nq) {
            if (MODE != kF64Exact) {
                const float2 p = a.xf[qs + lane];
                sq[w][lane] = make_float4(p.x, p.x, p.y, p.y);
            }
            if (F64) sqd[F64 ? w : 0][lane] = a.xd[qs + lane];
        }
        uint32_t my = 0;        // count: this lane's query's count; write: its offset within the group
        uint32_t* gout = nullptr;
        if (WRITE) {
            const uint64_t gb = off[qs];
            gout = out + (gb - out_base);
            if ((uint32_t)lane < nq) my = (uint32_t)(off[qs + lane] - gb);
        }
        __syncwarp();
#pragma unroll 1
        for (int r = 0; r < 3; ++r) {
            const uint2 sp = __ldg(&a.cspan[3 * c + r]);
            const uint32_t hi = sp.y;
#pragma unroll 1
            for (uint32_t c0 = sp.x; c0 < hi; c0 += 64) {
                const uint32_t j0 = c0 + lane, j1 = c0 + 32 + lane;
                const bool v0 = j0 < hi, v1 = j1 < hi;
                float2 p0 = make_float2(kFar, kFar), p1 = make_float2(kFar, kFar);
                double2 c0d = make_double2(0, 0), c1d = make_double2(0, 0);
                if (MODE == kF64Exact) {
                    if (v0) c0d = a.xd[j0];
                    if (v1) c1d = a.xd[j1];
                } else {
                    if (v0) p0 = a.xf[j0];
                    if (v1) p1 = a.xf[j1];
                }
                const u64x X = pack2(p0.x, p1.x);
                const u64x Y = pack2(p0.y, p1.y);
                uint32_t id0 = 0, id1 = 0;
                if (WRITE) {
                    if (v0) id0 = __ldg(&a.ids[j0]);
                    if (v1) id1 = __ldg(&a.ids[j1]);
                }
                if (!WRITE) tests += (unsigned long long)nq * min(64u, hi - c0);
#pragma unroll 2
                for (uint32_t i = 0; i < nq; ++i) {
                    float4 q = make_float4(0, 0, 0, 0);
                    if (MODE != kF64Exact) q = sq[w][i];
                    double2 qd = make_double2(0, 0);
                    if (F64) qd = sqd[F64 ? w : 0][i];
                    bool in0, in1;
                    test_pair<MODE>(a, q, X, Y, v0, v1, j0, j1, qd, c0d, c1d, in0, in1);
                    const unsigned m0 = __ballot_sync(FULL, in0);
                    const unsigned m1 = __ballot_sync(FULL, in1);
                    const uint32_t n0 = __popc(m0);
                    if (WRITE) {
                        const uint32_t b = __shfl_sync(FULL, my, i);
                        if (in0) gout[b + __popc(m0 & lt)] = id0;
                        if (in1) gout[b + n0 + __popc(m1 & lt)] = id1;
                    }
                    if ((uint32_t)lane == i) my += n0 + __popc(m1);
                }
            }
        }
        if (!WRITE && (uint32_t)lane < nq) cnt[qs + lane] = my;
    }
    if (!WRITE && tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

// a5: warp per sampled query (the paper's estimator kernel),
// exact predicate, lanes over candidates.
template <bool F64>
__global__ void __launch_bounds__(256) k_sample_count(SArgs a, uint64_t nne, uint64_t stride, uint64_t ns,
                                                      uint32_t* __restrict__ samp_cnt,
                                                      unsigned long long* __restrict__ sum) {
    const int lane = threadIdx.x & 31;
    const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    unsigned long long tot = 0;
    for (uint64_t j = wid; j < ns; j += nw) {
        const uint64_t s = j * stride;
        // cell of sorted position s: last c with cstart[c] <= s
        uint64_t lo = 0, hi = nne;
        while (hi - lo > 1) {
            uint64_t mid = (lo + hi) >> 1;
            if (__ldg(&a.cstart[mid]) <= s)
                lo = mid;
            else
                hi = mid;
        }
        const uint64_t c = lo;
        uint32_t cntv = 0;
        if (F64) {
            const double2 q = a.xd[s];
            for (int r = 0; r < 3; ++r) {
                const uint2 sp = a.cspan[3 * c + r];
                for (uint32_t k = sp.x + lane; k < sp.y; k += 32) {
                    const double2 p = a.xd[k];
                    cntv += pred_f64(q.x, q.y, p.x, p.y, a.e2d) ? 1u : 0u;
                }
            }
        } else {
            const float2 q = a.xf[s];
            for (int r = 0; r < 3; ++r) {
                const uint2 sp = a.cspan[3 * c + r];
                for (uint32_t k = sp.x + lane; k < sp.y; k += 32) {
                    const float2 p = a.xf[k];
                    cntv += pred_f32(q.x, q.y, p.x, p.y, a.e2f) ? 1u : 0u;
                }
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) cntv += __shfl_xor_sync(FULL, cntv, o);
        if (lane == 0 && samp_cnt) samp_cnt[j] = cntv;
        tot += cntv;
    }
    if (lane == 0 && tot) atomicAdd(sum, tot);
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
    uint64_t lo = 0, hi = ng;   // first group whose start is >= p
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
    const uint64_t o0 = off[q0];
    for (uint64_t q = q0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < q1;
         q += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t id = ids[q];
        begin[id] = off[q] - o0 + base;
        count[id] = cnt[q];
    }
}

SArgs args_of(const DevGrid& g) {
    SArgs a;
    a.xf = g.xf;
    a.xd = (const double2*)g.xy_s;
    a.ids = g.ids;
    a.cstart = g.cstart;
    a.cspan = g.cspan;
    a.gstart = g.gstart;
    a.gcell = g.gcell;
    a.e2f = g.e2_f;
    a.band = g.band;
    a.e2d = g.e2_d;
    return a;
}

unsigned search_grid(uint64_t ngroups) {
    uint64_t ctas = (ngroups + kWarps - 1) / kWarps;
    const uint64_t cap = 148ull * 8ull;   // 8 CTAs x 8 warps = 64 warps per SM
    if (ctas > cap) ctas = cap;
    return (unsigned)(ctas ? ctas : 1);
}

template <bool WRITE>
void launch_search(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                   const uint64_t* off, uint64_t out_base, uint32_t* out, bool force_exact, cudaStream_t s) {
    if (g1 <= g0) return;
    const unsigned grid = search_grid(g1 - g0);
    const SArgs a = args_of(g);
    const int mode = g.dtype == HDB_F32 ? kF32 : (g.filter && !force_exact ? kF64Filter : kF64Exact);
    if (mode == kF64Filter)
        k_search<kF64Filter, WRITE><<<grid, kSearchThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, cnt, tests, off,
                                                                     out_base, out);
    else if (mode == kF64Exact)
        k_search<kF64Exact, WRITE><<<grid, kSearchThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, cnt, tests, off,
                                                                    out_base, out);
    else
        k_search<kF32, WRITE><<<grid, kSearchThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, cnt, tests, off,
                                                               out_base, out);
    ++g_kernel_launches;
}

}  // namespace

void launch_sample_count(const DevGrid& g, uint64_t stride, uint64_t n_sample, uint32_t* samp_cnt,
                         unsigned long long* sum, cudaStream_t s) {
    if (n_sample == 0) return;
    uint64_t blocks = (n_sample + 7) / 8;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (g.dtype == HDB_F64)
        k_sample_count<true><<<(unsigned)blocks, 256, 0, s>>>(args_of(g), g.n_nonempty, stride, n_sample, samp_cnt,
                                                              sum);
    else
        k_sample_count<false><<<(unsigned)blocks, 256, 0, s>>>(args_of(g), g.n_nonempty, stride, n_sample, samp_cnt,
                                                               sum);
    ++g_kernel_launches;
}

// variant (hdb_opts.search_kernel): 0 = default, 1 = force the exact-f64-only kernel
void launch_count(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                  int variant, cudaStream_t s) {
    launch_search<false>(g, g0, g1, cnt, tests, nullptr, 0, nullptr, variant == 1, s);
}

void launch_write(const DevGrid& g, uint64_t g0, uint64_t g1, const uint64_t* off, uint64_t out_base,
                  uint32_t* out, int variant, cudaStream_t s) {
    launch_search<true>(g, g0, g1, nullptr, nullptr, off, out_base, out, variant == 1, s);
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
