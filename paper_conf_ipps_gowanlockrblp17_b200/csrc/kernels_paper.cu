// kernels_paper.cu -- the paper's two search kernels, compiled for sm_100a as
// the on-box baseline of Table II (NEXT-3); search_kernel 7 / 8.
//
//  * GPUCalcGlobal (Alg. 2, Sec. IV-A): one thread per point; the
//    point stays in registers (line 5); the thread scans the candidates of the
//    (at most 9) adjacent cells (lines 6-10) from global memory, tests each
//    (calcDistance, line 11) and appends every hit to the result set with an
//    atomic (line 13).
//  * GPUCalcShared (Alg. 3, Sec. IV-B): one block of blockDim = 256
//    threads per NON-EMPTY cell (schedule S, N = #non-empty cells x blockDim,
//    P:506-512); for every comparison cell the block pages the origin cell's
//    points and the comparison cell's points into shared memory in tiles of
//    blockDim (lines 11-18), synchronises, and each thread tests its origin
//    point against the whole comparison tile (lines 19-22) with an atomic
//    append.  Origin cells larger than blockDim take "an additional loop"
//    (reading R16).
//
// Both emit the paper's key/value result set R (key = the query's point id,
// value = a neighbour's point id); ConstructNeighborTable
// then needs R sorted by key (Alg. 4 line 7: the paper's Thrust sort_by_key),
// done here with the library's own LSD radix sort, and T's ranges are read off
// the sorted keys (k_rows_from_keys).
//
// Adaptations: the comparison cells of a row of the
// stencil are adjacent in the sorted order, so the 9 cells are visited as the
// grid's 3 row spans (the same candidates, the same tests); the distance test
// is the exact O1 predicate of the oracle (reading R1/R2) -- the paper's
// precision is unstated; the result-set append is `atomicAdd` on one global
// counter (nvcc aggregates it per warp), bounded by `cap` -- the counter keeps
// counting past the capacity, so the caller learns the exact |R| and reruns.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <type_traits>

#include "internal.h"
#include "predicate.cuh"

namespace hdb {

namespace {

constexpr int kPaperBlock = 256;   // the paper's block size

struct PArgs {
    const double2* xd;       // f64 mode: sorted exact coordinates
    const float2* xs;        // f32 mode
    const uint32_t* ids;     // A: sorted position -> point id
    const uint32_t* cstart;  // G: non-empty cell c holds sorted positions [cstart[c], cstart[c+1])
    const uint2* cspan;      // [nspan * n_nonempty] stencil row spans
    uint32_t nspan;
    uint64_t n_nonempty;
    double e2d;
    float e2f;
};

// atomic: gpuResultSet <- gpuResultSet u result   (Alg. 2 line 13, Alg. 3 line 22)
__device__ __forceinline__ void append(unsigned long long* ctr, uint64_t cap, uint32_t* rkey, uint32_t* rval,
                                       uint32_t key, uint32_t val) {
    const unsigned long long i = atomicAdd(ctr, 1ull);
    if (i < cap) {
        rkey[i] = key;
        rval[i] = val;
    }
}

// Alg. 2.  gid = sorted position (the points are in cell order, the paper's
// bin-sorted D); its cell by binary search in G (getNeighborCells).
template <bool F64>
__global__ void __launch_bounds__(kPaperBlock) k_paper_global(PArgs a, uint64_t n, unsigned long long* ctr,
                                                               uint64_t cap, uint32_t* rkey, uint32_t* rval) {
    const uint64_t gid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;   // line 2
    if (gid >= n) return;                                                  // line 3
    const uint32_t q = (uint32_t)gid;
    // line 6: the cell of the point -> its adjacent cells (row spans)
    uint64_t lo = 0, hi = a.n_nonempty;   // largest c with cstart[c] <= q
    while (hi - lo > 1) {
        const uint64_t mid = (lo + hi) >> 1;
        if (__ldg(&a.cstart[mid]) <= q) lo = mid;
        else hi = mid;
    }
    const uint32_t key = __ldg(&a.ids[q]);
    double2 pd = make_double2(0, 0);   // line 5: the point in registers
    float2 pf = make_float2(0, 0);
    if (F64) pd = a.xd[q];
    else pf = a.xs[q];
    for (uint32_t r = 0; r < a.nspan; ++r) {   // line 7
        const uint2 sp = __ldg(&a.cspan[(uint64_t)a.nspan * lo + r]);   // lines 8-9
        for (uint32_t k = sp.x; k < sp.y; ++k) {                       // line 10
            bool hit;                                                  // line 11
            if (F64) {
                const double2 v = a.xd[k];
                hit = pred_f64(pd.x, pd.y, v.x, v.y, a.e2d);
            } else {
                const float2 v = a.xs[k];
                hit = pred_f32(pf.x, pf.y, v.x, v.y, a.e2f);
            }
            if (hit) append(ctr, cap, rkey, rval, key, __ldg(&a.ids[k]));   // lines 12-13
        }
    }
}

// Alg. 3.  Block b processes non-empty cell S[b] = b (line 5).
template <bool F64>
__global__ void __launch_bounds__(kPaperBlock) k_paper_shared(PArgs a, unsigned long long* ctr, uint64_t cap,
                                                               uint32_t* rkey, uint32_t* rval) {
    using P2 = typename std::conditional<F64, double2, float2>::type;
    __shared__ P2 orig[kPaperBlock];     // line 6: pntsOriginCell
    __shared__ P2 comp[kPaperBlock];     // line 7: pntsCompCell
    __shared__ uint32_t comp_id[kPaperBlock];
    __shared__ uint2 cells[16];          // lines 8-9: cellIDsArr (row spans)
    const uint64_t c = blockIdx.x;
    const uint32_t t = threadIdx.x;
    if (t < a.nspan) cells[t] = __ldg(&a.cspan[(uint64_t)a.nspan * c + t]);
    const uint32_t o0 = __ldg(&a.cstart[c]), o1 = __ldg(&a.cstart[c + 1]);
    const P2* X = (const P2*)(F64 ? (const void*)a.xd : (const void*)a.xs);
    __syncthreads();   // line 10
    // "an additional loop" over origin tiles when the cell exceeds blockDim
    for (uint32_t ob = o0; ob < o1; ob += kPaperBlock) {
        const uint32_t q = ob + t;
        const bool has = q < o1;
        const uint32_t key = has ? __ldg(&a.ids[q]) : 0;
        for (uint32_t r = 0; r < a.nspan; ++r) {   // line 11: for cellID in cellIDsArr
            const uint2 sp = cells[r];
            for (uint32_t cb = sp.x; cb < sp.y; cb += kPaperBlock) {
                __syncthreads();   // the previous tile is no longer read
                if (has) orig[t] = X[q];                     // lines 12-14
                if (cb + t < sp.y) {                         // lines 15-17
                    comp[t] = X[cb + t];
                    comp_id[t] = __ldg(&a.ids[cb + t]);
                }
                __syncthreads();   // line 18
                if (has) {
                    const uint32_t m = min((uint32_t)kPaperBlock, sp.y - cb);
                    const P2 u = orig[t];
                    for (uint32_t j = 0; j < m; ++j) {   // lines 19-22
                        const P2 v = comp[j];
                        bool hit;
                        if (F64) hit = pred_f64(u.x, u.y, v.x, v.y, a.e2d);
                        else hit = pred_f32((float)u.x, (float)u.y, (float)v.x, (float)v.y, a.e2f);
                        if (hit) append(ctr, cap, rkey, rval, key, comp_id[j]);
                    }
                }
            }
        }
    }
}

// ConstructNeighborTable on R sorted by key: T_i^min / T_i^max of
// key i are the first / one-past-last positions of its run.  Every point is in
// its own list (self pair), so every key has a run.
__global__ void k_rows_from_keys(const uint32_t* __restrict__ key, uint64_t m, uint64_t* __restrict__ begin,
                                 uint32_t* __restrict__ count) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t k = key[i];
        if (i == 0 || key[i - 1] != k) begin[k] = i;
        if (i + 1 == m || key[i + 1] != k) count[k] = (uint32_t)(i + 1);   // end; minus begin below
    }
}
__global__ void k_rows_finish(uint64_t n, const uint64_t* __restrict__ begin, uint32_t* __restrict__ count) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        count[i] = (uint32_t)((uint64_t)count[i] - begin[i]);
}

PArgs pargs_of(const DevGrid& g) {
    PArgs a;
    a.xd = (const double2*)g.xy_s;
    a.xs = (const float2*)g.xy_s;
    a.ids = g.ids;
    a.cstart = g.cstart;
    a.cspan = g.cspan;
    a.nspan = g.nspan;
    a.n_nonempty = g.n_nonempty;
    a.e2d = g.e2_d;
    a.e2f = g.e2_f;
    return a;
}

}  // namespace

void launch_paper_search(const DevGrid& g, int which, unsigned long long* ctr, uint64_t cap, uint32_t* rkey,
                         uint32_t* rval, cudaStream_t s) {
    if (g.n == 0) return;
    const PArgs a = pargs_of(g);
    const bool f64 = g.dtype == HDB_F64;
    if (which == kPaperGlobal) {
        const unsigned blocks = (unsigned)((g.n + kPaperBlock - 1) / kPaperBlock);   // nGPU = |D| rounded up
        if (f64) k_paper_global<true><<<blocks, kPaperBlock, 0, s>>>(a, g.n, ctr, cap, rkey, rval);
        else k_paper_global<false><<<blocks, kPaperBlock, 0, s>>>(a, g.n, ctr, cap, rkey, rval);
    } else {
        const unsigned blocks = (unsigned)g.n_nonempty;   // N = #non-empty cells x blockDim
        if (f64) k_paper_shared<true><<<blocks, kPaperBlock, 0, s>>>(a, ctr, cap, rkey, rval);
        else k_paper_shared<false><<<blocks, kPaperBlock, 0, s>>>(a, ctr, cap, rkey, rval);
    }
    ++g_kernel_launches;
}

void launch_rows_from_keys(const uint32_t* key_sorted, uint64_t m, uint64_t n, uint64_t* begin, uint32_t* count,
                           cudaStream_t s) {
    if (m == 0) return;
    unsigned blocks = (unsigned)std::min<uint64_t>((m + 255) / 256, 148 * 32);
    k_rows_from_keys<<<blocks, 256, 0, s>>>(key_sorted, m, begin, count);
    blocks = (unsigned)std::min<uint64_t>((n + 255) / 256, 148 * 32);
    k_rows_finish<<<blocks, 256, 0, s>>>(n, begin, count);
    g_kernel_launches += 2;
}

}  // namespace hdb
