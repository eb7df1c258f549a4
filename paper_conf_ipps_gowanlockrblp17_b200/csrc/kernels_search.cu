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

#include <algorithm>
#include <cstdlib>

#include "internal.h"
#include "predicate.cuh"

namespace hdb {

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int kWarps = kSearchThreads / 32;

struct SArgs {
    const float4* xp;      // paired-SoA f32 coordinates {x_2k, x_2k+1, y_2k, y_2k+1}: filter coords (f64
                           // mode) / exact coords (f32 mode)
    const float2* xs;      // f32 mode: exact coordinates (sorted)
    const double2* xd;     // exact f64 coordinates (f64 mode)
    const uint32_t* ids;
    const uint32_t* cstart;
    const uint2* cspan;    // [nspan * non-empty cells]
    uint32_t nspan;        // 2k+1 stencil rows
    const uint32_t* gstart;
    const uint32_t* gcell;
    float e2f;             // f32 mode: fl32(eps^2); f64 mode: fl32(e2_d)
    float band;            // f64 mode, bbox-centre filter: decide in exact f64 when |t| <= band
    float band_l;          // f64 mode, group-local filter (count pass)
    float nb2_l;           //   -(band_l (1 + 2^-20))^2
    double e2d;            // fl64(eps^2)
    // dense/sparse hybrid (NEXT-1): the warp-per-group
    // kernels visit only the dense groups dl[dpre[g0] .. dpre[g1]) of a group range
    // (dl == null: every group); the sparse groups' queries sql[spre[g0] .. spre[g1])
    // = {sorted position, cell} go to the thread-per-query kernel k_sparse
    const uint32_t* dl;
    const uint32_t* dpre;
    // cost order (whole-range launches of the count / write pass): the dense groups, heaviest
    // first (group ids; the first dpre[ng] entries when dl is set) -- DESIGN.md "cost order"
    const uint32_t* ord;
    const uint2* sql;
    const uint32_t* spre;
    // query-lane blocks (k_qlanes): cell keys (row-major, < 2^30), grid width, points, and the
    // flag bound of the block-local filter (-(band_b (1 + 2^-20))^2)
    const uint64_t* ckey;
    uint32_t nx;
    uint32_t n;
    float nb2_b;
    // k_fused (f64 modes): the count phase stages each chunk's candidate pairs in shared
    // memory with cp.async one chunk ahead (the natural-order launches of large point sets,
    // whose candidates come from the L2 / DRAM rather than the L1)
    int pf;
    // position-space output (internal tables of the device sweep):
    // the single-pass kernels emit sorted positions instead of ids and write T by position
    int pos_out;
};

// the table entry for the point at sorted position s: its original id, or s itself
__device__ __forceinline__ uint32_t out_id(const SArgs& a, uint32_t s) { return a.pos_out ? s : __ldg(&a.ids[s]); }
template <bool POS>
__device__ __forceinline__ uint32_t qout(const SArgs& a, uint32_t s) {
    if (POS) return s;
    return __ldg(&a.ids[s]);
}

__device__ __forceinline__ void dense_range(const SArgs& a, uint32_t& i0, uint32_t& i1) {
    if (a.dl) {
        i0 = __ldg(&a.dpre[i0]);
        i1 = __ldg(&a.dpre[i1]);
    }
}

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
// predicated global store (keeps the st.global space after the pointer is laundered).
// No "memory" clobber: nothing in the kernels reads the output, and a clobber
// would pin every later shared/global load behind the store (serialising the
// emission loop on LDS latency).
__device__ __forceinline__ void stg_if(uint32_t* p, uint32_t v, bool f) {
    asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q st.global.u32 [%0], %1; }" ::"l"(p), "r"(v),
                 "r"((uint32_t)f));
}
// store v at p iff (m & bit) != 0 -- the mask test inside the asm keeps it one LOP3.P.
// HDB_STG_CS: the table's id stream is written with the streaming (evict-first)
// cache operator, so the GBs of output do not push the candidates out of the L2
#ifndef HDB_STG_CS
#define HDB_STG_CS 1
#endif
__device__ __forceinline__ void stg_if_bit(uint32_t* p, uint32_t v, uint32_t m, uint32_t bit) {
#if HDB_STG_CS
    asm volatile("{ .reg .pred q; .reg .b32 t; and.b32 t, %2, %3; setp.ne.b32 q, t, 0; @q st.global.cs.u32 [%0], %1; }" ::"l"(p),
                 "r"(v), "r"(m), "r"(bit));
#else
    asm volatile("{ .reg .pred q; .reg .b32 t; and.b32 t, %2, %3; setp.ne.b32 q, t, 0; @q st.global.u32 [%0], %1; }" ::"l"(p),
                 "r"(v), "r"(m), "r"(bit));
#endif
}
// HDB_LD_EL: candidate coordinates / ids read with an L2 evict-last policy (they are
// re-read by the neighbouring groups' stencils while the output streams past)
#ifndef HDB_LD_EL
#define HDB_LD_EL 1
#endif
#ifndef HDB_PF
#define HDB_PF 0   // 1: stage the natural-order launches' candidates via cp.async (A/B: C5 +0.4%, profiles/r2q)
#endif
__device__ __forceinline__ double2 ld_cand(const double2* p) {
#if HDB_LD_EL
    uint64_t pol;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    double2 r;
    asm("ld.global.nc.L2::cache_hint.v2.f64 {%0, %1}, [%2], %3;" : "=d"(r.x), "=d"(r.y) : "l"(p), "l"(pol));
    return r;
#else
    return __ldg(p);
#endif
}
__device__ __forceinline__ uint2 ld_ids(const uint2* p) {
#if HDB_LD_EL
    uint64_t pol;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    uint2 r;
    asm("ld.global.nc.L2::cache_hint.v2.u32 {%0, %1}, [%2], %3;" : "=r"(r.x), "=r"(r.y) : "l"(p), "l"(pol));
    return r;
#else
    return __ldg(p);
#endif
}
__device__ __forceinline__ u64x fma2(u64x a, u64x b, u64x c) {
    u64x r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const uint32_t sa = (uint32_t)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sa), "l"(gmem));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
    asm volatile("cp.async.wait_group %0;" ::"n"(N));
}

// Kernel modes: f32 input (exact f32 predicate), f64 input with the f32
// filter + exact f64 fallback, f64 input tested in exact f64 only (used when
// the filter bound is useless, e.g. extent/eps near 2^30 or huge coordinates).
enum Mode { kF32 = 0, kF64Filter = 1, kF64Exact = 2 };

// Dynamic work distribution: warps grab `chunk` consecutive query groups at a
// time from a global counter (heavy-tailed group costs: dense cells have up
// to ~60x the candidates of sparse ones, C2/C5).
__device__ __forceinline__ uint32_t grab(unsigned int* ctr, uint32_t chunk, int lane) {
    uint32_t v = 0;
    if (lane == 0) v = atomicAdd(ctr, chunk);
    return __shfl_sync(FULL, v, 0);
}

// Group feed with look-ahead (warp-per-group kernels).  Per group the warp
// used to wait on a chain of dependent loads before its first useful
// instruction -- the grab's atomic, then gstart / gcell / moff, then the spans
// and offsets; ncu put ~20% of the write pass's stall samples there.  Here the
// index stream runs two groups ahead (the next range's grab is issued one range
// early, the group id behind an index -- through the cost order or the dense
// list -- is loaded one group before its metadata) and the next group's level-1
// metadata (qs, nq, c, mask-table offsets) is loaded while the current group
// runs.  Holding reserved groups lengthens the tail only if the last groups are
// heavy; a.ord (heavy groups first, built with the grid) makes them light.
struct GMeta {
    uint32_t qs, nq, c;
    uint64_t ma, mb;   // mask-table words [ma, mb) (0 when moff is null)
};
__device__ __forceinline__ GMeta load_meta(const SArgs& a, const uint64_t* __restrict__ moff, uint32_t gi) {
    GMeta m;
    m.qs = __ldg(&a.gstart[gi]);
    m.nq = __ldg(&a.gstart[gi + 1]) - m.qs;   // groups tile the sorted order: gstart[ng] = n
    m.c = __ldg(&a.gcell[gi]);
    m.ma = moff ? __ldg(&moff[gi]) : 0;
    m.mb = moff ? __ldg(&moff[gi + 1]) : 0;
    return m;
}
template <class F>
__device__ __forceinline__ void for_each_group(const SArgs& a, const uint64_t* __restrict__ moff, uint32_t g0,
                                               uint32_t g1, uint32_t chunk, unsigned int* ctr, int lane, F&& body) {
    uint32_t i0 = g0, i1 = g1;
    dense_range(a, i0, i1);
    if (i1 <= i0) return;
    uint32_t tk = 0;   // lane 0: the pending grab (start of the range after the newest one)
    // the next index of the warp's stream after i (range end e); consumes the pending grab
    auto advance = [&](uint32_t& i, uint32_t& e) {
        uint32_t j = i + 1;
        if (j >= e) {
            j = i0 + __shfl_sync(FULL, tk, 0);
            e = min(j + chunk, i1);
            if (lane == 0 && j < i1) tk = atomicAdd(ctr, chunk);
        }
        i = j;
    };
    // group id of stream index i (clamped: look-ahead loads past the end stay in bounds)
    auto gid = [&](uint32_t i) -> uint32_t {
        i = min(i, i1 - 1);
        return a.ord ? __ldg(&a.ord[i]) : a.dl ? __ldg(&a.dl[i]) : i;
    };
    uint32_t ci = i0 + grab(ctr, chunk, lane), cend = min(ci + chunk, i1);
    if (lane == 0) tk = atomicAdd(ctr, chunk);
    uint32_t ni = ci, nend = cend;
    advance(ni, nend);
    GMeta m = load_meta(a, moff, gid(ci));
    uint32_t gn = gid(ni);
    while (ci < i1) {
        // unconditional (clamped) loads straight into the look-ahead registers: a
        // conditional load merged with a copy would wait for the data right here
        const GMeta mn = load_meta(a, moff, gn);   // gn arrived during the previous group
        uint32_t nni = ni, nnend = nend;
        advance(nni, nnend);                       // its grab was issued a range earlier
        const uint32_t gnn = gid(nni);
        body(m);
        ci = ni;
        m = mn;
        ni = nni;
        nend = nnend;
        gn = gnn;
    }
}

// Hit-mask table (count pass -> write pass).  Per group, chunks are grouped in
// windows of kWin; window v holds, for each query i, its kWin chunk masks
// contiguously: masks[v][i][kk] (uint2 = even / odd candidate halves).  The
// write pass then emits query by query inside a window, i.e. in runs of
// ~kWin * 27 consecutive ids per query (long sequential store streams).
constexpr int kWin = kMaskWin;

constexpr int kWinPad = kWin + 1;   // padded smem rows: 72-B stride, conflict-free per-lane access

// End of a window of the count pass: lane i (< nq) adds the popcounts of query
// i's kWin chunk masks to my (per window instead of per chunk: one warp
// barrier and shared load per window), stores them to the mask table (gmask
// non-null) and the window buffer is cleared for the next window.
// nck: the window's chunks (the rest of the row is zero)
__device__ __forceinline__ void flush_window(uint2 (*swin)[kWinPad], uint2* gmask, uint32_t v, uint32_t nq,
                                             uint32_t& my, int lane, bool clear = true, uint32_t nck = kWin) {
    __syncwarp();
    if ((uint32_t)lane < nq) {
        uint2 r[kWin];
#pragma unroll
        for (int kk = 0; kk < kWin; ++kk) {
            r[kk] = make_uint2(0, 0);
            if ((uint32_t)kk < nck) {
                r[kk] = swin[lane][kk];
                my += __popc(r[kk].x) + __popc(r[kk].y);
            }
        }
        if (gmask) {
            uint4* dst = (uint4*)(gmask + ((size_t)v * nq + lane) * kWin);
#pragma unroll
            for (int u = 0; u < kWin / 2; ++u)
                dst[u] = make_uint4(r[2 * u].x, r[2 * u].y, r[2 * u + 1].x, r[2 * u + 1].y);
        }
    }
    __syncwarp();
    // no clearing: every (query < nq, chunk < nck) entry is rewritten by the next window's
    // count loop before any reader looks at it, and readers stop at nck (a single-window
    // group of k_fused emits straight from swin: `clear` = false keeps that explicit)
    (void)clear;
}

// ---------------------------------------------------------------- virtual chunks
// A group's candidates are its 2k+1 row spans.  They are visited as ONE
// sequence of candidate pairs (2p, 2p+1) -- span r contributes the pairs
// lo_r/2 .. (hi_r-1)/2 -- cut into chunks of 32 pairs (one per lane), so only
// the group's last chunk is ragged (per-span chunks left ~17% of the lanes idle
// at k = 3).  VSpan r: [lo, hi) of the span, its first pair index and the
// position of that pair in the virtual sequence; entry nspan holds the total.
constexpr int kMaxSpans = 13;   // 2k + 1 for cell_split k <= 6
static_assert(kMaxSpans >= 2 * kMaxCellSplit + 1, "span table too small for the largest cell split");
struct VSpan {
    uint32_t lo, hi, pbase, vstart;
};

// lanes r < nspan load span r; warp prefix over the pair counts; returns the
// number of virtual pairs
// (ncand, optional: the group's candidate count, summed over the spans by one REDUX)
__device__ __forceinline__ uint32_t load_vspans(const SArgs& a, uint32_t c, VSpan* vs, int lane,
                                                uint32_t* ncand = nullptr) {
    uint32_t lo = 0, hi = 0, np = 0;
    if ((uint32_t)lane < a.nspan) {
        const uint2 sp = __ldg(&a.cspan[a.nspan * c + lane]);
        lo = sp.x;
        hi = sp.y;
        np = hi > lo ? ((hi + 1) >> 1) - (lo >> 1) : 0;
    }
    if (ncand) *ncand = __reduce_add_sync(FULL, hi - lo);   // empty spans have lo == hi
    static_assert(kMaxSpans + 1 <= 16, "the span prefix below covers 16 lanes");
    uint32_t incl = np;
#pragma unroll
    for (int o = 1; o < 16; o <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += y;
    }
    const uint32_t total = __shfl_sync(FULL, incl, a.nspan - 1);
    __syncwarp();
    if ((uint32_t)lane < a.nspan) vs[lane] = VSpan{lo, hi, lo >> 1, incl - np};
    if ((uint32_t)lane == a.nspan) vs[lane] = VSpan{0, 0, 0, total};
    __syncwarp();
    return total;
}

// Per-lane cursor over the virtual pair sequence: the lane's current span is
// cached in registers and only advanced when vp passes its end (vp grows by 32
// per chunk), so a chunk costs a compare and a few integer ops instead of a
// search over the span table (the search was ~15% of k_fused's instructions).
struct VCursor {
    uint32_t r;       // current span (~0 before the first)
    uint32_t next;    // first virtual pair after span r
    uint32_t delta;   // pbase - vstart of span r: s0 = 2 (vp + delta)
    uint32_t lo, hi;  // [lo, hi) of span r (lo = ~0, hi = 0 past the last span)
};
__device__ __forceinline__ void vc_init(VCursor& c) {
    c.r = ~0u;
    c.next = 0;
    c.delta = 0;
    c.lo = ~0u;
    c.hi = 0;
}
// candidate pair (s0, s0 + 1) of virtual pair vp (non-decreasing across calls) and
// its two validity flags.  Inside span r the pair index runs from lo/2 to (hi-1)/2,
// so s0 < hi and s0 + 1 >= lo always hold: v0 = s0 >= lo, v1 = s0 + 1 < hi.
__device__ __forceinline__ uint32_t vc_pair(VCursor& c, const VSpan* vs, uint32_t nspan, uint32_t vp, bool& v0,
                                            bool& v1) {
    while (vp >= c.next) {
        ++c.r;
        if (c.r >= nspan) {
            c.next = ~0u;
            c.delta = 0;
            c.lo = ~0u;
            c.hi = 0;
            break;
        }
        const VSpan e = vs[c.r];
        c.next = vs[c.r + 1].vstart;
        c.delta = e.pbase - e.vstart;
        c.lo = e.lo;
        c.hi = e.hi;
    }
    const uint32_t s0 = 2 * (vp + c.delta);
    v0 = s0 >= c.lo;
    v1 = s0 + 1 < c.hi;
    return s0;
}

// a6: the count pass.  Warp per query group; lane j holds the candidate PAIR
// (2k, 2k+1) of a 64-candidate chunk of the group's row spans (packed f32x2
// operands X = {x0, x1}, Y = {y0, y1}); every query of the group (broadcast
// from shared memory) is tested against the pair with FADD2/FFMA2, two
// ballots give the chunk's hit masks (lane 0 stores them to the window
// buffer), and at the end of the chunk lane i adds query i's popcounts.
// f64 mode: coordinates relative to the group's first query (|x - o| < 2w),
// so the f32 error band is ~1e-6 of eps^2; the band flag is accumulated per
// lane with one LOP3 (sign bit of fma(t, t, -B^2)) and checked once per chunk;
// the rare flagged chunk is replayed with the band tests in exact f64.
// Invalid candidate slots carry far coordinates (t = +inf): never hits, never flagged.
constexpr float kFarF = 1e30f;
constexpr double kFarD = 1e300;

// Count one query group (queries qs .. qs+nq-1 of non-empty cell c): hit masks
// to gmask (windowed layout; null = do not store), tests accumulated per lane;
// returns lane i's |N_eps(query i)| (0 for lanes >= nq).  swin needs no
// initialisation (every entry a reader looks at is written first); with
// keep_single and a single window (*nch_out <= kWin) the masks stay in swin
// (and are not stored to gmask) for the caller.
template <int MODE>
__device__ __forceinline__ uint32_t count_group(const SArgs& a, uint32_t qs, uint32_t c, uint32_t nq,
                                                uint2 (*swin)[kWinPad], VSpan* vsp, ulonglong2* sq, double2* sqd,
                                                uint2* gmask, unsigned long long& tests, int lane,
                                                bool keep_single = false, uint32_t* nch_out = nullptr,
                                                double2* cbuf = nullptr) {
    const ulonglong2* __restrict__ xp = (const ulonglong2*)a.xp;
    const u64x NE2 = pack2(-a.e2f, -a.e2f);
    const u64x NB2 = pack2(a.nb2_l, a.nb2_l);
    double2 o = make_double2(0, 0);
    if (MODE == kF64Filter) o = a.xd[qs];
    __syncwarp();
    if ((uint32_t)lane < nq) {
        const uint32_t q = qs + lane;
        if (MODE == kF32) {
            const float2 p = a.xs[q];
            sq[lane] = make_ulonglong2(pack2(p.x, p.x), pack2(p.y, p.y));
        } else {
            const double2 d = a.xd[q];
            sqd[lane] = d;
            if (MODE == kF64Filter) {
                const float qx = (float)__dsub_rn(d.x, o.x), qy = (float)__dsub_rn(d.y, o.y);
                sq[lane] = make_ulonglong2(pack2(qx, qx), pack2(qy, qy));
            }
        }
    }
    uint32_t my = 0;
    uint32_t ncand;
    const uint32_t npairs = load_vspans(a, c, vsp, lane, &ncand);
    const uint32_t nch = (npairs + 31) / 32;
    if (nch_out) *nch_out = nch;
    const bool keep = keep_single && nch <= kWin;
    if (keep) gmask = nullptr;
    if (lane == 0) tests += (unsigned long long)nq * ncand;   // candidate tests of the group
    VCursor cur;
    vc_init(cur);
    // cbuf (f64 modes, k_fused): each chunk's candidate pair is prefetched into the
    // warp's 2-stage buffer with cp.async one chunk ahead (lane j owns its slots, so
    // no warp barrier is needed), hiding the L2 / DRAM latency of the candidates
    const bool pf = MODE != kF32 && cbuf != nullptr;
    auto issue = [&](uint32_t kc) -> uint32_t {
        bool w0, w1;
        const uint32_t t0 = vc_pair(cur, vsp, a.nspan, 32 * kc + lane, w0, w1);
        double2* dst = cbuf + ((kc & 1) * 32 + lane) * 2;
        if (w0) cp_async16(dst, a.xd + t0);
        if (w1) cp_async16(dst + 1, a.xd + t0 + 1);
        cp_async_commit();
        return (uint32_t)w0 | ((uint32_t)w1 << 1);
    };
    uint32_t vf = (pf && nch) ? issue(0) : 0u;
    uint32_t k = 0;
#pragma unroll 1
    for (; k < nch; ++k) {
        const uint32_t kk = k % kWin;
        bool v0, v1;
        uint32_t s0 = 0;
        u64x X, Y;
        double2 d0 = make_double2(kFarD, kFarD), d1 = make_double2(kFarD, kFarD);
        ulonglong2 P = make_ulonglong2(0, 0);
        if (pf) {
            const uint32_t vfn = k + 1 < nch ? issue(k + 1) : (cp_async_commit(), 0u);
            cp_async_wait<1>();   // this lane's copies of chunk k have landed
            v0 = vf & 1u;
            v1 = vf & 2u;
            const double2* src = cbuf + ((k & 1) * 32 + lane) * 2;
            if (v0) d0 = src[0];
            if (v1) d1 = src[1];
            vf = vfn;
        } else {
            s0 = vc_pair(cur, vsp, a.nspan, 32 * k + lane, v0, v1);
            if (MODE == kF32) {
                if (v0 || v1) P = xp[s0 >> 1];
            } else {
                if (v0) d0 = ld_cand(a.xd + s0);
                if (v1) d1 = ld_cand(a.xd + s0 + 1);
            }
        }
        if (MODE == kF32) {
            const float2 px = unpack2(P.x), py = unpack2(P.y);
            X = pack2(v0 ? px.x : kFarF, v1 ? px.y : kFarF);
            Y = pack2(v0 ? py.x : kFarF, v1 ? py.y : kFarF);
        } else {
            if (MODE == kF64Filter) {
                X = pack2(v0 ? (float)__dsub_rn(d0.x, o.x) : kFarF, v1 ? (float)__dsub_rn(d1.x, o.x) : kFarF);
                Y = pack2(v0 ? (float)__dsub_rn(d0.y, o.y) : kFarF, v1 ? (float)__dsub_rn(d1.y, o.y) : kFarF);
            }
        }
        uint32_t acc = 0;   // f64 filter: sign bit set <=> some |t| <= band in this lane
        uint32_t i0 = 0;
        if (MODE == kF64Filter) {
            // four queries per step with their arithmetic issued before any ballot: the
            // ballots are warp-synchronous points the compiler does not schedule across, so
            // one query at a time left each FADD2 -> FFMA2 -> FFMA2 -> FSETP chain exposed
#pragma unroll 1
            for (; i0 + 4 <= nq; i0 += 4) {
                u64x tt[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const ulonglong2 Q = sq[i0 + j];
                    const u64x dx = sub2(Q.x, X);
                    const u64x dy = sub2(Q.y, Y);
                    tt[j] = fma2(dy, dy, fma2(dx, dx, NE2));   // (dx^2 - e2) + dy^2
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const float2 u = unpack2(fma2(tt[j], tt[j], NB2));   // t^2 - B^2 < 0  <=>  |t| < B
                    acc |= __float_as_uint(u.x) | __float_as_uint(u.y);
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const float2 t = unpack2(tt[j]);
                    const unsigned m0 = __ballot_sync(FULL, t.x < 0.f);
                    const unsigned m1 = __ballot_sync(FULL, t.y < 0.f);
                    if (lane == 0) swin[i0 + j][kk] = make_uint2(m0, m1);
                }
            }
        } else if (MODE == kF32) {
#pragma unroll 1
            for (; i0 + 4 <= nq; i0 += 4) {
                bool h0[4], h1[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const ulonglong2 Q = sq[i0 + j];
                    const u64x dx = sub2(Q.x, X);
                    const u64x dy = sub2(Q.y, Y);
                    // exact f32: fl(fl(dx^2) + fl(dy^2)), scalar add.rn (reading R2)
                    const float2 px = unpack2(mul2(dx, dx));
                    const float2 py = unpack2(mul2(dy, dy));
                    h0[j] = __fadd_rn(px.x, py.x) <= a.e2f;
                    h1[j] = __fadd_rn(px.y, py.y) <= a.e2f;
                }
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const unsigned m0 = __ballot_sync(FULL, h0[j]);
                    const unsigned m1 = __ballot_sync(FULL, h1[j]);
                    if (lane == 0) swin[i0 + j][kk] = make_uint2(m0, m1);
                }
            }
        }
#pragma unroll 4
        for (uint32_t i = i0; i < nq; ++i) {
            unsigned m0, m1;
            if (MODE == kF64Exact) {
                const double2 qd = sqd[i];
                m0 = __ballot_sync(FULL, pred_f64(qd.x, qd.y, d0.x, d0.y, a.e2d));
                m1 = __ballot_sync(FULL, pred_f64(qd.x, qd.y, d1.x, d1.y, a.e2d));
            } else {
                const ulonglong2 Q = sq[i];
                const u64x dx = sub2(Q.x, X);
                const u64x dy = sub2(Q.y, Y);
                if (MODE == kF64Filter) {
                    const u64x tt = fma2(dy, dy, fma2(dx, dx, NE2));   // (dx^2 - e2) + dy^2
                    const float2 t = unpack2(tt);
                    m0 = __ballot_sync(FULL, t.x < 0.f);
                    m1 = __ballot_sync(FULL, t.y < 0.f);
                    const float2 u = unpack2(fma2(tt, tt, NB2));         // t^2 - B^2 < 0  <=>  |t| < B
                    acc |= __float_as_uint(u.x) | __float_as_uint(u.y);
                } else {
                    // exact f32: fl(fl(dx^2) + fl(dy^2)) with scalar add.rn (ptxas would fuse
                    // mul.rn.f32x2 + add.rn.f32x2 into FFMA2 -- reading R2)
                    const float2 px = unpack2(mul2(dx, dx));
                    const float2 py = unpack2(mul2(dy, dy));
                    m0 = __ballot_sync(FULL, __fadd_rn(px.x, py.x) <= a.e2f);
                    m1 = __ballot_sync(FULL, __fadd_rn(px.y, py.y) <= a.e2f);
                }
            }
            if (lane == 0) swin[i][kk] = make_uint2(m0, m1);
        }
        if (MODE == kF64Filter && __any_sync(FULL, (int)acc < 0)) {
            // replay the chunk: tests in the band are decided in exact f64
#pragma unroll 1
            for (uint32_t i = 0; i < nq; ++i) {
                const ulonglong2 Q = sq[i];
                const u64x dx = sub2(Q.x, X);
                const u64x dy = sub2(Q.y, Y);
                const u64x tt = fma2(dy, dy, fma2(dx, dx, NE2));
                const float2 t = unpack2(tt);
                const float2 u = unpack2(fma2(tt, tt, NB2));
                const bool b0 = u.x < 0.f || __float_as_uint(u.x) == 0x80000000u;
                const bool b1 = u.y < 0.f || __float_as_uint(u.y) == 0x80000000u;
                if (!__any_sync(FULL, b0 | b1)) continue;
                const double2 qd = sqd[i];
                const bool e0 = b0 && pred_f64(qd.x, qd.y, d0.x, d0.y, a.e2d);
                const bool e1 = b1 && pred_f64(qd.x, qd.y, d1.x, d1.y, a.e2d);
                const unsigned m0 = (__ballot_sync(FULL, t.x < 0.f) & ~__ballot_sync(FULL, b0)) |
                                    __ballot_sync(FULL, e0);
                const unsigned m1 = (__ballot_sync(FULL, t.y < 0.f) & ~__ballot_sync(FULL, b1)) |
                                    __ballot_sync(FULL, e1);
                if (lane == 0) swin[i][kk] = make_uint2(m0, m1);
            }
        }
        if (kk == kWin - 1) flush_window(swin, gmask, k / kWin, nq, my, lane, !keep);
    }
    if ((k % kWin) != 0) flush_window(swin, gmask, k / kWin, nq, my, lane, !keep, k % kWin);
    return my;
}

template <int MODE>
__global__ void __launch_bounds__(kSearchThreads) k_count(SArgs a, uint32_t g0, uint32_t g1, uint32_t chunk,
                                                          unsigned int* __restrict__ ctr, uint32_t* __restrict__ cnt,
                                                          unsigned long long* __restrict__ tests_out,
                                                          uint2* __restrict__ masks, const uint64_t* __restrict__ moff) {
    constexpr bool F64 = MODE != kF32;
    __shared__ uint2 swin[kWarps][32][kWinPad];   // masks of the current window [query][chunk]
    __shared__ VSpan vsp[kWarps][kMaxSpans + 1];     // the group's spans as one pair sequence
    __shared__ ulonglong2 sq[kWarps][32];           // {{qx, qx}, {qy, qy}} packed f32 pairs
    __shared__ double2 sqd[F64 ? kWarps : 1][32];   // exact query coordinates (f64 modes)
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
#pragma unroll
    for (int kk = 0; kk < kWin; ++kk) swin[w][lane][kk] = make_uint2(0, 0);
    unsigned long long tests = 0;
    for_each_group(a, masks ? moff : nullptr, g0, g1, chunk, ctr, lane, [&](const GMeta& m) {
        uint2* gmask = masks ? masks + (m.ma >> 1) : nullptr;
        const uint32_t my =
            count_group<MODE>(a, m.qs, m.c, m.nq, swin[w], vsp[w], sq[w], sqd[F64 ? w : 0], gmask, tests, lane);
        if ((uint32_t)lane < m.nq) cnt[m.qs + lane] = my;
    });
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tests += __shfl_xor_sync(FULL, tests, o);
    if (tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

// a8 (recompute variant) / legacy count: warp per query group; lane j holds the candidate PAIR (2k, 2k+1)
// of the chunk (one 16-B load of the paired-SoA layout {x0, x1, y0, y1} gives
// the packed operands X = {x0, x1}, Y = {y0, y1} directly); each query is
// tested against 64 candidates with FADD2/FFMA2 and two ballots.
template <int MODE, bool WRITE>
__global__ void __launch_bounds__(kSearchThreads) k_search(SArgs a, uint32_t g0, uint32_t g1, uint32_t chunk,
                                                           unsigned int* __restrict__ ctr,
                                                           uint32_t* __restrict__ cnt,
                                                           unsigned long long* __restrict__ tests_out,
                                                           const uint64_t* __restrict__ off, uint64_t out_base,
                                                           uint32_t* __restrict__ out, uint2* __restrict__ masks,
                                                           const uint64_t* __restrict__ moff) {
    constexpr bool F64 = MODE != kF32;
    __shared__ uint2 swin[WRITE ? 1 : kWarps][32][kWinPad];   // count pass: masks of the current window
    __shared__ ulonglong2 sq[kWarps][32];          // {{qx, qx}, {qy, qy}} packed f32 pairs
    __shared__ double2 sqd[F64 ? kWarps : 1][32];  // exact query coordinates (f64 modes)
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    const ulonglong2* __restrict__ xp = (const ulonglong2*)a.xp;
    if (!WRITE) {
#pragma unroll
        for (int kk = 0; kk < kWin; ++kk) swin[WRITE ? 0 : w][lane][kk] = make_uint2(0, 0);
    }
    const u64x NE2 = pack2(-a.e2f, -a.e2f);
    const float band = a.band;
    unsigned long long tests = 0;
    uint32_t i0 = g0, i1 = g1;
    dense_range(a, i0, i1);
    uint32_t ii = i0 + grab(ctr, chunk, lane), iend = min(ii + chunk, i1);
    while (ii < i1) {
        const uint32_t gi = a.dl ? __ldg(&a.dl[ii]) : ii;
        const uint32_t qs = __ldg(&a.gstart[gi]);
        const uint32_t c = __ldg(&a.gcell[gi]);
        const uint32_t nq = min((uint32_t)kGroup, __ldg(&a.cstart[c + 1]) - qs);
        __syncwarp();
        if ((uint32_t)lane < nq) {
            const uint32_t q = qs + lane;
            const float4 P = a.xp[q >> 1];
            const float qx = (q & 1) ? P.y : P.x, qy = (q & 1) ? P.w : P.z;
            sq[w][lane] = make_ulonglong2(pack2(qx, qx), pack2(qy, qy));
            if (F64) sqd[F64 ? w : 0][lane] = a.xd[q];
        }
        uint32_t my = 0;        // count: this lane's query's count; write: its offset within the group
        uint32_t* gout = nullptr;
        if (WRITE) {
            const uint64_t gb = off[qs];
            gout = out + (gb - out_base);
            // materialise the group's base pointer so that every store address is one
            // IMAD.WIDE (32-bit index), not a 64-bit add chain re-derived from out_base
            asm volatile("mov.b64 %0, %0;" : "+l"(gout));
            if ((uint32_t)lane < nq) my = (uint32_t)(off[qs + lane] - gb);
        }
        // count pass: the hit masks of chunk k for query i go to masks[moff[gi]/2 + k*nq + i]
        uint2* gmask = (!WRITE && masks) ? masks + (__ldg(&moff[gi]) >> 1) : nullptr;
        uint32_t k = 0;
        __syncwarp();
#pragma unroll 1
        for (uint32_t r = 0; r < a.nspan; ++r) {
            const uint2 sp = __ldg(&a.cspan[a.nspan * c + r]);
            const uint32_t lo = sp.x, hi = sp.y;
            if (lo >= hi) continue;   // empty span: no chunk (the mask layout counts none)
#pragma unroll 1
            for (uint32_t c0 = lo & ~1u; c0 < hi; c0 += 64, ++k) {
                const uint32_t kk = k % kWin;   // count pass: chunk slot in the window buffer
                const uint32_t s0 = c0 + 2 * lane, s1 = s0 + 1;
                const bool v0 = s0 >= lo && s0 < hi, v1 = s1 >= lo && s1 < hi;
                ulonglong2 P = make_ulonglong2(0, 0);
                double2 d0 = make_double2(0, 0), d1 = make_double2(0, 0);
                if (v0 || v1) {
                    if (MODE == kF64Exact) {
                        d0 = a.xd[s0];
                        d1 = a.xd[s1];
                    } else {
                        P = xp[s0 >> 1];
                    }
                }
                uint2 id = make_uint2(0, 0);
                if (WRITE && (v0 || v1)) id = *(const uint2*)(a.ids + s0);
                if (!WRITE) tests += (unsigned long long)nq * (min(c0 + 64, hi) - max(c0, lo));
#pragma unroll 2
                for (uint32_t i = 0; i < nq; ++i) {
                    unsigned m0, m1;
                    if (MODE == kF64Exact) {
                        const double2 qd = sqd[F64 ? w : 0][i];
                        m0 = __ballot_sync(FULL, v0 && pred_f64(qd.x, qd.y, d0.x, d0.y, a.e2d));
                        m1 = __ballot_sync(FULL, v1 && pred_f64(qd.x, qd.y, d1.x, d1.y, a.e2d));
                    } else {
                        const ulonglong2 Q = sq[w][i];
                        const u64x dx = sub2(Q.x, P.x);
                        const u64x dy = sub2(Q.y, P.y);
                        if (MODE == kF64Filter) {
                            const float2 t = unpack2(fma2(dy, dy, fma2(dx, dx, NE2)));   // (dx^2 - e2) + dy^2
                            m0 = __ballot_sync(FULL, v0 && t.x < 0.f);
                            m1 = __ballot_sync(FULL, v1 && t.y < 0.f);
                            const float tm = fminf(v0 ? fabsf(t.x) : INFINITY, v1 ? fabsf(t.y) : INFINITY);
                            if (__any_sync(FULL, tm <= band)) {   // rare: decide these tests in exact f64
                                const bool b0 = v0 & (fabsf(t.x) <= band);
                                const bool b1 = v1 & (fabsf(t.y) <= band);
                                const double2 qd = sqd[F64 ? w : 0][i];
                                bool e0 = false, e1 = false;
                                if (b0) {
                                    const double2 p = a.xd[s0];
                                    e0 = pred_f64(qd.x, qd.y, p.x, p.y, a.e2d);
                                }
                                if (b1) {
                                    const double2 p = a.xd[s1];
                                    e1 = pred_f64(qd.x, qd.y, p.x, p.y, a.e2d);
                                }
                                m0 = (m0 & ~__ballot_sync(FULL, b0)) | __ballot_sync(FULL, e0);
                                m1 = (m1 & ~__ballot_sync(FULL, b1)) | __ballot_sync(FULL, e1);
                            }
                        } else {
                            // fl(fl(dx^2) + fl(dy^2)).  The sum is two scalar add.rn: ptxas fuses
                            // mul.rn.f32x2 + add.rn.f32x2 into FFMA2 (observed in SASS, even with
                            // --fmad=false), which would break the no-FMA contract (reading R2).
                            const float2 px = unpack2(mul2(dx, dx));
                            const float2 py = unpack2(mul2(dy, dy));
                            m0 = __ballot_sync(FULL, v0 && __fadd_rn(px.x, py.x) <= a.e2f);
                            m1 = __ballot_sync(FULL, v1 && __fadd_rn(px.y, py.y) <= a.e2f);
                        }
                    }
                    if (WRITE) {
                        // addresses computed by every lane, stores predicated (no branches)
                        const uint32_t n0 = __popc(m0);
                        const uint32_t b = __shfl_sync(FULL, my, i);
                        uint32_t* p0 = gout + (b + __popc(m0 & lt));
                        uint32_t* p1 = gout + (b + n0 + __popc(m1 & lt));
                        stg_if(p0, id.x, (m0 >> lane) & 1u);
                        stg_if(p1, id.y, (m1 >> lane) & 1u);
                        const uint32_t nn = n0 + __popc(m1);
                        my += ((uint32_t)lane == i) ? nn : 0u;
                    } else if (lane == 0) {
                        swin[WRITE ? 0 : w][i][kk] = make_uint2(m0, m1);   // one STS instead of per-lane selects
                    }
                }
                if (!WRITE) {
                    __syncwarp();
                    if ((uint32_t)lane < nq) {
                        const uint2 mk = swin[WRITE ? 0 : w][lane][kk];
                        my += __popc(mk.x) + __popc(mk.y);
                    }
                    uint32_t junk = 0;   // (counted above, per chunk)
                    if (gmask && kk == kWin - 1) flush_window(swin[WRITE ? 0 : w], gmask, k / kWin, nq, junk, lane);
                }
            }
        }
        uint32_t junk = 0;
        if (!WRITE && gmask && (k % kWin) != 0)
            flush_window(swin[WRITE ? 0 : w], gmask, k / kWin, nq, junk, lane, true, k % kWin);
        if (!WRITE && (uint32_t)lane < nq) cnt[qs + lane] = my;
        if (++ii >= iend) {
            ii = i0 + grab(ctr, chunk, lane);
            iend = min(ii + chunk, i1);
        }
    }
    if (!WRITE && tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

// a8 (mask path): emission only.  The count pass stored every query's hit
// masks per 64-candidate chunk (windowed layout above); this kernel replays the
// chunk order without any distance arithmetic.  Per window of kWin chunks the
// masks are staged in shared memory by cp.async (double-buffered, the next
// window's copy overlaps this window's stores), then the warp emits query by
// query: for query i the window's hits are one contiguous run of its CSR
// segment, written by ballot-free popc prefixes with all 32 lanes (lane j owns
// candidate pair (2j, 2j+1) of each chunk).  Long per-warp store streams keep
// L2 lines whole -- interleaving 32 query lists per chunk halved the store rate.
constexpr int kEmitThreads = 128;   // 4 warps per CTA (the padded window buffers are 28 KB per CTA)
constexpr int kEmitWarps = kEmitThreads / 32;

// Emission of one window for every query of the group: per query, the window's
// hits are one contiguous run of its list; per chunk, lane j stores its pair's
// hits at (run start + popc of the chunk's mask below j).  NCK = the window's
// chunks (a template: no per-chunk guards in the loop; emit_window picks one).
template <int NCK>
__device__ __forceinline__ void emit_rows(const uint2 (&ids)[kWin], const uint4 (*wq)[kWin + 1], uint32_t nq,
                                          uint32_t* gout, unsigned lt, unsigned lbit) {
#pragma unroll 1
    for (uint32_t i = 0; i < nq; ++i) {
#pragma unroll
        for (int kk = 0; kk < NCK; ++kk) {
            const uint4 e = wq[i][kk];   // broadcast
            stg_if_bit(gout + (e.z + __popc(e.x & lt)), ids[kk].x, e.x, lbit);
            stg_if_bit(gout + (e.w + __popc(e.y & lt)), ids[kk].y, e.y, lbit);
        }
    }
}
__device__ __forceinline__ void emit_window(uint32_t nck, const uint2 (&ids)[kWin], const uint4 (*wq)[kWin + 1],
                                            uint32_t nq, uint32_t* gout, unsigned lt, unsigned lbit) {
#define HDB_EMIT_CASE(N)                                                                   \
    case N:                                                                                \
        if (N < kWin) {                                                                    \
            emit_rows<(N < kWin ? N : kWin)>(ids, wq, nq, gout, lt, lbit);                 \
            break;                                                                         \
        }
    switch (nck) {
        HDB_EMIT_CASE(1)
        HDB_EMIT_CASE(2)
        HDB_EMIT_CASE(3)
        HDB_EMIT_CASE(4)
        HDB_EMIT_CASE(5)
        HDB_EMIT_CASE(6)
        HDB_EMIT_CASE(7)
        default: emit_rows<kWin>(ids, wq, nq, gout, lt, lbit); break;
    }
#undef HDB_EMIT_CASE
}

// this window's candidate ids: lane j holds pair (2j, 2j+1) of each of its nck chunks
__device__ __forceinline__ void window_ids(const SArgs& a, const VSpan* vsp, VCursor& cur, uint32_t v, uint32_t nck,
                                           uint2 (&ids)[kWin], int lane) {
#pragma unroll
    for (int kk = 0; kk < kWin; ++kk) {
        ids[kk] = make_uint2(0, 0);
        if ((uint32_t)kk < nck) {
            bool v0, v1;
            const uint32_t s0 = vc_pair(cur, vsp, a.nspan, 32 * (v * kWin + kk) + lane, v0, v1);
            if (v0 | v1) ids[kk] = a.pos_out ? make_uint2(s0, s0 + 1) : ld_ids((const uint2*)(a.ids + s0));
        }
    }
}

// Emit one query group from its hit masks: lane i starts query i's list at
// gout + my; raw / wq / vsp are the warp's buffers (see k_emit).
// nch: the group's chunk count when vsp already holds its spans (k_fused), else 0.
// swin (k_fused, single-window groups): the window's masks are still in the count
// phase's window buffer (count_group with keep_single) -- no mask round trip
// through the L2; gmask is unused then.
__device__ __forceinline__ void emit_group(const SArgs& a, uint32_t c, uint32_t nq, uint32_t nwin,
                                           const uint2* gmask, uint32_t* gout, uint32_t my,
                                           uint2 (*raw)[kWin + 2], uint4 (*wq)[kWin + 1], VSpan* vsp, int lane,
                                           uint32_t nch = 0, const uint2 (*swin)[kWinPad] = nullptr) {
    const unsigned lt = (1u << lane) - 1u, lbit = 1u << lane;
    // the group's spans as one sequence of candidate pairs (same chunks as the count pass)
    if (nch == 0) nch = (load_vspans(a, c, vsp, lane) + 31) / 32;
    VCursor cur;
    vc_init(cur);
    if (!swin) {
        __syncwarp();   // the previous group's buffers are no longer read
        if ((uint32_t)lane < nq) {   // prefetch window 0: lane i copies its 64-B mask row
            const uint4* src = (const uint4*)(gmask + (size_t)lane * kWin);
#pragma unroll
            for (int u = 0; u < kWin / 2; ++u) cp_async16(&raw[lane][2 * u], src + u);
        }
        cp_async_commit();
    }
#pragma unroll 1
    for (uint32_t v = 0; v < nwin; ++v) {
        // this window's candidate ids: lane j holds pair (2j, 2j+1) of each chunk
        const uint32_t nck = min((uint32_t)kWin, nch - v * kWin);
        uint2 ids[kWin];
        window_ids(a, vsp, cur, v, nck, ids, lane);
        if (!swin) cp_async_wait<0>();
        __syncwarp();
        // lane i turns its row of masks into output positions (all queries in parallel)
        if ((uint32_t)lane < nq) {
            const uint2* mrow = swin ? swin[lane] : raw[lane];
#pragma unroll
            for (int kk = 0; kk < kWin; ++kk) {
                if ((uint32_t)kk < nck) {
                    const uint2 m = mrow[kk];
                    const uint32_t p0 = my;
                    my += __popc(m.x);
                    wq[lane][kk] = make_uint4(m.x, m.y, p0, my);
                    my += __popc(m.y);
                }
            }
        }
        __syncwarp();
        // prefetch the next window's masks into the landing buffer (overlaps the stores)
        if (!swin) {
            if (v + 1 < nwin && (uint32_t)lane < nq) {
                const uint4* src = (const uint4*)(gmask + ((size_t)(v + 1) * nq + lane) * kWin);
#pragma unroll
                for (int u = 0; u < kWin / 2; ++u) cp_async16(&raw[lane][2 * u], src + u);
            }
            cp_async_commit();
        }
        // chunks of this window (the last window of a group is usually partial: short
        // groups, e.g. ~100-400 candidates on C5, have 2-7 of the 8 chunks)
        emit_window(nck, ids, wq, nq, gout, lt, lbit);
        __syncwarp();   // wq is rewritten for the next window
    }
    if (!swin) cp_async_wait<0>();
}

__global__ void __launch_bounds__(kEmitThreads) k_emit(SArgs a, uint32_t g0, uint32_t g1, uint32_t chunk,
                                                         unsigned int* __restrict__ ctr,
                                                         const uint64_t* __restrict__ off, uint64_t out_base,
                                                         uint32_t* __restrict__ out, const uint2* __restrict__ masks,
                                                         const uint64_t* __restrict__ moff,
                                                         uint64_t* __restrict__ begin, uint32_t* __restrict__ count) {
    // rows padded (80-B / 144-B strides) so the per-lane row accesses are bank-conflict free
    __shared__ __align__(16) uint2 raw[kEmitWarps][32][kWin + 2];   // cp.async landing buffer (next window's masks)
    __shared__ uint4 wq[kEmitWarps][32][kWin + 1];    // current window: {m0, m1, pos0, pos1} per (query, chunk)
    __shared__ VSpan vsp[kEmitWarps][kMaxSpans + 1];  // the group's spans as one pair sequence
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    auto body = [&](const GMeta& m) {
        const uint32_t nwin = (uint32_t)((m.mb - m.ma) / (2ull * m.nq * kWin));
        const uint64_t gb = off[m.qs];
        uint32_t* gout = out + (gb - out_base);
        asm volatile("mov.b64 %0, %0;" : "+l"(gout));
        uint32_t my = 0;   // lane i: output cursor of query i within the group
        if ((uint32_t)lane < m.nq) {
            const uint64_t b = off[m.qs + lane];
            my = (uint32_t)(b - gb);
            if (begin) {   // T by original id (a10): random 12-B writes overlapping the store stream
                const uint32_t id = __ldg(&a.ids[m.qs + lane]);
                begin[id] = b;
                count[id] = (uint32_t)(off[m.qs + lane + 1] - b);
            }
        }
        emit_group(a, m.c, m.nq, nwin, masks + (m.ma >> 1), gout, my, raw[w], wq[w], vsp[w], lane);
    };
    uint32_t i0 = g0, i1 = g1;
    dense_range(a, i0, i1);
    uint32_t ii = i0 + grab(ctr, chunk, lane), iend = min(ii + chunk, i1);
    while (ii < i1) {
        body(load_meta(a, moff, a.dl ? __ldg(&a.dl[ii]) : ii));
        if (++ii >= iend) {
            ii = i0 + grab(ctr, chunk, lane);
            iend = min(ii + chunk, i1);
        }
    }
}

// Single pass for a device-resident table (search_kernel 4, whole table):
// per group, count (hit masks to the group's slot of the mask table, which the
// same warp reads back right away -- it is still in L2), reserve the group's
// output with one atomicAdd on the pair counter, write begin/count by original
// id, then emit.  Rows land in reservation order (each list is still in
// candidate order).  If the reservation passes `cap` (the table was sized from
// the sampled estimate) the group is not emitted and *overflow is set; the
// host then rebuilds the table with the exact two-pass path.  Count work (FP32/
// ALU) of some warps overlaps the store streams of others.
constexpr int kFusedThreads = 128;
constexpr int kFusedWarps = kFusedThreads / 32;
#ifndef HDB_FUSED_MINB
#define HDB_FUSED_MINB (kWin <= 4 ? 8 : 7)
#endif
constexpr int kFusedMinBlocks = HDB_FUSED_MINB;
// per-warp shared memory: the count phase's buffers and the emit phase's share
// one union (the phases of a warp never overlap), so a CTA needs the larger of
// the two (~7 KB per warp) instead of their sum
struct FusedCount {
    uint2 swin[32][kWinPad];
    ulonglong2 sq[32];
    double2 sqd[32];
    double2 cand[2 * 32 * 2];   // count phase: 2-stage cp.async buffer of the candidate pairs (a.pf)
};
struct FusedEmit {
    uint2 raw[32][kWin + 2];
    uint4 wq[32][kWin + 1];
};
union __align__(16) FusedSmem {
    FusedCount c;
    FusedEmit e;
};
template <int MODE>
__global__ void __launch_bounds__(kFusedThreads, kFusedMinBlocks)
    k_fused(SArgs a, uint32_t g0, uint32_t g1, uint32_t chunk, unsigned int* __restrict__ ctr,
            uint32_t* __restrict__ cnt, unsigned long long* __restrict__ tests_out, uint2* __restrict__ masks,
            const uint64_t* __restrict__ moff, unsigned long long* __restrict__ pair_ctr, uint64_t cap,
            uint32_t* __restrict__ out, uint64_t* __restrict__ begin, uint32_t* __restrict__ count,
            unsigned int* __restrict__ overflow) {
    __shared__ FusedSmem sm[kFusedWarps];
    __shared__ VSpan vsp[kFusedWarps][kMaxSpans + 1];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    FusedSmem& my_sm = sm[w];
    unsigned long long tests = 0;
    for_each_group(a, moff, g0, g1, chunk, ctr, lane, [&](const GMeta& m) {
        // count (hit masks to the group's slot of the mask table)
        __syncwarp();   // the previous group's readers of the warp's buffers are done
        uint2* gmask = masks + (m.ma >> 1);
        uint32_t nch = 0;
        double2* cbuf = a.pf ? my_sm.c.cand : nullptr;   // stage the candidates with cp.async
        const uint32_t my = count_group<MODE>(a, m.qs, m.c, m.nq, my_sm.c.swin, vsp[w], my_sm.c.sq, my_sm.c.sqd,
                                              gmask, tests, lane, true, &nch, cbuf);
        // reserve the group's output
        uint32_t incl = my;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t total = __shfl_sync(FULL, incl, 31);
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(pair_ctr, (unsigned long long)total);
        base = __shfl_sync(FULL, base, 0);
        const uint32_t excl = incl - my;
        if ((uint32_t)lane < m.nq) {
            const uint32_t id = out_id(a, m.qs + lane);
            if (cnt) cnt[m.qs + lane] = my;   // counts in sorted order (optional)
#ifndef HDB_QX_NOT
            begin[id] = base + excl;
            count[id] = my;
#endif
        }
        if (base + total <= cap) {
            uint32_t* gout = out + base;
            asm volatile("mov.b64 %0, %0;" : "+l"(gout));
            const bool single = nch <= kWin;   // one window: its masks are still in swin
            if (!single) __threadfence_block();   // the masks this warp just stored are read back by cp.async
            __syncwarp();
            const uint32_t nwin = single ? 1u : (uint32_t)((m.mb - m.ma) / (2ull * m.nq * kWin));
            emit_group(a, m.c, m.nq, nwin, gmask, gout, excl, my_sm.e.raw, my_sm.e.wq, vsp[w], lane, nch,
                       single ? my_sm.c.swin : nullptr);
        } else if (lane == 0) {
            atomicOr(overflow, 1u);
        }
    });
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tests += __shfl_xor_sync(FULL, tests, o);
    if (tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

// Mask-table layout: words of group g = 2 * nq * kWin * (windows of kWin chunks of 32 virtual pairs)
__global__ void __launch_bounds__(256) k_mask_words(SArgs a, const uint32_t* __restrict__ ng_dev, uint64_t n,
                                                    uint32_t* __restrict__ words) {
    const uint64_t ng = *ng_dev;
    for (uint64_t g = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < n;
         g += (uint64_t)gridDim.x * blockDim.x) {
        if (g >= ng) {
            words[g] = 0;
            continue;
        }
        if (a.dl && a.dpre[g + 1] == a.dpre[g]) {   // sparse group: thread-per-query path, no masks
            words[g] = 0;
            continue;
        }
        const uint32_t qs = a.gstart[g], c = a.gcell[g];
        const uint32_t nq = min((uint32_t)kGroup, a.cstart[c + 1] - qs);
        uint32_t npairs = 0;
        for (uint32_t r = 0; r < a.nspan; ++r) {
            const uint2 sp = a.cspan[a.nspan * c + r];
            if (sp.y > sp.x) npairs += ((sp.y + 1) >> 1) - (sp.x >> 1);
        }
        const uint32_t ch = (npairs + 31) / 32;
        words[g] = 2 * nq * kWin * ((ch + kWin - 1) / kWin);
    }
}

// Sparse queries (NEXT-1, the dense/sparse hybrid):
// one thread per query of a sparse group -- GPUCalcGlobal's mapping (Alg. 2,
// P:443-450), which the paper found best where cells hold few points
// (Table II) -- scanning its cell's row spans with the exact
// predicate in the input precision.  Count pass: cnt[q]; write pass (same
// candidate order): out[off[q] - out_base ...].  A warp-per-group iteration
// costs ~300 instructions of set-up plus ~100 per 64-candidate chunk; a group
// of 2 queries with ~20 candidates (SDSS-like at eps 0.07) would use a whole
// warp for 40 tests.
template <bool F64, bool WRITE>
__global__ void __launch_bounds__(256) k_sparse(SArgs a, uint32_t g0, uint32_t g1, uint32_t* __restrict__ cnt,
                                                unsigned long long* __restrict__ tests_out,
                                                const uint64_t* __restrict__ off, uint64_t out_base,
                                                uint32_t* __restrict__ out, uint64_t* __restrict__ begin,
                                                uint32_t* __restrict__ count) {
    const uint32_t j0 = __ldg(&a.spre[g0]), j1 = __ldg(&a.spre[g1]);
    unsigned long long tests = 0;
    for (uint32_t j = j0 + blockIdx.x * blockDim.x + threadIdx.x; j < j1; j += gridDim.x * blockDim.x) {
        const uint2 e = __ldg(&a.sql[j]);
        const uint32_t q = e.x, c = e.y;
        double2 pd = make_double2(0, 0);
        float2 pf = make_float2(0, 0);
        if (F64) pd = a.xd[q];
        else pf = a.xs[q];
        uint32_t m = 0;
        uint32_t* o = nullptr;
        if (WRITE) {
            const uint64_t b = off[q];
            o = out + (b - out_base);
            if (begin) {   // T by original id (a10): the row's place in the table
                const uint32_t id = __ldg(&a.ids[q]);
                begin[id] = b;
                count[id] = (uint32_t)(off[q + 1] - b);
            }
        }
        auto test = [&](uint32_t k) -> bool {
            if (F64) {
                const double2 v = __ldg(&a.xd[k]);
                return pred_f64(pd.x, pd.y, v.x, v.y, a.e2d);
            }
            const float2 v = __ldg(&a.xs[k]);
            return pred_f32(pf.x, pf.y, v.x, v.y, a.e2f);
        };
        for (uint32_t r = 0; r < a.nspan; ++r) {
            const uint2 sp = __ldg(&a.cspan[a.nspan * c + r]);
            if (!WRITE) tests += sp.y - sp.x;
            uint32_t k = sp.x;
            // four candidates per step: the loads are issued together (memory-level parallelism;
            // a thread's candidates are a few short spans, so latency, not bandwidth, bounds it)
            for (; k + 4 <= sp.y; k += 4) {
                const bool h0 = test(k), h1 = test(k + 1), h2 = test(k + 2), h3 = test(k + 3);
                if (WRITE) {
                    if (h0) o[m++] = __ldg(&a.ids[k]);
                    if (h1) o[m++] = __ldg(&a.ids[k + 1]);
                    if (h2) o[m++] = __ldg(&a.ids[k + 2]);
                    if (h3) o[m++] = __ldg(&a.ids[k + 3]);
                } else {
                    m += (uint32_t)h0 + (uint32_t)h1 + (uint32_t)h2 + (uint32_t)h3;
                }
            }
            for (; k < sp.y; ++k) {
                if (test(k)) {
                    if (WRITE) o[m] = __ldg(&a.ids[k]);
                    ++m;
                }
            }
        }
        if (!WRITE) cnt[q] = m;
    }
    if (!WRITE && tests_out) {
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) tests += __shfl_xor_sync(FULL, tests, o);
        if ((threadIdx.x & 31) == 0 && tests) atomicAdd(tests_out, tests);
    }
}

// Single pass for the sparse queries of a device-resident table (the dense/sparse
// split with k_fused on the dense groups): a thread tests its query's candidates
// ONCE, keeping up to kSparseBuf hit ids in its shared-memory slot, reserves its
// row with a warp-aggregated atomicAdd on the pair counter shared with k_fused, and
// copies its hits out (a query with more hits re-scans its candidates for the
// copy).  The two-pass form tested every candidate twice (count, then write).
#ifndef HDB_SPARSE_BUF
#define HDB_SPARSE_BUF 16   // hit ids buffered per thread (16: C3L eps 0.07 -15%, eps 0.12 -21% vs the two passes)
#endif
#ifndef HDB_SPARSE_BLOCKS
#define HDB_SPARSE_BLOCKS 8
#endif
constexpr int kSparseBuf = HDB_SPARSE_BUF;
template <bool F64>
__global__ void __launch_bounds__(256) k_sparse_fused(SArgs a, uint32_t g0, uint32_t g1,
                                                      unsigned long long* __restrict__ tests_out,
                                                      unsigned long long* __restrict__ pair_ctr, uint64_t cap,
                                                      uint32_t* __restrict__ out, uint64_t* __restrict__ begin,
                                                      uint32_t* __restrict__ count, unsigned int* __restrict__ overflow) {
    __shared__ uint32_t sbuf[256][kSparseBuf + 1];   // +1: conflict-free per-thread rows
    uint32_t* buf = sbuf[threadIdx.x];
    const uint32_t j0 = __ldg(&a.spre[g0]), j1 = __ldg(&a.spre[g1]);   // the range's sparse queries
    const int lane = threadIdx.x & 31;
    unsigned long long tests = 0;
    // whole warps iterate (the reservation is warp-wide); idle lanes carry m = 0
    for (uint32_t jb = j0 + (blockIdx.x * blockDim.x + threadIdx.x) - lane; jb < j1; jb += gridDim.x * blockDim.x) {
        const uint32_t j = jb + lane;
        const bool act = j < j1;
        uint32_t q = 0, c = 0;
        if (act) {
            const uint2 e = __ldg(&a.sql[j]);
            q = e.x;
            c = e.y;
        }
        double2 pd = make_double2(0, 0);
        float2 pf = make_float2(0, 0);
        if (act) {
            if (F64) pd = a.xd[q];
            else pf = a.xs[q];
        }
        auto test = [&](uint32_t k) -> bool {
            if (F64) {
                const double2 v = __ldg(&a.xd[k]);
                return pred_f64(pd.x, pd.y, v.x, v.y, a.e2d);
            }
            const float2 v = __ldg(&a.xs[k]);
            return pred_f32(pf.x, pf.y, v.x, v.y, a.e2f);
        };
        uint32_t m = 0;
        if (act) {
            for (uint32_t r = 0; r < a.nspan; ++r) {
                const uint2 sp = __ldg(&a.cspan[a.nspan * c + r]);
                tests += sp.y - sp.x;
                uint32_t k = sp.x;
                for (; k + 4 <= sp.y; k += 4) {   // four loads in flight (latency-bound thread)
                    const bool h0 = test(k), h1 = test(k + 1), h2 = test(k + 2), h3 = test(k + 3);
                    if (h0) { if (m < kSparseBuf) buf[m] = out_id(a, k); ++m; }
                    if (h1) { if (m < kSparseBuf) buf[m] = out_id(a, k + 1); ++m; }
                    if (h2) { if (m < kSparseBuf) buf[m] = out_id(a, k + 2); ++m; }
                    if (h3) { if (m < kSparseBuf) buf[m] = out_id(a, k + 3); ++m; }
                }
                for (; k < sp.y; ++k)
                    if (test(k)) {
                        if (m < kSparseBuf) buf[m] = out_id(a, k);
                        ++m;
                    }
            }
        }
        // reserve the warp's rows: inclusive prefix of m, one atomic per warp
        uint32_t incl = m;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t total = __shfl_sync(FULL, incl, 31);
        unsigned long long base = 0;
        if (lane == 31 && total) base = atomicAdd(pair_ctr, (unsigned long long)total);
        base = __shfl_sync(FULL, base, 31);
        const uint64_t b = base + (incl - m);
        if (!act) continue;
        const uint32_t id = out_id(a, q);
        begin[id] = b;
        count[id] = m;
        if (base + total > cap) {   // the capacity bound failed: the host rebuilds exactly
            atomicOr(overflow, 1u);
            continue;
        }
        uint32_t* o = out + b;
        if (m <= kSparseBuf) {
            for (uint32_t i = 0; i < m; ++i) o[i] = buf[i];
        } else {   // more hits than the buffer: write them while re-testing (same order)
            uint32_t w = 0;
            for (uint32_t r = 0; r < a.nspan; ++r) {
                const uint2 sp = __ldg(&a.cspan[a.nspan * c + r]);
                for (uint32_t k = sp.x; k < sp.y; ++k)
                    if (test(k)) o[w++] = out_id(a, k);
            }
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) tests += __shfl_xor_sync(FULL, tests, o);
    if (tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
}

// ---------------------------------------------------------------- query-per-lane blocks
// Single pass for the SMALL groups of a device-resident table (DESIGN.md "query
// lanes"): Alg. 2's thread-per-query mapping with the candidates staged
// in shared memory as in Alg. 3.  Where cells hold few points (C5's
// sparse 99% of the area: ~11 queries, ~100 candidates per cell) a warp per cell
// leaves most lanes idle in the emission and pays its set-up per 11 queries; here
// a warp takes a BLOCK of up to 32 consecutive small queries of one cell row (up
// to kQCX cell columns apart), one query per lane:
//  * per stencil row r the union of the lanes' row spans (one contiguous range of
//    sorted positions: the spans of cells of one row are monotone) is staged in
//    shared memory as f32 pairs relative to the block's first query (f64 -> f32
//    once per candidate, so the filter band is that of a block-sized region, not
//    of the whole bounding box);
//  * each lane walks ITS span inside the staged union (broadcast-free per-lane
//    LDS.128, two candidates per FADD2/FFMA2) and shifts the sign bits of t into
//    per-lane hit words (SHF, no ballots); a word whose band flag is set is
//    replayed with the in-band tests decided in exact f64;
//  * one warp-wide reservation on the pair counter shared with k_fused, T by id,
//    then each lane walks its hit bits (FLO) writing ids into a shared-memory
//    stage at its list's offset, and the warp copies the stage out with aligned,
//    coalesced 16-B streaming stores -- the block's rows are one contiguous range.
// HDB_QX_CHECK: bounds-checking build (every shared / global index of k_qlanes checked, a
// violation traps) -- the substitute for compute-sanitizer runs (tools/qx_check.sh)
#ifdef HDB_QX_CHECK
#define QX_CHECK(c)                                                                         \
    do {                                                                                    \
        if (!(c)) {                                                                         \
            printf("k_qlanes bound check failed: %s (line %d)\n", #c, __LINE__);           \
            __trap();                                                                       \
        }                                                                                   \
    } while (0)
#else
#define QX_CHECK(c) ((void)0)
#endif
#ifndef HDB_QX_FULLB
#define HDB_QX_FULLB 1
#endif
constexpr int kQThreads = 128;
constexpr int kQWarps = kQThreads / 32;
#ifndef HDB_QX_GRAB
#define HDB_QX_GRAB 128
#endif
constexpr int kQGrab = HDB_QX_GRAB;   // small queries per grab (natural order: the L2 keeps the stencil rows);
                              // fewer when the warps would otherwise not all get work
// kQW, kQS, kQCX: internal.h (the grid build's classification bounds them)
constexpr int kQOut = 1280;                // output stage (ids): a block's rows in one round (C5: ~1,150)
static_assert(kQOut * 4 >= (kQS / 2 + 1 + 4) * 16, "the candidate stage overlays the output stage");
struct QSmem {
    uint32_t bits[kQW][32];    // hit words, [word][lane]
    uint32_t wtag[kQW][32];    // sorted position of the candidate of each word's MSB
    union {
        float4 cand[kQS / 2 + 1 + 4];   // testing: candidate pairs {x0, x1, y0, y1} of one row union
        uint32_t out[kQOut];   // emission: the block's ids in table order (offset by the misalignment)
    } st;
};
__device__ __forceinline__ void stg_cs_v4(uint32_t* p, uint4 v) {
    asm volatile("st.global.cs.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w));
}
__device__ __forceinline__ void stg_cs(uint32_t* p, uint32_t v) {
    asm volatile("st.global.cs.u32 [%0], %1;" ::"l"(p), "r"(v));
}
// (cur << 1) | (v >> 31): append the sign bit of v
__device__ __forceinline__ uint32_t push_sign(uint32_t cur, uint32_t v) {
    uint32_t r;
    asm("shf.l.wrap.b32 %0, %1, %2, 1;" : "=r"(r) : "r"(v), "r"(cur));
    return r;
}

#ifdef HDB_QX_PROF   // profiling build only: clock64 per phase, summed over warps, printed at the end
__device__ unsigned long long g_qx_prof[8];
__device__ unsigned int g_qx_done;
#define QX_T(i)                                         \
    do {                                                \
        const long long t_ = clock64();                 \
        if ((i) > 0) qx_acc[(i) - 1] += t_ - qx_last;   \
        qx_last = t_;                                   \
    } while (0)
#else
#define QX_T(i) ((void)0)
#endif
// MODE: kF64Filter (block-local f32 filter + exact f64 replay) or kF32 (exact f32);
// POS: position-space output (the device sweep's internal tables), a compile-time choice
template <int MODE, bool POS>
__global__ void __launch_bounds__(kQThreads, 7)   // 7 CTAs: 7 KB of shared memory per warp
    k_qlanes(SArgs a, uint32_t g0, uint32_t g1, uint32_t grab, unsigned int* __restrict__ ctr,
             unsigned long long* __restrict__ tests_out, unsigned long long* __restrict__ pair_ctr, uint64_t cap,
             uint32_t* __restrict__ out, uint64_t* __restrict__ begin, uint32_t* __restrict__ count,
             unsigned int* __restrict__ overflow) {
    __shared__ QSmem smem[kQWarps];
    const int lane = threadIdx.x & 31;
    QSmem& S = smem[threadIdx.x >> 5];
    const ulonglong2* const st2 = reinterpret_cast<const ulonglong2*>(S.st.cand);
    const u64x NE2 = pack2(-a.e2f, -a.e2f);
    const u64x NB2 = pack2(a.nb2_b, a.nb2_b);
    unsigned long long tests = 0;
#ifdef HDB_QX_PROF
    long long qx_acc[6] = {0, 0, 0, 0, 0, 0}, qx_last = 0;
#endif
    const uint32_t j0 = __ldg(&a.spre[g0]), j1 = __ldg(&a.spre[g1]);   // the range's small queries
    // work: grabs of `grab` small queries (the next grab is taken one grab early); the next
    // block's list entries, cell keys and first stencil rows are loaded while a block runs
    auto take = [&]() -> uint32_t {
        uint32_t v = 0;
        if (lane == 0) v = atomicAdd(ctr, grab);
        return j0 + __shfl_sync(FULL, v, 0);
    };
    constexpr int kPre = 3;   // stencil rows prefetched (k = 1: all)
    uint32_t j = take(), jn = take();
    uint32_t jend = min(j + grab, j1);
    uint2 e_n = make_uint2(0, 0), sp_n[kPre];
    uint32_t key_n = 0;
    double2 dq_n = make_double2(0, 0);   // f64 mode: the entry's query coordinates
    auto prefetch = [&](uint32_t jb, uint32_t je) {
        const bool in = jb + lane < je;
        e_n = in ? __ldg(&a.sql[jb + lane]) : make_uint2(0, 0);
        if (MODE == kF64Filter) dq_n = in ? __ldg(&a.xd[e_n.x]) : make_double2(0, 0);
        key_n = in ? (uint32_t)__ldg(&a.ckey[e_n.y]) : 0u;
#pragma unroll
        for (int r = 0; r < kPre; ++r)
            sp_n[r] = (in && (uint32_t)r < a.nspan) ? __ldg(&a.cspan[a.nspan * e_n.y + r]) : make_uint2(0, 0);
    };
    if (j < j1) prefetch(j, jend);
    while (j < j1) {
        {
            QX_T(0);
            // ---- the block: the leading run of queries in the row of the first one, at most
            // kQCX columns on, whose row spans stay within kQS of the first query's span starts
            const bool in = j + lane < jend;
            const uint2 e = e_n;
            const uint32_t key = key_n;
            const double2 dq0 = dq_n;
            const uint32_t key0 = __shfl_sync(FULL, key, 0);
            const uint32_t dk = key - key0;
            bool ok = in && dk <= (uint32_t)kQCX && key0 % a.nx + dk < a.nx;
            for (uint32_t r = 0; r < a.nspan; ++r) {
                uint2 sp;
                if (r < (uint32_t)kPre) {
                    sp = r == 0 ? sp_n[0] : r == 1 ? sp_n[1] : sp_n[2];
                } else {
                    sp = in ? __ldg(&a.cspan[a.nspan * e.y + r]) : make_uint2(0, 0);
                }
                const uint32_t lo0 = __shfl_sync(FULL, sp.x, 0);
                ok = ok && sp.x >= lo0 && sp.y - lo0 <= (uint32_t)kQS;
            }
            const unsigned okm = __ballot_sync(FULL, ok);
            uint32_t Q = ~okm ? (uint32_t)(__ffs(~okm) - 1) : 32u;
            if (Q == 0) {   // cannot happen for a classified small group; the host rebuilds exactly
                if (lane == 0) atomicOr(overflow, 1u);
                Q = 1;
            }
            // the next block's inputs (loads in flight while this block runs)
            {
                uint32_t jb = j + Q;
                if (jb >= jend) {
                    jb = jn;
                    jend = min(jn + grab, j1);
                    if (jn < j1) jn = take();
                }
                if (jb < j1) prefetch(jb, jend);
                if (Q == 1 && !(okm & 1u)) {   // (the Q == 0 case) skip the query
                    j = jb;
                    continue;
                }
                j = jb;   // (the current block's entries are e, Q, in registers)
            }
            QX_T(1);
            const bool act = (uint32_t)lane < Q;
            const uint32_t q = e.x, c = e.y;
            const uint32_t qid = act ? qout<POS>(a, q) : 0u;   // T by id (used after the reservation)
            double2 o = make_double2(0, 0);
            u64x QX, QY;
            if (MODE == kF64Filter) {
                const double2 dq = act ? dq0 : make_double2(0, 0);
                o.x = __shfl_sync(FULL, dq.x, 0);
                o.y = __shfl_sync(FULL, dq.y, 0);
                const float qx = (float)__dsub_rn(dq.x, o.x), qy = (float)__dsub_rn(dq.y, o.y);
                QX = pack2(qx, qx);
                QY = pack2(qy, qy);
            } else {
                const float2 p = act ? __ldg(&a.xs[q]) : make_float2(0, 0);
                QX = pack2(p.x, p.x);
                QY = pack2(p.y, p.y);
            }
            QX_T(2);
            // ---- per stencil row: the union [U0e, U1) of the lanes' spans is staged, then every
            // lane walks its own span inside it
            uint32_t my = 0, nw = 0;
            for (uint32_t r = 0; r < a.nspan; ++r) {
                const uint2 sp = act ? __ldg(&a.cspan[a.nspan * c + r]) : make_uint2(0, 0);
                const uint32_t U0 = __shfl_sync(FULL, sp.x, 0);
                const uint32_t U1 = __reduce_max_sync(FULL, act ? sp.y : 0u);
                const uint32_t U0e = U0 & ~1u;
                __syncwarp();   // the previous row's tests / the previous block's output copy are done
                if (U1 <= U0) continue;   // the row is empty for every lane (warp-uniform)
                if (act) tests += sp.y - sp.x;
                const uint32_t npu = (U1 - U0e + 1) >> 1;
                for (uint32_t p = lane; p < npu + 4; p += 32) {   // (+4 pairs of far-away padding: overrun)
                    float4 v = make_float4(kFarF, kFarF, kFarF, kFarF);
                    if (p < npu) {
                        const uint32_t s = U0e + 2 * p;
                        asm volatile("prefetch.global.L1 [%0];" ::"l"(a.ids + s));   // read by the emission
                        if (MODE == kF64Filter) {
                            const double2 c0 = ld_cand(a.xd + s);
                            v.x = (float)__dsub_rn(c0.x, o.x);
                            v.z = (float)__dsub_rn(c0.y, o.y);
                            if (s + 1 < a.n) {
                                const double2 c1 = ld_cand(a.xd + s + 1);
                                v.y = (float)__dsub_rn(c1.x, o.x);
                                v.w = (float)__dsub_rn(c1.y, o.y);
                            }
                        } else {
                            const float2 c0 = __ldg(&a.xs[s]);
                            v.x = c0.x;
                            v.z = c0.y;
                            if (s + 1 < a.n) {
                                const float2 c1 = __ldg(&a.xs[s + 1]);
                                v.y = c1.x;
                                v.w = c1.y;
                            }
                        }
                    }
                    QX_CHECK(p < (uint32_t)(kQS / 2 + 1 + 4));
                    S.st.cand[p] = v;
                }
                __syncwarp();
                // this lane's pairs [pa, pa + npl) of the staged union; the element before the
                // span (odd start) and after it (odd end) are masked off
                uint32_t npl = 0, pa = 0;
                if (act && sp.y > sp.x) {
                    pa = (sp.x - U0e) >> 1;
                    npl = ((sp.y - 1 - U0e) >> 1) - pa + 1;
                }
                uint32_t fix = ((sp.x - U0e) & 1u) ? 0x7fffffffu : ~0u;
                const bool odd_end = (sp.y - U0e) & 1u;
                for (uint32_t i = 0; i < npl; i += 16) {
                    const uint32_t cnt = min(16u, npl - i);
                    const ulonglong2* P = st2 + pa + i;
                    uint32_t cur = 0, acc = 0, proc = 0;
#pragma unroll 1
                    for (; proc < cnt; proc += 4) {
#pragma unroll
                        for (int u = 0; u < 4; ++u) {
                            QX_CHECK(pa + i + proc + u < npu + 4);
                            const ulonglong2 C = P[proc + u];
                            const u64x dx = sub2(QX, C.x);
                            const u64x dy = sub2(QY, C.y);
                            if (MODE == kF64Filter) {
                                const u64x tt = fma2(dy, dy, fma2(dx, dx, NE2));   // (dx^2 - e2) + dy^2
                                const float2 uu = unpack2(fma2(tt, tt, NB2));     // t^2 - B^2 < 0 <=> |t| < B
                                acc |= __float_as_uint(uu.x) | __float_as_uint(uu.y);
                                const float2 t = unpack2(tt);
                                cur = push_sign(cur, __float_as_uint(t.x));   // hit <=> t < 0 (t = +-0: in the band)
                                cur = push_sign(cur, __float_as_uint(t.y));
                            } else {
                                // exact f32 (reading R2): fl(fl(dx^2) + fl(dy^2)) <= e2; miss <=> e2 - s < 0
                                const float2 px = unpack2(mul2(dx, dx));
                                const float2 py = unpack2(mul2(dy, dy));
                                cur = push_sign(cur, __float_as_uint(__fsub_rn(a.e2f, __fadd_rn(px.x, py.x))));
                                cur = push_sign(cur, __float_as_uint(__fsub_rn(a.e2f, __fadd_rn(px.y, py.y))));
                            }
                        }
                    }
                    if (MODE == kF32) cur = ~cur;
                    cur <<= 2 * (16 - proc);   // bit 31 - 2p - e: element e of pair p
                    if (MODE == kF64Filter && (int)acc < 0) {
                        // a test of this word is within the band: decide the band tests in exact f64
                        const double2 dq = __ldg(&a.xd[q]);
                        for (uint32_t p = 0; p < cnt; ++p) {
                            const ulonglong2 C = P[p];
                            const u64x dx = sub2(QX, C.x);
                            const u64x dy = sub2(QY, C.y);
                            const u64x tt = fma2(dy, dy, fma2(dx, dx, NE2));
                            const float2 uu = unpack2(fma2(tt, tt, NB2));
#pragma unroll
                            for (int el = 0; el < 2; ++el) {
                                const float ue = el ? uu.y : uu.x;
                                const uint32_t sc = U0e + 2 * (pa + i + p) + el;
                                if ((ue < 0.f || __float_as_uint(ue) == 0x80000000u) && sc < a.n) {
                                    const double2 cd = __ldg(&a.xd[sc]);
                                    const uint32_t bit = 0x80000000u >> (2 * p + el);
                                    cur = pred_f64(dq.x, dq.y, cd.x, cd.y, a.e2d) ? (cur | bit) : (cur & ~bit);
                                }
                            }
                        }
                    }
                    uint32_t m = cnt == 16 ? ~0u : ~(~0u >> (2 * cnt));   // the word's 2 cnt elements
                    m &= fix;
                    fix = ~0u;
                    if (odd_end && i + 16 >= npl) m &= ~(1u << (32 - 2 * cnt));
                    cur &= m;
                    my += __popc(cur);
                    if (cur) {   // only words with hits are kept (the emission never skips a word)
                        QX_CHECK(nw < (uint32_t)kQW);
                        S.bits[nw][lane] = cur;
                        S.wtag[nw][lane] = U0e + 2 * (pa + i);
                        ++nw;
                    }
                }
            }
            QX_T(3);
            // ---- reserve the block's rows (one range: lane i's list at excl), T by id (a10)
            uint32_t incl = my;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(FULL, incl, d);
                if (lane >= d) incl += y;
            }
            const uint32_t total = __shfl_sync(FULL, incl, 31);
            unsigned long long base = 0;
#ifdef HDB_QX_NOATOM   // timing experiment only (wrong table): per-warp arenas instead of the counter
            {
                static __shared__ unsigned long long arena[kQWarps];
                const uint64_t wid = (uint64_t)blockIdx.x * kQWarps + (threadIdx.x >> 5);
                const uint64_t per = cap / ((uint64_t)gridDim.x * kQWarps);
                if (lane == 0) {
                    if (arena[threadIdx.x >> 5] + total > per || j == 0) arena[threadIdx.x >> 5] = 0;
                    base = wid * per + arena[threadIdx.x >> 5];
                    arena[threadIdx.x >> 5] += total;
                }
            }
#else
            if (lane == 0 && total) base = atomicAdd(pair_ctr, (unsigned long long)total);
#endif
            base = __shfl_sync(FULL, base, 0);
            const uint32_t excl = incl - my;
            if (base + total > cap) {   // the capacity bound failed: the host rebuilds exactly
                if (lane == 0) atomicOr(overflow, 1u);
                continue;
            }
#ifdef HDB_QX_NOEMIT   // timing experiment only (no table)
            continue;
#endif
            QX_T(4);
            // ---- emission in rounds of <= kQOut ids (one round unless the block is heavy): every
            // lane walks its hit bits (FLO) writing the ids (L1) into the output stage at its list's
            // offset (the stage is offset by the destination's misalignment); the stage is then
            // copied out with 16-B aligned streaming stores
            __syncwarp();   // (orders the words' stores before the reads below)
            uint32_t k = 0, cb = 0, src = 0, wi = 0;
            for (uint32_t r0 = 0; r0 < total;) {
                const uint32_t mis = (uint32_t)((base + r0) & 3u);
                const uint32_t cntr = min(total - r0, (uint32_t)kQOut - mis);
                const uint32_t rend = r0 + cntr;
                const uint32_t kend = min(my, rend > excl ? rend - excl : 0u);   // this round's hits: [k, kend)
                uint32_t* dst = S.st.out + mis + excl - r0;
                // kQB hits per step: positions first, then the id loads, then the stores
                constexpr int kQB = 8;
                // the next hit's sorted position (MSB first), loading the next word when cb runs out
                auto next_pos = [&]() -> uint32_t {
                    if (cb == 0) {
                        QX_CHECK(wi < nw);
                        cb = S.bits[wi][lane];
                        src = S.wtag[wi][lane];
                        ++wi;
                    }
                    uint32_t z;
                    asm("bfind.shiftamt.u32 %0, %1;" : "=r"(z) : "r"(cb));   // clz
                    cb ^= 0x80000000u >> z;
                    return src + z;
                };
#if HDB_QX_FULLB
                // whole batches without per-slot bounds, then the remainder one by one
                for (; k + kQB <= kend; k += kQB) {
                    uint32_t pos[kQB], v[kQB];
#pragma unroll
                    for (int u = 0; u < kQB; ++u) pos[u] = next_pos();
#pragma unroll
                    for (int u = 0; u < kQB; ++u) {
                        QX_CHECK(pos[u] < a.n);
                        v[u] = qout<POS>(a, pos[u]);   // (L1: prefetched by the staging)
                    }
#pragma unroll
                    for (int u = 0; u < kQB; ++u) {
                        QX_CHECK(mis + excl + k + u - r0 < (uint32_t)kQOut);
                        dst[k + u] = v[u];
                    }
                }
                for (; k < kend; ++k) dst[k] = qout<POS>(a, next_pos());
#else
                for (; k < kend; k += kQB) {
                    uint32_t pos[kQB];
#pragma unroll
                    for (int u = 0; u < kQB; ++u) {
                        pos[u] = 0;
                        if (k + u < kend) pos[u] = next_pos();
                    }
                    uint32_t v[kQB];
#pragma unroll
                    for (int u = 0; u < kQB; ++u)
                        if (k + u < kend) {
                            QX_CHECK(pos[u] < a.n);
                            v[u] = qout<POS>(a, pos[u]);   // (L1: prefetched by the staging)
                        }
#pragma unroll
                    for (int u = 0; u < kQB; ++u)
                        if (k + u < kend) {
                            QX_CHECK(mis + excl + k + u - r0 < (uint32_t)kQOut);
                            dst[k + u] = v[u];
                        }
                }
#endif
                k = kend;
                __syncwarp();
                QX_T(5);
                uint32_t* gd = out + (base + r0 - mis);   // 16-B aligned
                const uint32_t nch = (mis + cntr + 3) >> 2;
                for (uint32_t ch = lane; ch < nch; ch += 32) {
                    QX_CHECK(4 * ch + 3 < (uint32_t)kQOut);
                    const uint4 v = reinterpret_cast<const uint4*>(S.st.out)[ch];
                    const uint32_t e0 = 4 * ch;
                    if (e0 >= mis && e0 + 4 <= mis + cntr) {
                        stg_cs_v4(gd + e0, v);
                    } else {
                        const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                        for (int t = 0; t < 4; ++t)
                            if (e0 + t >= mis && e0 + t < mis + cntr) stg_cs(gd + e0 + t, w4[t]);
                    }
                }
                __syncwarp();   // the stage is rewritten by the next round / block
                QX_T(6);
                r0 = rend;
            }
#ifndef HDB_QX_NOT   // (timing experiment: no T by id)
            // T by id (a10), after the block's output (A/B against before it: equal)
            if (act) {
                begin[qid] = base + excl;
                count[qid] = my;
            }
#endif
        }
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) tests += __shfl_xor_sync(FULL, tests, d);
    if (tests_out && lane == 0 && tests) atomicAdd(tests_out, tests);
#ifdef HDB_QX_PROF
    if (lane == 0) {
        for (int i = 0; i < 6; ++i) atomicAdd(&g_qx_prof[i], (unsigned long long)qx_acc[i]);
        __threadfence();
        if (atomicAdd(&g_qx_done, 1u) + 1 == gridDim.x * kQWarps) {
            const char* nm[6] = {"formation", "query set-up", "stage+test", "reserve+T", "bit-walk", "copy-out"};
            unsigned long long t = 0;
            for (int i = 0; i < 6; ++i) t += g_qx_prof[i];
            for (int i = 0; i < 6; ++i)
                printf("qx_prof %-13s %6.2f%%  %.3e warp-cycles\n", nm[i], 100.0 * g_qx_prof[i] / t, (double)g_qx_prof[i]);
            for (int i = 0; i < 6; ++i) g_qx_prof[i] = 0;
            g_qx_done = 0;
        }
    }
#endif
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
        // cell of sorted position s: last c with cstart[c] <= s, by a 32-way warp search
        // (invariant cstart[lo] <= s < cstart[hi]; ~log32 steps of one load per lane)
        uint64_t lo = 0, hi = nne;
        while (hi - lo > 1) {
            const uint64_t step = (hi - lo + 31) / 32;
            const uint64_t idx = lo + (uint64_t)lane * step;
            const bool le = idx < hi && __ldg(&a.cstart[idx]) <= s;
            const uint32_t m = __popc(__ballot_sync(FULL, le));   // >= 1: lane 0 reads cstart[lo]
            const uint64_t nlo = lo + (uint64_t)(m - 1) * step;
            hi = min(hi, nlo + step);
            lo = nlo;
        }
        const uint64_t c = lo;
        uint32_t cntv = 0;
        if (F64) {
            const double2 q = a.xd[s];
            for (uint32_t r = 0; r < a.nspan; ++r) {
                const uint2 sp = a.cspan[a.nspan * c + r];
                for (uint32_t k = sp.x + lane; k < sp.y; k += 32) {
                    const double2 p = a.xd[k];
                    cntv += pred_f64(q.x, q.y, p.x, p.y, a.e2d) ? 1u : 0u;
                }
            }
        } else {
            const float2 q = a.xs[s];
            for (uint32_t r = 0; r < a.nspan; ++r) {
                const uint2 sp = a.cspan[a.nspan * c + r];
                for (uint32_t k = sp.x + lane; k < sp.y; k += 32) {
                    const float2 p = a.xs[k];
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



// The cost order (heavy groups first) trades the cell-sorted order's L2 locality
// for a shorter tail.  That pays while the point set stays L2-resident; beyond
// that the scattered visiting order re-reads each point's coordinates and id from
// DRAM for every stencil it is in (C5, 50M points: 14 GB of DRAM reads; natural order:
// single pass 14.5 -> 14.0 ms).  C3L (5M points, 100 MB) still gains from the order.
bool use_cost_order(const DevGrid& g) {
    const uint64_t esz = g.dtype == HDB_F64 ? 16 : 8;
    return g.ord && g.n * (esz + 4) <= (256ull << 20);
}

SArgs args_of(const DevGrid& g) {
    SArgs a;
    a.xp = g.xp;
    a.xs = (const float2*)g.xy_s;
    a.xd = (const double2*)g.xy_s;
    a.ids = g.ids;
    a.cstart = g.cstart;
    a.cspan = g.cspan;
    a.nspan = g.nspan;
    a.gstart = g.gstart;
    a.gcell = g.gcell;
    a.e2f = g.e2_f;
    a.band = g.band;
    a.band_l = g.band_l;
    a.nb2_l = g.nb2_l;
    a.e2d = g.e2_d;
    a.dl = g.dl;
    a.dpre = g.dpre;
    a.ord = nullptr;   // set by the whole-range count / write launches
    a.sql = g.sql;
    a.spre = g.spre;
    a.pf = 0;
    a.ckey = g.ckey;
    a.nx = g.nx;
    a.n = (uint32_t)g.n;
    a.nb2_b = g.nb2_b;
    a.pos_out = 0;
    return a;
}

// Groups the warp kernels visit in [g0, g1): all, or (dense/sparse split) the
// range's share of the dense groups -- sizes the grab chunk, so that a few
// heavy dense groups among many sparse ones still spread over every warp.
uint64_t dense_groups(const DevGrid& g, uint64_t g0, uint64_t g1) {
    if (!g.dl || g.n_groups == 0) return g1 - g0;
    return std::max<uint64_t>(1, (uint64_t)((double)(g1 - g0) * (double)g.n_dense_groups / (double)g.n_groups));
}

// One wave of resident CTAs; warps grab `chunk` groups at a time (~32 grabs
// per resident warp keeps the tail short while bounding counter atomics).
template <typename K>
void launch_groups(K kern, int& blocks_per_sm, uint64_t ng, uint32_t& chunk, unsigned& ctas,
                   int threads = kSearchThreads) {
    if (!blocks_per_sm) {
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks_per_sm, kern, threads, 0);
        if (blocks_per_sm < 1) blocks_per_sm = 1;
    }
    int dev = 0, nsm = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t wpb = (uint64_t)threads / 32;
    const uint64_t wave_warps = (uint64_t)nsm * blocks_per_sm * wpb;
    ctas = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((ng + wpb - 1) / wpb, (uint64_t)nsm * blocks_per_sm));
    chunk = (uint32_t)std::max<uint64_t>(1, ng / (wave_warps * 32));
}

template <int MODE, bool WRITE>
void launch_mode(const SArgs& a, uint64_t g0, uint64_t g1, uint64_t ngd, unsigned int* ctr, uint32_t* cnt,
                 unsigned long long* tests, const uint64_t* off, uint64_t out_base, uint32_t* out, uint2* masks,
                 const uint64_t* moff, cudaStream_t s) {
    static int bps = 0;
    uint32_t chunk;
    unsigned ctas;
    launch_groups(k_search<MODE, WRITE>, bps, ngd, chunk, ctas);
    k_search<MODE, WRITE><<<ctas, kSearchThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, chunk, ctr, cnt, tests, off,
                                                          out_base, out, masks, moff);
}

int mode_of(const DevGrid& g, bool force_exact) {
    return g.dtype == HDB_F32 ? kF32 : (g.filter && !force_exact ? kF64Filter : kF64Exact);
}

template <bool WRITE>
void launch_search(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                   const uint64_t* off, uint64_t out_base, uint32_t* out, bool force_exact, int slot, uint2* masks,
                   cudaStream_t s) {
    if (g1 <= g0) return;
    const SArgs a = args_of(g);
    unsigned int* ctr = g.counters + (slot % kCounterSlots);
    cudaMemsetAsync(ctr, 0, sizeof(unsigned int), s);
    const int mode = mode_of(g, force_exact);
    if (mode == kF64Filter)
        launch_mode<kF64Filter, WRITE>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, off, out_base, out, masks, g.moff, s);
    else if (mode == kF64Exact)
        launch_mode<kF64Exact, WRITE>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, off, out_base, out, masks, g.moff, s);
    else
        launch_mode<kF32, WRITE>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, off, out_base, out, masks, g.moff, s);
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

template <bool WRITE>
void launch_sparse(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                   const uint64_t* off, uint64_t out_base, uint32_t* out, cudaStream_t s, uint64_t* begin = nullptr,
                   uint32_t* count = nullptr) {
    if (!g.sql || g.n_sparse_q == 0 || g1 <= g0) return;
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((g.n_sparse_q + 255) / 256, 148 * 16));
    if (g.dtype == HDB_F64)
        k_sparse<true, WRITE><<<blocks, 256, 0, s>>>(args_of(g), (uint32_t)g0, (uint32_t)g1, cnt, tests, off, out_base,
                                                     out, begin, count);
    else
        k_sparse<false, WRITE><<<blocks, 256, 0, s>>>(args_of(g), (uint32_t)g0, (uint32_t)g1, cnt, tests, off,
                                                      out_base, out, begin, count);
    ++g_kernel_launches;
}

// variant (hdb_opts.search_kernel): 0 = default, 1 = force the exact-f64-only kernel
template <int MODE>
void launch_count_mode(const SArgs& a, uint64_t g0, uint64_t g1, uint64_t ngd, unsigned int* ctr, uint32_t* cnt,
                       unsigned long long* tests, uint2* masks, const uint64_t* moff, cudaStream_t s) {
    static int bps = 0;
    uint32_t chunk;
    unsigned ctas;
    launch_groups(k_count<MODE>, bps, ngd, chunk, ctas);
    k_count<MODE><<<ctas, kSearchThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, chunk, ctr, cnt, tests, masks, moff);
}

void launch_count(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests,
                  int variant, int slot, uint2* masks, cudaStream_t s) {
    if (g1 <= g0) return;
    SArgs a = args_of(g);
    if (g0 == 0 && g1 == g.n_groups && use_cost_order(g)) a.ord = g.ord;
    launch_sparse<false>(g, g0, g1, cnt, tests, nullptr, 0, nullptr, s);
    unsigned int* ctr = g.counters + (slot % kCounterSlots);
    cudaMemsetAsync(ctr, 0, sizeof(unsigned int), s);
    const int mode = g.dtype == HDB_F32 ? kF32 : (g.filter_l && variant != 1 ? kF64Filter : kF64Exact);
    if (mode == kF64Filter)
        launch_count_mode<kF64Filter>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, s);
    else if (mode == kF64Exact)
        launch_count_mode<kF64Exact>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, s);
    else
        launch_count_mode<kF32>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, s);
    ++g_kernel_launches;
}

// T by original id for the sorted positions of groups [g0, g1) (the recompute write
// variant; the default write kernels write it themselves): begin[ids[q]] = off[q],
// count[ids[q]] = off[q+1] - off[q], q in [gstart[g0], gstart[g1])
__global__ void __launch_bounds__(256) k_rows_direct(const uint32_t* __restrict__ ids,
                                                     const uint32_t* __restrict__ gstart, uint32_t g0, uint32_t g1,
                                                     const uint64_t* __restrict__ off, uint64_t* __restrict__ begin,
                                                     uint32_t* __restrict__ count) {
    const uint64_t q0 = gstart[g0], q1 = gstart[g1];
    for (uint64_t q = q0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; q < q1;
         q += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t id = ids[q];
        const uint64_t b = off[q];
        begin[id] = b;
        count[id] = (uint32_t)(off[q + 1] - b);
    }
}

void launch_rows_direct(const DevGrid& g, uint64_t g0, uint64_t g1, const uint64_t* off, uint64_t* begin,
                        uint32_t* count, cudaStream_t s) {
    const unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((g.n + 255) / 256, 148 * 16));
    k_rows_direct<<<blocks, 256, 0, s>>>(g.ids, g.gstart, (uint32_t)g0, (uint32_t)g1, off, begin, count);
    ++g_kernel_launches;
}

// masks != null: emission from the count pass's hit masks (k_emit); else the
// write pass recomputes the distance tests (k_search<WRITE>).
void launch_write(const DevGrid& g, uint64_t g0, uint64_t g1, const uint64_t* off, uint64_t out_base,
                  uint32_t* out, int variant, int slot, const uint2* masks, cudaStream_t s, uint64_t* begin,
                  uint32_t* count) {
    launch_sparse<true>(g, g0, g1, nullptr, nullptr, off, out_base, out, s, begin, count);
    if (!masks) {
        launch_search<true>(g, g0, g1, nullptr, nullptr, off, out_base, out, variant == 1, slot, nullptr, s);
        if (begin && g1 > g0) {   // the recompute variant leaves T by id to a direct pass
            launch_rows_direct(g, g0, g1, off, begin, count, s);
        }
        return;
    }
    if (g1 <= g0) return;
    unsigned int* ctr = g.counters + (slot % kCounterSlots);
    cudaMemsetAsync(ctr, 0, sizeof(unsigned int), s);
    // the write pass keeps the natural (cell-sorted) group order without look-ahead:
    // measured on B200 (tools/ab.sh), both cost order and look-ahead slowed the
    // store streams (C2 eps 0.45: 1.48 ms plain vs 1.55 ordered vs 1.56 look-ahead)
    const SArgs a = args_of(g);
    static int bps = 0;
    uint32_t chunk;
    unsigned ctas;
    launch_groups(k_emit, bps, dense_groups(g, g0, g1), chunk, ctas, kEmitThreads);
    k_emit<<<ctas, kEmitThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, chunk, ctr, off, out_base, out, masks,
                                         g.moff, begin, count);
    ++g_kernel_launches;
}

template <int MODE>
void launch_fused_mode(const SArgs& a, uint64_t g0, uint64_t g1, uint64_t ngd, unsigned int* ctr, uint32_t* cnt,
                       unsigned long long* tests, uint2* masks, const uint64_t* moff, unsigned long long* pair_ctr,
                       uint64_t cap, uint32_t* out, uint64_t* begin, uint32_t* count, unsigned int* overflow,
                       cudaStream_t s) {
    static int bps = 0;
    uint32_t chunk;
    unsigned ctas;
    // grabs sized by the groups the warps actually visit (the dense ones under the split)
    launch_groups(k_fused<MODE>, bps, ngd, chunk, ctas, kFusedThreads);
    // natural (cell-sorted) order: small grabs keep the front of groups in flight spatially
    // narrow, so the stencil rows above / below a group are still in the L2 (C5: grabs of
    // 31 / 16 / 8 / 4 groups: 16.13 / 15.71 / 15.60 / 15.48 ms per step)
    if (!a.ord) chunk = std::min<uint32_t>(chunk, 4);
    static const uint32_t chunk_env = [] {
        const char* e = std::getenv("HDB_FUSED_CHUNK");   // tuning knob (A/B runs)
        return e ? (uint32_t)std::strtoul(e, nullptr, 10) : 0u;
    }();
    if (chunk_env) chunk = chunk_env;
    k_fused<MODE><<<ctas, kFusedThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, chunk, ctr, cnt, tests, masks, moff,
                                                 pair_ctr, cap, out, begin, count, overflow);
}

void launch_fused(const DevGrid& g, uint64_t g0, uint64_t g1, uint32_t* cnt, unsigned long long* tests, uint2* masks,
                  unsigned long long* pair_ctr, uint64_t cap, uint32_t* out, uint64_t* begin, uint32_t* count,
                  unsigned int* overflow, cudaStream_t s, bool pos_out) {
    if (g1 <= g0) return;
    SArgs a = args_of(g);
    a.pos_out = pos_out ? 1 : 0;
    // heavy groups first (whole ranges only: ord lists every group): C2 eps 0.45 2.50 -> 2.10 ms
    if (g0 == 0 && g1 == g.n_groups && use_cost_order(g)) a.ord = g.ord;
    a.pf = HDB_PF && !a.ord && g.dtype == HDB_F64;   // the natural order: point sets beyond the L2
    unsigned int* ctr = g.counters;
    cudaMemsetAsync(ctr, 0, sizeof(unsigned int), s);
    const int mode = g.dtype == HDB_F32 ? kF32 : (g.filter_l ? kF64Filter : kF64Exact);
    if (mode == kF64Filter)
        launch_fused_mode<kF64Filter>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, pair_ctr, cap, out, begin, count,
                                      overflow, s);
    else if (mode == kF64Exact)
        launch_fused_mode<kF64Exact>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, pair_ctr, cap, out, begin, count,
                                     overflow, s);
    else
        launch_fused_mode<kF32>(a, g0, g1, dense_groups(g, g0, g1), ctr, cnt, tests, masks, g.moff, pair_ctr, cap, out, begin, count, overflow,
                                s);
    ++g_kernel_launches;
}

void launch_sparse_fused(const DevGrid& g, uint64_t g0, uint64_t g1, unsigned long long* tests,
                         unsigned long long* pair_ctr, uint64_t cap, uint32_t* out, uint64_t* begin, uint32_t* count,
                         unsigned int* overflow, cudaStream_t s, bool pos_out) {
    if (!g.sql || g.n_sparse_q == 0 || g1 <= g0) return;
    if (g.qsplit && (g.dtype == HDB_F32 || g.filter_b)) {
        // small groups (query-lane classification): blocks of up to 32 queries, one per lane
        SArgs a = args_of(g);
        a.pos_out = pos_out ? 1 : 0;
        static int bps[2] = {0, 0};
        const int f64 = g.dtype == HDB_F64;
        if (!bps[f64]) {
            if (f64) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps[1], k_qlanes<kF64Filter, false>, kQThreads, 0);
            else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps[0], k_qlanes<kF32, false>, kQThreads, 0);
            if (bps[f64] < 1) bps[f64] = 1;
        }
        // the range's small queries (whole range: all of them; a band's share is ~ its groups')
        const uint64_t nq = (g0 == 0 && g1 == g.n_groups)
                                ? g.n_sparse_q
                                : (uint64_t)((double)g.n_sparse_q * (double)(g1 - g0) / (double)g.n_groups) + 1;
        unsigned int* ctr = g.counters + (kCounterSlots - 1);
        HDB_CUDA(cudaMemsetAsync(ctr, 0, sizeof(unsigned int), s));
        const uint64_t warps = (uint64_t)148 * bps[f64] * kQWarps;
        const uint32_t grab = (uint32_t)std::max<uint64_t>(32, std::min<uint64_t>(kQGrab, nq / warps / 32 * 32));
        const uint64_t need = (nq + grab - 1) / grab;   // grabs (extra CTAs of a band exit at once)
        const unsigned ctas = (unsigned)std::max<uint64_t>(
            1, std::min<uint64_t>((uint64_t)148 * bps[f64], (need + kQWarps - 1) / kQWarps));
        auto go = [&](auto kern) {
            kern<<<ctas, kQThreads, 0, s>>>(a, (uint32_t)g0, (uint32_t)g1, grab, ctr, tests, pair_ctr, cap, out, begin,
                                            count, overflow);
        };
        if (f64) {
            if (pos_out) go(k_qlanes<kF64Filter, true>);
            else go(k_qlanes<kF64Filter, false>);
        } else {
            if (pos_out) go(k_qlanes<kF32, true>);
            else go(k_qlanes<kF32, false>);
        }
        ++g_kernel_launches;
        return;
    }
    SArgs as = args_of(g);
    as.pos_out = pos_out ? 1 : 0;
    const unsigned blocks =
        (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((g.n_sparse_q + 255) / 256, 148 * HDB_SPARSE_BLOCKS));
    if (g.dtype == HDB_F64)
        k_sparse_fused<true><<<blocks, 256, 0, s>>>(as, (uint32_t)g0, (uint32_t)g1, tests, pair_ctr, cap, out,
                                                    begin, count, overflow);
    else
        k_sparse_fused<false><<<blocks, 256, 0, s>>>(as, (uint32_t)g0, (uint32_t)g1, tests, pair_ctr, cap, out,
                                                     begin, count, overflow);
    ++g_kernel_launches;
}

void launch_mask_words(const DevGrid& g, const uint32_t* ng_dev, uint64_t n, uint32_t* words, cudaStream_t s) {
    unsigned blocks = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 148 * 16));
    k_mask_words<<<blocks, 256, 0, s>>>(args_of(g), ng_dev, n, words);
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


}  // namespace hdb
