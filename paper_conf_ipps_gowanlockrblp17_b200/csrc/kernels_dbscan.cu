// kernels_dbscan.cu -- DBSCAN on a DEVICE-resident neighbour table (NEXT-4,
// SURVEY 8(f)): the paper's modified DBSCAN (Alg. 1 with lookups in T,
// P:651-655) without moving T over PCIe, which the paper names as its
// bottleneck.  Same canonical labelling as the host code
// (R7): core <=> |N_eps(p)| >= minpts; clusters = components of the
// core-core graph numbered by increasing minimum core id; a border point takes
// the lowest-numbered cluster among its core neighbours; noise = -1.
//
//   k_core_init   core flags, parent[p] = p
//   k_sample_link every core u unites with 2 sampled core neighbours (Afforest-style
//                 pre-pass: assembles most of every dense cluster cheaply)
//   k_giant       the two most frequent roots among 1024 sampled points = the giant
//                 components A, B; k_giant_bits: their membership bitmaps
//   k_union       warp per core row (rows taken in the table's cell-sorted production
//                 order); each core-core edge not inside A or B is taken once
//                 (rule at k_union): union(u, v) by hooking the larger root under the smaller
//                 (atomicCAS), so every root stays the minimum id of its tree
//                 (ECL-CC style, path halving)
//   k_flatten     root[p] = root(p) for cores (read-only find); root flags
//   scan          cluster number of each root = rank of its id among the roots
//   k_labels      cores: number of their root; non-cores (lists < minpts long):
//                 min over core neighbours, or -1
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace hdb {

namespace {

constexpr unsigned FULL = 0xffffffffu;

// parent[] is read and written through L2 only (.cg): L1 is not coherent across
// SMs and a stale root would make unite() spin.
__device__ __forceinline__ uint32_t find_root(uint32_t* __restrict__ parent, uint32_t x) {
    uint32_t p = __ldcg(&parent[x]);
    while (p != x) {
        const uint32_t gp = __ldcg(&parent[p]);
        if (gp != p) __stcg(&parent[x], gp);   // path halving: gp is an ancestor (benign race)
        x = p;
        p = gp;
    }
    return x;
}

// Read-only root lookup through L1 (possibly stale).  Roots only ever merge, so
// if two stale lookups agree the elements ARE in one component; if they differ,
// unite() re-checks coherently.  This keeps the giant components' root entries
// (read by every edge) out of a single hot L2 line.
__device__ __forceinline__ uint32_t find_fast(const uint32_t* __restrict__ parent, uint32_t x) {
    uint32_t p = __ldca(&parent[x]);
    while (p != x) {
        x = p;
        p = __ldca(&parent[x]);
    }
    return x;
}

// key: null in id space (an element's id is its index); in position space the ids of the
// positions, so that a root is always its component's minimum core ID either way
__device__ __forceinline__ void unite(uint32_t* __restrict__ parent, uint32_t a, uint32_t b,
                                      const uint32_t* __restrict__ key) {
    while (true) {
        a = find_root(parent, a);
        b = find_root(parent, b);
        if (a == b) return;
        if (key ? __ldg(&key[a]) < __ldg(&key[b]) : a < b) {
            const uint32_t t = a;
            a = b;
            b = t;
        }
        // hang the larger root a under the smaller root b
        if (atomicCAS(&parent[a], a, b) == a) return;
    }
}

// parent[p] of a non-core point is kNonCore for the whole union phase: one
// load of parent[v] then answers both "is v core" and "where is v's root".
constexpr uint32_t kNonCore = 0xffffffffu;

__global__ void __launch_bounds__(256) k_core_init(const uint32_t* __restrict__ count, uint64_t n, uint32_t minpts,
                                                   uint8_t* __restrict__ core, uint32_t* __restrict__ parent) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        const bool c = count[p] >= minpts;
        core[p] = c ? 1 : 0;
        parent[p] = c ? (uint32_t)p : kNonCore;
    }
}

// True if x's root is `r` (read-only, possibly stale L1 reads): stops as soon
// as the chain reaches r, so the common case -- x hangs directly under the
// root already found for u -- costs one load.
__device__ __forceinline__ bool reaches(const uint32_t* __restrict__ parent, uint32_t x, uint32_t r) {
    uint32_t p = __ldca(&parent[x]);
    while (p != x) {
        if (p == r) return true;
        x = p;
        p = __ldca(&parent[x]);
    }
    return x == r;
}

// Walk order of the per-point passes (sampled links, labels).  The id-indexed arrays
// (begin, count, parent: 16 B per point) are read at u in either order; in the table's
// production (cell-sorted) order u is a random id but the lists stream, in id order u
// streams but the sampled list entry is a random read.  When those arrays fit in the L2
// the random id accesses are L2 hits and the production order wins (C2, 1.86M points:
// sampled links 0.93 vs 1.30 ms); beyond it (C5, 50M points, 800 MB) id order makes
// three of the four accesses coalesced (sampled links 17 -> 8.3 ms, labels 3.3 -> 0.26 ms).
constexpr double kIdOrderBytes = 48e6;// Consecutive (cell-sorted) rows per warp grab (<= 32: one per lane for the skip test --
// rows in A and non-core rows add no edge).  Short lists (mostly rows that are skipped,
// C5: 79 pairs per row, one giant): 32 rows, so the skip tests run 32 at a time; long lists
// (C2: 700-4,600 pairs per row, edge-bound): 4 rows, so the rows in flight on an SM stay
// few and their neighbours' parent entries stay in its L1.  Measured on one B200
// (device DBSCAN ms, grab 4 / 32): C5 16.6 / 12.4, C2 eps 0.45 3.8 / 7.1, eps 1.40 12.9 / 19.4.
constexpr uint32_t kGrabShort = 32, kGrabLong = 4;
constexpr double kLongListPairs = 256.0;
constexpr int kUnionThreads = 1024;       // one CTA per SM

// first row r in [0, n) with pre[r] >= x (pre = exclusive prefix of the list
// lengths along the walk order)
__device__ uint32_t row_of_pair(const uint64_t* __restrict__ pre, uint32_t n, uint64_t x) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = lo + (hi - lo) / 2;
        if (pre[mid] < x) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// list lengths along the walk order (rows[], identity if null)
__global__ void __launch_bounds__(256) k_row_counts(const uint32_t* __restrict__ count,
                                                    const uint32_t* __restrict__ rows, uint64_t n,
                                                    uint32_t* __restrict__ out) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        out[i] = count[rows ? rows[i] : i];
}

constexpr uint32_t kSampleLinks = 2;   // edges per core linked before the full pass

// Afforest-style pre-pass (Sutton et al., IPDPS 2018): every core u unites with
// kSampleLinks of its core neighbours, taken at evenly spaced list positions.
// On an eps-graph this already assembles most of every dense cluster.  The
// read-only root test first keeps the CAS traffic off the giant roots.
// Round k links every core u with its list entry at position m*k/(kSampleLinks+1);
// k_compress between rounds points every core straight at its root.
__global__ void __launch_bounds__(256) k_sample_link(const uint64_t* __restrict__ begin,
                                                     const uint32_t* __restrict__ count,
                                                     const uint32_t* __restrict__ nbrs,
                                                     const uint32_t* __restrict__ rows, uint64_t n, uint32_t k,
                                                     uint32_t* __restrict__ parent, const uint32_t* __restrict__ key) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t u = rows ? rows[i] : (uint32_t)i;
        const uint32_t pu = __ldcg(&parent[u]);
        if (pu == kNonCore) continue;
        const uint32_t v = nbrs[begin[u] + (uint64_t)count[u] * k / (kSampleLinks + 1)];
        const uint32_t pv = __ldcg(&parent[v]);
        if (v != u && pv != kNonCore && pv != pu) unite(parent, u, v, key);
    }
}

__global__ void __launch_bounds__(256) k_compress(uint64_t n, uint32_t* __restrict__ parent) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t q = __ldcg(&parent[p]);
        if (q == kNonCore || q == (uint32_t)p) continue;
        uint32_t r = q, x = __ldcg(&parent[r]);
        while (x != r) {
            r = x;
            x = __ldcg(&parent[r]);
        }
        if (r != q) __stcg(&parent[p], r);
    }
}

// One CTA: the two most frequent roots among 1024 sampled points after the
// pre-pass (the "giant" components A = giant[0], B = giant[1]; kNonCore if a
// root holds fewer than kGiantMin samples).
constexpr int kGiantSamples = 1024;
constexpr unsigned long long kGiantMin = kGiantSamples / 8;
__global__ void __launch_bounds__(kGiantSamples) k_giant(const uint32_t* __restrict__ rows, uint64_t n,
                                                         uint32_t* __restrict__ parent, uint32_t* __restrict__ giant) {
    __shared__ uint32_t sv[kGiantSamples];
    __shared__ unsigned long long best, second;
    const uint32_t t = threadIdx.x;
    const uint64_t i = (uint64_t)t * n / kGiantSamples;
    uint32_t r = kNonCore;
    if (i < n) {
        const uint32_t p = rows ? rows[i] : (uint32_t)i;
        if (__ldcg(&parent[p]) != kNonCore) r = find_root(parent, p);
    }
    sv[t] = r;
    if (t == 0) best = second = 0;
    __syncthreads();
    for (int k = 2; k <= kGiantSamples; k <<= 1)   // bitonic sort
        for (int j = k >> 1; j > 0; j >>= 1) {
            const uint32_t o = t ^ j;
            if (o > t) {
                const uint32_t x = sv[t], y = sv[o];
                if (((t & k) == 0) == (x > y)) {
                    sv[t] = y;
                    sv[o] = x;
                }
            }
            __syncthreads();
        }
    unsigned long long run = 0;
    if (sv[t] != kNonCore && (t == 0 || sv[t - 1] != sv[t])) {
        uint32_t e = t + 1;
        while (e < kGiantSamples && sv[e] == sv[t]) ++e;
        run = ((unsigned long long)(e - t) << 32) | sv[t];
        atomicMax(&best, run);
    }
    __syncthreads();
    if (run && run != best) atomicMax(&second, run);
    __syncthreads();
    if (t == 0) {
        giant[0] = (best >> 32) >= kGiantMin ? (uint32_t)best : kNonCore;
        giant[1] = (second >> 32) >= kGiantMin ? (uint32_t)second : kNonCore;
    }
}

// Membership bitmaps of A and B after the pre-pass (bit p of word p/32).
__global__ void __launch_bounds__(256) k_giant_bits(uint64_t n, const uint32_t* __restrict__ parent,
                                                    const uint32_t* __restrict__ giant, uint32_t* __restrict__ bits_a,
                                                    uint32_t* __restrict__ bits_b) {
    const uint32_t A = giant[0], B = giant[1];
    const uint64_t nw = (n + 31) / 32;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < 32 * nw;
         i += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t r = kNonCore;
        if (i < n && A != kNonCore && __ldcg(&parent[i]) != kNonCore) r = find_fast(parent, (uint32_t)i);
        const unsigned ma = __ballot_sync(FULL, r == A && r != kNonCore);
        const unsigned mb = __ballot_sync(FULL, r == B && r != kNonCore);
        if ((threadIdx.x & 31) == 0) {
            bits_a[i / 32] = ma;
            bits_b[i / 32] = mb;
        }
    }
}

__device__ __forceinline__ bool bit_of(const uint32_t* __restrict__ bits, uint32_t v) {
    return (__ldg(&bits[v >> 5]) >> (v & 31)) & 1u;
}

// Work regions of k_union: region c = rows [sched[c], sched[G + c]) of the
// production order holding ~1/G of the pairs; sched[c] doubles as the region's
// grab counter.
__global__ void k_sched_init(const uint64_t* __restrict__ pre, uint32_t n, uint64_t npairs, uint32_t G,
                             uint32_t* __restrict__ sched) {
    for (uint32_t c = threadIdx.x; c < G; c += blockDim.x) {
        sched[c] = row_of_pair(pre, n, npairs * c / G);
        sched[G + c] = c + 1 == G ? n : row_of_pair(pre, n, npairs * (c + 1) / G);
    }
}

// Main pass.  CTA c (one per SM) starts in region c; its warps take
// kRowsPerGrab consecutive rows at a time from the region's counter, so an SM
// works in one small region of space and its random parent[v] reads share L1.
// A warp whose region is exhausted moves on to region c+1, c+2, ... (work
// stealing without barriers).
//
// Which core-core edges (u, v) a row u processes, with A, B the giant
// components of the pre-pass (each edge of the graph ends up processed once,
// or is already inside one component):
//   u in A:        none           (A-A: one component; A-x: done by x's side)
//   u in B:        v in A         (B-B: one component; B-other: done by other's side)
//   u elsewhere:   v in A or B, or v < u (other-other edges from the larger end)
// Processing = one load of parent[v] (kNonCore: v not core); skip if v hangs
// under u's root; else follow the chain and unite if the roots differ.
__global__ void __launch_bounds__(kUnionThreads, 1)
    k_union(const uint64_t* __restrict__ begin, const uint32_t* __restrict__ count, const uint32_t* __restrict__ nbrs,
            const uint32_t* __restrict__ rows, uint32_t* __restrict__ parent, const uint32_t* __restrict__ giant,
            const uint32_t* __restrict__ bits_a, const uint32_t* __restrict__ bits_b, uint32_t* __restrict__ sched,
            uint32_t kRowsPerGrab, const uint32_t* __restrict__ key) {
    const bool have_a = giant[0] != kNonCore, have_b = giant[1] != kNonCore;
    const uint32_t G = gridDim.x;
    const int lane = threadIdx.x & 31;
    uint32_t region = blockIdx.x, visited = 0;
    while (visited < G) {
        {
            uint32_t r0 = 0;
            if (lane == 0) r0 = atomicAdd(&sched[region], kRowsPerGrab);
            r0 = __shfl_sync(FULL, r0, 0);
            const uint32_t end = __ldg(&sched[G + region]);
            if (r0 >= end) {
                region = region + 1 == G ? 0 : region + 1;
                ++visited;
                continue;
            }
            const uint32_t r1 = min(end, r0 + kRowsPerGrab);
            // the skip test for all 32 rows at once (one row per lane), then the warp walks the
            // lists of the rows that remain -- at C5 (one giant component) nearly every row is
            // in A, and testing them one after the other was a chain of dependent loads per row
            const uint32_t rl = r0 + lane;
            uint32_t ul = 0;
            bool keep = false;
            if (rl < r1) {
                ul = rows ? __ldg(&rows[rl]) : rl;
                keep = !(have_a && bit_of(bits_a, ul)) && __ldca(&parent[ul]) != kNonCore;
            }
            for (unsigned todo = __ballot_sync(FULL, keep); todo; todo &= todo - 1) {
                const uint32_t u = __shfl_sync(FULL, ul, __ffs(todo) - 1);
                const bool in_b = have_b && bit_of(bits_b, u);
                const uint32_t* L = nbrs + begin[u];
                const uint32_t m = count[u];
                uint32_t ru = find_fast(parent, u);
                for (uint32_t j0 = 0; j0 < m; j0 += 128) {
                    uint32_t v[4], p[4];
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const uint32_t j = j0 + lane + 32 * k;
                        v[k] = j < m ? __ldg(&L[j]) : 0xffffffffu;
                    }
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        bool take = false;
                        if (v[k] != 0xffffffffu) {
                            const bool va = have_a && bit_of(bits_a, v[k]);
                            take = in_b ? va : (va || v[k] < u || (have_b && bit_of(bits_b, v[k])));
                        }
                        p[k] = take ? __ldca(&parent[v[k]]) : kNonCore;
                    }
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        // skip non-cores and v hanging directly under u's root; else follow the chain
                        if (p[k] != kNonCore && p[k] != ru && !(p[k] != v[k] && reaches(parent, p[k], ru))) {
                            unite(parent, u, v[k], key);
                            ru = find_fast(parent, u);
                        }
                    }
                }
            }
        }
    }
}

// Roots into a separate array with a read-only find: path-halving writes racing
// with a "parent[p] = root" store could leave a non-root in parent[p].
__global__ void __launch_bounds__(256) k_flatten(const uint8_t* __restrict__ core, uint64_t n,
                                                 const uint32_t* __restrict__ parent, uint32_t* __restrict__ root,
                                                 uint32_t* __restrict__ is_root) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t r = 0, rt = (uint32_t)p;
        if (core[p]) {
            rt = find_fast(parent, (uint32_t)p);   // no writer is left: L1 reads are coherent here
            r = rt == (uint32_t)p ? 1u : 0u;
        }
        root[p] = rt;
        is_root[p] = r;
    }
}

// thread per point: cores read their root's rank; non-cores scan their (short) list
__global__ void __launch_bounds__(256) k_labels(const uint64_t* __restrict__ begin, const uint32_t* __restrict__ count,
                                                const uint32_t* __restrict__ nbrs, const uint32_t* __restrict__ rows,
                                                const uint8_t* __restrict__ core,
                                                const uint32_t* __restrict__ parent, const uint32_t* __restrict__ rank,
                                                uint64_t n, int32_t* __restrict__ labels) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t p = rows ? rows[i] : i;
        int32_t lab = -1;
        if (core[p]) {
            lab = (int32_t)rank[parent[p]];
        } else {
            const uint32_t* L = nbrs + begin[p];
            const uint32_t m = count[p];
            for (uint32_t j = 0; j < m; ++j) {
                const uint32_t v = L[j];
                if (core[v]) {
                    const int32_t c = (int32_t)rank[parent[v]];
                    if (lab < 0 || c < lab) lab = c;
                }
            }
        }
        labels[p] = lab;
    }
}

// Position space: roots are positions whose id is their
// component's minimum core id; the root flags and the labels / core flags go out by id.
__global__ void __launch_bounds__(256) k_flatten_pos(const uint8_t* __restrict__ core, uint64_t n,
                                                     const uint32_t* __restrict__ parent, const uint32_t* __restrict__ key,
                                                     uint32_t* __restrict__ root, uint32_t* __restrict__ is_root_id) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        uint32_t rt = (uint32_t)p;
        if (core[p]) {
            rt = find_fast(parent, (uint32_t)p);
            if (rt == (uint32_t)p) is_root_id[key[p]] = 1u;   // (is_root_id zeroed before)
        }
        root[p] = rt;
    }
}
__global__ void __launch_bounds__(256) k_labels_pos(const uint64_t* __restrict__ begin,
                                                    const uint32_t* __restrict__ count,
                                                    const uint32_t* __restrict__ nbrs, const uint8_t* __restrict__ core,
                                                    const uint32_t* __restrict__ root, const uint32_t* __restrict__ rank,
                                                    const uint32_t* __restrict__ key, uint64_t n,
                                                    int32_t* __restrict__ labels, uint8_t* __restrict__ core_out) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        int32_t lab = -1;
        const bool c = core[p];
        if (c) {
            lab = (int32_t)rank[key[root[p]]];
        } else {
            const uint32_t* L = nbrs + begin[p];
            const uint32_t m = count[p];
            for (uint32_t j = 0; j < m; ++j) {
                const uint32_t v = L[j];
                if (core[v]) {
                    const int32_t cl = (int32_t)rank[key[root[v]]];
                    if (lab < 0 || cl < lab) lab = cl;
                }
            }
        }
        const uint32_t id = key[p];
        labels[id] = lab;
        if (core_out) core_out[id] = c ? 1 : 0;
    }
}

inline unsigned blocks_for(uint64_t n, unsigned cap = 148u * 16u) {
    uint64_t b = (n + 255) / 256;
    return (unsigned)(b < 1 ? 1 : (b < cap ? b : cap));
}

}  // namespace

void launch_dbscan_device(const uint64_t* begin, const uint32_t* count, const uint32_t* nbrs, const uint32_t* rows,
                          uint64_t n, uint64_t npairs, uint32_t minpts, uint8_t* core, uint32_t* parent, uint32_t* root,
                          uint32_t* is_root, uint32_t* rank, uint32_t* giant, uint32_t* bits, uint32_t* sched,
                          uint64_t* pre, void* scan_temp, int32_t* labels, cudaStream_t s, bool pos_space,
                          uint8_t* core_out) {
    if (n == 0) return;
    // position space: every per-point pass walks positions (the production order itself), roots
    // are hooked by id (key = rows: position -> id)
    const uint32_t* key = pos_space ? rows : nullptr;
    if (pos_space) rows = nullptr;
    k_core_init<<<blocks_for(n), 256, 0, s>>>(count, n, minpts, core, parent);
    const uint32_t* walk = 16.0 * (double)n > kIdOrderBytes ? nullptr : rows;   // null: index order
    for (uint32_t k = 1; k <= kSampleLinks; ++k) {
        k_sample_link<<<blocks_for(n), 256, 0, s>>>(begin, count, nbrs, walk, n, k, parent, key);
        k_compress<<<blocks_for(n), 256, 0, s>>>(n, parent);
    }
    k_giant<<<1, kGiantSamples, 0, s>>>(rows, n, parent, giant);
    k_giant_bits<<<blocks_for(n), 256, 0, s>>>(n, parent, giant, bits, bits + (n + 31) / 32);
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaFuncSetAttribute(k_union, cudaFuncAttributePreferredSharedMemoryCarveout, 0);   // all of it as L1
        if (sms <= 0) sms = 148;
    }
    // pair-balanced regions: prefix of the list lengths along the walk order
    k_row_counts<<<blocks_for(n), 256, 0, s>>>(count, rows, n, (uint32_t*)root);   // root[] is free until k_flatten
    scan_u32_to_u64((const uint32_t*)root, pre, n, scan_temp, s);
    k_sched_init<<<1, 256, 0, s>>>(pre, (uint32_t)n, npairs, (uint32_t)sms, sched);
    const uint32_t grab = (double)npairs >= kLongListPairs * (double)n ? kGrabLong : kGrabShort;
    k_union<<<sms, kUnionThreads, 0, s>>>(begin, count, nbrs, rows, parent, giant, bits, bits + (n + 31) / 32, sched,
                                          grab, key);
    if (pos_space) {
        cudaMemsetAsync(is_root, 0, 4 * n, s);
        k_flatten_pos<<<blocks_for(n), 256, 0, s>>>(core, n, parent, key, root, is_root);
        scan_u32_to_u32(is_root, rank, n, scan_temp, s);
        k_labels_pos<<<blocks_for(n), 256, 0, s>>>(begin, count, nbrs, core, root, rank, key, n, labels, core_out);
    } else {
        k_flatten<<<blocks_for(n), 256, 0, s>>>(core, n, parent, root, is_root);
        scan_u32_to_u32(is_root, rank, n, scan_temp, s);
        k_labels<<<blocks_for(n), 256, 0, s>>>(begin, count, nbrs, walk, core, root, rank, n, labels);
    }
    g_kernel_launches += 8 + 2 * kSampleLinks;
}

}  // namespace hdb
