// kernels_dbscan.cu -- DBSCAN on a DEVICE-resident neighbour table (NEXT-4,
// SURVEY 8(f)): the paper's modified DBSCAN (Alg. 1 with lookups in T,
// P:651-655) without moving T over PCIe, which the paper names as its
// bottleneck.  Same canonical labelling as the host code
// (R7): core <=> |N_eps(p)| >= minpts; clusters = components of the
// core-core graph numbered by increasing minimum core id; a border point takes
// the lowest-numbered cluster among its core neighbours; noise = -1.
//
//   k_core_init   core flags, parent[p] = p
//   k_union       warp per core u (rows taken in the table's cell-sorted production
//                 order): for every core neighbour v < u, union(u, v) by
//                 hooking the larger root under the smaller (atomicCAS), so every
//                 root stays the minimum id of its tree (ECL-CC style, path halving)
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

__device__ __forceinline__ void unite(uint32_t* __restrict__ parent, uint32_t a, uint32_t b) {
    while (true) {
        a = find_root(parent, a);
        b = find_root(parent, b);
        if (a == b) return;
        if (a < b) {
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

constexpr uint32_t kRowsPerGrab = 4;      // consecutive (cell-sorted) rows per warp grab
constexpr int kUnionThreads = 1024;       // one CTA per SM

// first row r in [0, n) with begin[rows[r]] >= x (begin is non-decreasing
// along the production order of a whole table)
__device__ uint32_t row_of_pair(const uint64_t* __restrict__ begin, const uint32_t* __restrict__ rows, uint32_t n,
                                uint64_t x) {
    uint32_t lo = 0, hi = n;
    while (lo < hi) {
        const uint32_t mid = lo + (hi - lo) / 2;
        if (begin[rows[mid]] < x) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// One CTA per SM owns a contiguous range of the production (cell-sorted) order
// holding ~1/G of the pairs; its warps take kRowsPerGrab consecutive rows at a
// time from a shared counter.  All warps of an SM therefore work in one small
// region of space at any moment and their random parent[v] reads share L1.
// For core u, lanes stride over u's list (4 independent edges per lane per
// pass); every core neighbour v < u whose root differs is united with u.
__global__ void __launch_bounds__(kUnionThreads, 1)
    k_union(const uint64_t* __restrict__ begin, const uint32_t* __restrict__ count, const uint32_t* __restrict__ nbrs,
            const uint32_t* __restrict__ rows, uint32_t n, uint64_t npairs, uint32_t* __restrict__ parent) {
    __shared__ uint32_t s_next, s_end;
    const int lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        const uint64_t G = gridDim.x, c = blockIdx.x;
        if (rows) {
            s_next = row_of_pair(begin, rows, n, npairs * c / G);
            s_end = c + 1 == G ? n : row_of_pair(begin, rows, n, npairs * (c + 1) / G);
        } else {
            s_next = (uint32_t)((uint64_t)n * c / G);
            s_end = (uint32_t)((uint64_t)n * (c + 1) / G);
        }
    }
    __syncthreads();
    const uint32_t end = s_end;
    while (true) {
        uint32_t r0 = 0;
        if (lane == 0) r0 = atomicAdd(&s_next, kRowsPerGrab);
        r0 = __shfl_sync(FULL, r0, 0);
        if (r0 >= end) return;
        const uint32_t r1 = min(end, r0 + kRowsPerGrab);
        for (uint32_t r = r0; r < r1; ++r) {
            const uint32_t u = rows ? __ldg(&rows[r]) : r;
            if (__ldca(&parent[u]) == kNonCore) continue;   // uniform: non-core rows add no edge
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
                for (int k = 0; k < 4; ++k) p[k] = v[k] < u ? __ldca(&parent[v[k]]) : kNonCore;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    // skip non-cores and v hanging directly under u's root; else follow the chain
                    if (p[k] != kNonCore && p[k] != ru && !(p[k] != v[k] && reaches(parent, p[k], ru))) {
                        unite(parent, u, v[k]);
                        ru = find_fast(parent, u);
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

inline unsigned blocks_for(uint64_t n, unsigned cap = 148u * 16u) {
    uint64_t b = (n + 255) / 256;
    return (unsigned)(b < 1 ? 1 : (b < cap ? b : cap));
}

}  // namespace

void launch_dbscan_device(const uint64_t* begin, const uint32_t* count, const uint32_t* nbrs, const uint32_t* rows,
                          uint64_t n, uint64_t npairs, uint32_t minpts, uint8_t* core, uint32_t* parent, uint32_t* root,
                          uint32_t* is_root, uint32_t* rank, void* scan_temp, int32_t* labels, cudaStream_t s) {
    if (n == 0) return;
    k_core_init<<<blocks_for(n), 256, 0, s>>>(count, n, minpts, core, parent);
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaFuncSetAttribute(k_union, cudaFuncAttributePreferredSharedMemoryCarveout, 0);   // all of it as L1
        if (sms <= 0) sms = 148;
    }
    k_union<<<sms, kUnionThreads, 0, s>>>(begin, count, nbrs, rows, (uint32_t)n, npairs, parent);
    k_flatten<<<blocks_for(n), 256, 0, s>>>(core, n, parent, root, is_root);
    scan_u32_to_u32(is_root, rank, n, scan_temp, s);
    k_labels<<<blocks_for(n), 256, 0, s>>>(begin, count, nbrs, rows, core, root, rank, n, labels);
    g_kernel_launches += 4;
}

}  // namespace hdb
