// kernels_dbscan.cu -- DBSCAN on a DEVICE-resident neighbour table (NEXT-4,
// SURVEY 8(f)): the paper's modified DBSCAN (Alg. 1 with lookups in T,
// P:651-655) without moving T over PCIe, which the paper names as its
// bottleneck.  Same canonical labelling as the host code
// (R7): core <=> |N_eps(p)| >= minpts; clusters = components of the
// core-core graph numbered by increasing minimum core id; a border point takes
// the lowest-numbered cluster among its core neighbours; noise = -1.
//
//   k_core_init   core flags, parent[p] = p
//   k_union       warp per core u: for every core neighbour v < u, union(u, v) by
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

__global__ void __launch_bounds__(256) k_core_init(const uint32_t* __restrict__ count, uint64_t n, uint32_t minpts,
                                                   uint8_t* __restrict__ core, uint32_t* __restrict__ parent) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
        core[p] = count[p] >= minpts ? 1 : 0;
        parent[p] = (uint32_t)p;
    }
}

// warp per core vertex u (grid-stride over ids); lanes stride over u's list
__global__ void __launch_bounds__(256) k_union(const uint64_t* __restrict__ begin, const uint32_t* __restrict__ count,
                                               const uint32_t* __restrict__ nbrs, const uint8_t* __restrict__ core,
                                               uint64_t n, uint32_t* __restrict__ parent) {
    const int lane = threadIdx.x & 31;
    const uint64_t wid = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    for (uint64_t u = wid; u < n; u += nw) {
        if (!core[u]) continue;   // uniform
        const uint32_t* L = nbrs + begin[u];
        const uint32_t m = count[u];
        uint32_t ru = find_fast(parent, (uint32_t)u);
        for (uint32_t j = lane; j < m; j += 32) {
            const uint32_t v = __ldg(&L[j]);
            if (v < u && core[v]) {
                const uint32_t rv = find_fast(parent, v);
                if (rv != ru) {
                    unite(parent, (uint32_t)u, v);
                    ru = find_fast(parent, (uint32_t)u);
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
                                                const uint32_t* __restrict__ nbrs, const uint8_t* __restrict__ core,
                                                const uint32_t* __restrict__ parent, const uint32_t* __restrict__ rank,
                                                uint64_t n, int32_t* __restrict__ labels) {
    for (uint64_t p = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; p < n; p += (uint64_t)gridDim.x * blockDim.x) {
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

void launch_dbscan_device(const uint64_t* begin, const uint32_t* count, const uint32_t* nbrs, uint64_t n,
                          uint32_t minpts, uint8_t* core, uint32_t* parent, uint32_t* root, uint32_t* is_root,
                          uint32_t* rank, void* scan_temp, int32_t* labels, cudaStream_t s) {
    if (n == 0) return;
    k_core_init<<<blocks_for(n), 256, 0, s>>>(count, n, minpts, core, parent);
    k_union<<<148 * 8, 256, 0, s>>>(begin, count, nbrs, core, n, parent);
    k_flatten<<<blocks_for(n), 256, 0, s>>>(core, n, parent, root, is_root);
    scan_u32_to_u32(is_root, rank, n, scan_temp, s);
    k_labels<<<blocks_for(n), 256, 0, s>>>(begin, count, nbrs, core, root, rank, n, labels);
    g_kernel_launches += 4;
}

}  // namespace hdb
