// cellkey.cuh -- the cell of a point (reading R9): shared by the
// grid build's sort (kernels_grid.cu) and the process-shard band selection
// (kernels_scan.cu), so that both put every point in the same cell.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace hdb {

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

struct KeyParams {
    double xmin, ymin, inv_w;
    uint32_t nx, ny;
};

// cx = floor(fl(fl(x - xmin) * fl(1/w))) clamped to [0, nx-1], FP64 with explicitly
// rounded ops (no FMA); the same for cy.  w = eps_F (1 + 2^-19) / k (reading R9).
template <typename T>
__device__ __forceinline__ void cell_xy(const typename V2<T>::type p, const KeyParams& kp, uint64_t& cx,
                                        uint64_t& cy) {
    const double tx = floor(__dmul_rn(__dsub_rn((double)p.x, kp.xmin), kp.inv_w));
    const double ty = floor(__dmul_rn(__dsub_rn((double)p.y, kp.ymin), kp.inv_w));
    cx = (uint64_t)fmin(fmax(tx, 0.0), (double)(kp.nx - 1));
    cy = (uint64_t)fmin(fmax(ty, 0.0), (double)(kp.ny - 1));
}

// row-major cell key h = cy * nx + cx
template <typename T, typename K>
__device__ __forceinline__ K cell_key(const typename V2<T>::type p, const KeyParams& kp) {
    uint64_t cx, cy;
    cell_xy<T>(p, kp, cx, cy);
    return (K)(cy * kp.nx + cx);
}

}  // namespace hdb
