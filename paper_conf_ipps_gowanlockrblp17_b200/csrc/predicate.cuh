// predicate.cuh -- the neighbour predicate O1 (R1/R2):
// q in N_eps(p) <=> fl(fl(dx*dx) + fl(dy*dy)) <= fl(eps*eps), dx = fl(x_p - x_q),
// dy = fl(y_p - y_q), round-to-nearest-even in the input precision, no FMA
// (explicit _rn intrinsics cannot be contracted).  Dist <= eps is P:147-148.
#pragma once

namespace hdb {

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

}  // namespace hdb
