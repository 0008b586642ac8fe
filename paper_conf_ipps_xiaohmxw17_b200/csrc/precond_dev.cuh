// A3/A5/A7 device routines shared by the standalone preconditioner kernels and
// the persistent PCG kernel.
//
// Thread maps:
//  * "row warp": one warp per block row (spmv_row); lanes 0..5 end up owning
//    DOF a = lane of the row;
//  * "5-row warp": lanes 0..29 own DOF a = lane % 6 of block row 5*grp + lane/6
//    (30 consecutive doubles per warp access: coalesced); the 6 DOFs of a block
//    sit in one warp so D_i^{-1} r_i is done with shuffles.
#pragma once
#include "spmv_warp.cuh"

namespace dda {

struct XCg {   // coherent vector loads (the vector may have been written in this kernel)
    const double* __restrict__ x;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        return ld_cg2(x + 6 * (size_t)vec + 2 * pair);
    }
};

struct Row5 {
    int i;       // block row of this lane (may be >= n: invalid)
    int a;       // DOF within the row
    int base;    // first lane of this row's 6-lane group
    bool valid;
    size_t idx;  // 6*i + a
};

__device__ __forceinline__ Row5 row5(int grp, int lane, int n) {
    Row5 r;
    const int k = lane < 30 ? lane / 6 : 4;
    r.a = lane < 30 ? lane - 6 * k : 0;
    r.base = 6 * k;
    r.i = 5 * grp + k;
    r.valid = lane < 30 && r.i < n;
    r.idx = 6 * (size_t)(r.valid ? r.i : 0) + r.a;
    return r;
}

// Row a of the packed D_i^{-1} for the lane's DOF (6 values), loaded ahead of use
struct DinvRow {
    double v[6];
};
__device__ __forceinline__ DinvRow dinv_row(const double* __restrict__ dinv, const Row5& R) {
    const double* blk = dinv + (size_t)kDinv * (R.valid ? R.i : 0);
    DinvRow d;
#pragma unroll
    for (int c = 0; c < 6; ++c) {
        const int r0 = R.a < c ? R.a : c, c0 = R.a < c ? c : R.a;
        d.v[c] = __ldg(blk + pk_off(r0, c0));
    }
    return d;
}
// z_a = sum_c D[a][c] v_c with the preloaded row; every lane of the warp must call
__device__ __forceinline__ double dinv_row_apply(const DinvRow& d, double v, const Row5& R) {
    double z = 0.0;
#pragma unroll
    for (int c = 0; c < 6; ++c) z = fma(d.v[c], __shfl_sync(0xffffffffu, v, R.base + c), z);
    return z;
}

// z = D_i^{-1} v for the lane's DOF (packed inverse); all lanes must call
__device__ __forceinline__ double bj_lane(const double* __restrict__ dinv, const Row5& R, double v) {
    const double* blk = dinv + (size_t)kDinv * (R.valid ? R.i : 0);
    return dinv_apply6(blk, v, R.a, R.base);
}

// SSOR-AI lower half-pass epilogue (reading Z14, A7 steps 2-3) for the lane's
// group row i, given (y0, y1) = the SPMV_LOWER_T row product of t:
//   s_i = r_i - omega * sum_{k<i} V_ki^T t_k ;  w_i = D_i^{-1} s_i
__device__ __forceinline__ void ssor_lower_row(const double* __restrict__ dinv, int i, bool ok, double y0, double y1,
                                               const double* r, double omega, double* w, int lane) {
    const double lt = pairs_to_dof(y0, y1, lane);
    const int q = q_of(lane);
    const int a = q < 6 ? q : 0;
    const bool mine = ok && q < 6;
    const double s = mine ? ld_cg(r + 6 * (size_t)i + a) - omega * lt : 0.0;
    const double wv = dinv_apply6(dinv + (size_t)kDinv * (ok ? i : 0), s, a, 9 * grp_of(lane));
    if (mine) w[6 * (size_t)i + a] = wv;
}

// SSOR-AI upper half-pass epilogue (A7 step 4) for the lane's group row i, given
// (y0, y1) = the SPMV_UPPER row product of w:
//   z_i = w_i - omega * D_i^{-1} sum_{j>i} V_ij w_j   (valid on lanes q < 6 of groups with a row)
__device__ __forceinline__ double ssor_upper_row(const double* __restrict__ dinv, int i, bool ok, double y0,
                                                 double y1, const double* w, double omega, int lane) {
    const double uw = pairs_to_dof(y0, y1, lane);
    const int q = q_of(lane);
    const int a = q < 6 ? q : 0;
    const double du = dinv_apply6(dinv + (size_t)kDinv * (ok ? i : 0), uw, a, 9 * grp_of(lane));
    return (ok && q < 6) ? ld_cg(w + 6 * (size_t)i + a) - omega * du : 0.0;
}

}  // namespace dda
