// A4 — warp-cooperative symmetric BSR6 block-row product (§IV.B).
//
//   y_i = D_i x_i + sum_{j in R_i} V_ij x_j + sum_{k in L_i} V_ki^T x_k
//
// computed from the upper storage only ("need not recover the global stiffness
// matrix"), with no atomics and no intermediate up-res / low-res arrays
// (the paper's two-stage scheme, is prior art: on B200 its extra
// 96 B/block round trip costs more than re-reading the transposed block from L2).
//
// One warp owns one block row.  Lanes 0..26 form three 9-lane groups; lane
// (g, q = 3R + C) loads chunk q (a 2x2 sub-block, one 256-bit load) of block
// number b = g, g+3, g+6, ... of the row's list [D_i, V_i*, V_*i]; lanes 27..31
// idle.  A forward block adds its 2x2 chunk times x_j[2C..2C+1] to the row
// pair R; a transposed block adds chunk^T times x_k[2R..2R+1] to the row pair C.
// The 27 partial pairs are combined in a fixed order (transpose-shuffle, sum
// over groups, sum over C), so the result is bitwise deterministic.
#pragma once
#include "dda_internal.cuh"

namespace dda {

enum SpmvMode { SPMV_FULL = 0, SPMV_LOWER_T = 1, SPMV_UPPER = 2 };

struct BsrView {
    int32_t n;
    const int32_t* __restrict__ row_ptr;
    const int32_t* __restrict__ col_idx;
    const int32_t* __restrict__ low_ptr;
    const int32_t* __restrict__ low_row;
    const int32_t* __restrict__ low_to_up;
    const double* __restrict__ diag;
    const double* __restrict__ upper;
};

__host__ inline BsrView view_of(const dda_matrix* K) {
    return BsrView{K->n, K->row_ptr, K->col_idx, K->low_ptr, K->low_row, K->low_to_up, K->diag, K->upper};
}

// XLoad: functor  double2 operator()(int vec_block, int pair) -> x[6*vec + 2*pair .. +1]
// On return, lanes 0, 3, 6 (pair R = lane/3) hold (y[2R], y[2R+1]) in (y0, y1).
template <int MODE, class XLoad>
__device__ __forceinline__ void spmv_row(const BsrView& A, int i, const XLoad& xload, int lane,
                                         double& y0, double& y1) {
    const int g = lane / 9;
    const int q = lane - 9 * g;
    const int R = q / 3;
    const int C = q - 3 * R;
    int up0 = 0, nu = 0, lo0 = 0, nl = 0;
    if (MODE != SPMV_LOWER_T) { up0 = __ldg(A.row_ptr + i); nu = __ldg(A.row_ptr + i + 1) - up0; }
    if (MODE != SPMV_UPPER)   { lo0 = __ldg(A.low_ptr + i); nl = __ldg(A.low_ptr + i + 1) - lo0; }
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const int nb = (lane < 27) ? nd + nu + nl : 0;
    double f0 = 0.0, f1 = 0.0, t0 = 0.0, t1 = 0.0;
    for (int b = g; b < nb; b += 3) {
        const double* blk;
        int vec;
        bool trans;
        if (nd && b < nd) {
            blk = A.diag + (size_t)kBlk * i; vec = i; trans = false;
        } else if (b < nd + nu) {
            const int u = up0 + b - nd;
            blk = A.upper + (size_t)kBlk * u; vec = __ldg(A.col_idx + u); trans = false;
        } else {
            const int t = lo0 + b - nd - nu;
            blk = A.upper + (size_t)kBlk * __ldg(A.low_to_up + t); vec = __ldg(A.low_row + t); trans = true;
        }
        const double4 a = ld_chunk(blk + 4 * q);
        const double2 xv = xload(vec, trans ? R : C);
        if (!trans) {
            f0 = fma(a.x, xv.x, fma(a.y, xv.y, f0));
            f1 = fma(a.z, xv.x, fma(a.w, xv.y, f1));
        } else {
            t0 = fma(a.x, xv.x, fma(a.z, xv.y, t0));
            t1 = fma(a.y, xv.x, fma(a.w, xv.y, t1));
        }
    }
    const unsigned full = 0xffffffffu;
    // (1) transposed partials of lane (g,C,R) target pair R of lane (g,R,C)
    const int src = (lane < 27) ? 9 * g + 3 * C + R : lane;
    double v0 = f0 + __shfl_sync(full, t0, src);
    double v1 = f1 + __shfl_sync(full, t1, src);
    // (2) sum over the three groups, into lanes 0..8
    const int s1 = (lane + 9) & 31, s2 = (lane + 18) & 31;
    const double a0 = __shfl_sync(full, v0, s1), a1 = __shfl_sync(full, v1, s1);
    const double b0 = __shfl_sync(full, v0, s2), b1 = __shfl_sync(full, v1, s2);
    v0 = (v0 + a0) + b0;
    v1 = (v1 + a1) + b1;
    // (3) sum over C, into lanes 0, 3, 6
    const int c1 = (lane + 1) & 31, c2 = (lane + 2) & 31;
    const double d0 = __shfl_sync(full, v0, c1), d1 = __shfl_sync(full, v1, c1);
    const double e0 = __shfl_sync(full, v0, c2), e1 = __shfl_sync(full, v1, c2);
    y0 = (v0 + d0) + e0;
    y1 = (v1 + d1) + e1;
}

// Move the row result from lanes 0/3/6 (pairs) to lanes 0..5 (one DOF each).
__device__ __forceinline__ double pairs_to_dof(double y0, double y1, int lane) {
    const int a = lane < 6 ? lane : 0;
    const double lo = __shfl_sync(0xffffffffu, y0, 3 * (a >> 1));
    const double hi = __shfl_sync(0xffffffffu, y1, 3 * (a >> 1));
    return (a & 1) ? hi : lo;
}

// z_a = sum_c Dinv[a][c] v_c for the 6 DOFs held by lanes base..base+5 (packed
// upper-triangle Dinv of that block); every lane of the warp must call it.
__device__ __forceinline__ double dinv_apply6(const double* __restrict__ dinv_blk, double v, int a, int base) {
    double z = 0.0;
#pragma unroll
    for (int c = 0; c < 6; ++c) {
        const double vc = __shfl_sync(0xffffffffu, v, base + c);
        const int r0 = a < c ? a : c, c0 = a < c ? c : a;
        z = fma(__ldg(dinv_blk + pk_off(r0, c0)), vc, z);
    }
    return z;
}

}  // namespace dda
