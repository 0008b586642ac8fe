// A4 — warp-cooperative symmetric BSR6 block-row product (§IV.B).
//
//   y_i = D_i x_i + sum_{j in R_i} V_ij x_j + sum_{k in L_i} V_ki^T x_k
//
// computed from the upper storage only ("need not recover the global stiffness
// matrix"), with no atomics and no intermediate up-res / low-res arrays
// (the paper's two-stage scheme, is prior art: on B200 its extra
// 96 B/block round trip costs more than re-reading the transposed block from L2).
//
// Thread map: a warp is three 9-lane groups; group g owns block
// row i = 3*step + g.  Lane q = 3R + C of the group loads ONE 256-bit chunk of
// the row's b-th block per round (the whole 288 B block in one warp instruction,
// i.e. the minimum number of L1 wavefronts), and always accumulates into the row
// pair R with x_vec[2C..2C+1]:
//   forward block  (D_i, V_ij):  chunk (R, C)            -> += chunk   * x_j
//   transposed     (V_ki^T)   :  chunk (C, R), used ^T   -> += chunk^T * x_k
// so the only cross-lane step per row is the sum over C (2 shuffles of a pair,
// shared by the three rows of the warp).  The group's block list (block index,
// vector index, transposed flag) is fetched with one coalesced load per 9
// entries and broadcast by shuffles, so each round's chunk and x loads depend
// on nothing but registers.  Fixed summation order: bitwise deterministic.
#pragma once
#include "dda_internal.cuh"

namespace dda {

// SPMV_OFFDIAG: both triangles without the diagonal block (the scaled BJ engine, whose
// diagonal blocks are the identity and are applied by the caller)
enum SpmvMode { SPMV_FULL = 0, SPMV_LOWER_T = 1, SPMV_UPPER = 2, SPMV_OFFDIAG = 3 };

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

struct RowBounds {
    int up0, nu, lo0, nl;
};

template <int MODE>
__device__ __forceinline__ RowBounds row_bounds(const BsrView& A, int i, bool ok) {
    RowBounds b{0, 0, 0, 0};
    if (ok && i < A.n) {
        if (MODE != SPMV_LOWER_T) {
            b.up0 = __ldg(A.row_ptr + i);
            b.nu = __ldg(A.row_ptr + i + 1) - b.up0;
        }
        if (MODE != SPMV_UPPER) {
            b.lo0 = __ldg(A.low_ptr + i);
            b.nl = __ldg(A.low_ptr + i + 1) - b.lo0;
        }
    }
    return b;
}

// lane roles
__device__ __forceinline__ int grp_of(int lane) { return lane < 27 ? lane / 9 : 2; }
__device__ __forceinline__ int q_of(int lane) { return lane < 27 ? lane - 9 * (lane / 9) : 8; }
// lanes that hold a row result pair after spmv: q in {0,3,6} of groups 0..2
__device__ __forceinline__ bool is_out_lane(int lane) { return lane < 27 && (q_of(lane) % 3) == 0; }

// XLoad: functor  double2 operator()(int vec_block, int pair) -> x[6*vec + 2*pair .. +1]
// Computes the product for row i (this lane's group row; `ok` false for no row).
// On return, lanes q = 3R of the group hold (y[2R], y[2R+1]) in (y0, y1).
template <int MODE, class XLoad>
__device__ __forceinline__ void spmv_row_g(const BsrView& A, int i, bool ok, const RowBounds& rb,
                                           const XLoad& xload, int lane, double& y0, double& y1) {
    const unsigned full = 0xffffffffu;
    const int g = grp_of(lane);
    const int q = q_of(lane);
    const int R = q / 3;
    const int C = q - 3 * R;
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const int nb = (ok && lane < 27) ? nd + rb.nu + rb.nl : 0;
    int nbmax = __reduce_max_sync(full, nb);
    double f0 = 0.0, f1 = 0.0;
    for (int e0 = 0; e0 < nbmax; e0 += 9) {
        // this lane fetches entry e0+q of its group's list
        int ent_blk = 0, ent_vec = 0;   // ent_blk: upper index, or -(i+1) for the diagonal; ent_vec < 0: transposed
        {
            const int e = e0 + q;
            if (e < nb) {
                if (nd && e < nd) {
                    ent_blk = -(i + 1);
                    ent_vec = i;
                } else if (e < nd + rb.nu) {
                    const int u = rb.up0 + e - nd;
                    ent_blk = u;
                    ent_vec = __ldg(A.col_idx + u);
                } else {
                    const int t = rb.lo0 + e - nd - rb.nu;
                    ent_blk = __ldg(A.low_to_up + t);
                    ent_vec = ~__ldg(A.low_row + t);
                }
            }
        }
        const int rounds = min(9, nbmax - e0);
#pragma unroll 3
        for (int b = 0; b < rounds; ++b) {
            const int src = 9 * g + b;
            const int blk = __shfl_sync(full, ent_blk, src);
            const int vec = __shfl_sync(full, ent_vec, src);
            if (e0 + b < nb) {
                const bool tr = vec < 0;
                const int v = tr ? ~vec : vec;
                const double* bp = (blk < 0) ? A.diag + (size_t)kBlk * (-blk - 1) : A.upper + (size_t)kBlk * blk;
                const double4 a = ld_chunk(bp + 4 * (tr ? 3 * C + R : q));
                const double2 xv = xload(v, C);
                const double m01 = tr ? a.z : a.y;
                const double m10 = tr ? a.y : a.z;
                f0 = fma(a.x, xv.x, fma(m01, xv.y, f0));
                f1 = fma(m10, xv.x, fma(a.w, xv.y, f1));
            }
        }
    }
    // sum over C within the group, into lanes q = 3R
    const int c1 = (lane + 1) & 31, c2 = (lane + 2) & 31;
    const double d0 = __shfl_sync(full, f0, c1), d1 = __shfl_sync(full, f1, c1);
    const double e0_ = __shfl_sync(full, f0, c2), e1 = __shfl_sync(full, f1, c2);
    y0 = (f0 + d0) + e0_;
    y1 = (f1 + d1) + e1;
}

// Row loop: warp w takes rows 3w..3w+2, then 3(w+W).., the whole grid sweeping
// the rows in increasing order; the bounds of the next rows are prefetched.
// body(i, ok, y0, y1) is called by every lane (ok: the lane's group has a row).
template <int MODE, class XLoad, class Body>
__device__ __forceinline__ void for_rows(const BsrView& A, int w, int W, const XLoad& xload, int lane,
                                         const Body& body) {
    const int g = grp_of(lane);
    const bool lane_ok = lane < 27;
    int i = 3 * w + g;
    RowBounds nxt = row_bounds<MODE>(A, i, lane_ok);
    for (int base = 3 * w; base < A.n; base += 3 * W) {
        i = base + g;
        const bool ok = lane_ok && i < A.n;
        const RowBounds cur = nxt;
        nxt = row_bounds<MODE>(A, i + 3 * W, lane_ok);
        double y0, y1;
        spmv_row_g<MODE>(A, i, ok, cur, xload, lane, y0, y1);
        body(i, ok, y0, y1);
    }
}

// Move a group's row result from lanes q = 0/3/6 (pairs) to lanes q = 0..5 (one DOF each).
__device__ __forceinline__ double pairs_to_dof(double y0, double y1, int lane) {
    const int g = grp_of(lane);
    const int q = q_of(lane);
    const int a = q < 6 ? q : 0;
    const int src = 9 * g + 3 * (a >> 1);
    const double lo = __shfl_sync(0xffffffffu, y0, src);
    const double hi = __shfl_sync(0xffffffffu, y1, src);
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
