// A4 — symmetric BSR6 block-row product, "column-pair" thread map (v3).
//
// Same product as spmv_warp.cuh (§IV.B):
//   y_i = D_i x_i + sum_{j in R_i} V_ij x_j + sum_{k in L_i} V_ki^T x_k
//
// Why a second map: the symmetric SpMV is bound by the L1 data pipe (register
// write-back of loaded bytes), not by HBM — ncu: ~58 LSU wavefronts per block row
// with the 9-lanes-per-block map, where each x pair is delivered to 3 lanes and
// the row bounds to all 27.  Here every loaded byte lands in exactly one lane:
//
//   a warp = 10 groups of 3 lanes; group h owns block row i = 10*step + h;
//   lane C (0..2) of the group owns COLUMN pair C of every block of the row:
//     forward block  (D_i, V_ij): chunks (0,C),(1,C),(2,C)  x_j[2C..2C+1]
//     transposed     (V_ki^T)   : chunks (C,0),(C,1),(C,2)  x_k[2C..2C+1]
//   (three 256-bit chunk loads + one 128-bit x load per lane per block), and
//   accumulates all six row partials; one 3-lane reduce-scatter per row leaves
//   y[2C..2C+1] in lane C.  Fixed summation order: bitwise deterministic.
//   (Fetching the row's block list up front and broadcasting it spills at 48
//   registers and measured slower: 0.296 vs 0.269 ms at 1M blocks.)
#pragma once
#include "spmv_warp.cuh"

namespace dda {

__device__ __forceinline__ int cgrp_of(int lane) { return lane < 30 ? lane / 3 : 9; }
__device__ __forceinline__ int ccol_of(int lane) { return lane < 30 ? lane - 3 * (lane / 3) : 2; }

// pair p of the 6 accumulators (p in 0..2, runtime) without dynamic register indexing
__device__ __forceinline__ double2 pick_pair(const double (&a)[6], int p) {
    return make_double2(p == 0 ? a[0] : (p == 1 ? a[2] : a[4]), p == 0 ? a[1] : (p == 1 ? a[3] : a[5]));
}

template <int MODE, class XLoad>
__device__ __forceinline__ void spmv_row_c(const BsrView& A, int i, bool ok, const RowBounds& rb,
                                           const XLoad& xload, int lane, double& y0, double& y1) {
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane);
    const int C = ccol_of(lane);
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const int nb = (ok && lane < 30) ? nd + rb.nu + rb.nl : 0;
    const int nbmax = __reduce_max_sync(full, nb);
    double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
#pragma unroll 2
    for (int b = 0; b < nbmax; ++b) {
        if (b < nb) {
            const double* blk;
            int vec;
            bool tr = false;
            if (nd && b < nd) {
                blk = A.diag + (size_t)kBlk * i;
                vec = i;
            } else if (b < nd + rb.nu) {
                const int u = rb.up0 + b - nd;
                blk = A.upper + (size_t)kBlk * u;
                vec = __ldg(A.col_idx + u);
            } else {
                const int t = rb.lo0 + b - nd - rb.nu;
                blk = A.upper + (size_t)kBlk * __ldg(A.low_to_up + t);
                vec = __ldg(A.low_row + t);
                tr = true;
            }
            const double2 xv = xload(vec, C);
#pragma unroll
            for (int k = 0; k < 3; ++k) {
                const double4 c = ld_chunk(blk + 4 * (tr ? 3 * C + k : 3 * k + C));
                const double m01 = tr ? c.z : c.y;
                const double m10 = tr ? c.y : c.z;
                acc[2 * k] = fma(c.x, xv.x, fma(m01, xv.y, acc[2 * k]));
                acc[2 * k + 1] = fma(m10, xv.x, fma(c.w, xv.y, acc[2 * k + 1]));
            }
        }
    }
    // 3-lane reduce-scatter: lane C collects pair C from lanes C+1 and C+2 (mod 3).  In step 1 a
    // lane is read by lane C-1, so it exports its pair C-1; in step 2 it is read by lane C+1.
    const int c1 = C == 2 ? 0 : C + 1, c2 = C == 0 ? 2 : C - 1;
    const int s1 = lane < 30 ? 3 * h + c1 : lane, s2 = lane < 30 ? 3 * h + c2 : lane;
    const double2 v1 = pick_pair(acc, c2);
    const double r1x = __shfl_sync(full, v1.x, s1), r1y = __shfl_sync(full, v1.y, s1);
    const double2 v2 = pick_pair(acc, c1);
    const double r2x = __shfl_sync(full, v2.x, s2), r2y = __shfl_sync(full, v2.y, s2);
    const double2 own = pick_pair(acc, C);
    y0 = (own.x + r1x) + r2x;
    y1 = (own.y + r1y) + r2y;
}

// v4: the same map and the same per-lane summation order, with the block list decoded one block
// AHEAD: the index loads of block b+1 (col_idx / low_to_up / low_row) are in flight while block
// b's chunks and x are loaded and consumed, so each block costs one memory round trip instead of
// two (ncu on v3: the consumer of the col_idx load was the top stall).  Lanes past the end of
// their row's list issue no chunk loads (predicated off: zeros) and add exact zeros.
struct CEnt {
    int blk;   // upper block index, or ~row for a diagonal block
    int vec;   // block row of x, or ~row when the block is used transposed
};

template <int MODE>
__device__ __forceinline__ CEnt cent_decode(const BsrView& A, int i, const RowBounds& rb, int b, int nb) {
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const bool valid = b < nb;
    const int k = b - nd;
    const bool isd = valid && nd && k < 0;
    const bool isu = valid && !isd && k < rb.nu;
    const bool isl = valid && !isd && !isu;
    const int u = rb.up0 + k;
    const int t = rb.lo0 + k - rb.nu;
    const int vu = isu ? __ldg(A.col_idx + u) : 0;
    const int bl = isl ? __ldg(A.low_to_up + t) : 0;
    const int vl = isl ? __ldg(A.low_row + t) : 0;
    CEnt e;
    e.blk = isu ? u : (isl ? bl : ~(isd ? i : 0));
    e.vec = isu ? vu : (isl ? ~vl : (isd ? i : 0));
    return e;
}

template <int MODE, class XLoad>
__device__ __forceinline__ void spmv_row_c4(const BsrView& A, int i, bool ok, const RowBounds& rb,
                                            const XLoad& xload, int lane, double& y0, double& y1) {
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane);
    const int C = ccol_of(lane);
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const int nb = (ok && lane < 30) ? nd + rb.nu + rb.nl : 0;
    const int nbmax = __reduce_max_sync(full, nb);
    double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    CEnt nx = cent_decode<MODE>(A, i, rb, 0, nb);
    for (int b = 0; b < nbmax; ++b) {
        const CEnt e = nx;
        const bool valid = b < nb;
        const bool tr = e.vec < 0;
        const double* blk = e.blk >= 0 ? A.upper + (size_t)kBlk * e.blk : A.diag + (size_t)kBlk * ~e.blk;
        const double2 xv = xload(tr ? ~e.vec : e.vec, C);
        const int q0 = tr ? 3 * C : C, qs = tr ? 1 : 3;
        const double4 c0 = ld_chunk_if(blk + 4 * q0, valid);
        const double4 c1 = ld_chunk_if(blk + 4 * (q0 + qs), valid);
        const double4 c2 = ld_chunk_if(blk + 4 * (q0 + 2 * qs), valid);
        nx = cent_decode<MODE>(A, i, rb, b + 1, nb);
        const double4 cs[3] = {c0, c1, c2};
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const double4 c = cs[k];
            const double m01 = tr ? c.z : c.y;
            const double m10 = tr ? c.y : c.z;
            acc[2 * k] = fma(c.x, xv.x, fma(m01, xv.y, acc[2 * k]));
            acc[2 * k + 1] = fma(m10, xv.x, fma(c.w, xv.y, acc[2 * k + 1]));
        }
    }
    const int c1 = C == 2 ? 0 : C + 1, c2 = C == 0 ? 2 : C - 1;
    const int s1 = lane < 30 ? 3 * h + c1 : lane, s2 = lane < 30 ? 3 * h + c2 : lane;
    const double2 v1 = pick_pair(acc, c2);
    const double r1x = __shfl_sync(full, v1.x, s1), r1y = __shfl_sync(full, v1.y, s1);
    const double2 v2 = pick_pair(acc, c1);
    const double r2x = __shfl_sync(full, v2.x, s2), r2y = __shfl_sync(full, v2.y, s2);
    const double2 own = pick_pair(acc, C);
    y0 = (own.x + r1x) + r2x;
    y1 = (own.y + r1y) + r2y;
}

// v5: v4 plus data double-buffering: block b+1's chunks and x are loaded before block b is
// consumed (two blocks in flight per lane; ~80 registers).  XLoad::raw loads the x operand and
// XLoad::cook finishes it when the block is consumed (the functor decides how much work is
// deferred; see XFusedG in pcg_graph.cu).
template <class XLoad>
struct CData {
    double4 c0, c1, c2;
    typename XLoad::Raw x;
    bool tr;
};

template <int MODE, class XLoad>
__device__ __forceinline__ CData<XLoad> cdata_load(const BsrView& A, const CEnt& e, bool valid, const XLoad& xload,
                                                   int C) {
    CData<XLoad> d;
    d.tr = e.vec < 0;
    const double* blk = e.blk >= 0 ? A.upper + (size_t)kBlk * e.blk : A.diag + (size_t)kBlk * ~e.blk;
    d.x = xload.raw(d.tr ? ~e.vec : e.vec, C);
    const int q0 = d.tr ? 3 * C : C, qs = d.tr ? 1 : 3;
    d.c0 = ld_chunk_if(blk + 4 * q0, valid);
    d.c1 = ld_chunk_if(blk + 4 * (q0 + qs), valid);
    d.c2 = ld_chunk_if(blk + 4 * (q0 + 2 * qs), valid);
    return d;
}

template <int MODE, class XLoad>
__device__ __forceinline__ void spmv_row_c5(const BsrView& A, int i, bool ok, const RowBounds& rb,
                                            const XLoad& xload, int lane, double& y0, double& y1) {
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane);
    const int C = ccol_of(lane);
    constexpr int nd = (MODE == SPMV_FULL) ? 1 : 0;
    const int nb = (ok && lane < 30) ? nd + rb.nu + rb.nl : 0;
    const int nbmax = __reduce_max_sync(full, nb);
    double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    CEnt e1 = cent_decode<MODE>(A, i, rb, 0, nb);
    CData<XLoad> d0 = cdata_load<MODE>(A, e1, 0 < nb, xload, C);
    e1 = cent_decode<MODE>(A, i, rb, 1, nb);
    for (int b = 0; b < nbmax; ++b) {
        const CEnt e2 = cent_decode<MODE>(A, i, rb, b + 2, nb);
        const CData<XLoad> d1 = cdata_load<MODE>(A, e1, b + 1 < nb, xload, C);
        const double4 cs[3] = {d0.c0, d0.c1, d0.c2};
        const double2 xv = xload.cook(d0.x);
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const double4 c = cs[k];
            const double m01 = d0.tr ? c.z : c.y;
            const double m10 = d0.tr ? c.y : c.z;
            acc[2 * k] = fma(c.x, xv.x, fma(m01, xv.y, acc[2 * k]));
            acc[2 * k + 1] = fma(m10, xv.x, fma(c.w, xv.y, acc[2 * k + 1]));
        }
        d0 = d1;
        e1 = e2;
    }
    const int c1 = C == 2 ? 0 : C + 1, c2 = C == 0 ? 2 : C - 1;
    const int s1 = lane < 30 ? 3 * h + c1 : lane, s2 = lane < 30 ? 3 * h + c2 : lane;
    const double2 v1 = pick_pair(acc, c2);
    const double r1x = __shfl_sync(full, v1.x, s1), r1y = __shfl_sync(full, v1.y, s1);
    const double2 v2 = pick_pair(acc, c1);
    const double r2x = __shfl_sync(full, v2.x, s2), r2y = __shfl_sync(full, v2.y, s2);
    const double2 own = pick_pair(acc, C);
    y0 = (own.x + r1x) + r2x;
    y1 = (own.y + r1y) + r2y;
}

// Row loop for the column-pair map: warp w takes rows 10w..10w+9, then +10W.
// body(i, ok, y0, y1) on every lane; lanes with ok hold pair ccol_of(lane) of row i.
template <int MODE, int V = 4, class XLoad, class Body>
__device__ __forceinline__ void for_rows_c(const BsrView& A, int w, int W, const XLoad& xload, int lane,
                                           const Body& body) {
    const int h = cgrp_of(lane);
    const bool lane_ok = lane < 30;
    RowBounds nxt = row_bounds<MODE>(A, 10 * w + h, lane_ok);
    for (int base = 10 * w; base < A.n; base += 10 * W) {
        const int i = base + h;
        const bool ok = lane_ok && i < A.n;
        const RowBounds cur = nxt;
        nxt = row_bounds<MODE>(A, i + 10 * W, lane_ok);
        double y0, y1;
        if (V == 5)
            spmv_row_c5<MODE>(A, i, ok, cur, xload, lane, y0, y1);
        else if (V == 4)
            spmv_row_c4<MODE>(A, i, ok, cur, xload, lane, y0, y1);
        else
            spmv_row_c<MODE>(A, i, ok, cur, xload, lane, y0, y1);
        body(i, ok, y0, y1);
    }
}

// for_rows_c over a row subset: logical rows t in [t0, t1) (ten per warp step, warp-strided), mapped to
// matrix rows i = t < ilo ? t : t + gap — the interior range [ilo, ihi) of a partition with gap = 0
// (t0 = ilo, t1 = ihi), or the rows around it with gap = ihi - ilo (t0 = 0, t1 = n - gap)
template <int MODE, class XLoad, class Body>
__device__ __forceinline__ void for_rows_cr(const BsrView& A, int t0, int t1, int ilo, int gap, int w, int W,
                                            const XLoad& xload, int lane, const Body& body) {
    const int h = cgrp_of(lane);
    const bool lane_ok = lane < 30;
    auto row_of = [&](int t) { return t < ilo ? t : t + gap; };
    int t = t0 + 10 * w + h;
    RowBounds nxt = row_bounds<MODE>(A, row_of(t), lane_ok && t < t1);
    for (int base = t0 + 10 * w; base < t1; base += 10 * W) {
        t = base + h;
        const bool ok = lane_ok && t < t1;
        const int i = ok ? row_of(t) : A.n;
        const RowBounds cur = nxt;
        const int tn = t + 10 * W;
        nxt = row_bounds<MODE>(A, row_of(tn), lane_ok && tn < t1);
        double y0, y1;
        spmv_row_c5<MODE>(A, i, ok, cur, xload, lane, y0, y1);
        body(i, ok, y0, y1);
    }
}

}  // namespace dda
