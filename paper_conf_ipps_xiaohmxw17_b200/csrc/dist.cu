// §8(e) — block-row partitioned PCG across GPUs (beyond the paper: multi-GPU is
// its future work; the related multi-GPU CG of ref [28] is only cited).
//
// Each partition is an ordinary dda_matrix built on the rank's LOCAL numbering
// (own rows first, then halo rows grouped by owning peer — see partition.py);
// its own rows are exact global rows.  Per PCG iteration:
//   halo(p)      pack the own rows each peer needs -> send; receive peers' rows
//                straight into p[n_own:] (contiguous per peer: no unpack)
//   q = K p      the symmetric SpMV of spmv_warp.cuh over own rows only
//   sigma        CTA partials -> fixed-order sum -> allreduce (NCCL sum over ranks)
//   update       d += alpha p; r -= alpha q; z = D^{-1} r; (rr, rz) -> allreduce
//   p = z + beta p
// Two transports share the driver: NCCL (one partition per process / GPU) and
// LOOPBACK (all partitions in one process on one GPU; the exchange is a device
// copy and the "allreduce" a device sum in partition order) — the loopback runs
// the identical partitioned algorithm where only one GPU is available.
// v2: the CG scalars never leave the device.  After each allreduce a one-thread
// kernel (k_scal_alpha / k_scal_beta) turns the reduced sums into alpha, beta,
// the stopping test and the loop state (identical on every partition / rank);
// the vector kernels read them from device memory and return at once when the
// solve has finished.  The host issues iterations in chunks and reads the
// state once per chunk (DDA_DIST_CHUNK, default 8) instead of twice per
// iteration.  The SpMV is the column-pair map (spmv_col.cuh, v5) over own rows.
#include <cooperative_groups.h>
#include <nccl.h>

#include <cmath>
#include <cstring>
#include <vector>

#include "precond_dev.cuh"
#include "spmv_col.cuh"

namespace cg = cooperative_groups;

namespace dda {
namespace {

constexpr int WPB = DDA_THREADS / 32;

struct XLd {
    const double* __restrict__ x;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
};

__device__ __forceinline__ void cta_partial(double v, double* part, int slot_stride, int k, double* red) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    v = warp_sum(v);
    if (lane == 0) red[wib] = v;
    cta_barrier();
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int w = 0; w < WPB; ++w) s += red[w];
        part[k * slot_stride + blockIdx.x] = s;
    }
    cta_barrier();
}


// q = K x over own rows (A.n = n_own); optional partial of x^T q
__global__ void __launch_bounds__(DDA_THREADS, 6) k_spmv_own(BsrView A, const double* __restrict__ x,
                                                             double* __restrict__ q, double* part, int dot) {
    __shared__ double red[WPB];
    const int lane = threadIdx.x & 31;
    double acc = 0.0;
    const XLd xf{x};
    for_rows<SPMV_FULL>(A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, xf, lane,
                        [&](int i, bool ok, double y0, double y1) {
                            if (ok && is_out_lane(lane)) {
                                const size_t o = 6 * (size_t)i + 2 * (q_of(lane) / 3);
                                *reinterpret_cast<double2*>(q + o) = make_double2(y0, y1);
                                if (dot) {
                                    const double2 xv = xf(i, q_of(lane) / 3);
                                    acc += xv.x * y0 + xv.y * y1;
                                }
                            }
                        });
    if (dot) cta_partial(acc, part, gridDim.x, 0, red);
}

// setup over own rows: d = d0 | 0, r = F - q | F, z = M^{-1} r, p = z; partials FF, rr, rz
__global__ void __launch_bounds__(DDA_THREADS) k_init_own(int n, const double* __restrict__ dinv, int use_bj,
                                                          const double* __restrict__ F, const double* d0, double* d,
                                                          const double* __restrict__ q, double* r, double* z,
                                                          double* p, double* part) {
    __shared__ double red[WPB];
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double FF = 0, rr = 0, rz = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0, fv = 0.0;
        if (R.valid) {
            fv = F[R.idx];
            const double dv = d0 ? d0[R.idx] : 0.0;
            if (d != d0) d[R.idx] = dv;
            rv = d0 ? fv - q[R.idx] : fv;
            r[R.idx] = rv;
        }
        FF += fv * fv;
        rr += rv * rv;
        const double zz = use_bj ? bj_lane(dinv, R, rv) : rv;
        if (R.valid) {
            z[R.idx] = zz;
            p[R.idx] = zz;
        }
        rz += rv * zz;
    }
    cta_partial(FF, part, gridDim.x, 0, red);
    cta_partial(rr, part, gridDim.x, 1, red);
    cta_partial(rz, part, gridDim.x, 2, red);
}

__global__ void __launch_bounds__(DDA_THREADS) k_update_own(int n, const double* __restrict__ dinv, int use_bj,
                                                            double alpha, const double* __restrict__ p,
                                                            const double* __restrict__ q, double* d, double* r,
                                                            double* z, double* part) {
    __shared__ double red[WPB];
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rr = 0, rz = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0;
        if (R.valid) {
            d[R.idx] = d[R.idx] + alpha * p[R.idx];
            rv = r[R.idx] - alpha * q[R.idx];
            r[R.idx] = rv;
        }
        rr += rv * rv;
        const double zz = use_bj ? bj_lane(dinv, R, rv) : rv;
        if (R.valid) z[R.idx] = zz;
        rz += rv * zz;
    }
    cta_partial(rr, part, gridDim.x, 0, red);
    cta_partial(rz, part, gridDim.x, 1, red);
}

__global__ void __launch_bounds__(DDA_THREADS) k_resid_own(int n, const double* __restrict__ F,
                                                           const double* __restrict__ q, double* part) {
    __shared__ double red[WPB];
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double acc = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) {
            const double e = F[R.idx] - q[R.idx];
            acc += e * e;
        }
    }
    cta_partial(acc, part, gridDim.x, 0, red);
}

// out[k] = fixed-order sum of part[k*G .. k*G+G), k < nv (one CTA)
__global__ void k_sum_parts(const double* part, int G, int nv, double* out) {
    __shared__ double red[DDA_THREADS];
    for (int k = 0; k < nv; ++k) {
        double s = 0.0;
        for (int j = threadIdx.x; j < G; j += blockDim.x) s += part[k * G + j];
        red[threadIdx.x] = s;
        cta_barrier();
        for (int h = blockDim.x / 2; h > 0; h >>= 1) {
            if (threadIdx.x < h) red[threadIdx.x] += red[threadIdx.x + h];
            cta_barrier();
        }
        if (threadIdx.x == 0) out[k] = red[0];
        cta_barrier();
    }
}

// ---- v2: device-side CG state (one copy per partition; every copy evolves identically)
struct DState {
    double rho, alpha, beta, bnorm, tol, rr;
    int k, maxit, done, status, iters, pad;
};

struct XLdC {   // x (p and its halo) is written by earlier kernels / NCCL: read-only here
    const double* __restrict__ x;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// q = K x over own rows, column-pair map; partial of x^T q.  Skipped once the solve is done.
__global__ void __launch_bounds__(DDA_THREADS, 3) k_spmv_own2(BsrView A, const double* __restrict__ x,
                                                              double* __restrict__ q, double* part,
                                                              const DState* st) {
    __shared__ double red[WPB];
    if (st && st->done) return;
    const int lane = threadIdx.x & 31;
    const XLdC xf{x};
    double acc = 0.0;
    for_rows_c<SPMV_FULL, 5>(A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, xf, lane,
                             [&](int i, bool ok, double y0, double y1) {
                                 if (ok) {
                                     const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                                     *reinterpret_cast<double2*>(q + o) = make_double2(y0, y1);
                                     const double2 xv = xf(i, ccol_of(lane));
                                     acc += xv.x * y0 + xv.y * y1;
                                 }
                             });
    cta_partial(acc, part, gridDim.x, 0, red);
}

// after the sigma allreduce: alpha = rho / sigma (breakdown: done)
__global__ void k_scal_alpha(DState* st, const double* red) {
    if (st->done) return;
    const double sigma = red[0];
    if (!(sigma > 0.0) || !isfinite(sigma)) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; return; }
    st->alpha = st->rho / sigma;
}

__global__ void __launch_bounds__(DDA_THREADS) k_update_own2(int n, const double* __restrict__ dinv, int use_bj,
                                                             const DState* stt, const double* __restrict__ p,
                                                             const double* __restrict__ q, double* d, double* r,
                                                             double* z, double* part) {
    __shared__ double red[WPB];
    if (stt->done) return;
    const double alpha = stt->alpha;
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rr = 0, rz = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0;
        if (R.valid) {
            d[R.idx] = d[R.idx] + alpha * p[R.idx];
            rv = r[R.idx] - alpha * q[R.idx];
            r[R.idx] = rv;
        }
        rr += rv * rv;
        const double zz = use_bj ? bj_lane(dinv, R, rv) : rv;
        if (R.valid) z[R.idx] = zz;
        rz += rv * zz;
    }
    cta_partial(rr, part, gridDim.x, 0, red);
    cta_partial(rz, part, gridDim.x, 1, red);
}

// after the (rr, rz) allreduce: stopping test (reading Z1), breakdown, beta, iteration cap
__global__ void k_scal_beta(DState* st, const double* red) {
    if (st->done) return;
    const double rr = red[0], rz = red[1];
    st->rr = rr;
    st->iters = st->k + 1;
    st->k = st->k + 1;
    if (sqrt(rr) <= st->tol * st->bnorm) { st->status = DDA_OK; st->done = 1; return; }
    if (!(rz > 0.0) || !isfinite(rz)) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; return; }
    st->beta = rz / st->rho;
    st->rho = rz;
    if (st->k >= st->maxit) { st->status = DDA_ERR_NO_CONVERGENCE; st->done = 1; }
}

__global__ void k_pupd_own2(int n6, const DState* st, const double* __restrict__ z, double* p) {
    if (st->done) return;
    const double beta = st->beta;
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < n6; t += gridDim.x * blockDim.x)
        p[t] = fma(beta, p[t], z[t]);
}

// loopback "allreduce": red[0..nv) = sum over partitions, in partition order, of scal[p][0..nv)
__global__ void k_sum_loopback(const double* const* scal, int P, int nv, double* red) {
    const int k = threadIdx.x;
    if (k >= nv) return;
    double s = 0.0;
    for (int p = 0; p < P; ++p) s += scal[p][k];
    red[k] = s;
}

// ---- v3: the scaled block-Jacobi engine per partition (PCG on S K S^T, reading Z25)
//
// Each partition runs the single-GPU scaled iteration on its own rows: phase A forms p = r~ + beta
// p_old for own and gathered rows (halo rows of r~ and p_old come from the exchange), q = Ks p, and
// applies the deferred x += alpha p_old; phase B updates r~ and sums rho' and the w-bound of the
// stopping test; the exact test |L r~| runs only when that bound allows it.  The block scaling needs
// S_j of the halo rows (their diagonal blocks are complete only on the owner): exchanged once per solve.
struct SState {
    double rho, alpha, beta, bnorm, tol, rr, rho_new;
    int k, maxit, done, status, iters, maybe, pend, checks;
};

__global__ void k_pack_w(int n_send, int w, const int* __restrict__ idx, const double* __restrict__ x,
                         double* __restrict__ buf) {
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < w * n_send; t += gridDim.x * blockDim.x)
        buf[t] = x[(size_t)w * idx[t / w] + t % w];
}

// row a of the packed lower-triangular M (TR = false: M[a][c], c <= a) or of its transpose (TR: M[c][a],
// c >= a) applied to the 6-vector spread over the row's lanes; every lane of the warp must call
__device__ __forceinline__ double tri_apply(const double* __restrict__ M, const Row5& R, double v, bool tr) {
    const double* blk = M + (size_t)kDinv * (R.valid ? R.i : 0);
    double z = 0.0;
#pragma unroll
    for (int c = 0; c < 6; ++c) {
        const bool nz = tr ? (c >= R.a) : (c <= R.a);
        const double m = nz ? __ldg(blk + (tr ? lo_off(c, R.a) : lo_off(R.a, c))) : 0.0;
        z = fma(m, __shfl_sync(0xffffffffu, v, R.base + c), z);
    }
    return z;
}

// r = F - q (or F); r~ = S r -> rt, p0; x = L^T d0 (or 0) -> d; partials FF, |r|^2, |r~|^2
__global__ void __launch_bounds__(DDA_THREADS) k_v3_init(int n, const double* __restrict__ F,
                                                         const double* __restrict__ q, const double* d0, double* d,
                                                         const double* __restrict__ sfac,
                                                         const double* __restrict__ lfac, double* rt, double* p0,
                                                         double* part) {
    __shared__ double red[WPB];
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double FF = 0, rr = 0, rz = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double fv = 0.0, rv = 0.0, dv = 0.0;
        if (R.valid) {
            fv = F[R.idx];
            rv = q ? fv - q[R.idx] : fv;
            if (d0) dv = d0[R.idx];
        }
        FF += fv * fv;
        rr += rv * rv;
        const double t0 = tri_apply(sfac, R, rv, false);
        const double t = R.valid ? t0 : 0.0;
        const double x0 = tri_apply(lfac, R, dv, true);
        if (R.valid) {
            rt[R.idx] = t;
            p0[R.idx] = t;
            d[R.idx] = d0 ? x0 : 0.0;
        }
        rz += t * t;
    }
    cta_partial(FF, part, gridDim.x, 0, red);
    cta_partial(rr, part, gridDim.x, 1, red);
    cta_partial(rz, part, gridDim.x, 2, red);
}

struct XFusedLdg {   // x = r~ + beta p_old (k = 0: p_old = r~, beta = 0)
    const double* __restrict__ z;
    const double* __restrict__ p;
    double beta;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const size_t o = 6 * (size_t)vec + 2 * pair;
        const double2 zz = __ldg(reinterpret_cast<const double2*>(z + o));
        const double2 pp = __ldg(reinterpret_cast<const double2*>(p + o));
        return make_double2(fma(beta, pp.x, zz.x), fma(beta, pp.y, zz.y));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// phase A over own rows (A.upper = the scaled blocks)
// p_k lives in buffer (k & 1) ? PB : PA; p_old of iteration k >= 1 is p_{k-1}
__global__ void __launch_bounds__(DDA_THREADS, 3) k_v3_a(BsrView A, const double* rt, double* PA, double* PB,
                                                         double* q, double* x, const SState* st, double* part) {
    __shared__ double red[WPB];
    if (st->done) return;
    const int k = st->k;
    const double* pold = k == 0 ? rt : ((k & 1) ? PA : PB);
    double* pnew = (k & 1) ? PB : PA;
    const double beta = k == 0 ? 0.0 : st->beta;
    const double ap = st->pend ? st->alpha : 0.0;
    const int lane = threadIdx.x & 31;
    const XFusedLdg xf{rt, pold, beta};
    double acc = 0.0;
    for_rows_c<SPMV_OFFDIAG, 5>(A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, xf, lane,
                                [&](int i, bool ok, double y0, double y1) {
                                    if (ok) {
                                        const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                                        const double2 pv = xf(i, ccol_of(lane));
                                        y0 += pv.x;
                                        y1 += pv.y;
                                        if (ap != 0.0) {
                                            const double2 po = __ldg(reinterpret_cast<const double2*>(pold + o));
                                            const double2 xo = *reinterpret_cast<const double2*>(x + o);
                                            *reinterpret_cast<double2*>(x + o) =
                                                make_double2(xo.x + ap * po.x, xo.y + ap * po.y);
                                        }
                                        *reinterpret_cast<double2*>(q + o) = make_double2(y0, y1);
                                        *reinterpret_cast<double2*>(pnew + o) = pv;
                                        acc += pv.x * y0 + pv.y * y1;
                                    }
                                });
    cta_partial(acc, part, gridDim.x, 0, red);
}

__global__ void k_v3_alpha(SState* st, const double* red) {
    if (st->done) return;
    st->pend = 0;                                           // phase A applied the deferred x update
    const double sigma = red[0];
    if (!(sigma > 0.0) || !isfinite(sigma)) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; return; }
    st->alpha = st->rho / sigma;
}

// phase B: r~ -= alpha q; partials |r~|^2 and sum_i w_i |r~_i|^2
__global__ void __launch_bounds__(DDA_THREADS) k_v3_b(int n, double* rt, const double* __restrict__ q,
                                                      const double* __restrict__ w, const SState* st, double* part) {
    __shared__ double red[WPB];
    if (st->done) return;
    const double alpha = st->alpha;
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rz = 0.0, lb = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) {
            const double rv = rt[R.idx] - alpha * q[R.idx];
            rt[R.idx] = rv;
            rz += rv * rv;
            lb += __ldg(w + R.i) * (rv * rv);
        }
    }
    cta_partial(rz, part, gridDim.x, 0, red);
    cta_partial(lb, part, gridDim.x, 1, red);
}

__global__ void k_v3_rho(SState* st, const double* red) {
    if (st->done) return;
    const double rho1 = red[0];
    const double thr = st->tol * st->bnorm;
    st->pend = 1;                                           // x += alpha p_k: next phase A or k_v3_final
    st->iters = st->k + 1;
    st->rho_new = rho1;
    st->maybe = 0;
    if (rho1 == 0.0) { st->rr = 0.0; st->status = DDA_OK; st->k = st->k + 1; st->done = 1; return; }
    st->maybe = (isfinite(rho1) && !(0.999 * red[1] > thr * thr)) ? 1 : 0;
}

// the exact stopping test share |L r~|^2 (only when k_v3_rho flagged it)
__global__ void __launch_bounds__(DDA_THREADS) k_v3_c(int n, const double* __restrict__ rt,
                                                      const double* __restrict__ lfac, const SState* st,
                                                      double* part) {
    __shared__ double red[WPB];
    const bool on = !st->done && st->maybe;
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rl = 0.0;
    if (on) {
        for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
            const Row5 R = row5(grp, lane, n);
            const double rv = R.valid ? rt[R.idx] : 0.0;
            const double o0 = tri_apply(lfac, R, rv, false);
            const double o = R.valid ? o0 : 0.0;
            rl += o * o;
        }
    }
    cta_partial(rl, part, gridDim.x, 0, red);
}

__global__ void k_v3_check(SState* st, const double* red) {
    if (st->done) return;
    if (st->maybe) {
        st->checks = st->checks + 1;
        st->rr = red[0];
        if (sqrt(red[0]) <= st->tol * st->bnorm) { st->status = DDA_OK; st->k = st->k + 1; st->done = 1; return; }
    }
    const double rho1 = st->rho_new;
    st->k = st->k + 1;
    if (!(rho1 > 0.0) || !isfinite(rho1)) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; return; }
    st->beta = rho1 / st->rho;
    st->rho = rho1;
    if (st->k >= st->maxit) { st->status = DDA_ERR_NO_CONVERGENCE; st->done = 1; }
}

// the pending x += alpha p of the last iteration, then d = S^T x (own rows)
__global__ void __launch_bounds__(DDA_THREADS) k_v3_final(int n, double* d, const double* pA, const double* pB,
                                                          const double* __restrict__ sfac, const SState* st) {
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool pend = st->pend;
    const double alpha = st->alpha;
    const double* pk = ((st->k - 1) & 1) ? pB : pA;        // p of the last phase A (iteration k - 1)
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double xv = R.valid ? (pend ? d[R.idx] + alpha * pk[R.idx] : d[R.idx]) : 0.0;
        const double dv = tri_apply(sfac, R, xv, true);
        if (R.valid) d[R.idx] = dv;
    }
}

// ---- v4: one halo and one allreduce per iteration
//
// Iteration k on each partition (own rows), with p_k of own and halo rows in place:
//   A_k  q = Ks p_k; partials sigma = p.q, r~.q, q.q                       -> scal[0..2]
//   allreduce scal[0..5]   (slots 3..5: B_{k-1}'s |r~_k|^2, w-bound, |L r~_k|^2, moved from 8..10 by A_k)
//   B_k  (every CTA derives the same scalars from the reduced sums)
//        stopping test on r~_k (reading Z1 with the w-bound of the single-GPU engine; the exact
//        |L r~_k|^2 was computed speculatively by B_{k-1} once the bound came within a factor 4 of
//        the threshold; if it is missing, B_k only computes it and the next pass repeats A_k, B_k);
//        alpha = rho_k / sigma with the exact rho_k = |r~_k|^2; beta = rho^_{k+1} / rho_k with
//        rho^_{k+1} = rho_k - 2 alpha r~.q + alpha^2 q.q (the recurrence: rho_{k+1} itself is
//        only reduced in the next allreduce);
//        r~' = r~ - alpha q, p_{k+1} = r~' + beta p_k, x += alpha p_k; partials of r~'  -> scal[3..5]
//   halo  of p_{k+1} (pack + one grouped send / receive)
// Partial sums: every CTA writes its partials, the last CTA to arrive (ticket) adds them in CTA
// order and writes the partition's slots: no separate reduction launch.  Per iteration: 3 kernels
// (pack, A, B) and 2 NCCL calls (the halo group, the allreduce).
struct S4 {
    double rho, bnorm, tol, rr;
    double alpha, beta, rho_hat;
    int k, maxit, done, status, iters, checks, spec, retry;
};

// CTA partials -> part[k * G + cta]; the last CTA to arrive (ticket) writes out[k] = the sum over CTAs
// in CTA order and returns true (in every thread of that CTA), after all other CTAs have finished
template <int NV>
__device__ __forceinline__ bool last_cta_sum(double (&v)[NV], double* part, int G, unsigned* ticket, double* out) {
    __shared__ double red[NV][WPB];
    __shared__ bool last;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = warp_sum(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[k][wib] = v[k];
    }
    cta_barrier();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int w = 0; w < WPB; ++w) s += red[k][w];
            part[k * G + blockIdx.x] = s;
        }
        __threadfence();
        last = atomicAdd(ticket, 1u) == (unsigned)G - 1;
    }
    cta_barrier();
    if (!last) return false;
    __threadfence();
    // the whole last CTA adds the G partials: strided per thread, then a fixed-shape tree
    __shared__ double tr[NV][DDA_THREADS];
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        double s = 0.0;
        for (int j = threadIdx.x; j < G; j += DDA_THREADS) s += __ldcg(part + k * G + j);
        tr[k][threadIdx.x] = s;
    }
    cta_barrier();
    for (int h = DDA_THREADS / 2; h > 0; h >>= 1) {
        if (threadIdx.x < h) {
#pragma unroll
            for (int k = 0; k < NV; ++k) tr[k][threadIdx.x] += tr[k][threadIdx.x + h];
        }
        cta_barrier();
    }
    if (threadIdx.x < NV) out[threadIdx.x] = tr[threadIdx.x][0];
    if (threadIdx.x == 0) *ticket = 0u;
    return true;
}

// v5 (loopback): halo rows read straight from the owner partition's p (a pointer per halo row into
// the owner's own rows) instead of a packed copy — the peer-load halo an NVLink-mapped multi-GPU
// version performs over peer memory
struct XPeer {
    const double* __restrict__ x;             // own rows
    const double* const* __restrict__ hsrc;   // [n_halo] the owner's row
    int n_own;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const double* row = vec < n_own ? x + 6 * (size_t)vec : hsrc[vec - n_own];
        return __ldg(reinterpret_cast<const double2*>(row + 2 * pair));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// A_k: q = Ks p_k over own rows (p_k own + halo through XL), partials sigma, r~.q, q.q -> scal[0..2]
// rows: logical range [t0, t1) mapped as in for_rows_cr (t1 < 0: every own row).  mode 0: the only
// launch (sums -> scal[0..2], moves 8..10 -> 3..5); mode 1: the interior launch of the halo overlap
// (sums -> scal[12..14]); mode 2: the boundary launch (scal[0..2] = scal[12..14] + its sums, in that
// order, and the move)
template <class XL>
__global__ void __launch_bounds__(DDA_THREADS, 3) k_v4_a(BsrView A, const double* __restrict__ rt, const XL xf,
                                                         double* __restrict__ q, const S4* st, double* part,
                                                         unsigned* ticket, double* scal, int t0, int t1, int ilo,
                                                         int gap, int mode) {
    if (st->done) return;
    const int lane = threadIdx.x & 31;
    double s0 = 0.0, s1 = 0.0, s2 = 0.0;
    auto rowA = [&](int i, bool ok, double y0, double y1) {
                                    if (ok) {
                                        const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                                        const double2 pv = xf(i, ccol_of(lane));
                                        y0 += pv.x;
                                        y1 += pv.y;
                                        *reinterpret_cast<double2*>(q + o) = make_double2(y0, y1);
                                        const double2 rv = __ldg(reinterpret_cast<const double2*>(rt + o));
                                        s0 += pv.x * y0 + pv.y * y1;
                                        s1 += rv.x * y0 + rv.y * y1;
                                        s2 += y0 * y0 + y1 * y1;
                                    }
                                };
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    if (t1 < 0) for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, rowA);
    else for_rows_cr<SPMV_OFFDIAG>(A, t0, t1, ilo, gap, w0, W, xf, lane, rowA);
    double v[3] = {s0, s1, s2};
    double* out = mode == 1 ? scal + 12 : (mode == 2 ? scal + 16 : scal);
    if (last_cta_sum<3>(v, part, gridDim.x, ticket, out) && mode != 1 && threadIdx.x < 3) {
        if (mode == 2) scal[threadIdx.x] = scal[12 + threadIdx.x] + scal[16 + threadIdx.x];
        scal[3 + threadIdx.x] = scal[8 + threadIdx.x];    // B_{k-1}'s partials (written to 8..10)
    }
}

// flag[i] = own row i references a halo row (a forward column or a transposed source >= n_own)
__global__ void k_boundary_rows(int n_own, const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ col,
                                const int32_t* __restrict__ low_ptr, const int32_t* __restrict__ low_row,
                                uint8_t* __restrict__ flag) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n_own; i += gridDim.x * blockDim.x) {
        bool b = false;
        for (int u = row_ptr[i]; u < row_ptr[i + 1]; ++u) b = b || col[u] >= n_own;
        for (int t = low_ptr[i]; t < low_ptr[i + 1]; ++t) b = b || low_row[t] >= n_own;
        flag[i] = b ? 1 : 0;
    }
}

// B_k (see above); red = the allreduced scal[0..5].  Every CTA reads the state at entry and takes the
// same decisions; only the last CTA (after all others have arrived) writes the state.
// red: the allreduced sums, or (red_all != null, v5) the sums of the partitions' slots red_all[p][0..5]
// taken here in partition order: the one-shot allreduce, identical in every CTA of every partition
__global__ void __launch_bounds__(DDA_THREADS) k_v4_b(int n, double* rt, double* P, const double* __restrict__ q,
                                                      double* x, const double* __restrict__ w,
                                                      const double* __restrict__ lfac, S4* st, const double* red_in,
                                                      const double* const* red_all, int nparts, double* part,
                                                      unsigned* ticket, double* scal) {
    if (st->done) return;
    __shared__ double red_sh[6];
    const double* red = red_in;
    if (red_all) {
        if (threadIdx.x < 6) {
            double s = 0.0;
            for (int p = 0; p < nparts; ++p) s += red_all[p][threadIdx.x];
            red_sh[threadIdx.x] = s;
        }
        __syncthreads();
        red = red_sh;
    }
    const int k = st->k;
    const int spec = st->spec;
    const double thr = st->tol * st->bnorm;
    // ---- the stopping test on r~_k (k = 0: decided at setup)
    bool need_exact = false, stop = false;
    double rho = st->rho;
    if (k > 0) {
        rho = red[3];
        if (rho == 0.0) stop = true;
        else if (isfinite(rho) && !(0.999 * red[4] > thr * thr)) {       // the bound allows convergence
            if (spec) stop = sqrt(red[5]) <= thr;
            else need_exact = true;
        }
    }
    const double sigma = red[0];
    const bool breakdown = !stop && !need_exact &&
                           (!(sigma > 0.0) || !isfinite(sigma) || !(rho > 0.0) || !isfinite(rho));
    const bool maxed = !stop && !need_exact && !breakdown && k >= st->maxit;
    const bool finish = stop || breakdown || maxed;
    const bool update = !finish && !need_exact;
    const double alpha = rho / sigma;
    const double rho_hat = rho - 2.0 * alpha * red[1] + alpha * alpha * red[2];
    const double beta = rho_hat / rho;
    // the exact norm of the NEXT residual is computed speculatively once the bound is within 4x
    const bool spec_next = !(0.999 * red[4] > 16.0 * thr * thr);
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rz = 0.0, lb = 0.0, rl = 0.0;
    if (!finish) {
        const bool exact = need_exact || spec_next;
        for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
            const Row5 R = row5(grp, lane, n);
            double rv = 0.0;
            if (R.valid) {
                rv = rt[R.idx];
                if (update) {          // r~' = r~ - alpha q, p' = r~' + beta p, x += alpha p
                    const double pk = P[R.idx];
                    rv = rv - alpha * q[R.idx];
                    rt[R.idx] = rv;
                    P[R.idx] = fma(beta, pk, rv);
                    x[R.idx] = x[R.idx] + alpha * pk;
                }
                rz += rv * rv;
                lb += __ldg(w + R.i) * (rv * rv);
            }
            if (exact) {               // uniform branch: every lane shuffles
                const double o0 = tri_apply(lfac, R, rv, false);
                const double o = R.valid ? o0 : 0.0;
                rl += o * o;
            }
        }
    }
    // need_exact: r~_k is unchanged and its |r~|^2 and bound are recomputed bit-identically, so the
    // next pass (A_k again, then B_k) finds the same sums plus the exact norm
    // the partials of the next residual go to slots 8..10; the next A moves them to 3..5 once every
    // B of this pass has read 3..5 (the loopback one-shot sum reads the other partitions' slots)
    double v[3] = {rz, lb, rl};
    if (last_cta_sum<3>(v, part, gridDim.x, ticket, scal + 8) && threadIdx.x == 0) {
        if (finish) {
            st->done = 1;
            st->status = stop ? DDA_OK : (breakdown ? DDA_ERR_BREAKDOWN : DDA_ERR_NO_CONVERGENCE);
            st->iters = k;
            if (k > 0 && spec && !(0.999 * red[4] > thr * thr)) { st->checks = st->checks + 1; st->rr = red[5]; }
        } else if (need_exact) {
            st->spec = 1;
            st->retry = st->retry + 1;
        } else {
            if (k > 0 && spec && !(0.999 * red[4] > thr * thr)) { st->checks = st->checks + 1; st->rr = red[5]; }
            st->alpha = alpha;
            st->beta = beta;
            st->rho_hat = rho_hat;
            st->rho = rho;
            st->k = k + 1;
            st->iters = k + 1;
            st->spec = spec_next ? 1 : 0;
        }
    }
}

// r = F - q (or F); r~ = S r -> rt and P (p_0); x = L^T d0 (or 0) -> d; scal[3] = |r~|^2, scal[4] =
// the w-bound, scal[5] = |r|^2 (the exact test of r~_0), scal[6] = FF
__global__ void __launch_bounds__(DDA_THREADS) k_v4_init(int n, const double* __restrict__ F,
                                                         const double* __restrict__ q, const double* d0, double* d,
                                                         const double* __restrict__ sfac,
                                                         const double* __restrict__ lfac,
                                                         const double* __restrict__ w, double* rt, double* P,
                                                         double* part, unsigned* ticket, double* scal) {
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double FF = 0, rr = 0, rz = 0, lb = 0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double fv = 0.0, rv = 0.0, dv = 0.0;
        if (R.valid) {
            fv = F[R.idx];
            rv = q ? fv - q[R.idx] : fv;
            if (d0) dv = d0[R.idx];
        }
        FF += fv * fv;
        rr += rv * rv;
        const double t0 = tri_apply(sfac, R, rv, false);
        const double t = R.valid ? t0 : 0.0;
        const double x0 = tri_apply(lfac, R, dv, true);
        if (R.valid) {
            rt[R.idx] = t;
            P[R.idx] = t;
            d[R.idx] = d0 ? x0 : 0.0;
            lb += __ldg(w + R.i) * (t * t);
        }
        rz += t * t;
    }
    double v[4] = {rz, lb, rr, FF};
    last_cta_sum<4>(v, part, gridDim.x, ticket, scal + 8);  // slots 8..11 (A_0 moves 8..10 to 3..5)
}

// d = S^T x (own rows; every x update was applied in B)
__global__ void __launch_bounds__(DDA_THREADS) k_v4_final(int n, double* d, const double* __restrict__ sfac) {
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double xv = R.valid ? d[R.idx] : 0.0;
        const double dv = tri_apply(sfac, R, xv, true);
        if (R.valid) d[R.idx] = dv;
    }
}

// ---- v6 (loopback): every partition in ONE persistent cooperative kernel.
//
// The single-GPU scaled engine (k_sp_loop, pcg_graph.cu) run over partitions: CTA range [c0, c1) of the
// grid serves partition p's own rows; a halo row of p is read straight from its owner's r~ and p_old
// (pointer tables: owner partition, owner's local row), so p_k = r~_k + beta p_{k-1} is formed on the
// fly for halo rows exactly as for own rows and no halo is ever copied; every grid-wide sum is a
// fixed-order read of all partitions' CTA partials (the allreduce).  Per iteration:
//   A  p_k (own, written to the ping-pong buffer), q = Ks p_k over own rows, x += alpha_{k-1} p_{k-1}
//      | grid barrier, sigma
//   B  r~ -= alpha q; |r~|^2 and the w-bound                     | grid barrier
//   C  (rare) the exact test |L r~| (reading Z1)                 | grid barrier
// Two barriers per iteration, as on one GPU.  On separate GPUs the same kernel needs the peer
// pointers mapped over NVLink and the grid barrier extended by a flag exchange between ranks.
struct DPart {
    BsrView A;            // Ks over own rows (local columns: own, then halo)
    double *rt, *p0, *p1, *q, *x;
    const double* w;      // the w-bound weights (bj_setup)
    const double* lfac;
    const int2* hmap;     // [n_halo]: (owner partition, owner's local row)
    int n_own, c0, c1;
};
struct DPState {
    double alpha, beta, rho, rr;
    int k, iters, status, pend, checks;
    unsigned epoch_end;   // v7: the arrival epoch the loop ended at (the IPC transport continues from it)
};
constexpr int kDPMax = 8;   // partitions held in the kernel's parameter block (more: v5)
struct DPArgs {
    DPart parts[kDPMax];
    const DPart* gparts;  // the same table in global memory (halo owners' arrays)
    int P;
    double* part;         // [4][gridDim] CTA partials
    DPState* st;
    double rho0, thr;
    int maxit;
};

// p = r~ + beta p_old for own and halo rows (sel: 0 -> p_old = r~ (k = 0), 1 -> p0, 2 -> p1)
struct XFusedPeer {
    const DPart* parts;
    const double* rt;
    const double* pold;
    const int2* hmap;
    int n_own, sel;
    double beta;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const double* z;
        const double* p;
        size_t o;
        if (vec < n_own) {
            z = rt;
            p = pold;
            o = 6 * (size_t)vec + 2 * pair;
        } else {
            const int2 h = __ldg(hmap + (vec - n_own));
            const DPart& Q = parts[h.x];
            z = Q.rt;
            p = sel == 0 ? Q.rt : (sel == 1 ? Q.p0 : Q.p1);
            o = 6 * (size_t)h.y + 2 * pair;
        }
        const double2 zz = *reinterpret_cast<const double2*>(z + o), pp = *reinterpret_cast<const double2*>(p + o);
        return make_double2(fma(beta, pp.x, zz.x), fma(beta, pp.y, zz.y));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// fixed-order grid sum of NV values (every CTA gets the same totals): partials -> part[(slot+k)*G + cta]
template <int NV>
__device__ __forceinline__ void dp_allsum(const DPArgs& a, cg::grid_group& grid, int slot, double (&v)[NV],
                                          double (&tot)[NV]) {
    __shared__ double red[NV][DDA_THREADS];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5, G = gridDim.x;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = warp_sum(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[k][wib] = v[k];
    }
    cta_barrier();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int w = 0; w < WPB; ++w) s += red[k][w];
            a.part[(size_t)(slot + k) * G + blockIdx.x] = s;
        }
    }
    grid.sync();
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        const double* part = a.part + (size_t)(slot + k) * G;
        double s = 0.0;
        for (int j = threadIdx.x; j < G; j += DDA_THREADS) s += *(volatile const double*)(part + j);
        red[k][threadIdx.x] = s;
    }
    cta_barrier();
    for (int h = DDA_THREADS / 2; h > 0; h >>= 1) {
        if (threadIdx.x < h) {
#pragma unroll
            for (int k = 0; k < NV; ++k) red[k][threadIdx.x] += red[k][threadIdx.x + h];
        }
        cta_barrier();
    }
#pragma unroll
    for (int k = 0; k < NV; ++k) tot[k] = red[k][0];
    cta_barrier();
}

__global__ void __launch_bounds__(DDA_THREADS, 3) k_dist_loop(const DPArgs a) {
    cg::grid_group grid = cg::this_grid();
    int pi = 0;
#pragma unroll
    for (int q = 0; q + 1 < kDPMax; ++q)
        if (q + 1 < a.P && (int)blockIdx.x >= a.parts[q].c1) pi = q + 1;
    const DPart& D = a.parts[pi];
    const int lane = threadIdx.x & 31;
    const int w0 = ((int)blockIdx.x - D.c0) * WPB + (threadIdx.x >> 5), W = (D.c1 - D.c0) * WPB;
    const int n = D.n_own, ngrp = (n + 4) / 5;
    const double thr = a.thr;
    double rho = a.rho0, alpha = 0.0, beta = 0.0, rr_last = 0.0;
    int k = 0, status = DDA_ERR_NO_CONVERGENCE, iters = 0, checks = 0, pend = 0;
    for (;;) {
        double* pnew = (k & 1) ? D.p1 : D.p0;
        const double* pold = k == 0 ? D.rt : ((k & 1) ? D.p0 : D.p1);
        const XFusedPeer xf{a.gparts, D.rt, pold, D.hmap, n, k == 0 ? 0 : ((k & 1) ? 1 : 2), beta};
        const double ap = alpha;
        double acc = 0.0;
        for_rows_c<SPMV_OFFDIAG, 5>(D.A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                y0 += pv.x;
                y1 += pv.y;
                const double2 po = *reinterpret_cast<const double2*>(pold + o);
                const double2 xo = *reinterpret_cast<const double2*>(D.x + o);
                *reinterpret_cast<double2*>(D.x + o) = make_double2(xo.x + ap * po.x, xo.y + ap * po.y);
                *reinterpret_cast<double2*>(D.q + o) = make_double2(y0, y1);
                *reinterpret_cast<double2*>(pnew + o) = pv;
                acc += pv.x * y0 + pv.y * y1;
            }
        });
        double sv[1] = {acc}, stot[1];
        dp_allsum<1>(a, grid, 0, sv, stot);
        const double sigma = stot[0];
        pend = 0;
        if (!(sigma > 0.0) || !isfinite(sigma)) { status = DDA_ERR_BREAKDOWN; break; }
        alpha = rho / sigma;
        double rz = 0.0, lb = 0.0;
        for (int grp = w0; grp < ngrp; grp += 2 * W) {     // two row groups in flight per warp
            const Row5 RA = row5(grp, lane, n);
            const Row5 RB = row5(grp + W, lane, n);
            double ra = 0, qa = 0, rb = 0, qb = 0, wa = 0, wb = 0;
            if (RA.valid) { ra = D.rt[RA.idx]; qa = D.q[RA.idx]; wa = __ldg(D.w + RA.i); }
            if (RB.valid) { rb = D.rt[RB.idx]; qb = D.q[RB.idx]; wb = __ldg(D.w + RB.i); }
            const double rva = RA.valid ? ra - alpha * qa : 0.0;
            const double rvb = RB.valid ? rb - alpha * qb : 0.0;
            if (RA.valid) D.rt[RA.idx] = rva;
            if (RB.valid) D.rt[RB.idx] = rvb;
            rz += rva * rva + rvb * rvb;
            lb += wa * (rva * rva) + wb * (rvb * rvb);
        }
        double bv[2] = {rz, lb}, btot[2];
        dp_allsum<2>(a, grid, 1, bv, btot);
        const double rho1 = btot[0];
        pend = 1;
        iters = k + 1;
        if (rho1 == 0.0) { status = DDA_OK; rr_last = 0.0; k = k + 1; break; }
        if (isfinite(rho1) && !(0.999 * btot[1] > thr * thr)) {   // the exact test (reading Z1)
            double rl = 0.0;
            for (int grp = w0; grp < ngrp; grp += W) {
                const Row5 R = row5(grp, lane, n);
                const double rv = R.valid ? D.rt[R.idx] : 0.0;
                const double o0 = tri_apply(D.lfac, R, rv, false);
                const double o = R.valid ? o0 : 0.0;
                rl += o * o;
            }
            double cv[1] = {rl}, ctot[1];
            dp_allsum<1>(a, grid, 3, cv, ctot);
            checks += 1;
            rr_last = ctot[0];
            if (sqrt(ctot[0]) <= thr) { status = DDA_OK; k = k + 1; break; }
        }
        k = k + 1;
        if (!(rho1 > 0.0) || !isfinite(rho1)) { status = DDA_ERR_BREAKDOWN; break; }
        beta = rho1 / rho;
        rho = rho1;
        if (k >= a.maxit) { status = DDA_ERR_NO_CONVERGENCE; break; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        DPState* st = a.st;
        st->k = k;
        st->iters = iters;
        st->status = status;
        st->alpha = alpha;
        st->beta = beta;
        st->rho = rho;
        st->rr = rr_last;
        st->pend = pend;
        st->checks = checks;
    }
}

// the pending x += alpha p_{k-1} of the last iteration, then d = S^T x (own rows)
__global__ void __launch_bounds__(DDA_THREADS) k_dp_final(int n, double* d, const double* __restrict__ pk,
                                                          const DPState* st, const double* __restrict__ sfac) {
    const bool pend = st->pend;
    const double alpha = st->alpha;
    const int lane = threadIdx.x & 31, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double xv = R.valid ? (pend ? d[R.idx] + alpha * pk[R.idx] : d[R.idx]) : 0.0;
        const double dv = tri_apply(sfac, R, xv, true);
        if (R.valid) d[R.idx] = dv;
    }
}

// ---- v7 (loopback): one persistent cooperative kernel PER PARTITION ("rank"), the launches running
// concurrently on their own streams, exactly the structure one process per GPU would run.
//
// Each rank's kernel runs k_sp_loop's iteration over its own rows with its own grid.  What crosses
// ranks: the halo rows (read from the owners' r~ / p_old through the partition table, as in v6) and
// every reduction, taken as a two-level fixed-order sum: the rank's CTA partials (grid barrier),
// then the ranks' totals, which each rank's leader publishes to a slot set and announces on a shared
// arrival counter; every CTA of every rank waits for all P arrivals of that epoch and sums the P
// totals in rank order (a one-shot deterministic allreduce, identical everywhere).  The arrival
// wait is also the inter-rank barrier that orders one phase's halo writes before the next phase's
// reads.  Across GPUs the same code needs the partition table and the slot / counter words mapped over
// NVLink (IPC handles) and system-scope fences; here they are one device's memory.  Every wait is
// bounded (an error flag instead of a hang).
// one arrival on the (possibly peer-mapped) counter with release semantics at system scope: cumulative
// over this thread's earlier writes and everything ordered before them (the CTA barrier, the grid
// barrier), cheaper than a full system fence followed by an atomic
__device__ __forceinline__ void arrive_release_sys(unsigned* p) {
    asm volatile("red.release.sys.global.add.u32 [%0], 1;" :: "l"(p) : "memory");
}
__device__ __forceinline__ int ld_acquire(const int* p) {   // system scope: the counter may be a peer's
    int v;
    asm volatile("ld.acquire.sys.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
constexpr int kSlotStride = 16;              // doubles per rank in a slot set
constexpr size_t kSyncHdr = 64;              // IPC sync buffer: counter, error flag; the slot sets follow
constexpr int kRankSets = 4;                 // slot sets in rotation (a rank is at most one epoch ahead)
struct RArgs {
    const DPart* parts;                       // every rank's table entry (the owners' arrays)
    int P, rank;
    double* part;                             // this rank's CTA partials [4][gridDim]
    double* slots;                            // [kRankSets][P][kSlotStride] rank totals
    unsigned* arrive;                         // shared arrival counter (monotone over epochs)
    unsigned epoch0;                          // epochs already consumed on this counter
    DPState* st;                              // this rank's result
    int* err;                                 // set when a wait hit its bound
    double rho0, thr;
    int maxit;
};

template <int NV>
__device__ __forceinline__ void rank_allsum(const RArgs& a, cg::grid_group& grid, int slot, unsigned& epoch,
                                            double (&v)[NV], double (&tot)[NV]) {
    __shared__ double red[NV][DDA_THREADS];
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5, G = gridDim.x;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = warp_sum(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[k][wib] = v[k];
    }
    cta_barrier();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int w = 0; w < WPB; ++w) s += red[k][w];
            a.part[(size_t)(slot + k) * G + blockIdx.x] = s;
        }
    }
    grid.sync();
    epoch += 1;
    double* set = a.slots + (size_t)(epoch % kRankSets) * a.P * kSlotStride;
    if (blockIdx.x == 0) {                   // the rank's total, in CTA order (a fixed-shape tree)
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            const double* part = a.part + (size_t)(slot + k) * G;
            double s = 0.0;
            for (int j = threadIdx.x; j < G; j += DDA_THREADS) s += *(volatile const double*)(part + j);
            red[k][threadIdx.x] = s;
        }
        cta_barrier();
        for (int h = DDA_THREADS / 2; h > 0; h >>= 1) {
            if (threadIdx.x < h) {
#pragma unroll
                for (int k = 0; k < NV; ++k) red[k][threadIdx.x] += red[k][threadIdx.x + h];
            }
            cta_barrier();
        }
        if (threadIdx.x == 0) {
#pragma unroll
            for (int k = 0; k < NV; ++k) set[(size_t)a.rank * kSlotStride + k] = red[k][0];
            arrive_release_sys(a.arrive);    // the slot (and the rank's phase writes) before the arrival
        }
        cta_barrier();
    }
    if (threadIdx.x == 0) {                  // every rank's total of this epoch has arrived
        const unsigned target = epoch * (unsigned)a.P;
        unsigned long long spins = 0;
        while ((int)(ld_acquire(reinterpret_cast<const int*>(a.arrive)) - (int)target) < 0) {
            if (++spins > (1ull << 28)) { atomicExch(a.err, 1); break; }
            __nanosleep(32);
        }
    }
    cta_barrier();
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        double s = 0.0;
        for (int q = 0; q < a.P; ++q) s += *(volatile const double*)(set + (size_t)q * kSlotStride + k);
        tot[k] = s;
    }
}

__global__ void __launch_bounds__(DDA_THREADS, 3) k_rank_loop(const RArgs a) {
    cg::grid_group grid = cg::this_grid();
    const DPart& D = a.parts[a.rank];
    const int lane = threadIdx.x & 31;
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    const int n = D.n_own, ngrp = (n + 4) / 5;
    const double thr = a.thr;
    double rho = a.rho0, alpha = 0.0, beta = 0.0, rr_last = 0.0;
    int k = 0, status = DDA_ERR_NO_CONVERGENCE, iters = 0, checks = 0, pend = 0;
    unsigned epoch = a.epoch0;
    for (;;) {
        double* pnew = (k & 1) ? D.p1 : D.p0;
        const double* pold = k == 0 ? D.rt : ((k & 1) ? D.p0 : D.p1);
        const XFusedPeer xf{a.parts, D.rt, pold, D.hmap, n, k == 0 ? 0 : ((k & 1) ? 1 : 2), beta};
        const double ap = alpha;
        double acc = 0.0;
        for_rows_c<SPMV_OFFDIAG, 5>(D.A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                y0 += pv.x;
                y1 += pv.y;
                const double2 po = *reinterpret_cast<const double2*>(pold + o);
                const double2 xo = *reinterpret_cast<const double2*>(D.x + o);
                *reinterpret_cast<double2*>(D.x + o) = make_double2(xo.x + ap * po.x, xo.y + ap * po.y);
                *reinterpret_cast<double2*>(D.q + o) = make_double2(y0, y1);
                *reinterpret_cast<double2*>(pnew + o) = pv;
                acc += pv.x * y0 + pv.y * y1;
            }
        });
        double sv[1] = {acc}, stot[1];
        rank_allsum<1>(a, grid, 0, epoch, sv, stot);
        const double sigma = stot[0];
        pend = 0;
        if (!(sigma > 0.0) || !isfinite(sigma)) { status = DDA_ERR_BREAKDOWN; break; }
        alpha = rho / sigma;
        double rz = 0.0, lb = 0.0;
        for (int grp = w0; grp < ngrp; grp += 2 * W) {
            const Row5 RA = row5(grp, lane, n);
            const Row5 RB = row5(grp + W, lane, n);
            double ra = 0, qa = 0, rb = 0, qb = 0, wa = 0, wb = 0;
            if (RA.valid) { ra = D.rt[RA.idx]; qa = D.q[RA.idx]; wa = __ldg(D.w + RA.i); }
            if (RB.valid) { rb = D.rt[RB.idx]; qb = D.q[RB.idx]; wb = __ldg(D.w + RB.i); }
            const double rva = RA.valid ? ra - alpha * qa : 0.0;
            const double rvb = RB.valid ? rb - alpha * qb : 0.0;
            if (RA.valid) D.rt[RA.idx] = rva;
            if (RB.valid) D.rt[RB.idx] = rvb;
            rz += rva * rva + rvb * rvb;
            lb += wa * (rva * rva) + wb * (rvb * rvb);
        }
        double bv[2] = {rz, lb}, btot[2];
        rank_allsum<2>(a, grid, 1, epoch, bv, btot);
        const double rho1 = btot[0];
        pend = 1;
        iters = k + 1;
        if (rho1 == 0.0) { status = DDA_OK; rr_last = 0.0; k = k + 1; break; }
        if (isfinite(rho1) && !(0.999 * btot[1] > thr * thr)) {   // the exact test (reading Z1)
            double rl = 0.0;
            for (int grp = w0; grp < ngrp; grp += W) {
                const Row5 R = row5(grp, lane, n);
                const double rv = R.valid ? D.rt[R.idx] : 0.0;
                const double o0 = tri_apply(D.lfac, R, rv, false);
                const double o = R.valid ? o0 : 0.0;
                rl += o * o;
            }
            double cv[1] = {rl}, ctot[1];
            rank_allsum<1>(a, grid, 3, epoch, cv, ctot);
            checks += 1;
            rr_last = ctot[0];
            if (sqrt(ctot[0]) <= thr) { status = DDA_OK; k = k + 1; break; }
        }
        k = k + 1;
        if (!(rho1 > 0.0) || !isfinite(rho1)) { status = DDA_ERR_BREAKDOWN; break; }
        beta = rho1 / rho;
        rho = rho1;
        if (k >= a.maxit) { status = DDA_ERR_NO_CONVERGENCE; break; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        DPState* st = a.st;
        st->k = k;
        st->iters = iters;
        st->status = status;
        st->alpha = alpha;
        st->beta = beta;
        st->rho = rho;
        st->rr = rr_last;
        st->pend = pend;
        st->checks = checks;
        st->epoch_end = epoch;
    }
}

__global__ void k_ipc_coll(const double* in, int nv, double* out, char* sync, int P, int rank, unsigned epoch) {
    unsigned* arrive = reinterpret_cast<unsigned*>(sync);
    int* err = reinterpret_cast<int*>(sync + 16);
    double* set = reinterpret_cast<double*>(sync + kSyncHdr) + (size_t)(epoch % kRankSets) * P * kSlotStride;
    for (int k = 0; k < nv; ++k) set[(size_t)rank * kSlotStride + k] = in[k];
    arrive_release_sys(arrive);
    const unsigned target = epoch * (unsigned)P;
    unsigned long long spins = 0;
    while ((int)(ld_acquire(reinterpret_cast<const int*>(arrive)) - (int)target) < 0) {
        if (++spins > (1ull << 28)) { atomicExch_system(err, 1); break; }
        __nanosleep(64);
    }
    for (int k = 0; k < nv; ++k) {
        double acc = 0.0;
        for (int q = 0; q < P; ++q) acc += *(volatile const double*)(set + (size_t)q * kSlotStride + k);
        out[k] = acc;
    }
}

__global__ void k_ipc_hmap(int n, int q, const int* __restrict__ peer_idx, int2* __restrict__ out) {
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < n; t += gridDim.x * blockDim.x)
        out[t] = make_int2(q, peer_idx[t]);
}

int grid_of(const void* k, int cap_per_sm) {
    int per = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k, DDA_THREADS, 0);
    if (per < 1) per = 1;
    if (per > cap_per_sm) per = cap_per_sm;
    return device_sms() * per;
}

}  // namespace

dda_status_t bj_setup_rows(dda_matrix* K, int32_t nrows, cudaStream_t st, int32_t* bad_block);

}  // namespace dda

using namespace dda;

struct DistPart {
    dda_matrix* K = nullptr;
    int n_own = 0, n_local = 0;
    std::vector<int> send_counts, recv_counts, send_off, recv_off;
    int n_send = 0;
    int* send_idx = nullptr;     // device
    double* sendbuf = nullptr;   // device [6 n_send]
    double* x = nullptr;         // device [6 n_local]: p (own) + halo
    double *q = nullptr, *r = nullptr, *z = nullptr, *part = nullptr, *scal = nullptr;
    double* red = nullptr;       // device: allreduced scalars (v2)
    void* dst = nullptr;         // device DState (v2)
    const double** scal_ptrs = nullptr;   // device [P] (loopback: every partition's scal)
    double *rt = nullptr, *pA = nullptr, *pB = nullptr;   // v3: r~, p ping-pong over local rows (own + halo)
    unsigned* ticket = nullptr;  // v4: last-CTA ticket of the partial sums
    unsigned* ticket2 = nullptr; // v4 halo overlap: the interior launch's ticket
    int ilo = 0, ihi = 0;        // v4 halo overlap: the longest run of own rows that read no halo row
    std::vector<int> h_send_idx; // host copy of send_idx (v5 peer tables)
    const double** hsrc = nullptr;   // v5: [n_halo] device pointers to the owners' rows of p
    int G_spmv = 0, G_vec = 0, G_spmv2 = 0, G_a3 = 0;
    bool ipc_alloc = false;      // sendbuf, rt, pA, pB, send_idx from cudaMalloc (exported through IPC handles)
};

// release a partition's device buffers (the IPC-exported ones were cudaMalloc'd)
static void free_part(DistPart& p) {
    void* exported[] = {p.send_idx, p.sendbuf, p.rt, p.pA, p.pB};
    void* pooled[] = {p.x, p.q, p.r, p.z, p.part, p.scal, p.red, p.dst, (void*)p.scal_ptrs, p.ticket,
                      (void*)p.hsrc, p.ticket2};
    for (void* v : exported)
        if (v) { if (p.ipc_alloc) cudaFree(v); else dda::dev_free(v); }
    for (void* v : pooled)
        if (v) dda::dev_free(v);
}

// IPC transport (one partition per process; peers' buffers mapped with CUDA IPC handles): what this
// rank reads of peer q
struct IpcPeer {
    double* sendbuf = nullptr;   // q's packed halo rows, in q's send order
    double *rt = nullptr, *pA = nullptr, *pB = nullptr;   // q's r~ and p ping-pong (own rows first)
    int* send_idx = nullptr;     // q's send lists (local rows), concatenated by destination
    std::vector<int> send_off;   // [P + 1] q's send offsets
    std::vector<void*> opened;   // mapped handles to close
};

struct dda_comm {
    bool loopback = false;
    bool ipc = false;            // IPC transport (dda_comm_init_ipc)
    bool ipc_ready = false;      // peers mapped (dda_comm_ipc_import)
    std::vector<IpcPeer> peers;  // [P] (own entry: own pointers)
    char* sync = nullptr;        // rank 0's arrival counter + slot sets (mapped on the other ranks)
    bool sync_owned = false;
    unsigned epoch = 0;          // arrival epochs consumed (identical on every rank)
    int last_checks = 0;         // v4: exact stopping tests of the last solve
    double prof_ms[4] = {0, 0, 0, 0};   // v4 with DDA_DIST_PROFILE=1: halo, A, allreduce, B (summed, ms)
    int nranks = 1, rank = 0;    // NCCL: world; loopback: nranks = partitions, rank unused
    ncclComm_t nccl = nullptr;
    std::vector<DistPart> parts;
};

int dda::comm_nparts(const dda_comm* c) { return c->nranks; }
int dda::comm_part_index(const dda_comm* c, int part) {
    if (c->loopback) return (part >= 0 && part < c->nranks) ? part : -1;
    return part == 0 ? c->rank : -1;
}

static dda_status_t nccl_fail(ncclResult_t r) {
    (void)r;
    return DDA_ERR_NCCL;
}
#define DDA_NCCL(call)                              \
    do {                                            \
        ncclResult_t _r = (call);                   \
        if (_r != ncclSuccess) return nccl_fail(_r); \
    } while (0)

extern "C" dda_status_t dda_comm_unique_id(void* id128) {
    if (!id128) return DDA_ERR_ARG;
    ncclUniqueId id;
    DDA_NCCL(ncclGetUniqueId(&id));
    std::memcpy(id128, &id, sizeof id);
    return DDA_OK;
}

extern "C" dda_status_t dda_comm_init(int32_t nranks, int32_t rank, const void* id128, dda_comm_t* out) {
    if (!out || !id128 || nranks < 1 || rank < 0 || rank >= nranks) return DDA_ERR_ARG;
    *out = nullptr;
    dda_comm* c = new dda_comm();
    c->nranks = nranks;
    c->rank = rank;
    ncclUniqueId id;
    std::memcpy(&id, id128, sizeof id);
    ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, id, rank);
    if (r != ncclSuccess) { delete c; return DDA_ERR_NCCL; }
    c->parts.resize(1);
    *out = c;
    return DDA_OK;
}

extern "C" dda_status_t dda_comm_init_loopback(int32_t nparts, dda_comm_t* out) {
    if (!out || nparts < 1) return DDA_ERR_ARG;
    dda_comm* c = new dda_comm();
    c->loopback = true;
    c->nranks = nparts;
    c->parts.resize(nparts);
    *out = c;
    return DDA_OK;
}

extern "C" dda_status_t dda_comm_init_ipc(int32_t nranks, int32_t rank, dda_comm_t* out) {
    if (!out || nranks < 1 || nranks > kDPMax || rank < 0 || rank >= nranks) return DDA_ERR_ARG;
    dda_comm* c = new dda_comm();
    c->ipc = true;
    c->nranks = nranks;
    c->rank = rank;
    c->parts.resize(1);
    c->peers.resize(nranks);
    *out = c;
    return DDA_OK;
}

static constexpr uint32_t kIpcMagic = 0x44444149u;   // "DDAI"
struct IpcBlob {   // what dda_comm_ipc_export writes: this rank's exchange plan and buffer handles
    uint32_t magic;
    int32_t rank, nranks, n_send, has_sync;
    int32_t send_off[kDPMax + 1];
    cudaIpcMemHandle_t sendbuf, rt, pA, pB, send_idx, sync;
};

extern "C" dda_status_t dda_comm_ipc_export(dda_comm_t c, void* blob, int64_t* bytes) {
    if (!c || !c->ipc || !bytes) return DDA_ERR_ARG;
    const int64_t need = (int64_t)sizeof(IpcBlob);
    if (!blob) { *bytes = need; return DDA_OK; }
    if (*bytes < need) return DDA_ERR_ARG;
    DistPart& D = c->parts[0];
    if (!D.K || !D.ipc_alloc) return DDA_ERR_ARG;          // attach (or build) this rank's partition first
    IpcBlob b{};
    b.magic = kIpcMagic;
    b.rank = c->rank;
    b.nranks = c->nranks;
    b.n_send = D.n_send;
    for (int q = 0; q <= c->nranks; ++q) b.send_off[q] = D.send_off[q];
    if (c->rank == 0 && !c->sync) {   // rank 0 owns the arrival counter and the slot sets
        const size_t sb = kSyncHdr + sizeof(double) * kRankSets * kSlotStride * (size_t)c->nranks;
        DDA_CK(cudaMalloc(reinterpret_cast<void**>(&c->sync), sb));
        DDA_CK(cudaMemset(c->sync, 0, sb));
        c->sync_owned = true;
    }
    DDA_CK(cudaDeviceSynchronize());
    DDA_CK(cudaIpcGetMemHandle(&b.sendbuf, D.sendbuf));
    DDA_CK(cudaIpcGetMemHandle(&b.rt, D.rt));
    DDA_CK(cudaIpcGetMemHandle(&b.pA, D.pA));
    DDA_CK(cudaIpcGetMemHandle(&b.pB, D.pB));
    DDA_CK(cudaIpcGetMemHandle(&b.send_idx, D.send_idx));
    b.has_sync = c->rank == 0;
    if (b.has_sync) DDA_CK(cudaIpcGetMemHandle(&b.sync, c->sync));
    std::memcpy(blob, &b, sizeof b);
    *bytes = need;
    return DDA_OK;
}

extern "C" dda_status_t dda_comm_ipc_import(dda_comm_t c, const void* blobs, int64_t bytes) {
    if (!c || !c->ipc || !blobs || bytes != (int64_t)sizeof(IpcBlob) || c->ipc_ready) return DDA_ERR_ARG;
    DistPart& D = c->parts[0];
    if (!D.K) return DDA_ERR_ARG;
    const int P = c->nranks, me = c->rank;
    std::vector<IpcBlob> b(P);
    for (int q = 0; q < P; ++q) {
        std::memcpy(&b[q], static_cast<const char*>(blobs) + (size_t)q * sizeof(IpcBlob), sizeof(IpcBlob));
        if (b[q].magic != kIpcMagic || b[q].rank != q || b[q].nranks != P) return DDA_ERR_ARG;
        // q's send list to this rank must match this rank's receive list from q
        if (q != me && b[q].send_off[me + 1] - b[q].send_off[me] != D.recv_counts[q]) return DDA_ERR_ARG;
    }
    if (!b[0].has_sync) return DDA_ERR_ARG;
    auto open = [&](IpcPeer& Q, const cudaIpcMemHandle_t& h, void** out) -> cudaError_t {
        cudaError_t e = cudaIpcOpenMemHandle(out, h, cudaIpcMemLazyEnablePeerAccess);
        if (e == cudaSuccess) Q.opened.push_back(*out);
        return e;
    };
    for (int q = 0; q < P; ++q) {
        IpcPeer& Q = c->peers[q];
        Q.send_off.assign(b[q].send_off, b[q].send_off + P + 1);
        if (q == me) {
            Q.sendbuf = D.sendbuf; Q.rt = D.rt; Q.pA = D.pA; Q.pB = D.pB; Q.send_idx = D.send_idx;
            continue;
        }
        DDA_CK(open(Q, b[q].sendbuf, reinterpret_cast<void**>(&Q.sendbuf)));
        DDA_CK(open(Q, b[q].rt, reinterpret_cast<void**>(&Q.rt)));
        DDA_CK(open(Q, b[q].pA, reinterpret_cast<void**>(&Q.pA)));
        DDA_CK(open(Q, b[q].pB, reinterpret_cast<void**>(&Q.pB)));
        DDA_CK(open(Q, b[q].send_idx, reinterpret_cast<void**>(&Q.send_idx)));
    }
    if (me != 0) DDA_CK(cudaIpcOpenMemHandle(reinterpret_cast<void**>(&c->sync), b[0].sync, cudaIpcMemLazyEnablePeerAccess));
    c->epoch = 0;
    c->ipc_ready = true;
    return DDA_OK;
}

extern "C" void dda_comm_free(dda_comm_t c) {
    if (!c) return;
    cudaDeviceSynchronize();
    for (IpcPeer& q : c->peers)
        for (void* v : q.opened) cudaIpcCloseMemHandle(v);
    if (c->sync && !c->sync_owned) cudaIpcCloseMemHandle(c->sync);
    for (DistPart& p : c->parts) free_part(p);
    if (c->sync && c->sync_owned) cudaFree(c->sync);
    if (c->nccl) ncclCommDestroy(c->nccl);
    delete c;
}

extern "C" dda_status_t dda_dist_info(dda_comm_t c, int32_t part, int32_t* n_own, int32_t* n_halo,
                                      int32_t* send_counts, int32_t* recv_counts, int32_t* send_idx) {
    if (!c) return DDA_ERR_ARG;
    const int slot = c->loopback ? part : 0;
    if (slot < 0 || slot >= (int)c->parts.size() || (!c->loopback && part != 0)) return DDA_ERR_ARG;
    const DistPart& D = c->parts[slot];
    if (!D.K) return DDA_ERR_ARG;
    if (n_own) *n_own = D.n_own;
    if (n_halo) *n_halo = D.n_local - D.n_own;
    for (int q = 0; q < c->nranks; ++q) {
        if (send_counts) send_counts[q] = D.send_counts[q];
        if (recv_counts) recv_counts[q] = D.recv_counts[q];
    }
    if (send_idx && D.n_send) {
        if (cudaMemcpy(send_idx, D.send_idx, D.n_send * sizeof(int), cudaMemcpyDeviceToHost) != cudaSuccess)
            return DDA_ERR_CUDA;
    }
    return DDA_OK;
}

extern "C" dda_status_t dda_dist_attach(dda_comm_t c, int32_t part, dda_matrix_t K, int32_t n_own,
                                        const int32_t* send_counts, const int32_t* send_idx,
                                        const int32_t* recv_counts, void* stream) {
    if (!c || !K || !send_counts || !recv_counts) return DDA_ERR_ARG;
    if (K->rperm) return DDA_ERR_ARG;            // partitions are built in their own local numbering
    const int P = c->nranks;
    const int slot = c->loopback ? part : 0;
    if (slot < 0 || slot >= (int)c->parts.size() || n_own < 1 || n_own > K->n) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    DistPart& D = c->parts[slot];
    // re-attach (e.g. the matrix rebuilt for the next step): release the old buffers.  Under a mapped IPC
    // transport the exported ones stay (peers hold their handles): the new partition must have the same
    // sizes and exchange plan
    double *keep_sendbuf = nullptr, *keep_rt = nullptr, *keep_pA = nullptr, *keep_pB = nullptr;
    int* keep_send_idx = nullptr;
    if (D.K) {
        cudaStreamSynchronize(st);
        if (c->ipc_ready) {
            if (n_own != D.n_own || K->n != D.n_local) return DDA_ERR_ARG;
            for (int q = 0; q < P; ++q)
                if (send_counts[q] != D.send_counts[q] || recv_counts[q] != D.recv_counts[q]) return DDA_ERR_ARG;
            keep_sendbuf = D.sendbuf; keep_rt = D.rt; keep_pA = D.pA; keep_pB = D.pB; keep_send_idx = D.send_idx;
            D.sendbuf = D.rt = D.pA = D.pB = nullptr;
            D.send_idx = nullptr;
        }
        free_part(D);
        D = DistPart();
    }
    for (int q = 0; q < P; ++q)
        if (send_counts[q] < 0 || recv_counts[q] < 0 || (q == c->rank && !c->loopback && (send_counts[q] || recv_counts[q])))
            return DDA_ERR_ARG;
    {   // every send index is an own row (k_pack_w gathers them without bounds checks)
        int64_t ns = 0;
        for (int q = 0; q < P; ++q) ns += send_counts[q];
        if (ns && !send_idx) return DDA_ERR_ARG;
        for (int64_t t = 0; t < ns; ++t)
            if (send_idx[t] < 0 || send_idx[t] >= n_own) return DDA_ERR_ARG;
    }
    D.K = K;
    D.n_own = n_own;
    D.n_local = K->n;
    D.send_counts.assign(send_counts, send_counts + P);
    D.recv_counts.assign(recv_counts, recv_counts + P);
    D.send_off.assign(P + 1, 0);
    D.recv_off.assign(P + 1, 0);
    for (int q = 0; q < P; ++q) {
        D.send_off[q + 1] = D.send_off[q] + D.send_counts[q];
        D.recv_off[q + 1] = D.recv_off[q] + D.recv_counts[q];
    }
    D.n_send = D.send_off[P];
    if (D.n_send && send_idx) D.h_send_idx.assign(send_idx, send_idx + D.n_send);
    if (D.recv_off[P] != K->n - n_own) return DDA_ERR_ARG;   // halo rows = received rows
    if (D.n_send && !send_idx) return DDA_ERR_ARG;
    const size_t nl6 = 6 * (size_t)K->n, no6 = 6 * (size_t)n_own;
    D.G_spmv = grid_of((const void*)k_spmv_own, 6);
    D.G_vec = grid_of((const void*)k_update_own, 8);
    D.G_spmv2 = grid_of((const void*)k_spmv_own2, 3);
    {   // no more CTAs than ten-row groups of own rows
        const int need = (n_own + 10 * WPB - 1) / (10 * WPB);
        if (D.G_spmv2 > need) D.G_spmv2 = need > 0 ? need : 1;
    }
    D.G_a3 = grid_of((const void*)k_v3_a, 3);
    {
        const int need = (n_own + 10 * WPB - 1) / (10 * WPB);
        if (D.G_a3 > need) D.G_a3 = need > 0 ? need : 1;
    }
    int Gm = D.G_spmv > D.G_vec ? D.G_spmv : D.G_vec;
    if (D.G_spmv2 > Gm) Gm = D.G_spmv2;
    if (D.G_a3 > Gm) Gm = D.G_a3;
    // the buffers peers read in place under the IPC transport come from cudaMalloc (an IPC handle maps a
    // whole allocation); everything else from the stream-ordered pool
    D.ipc_alloc = c->ipc;
    auto xalloc = [&](void** ptr, size_t bytes) -> cudaError_t {
        return c->ipc ? cudaMalloc(ptr, bytes) : dev_alloc(ptr, bytes, st);
    };
    if (keep_send_idx) { D.send_idx = keep_send_idx; D.sendbuf = keep_sendbuf; }
    else {
        DDA_CK(xalloc(reinterpret_cast<void**>(&D.send_idx), (D.n_send + 1) * sizeof(int)));
        DDA_CK(xalloc(reinterpret_cast<void**>(&D.sendbuf), (24 * (size_t)D.n_send + 1) * sizeof(double)));
    }
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.x), nl6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.q), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.r), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.z), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.part), 4 * (size_t)Gm * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.ticket), sizeof(unsigned), st));
    DDA_CK(cudaMemsetAsync(D.ticket, 0, sizeof(unsigned), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.ticket2), sizeof(unsigned), st));
    DDA_CK(cudaMemsetAsync(D.ticket2, 0, sizeof(unsigned), st));
    {   // the interior rows for the halo overlap: the longest run of rows that read no halo row
        uint8_t* flag = nullptr;
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&flag), (size_t)n_own + 1, st));
        k_boundary_rows<<<(n_own + 255) / 256, 256, 0, st>>>(n_own, K->row_ptr, K->col_idx, K->low_ptr, K->low_row,
                                                            flag);
        DDA_LAUNCHED();
        std::vector<uint8_t> hf(n_own);
        DDA_CK(cudaMemcpyAsync(hf.data(), flag, n_own, cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        dev_free_on(flag, st);
        int best_lo = 0, best_len = 0;
        for (int i = 0; i < n_own;) {
            if (hf[i]) { ++i; continue; }
            int j = i;
            while (j < n_own && !hf[j]) ++j;
            if (j - i > best_len) { best_len = j - i; best_lo = i; }
            i = j;
        }
        D.ilo = best_lo;
        D.ihi = best_lo + best_len;
    }
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.scal), 16 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.red), 8 * sizeof(double), st));
    {
        size_t ds = sizeof(DState) > sizeof(SState) ? sizeof(DState) : sizeof(SState);
        if (sizeof(S4) > ds) ds = sizeof(S4);
        DDA_CK(dev_alloc(&D.dst, ds, st));
    }
    if (keep_rt) { D.rt = keep_rt; D.pA = keep_pA; D.pB = keep_pB; }
    else {
        DDA_CK(xalloc(reinterpret_cast<void**>(&D.rt), nl6 * sizeof(double)));
        DDA_CK(xalloc(reinterpret_cast<void**>(&D.pA), nl6 * sizeof(double)));
        DDA_CK(xalloc(reinterpret_cast<void**>(&D.pB), nl6 * sizeof(double)));
    }
    DDA_CK(cudaMemsetAsync(D.rt, 0, nl6 * sizeof(double), st));
    DDA_CK(cudaMemsetAsync(D.pA, 0, nl6 * sizeof(double), st));
    DDA_CK(cudaMemsetAsync(D.pB, 0, nl6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.scal_ptrs), (P + 1) * sizeof(double*), st));
    if (D.n_send)
        DDA_CK(cudaMemcpyAsync(D.send_idx, send_idx, D.n_send * sizeof(int), cudaMemcpyHostToDevice, st));
    DDA_CK(cudaMemsetAsync(D.x, 0, nl6 * sizeof(double), st));
    if (!c->loopback && !c->ipc && P > 1) {   // the peers' send counts must equal this rank's receive counts
        int* cnt = nullptr;
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&cnt), (size_t)P * (P + 1) * sizeof(int), st));
        DDA_CK(cudaMemcpyAsync(cnt, send_counts, P * sizeof(int), cudaMemcpyHostToDevice, st));
        const ncclResult_t r = ncclAllGather(cnt, cnt + P, P, ncclInt32, c->nccl, st);
        std::vector<int> all((size_t)P * P);
        if (r == ncclSuccess)
            DDA_CK(cudaMemcpyAsync(all.data(), cnt + P, (size_t)P * P * sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        dev_free_on(cnt, st);
        if (r != ncclSuccess) return DDA_ERR_NCCL;
        for (int q = 0; q < P; ++q)
            if (all[(size_t)q * P + c->rank] != recv_counts[q]) return DDA_ERR_ARG;
    }
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

namespace {

double* part_buf(DistPart& D, int which) {
    switch (which) {
        case 1: return D.rt;
        case 2: return D.pA;
        case 3: return D.pB;
        case 4: return D.K->sfac;
        default: return D.x;
    }
}

// fill rows n_own.. of buffer `which` (w doubles per row) of every local partition from the peers' own rows
// IPC transport collective (one thread): publish nv values to this rank's slot of the epoch's set,
// announce the arrival on rank 0's counter, wait for all P ranks (bounded), sum the P slots in rank
// order into out (nv = 0: a barrier).  epoch is the 1-based arrival epoch this call completes.
#define DDA_TRY_S(expr)                    \
    do {                                   \
        dda_status_t _s = (expr);          \
        if (_s != DDA_OK) return _s;       \
    } while (0)
dda_status_t ipc_coll(dda_comm* c, const double* in, int nv, double* out, cudaStream_t st) {
    if (nv > kSlotStride) return DDA_ERR_ARG;
    c->epoch += 1;
    k_ipc_coll<<<1, 1, 0, st>>>(in, nv, out, c->sync, c->nranks, c->rank, c->epoch);
    DDA_LAUNCHED();
    return DDA_OK;
}

dda_status_t halo_exchange_w(dda_comm* c, cudaStream_t st, int which, int w) {
    const int P = c->nranks;
    for (DistPart& D : c->parts) {
        if (D.n_send) {
            const int items = w * D.n_send;
            k_pack_w<<<(items + 255) / 256 < 1024 ? (items + 255) / 256 : 1024, 256, 0, st>>>(
                D.n_send, w, D.send_idx, part_buf(D, which), D.sendbuf);
            DDA_LAUNCHED();
        }
    }
    if (c->ipc) {   // packed by every rank -> each copies its halo from the peers' send buffers -> released
        if (!c->ipc_ready) return DDA_ERR_ARG;
        DistPart& D = c->parts[0];
        DDA_TRY_S(ipc_coll(c, nullptr, 0, nullptr, st));
        for (int q = 0; q < P; ++q) {
            if (q == c->rank || !D.recv_counts[q]) continue;
            const IpcPeer& Q = c->peers[q];
            DDA_CK(cudaMemcpyAsync(part_buf(D, which) + (size_t)w * ((size_t)D.n_own + D.recv_off[q]),
                                   Q.sendbuf + (size_t)w * Q.send_off[c->rank],
                                   (size_t)w * sizeof(double) * D.recv_counts[q], cudaMemcpyDeviceToDevice, st));
        }
        DDA_TRY_S(ipc_coll(c, nullptr, 0, nullptr, st));
        return DDA_OK;
    }
    if (c->loopback) {
        for (int p = 0; p < P; ++p)
            for (int q = 0; q < P; ++q) {
                if (p == q) continue;
                DistPart& S = c->parts[p];
                DistPart& R = c->parts[q];
                if (S.send_counts[q] != R.recv_counts[p]) return DDA_ERR_ARG;
                if (!S.send_counts[q]) continue;
                DDA_CK(cudaMemcpyAsync(part_buf(R, which) + (size_t)w * ((size_t)R.n_own + R.recv_off[p]),
                                       S.sendbuf + (size_t)w * S.send_off[q], (size_t)w * sizeof(double) * S.send_counts[q],
                                       cudaMemcpyDeviceToDevice, st));
            }
        return DDA_OK;
    }
    DistPart& D = c->parts[0];
    double* dst = part_buf(D, which);
    DDA_NCCL(ncclGroupStart());
    for (int q = 0; q < P; ++q) {
        if (q == c->rank) continue;
        if (D.send_counts[q])
            DDA_NCCL(ncclSend(D.sendbuf + (size_t)w * D.send_off[q], (size_t)w * D.send_counts[q], ncclDouble, q,
                              c->nccl, st));
        if (D.recv_counts[q])
            DDA_NCCL(ncclRecv(dst + (size_t)w * ((size_t)D.n_own + D.recv_off[q]), (size_t)w * D.recv_counts[q],
                              ncclDouble, q, c->nccl, st));
    }
    DDA_NCCL(ncclGroupEnd());
    return DDA_OK;
}

// fill x[n_own:] of every local partition from the peers' own rows
dda_status_t halo_exchange(dda_comm* c, cudaStream_t st) { return halo_exchange_w(c, st, 0, 6); }

// sum of the nv scalars D.scal[0..nv) over all partitions / ranks, to the host
dda_status_t allreduce_host(dda_comm* c, int nv, double* out, cudaStream_t st) {
    for (int k = 0; k < nv; ++k) out[k] = 0.0;
    if (c->loopback) {
        std::vector<double> tmp(nv * c->parts.size());
        for (size_t p = 0; p < c->parts.size(); ++p)
            DDA_CK(cudaMemcpyAsync(tmp.data() + p * nv, c->parts[p].scal, nv * sizeof(double), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        for (size_t p = 0; p < c->parts.size(); ++p)
            for (int k = 0; k < nv; ++k) out[k] += tmp[p * nv + k];
        return DDA_OK;
    }
    DistPart& D = c->parts[0];
    if (c->ipc) DDA_TRY_S(ipc_coll(c, D.scal, nv, D.scal, st));
    else if (c->nranks > 1) DDA_NCCL(ncclAllReduce(D.scal, D.scal, nv, ncclDouble, ncclSum, c->nccl, st));
    DDA_CK(cudaMemcpyAsync(out, D.scal, nv * sizeof(double), cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

// the sum over all partitions / ranks of D.scal[off .. off+nv), to the host; D.scal is not modified
// (the NCCL sum goes to D.red)
dda_status_t allreduce_host_at(dda_comm* c, int off, int nv, double* out, cudaStream_t st) {
    for (int k = 0; k < nv; ++k) out[k] = 0.0;
    if (c->loopback) {
        std::vector<double> tmp(nv * c->parts.size());
        for (size_t p = 0; p < c->parts.size(); ++p)
            DDA_CK(cudaMemcpyAsync(tmp.data() + p * nv, c->parts[p].scal + off, nv * sizeof(double),
                                   cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        for (size_t p = 0; p < c->parts.size(); ++p)
            for (int k = 0; k < nv; ++k) out[k] += tmp[p * nv + k];
        return DDA_OK;
    }
    DistPart& D = c->parts[0];
    if (c->ipc) DDA_TRY_S(ipc_coll(c, D.scal + off, nv, D.red, st));
    else if (c->nranks > 1) DDA_NCCL(ncclAllReduce(D.scal + off, D.red, nv, ncclDouble, ncclSum, c->nccl, st));
    else DDA_CK(cudaMemcpyAsync(D.red, D.scal + off, nv * sizeof(double), cudaMemcpyDeviceToDevice, st));
    DDA_CK(cudaMemcpyAsync(out, D.red, nv * sizeof(double), cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

// v2: D.red[0..nv) = the sum over all partitions / ranks of D.scal[0..nv), on the device
dda_status_t allreduce_dev(dda_comm* c, int nv, cudaStream_t st) {
    if (c->loopback) {
        for (DistPart& D : c->parts) {
            k_sum_loopback<<<1, 32, 0, st>>>(D.scal_ptrs, (int)c->parts.size(), nv, D.red);
            DDA_LAUNCHED();
        }
        return DDA_OK;
    }
    DistPart& D = c->parts[0];
    if (c->ipc) return ipc_coll(c, D.scal, nv, D.red, st);
    if (c->nranks > 1) DDA_NCCL(ncclAllReduce(D.scal, D.red, nv, ncclDouble, ncclSum, c->nccl, st));
    else DDA_CK(cudaMemcpyAsync(D.red, D.scal, nv * sizeof(double), cudaMemcpyDeviceToDevice, st));
    return DDA_OK;
}

BsrView own_view(const DistPart& D) {
    BsrView A = view_of(D.K);
    A.n = D.n_own;
    return A;
}

dda_status_t spmv_parts(dda_comm* c, bool dot, cudaStream_t st) {
    for (DistPart& D : c->parts) {
        k_spmv_own<<<D.G_spmv, DDA_THREADS, 0, st>>>(own_view(D), D.x, D.q, D.part, dot ? 1 : 0);
        DDA_LAUNCHED();
        if (dot) {
            k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_spmv, 1, D.scal);
            DDA_LAUNCHED();
        }
    }
    return DDA_OK;
}

}  // namespace

#define DDA_TRY(expr)                      \
    do {                                   \
        dda_status_t _s = (expr);          \
        if (_s != DDA_OK) return _s;       \
    } while (0)

extern "C" dda_status_t dda_spmv_dist(dda_comm_t c, const double* const* x_own, double* const* y_own, void* stream) {
    DDA_NVTX("dda_spmv_dist");
    if (!c || !x_own || !y_own) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        if (!D.K) return DDA_ERR_ARG;
        DDA_CK(cudaMemcpyAsync(D.x, x_own[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
    }
    DDA_TRY(halo_exchange(c, st));
    DDA_TRY(spmv_parts(c, false, st));
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        DDA_CK(cudaMemcpyAsync(y_own[p], D.q, 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
    }
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

namespace {

BsrView own_view_sc(const DistPart& D) {
    BsrView A = view_of(D.K);
    A.n = D.n_own;
    A.upper = D.K->sc_upper;
    return A;
}

// v3 solve (BJ, scaled engine per partition): fills d, *status, *it; *zero = F was 0 (d = 0 set)
dda_status_t dist_scaled_solve(dda_comm* c, const double* const* F, const double* const* d0, double* const* d,
                               double tol, int32_t maxit, dda_status_t* status, int* it, bool* zero,
                               double* bnorm_out, cudaStream_t st) {
    *zero = false;
    *it = 0;
    // S_j of the halo rows from their owners, then the scaled blocks S_i V_ij S_j^T of every local block
    DDA_TRY(halo_exchange_w(c, st, 4, kDinv));
    for (DistPart& D : c->parts) {
        D.K->scaled_valid = false;
        DDA_TRY(scaled_setup(D.K, st));
    }
    const bool have_d0 = d0 != nullptr;
    if (have_d0) {                                          // q = K d0 over own rows (unscaled)
        for (size_t p = 0; p < c->parts.size(); ++p) {
            DistPart& D = c->parts[p];
            if (d0[p]) DDA_CK(cudaMemcpyAsync(D.x, d0[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
            else DDA_CK(cudaMemsetAsync(D.x, 0, 6 * sizeof(double) * D.n_own, st));
        }
        DDA_TRY(halo_exchange(c, st));
        DDA_TRY(spmv_parts(c, false, st));
    }
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        k_v3_init<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[p], have_d0 ? D.q : nullptr, have_d0 ? d0[p] : nullptr,
                                                   d[p], D.K->sfac, D.K->lfac, D.rt, D.pA, D.part);
        DDA_LAUNCHED();
        k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 3, D.scal);
        DDA_LAUNCHED();
    }
    double s3[3];
    DDA_TRY(allreduce_host(c, 3, s3, st));
    const double FF = s3[0], bnorm = std::sqrt(FF), rr = s3[1], rho = s3[2];
    *bnorm_out = bnorm;
    if (FF == 0.0) {                                        // reading Z2
        for (size_t p = 0; p < c->parts.size(); ++p)
            DDA_CK(cudaMemsetAsync(d[p], 0, 6 * sizeof(double) * c->parts[p].n_own, st));
        DDA_CK(cudaStreamSynchronize(st));
        *zero = true;
        *status = DDA_OK;
        return DDA_OK;
    }
    SState h{};
    h.rho = rho; h.bnorm = bnorm; h.tol = tol; h.rr = rr; h.maxit = maxit;
    h.status = DDA_ERR_NO_CONVERGENCE;
    if (std::sqrt(rr) <= tol * bnorm) { h.status = DDA_OK; h.done = 1; }
    else if (!(rho > 0.0) || !std::isfinite(rho)) { h.status = DDA_ERR_BREAKDOWN; h.done = 1; }
    else if (maxit <= 0) { h.done = 1; }
    std::vector<const double*> sp;
    for (DistPart& D : c->parts) sp.push_back(D.scal);
    for (DistPart& D : c->parts) {
        DDA_CK(cudaMemcpyAsync(D.dst, &h, sizeof h, cudaMemcpyHostToDevice, st));
        if (c->loopback)
            DDA_CK(cudaMemcpyAsync(D.scal_ptrs, sp.data(), sp.size() * sizeof(double*), cudaMemcpyHostToDevice, st));
    }
    int chunk = 8;
    if (const char* e = getenv("DDA_DIST_CHUNK")) chunk = atoi(e) > 0 ? atoi(e) : 8;
    SState out = h;
    for (int k = 0; !h.done && k < maxit; k += chunk) {
        for (int ci = 0; ci < chunk && k + ci < maxit; ++ci) {
            const int j = k + ci;
            DDA_TRY(halo_exchange_w(c, st, 1, 6));                               // r~
            if (j >= 1) DDA_TRY(halo_exchange_w(c, st, ((j - 1) & 1) ? 3 : 2, 6));   // p_{j-1}
            for (size_t p = 0; p < c->parts.size(); ++p) {
                DistPart& D = c->parts[p];
                SState* ds = reinterpret_cast<SState*>(D.dst);
                k_v3_a<<<D.G_a3, DDA_THREADS, 0, st>>>(own_view_sc(D), D.rt, D.pA, D.pB, D.q, d[p], ds, D.part);
                DDA_LAUNCHED();
                k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_a3, 1, D.scal);
                DDA_LAUNCHED();
            }
            DDA_TRY(allreduce_dev(c, 1, st));
            for (DistPart& D : c->parts) {
                SState* ds = reinterpret_cast<SState*>(D.dst);
                k_v3_alpha<<<1, 1, 0, st>>>(ds, D.red);
                DDA_LAUNCHED();
                k_v3_b<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, D.rt, D.q, D.K->bj_w, ds, D.part);
                DDA_LAUNCHED();
                k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 2, D.scal);
                DDA_LAUNCHED();
            }
            DDA_TRY(allreduce_dev(c, 2, st));
            for (DistPart& D : c->parts) {
                SState* ds = reinterpret_cast<SState*>(D.dst);
                k_v3_rho<<<1, 1, 0, st>>>(ds, D.red);
                DDA_LAUNCHED();
                k_v3_c<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, D.rt, D.K->lfac, ds, D.part);
                DDA_LAUNCHED();
                k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 1, D.scal);
                DDA_LAUNCHED();
            }
            DDA_TRY(allreduce_dev(c, 1, st));
            for (DistPart& D : c->parts) {
                k_v3_check<<<1, 1, 0, st>>>(reinterpret_cast<SState*>(D.dst), D.red);
                DDA_LAUNCHED();
            }
        }
        DDA_CK(cudaMemcpyAsync(&out, c->parts[0].dst, sizeof out, cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        if (out.done) break;
    }
    for (size_t p = 0; p < c->parts.size(); ++p) {          // d = S^T x (after the pending x update)
        DistPart& D = c->parts[p];
        k_v3_final<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, d[p], D.pA, D.pB, D.K->sfac,
                                                    reinterpret_cast<SState*>(D.dst));
        DDA_LAUNCHED();
    }
    DDA_CK(cudaMemcpyAsync(&out, c->parts[0].dst, sizeof out, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    *status = (dda_status_t)out.status;
    *it = out.iters;
    return DDA_OK;
}

// v4 solve (BJ, scaled engine per partition, one halo + one allreduce per iteration)
dda_status_t dist_v4_solve(dda_comm* c, const double* const* F, const double* const* d0, double* const* d,
                           double tol, int32_t maxit, dda_status_t* status, int* it, bool* zero, double* bnorm_out,
                           int* checks_out, cudaStream_t st) {
    *zero = false;
    *it = 0;
    DDA_TRY(halo_exchange_w(c, st, 4, kDinv));             // S_j of the halo rows
    for (DistPart& D : c->parts) {
        D.K->scaled_valid = false;
        DDA_TRY(scaled_setup(D.K, st));
    }
    const bool have_d0 = d0 != nullptr;
    if (have_d0) {                                          // q = K d0 over own rows (unscaled)
        for (size_t p = 0; p < c->parts.size(); ++p) {
            DistPart& D = c->parts[p];
            if (d0[p]) DDA_CK(cudaMemcpyAsync(D.x, d0[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
            else DDA_CK(cudaMemsetAsync(D.x, 0, 6 * sizeof(double) * D.n_own, st));
        }
        DDA_TRY(halo_exchange(c, st));
        DDA_TRY(spmv_parts(c, false, st));
    }
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        k_v4_init<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[p], have_d0 ? D.q : nullptr,
                                                   have_d0 ? d0[p] : nullptr, d[p], D.K->sfac, D.K->lfac,
                                                   D.K->bj_w, D.rt, D.pA, D.part, D.ticket, D.scal);
        DDA_LAUNCHED();
    }
    double s4[4];
    DDA_TRY(allreduce_host_at(c, 8, 4, s4, st));
    const double rho = s4[0], rr = s4[2], FF = s4[3], bnorm = std::sqrt(FF);
    *bnorm_out = bnorm;
    if (FF == 0.0) {                                        // reading Z2
        for (size_t p = 0; p < c->parts.size(); ++p)
            DDA_CK(cudaMemsetAsync(d[p], 0, 6 * sizeof(double) * c->parts[p].n_own, st));
        DDA_CK(cudaStreamSynchronize(st));
        *zero = true;
        *status = DDA_OK;
        return DDA_OK;
    }
    S4 h{};
    h.rho = rho; h.bnorm = bnorm; h.tol = tol; h.rr = rr; h.maxit = maxit;
    h.status = DDA_ERR_NO_CONVERGENCE;
    if (std::sqrt(rr) <= tol * bnorm) { h.status = DDA_OK; h.done = 1; }
    else if (!(rho > 0.0) || !std::isfinite(rho)) { h.status = DDA_ERR_BREAKDOWN; h.done = 1; }
    else if (maxit <= 0) { h.done = 1; }
    std::vector<const double*> sp;
    for (DistPart& D : c->parts) sp.push_back(D.scal);
    for (DistPart& D : c->parts) {
        DDA_CK(cudaMemcpyAsync(D.dst, &h, sizeof h, cudaMemcpyHostToDevice, st));
        if (c->loopback)
            DDA_CK(cudaMemcpyAsync(D.scal_ptrs, sp.data(), sp.size() * sizeof(double*), cudaMemcpyHostToDevice, st));
    }
    // v5 (loopback, default there; DDA_DIST_VERSION=4 keeps the copies): halo by peer loads, one-shot
    // allreduce inside B.  The pointer tables follow the exchange plan: halo row recv_off[q] + t of p
    // is q's own row send_idx_q[send_off_q[p] + t]
    const char* dve = getenv("DDA_DIST_VERSION");
    const bool peer = c->loopback && !(dve && dve[0] == '4');
    if (peer) {
        const int P = (int)c->parts.size();
        for (int p = 0; p < P; ++p) {
            DistPart& D = c->parts[p];
            const int nh = D.n_local - D.n_own;
            if (!D.hsrc) DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.hsrc), (nh + 1) * sizeof(double*), st));
            std::vector<const double*> tab(nh + 1, nullptr);
            for (int q = 0; q < P; ++q) {
                if (q == p) continue;
                const DistPart& S = c->parts[q];
                for (int t = 0; t < D.recv_counts[q]; ++t)
                    tab[D.recv_off[q] + t] = S.pA + 6 * (size_t)S.h_send_idx[S.send_off[p] + t];
            }
            DDA_CK(cudaMemcpyAsync(D.hsrc, tab.data(), (nh + 1) * sizeof(double*), cudaMemcpyHostToDevice, st));
        }
        DDA_CK(cudaStreamSynchronize(st));                  // the host table must outlive the copies
    }
    // halo overlap (v4 with halo copies or NCCL; DDA_DIST_OVERLAP=0 disables): phase A of the interior
    // rows runs while the halo is in flight on a second stream
    const char* ove = getenv("DDA_DIST_OVERLAP");
    bool overlap = !peer && !(ove && ove[0] == '0');
    if (overlap) {
        bool any_halo = false;
        for (DistPart& D : c->parts) any_halo = any_halo || D.n_local > D.n_own;
        overlap = any_halo;
    }
    cudaStream_t cs = nullptr;
    cudaEvent_t ev_a = nullptr, ev_b = nullptr;
    struct StreamGuard {
        cudaStream_t& s; cudaEvent_t& a; cudaEvent_t& b;
        ~StreamGuard() { if (a) cudaEventDestroy(a); if (b) cudaEventDestroy(b); if (s) cudaStreamDestroy(s); }
    } sguard{cs, ev_a, ev_b};
    if (overlap) {
        DDA_CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
        DDA_CK(cudaEventCreateWithFlags(&ev_a, cudaEventDisableTiming));
        DDA_CK(cudaEventCreateWithFlags(&ev_b, cudaEventDisableTiming));
    }
    int chunk = 8;
    if (const char* e = getenv("DDA_DIST_CHUNK")) chunk = atoi(e) > 0 ? atoi(e) : 8;
    S4 out = h;
    // DDA_DIST_PROFILE=1: CUDA events between the four steps of every iteration (a diagnostic solve:
    // the comm / compute split of bench.py's N > 1 line), summed per step
    const char* pe = getenv("DDA_DIST_PROFILE");
    const bool prof = pe && pe[0] == '1';
    std::vector<cudaEvent_t> ev;
    std::vector<int> ev_step;
    for (int q = 0; q < 4; ++q) c->prof_ms[q] = 0.0;
    auto mark = [&](int step) {
        if (!prof) return;
        cudaEvent_t e;
        cudaEventCreate(&e);
        cudaEventRecord(e, st);
        ev.push_back(e);
        ev_step.push_back(step);
    };
    // passes: maxit iterations + the pass that finds the final test + the rare exact-test retries
    for (int k = 0; !out.done && k < maxit + 64; k += chunk) {
        for (int ci = 0; ci < chunk; ++ci) {
            mark(-1);
            if (overlap) {
                // the halo of p_k on the comm stream while the interior rows (which read no halo row)
                // run phase A; then the boundary rows
                DDA_CK(cudaEventRecord(ev_a, st));
                DDA_CK(cudaStreamWaitEvent(cs, ev_a, 0));
                DDA_TRY(halo_exchange_w(c, cs, 2, 6));
                DDA_CK(cudaEventRecord(ev_b, cs));
                for (DistPart& D : c->parts) {
                    const XLdC xf{D.pA};
                    k_v4_a<XLdC><<<D.G_a3, DDA_THREADS, 0, st>>>(own_view_sc(D), D.rt, xf, D.q,
                                                                 reinterpret_cast<S4*>(D.dst), D.part, D.ticket2,
                                                                 D.scal, D.ilo, D.ihi, D.ihi, 0, 1);
                    DDA_LAUNCHED();
                }
                mark(0);
                DDA_CK(cudaStreamWaitEvent(st, ev_b, 0));
                for (DistPart& D : c->parts) {
                    const XLdC xf{D.pA};
                    const int gap = D.ihi - D.ilo;
                    k_v4_a<XLdC><<<D.G_a3, DDA_THREADS, 0, st>>>(own_view_sc(D), D.rt, xf, D.q,
                                                                 reinterpret_cast<S4*>(D.dst), D.part, D.ticket,
                                                                 D.scal, 0, D.n_own - gap, D.ilo, gap, 2);
                    DDA_LAUNCHED();
                }
            } else {
                if (!peer) DDA_TRY(halo_exchange_w(c, st, 2, 6));                    // p_k
                mark(0);
                for (DistPart& D : c->parts) {
                    if (peer) {
                        const XPeer xf{D.pA, D.hsrc, D.n_own};
                        k_v4_a<XPeer><<<D.G_a3, DDA_THREADS, 0, st>>>(own_view_sc(D), D.rt, xf, D.q,
                                                                      reinterpret_cast<S4*>(D.dst), D.part,
                                                                      D.ticket, D.scal, 0, -1, 0, 0, 0);
                    } else {
                        const XLdC xf{D.pA};
                        k_v4_a<XLdC><<<D.G_a3, DDA_THREADS, 0, st>>>(own_view_sc(D), D.rt, xf, D.q,
                                                                     reinterpret_cast<S4*>(D.dst), D.part,
                                                                     D.ticket, D.scal, 0, -1, 0, 0, 0);
                    }
                    DDA_LAUNCHED();
                }
            }
            mark(1);
            if (!peer) DDA_TRY(allreduce_dev(c, 6, st));
            mark(2);
            for (size_t p = 0; p < c->parts.size(); ++p) {
                DistPart& D = c->parts[p];
                k_v4_b<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, D.rt, D.pA, D.q, d[p], D.K->bj_w, D.K->lfac,
                                                        reinterpret_cast<S4*>(D.dst), D.red,
                                                        peer ? D.scal_ptrs : nullptr, (int)c->parts.size(),
                                                        D.part, D.ticket, D.scal);
                DDA_LAUNCHED();
            }
            mark(3);
        }
        DDA_CK(cudaMemcpyAsync(&out, c->parts[0].dst, sizeof out, cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        if (prof) {
            for (size_t q = 1; q < ev.size(); ++q) {
                if (ev_step[q] < 0) continue;
                float ms = 0.0f;
                cudaEventElapsedTime(&ms, ev[q - 1], ev[q]);
                c->prof_ms[ev_step[q]] += ms;
            }
            for (cudaEvent_t e : ev) cudaEventDestroy(e);
            ev.clear();
            ev_step.clear();
        }
    }
    for (size_t p = 0; p < c->parts.size(); ++p) {          // d = S^T x
        DistPart& D = c->parts[p];
        k_v4_final<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, d[p], D.K->sfac);
        DDA_LAUNCHED();
    }
    DDA_CK(cudaStreamSynchronize(st));
    *status = out.done ? (dda_status_t)out.status : DDA_ERR_NO_CONVERGENCE;
    *it = out.iters;
    *checks_out = out.checks;
    return DDA_OK;
}

// v6 solve (loopback, BJ): the whole iteration loop in one cooperative launch (k_dist_loop).  *ran is
// false (nothing done) when the cooperative grid cannot give every partition a CTA: the caller runs v5.
dda_status_t dist_v6_solve(dda_comm* c, const double* const* F, const double* const* d0, double* const* d,
                           double tol, int32_t maxit, dda_status_t* status, int* it, bool* zero, double* bnorm_out,
                           int* checks_out, bool* ran, cudaStream_t st, bool per_rank = false) {
    *zero = false;
    *it = 0;
    *ran = false;
    const int P = (int)c->parts.size();
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, per_rank ? (const void*)k_rank_loop : (const void*)k_dist_loop,
                                                  DDA_THREADS, 0);
    if (per_sm > 3) per_sm = 3;
    const int G = device_sms() * per_sm;
    if (per_sm < 1 || G < P || P > kDPMax) return DDA_OK;   // not co-resident / too many: the caller runs v5
    *ran = true;
    DDA_TRY(halo_exchange_w(c, st, 4, kDinv));             // S_j of the halo rows
    for (DistPart& D : c->parts) {
        D.K->scaled_valid = false;
        DDA_TRY(scaled_setup(D.K, st));
    }
    const bool have_d0 = d0 != nullptr;
    if (have_d0) {                                          // q = K d0 over own rows (unscaled)
        for (int p = 0; p < P; ++p) {
            DistPart& D = c->parts[p];
            if (d0[p]) DDA_CK(cudaMemcpyAsync(D.x, d0[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
            else DDA_CK(cudaMemsetAsync(D.x, 0, 6 * sizeof(double) * D.n_own, st));
        }
        DDA_TRY(halo_exchange(c, st));
        DDA_TRY(spmv_parts(c, false, st));
    }
    for (int p = 0; p < P; ++p) {
        DistPart& D = c->parts[p];
        k_v4_init<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[p], have_d0 ? D.q : nullptr,
                                                   have_d0 ? d0[p] : nullptr, d[p], D.K->sfac, D.K->lfac,
                                                   D.K->bj_w, D.rt, D.pA, D.part, D.ticket, D.scal);
        DDA_LAUNCHED();
    }
    double s4[4];
    DDA_TRY(allreduce_host_at(c, 8, 4, s4, st));
    const double rho = s4[0], rr = s4[2], FF = s4[3], bnorm = std::sqrt(FF);
    *bnorm_out = bnorm;
    *checks_out = 0;
    if (FF == 0.0) {                                        // reading Z2
        for (int p = 0; p < P; ++p) DDA_CK(cudaMemsetAsync(d[p], 0, 6 * sizeof(double) * c->parts[p].n_own, st));
        DDA_CK(cudaStreamSynchronize(st));
        *zero = true;
        *status = DDA_OK;
        return DDA_OK;
    }
    // decided at setup (converged at the start, breakdown, maxit = 0): no loop, d = S^T x0 below
    int pre = -1;
    if (std::sqrt(rr) <= tol * bnorm) pre = DDA_OK;
    else if (!(rho > 0.0) || !std::isfinite(rho)) pre = DDA_ERR_BREAKDOWN;
    else if (maxit <= 0) pre = DDA_ERR_NO_CONVERGENCE;
    // device tables: the partitions, their halo maps (owner partition, owner's local row), the CTA split
    std::vector<DPart> h(P);
    int64_t tot = 0;
    for (DistPart& D : c->parts) tot += D.n_own;
    int64_t cum = 0;
    int prev = 0;
    std::vector<int2> hm;
    std::vector<size_t> hoff(P + 1, 0);
    for (int p = 0; p < P; ++p) {
        DistPart& D = c->parts[p];
        const int nh = D.n_local - D.n_own;
        hoff[p] = hm.size();
        hm.resize(hm.size() + nh);
        for (int q = 0; q < P; ++q) {
            if (q == p) continue;
            const DistPart& S = c->parts[q];
            for (int t = 0; t < D.recv_counts[q]; ++t)
                hm[hoff[p] + D.recv_off[q] + t] = make_int2(q, S.h_send_idx[S.send_off[p] + t]);
        }
        cum += D.n_own;
        int c1 = (int)((G * cum) / (tot > 0 ? tot : 1));
        if (c1 < prev + 1) c1 = prev + 1;                   // at least one CTA per partition ...
        if (c1 > G - (P - 1 - p)) c1 = G - (P - 1 - p);     // ... and one left for each later one
        if (p == P - 1) c1 = G;
        h[p].A = own_view_sc(D);
        h[p].rt = D.rt; h[p].p0 = D.pA; h[p].p1 = D.pB; h[p].q = D.q; h[p].x = d[p];
        h[p].w = D.K->bj_w; h[p].lfac = D.K->lfac;
        h[p].n_own = D.n_own; h[p].c0 = prev; h[p].c1 = c1;
        prev = c1;
    }
    hoff[P] = hm.size();
    const size_t tb = sizeof(DPart) * P, hb = sizeof(int2) * (hm.size() + 1), pb = sizeof(double) * 4 * (size_t)G;
    char* ws = nullptr;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&ws), tb + hb + pb + sizeof(DPState) + 256, st));
    struct WsFree { char* b; cudaStream_t s; ~WsFree() { cudaStreamSynchronize(s); dev_free_on(b, s); } } wf{ws, st};
    DPart* dparts = reinterpret_cast<DPart*>(ws);
    int2* dh = reinterpret_cast<int2*>(ws + ((tb + 15) / 16) * 16);
    double* dpart = reinterpret_cast<double*>(ws + ((tb + 15) / 16) * 16 + ((hb + 15) / 16) * 16);
    DPState* dst = reinterpret_cast<DPState*>(dpart + 4 * (size_t)G);
    for (int p = 0; p < P; ++p) h[p].hmap = dh + hoff[p];
    DDA_CK(cudaMemcpyAsync(dparts, h.data(), tb, cudaMemcpyHostToDevice, st));
    if (!hm.empty()) DDA_CK(cudaMemcpyAsync(dh, hm.data(), sizeof(int2) * hm.size(), cudaMemcpyHostToDevice, st));
    DPArgs a{};
    for (int p = 0; p < P; ++p) a.parts[p] = h[p];
    a.gparts = dparts;
    a.P = P;
    a.part = dpart;
    a.st = dst;
    a.rho0 = rho;
    a.thr = tol * bnorm;
    a.maxit = maxit;
    DPState z{};
    DDA_CK(cudaMemsetAsync(dst, 0, sizeof(DPState), st));   // (struct padding: every byte defined)
    if (pre < 0 && per_rank) {
        // v7: one cooperative kernel per rank, each on its own stream, all resident together (the grid is
        // split evenly); the ranks meet only through the slot sets and the arrival counter
        const int Gr = G / P;
        const size_t pb_r = sizeof(double) * 4 * (size_t)Gr, sb = sizeof(double) * kRankSets * kSlotStride * (size_t)P;
        char* rw = nullptr;
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&rw), P * (pb_r + sizeof(DPState) + 64) + sb + 64, st));
        struct RwFree { char* b; cudaStream_t s; ~RwFree() { cudaStreamSynchronize(s); dev_free_on(b, s); } } rf{rw, st};
        double* slots = reinterpret_cast<double*>(rw);
        unsigned* arrive = reinterpret_cast<unsigned*>(rw + sb);
        int* err = reinterpret_cast<int*>(rw + sb + 16);
        char* base = rw + sb + 64;
        DDA_CK(cudaMemsetAsync(rw + sb, 0, 64, st));
        std::vector<cudaStream_t> rs(P, nullptr);
        cudaEvent_t ev0 = nullptr;
        struct RsFree {
            std::vector<cudaStream_t>& v; cudaEvent_t& e;
            ~RsFree() { for (cudaStream_t x : v) if (x) cudaStreamDestroy(x); if (e) cudaEventDestroy(e); }
        } rsf{rs, ev0};
        DDA_CK(cudaEventCreateWithFlags(&ev0, cudaEventDisableTiming));
        DDA_CK(cudaEventRecord(ev0, st));
        std::vector<RArgs> ra(P);
        for (int p = 0; p < P; ++p) {
            DDA_CK(cudaStreamCreateWithFlags(&rs[p], cudaStreamNonBlocking));
            DDA_CK(cudaStreamWaitEvent(rs[p], ev0, 0));
            char* mine = base + (size_t)p * (pb_r + sizeof(DPState) + 64);
            DPState* rst = reinterpret_cast<DPState*>(mine + pb_r);
            DDA_CK(cudaMemsetAsync(rst, 0, sizeof(DPState), rs[p]));
            ra[p] = RArgs{dparts, P, p, reinterpret_cast<double*>(mine), slots, arrive, 0u, rst, err, rho, tol * bnorm, maxit};
        }
        for (int p = 0; p < P; ++p) {       // all ranks are launched before any is waited on
            void* args[] = {&ra[p]};
            DDA_CK(cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(k_rank_loop), dim3(Gr),
                                               dim3(DDA_THREADS), args, 0, rs[p]));
            note_launch();
        }
        for (int p = 0; p < P; ++p) {
            cudaEvent_t e;
            DDA_CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
            DDA_CK(cudaEventRecord(e, rs[p]));
            DDA_CK(cudaStreamWaitEvent(st, e, 0));
            cudaEventDestroy(e);
        }
        DDA_CK(cudaMemcpyAsync(dst, ra[0].st, sizeof(DPState), cudaMemcpyDeviceToDevice, st));   // rank 0's copy
        int herr = 0;
        DDA_CK(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        if (herr) return DDA_ERR_CUDA;      // a rank waited past the bound on the others
    } else if (pre < 0) {
        void* args[] = {&a};
        DDA_CK(cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(k_dist_loop), dim3(G), dim3(DDA_THREADS),
                                           args, 0, st));
        note_launch();
    } else {
        z.status = pre;
        z.rr = rr;
        DDA_CK(cudaMemcpyAsync(dst, &z, sizeof z, cudaMemcpyHostToDevice, st));
    }
    DPState out{};
    DDA_CK(cudaMemcpyAsync(&out, dst, sizeof out, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    for (int p = 0; p < P; ++p) {
        DistPart& D = c->parts[p];
        k_dp_final<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, d[p], ((out.k - 1) & 1) ? D.pB : D.pA, dst, D.K->sfac);
        DDA_LAUNCHED();
    }
    DDA_CK(cudaStreamSynchronize(st));
    *status = (dda_status_t)out.status;
    *it = out.iters;
    *checks_out = out.checks;
    return DDA_OK;
}

// ---- IPC transport solve: this process's rank of the v7 loop (one persistent kernel per rank); the
// peers' r~ / p rows are read through their IPC-mapped arrays, every reduction through rank 0's
// mapped counter and slot sets
dda_status_t dist_ipc_solve(dda_comm* c, const double* const* F, const double* const* d0, double* const* d,
                            double tol, int32_t maxit, dda_status_t* status, int* it, bool* zero, double* bnorm_out,
                            int* checks_out, cudaStream_t st) {
    *zero = false;
    *it = 0;
    const int P = c->nranks, me = c->rank;
    DistPart& D = c->parts[0];
    if (!c->ipc_ready || !D.K || P > kDPMax) return DDA_ERR_ARG;
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_rank_loop, DDA_THREADS, 0);
    if (per_sm > 3) per_sm = 3;
    if (per_sm < 1) return DDA_ERR_CUDA;
    const int G = device_sms() * per_sm;
    DDA_TRY_S(halo_exchange_w(c, st, 4, kDinv));           // S_j of the halo rows
    D.K->scaled_valid = false;
    DDA_TRY_S(scaled_setup(D.K, st));
    const bool have_d0 = d0 != nullptr && d0[0] != nullptr;
    if (have_d0) {
        DDA_CK(cudaMemcpyAsync(D.x, d0[0], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
        DDA_TRY_S(halo_exchange(c, st));
        DDA_TRY_S(spmv_parts(c, false, st));
    }
    k_v4_init<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[0], have_d0 ? D.q : nullptr, have_d0 ? d0[0] : nullptr,
                                               d[0], D.K->sfac, D.K->lfac, D.K->bj_w, D.rt, D.pA, D.part, D.ticket,
                                               D.scal);
    DDA_LAUNCHED();
    double s4[4];
    DDA_TRY_S(allreduce_host_at(c, 8, 4, s4, st));
    const double rho = s4[0], rr = s4[2], FF = s4[3], bnorm = std::sqrt(FF);
    *bnorm_out = bnorm;
    *checks_out = 0;
    if (FF == 0.0) {                                        // reading Z2
        DDA_CK(cudaMemsetAsync(d[0], 0, 6 * sizeof(double) * D.n_own, st));
        DDA_CK(cudaStreamSynchronize(st));
        *zero = true;
        *status = DDA_OK;
        return DDA_OK;
    }
    int pre = -1;
    if (std::sqrt(rr) <= tol * bnorm) pre = DDA_OK;
    else if (!(rho > 0.0) || !std::isfinite(rho)) pre = DDA_ERR_BREAKDOWN;
    else if (maxit <= 0) pre = DDA_ERR_NO_CONVERGENCE;
    // the rank table: own entry complete; a peer's entry carries its mapped r~ / p arrays
    std::vector<DPart> h(P);
    for (int q = 0; q < P; ++q) {
        h[q] = DPart{};
        h[q].rt = c->peers[q].rt;
        h[q].p0 = c->peers[q].pA;
        h[q].p1 = c->peers[q].pB;
    }
    const int nh = D.n_local - D.n_own;
    const size_t tb = sizeof(DPart) * P, hb = sizeof(int2) * (nh + 1), pb = sizeof(double) * 4 * (size_t)G;
    char* ws = nullptr;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&ws), tb + hb + pb + 2 * sizeof(DPState) + 256, st));
    struct WsFree { char* b; cudaStream_t s; ~WsFree() { cudaStreamSynchronize(s); dev_free_on(b, s); } } wf{ws, st};
    DPart* dparts = reinterpret_cast<DPart*>(ws);
    int2* dh = reinterpret_cast<int2*>(ws + ((tb + 15) / 16) * 16);
    double* dpart = reinterpret_cast<double*>(ws + ((tb + 15) / 16) * 16 + ((hb + 15) / 16) * 16);
    DPState* dst = reinterpret_cast<DPState*>(dpart + 4 * (size_t)G);
    for (int q = 0; q < P; ++q) {       // halo rows from q -> (q, q's local row) read from q's send list
        if (q == me || !D.recv_counts[q]) continue;
        const IpcPeer& Q = c->peers[q];
        k_ipc_hmap<<<(D.recv_counts[q] + 255) / 256, 256, 0, st>>>(D.recv_counts[q], q, Q.send_idx + Q.send_off[me],
                                                                     dh + D.recv_off[q]);
        DDA_LAUNCHED();
    }
    h[me].A = own_view_sc(D);
    h[me].rt = D.rt; h[me].p0 = D.pA; h[me].p1 = D.pB; h[me].q = D.q; h[me].x = d[0];
    h[me].w = D.K->bj_w; h[me].lfac = D.K->lfac; h[me].hmap = dh;
    h[me].n_own = D.n_own; h[me].c0 = 0; h[me].c1 = G;
    DDA_CK(cudaMemcpyAsync(dparts, h.data(), tb, cudaMemcpyHostToDevice, st));
    DDA_CK(cudaMemsetAsync(dst, 0, sizeof(DPState), st));
    int* err = reinterpret_cast<int*>(c->sync + 16);
    if (pre < 0) {
        RArgs ra{dparts, P, me, dpart, reinterpret_cast<double*>(c->sync + kSyncHdr),
                 reinterpret_cast<unsigned*>(c->sync), c->epoch, dst, err, rho, tol * bnorm, maxit};
        void* args[] = {&ra};
        DDA_CK(cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(k_rank_loop), dim3(G), dim3(DDA_THREADS),
                                           args, 0, st));
        note_launch();
    } else {
        DPState z{};
        z.status = pre;
        z.rr = rr;
        z.epoch_end = c->epoch;
        DDA_CK(cudaMemcpyAsync(dst, &z, sizeof z, cudaMemcpyHostToDevice, st));
    }
    DPState out{};
    int herr = 0;
    DDA_CK(cudaMemcpyAsync(&out, dst, sizeof out, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    if (herr) return DDA_ERR_CUDA;                        // a wait on the other ranks hit its bound
    c->epoch = out.epoch_end;
    k_dp_final<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, d[0], ((out.k - 1) & 1) ? D.pB : D.pA, dst, D.K->sfac);
    DDA_LAUNCHED();
    DDA_CK(cudaStreamSynchronize(st));
    *status = (dda_status_t)out.status;
    *it = out.iters;
    *checks_out = out.checks;
    return DDA_OK;
}

}  // namespace

extern "C" dda_status_t dda_pcg_solve_dist(dda_comm_t c, const double* const* F, const double* const* d0,
                                           double* const* d, double tol, int32_t maxit, dda_precond_t pc,
                                           int32_t* iters, double* rel_res, void* stream) {
    DDA_NVTX("dda_pcg_solve_dist");
    if (iters) *iters = 0;
    if (rel_res) *rel_res = 0.0;
    if (!c || !F || !d || !(tol > 0.0) || maxit < 0) return DDA_ERR_ARG;
    if (pc != DDA_PC_BJ && pc != DDA_PC_NONE) return DDA_ERR_ARG;   // SSOR-AI / ILU(0): single GPU only
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const int use_bj = pc == DDA_PC_BJ;
    for (DistPart& D : c->parts)
        if (!D.K) return DDA_ERR_ARG;
    if (use_bj)
        for (DistPart& D : c->parts) DDA_TRY(bj_setup_rows(D.K, D.n_own, st, nullptr));
    // v4 (default for block-Jacobi): one halo + one allreduce per iteration; DDA_DIST_VERSION=3 selects
    // v3 (two halos, three allreduces); DDA_DIST_SCALED=0 selects the unscaled v2
    const char* dse = getenv("DDA_DIST_SCALED");
    const char* dve = getenv("DDA_DIST_VERSION");
    const bool v3 = dve && dve[0] == '3';
    if (use_bj && !(dse && dse[0] == '0')) {
        dda_status_t status = DDA_ERR_NO_CONVERGENCE;
        int it = 0, checks = 0;
        bool zero = false;
        double bnorm = 0.0;
        // v6 (loopback default): one persistent kernel for every partition; DDA_DIST_VERSION=5 / 4 / 3
        // select the per-iteration launches (v5: peer-load halo, v4: halo copies, v3)
        bool ran = false;
        if (c->ipc && !(dve && (dve[0] == '3' || dve[0] == '4'))) {   // the IPC transport: v7, this process's rank
            DDA_TRY(dist_ipc_solve(c, F, d0, d, tol, maxit, &status, &it, &zero, &bnorm, &checks, st));
            ran = true;
        } else if (c->loopback && !(dve && (dve[0] == '3' || dve[0] == '4' || dve[0] == '5')))
            DDA_TRY(dist_v6_solve(c, F, d0, d, tol, maxit, &status, &it, &zero, &bnorm, &checks, &ran, st,
                                  dve && dve[0] == '7'));
        if (ran) {
        } else if (v3) DDA_TRY(dist_scaled_solve(c, F, d0, d, tol, maxit, &status, &it, &zero, &bnorm, st));
        else DDA_TRY(dist_v4_solve(c, F, d0, d, tol, maxit, &status, &it, &zero, &bnorm, &checks, st));
        c->last_checks = checks;
        if (zero) return DDA_OK;
        // true residual ||F - K d|| / ||F|| (unscaled, over the partitions)
        for (size_t p = 0; p < c->parts.size(); ++p) {
            DistPart& D = c->parts[p];
            DDA_CK(cudaMemcpyAsync(D.x, d[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
        }
        DDA_TRY(halo_exchange(c, st));
        DDA_TRY(spmv_parts(c, false, st));
        for (size_t p = 0; p < c->parts.size(); ++p) {
            DistPart& D = c->parts[p];
            k_resid_own<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[p], D.q, D.part);
            DDA_LAUNCHED();
            k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 1, D.scal);
            DDA_LAUNCHED();
        }
        double res;
        DDA_TRY(allreduce_host(c, 1, &res, st));
        if (iters) *iters = it;
        if (rel_res) *rel_res = std::sqrt(res) / bnorm;
        return status;
    }
    const bool have_d0 = d0 != nullptr;
    // ---- setup: r = F - K d0
    if (have_d0) {
        for (size_t p = 0; p < c->parts.size(); ++p) {
            DistPart& D = c->parts[p];
            if (d0[p]) DDA_CK(cudaMemcpyAsync(D.x, d0[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
            else DDA_CK(cudaMemsetAsync(D.x, 0, 6 * sizeof(double) * D.n_own, st));
        }
        DDA_TRY(halo_exchange(c, st));
        DDA_TRY(spmv_parts(c, false, st));
    }
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        const double* dd0 = have_d0 ? d0[p] : nullptr;
        if (have_d0 && !dd0) DDA_CK(cudaMemsetAsync(d[p], 0, 6 * sizeof(double) * D.n_own, st));
        k_init_own<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, D.K->dinv, use_bj, F[p], dd0, d[p],
                                                    have_d0 ? D.q : nullptr, D.r, D.z, D.x, D.part);
        DDA_LAUNCHED();
        k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 3, D.scal);
        DDA_LAUNCHED();
    }
    double s3[3];
    DDA_TRY(allreduce_host(c, 3, s3, st));
    const double FF = s3[0], bnorm = std::sqrt(FF);
    double rr = s3[1], rho = s3[2];
    dda_status_t status = DDA_ERR_NO_CONVERGENCE;
    int it = 0;
    if (FF == 0.0) {
        for (size_t p = 0; p < c->parts.size(); ++p)
            DDA_CK(cudaMemsetAsync(d[p], 0, 6 * sizeof(double) * c->parts[p].n_own, st));
        DDA_CK(cudaStreamSynchronize(st));
        return DDA_OK;
    }
    if (std::sqrt(rr) <= tol * bnorm) {
        status = DDA_OK;
    } else if (!(rho > 0.0) || !std::isfinite(rho)) {
        status = DDA_ERR_BREAKDOWN;
    } else if (maxit > 0) {
        // v2: device-side scalars; the host reads the state once per chunk of iterations
        DState h{};
        h.rho = rho; h.bnorm = bnorm; h.tol = tol; h.rr = rr; h.maxit = maxit;
        h.status = DDA_ERR_NO_CONVERGENCE;
        std::vector<const double*> sp;
        for (DistPart& D : c->parts) sp.push_back(D.scal);
        for (DistPart& D : c->parts) {
            DDA_CK(cudaMemcpyAsync(D.dst, &h, sizeof h, cudaMemcpyHostToDevice, st));
            if (c->loopback)
                DDA_CK(cudaMemcpyAsync(D.scal_ptrs, sp.data(), sp.size() * sizeof(double*), cudaMemcpyHostToDevice,
                                       st));
        }
        int chunk = 8;
        if (const char* e = getenv("DDA_DIST_CHUNK")) chunk = atoi(e) > 0 ? atoi(e) : 8;
        DState out{};
        for (int k = 0; k < maxit; k += chunk) {
            for (int ci = 0; ci < chunk && k + ci < maxit; ++ci) {
                DDA_TRY(halo_exchange(c, st));                    // p halo
                for (DistPart& D : c->parts) {                    // q = K p, p^T q
                    k_spmv_own2<<<D.G_spmv2, DDA_THREADS, 0, st>>>(own_view(D), D.x, D.q, D.part,
                                                                  reinterpret_cast<DState*>(D.dst));
                    DDA_LAUNCHED();
                    k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_spmv2, 1, D.scal);
                    DDA_LAUNCHED();
                }
                DDA_TRY(allreduce_dev(c, 1, st));
                for (DistPart& D : c->parts) {
                    k_scal_alpha<<<1, 1, 0, st>>>(reinterpret_cast<DState*>(D.dst), D.red);
                    DDA_LAUNCHED();
                    k_update_own2<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, D.K->dinv, use_bj,
                                                                   reinterpret_cast<DState*>(D.dst), D.x, D.q,
                                                                   d[&D - &c->parts[0]], D.r, D.z, D.part);
                    DDA_LAUNCHED();
                    k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 2, D.scal);
                    DDA_LAUNCHED();
                }
                DDA_TRY(allreduce_dev(c, 2, st));
                for (DistPart& D : c->parts) {
                    k_scal_beta<<<1, 1, 0, st>>>(reinterpret_cast<DState*>(D.dst), D.red);
                    DDA_LAUNCHED();
                    k_pupd_own2<<<2 * device_sms(), 256, 0, st>>>(6 * D.n_own, reinterpret_cast<DState*>(D.dst),
                                                                  D.z, D.x);
                    DDA_LAUNCHED();
                }
            }
            DDA_CK(cudaMemcpyAsync(&out, c->parts[0].dst, sizeof out, cudaMemcpyDeviceToHost, st));
            DDA_CK(cudaStreamSynchronize(st));
            if (out.done) break;
        }
        status = (dda_status_t)out.status;
        it = out.iters;
    }
    // ---- true residual
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        DDA_CK(cudaMemcpyAsync(D.x, d[p], 6 * sizeof(double) * D.n_own, cudaMemcpyDeviceToDevice, st));
    }
    DDA_TRY(halo_exchange(c, st));
    DDA_TRY(spmv_parts(c, false, st));
    for (size_t p = 0; p < c->parts.size(); ++p) {
        DistPart& D = c->parts[p];
        k_resid_own<<<D.G_vec, DDA_THREADS, 0, st>>>(D.n_own, F[p], D.q, D.part);
        DDA_LAUNCHED();
        k_sum_parts<<<1, DDA_THREADS, 0, st>>>(D.part, D.G_vec, 1, D.scal);
        DDA_LAUNCHED();
    }
    double res;
    DDA_TRY(allreduce_host(c, 1, &res, st));
    if (iters) *iters = it;
    if (rel_res) *rel_res = std::sqrt(res) / bnorm;
    return status;
}

// internal hook: the step times of the last profiled v4 solve (DDA_DIST_PROFILE=1): halo, A, allreduce, B
extern "C" int dda__dist_profile(dda_comm_t c, double* ms4) {
    if (!c || !ms4) return -1;
    for (int q = 0; q < 4; ++q) ms4[q] = c->prof_ms[q];
    return c->last_checks;
}
