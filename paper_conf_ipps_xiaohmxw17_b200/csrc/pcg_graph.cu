// A5/A6 — PCG (§IV.A; textbook PCG, Saad Alg. 9.1) as a
// CUDA graph with a device-side while loop (conditional node): the iteration
// runs entirely on the GPU, each phase is its own kernel with its own register
// budget and occupancy, and the host reads the outcome once.
//
//   prelude  (stream)   [q = K d0] -> init vectors (+ FF, rr, rho) -> [SSOR halves (rho)]
//   while (cond) {      k_g_spmv:   p^(k) = z + beta p^(k-1) on the fly (k > 0), q = K p^(k); sigma -> alpha
//                       k_g_update: d += alpha p; r -= alpha q; z = D^{-1} r; rr, rz -> convergence test
//                                   ||r|| <= tol ||F||, beta, cudaGraphSetConditional
//                       [k_g_ssor_lower, k_g_ssor_upper]  (SSOR-AI: z = M^{-1} r; rz -> beta, condition) }
//   epilogue (stream)   q = K d -> ||F - q|| / ||F||, status
//
// Scalar reductions use a deterministic "last CTA done" scheme: every CTA
// writes its partial, the last CTA to arrive (atomic ticket) sums all partials
// in one fixed order with the whole CTA and publishes the scalars (and the loop
// condition) in a device State — no separate check kernel, no per-CTA
// re-summing.  Per-call pointers (F, d0, d) and tol / maxit / omega travel
// in a device CallArgs block, so one instantiated graph per (matrix, precond)
// is reused across solves.
#include <cooperative_groups.h>

#include <cmath>
#include <cstdlib>

#include "ilu_dev.cuh"
#include "spmv_col.cuh"

namespace cg = cooperative_groups;

namespace dda {
namespace {

constexpr int WPB = DDA_THREADS / 32;
// largest power of two <= DDA_THREADS (the CTA tree sums; the library is built with 256)
constexpr int kTreeP2 = DDA_THREADS >= 512 ? 512 : DDA_THREADS >= 256 ? 256 : DDA_THREADS >= 128 ? 128 : 64;

struct CallArgs {
    const double* F;
    const double* d0;
    double* d;
    double tol;
    double omega;
    int maxit;
};

struct State {
    double rho, beta, alpha, FF, bnorm, rr, rel;
    int k, done, status, iters, zero_d;
    unsigned ticket;
    // scaled engine: lam = a lower bound of min_i lambda_min(D_i); maybe = the exact stopping test
    // is due (k_s_check); pend_rz = the new rho waiting for it
    double lam, pend_rz;
    int maybe;
    int checks;   // exact stopping tests evaluated (k_s_check passes that did work)
    int pend;   // scaled engine: x += alpha p of the last k_s_update still to apply (k_s_final)
};

struct GArgs {           // constant for a (matrix, preconditioner): baked into the graph
    BsrView A;
    const double* dinv;
    double *r, *z, *p0, *p1, *q, *t, *w;
    double* part;        // [8][Gmax] CTA partials
    int Gmax;
    int pc;
    State* st;
    const CallArgs* ca;
    int* out;            // iters, status, rel (double at +8 bytes)
    const double* ilu_up;
    const double* ilu_inv;
    int* ilu_flags_f;    // forward / backward ready flags and their row counters
    int* ilu_flags_b;
    int* ilu_counters;
    const int* ilu_order;
    const double* su;    // scaled BJ engine: S_i V_ij S_j^T (tiled, upper pattern)
    const double* lfac;  // packed lower L_i (D_i = L_i L_i^T)
    const double* sfac;  // packed lower S_i = L_i^{-1}
    const unsigned long long* dinv_fmax;   // bits of max_i ||D_i^{-1}||_F (bj_setup)
    const double* bj_w;  // [n] w_i <= lambda_min(D_i) (bj_setup): sum_i w_i |r~_i|^2 <= |L r~|^2
    int use_cond;        // 0 only for the internal phase-timing hook (kernels launched outside the graph)
    unsigned long long* trace;   // k_sp_loop timeline [iter][cta][4] (%globaltimer), null = off (internal hook)
    int trace_iters;
    double* hist;        // residual history [hist_cap][2] (dda_pcg_set_history), null = off
    int hist_cap;
    // k_sp_loop push form (phase_a_lr): entries, their offsets per upper block, per-step counters
    double2* lr;
    const int* lr_off;
    unsigned* lr_cnt;
    int lr_discard;
    int lr_sync;
};

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ void set_cond(const GArgs& a, cudaGraphConditionalHandle h, unsigned v) {
    if (a.use_cond) cudaGraphSetConditional(h, v);
}

__device__ __forceinline__ bool loop_done(const State* st) { return *reinterpret_cast<volatile const int*>(&st->done); }

// Programmatic dependent launch: wait for the previous kernel of the loop body
// (all its memory operations visible), then allow the next one to be launched
// and staged while this one runs.  No-ops when launched without the attribute.
__device__ __forceinline__ void pdl_enter() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// Deterministic grid reduction of NV values: CTA partials -> part[k*Gmax + blockIdx.x];
// returns true in the last CTA to finish, where tot[] then holds the fixed-order sums
// (every thread of that CTA sees them).
template <int NV>
__device__ __forceinline__ bool grid_reduce_last(const GArgs& a, double (&v)[NV], double (&tot)[NV]) {
    __shared__ double red[NV][DDA_THREADS];
    __shared__ bool last;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = warp_sum(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[k][wib] = v[k];
    }
    cta_barrier_na();
    if (threadIdx.x == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int w = 0; w < WPB; ++w) s += red[k][w];
            a.part[k * a.Gmax + blockIdx.x] = s;
        }
        __threadfence();
        const unsigned t = atomicAdd(&a.st->ticket, 1u);
        last = (t == gridDim.x - 1);
    }
    cta_barrier_na();
    if (!last) return false;
    __threadfence();
    const int G = gridDim.x;
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        double s = 0.0;
        for (int j = threadIdx.x; j < G; j += DDA_THREADS) s += __ldcg(a.part + k * a.Gmax + j);
        red[k][threadIdx.x] = s;
    }
    cta_barrier_na();
    if (kTreeP2 < DDA_THREADS) {                          // fold a non-power-of-two CTA first
        if ((int)threadIdx.x < DDA_THREADS - kTreeP2) {
#pragma unroll
            for (int k = 0; k < NV; ++k) red[k][threadIdx.x] += red[k][threadIdx.x + kTreeP2];
        }
        cta_barrier_na();
    }
    for (int h = kTreeP2 / 2; h > 0; h >>= 1) {           // fixed-shape tree
        if (threadIdx.x < h) {
#pragma unroll
            for (int k = 0; k < NV; ++k) red[k][threadIdx.x] += red[k][threadIdx.x + h];
        }
        cta_barrier_na();
    }
#pragma unroll
    for (int k = 0; k < NV; ++k) tot[k] = red[k][0];
    if (threadIdx.x == 0) a.st->ticket = 0u;
    return true;
}

struct XPlain {
    const double* __restrict__ x;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};
// x = z + beta p_old, formed on the fly for every gathered neighbour (the fused p-update).  Formed
// at load time (Raw = the combined pair): keeping z and p raw until the block is consumed costs 8
// registers and measured slower (250 vs 240 us at 1M blocks, scaled engine).
struct XFusedG {
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

// ---------------------------------------------------------------- loop body

// phase A: p^(k) (fused p-update for k > 0), q = K p^(k); last CTA: sigma = p^T q, alpha = rho / sigma.
// SC (scaled BJ engine): the matrix is S K S^T, whose diagonal blocks are the identity, so the
// off-diagonal product (SPMV_OFFDIAG over the scaled blocks) is completed by q_i += p_i and the
// "preconditioned residual" gathered for p is the scaled residual itself (a.z == a.r).
template <int MINB, bool SC, int V = 4>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_g_spmv(const GArgs a, cudaGraphConditionalHandle h) {
    pdl_enter();
    if (loop_done(a.st)) {                 // finished at setup: leave the loop
        if (blockIdx.x == 0 && threadIdx.x == 0) set_cond(a, h, 0);
        return;
    }
    constexpr int MODE = SC ? SPMV_OFFDIAG : SPMV_FULL;
    BsrView A = a.A;
    if (SC) A.upper = a.su;
    const int k = a.st->k;
    const double beta = a.st->beta;
    const int lane = threadIdx.x & 31;
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    double acc = 0.0;
    // column-pair map (spmv_col.cuh): 10 rows per warp, lane C holds pair C of its group's row
    if (k == 0) {
        const XPlain xf{a.p0};
        for_rows_c<MODE, V>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                if (SC) { y0 += pv.x; y1 += pv.y; }
                *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
                acc += pv.x * y0 + pv.y * y1;
            }
        });
    } else {
        double* pnew = (k & 1) ? a.p1 : a.p0;
        const double* pold = (k & 1) ? a.p0 : a.p1;
        const XFusedG xf{SC ? a.r : a.z, pold, beta};
        // scaled engine: the solution update of the previous iteration, x += alpha_{k-1} p_{k-1}, is
        // applied here for the own rows (p_{k-1} is read here anyway), not in k_s_update
        const double alpha_prev = a.st->alpha;
        double* x = a.ca->d;
        for_rows_c<MODE, V>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                if (SC) {
                    y0 += pv.x;
                    y1 += pv.y;
                    const double2 po = __ldg(reinterpret_cast<const double2*>(pold + o));
                    const double2 xo = *reinterpret_cast<const double2*>(x + o);
                    *reinterpret_cast<double2*>(x + o) = make_double2(xo.x + alpha_prev * po.x,
                                                                      xo.y + alpha_prev * po.y);
                }
                *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
                *reinterpret_cast<double2*>(pnew + o) = pv;
                acc += pv.x * y0 + pv.y * y1;
            }
        });
    }
    double v[1] = {acc}, tot[1];
    if (grid_reduce_last<1>(a, v, tot) && threadIdx.x == 0) {
        State* st = a.st;
        st->pend = 0;                                      // the pending solution update is applied
        const double sigma = tot[0];
        if (!(sigma > 0.0) || !isfinite(sigma)) {          // reading Z19: d stays the last iterate
            st->status = DDA_ERR_BREAKDOWN;
            st->done = 1;
            set_cond(a, h, 0);
        } else {
            st->alpha = st->rho / sigma;
        }
    }
}

// last-CTA scalar step after r^T z is known: breakdown, beta, iteration cap, loop condition
__device__ __forceinline__ void finish_iteration(const GArgs& a, double rz, cudaGraphConditionalHandle h) {
    State* st = a.st;
    int done = 0;
    if (!(rz > 0.0) || !isfinite(rz)) {
        st->status = DDA_ERR_BREAKDOWN; done = 1;
    } else {
        st->beta = rz / st->rho;
        st->rho = rz;
        if (st->k + 1 >= a.ca->maxit) { st->status = DDA_ERR_NO_CONVERGENCE; done = 1; }
    }
    st->k = st->k + 1;
    st->done = done;
    set_cond(a, h, done ? 0 : 1);
}

// phase B: d += alpha p; r -= alpha q; z = D^{-1} r (BJ) / t = D^{-1} r (SSOR) / z = r;
// last CTA: rr, rz -> convergence test, (BJ / none) beta and the loop condition
__global__ void __launch_bounds__(DDA_THREADS) k_g_update(const GArgs a, cudaGraphConditionalHandle h) {
    pdl_enter();
    if (loop_done(a.st)) return;
    const int k = a.st->k;
    const double alpha = a.st->alpha;
    const double* pk = (k & 1) ? a.p1 : a.p0;
    double* d = a.ca->d;
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool use_dinv = (a.pc == DDA_PC_BJ || a.pc == DDA_PC_SSOR_AI);
    double rr = 0.0, rz = 0.0;
    // two 5-row groups per warp iteration, every load issued before any shuffle / arithmetic
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += 2 * W) {
        const Row5 RA = row5(grp, lane, n);
        const Row5 RB = row5(grp + W, lane, n);
        double pa = 0, da = 0, ra = 0, qa = 0, pb = 0, db = 0, rb = 0, qb = 0;
        if (RA.valid) { pa = pk[RA.idx]; da = d[RA.idx]; ra = a.r[RA.idx]; qa = a.q[RA.idx]; }
        if (RB.valid) { pb = pk[RB.idx]; db = d[RB.idx]; rb = a.r[RB.idx]; qb = a.q[RB.idx]; }
        DinvRow DA, DB;
        if (use_dinv) { DA = dinv_row(a.dinv, RA); DB = dinv_row(a.dinv, RB); }
        const double rva = RA.valid ? ra - alpha * qa : 0.0;
        const double rvb = RB.valid ? rb - alpha * qb : 0.0;
        if (RA.valid) { d[RA.idx] = da + alpha * pa; a.r[RA.idx] = rva; }
        if (RB.valid) { d[RB.idx] = db + alpha * pb; a.r[RB.idx] = rvb; }
        rr += rva * rva + rvb * rvb;
        const double tza = use_dinv ? dinv_row_apply(DA, rva, RA) : rva;
        const double tzb = use_dinv ? dinv_row_apply(DB, rvb, RB) : rvb;
        if (a.pc == DDA_PC_SSOR_AI) {
            if (RA.valid) a.t[RA.idx] = tza;
            if (RB.valid) a.t[RB.idx] = tzb;
        } else if (a.pc != DDA_PC_ILU0) {
            if (RA.valid) a.z[RA.idx] = tza;
            if (RB.valid) a.z[RB.idx] = tzb;
            rz += rva * tza + rvb * tzb;
        }
    }
    double v[2] = {rr, rz}, tot[2];
    if (grid_reduce_last<2>(a, v, tot) && threadIdx.x == 0) {
        State* st = a.st;
        st->rr = tot[0];
        st->iters = k + 1;
        if (sqrt(tot[0]) <= a.ca->tol * st->bnorm) {
            st->status = DDA_OK;
            st->k = k + 1;
            st->done = 1;
            set_cond(a, h, 0);
        } else if (a.pc != DDA_PC_SSOR_AI && a.pc != DDA_PC_ILU0) {
            finish_iteration(a, tot[1], h);
        }
    }
}

// SSOR-AI halves (INIT: at setup, also p0 = z and rho = r^T z)
template <bool INIT>
__global__ void __launch_bounds__(DDA_THREADS) k_g_ssor_lower(const GArgs a) {
    pdl_enter();
    if (!INIT && loop_done(a.st)) return;
    const int lane = threadIdx.x & 31;
    const double omega = a.ca->omega;
    for_rows<SPMV_LOWER_T>(a.A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, XPlain{a.t}, lane,
                           [&](int i, bool ok, double y0, double y1) {
                               ssor_lower_row(a.dinv, i, ok, y0, y1, a.r, omega, a.w, lane);
                           });
}

template <bool INIT>
__global__ void __launch_bounds__(DDA_THREADS) k_g_ssor_upper(const GArgs a, cudaGraphConditionalHandle h) {
    pdl_enter();
    if (loop_done(a.st)) return;   // at setup: done means converged / F = 0 already
    const int lane = threadIdx.x & 31;
    const double omega = a.ca->omega;
    double rz = 0.0;
    for_rows<SPMV_UPPER>(a.A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, XPlain{a.w}, lane,
                         [&](int i, bool ok, double y0, double y1) {
                             const double zz = ssor_upper_row(a.dinv, i, ok, y0, y1, a.w, omega, lane);
                             if (ok && q_of(lane) < 6) {
                                 const size_t idx = 6 * (size_t)i + q_of(lane);
                                 a.z[idx] = zz;
                                 if (INIT) a.p0[idx] = zz;
                                 rz += a.r[idx] * zz;
                             }
                         });
    double v[1] = {rz}, tot[1];
    if (grid_reduce_last<1>(a, v, tot) && threadIdx.x == 0) {
        if (INIT) {
            State* st = a.st;
            st->rho = tot[0];
            if (!(tot[0] > 0.0) || !isfinite(tot[0])) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; }
        } else {
            finish_iteration(a, tot[0], h);
        }
    }
}

// ILU(0) sweeps (sync-free, ilu.cu): y = t, yh = w scratch; z (and p0 at setup); rz -> beta / rho
template <bool INIT>
__global__ void __launch_bounds__(DDA_THREADS) k_g_ilu_fwd(const GArgs a) {
    if (loop_done(a.st)) return;
    ilu_forward_rows(a.A, a.ilu_up, a.ilu_inv, a.r, a.t, a.w, a.ilu_flags_f, a.ilu_counters, a.ilu_order);
}

template <bool INIT>
__global__ void __launch_bounds__(DDA_THREADS) k_g_ilu_bwd(const GArgs a, cudaGraphConditionalHandle h) {
    if (loop_done(a.st)) return;
    const double rz = ilu_backward_rows(a.A, a.ilu_up, a.ilu_inv, a.t, a.z, a.r, INIT ? a.p0 : nullptr,
                                        a.ilu_flags_b, a.ilu_counters + 1, a.ilu_order + a.A.n);
    double v[1] = {rz}, tot[1];
    if (grid_reduce_last<1>(a, v, tot) && threadIdx.x == 0) {
        if (INIT) {
            State* st = a.st;
            st->rho = tot[0];
            if (!(tot[0] > 0.0) || !isfinite(tot[0])) { st->status = DDA_ERR_BREAKDOWN; st->done = 1; }
        } else {
            finish_iteration(a, tot[0], h);
        }
    }
}

// ---------------------------------------------------------------- prelude / epilogue

__device__ __noinline__ void init_decide(const GArgs& a, const double (&tot)[3]);

// d = d0 (or 0), r = F - q (or F); BJ/none: z = p0 = M^{-1} r; SSOR: t = D^{-1} r;
// last CTA: FF, rr, rho and the setup decisions (F = 0, converged at start, breakdown, maxit = 0)
__global__ void __launch_bounds__(DDA_THREADS) k_g_init(const GArgs a) {
    const CallArgs* ca = a.ca;
    const double* d0 = ca->d0;
    double* d = ca->d;
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool use_dinv = (a.pc == DDA_PC_BJ || a.pc == DDA_PC_SSOR_AI);
    double FF = 0.0, rr = 0.0, rz = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0, fv = 0.0;
        if (R.valid) {
            fv = ca->F[R.idx];
            const double dv = d0 ? d0[R.idx] : 0.0;
            if (d != d0) d[R.idx] = dv;
            rv = d0 ? fv - a.q[R.idx] : fv;
            a.r[R.idx] = rv;
        }
        FF += fv * fv;
        rr += rv * rv;
        const double tz = use_dinv ? bj_lane(a.dinv, R, rv) : rv;
        if (R.valid) {
            if (a.pc == DDA_PC_SSOR_AI) {
                a.t[R.idx] = tz;
            } else if (a.pc != DDA_PC_ILU0) {
                a.z[R.idx] = tz;
                a.p0[R.idx] = tz;
                rz += rv * tz;
            }
        }
    }
    double v[3] = {FF, rr, rz}, tot[3];
    if (grid_reduce_last<3>(a, v, tot) && threadIdx.x == 0) init_decide(a, tot);
}

// setup decisions from (FF, rr, rho): F = 0, converged at start, breakdown, maxit = 0
__device__ __noinline__ void init_decide(const GArgs& a, const double (&tot)[3]) {
    const CallArgs* ca = a.ca;
    {
        State* st = a.st;
        st->FF = tot[0];
        st->bnorm = sqrt(tot[0]);
        st->rr = tot[1];
        st->rho = tot[2];
        st->beta = 0.0;
        st->alpha = 0.0;
        st->k = 0;
        st->iters = 0;
        st->rel = 0.0;
        st->zero_d = 0;
        st->done = 0;
        st->maybe = 0;
        st->checks = 0;
        st->pend = 0;
        st->pend_rz = 0.0;
        st->status = DDA_ERR_NO_CONVERGENCE;
        if (tot[0] == 0.0) {                                   // reading Z2
            st->zero_d = 1; st->status = DDA_OK; st->done = 1;
        } else if (sqrt(tot[1]) <= ca->tol * st->bnorm) {
            st->status = DDA_OK; st->done = 1;
        } else if (a.pc != DDA_PC_SSOR_AI && a.pc != DDA_PC_ILU0 && (!(tot[2] > 0.0) || !isfinite(tot[2]))) {
            st->status = DDA_ERR_BREAKDOWN; st->done = 1;
        } else if (ca->maxit <= 0) {
            st->status = DDA_ERR_NO_CONVERGENCE; st->done = 1;
        }
    }
}

// q = K x with x = d0 (prelude, D0 = true) or x = d (true residual; skipped when d = 0 by reading Z2)
template <bool D0>
__global__ void __launch_bounds__(DDA_THREADS, 3) k_g_spmv_x(const GArgs a) {
    if (!D0 && a.st->zero_d) return;
    const int lane = threadIdx.x & 31;
    const XPlain xf{D0 ? a.ca->d0 : a.ca->d};
    for_rows_c<SPMV_FULL, 5>(a.A, blockIdx.x * WPB + (threadIdx.x >> 5), gridDim.x * WPB, xf, lane,
                             [&](int i, bool ok, double y0, double y1) {
                                 if (ok)
                                     *reinterpret_cast<double2*>(a.q + 6 * (size_t)i + 2 * ccol_of(lane)) =
                                         make_double2(y0, y1);
                             });
}

// ||F - q||^2 (or d = 0 when F = 0); last CTA writes rel_res, iterations and status
__global__ void __launch_bounds__(DDA_THREADS) k_g_resid(const GArgs a) {
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool zero = a.st->zero_d;
    double acc = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) {
            if (zero) {
                a.ca->d[R.idx] = 0.0;
            } else {
                const double e = a.ca->F[R.idx] - a.q[R.idx];
                acc += e * e;
            }
        }
    }
    double v[1] = {acc}, tot[1];
    if (grid_reduce_last<1>(a, v, tot) && threadIdx.x == 0) {
        State* st = a.st;
        st->rel = zero ? 0.0 : sqrt(tot[0]) / st->bnorm;
        a.out[0] = st->iters;
        a.out[1] = st->status;
        *reinterpret_cast<double*>(a.out + 2) = st->rel;
        a.out[4] = st->checks;
        a.out[5] = 0;                                  // (padding of the host result struct: initcheck)
    }
}

// ---------------------------------------------------------------- scaled block-Jacobi engine
//
// Block-Jacobi PCG on K d = F (M = D = blockdiag(D_i), D_i = L_i L_i^T) is, in exact
// arithmetic, plain CG on the block-scaled system  Ks x = S F,  Ks = S K S^T,  S = blockdiag(L_i^{-1}),
// d = S^T x: every iterate maps one to one (r~ = S r, p~ = L^T p, z = S^T r~, rho = r^T z = |r~|^2,
// sigma = p^T K p = p~^T Ks p~), so alpha, beta and the iteration count are those of BJ-PCG.
// Ks has identity diagonal blocks, so the loop streams no D_i and no D_i^{-1} and writes no z:
// 1916 -> 1580 algorithmic bytes per block row and iteration.  The stopping test
// stays reading Z1 on the ORIGINAL residual, ||r|| = ||L r~||, from the packed L_i.

// row a of a packed lower-triangular block (M[a][c], zero for c > a)
__device__ __forceinline__ DinvRow tri_row(const double* __restrict__ M, const Row5& R) {
    const double* blk = M + (size_t)kDinv * (R.valid ? R.i : 0);
    DinvRow d;
#pragma unroll
    for (int c = 0; c < 6; ++c) d.v[c] = c <= R.a ? __ldg(blk + lo_off(R.a, c)) : 0.0;
    return d;
}
// row a of the transpose of a packed lower-triangular block (M[c][a], zero for c < a)
__device__ __forceinline__ DinvRow tri_col(const double* __restrict__ M, const Row5& R) {
    const double* blk = M + (size_t)kDinv * (R.valid ? R.i : 0);
    DinvRow d;
#pragma unroll
    for (int c = 0; c < 6; ++c) d.v[c] = c >= R.a ? __ldg(blk + lo_off(c, R.a)) : 0.0;
    return d;
}

// Vs_ij = S_i V_ij S_j^T for every stored upper block (one thread per block, in registers)
__global__ void __launch_bounds__(128) k_scale_upper(int64_t nnzb, const int32_t* __restrict__ urow,
                                                     const int32_t* __restrict__ col,
                                                     const double* __restrict__ upper,
                                                     const double* __restrict__ sfac, double* __restrict__ su) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < nnzb;
         u += (int64_t)gridDim.x * blockDim.x) {
        const double* V = upper + (size_t)kBlk * u;
        double A[6][6];
#pragma unroll
        for (int q = 0; q < 9; ++q) {
            const double4 v = ld_chunk(V + 4 * q);
            const int R = q / 3, C = q % 3;
            A[2 * R][2 * C] = v.x; A[2 * R][2 * C + 1] = v.y;
            A[2 * R + 1][2 * C] = v.z; A[2 * R + 1][2 * C + 1] = v.w;
        }
        const double* Si = sfac + (size_t)kDinv * __ldg(urow + u);
        const double* Sj = sfac + (size_t)kDinv * __ldg(col + u);
        double s[21];
#pragma unroll
        for (int k = 0; k < 21; ++k) s[k] = __ldg(Si + k);
        // A <- S_i A, rows in decreasing order (row r needs the original rows 0..r)
#pragma unroll
        for (int r = 5; r >= 0; --r)
#pragma unroll
            for (int c = 0; c < 6; ++c) {
                double t = 0.0;
#pragma unroll
                for (int k = 0; k <= r; ++k) t = fma(s[lo_off(r, k)], A[k][c], t);
                A[r][c] = t;
            }
#pragma unroll
        for (int k = 0; k < 21; ++k) s[k] = __ldg(Sj + k);
        // A <- A S_j^T: (A S^T)[r][c] = sum_{k<=c} A[r][k] S[c][k], columns in decreasing order
#pragma unroll
        for (int r = 0; r < 6; ++r)
#pragma unroll
            for (int c = 5; c >= 0; --c) {
                double t = 0.0;
#pragma unroll
                for (int k = 0; k <= c; ++k) t = fma(A[r][k], s[lo_off(c, k)], t);
                A[r][c] = t;
            }
        double* out = su + (size_t)kBlk * u;
#pragma unroll
        for (int q = 0; q < 9; ++q) {
            const int R = q / 3, C = q % 3;
            reinterpret_cast<double4*>(out)[q] = make_double4(A[2 * R][2 * C], A[2 * R][2 * C + 1],
                                                              A[2 * R + 1][2 * C], A[2 * R + 1][2 * C + 1]);
        }
    }
}

// prelude: r = F - K d0 (or F); r~ = S r -> r, p0; x = L^T d0 (or 0) -> d; FF, rr = |r|^2, rho = |r~|^2
__global__ void __launch_bounds__(DDA_THREADS) k_s_init(const GArgs a) {
    const CallArgs* ca = a.ca;
    const double* d0 = ca->d0;
    double* d = ca->d;
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double FF = 0.0, rr = 0.0, rz = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0, fv = 0.0, dv = 0.0;
        if (R.valid) {
            fv = ca->F[R.idx];
            if (d0) dv = d0[R.idx];
            rv = d0 ? fv - a.q[R.idx] : fv;
        }
        const DinvRow Srow = tri_row(a.sfac, R);
        FF += fv * fv;
        rr += rv * rv;
        // (lanes without a row, e.g. 30 and 31, shuffle a neighbour's values: mask them out)
        const double rt0 = dinv_row_apply(Srow, rv, R);
        const double rt = R.valid ? rt0 : 0.0;
        double xt = 0.0;
        if (d0) {                                  // uniform branch: every lane shuffles
            const DinvRow Lcol = tri_col(a.lfac, R);
            xt = dinv_row_apply(Lcol, dv, R);
        }
        if (R.valid) {
            a.r[R.idx] = rt;
            a.p0[R.idx] = rt;
            d[R.idx] = xt;
        }
        rz += rt * rt;
    }
    double v[3] = {FF, rr, rz}, tot[3];
    if (grid_reduce_last<3>(a, v, tot) && threadIdx.x == 0) {
        init_decide(a, tot);
        const double lam = 1.0 / __longlong_as_double((long long)*a.dinv_fmax);
        a.st->lam = (isfinite(lam) && lam > 0.0) ? lam : 0.0;   // 0: the exact test in every iteration
    }
}

// phase B: r~ -= alpha q~; rho' = |r~|^2 (x += alpha p~ is applied by the next SpMV or k_s_final).
// The stopping test (reading Z1) is on the ORIGINAL residual r = L r~, whose norm costs the packed
// L_i (192 B per row).  It is evaluated only when it can succeed: |L_i r~_i|^2 >= lambda_min(D_i)
// |r~_i|^2 >= w_i |r~_i|^2 (w_i = 1 / min(||D_i^{-1}||_F, ||D_i^{-1}||_inf), bj_setup), so while
// 0.999 sum_i w_i |r~_i|^2 > tol^2 ||F||^2 the iteration cannot have converged and L is not read
// (8 B of w per row instead of 192 B of L).  Otherwise k_s_check evaluates |L r~| exactly (the
// decision, the iteration count and the solution are those of the plain test).
__global__ void __launch_bounds__(DDA_THREADS, 4) k_s_update(const GArgs a, cudaGraphConditionalHandle h) {
    pdl_enter();
    if (loop_done(a.st)) return;
    const int k = a.st->k;
    const double alpha = a.st->alpha;
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rz = 0.0, lb = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += 2 * W) {
        const Row5 RA = row5(grp, lane, n);
        const Row5 RB = row5(grp + W, lane, n);
        double ra = 0, qa = 0, rb = 0, qb = 0, wa = 0, wb = 0;
        if (RA.valid) { ra = a.r[RA.idx]; qa = a.q[RA.idx]; wa = __ldg(a.bj_w + RA.i); }
        if (RB.valid) { rb = a.r[RB.idx]; qb = a.q[RB.idx]; wb = __ldg(a.bj_w + RB.i); }
        const double rva = RA.valid ? ra - alpha * qa : 0.0;
        const double rvb = RB.valid ? rb - alpha * qb : 0.0;
        if (RA.valid) a.r[RA.idx] = rva;
        if (RB.valid) a.r[RB.idx] = rvb;
        rz += rva * rva + rvb * rvb;
        lb += wa * (rva * rva) + wb * (rvb * rvb);
    }
    double v[2] = {rz, lb}, tot[2];
    if (grid_reduce_last<2>(a, v, tot) && threadIdx.x == 0) {
        State* st = a.st;
        st->pend = 1;                                       // x += alpha p_k: next SpMV or k_s_final
        const double rho1 = tot[0];
        if (a.hist && k < a.hist_cap) {
            a.hist[2 * (size_t)k] = rho1;
            a.hist[2 * (size_t)k + 1] = __longlong_as_double(0x7FF8000000000000ll);
        }
        st->iters = k + 1;
        const double thr = a.ca->tol * st->bnorm;
        if (rho1 == 0.0) {                                  // r~ = 0 exactly: r = L r~ = 0
            st->rr = 0.0;
            st->status = DDA_OK;
            st->k = k + 1;
            st->done = 1;
            set_cond(a, h, 0);
        } else if (isfinite(rho1) && !(0.999 * tot[1] > thr * thr)) {
            st->maybe = 1;                                  // k_s_check decides
            st->pend_rz = rho1;
        } else {
            finish_iteration(a, rho1, h);                   // cannot have converged (or breakdown)
        }
    }
}

// the exact stopping test |L r~| <= tol ||F|| when k_s_update flagged it; then beta / the loop
// condition as k_s_update would have set them
__global__ void __launch_bounds__(DDA_THREADS, 4) k_s_check(const GArgs a, cudaGraphConditionalHandle h) {
    pdl_enter();
    if (loop_done(a.st) || !*reinterpret_cast<volatile const int*>(&a.st->maybe)) return;
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double rr = 0.0;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double rv = R.valid ? a.r[R.idx] : 0.0;
        const DinvRow Lrow = tri_row(a.lfac, R);
        const double o0 = dinv_row_apply(Lrow, rv, R);
        const double o = R.valid ? o0 : 0.0;
        rr += o * o;
    }
    double v[1] = {rr}, tot[1];
    if (grid_reduce_last<1>(a, v, tot) && threadIdx.x == 0) {
        State* st = a.st;
        st->maybe = 0;
        st->checks += 1;
        st->rr = tot[0];
        if (a.hist && st->k < a.hist_cap) a.hist[2 * (size_t)st->k + 1] = tot[0];
        if (sqrt(tot[0]) <= a.ca->tol * st->bnorm) {
            st->status = DDA_OK;
            st->k = st->k + 1;
            st->done = 1;
            set_cond(a, h, 0);
        } else {
            finish_iteration(a, st->pend_rz, h);
        }
    }
}

// epilogue: the pending x += alpha p of the last iteration, then d = S^T x in place (before the
// true residual)
__global__ void __launch_bounds__(DDA_THREADS) k_s_final(const GArgs a) {
    if (a.st->zero_d) return;
    double* d = a.ca->d;
    const bool pend = a.st->pend;
    const double alpha = a.st->alpha;
    const double* pk = ((a.st->k - 1) & 1) ? a.p1 : a.p0;   // p of the last k_s_update (iteration k-1)
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    for (int grp = blockIdx.x * WPB + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double xv = R.valid ? (pend ? d[R.idx] + alpha * pk[R.idx] : d[R.idx]) : 0.0;
        const DinvRow Scol = tri_col(a.sfac, R);
        const double dv = dinv_row_apply(Scol, xv, R);
        if (R.valid) d[R.idx] = dv;
    }
}

// ---------------------------------------------------------------- scaled engine, persistent loop
//
// The same iteration as the graph loop above (k_g_spmv<SC> -> k_s_update -> [k_s_check]) with the
// kernel boundaries replaced by grid barriers: ONE cooperative launch runs every iteration.  At 1M
// blocks the graph loop spends ~45 us per iteration (of 323) between its kernels (drain / fill of
// three grids, the while-loop back edge); a grid barrier costs a few us.  Every CTA sums the CTA
// partials itself in one fixed order, so all CTAs take the same branches.  Vectors written in
// this launch (p, q, r~, x) are read with weak loads after the barrier (grid.sync is a gpu-scope
// fence), never through the read-only path; the matrix is read-only and keeps its .nc loads.

// x = r~ + beta p_old with coherent loads (k = 0: p = r~, beta = 0 gives r~ exactly)
struct XFusedW {
    const double* z;
    const double* p;
    double beta;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const size_t o = 6 * (size_t)vec + 2 * pair;
        const double2 zz = ld_cg2(z + o), pp = ld_cg2(p + o);
        return make_double2(fma(beta, pp.x, zz.x), fma(beta, pp.y, zz.y));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// Fixed-order grid sums of NV values per thread: CTA partials -> part[(slot+k)*Gmax + cta], grid
// barrier, then every CTA sums the G partials in the order grid_reduce_last uses.  k_sp_loop slots:
// 0 (phase A), 1-2 (phase B), 3 (phase C).  A CTA writes slot s only after passing at least one
// barrier that follows every read of s: phase A's slot 0 is read before barrier B, phase B's slots
// before barrier C or the next iteration's barrier A, phase C's slot 3 before the next barrier A.
// (Phase C on slot 0 would race: a fast CTA's next phase A rewrites slot 0 while a slow CTA is
// still summing the exact-test partials, and the CTAs could then disagree on the stop decision.)
// k_sp_ssor: 0 (A), 1-2 (L), 0 (C, followed by the U barrier before the next A), 3 (U).
template <int NV>
__device__ __forceinline__ void grid_allsum(const GArgs& a, cg::grid_group& grid, int slot, double (&v)[NV],
                                            double (&tot)[NV]) {
    __shared__ double red[NV][DDA_THREADS];
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
            a.part[(size_t)(slot + k) * a.Gmax + blockIdx.x] = s;
        }
    }
    grid.sync();
    const int G = gridDim.x;
#pragma unroll
    for (int k = 0; k < NV; ++k) {
        const double* part = a.part + (size_t)(slot + k) * a.Gmax;
        double s = 0.0;
        for (int j = threadIdx.x; j < G; j += DDA_THREADS) s += ld_cg(part + j);
        red[k][threadIdx.x] = s;
    }
    cta_barrier();
    if (kTreeP2 < DDA_THREADS) {
        if ((int)threadIdx.x < DDA_THREADS - kTreeP2) {
#pragma unroll
            for (int k = 0; k < NV; ++k) red[k][threadIdx.x] += red[k][threadIdx.x + kTreeP2];
        }
        cta_barrier();
    }
    for (int h = kTreeP2 / 2; h > 0; h >>= 1) {
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

// ---- phase A with the transposed products pushed, not pulled ("low-res" in L2)
//
// The paper's two-stage SpMV applies every stored block once in both directions and
// parks the transposed product V_ij^T x_i in a low-res array that a second stage sums per row.
// k_sp_loop's pull form instead re-reads each V_ki through low_to_up from L2 (0.86 GB per iteration
// at 1M) and gathers the lower neighbours' r~ / p_old, which puts phase A at the L2 sector cap
// (DESIGN.md §10).  Here one sweep does both stages, ten block rows per warp step:
//   produce (step s):  p_i (own rows), the forward products V_ij p_j, and the 48 B push
//                      lr[slot(ij)] = V_ij^T p_i for every upper block, in the same registers;
//   consume (step s-1): q_j = p_j + (its forward sum, kept in registers) + sum over its lower
//                      blocks of the pushed entries, in lower-CSR order (deterministic).
// A row's lower blocks all belong to rows with a smaller index, so to steps <= its own; one step of
// lag plus an ordering of the pushes before the reads replaces a grid barrier: per-group ready flags
// (release by the producing warp, acquire per pushing group by the consumer; default), per-step
// arrival counters, or entries tagged with the iteration parity in their last mantissa bit (the
// data is its own flag; results then differ from the untagged form by <= 1 ulp per entry).  The
// entries are laid out by CONSUMER group, each ten-row group's run 128 B aligned
// (base(g) = roundup128(48 lo(10g) + 128 g)), and the consuming warp may discard its lines from L2
// after reading them (discard.global.L2; not with tags) so they never reach HBM.
// Measured at 1M (profiles/r02_push_form.md): correct, but slower than the pull form
// (373-399 vs 304 us per iteration; 327 with no ordering at all): the producer holds p_i, the
// pending group and two blocks in flight in 128 registers, so 16 warps per SM instead of 24, and
// the 16 B entry accesses give back most of the L2 sectors the transposed re-reads cost.  Opt-in.
struct LrArgs {
    double2* lr;           // pushed entries (16 B units)
    const int* lr_off;     // [nnzb] entry of upper block u, in 16 B units
    unsigned* cnt;         // [ngrp] per-group ready flags (epoch), or [nsteps] per-step counters; zeroed per launch
    int discard;           // discard consumed lines from L2
    int sync;              // 0 per-group flags, 1 per-step counters, 2 none (timing diagnostic only: wrong results)
};

__device__ __forceinline__ void red_release_add(unsigned* p, unsigned v) {
    asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned ld_acquire_u(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void l2_discard(const void* p) {
    asm volatile("discard.global.L2 [%0], 128;" ::"l"(p) : "memory");
}
__device__ __forceinline__ double tag_lsb(double v, int t) {
    return __longlong_as_double((__double_as_longlong(v) & ~1ll) | (long long)t);
}
__device__ __forceinline__ void st_relaxed2(double2* p, double x, double y) {
    asm volatile("st.relaxed.gpu.global.v2.f64 [%0], {%1, %2};" ::"l"(p), "d"(x), "d"(y) : "memory");
}
__device__ __forceinline__ double2 ld_relaxed2(const double2* p) {
    double2 v;
    asm volatile("ld.relaxed.gpu.global.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ long long lr_base16(int lo_first, int g) {   // group g's first entry, 16 B units
    return ((48ll * lo_first + 128ll * g + 127) >> 7) << 3;
}

// Forward products and pushes of row i (group lanes; lane C owns column pair C of every block):
// y (pair C after the 3-lane reduce-scatter) = sum_j V_ij p_j, and lr entry of block ij, pair C,
// = sum_r V_ij[r][2C..2C+1] p_i[r] (the lane holds column pair C of all six rows).  Two blocks in
// flight per lane, the block list decoded one block ahead (as spmv_row_c5).
template <bool DEEP, class XLoad>
__device__ __forceinline__ void lr_row_produce(const BsrView& A, const LrArgs& L, int i, bool ok, const RowBounds& rb,
                                               const XLoad& xload, int lane, const double (&p6)[6], double& y0,
                                               double& y1, int tag) {
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane);
    const int C = ccol_of(lane);
    const int nb = (ok && lane < 30) ? rb.nu : 0;
    const int nbmax = __reduce_max_sync(full, nb);
    double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    auto decode = [&](int b, int& vec, int& off) {
        const bool v = b < nb;
        vec = v ? __ldg(A.col_idx + rb.up0 + b) : 0;
        off = v ? __ldg(L.lr_off + rb.up0 + b) : 0;
    };
    struct D {
        double4 c0, c1, c2;
        double2 x;
    };
    auto load = [&](int b, int vec) {
        D d;
        const bool v = b < nb;
        const double* blk = A.upper + (size_t)kBlk * (rb.up0 + (v ? b : 0));
        d.x = v ? xload.raw(vec, C) : make_double2(0.0, 0.0);
        d.c0 = ld_chunk_if(blk + 4 * C, v);
        d.c1 = ld_chunk_if(blk + 4 * (3 + C), v);
        d.c2 = ld_chunk_if(blk + 4 * (6 + C), v);
        return d;
    };
    int v1, o1, o0;
    decode(0, v1, o0);
    D d0 = load(0, v1);
    decode(1, v1, o1);
    for (int b = 0; b < nbmax; ++b) {
        int v2, o2;
        decode(b + 2, v2, o2);
        D d1;
        if (DEEP) d1 = load(b + 1, v1);   // two blocks in flight (else the next block loads after use)
        const double4 cs[3] = {d0.c0, d0.c1, d0.c2};
        const double2 xv = d0.x;
        double e0 = 0.0, e1 = 0.0;
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const double4 c = cs[k];
            acc[2 * k] = fma(c.x, xv.x, fma(c.y, xv.y, acc[2 * k]));
            acc[2 * k + 1] = fma(c.z, xv.x, fma(c.w, xv.y, acc[2 * k + 1]));
            e0 = fma(c.z, p6[2 * k + 1], fma(c.x, p6[2 * k], e0));
            e1 = fma(c.w, p6[2 * k + 1], fma(c.y, p6[2 * k], e1));
        }
        if (b < nb) {
            if (tag >= 0)   // last mantissa bit = iteration parity (the entry is its own ready flag)
                st_relaxed2(L.lr + (size_t)o0 + C, tag_lsb(e0, tag), tag_lsb(e1, tag));
            else
                L.lr[(size_t)o0 + C] = make_double2(e0, e1);
        }
        if (!DEEP) d1 = load(b + 1, v1);
        d0 = d1;
        v1 = v2;
        o0 = o1;
        o1 = o2;
    }
    const int c1 = C == 2 ? 0 : C + 1, c2 = C == 0 ? 2 : C - 1;
    const int s1 = lane < 30 ? 3 * h + c1 : lane, s2 = lane < 30 ? 3 * h + c2 : lane;
    const double2 w1 = pick_pair(acc, c2);
    const double r1x = __shfl_sync(full, w1.x, s1), r1y = __shfl_sync(full, w1.y, s1);
    const double2 w2 = pick_pair(acc, c1);
    const double r2x = __shfl_sync(full, w2.x, s2), r2y = __shfl_sync(full, w2.y, s2);
    const double2 own = pick_pair(acc, C);
    y0 = (own.x + r1x) + r2x;
    y1 = (own.y + r1y) + r2y;
}

// Phase A of k_sp_loop in the push form; returns this thread's partial of sigma = p.q.  `target` is
// the per-step counter value that means "every warp has produced this step in this iteration".
template <bool DEEP>
__device__ __forceinline__ double phase_a_lr(const GArgs& a, const LrArgs& L, const BsrView& A, const XFusedW& xf,
                                             const double* pold, double* pnew, double* x, double ap, int w0, int W,
                                             int lane, unsigned epoch) {
    const unsigned target = epoch * (unsigned)W;   // per-step counters: every warp produced the step
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane), C = ccol_of(lane);
    const bool lane_ok = lane < 30;
    const int n = A.n, ngrp = (n + 9) / 10, nsteps = (ngrp + W - 1) / W;
    double acc = 0.0;
    bool have = false;                      // a produced group waiting for its lower pushes
    int pg = 0, plo = 0, pnl = 0;
    double py0 = 0.0, py1 = 0.0, pp0 = 0.0, pp1 = 0.0;
    // consume, first half: wait for the pushes into the pending group's rows (sync 0 / 1), then issue
    // the loads of up to three of each row's entries, which stay in flight while the next group is
    // produced; sync 3 tags every pushed double with the iteration parity in its last mantissa bit
    // and the reader re-loads until the tag matches (the data is its own ready flag)
    const unsigned par = epoch & 1u;
    double2 lv[3];
    long long cb16 = 0;
    auto consume_begin = [&](int s) {
        const int j = 10 * pg + h;
        const bool ok = lane_ok && j < n;
        if (L.sync == 1 && lane == 0) {
            unsigned spins = 0;
            while ((int)(ld_acquire_u(L.cnt + s) - target) < 0) {
                __nanosleep(32);
                if (++spins > (1u << 26)) __trap();   // a lost arrival: fail loudly, never hang the GPU
            }
        } else if (L.sync == 0 && ok) {
            // the groups that pushed into this row (other than this warp's own, ordered by __syncwarp)
            for (int e = C; e < pnl; e += 3) {
                const int pgrp = __ldg(A.low_row + plo + e) / 10;
                if (pgrp == pg) continue;
                unsigned spins = 0;
                while ((int)(ld_acquire_u(L.cnt + pgrp) - epoch) < 0) {
                    __nanosleep(32);
                    if (++spins > (1u << 26)) __trap();
                }
            }
        }
        __syncwarp();
        const int lo_first = __shfl_sync(full, plo, 0);   // lane 0 holds row 10 pg (always < n)
        cb16 = lr_base16(lo_first, pg);
        const double2* src = L.lr + cb16 + 3ll * (plo - lo_first) + C;
        const int nl = ok ? pnl : 0;
#pragma unroll
        for (int t = 0; t < 3; ++t)
            lv[t] = t < nl ? (L.sync == 3 ? ld_relaxed2(src + 3 * t) : __ldcg(src + 3 * t)) : make_double2(0.0, 0.0);
    };
    auto consume_end = [&]() {
        const int j = 10 * pg + h;
        const bool ok = lane_ok && j < n;
        const int lo_first = __shfl_sync(full, plo, 0);
        const int lo_end = __reduce_max_sync(full, ok ? plo + pnl : 0);
        const double2* src = L.lr + cb16 + 3ll * (plo - lo_first) + C;
        const int nl = ok ? pnl : 0;
        double y0 = py0, y1 = py1;
        for (int e = 0; e < nl; ++e) {
            double2 v = e < 3 ? (e == 0 ? lv[0] : (e == 1 ? lv[1] : lv[2]))
                              : (L.sync == 3 ? ld_relaxed2(src + 3 * e) : __ldcg(src + 3 * e));
            if (L.sync == 3) {
                unsigned spins = 0;
                while (((unsigned)__double_as_longlong(v.x) & 1u) != par || ((unsigned)__double_as_longlong(v.y) & 1u) != par) {
                    if (++spins > (1u << 26)) __trap();
                    v = ld_relaxed2(src + 3 * e);
                }
            }
            y0 += v.x;
            y1 += v.y;
        }
        if (ok) {
            const size_t o = 6 * (size_t)j + 2 * C;
            *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
            acc += pp0 * y0 + pp1 * y1;
        }
        if (L.discard && L.sync != 3) {
            __syncwarp();
            const int nlines = (int)((48ll * (lo_end - lo_first) + 127) >> 7);
            const char* base = reinterpret_cast<const char*>(L.lr + cb16);
            for (int l = lane; l < nlines; l += 32) l2_discard(base + 128 * (size_t)l);
        }
    };
    RowBounds nxt = row_bounds<SPMV_OFFDIAG>(A, 10 * w0 + h, lane_ok);
    for (int s = 0; s < nsteps; ++s) {
        const int g = w0 + s * W;
        const int i = 10 * g + h;
        const bool ok = lane_ok && i < n;
        const RowBounds cur = nxt;
        nxt = row_bounds<SPMV_OFFDIAG>(A, i + 10 * W, lane_ok);
        // own p_i pair (x = r~ + beta p_old, as the gathers form it) and x += alpha_prev p_old
        double2 pv = make_double2(0.0, 0.0);
        if (ok) {
            const size_t o = 6 * (size_t)i + 2 * C;
            const double2 po = ld_cg2(pold + o);
            const double2 rr = ld_cg2(a.r + o);
            pv = make_double2(fma(xf.beta, po.x, rr.x), fma(xf.beta, po.y, rr.y));
            const double2 xo = ld_cg2(x + o);
            *reinterpret_cast<double2*>(x + o) = make_double2(xo.x + ap * po.x, xo.y + ap * po.y);
            *reinterpret_cast<double2*>(pnew + o) = pv;
        }
        double p6[6];
        {
            const int b0 = lane_ok ? 3 * h : lane;
#pragma unroll
            for (int c = 0; c < 3; ++c) {
                p6[2 * c] = __shfl_sync(full, pv.x, lane_ok ? b0 + c : lane);
                p6[2 * c + 1] = __shfl_sync(full, pv.y, lane_ok ? b0 + c : lane);
            }
        }
        if (have) consume_begin(s - 1);
        double y0, y1;
        lr_row_produce<DEEP>(A, L, i, ok, cur, xf, lane, p6, y0, y1, L.sync == 3 ? (int)par : -1);
        __syncwarp();
        if (lane == 0) {
            if (L.sync == 1)
                red_release_add(L.cnt + s, 1u);
            else if (L.sync == 0 && g < ngrp)
                st_release(reinterpret_cast<int*>(L.cnt + g), (int)epoch);
        }
        if (have) consume_end();
        have = g < ngrp;
        pg = g;
        plo = cur.lo0;
        pnl = cur.nl;
        py0 = y0 + pv.x;
        py1 = y1 + pv.y;
        pp0 = pv.x;
        pp1 = pv.y;
    }
    if (have) {
        consume_begin(nsteps - 1);
        consume_end();
    }
    return acc;
}

// lr_off[u] for every upper block u = (i, j): the position of u in row j's lower list (lower CSR
// index t), inside consumer group j / 10's 128 B-aligned run
__global__ void k_lr_off(int64_t nnzb, const int32_t* __restrict__ low_ptr, const int32_t* __restrict__ low_to_up,
                         const int32_t* __restrict__ col_idx, int32_t* __restrict__ lr_off) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nnzb; t += (int64_t)gridDim.x * blockDim.x) {
        const int u = __ldg(low_to_up + t);
        const int j = __ldg(col_idx + u);
        const int g = j / 10;
        const int lo_first = __ldg(low_ptr + 10 * g);
        lr_off[u] = (int32_t)(lr_base16(lo_first, g) + 3 * (t - lo_first));
    }
}

// LR: 0 = phase A in the pull form (for_rows_c), 1 = push form (phase_a_lr) with one block in flight
// per lane, 2 = with two (the opt-in variant: 128 registers, 2 CTAs/SM)
template <int MINB, int LR>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_sp_loop(const GArgs a) {
    const LrArgs L{a.lr, a.lr_off, a.lr_cnt, a.lr_discard, a.lr_sync};
    cg::grid_group grid = cg::this_grid();
    State* st = a.st;
    unsigned long long* tr_k = (a.trace && blockIdx.x == 0 && threadIdx.x == 0)
                                   ? a.trace + 4 * (size_t)a.trace_iters * gridDim.x : nullptr;
    if (tr_k) tr_k[0] = gtimer();                           // kernel entry / exit stamps (after the rows)
    if (st->done) return;                                   // decided at setup (uniform: no barrier reached)
    double rho = st->rho, alpha = 0.0, beta = 0.0, rr_last = st->rr;
    const double thr = a.ca->tol * st->bnorm;
    const int maxit = a.ca->maxit;
    BsrView A = a.A;
    A.upper = a.su;
    const int lane = threadIdx.x & 31;
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    const int n = A.n, ngrp = (n + 4) / 5;
    double* x = a.ca->d;
    int k = 0, status = DDA_ERR_NO_CONVERGENCE, iters = 0, checks = 0, pend = 0;
    unsigned long long* tr = nullptr;
    for (;;) {
        tr = (a.trace && k < a.trace_iters && threadIdx.x == 0)
                 ? a.trace + 4 * ((size_t)k * gridDim.x + blockIdx.x) : nullptr;
        if (tr) tr[0] = gtimer();
        // phase A: p_k = r~ + beta p_{k-1} (own rows written), q = Ks p_k, x += alpha_{k-1} p_{k-1}
        double* pnew = (k & 1) ? a.p1 : a.p0;
        const double* pold = k == 0 ? a.r : ((k & 1) ? a.p0 : a.p1);
        const XFusedW xf{a.r, pold, beta};
        const double ap = alpha;
        double acc = 0.0;
        auto rowA = [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                y0 += pv.x;
                y1 += pv.y;
                const double2 po = ld_cg2(pold + o);
                const double2 xo = ld_cg2(x + o);
                *reinterpret_cast<double2*>(x + o) = make_double2(xo.x + ap * po.x, xo.y + ap * po.y);
                *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
                *reinterpret_cast<double2*>(pnew + o) = pv;
                acc += pv.x * y0 + pv.y * y1;
            }
        };
        if (LR)
            acc = phase_a_lr<LR == 2>(a, L, A, xf, pold, pnew, x, ap, w0, W, lane, (unsigned)(k + 1));
        else
            for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, rowA);
        if (tr) tr[1] = gtimer();
        double sv[1] = {acc}, stot[1];
        grid_allsum<1>(a, grid, 0, sv, stot);
        const double sigma = stot[0];
        if (tr) tr[2] = gtimer();
        pend = 0;
        if (!(sigma > 0.0) || !isfinite(sigma)) { status = DDA_ERR_BREAKDOWN; break; }   // reading Z19
        alpha = rho / sigma;
        // phase B: r~ -= alpha q; rho' = |r~|^2 and the lower bound sum_i w_i |r~_i|^2 of |L r~|^2
        double rz = 0.0, lb = 0.0;
        for (int grp = w0; grp < ngrp; grp += 2 * W) {
            const Row5 RA = row5(grp, lane, n);
            const Row5 RB = row5(grp + W, lane, n);
            double ra = 0, qa = 0, rb = 0, qb = 0, wa = 0, wb = 0;
            if (RA.valid) { ra = ld_cg(a.r + RA.idx); qa = ld_cg(a.q + RA.idx); wa = __ldg(a.bj_w + RA.i); }
            if (RB.valid) { rb = ld_cg(a.r + RB.idx); qb = ld_cg(a.q + RB.idx); wb = __ldg(a.bj_w + RB.i); }
            const double rva = RA.valid ? ra - alpha * qa : 0.0;
            const double rvb = RB.valid ? rb - alpha * qb : 0.0;
            if (RA.valid) a.r[RA.idx] = rva;
            if (RB.valid) a.r[RB.idx] = rvb;
            rz += rva * rva + rvb * rvb;
            lb += wa * (rva * rva) + wb * (rvb * rvb);
        }
        if (tr) tr[3] = gtimer();
        double bv[2] = {rz, lb}, btot[2];
        grid_allsum<2>(a, grid, 1, bv, btot);
        const double rho1 = btot[0];
        pend = 1;                                           // x += alpha p_k: next phase A or k_s_final
        iters = k + 1;
        if (a.hist && k < a.hist_cap && blockIdx.x == 0 && threadIdx.x == 0) {
            a.hist[2 * (size_t)k] = rho1;
            a.hist[2 * (size_t)k + 1] = __longlong_as_double(0x7FF8000000000000ll);
        }
        if (rho1 == 0.0) { status = DDA_OK; rr_last = 0.0; k = k + 1; break; }
        if (isfinite(rho1) && !(0.999 * btot[1] > thr * thr)) {
            // phase C (rare): the exact stopping test |L r~| <= tol ||F|| (reading Z1; see k_s_update)
            double rl = 0.0;
            for (int grp = w0; grp < ngrp; grp += W) {
                const Row5 R = row5(grp, lane, n);
                const double rv = R.valid ? ld_cg(a.r + R.idx) : 0.0;
                const DinvRow Lrow = tri_row(a.lfac, R);
                const double o0 = dinv_row_apply(Lrow, rv, R);
                const double o = R.valid ? o0 : 0.0;
                rl += o * o;
            }
            double cv[1] = {rl}, ctot[1];
            grid_allsum<1>(a, grid, 3, cv, ctot);   // slot 3: slot 0 is rewritten by the next phase A
            const double rr = ctot[0];
            if (a.hist && k < a.hist_cap && blockIdx.x == 0 && threadIdx.x == 0) a.hist[2 * (size_t)k + 1] = rr;
            checks += 1;
            rr_last = rr;
            if (sqrt(rr) <= thr) { status = DDA_OK; k = k + 1; break; }
        }
        // finish_iteration
        k = k + 1;
        if (!(rho1 > 0.0) || !isfinite(rho1)) { status = DDA_ERR_BREAKDOWN; break; }
        beta = rho1 / rho;
        rho = rho1;
        if (k >= maxit) { status = DDA_ERR_NO_CONVERGENCE; break; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {              // the State k_s_final / k_g_resid read
        st->k = k;
        st->iters = iters;
        st->status = status;
        st->done = 1;
        st->alpha = alpha;
        st->beta = beta;
        st->rho = rho;
        st->rr = rr_last;
        st->pend = pend;
        st->checks = checks;
    }
    if (tr_k) tr_k[1] = gtimer();
}

// ---- scaled SSOR-AI (A7) in one persistent kernel
//
// The SSOR approximate inverse of reading Z14, M^{-1} = (I - w D^{-1} U) D^{-1} (I - w U^T D^{-1}),
// is, with D^{-1} = S^T S (S = L^{-1}) and Us = S U S^T (the scaled upper blocks, sc_upper),
//   M^{-1} = S^T (I - w Us)(I - w Us^T) S,
// so SSOR-AI PCG on K d = F is PCG on Ks x = S F with M~^{-1} = (I - w Us)(I - w Us^T): the same
// iterates under r~ = S r, z = S^T z~ (exact arithmetic), and the apply streams no D^{-1}.
// Per iteration (three grid barriers, three passes over the upper storage):
//   A  p = z~ + beta p_old (on the fly), q = Ks p, x += alpha_prev p_old; sigma      | barrier
//   L  r~' = r~ - alpha q (on the fly for gathered lower neighbours, ping-pong r~),
//      t = r~' - w Us^T r~' (transposed half pass); |r~'|^2 and the w-bound          | barrier
//      [C: the exact stopping test |L r~'| when the bound allows it                  | barrier]
//   U  z~ = t - w Us t (upper half pass); rho' = r~' . z~ -> beta                    | barrier
// Before the loop the same L and U passes with alpha = 0 give z~0 = M~^{-1} r~0.

// x = r - alpha q formed on the fly (the residual update fused into the lower half pass)
struct XUpdW {
    const double* r;
    const double* q;
    double alpha;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const size_t o = 6 * (size_t)vec + 2 * pair;
        const double2 rr = ld_cg2(r + o), qq = ld_cg2(q + o);
        return make_double2(fma(-alpha, qq.x, rr.x), fma(-alpha, qq.y, rr.y));
    }
    __device__ __forceinline__ double2 cook(const Raw& v) const { return v; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};
struct XPlainW {   // coherent loads of a vector written in this launch
    const double* x;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const { return ld_cg2(x + 6 * (size_t)vec + 2 * pair); }
    __device__ __forceinline__ double2 cook(const Raw& v) const { return v; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

// L pass: r~' (written to rn), t = r~' - w Us^T r~'; returns (|r~'|^2, sum w_i |r~'_i|^2) partials
__device__ __forceinline__ double2 ssor_lower_pass(const GArgs& a, const BsrView& A, const double* rc, double* rn,
                                                   const double* qv, double alpha, double omega, int w0, int W) {
    const int lane = threadIdx.x & 31;
    const XUpdW xf{rc, qv, alpha};
    double rr = 0.0, lb = 0.0;
    for_rows_c<SPMV_LOWER_T, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
        if (ok) {
            const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
            const double2 rv = xf(i, ccol_of(lane));
            *reinterpret_cast<double2*>(rn + o) = rv;
            *reinterpret_cast<double2*>(a.t + o) = make_double2(fma(-omega, y0, rv.x), fma(-omega, y1, rv.y));
            const double s = rv.x * rv.x + rv.y * rv.y;
            rr += s;
            lb += __ldg(a.bj_w + i) * s;
        }
    });
    return make_double2(rr, lb);
}

// U pass: z~ = t - w Us t (written to z); returns this lane's share of r~' . z~
__device__ __forceinline__ double ssor_upper_pass(const GArgs& a, const BsrView& A, const double* rn, double omega,
                                               int w0, int W) {
    const int lane = threadIdx.x & 31;
    const XPlainW xf{a.t};
    double rz = 0.0;
    for_rows_c<SPMV_UPPER, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
        if (ok) {
            const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
            const double2 tv = xf(i, ccol_of(lane));
            const double2 zv = make_double2(fma(-omega, y0, tv.x), fma(-omega, y1, tv.y));
            *reinterpret_cast<double2*>(a.z + o) = zv;
            const double2 rv = ld_cg2(rn + o);
            rz += rv.x * zv.x + rv.y * zv.y;
        }
    });
    return rz;
}

// A pass: p = z~ + beta p_old (own rows written), q = Ks p, x += alpha_prev p_old; returns sigma share
__device__ __forceinline__ double ssor_spmv_pass(const GArgs& a, const BsrView& A, const double* pold, double* pnew,
                                              double beta, double alpha_prev, int w0, int W) {
    const int lane = threadIdx.x & 31;
    const XFusedW xf{a.z, pold, beta};
    double* x = a.ca->d;
    double acc = 0.0;
    for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
        if (ok) {
            const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
            const double2 pv = xf(i, ccol_of(lane));
            y0 += pv.x;
            y1 += pv.y;
            const double2 po = ld_cg2(pold + o);
            const double2 xo = ld_cg2(x + o);
            *reinterpret_cast<double2*>(x + o) = make_double2(xo.x + alpha_prev * po.x, xo.y + alpha_prev * po.y);
            *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
            *reinterpret_cast<double2*>(pnew + o) = pv;
            acc += pv.x * y0 + pv.y * y1;
        }
    });
    return acc;
}

// exact stopping test share: |L r~|^2 over this thread's rows
__device__ __forceinline__ double exact_rr_pass(const GArgs& a, const double* rn, int w0, int W) {
    const int lane = threadIdx.x & 31;
    const int n = a.A.n, ngrp = (n + 4) / 5;
    double rl = 0.0;
    for (int grp = w0; grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double rv = R.valid ? ld_cg(rn + R.idx) : 0.0;
        const DinvRow Lrow = tri_row(a.lfac, R);
        const double o0 = dinv_row_apply(Lrow, rv, R);
        const double o = R.valid ? o0 : 0.0;
        rl += o * o;
    }
    return rl;
}

// ---- scaled BJ, single-reduction variant (Chronopoulos-Gear CG on Ks; A/B tuning aid, DDA_SCALED_CG1=1)
//
// The same Krylov iterates in exact arithmetic with ONE grid barrier per iteration instead of two:
// s = Ks r is carried instead of q = Ks p (q_k = s_k + beta_k q_{k-1}), so the SpMV operand of pass k
// is r_{k+1} = r_k - alpha_k (s_k + beta_k q_{k-1}), formed on the fly from vectors of pass k - 1,
// and both inner products of the next step (rho = r.r, mu = r.s) come out of the same pass:
//   beta_{k+1} = rho_{k+1} / rho_k,  alpha_{k+1} = rho_{k+1} / (mu_{k+1} - beta_{k+1} rho_{k+1} / alpha_k).
// Pass k per row: q_k, p_k (own), x += alpha_k p_k, r_{k+1}, s_{k+1} = Ks r_{k+1}; partials rho, mu, w-bound.
// r, s, q are ping-ponged (neighbours read pass k - 1's values while owners write pass k's); p and
// x are own-row only and updated in place.  Partial slots alternate between passes (1-3 / 4-6) so a
// fast CTA never overwrites partials a slow CTA is still summing; phase C keeps slot 0.
struct XCg1 {   // r_{k+1} = r_k - alpha (s_k + beta q_{k-1}) (first pass: q_0 = s_0)
    const double *r, *s, *q;
    double alpha, beta;
    bool first;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        const size_t o = 6 * (size_t)vec + 2 * pair;
        const double2 rr = ld_cg2(r + o), ss = ld_cg2(s + o);
        double2 qk = ss;
        if (!first) {
            const double2 qq = ld_cg2(q + o);
            qk = make_double2(fma(beta, qq.x, ss.x), fma(beta, qq.y, ss.y));
        }
        return make_double2(fma(-alpha, qk.x, rr.x), fma(-alpha, qk.y, rr.y));
    }
    __device__ __forceinline__ double2 cook(const Raw& v) const { return v; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

template <int TPB, class Sync>
__device__ __forceinline__ void sp_cg1_body(const GArgs& a, Sync& sync) {
    constexpr int WPBT = TPB / 32;
    State* st = a.st;
    if (st->done) return;
    double rho = st->rho, alpha = 0.0, beta = 0.0, rr_last = st->rr;
    const double thr = a.ca->tol * st->bnorm;
    const int maxit = a.ca->maxit;
    BsrView A = a.A;
    A.upper = a.su;
    const int lane = threadIdx.x & 31;
    const int w0 = blockIdx.x * WPBT + (threadIdx.x >> 5), W = gridDim.x * WPBT;
    const int n = A.n, ngrp = (n + 4) / 5;
    double* x = a.ca->d;
    double* Rb[2] = {a.r, a.z};
    double* Sb[2] = {a.t, a.w};
    double* Qb[2] = {a.q, a.p1};
    double* P = a.p0;
    int k = 0, status = DDA_ERR_NO_CONVERGENCE, iters = 0, checks = 0;
    {   // pass 0: s_0 = Ks r_0, mu_0 = r_0 . s_0
        const XPlainW xf{a.r};
        double mu = 0.0;
        for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 rv = xf(i, ccol_of(lane));
                const double2 sv = make_double2(y0 + rv.x, y1 + rv.y);
                *reinterpret_cast<double2*>(Sb[0] + o) = sv;
                mu += rv.x * sv.x + rv.y * sv.y;
            }
        });
        double v[1] = {mu}, tot[1];
        sync.template allsum<1>(4, v, tot);
        if (!(tot[0] > 0.0) || !isfinite(tot[0])) status = DDA_ERR_BREAKDOWN;
        alpha = rho / tot[0];
    }
    while (status != DDA_ERR_BREAKDOWN) {
        const int cur = k & 1, nxt = cur ^ 1;
        const bool first = k == 0;
        const XCg1 xf{Rb[cur], Sb[cur], Qb[nxt], alpha, beta, first};
        const double* rk_ = Rb[cur];
        const double* sk_ = Sb[cur];
        const double* qp_ = Qb[nxt];
        double* qk_ = Qb[cur];
        double* r1_ = Rb[nxt];
        double* s1_ = Sb[nxt];
        double rz = 0.0, mu = 0.0, lb = 0.0;
        for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 rk = ld_cg2(rk_ + o), sk = ld_cg2(sk_ + o);
                double2 qk = sk, pk = rk;
                if (!first) {
                    const double2 qp = ld_cg2(qp_ + o), pp = ld_cg2(P + o);
                    qk = make_double2(fma(beta, qp.x, sk.x), fma(beta, qp.y, sk.y));
                    pk = make_double2(fma(beta, pp.x, rk.x), fma(beta, pp.y, rk.y));
                }
                const double2 r1 = make_double2(fma(-alpha, qk.x, rk.x), fma(-alpha, qk.y, rk.y));
                const double2 s1 = make_double2(y0 + r1.x, y1 + r1.y);
                const double2 xo = ld_cg2(x + o);
                *reinterpret_cast<double2*>(x + o) = make_double2(xo.x + alpha * pk.x, xo.y + alpha * pk.y);
                *reinterpret_cast<double2*>(P + o) = pk;
                *reinterpret_cast<double2*>(qk_ + o) = qk;
                *reinterpret_cast<double2*>(r1_ + o) = r1;
                *reinterpret_cast<double2*>(s1_ + o) = s1;
                const double rr2 = r1.x * r1.x + r1.y * r1.y;
                rz += rr2;
                mu += r1.x * s1.x + r1.y * s1.y;
                lb += __ldg(a.bj_w + i) * rr2;
            }
        });
        double bv[3] = {rz, mu, lb}, btot[3];
        sync.template allsum<3>(cur ? 4 : 1, bv, btot);
        const double rho1 = btot[0];
        iters = k + 1;
        if (a.hist && k < a.hist_cap && blockIdx.x == 0 && threadIdx.x == 0) {
            a.hist[2 * (size_t)k] = rho1;
            a.hist[2 * (size_t)k + 1] = __longlong_as_double(0x7FF8000000000000ll);
        }
        if (rho1 == 0.0) { status = DDA_OK; rr_last = 0.0; k = k + 1; break; }
        if (isfinite(rho1) && !(0.999 * btot[2] > thr * thr)) {
            double rl = 0.0;   // phase C: the exact test |L r~| <= tol ||F|| (reading Z1)
            for (int grp = w0; grp < ngrp; grp += W) {
                const Row5 R = row5(grp, lane, n);
                const double rv = R.valid ? ld_cg(r1_ + R.idx) : 0.0;
                const DinvRow Lrow = tri_row(a.lfac, R);
                const double o0 = dinv_row_apply(Lrow, rv, R);
                const double o = R.valid ? o0 : 0.0;
                rl += o * o;
            }
            double cv[1] = {rl}, ctot[1];
            sync.template allsum<1>(0, cv, ctot);
            if (a.hist && k < a.hist_cap && blockIdx.x == 0 && threadIdx.x == 0) a.hist[2 * (size_t)k + 1] = ctot[0];
            checks += 1;
            rr_last = ctot[0];
            if (sqrt(ctot[0]) <= thr) { status = DDA_OK; k = k + 1; break; }
        }
        k = k + 1;
        if (!(rho1 > 0.0) || !isfinite(rho1)) { status = DDA_ERR_BREAKDOWN; break; }
        const double b1 = rho1 / rho;
        const double den = btot[1] - b1 * rho1 / alpha;
        if (!(den > 0.0) || !isfinite(den)) { status = DDA_ERR_BREAKDOWN; break; }   // p.Ks p <= 0
        beta = b1;
        alpha = rho1 / den;
        rho = rho1;
        if (k >= maxit) { status = DDA_ERR_NO_CONVERGENCE; break; }
    }
    sync.finish();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        st->k = k;
        st->iters = iters;
        st->status = status;
        st->done = 1;
        st->alpha = alpha;
        st->beta = beta;
        st->rho = rho;
        st->rr = rr_last;
        st->pend = 0;   // x already holds x_{k}
        st->checks = checks;
    }
}


// the grid-wide form: cooperative grid, fixed-order sums of the CTA partials in global memory
struct GridSyncCg1 {
    const GArgs& a;
    cg::grid_group grid;
    __device__ __forceinline__ void finish() {}
    template <int NV>
    __device__ __forceinline__ void allsum(int slot, double (&v)[NV], double (&tot)[NV]) {
        grid_allsum<NV>(a, grid, slot, v, tot);
    }
};

template <int MINB>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_sp_cg1(const GArgs a) {
    GridSyncCg1 s{a, cg::this_grid()};
    sp_cg1_body<DDA_THREADS>(a, s);
}

// Small systems (the paper's case-1 scale): ONE thread-block cluster runs the whole loop.  The
// cluster barrier (barrier.cluster, hardware) replaces the grid barrier, and every reduction reads
// the cluster's CTA partials from their shared memory through DSMEM (map_shared_rank) in rank order:
// deterministic, no global partials, no grid-wide barrier.  Vectors written by other CTAs of the
// cluster are read after barrier.cluster's release / acquire (cluster scope).
constexpr int kClThreads = 512;   // 16 warps per CTA
struct ClusterSyncCg1 {
    cg::cluster_group cl;
    // no CTA may exit while another can still read its shared memory through DSMEM
    __device__ __forceinline__ void finish() { cl.sync(); }
    template <int NV>
    __device__ __forceinline__ void allsum(int slot, double (&v)[NV], double (&tot)[NV]) {
        __shared__ double red[NV][kClThreads / 32];
        __shared__ double cpart[8];
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
                for (int w = 0; w < kClThreads / 32; ++w) s += red[k][w];
                cpart[slot + k] = s;
            }
        }
        cl.sync();
        const int nr = (int)cl.num_blocks();
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int r = 0; r < nr; ++r) s += *cl.map_shared_rank(&cpart[slot + k], r);
            tot[k] = s;
        }
    }
};

__global__ void __launch_bounds__(kClThreads, 1) k_sp_cg1_cl(const GArgs a) {
    ClusterSyncCg1 s{cg::this_cluster()};
    sp_cg1_body<kClThreads>(a, s);
}

__global__ void __launch_bounds__(DDA_THREADS, 3) k_sp_ssor(const GArgs a) {
    cg::grid_group grid = cg::this_grid();
    State* st = a.st;
    if (st->done) return;                                   // decided at setup (uniform: no barrier reached)
    const double thr = a.ca->tol * st->bnorm, omega = a.ca->omega;
    const int maxit = a.ca->maxit;
    BsrView A = a.A;
    A.upper = a.su;
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    double* rb[2] = {a.r, a.w};                             // r~ ping-pong (a.w is free in this engine)
    int ri = 0;
    double rho, alpha = 0.0, beta = 0.0, rr_last = st->rr;
    int k = 0, status = DDA_ERR_NO_CONVERGENCE, iters = 0, checks = 0, pend = 0;
    {   // z~0 = M~^{-1} r~0, rho0 = r~0 . z~0
        const double2 lr = ssor_lower_pass(a, A, rb[ri], rb[ri ^ 1], rb[ri], 0.0, omega, w0, W);   // q = r: no NaN
        (void)lr;
        ri ^= 1;
        grid.sync();
        const double rz0 = ssor_upper_pass(a, A, rb[ri], omega, w0, W);
        double v[1] = {rz0}, t[1];
        grid_allsum<1>(a, grid, 3, v, t);
        rho = t[0];
        if (!(rho > 0.0) || !isfinite(rho)) status = DDA_ERR_BREAKDOWN;
    }
    while (status != DDA_ERR_BREAKDOWN) {
        double* pnew = (k & 1) ? a.p1 : a.p0;
        const double* pold = k == 0 ? a.z : ((k & 1) ? a.p0 : a.p1);
        const double sg = ssor_spmv_pass(a, A, pold, pnew, beta, alpha, w0, W);
        double sv[1] = {sg}, stt[1];
        grid_allsum<1>(a, grid, 0, sv, stt);
        pend = 0;
        const double sigma = stt[0];
        if (!(sigma > 0.0) || !isfinite(sigma)) { status = DDA_ERR_BREAKDOWN; break; }   // reading Z19
        alpha = rho / sigma;
        const double2 lr = ssor_lower_pass(a, A, rb[ri], rb[ri ^ 1], a.q, alpha, omega, w0, W);
        ri ^= 1;
        double lv[2] = {lr.x, lr.y}, lt[2];
        grid_allsum<2>(a, grid, 1, lv, lt);
        pend = 1;                                           // x += alpha p_k: next A pass or k_s_final
        iters = k + 1;
        const double rr1 = lt[0];
        if (rr1 == 0.0) { status = DDA_OK; rr_last = 0.0; k = k + 1; break; }
        if (isfinite(rr1) && !(0.999 * lt[1] > thr * thr)) {
            const double rl = exact_rr_pass(a, rb[ri], w0, W);
            double cv[1] = {rl}, ct[1];
            grid_allsum<1>(a, grid, 0, cv, ct);
            checks += 1;
            rr_last = ct[0];
            if (sqrt(ct[0]) <= thr) { status = DDA_OK; k = k + 1; break; }
        }
        const double rz = ssor_upper_pass(a, A, rb[ri], omega, w0, W);
        double uv[1] = {rz}, ut[1];
        grid_allsum<1>(a, grid, 3, uv, ut);
        const double rho1 = ut[0];
        k = k + 1;
        if (!(rho1 > 0.0) || !isfinite(rho1)) { status = DDA_ERR_BREAKDOWN; break; }
        beta = rho1 / rho;
        rho = rho1;
        if (k >= maxit) { status = DDA_ERR_NO_CONVERGENCE; break; }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {              // the State k_s_final / k_g_resid read
        st->k = k;
        st->iters = iters;
        st->status = status;
        st->done = 1;
        st->alpha = alpha;
        st->beta = beta;
        st->rr = rr_last;
        st->pend = pend;
        st->checks = checks;
    }
}

// Experiment kernels (internal timing hook dda__time_ks_variants): the bare off-diagonal Ks product
// q = Ks p with sigma, gathering ONE vector, through the read-only path (LDG) or coherent loads.
template <bool LDG, int MINB>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_x_ks(const GArgs a) {
    BsrView A = a.A;
    A.upper = a.su;
    const int lane = threadIdx.x & 31;
    const int w0 = blockIdx.x * WPB + (threadIdx.x >> 5), W = gridDim.x * WPB;
    double acc = 0.0;
    auto body = [&](const auto& xf) {
        for_rows_c<SPMV_OFFDIAG, 5>(A, w0, W, xf, lane, [&](int i, bool ok, double y0, double y1) {
            if (ok) {
                const size_t o = 6 * (size_t)i + 2 * ccol_of(lane);
                const double2 pv = xf(i, ccol_of(lane));
                y0 += pv.x;
                y1 += pv.y;
                *reinterpret_cast<double2*>(a.q + o) = make_double2(y0, y1);
                acc += pv.x * y0 + pv.y * y1;
            }
        });
    };
    if (LDG) body(XPlain{a.p0}); else body(XPlainW{a.p0});
    if (acc == 12345.678) a.part[0] = acc;   // keep the dot product live
}

// loop-body SpMV kernel variants (tuning aid, DDA_GSPMV_VARIANT): occupancy / register budget
typedef void (*GSpmvKernel)(const GArgs, cudaGraphConditionalHandle);
struct GSpmvVariant { GSpmvKernel plain, scaled; int minb; };
// default: v5 row product (look-ahead decode, two blocks in flight) at 3 CTAs/SM (no spills): 317.6
// us per whole scaled-engine iteration at 1M blocks vs 330.8 with v4 (one block in flight) since the
// SpMV also applies the deferred x += alpha p; v3 at 4 CTAs/SM: 282 us for the SpMV alone (v4: 240).
const GSpmvVariant kGSpmv[] = {
    {k_g_spmv<3, false, 5>, k_g_spmv<3, true, 5>, 3},
    {k_g_spmv<3, false>, k_g_spmv<3, true>, 3},
    {k_g_spmv<4, false>, k_g_spmv<4, true>, 4},
    {k_g_spmv<2, false, 5>, k_g_spmv<2, true, 5>, 2},
};
const GSpmvVariant& gspmv_variant() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("DDA_GSPMV_VARIANT");
        v = e ? atoi(e) : 0;
        if (v < 0 || v >= (int)(sizeof(kGSpmv) / sizeof(kGSpmv[0]))) v = 0;
    }
    return kGSpmv[v];
}

int env_int(const char* name, int dflt) {
    const char* e = getenv(name);
    return e ? atoi(e) : dflt;
}

int occ_grid(const void* k, int minb_cap) {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, DDA_THREADS, 0);
    if (per_sm < 1) per_sm = 1;
    if (minb_cap > 0 && per_sm > minb_cap) per_sm = minb_cap;
    return device_sms() * per_sm;
}

}  // namespace

// scaled-engine loop: 1 = persistent cooperative kernel, 0 = CUDA-graph while loop, -1 = from
// DDA_SCALED_LOOP (default persistent); set by the internal hook dda__set_scaled_loop
int g_scaled_loop = -1;
unsigned long long* g_trace = nullptr;   // k_sp_loop timeline (internal hook dda__set_loop_trace)
int g_trace_iters = 0;

#ifndef DDA_SPLOOP_MINB
#define DDA_SPLOOP_MINB 3
#endif
constexpr int kSpLoopMinb = DDA_SPLOOP_MINB;   // CTAs per SM of the persistent loops (tuning build flag)
constexpr int kCg1Rows = 60000;   // k_sp_cg1 below this many block rows (see pcg_graph_solve)
constexpr int kClMaxRows = 65536; // k_sp_cg1_cl (one cluster, opt-in) up to this many block rows
constexpr int kClCtas = 16;       // the cluster: 16 CTAs of kClThreads (non-portable size)
bool cluster_size_ok() {
    static int ok = -1;
    if (ok < 0) {
        cudaFuncSetAttribute(k_sp_cg1_cl, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(kClCtas);
        cfg.blockDim = dim3(kClThreads);
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = kClCtas;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        int nclusters = 0;
        ok = (cudaOccupancyMaxActiveClusters(&nclusters, k_sp_cg1_cl, &cfg) == cudaSuccess && nclusters >= 1) ? 1 : 0;
        cudaGetLastError();
    }
    return ok == 1;
}

// Per-handle cached graph engine
struct PcgGraph {
    int pc = -1;
    GArgs a{};
    cudaGraphExec_t exec = nullptr;
    cudaGraph_t graph = nullptr;
    cudaGraphConditionalHandle h = 0;
    int G_spmv = 0, G_vec = 0, g_ilu = 0;
    int G_persist = 0;   // scaled engine, persistent loop: cooperative grid (0: graph loop)
    bool cluster = false;   // the persistent loop is k_sp_cg1_cl in one thread-block cluster
    int body_iters = 2;
};

void pcg_graph_free(void* p) {
    PcgGraph* g = reinterpret_cast<PcgGraph*>(p);
    if (!g) return;
    if (g->exec) cudaGraphExecDestroy(g->exec);
    if (g->graph) cudaGraphDestroy(g->graph);
    delete g;
}

// S_i V_ij S_j^T for the scaled BJ engine (needs the factors from bj_setup); cached until the values change
dda_status_t scaled_setup(dda_matrix* K, cudaStream_t st) {
    if (K->scaled_valid) return DDA_OK;
    if (!K->sc_upper && K->nnzb > 0)
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->sc_upper), sizeof(double) * kBlk * (size_t)K->nnzb, st));
    if (K->nnzb > 0) {
        int g = (int)((K->nnzb + 127) / 128);
        const int cap = device_sms() * 16;
        if (g > cap) g = cap;
        k_scale_upper<<<g, 128, 0, st>>>(K->nnzb, K->urow, K->col_idx, K->upper, K->sfac, K->sc_upper);
        DDA_LAUNCHED();
    }
    K->scaled_valid = true;
    return DDA_OK;
}

// The push-form phase A's entry map and buffers (structure only: built once per matrix)
dda_status_t lr_setup(dda_matrix* K, cudaStream_t st) {
    if (K->lr_off || K->nnzb == 0) return DDA_OK;
    const int64_t ngrp = (K->n + 9) / 10;
    const size_t ebytes = (size_t)(48 * K->nnzb + 128 * ngrp + 256);
    if ((int64_t)(ebytes / 16) > INT32_MAX) return DDA_ERR_ARG;   // 16 B offsets are int32
    const size_t cbytes = sizeof(unsigned) * (size_t)(ngrp + 1);
    void* buf = nullptr;
    void* off = nullptr;
    DDA_CK(dev_alloc(&buf, ebytes + cbytes, st));
    cudaError_t e = dev_alloc(&off, sizeof(int32_t) * (size_t)K->nnzb, st);
    if (e != cudaSuccess) {   // publish both or neither (lr_off set means the map is built)
        dev_free_on(buf, st);
        return cuda_fail(e);
    }
    K->lr_buf = buf;
    K->lr_off = reinterpret_cast<int32_t*>(off);
    K->lr_bytes = ebytes;
    int g = (int)((K->nnzb + 255) / 256);
    const int cap = device_sms() * 8;
    if (g > cap) g = cap;
    k_lr_off<<<g, 256, 0, st>>>(K->nnzb, K->low_ptr, K->low_to_up, K->col_idx, K->lr_off);
    DDA_LAUNCHED();
    return DDA_OK;
}

dda_status_t pcg_graph_solve(dda_matrix* K, const double* F, const double* d0, double* d, double tol,
                             int32_t maxit, dda_precond_t pc, double omega, int32_t* iters, double* rel_res,
                             cudaStream_t st, bool scaled) {
    const size_t N = 6 * (size_t)K->n;
    if (scaled) {
        if (pc != DDA_PC_BJ && pc != DDA_PC_SSOR_AI) return DDA_ERR_ARG;
        dda_status_t s = scaled_setup(K, st);
        if (s != DDA_OK) return s;
    }
    trace("solve: enter");
    // scaled engine loop: one persistent cooperative kernel (default) or the CUDA-graph while loop
    // (DDA_SCALED_LOOP=graph)
    if (g_scaled_loop < 0) {
        const char* e = getenv("DDA_SCALED_LOOP");
        g_scaled_loop = (e && (e[0] == 'g' || e[0] == '0')) ? 0 : 1;
    }
    // scaled SSOR-AI exists as a persistent kernel only (k_sp_ssor)
    bool persist = scaled && (g_scaled_loop == 1 || pc == DDA_PC_SSOR_AI);
    // scaled BJ engine: the single-reduction loop (one grid barrier per iteration, one more gathered
    // vector per block) below kCg1Rows block rows, where the iteration is barrier-latency bound; the
    // two-phase k_sp_loop above, where the gathers' L2 traffic decides (measured
    // crossover).  DDA_SCALED_CG1 = 0 / 1 forces either (tests, A/B).
    const int cg1_env = env_int("DDA_SCALED_CG1", -1);
    const bool cg1 = scaled && pc == DDA_PC_BJ && (cg1_env >= 0 ? cg1_env != 0 : K->n < kCg1Rows);
    // the single-reduction loop in ONE thread-block cluster (k_sp_cg1_cl): opt-in (DDA_SCALED_CLUSTER=1,
    // up to kClMaxRows), measured slower than the grid form at every size
    const bool cl = cg1 && g_scaled_loop != 0 && K->n <= kClMaxRows && env_int("DDA_SCALED_CLUSTER", 0) == 1 &&
                    cluster_size_ok();
    // the two-phase loop's phase A in the pull form (default) or the push form (phase_a_lr, opt-in
    // DDA_SP_LR=1: measured slower); DDA_LR_SYNC selects its ordering (0 ready flags,
    // 1 step counters, 3 parity-tagged entries), DDA_LR_DISCARD=0 keeps consumed entries in L2
    const bool lr = scaled && pc == DDA_PC_BJ && !cg1 && K->nnzb > 0 && env_int("DDA_SP_LR", 0) != 0;
    const void* persist_kernel = pc == DDA_PC_SSOR_AI ? reinterpret_cast<const void*>(k_sp_ssor)
                                 : cg1                ? reinterpret_cast<const void*>(k_sp_cg1<3>)
                                 : lr                 ? reinterpret_cast<const void*>(k_sp_loop<2, 2>)
                                                      : reinterpret_cast<const void*>(k_sp_loop<kSpLoopMinb, 0>);
    if (persist) {
        // The persistent kernels need every CTA co-resident (cooperative launch).  If not even one CTA
        // per SM fits (e.g. a smaller shared-memory carve-out forced by the caller's context), fall
        // back before any state is written: scaled BJ to the CUDA-graph while loop (same phases as
        // kernels), SSOR-AI to the unscaled graph engine.
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, persist_kernel, DDA_THREADS, 0);
        if (env_int("DDA_SIMULATE_NO_COOP", 0)) per_sm = 0;   // test hook: exercise the fallback
        if (per_sm < 1) {
            trace("solve: cooperative grid does not fit, graph loop fallback");
            if (pc == DDA_PC_SSOR_AI)
                return pcg_graph_solve(K, F, d0, d, tol, maxit, pc, omega, iters, rel_res, st, false);
            persist = false;
        }
    }
    const int key = (scaled ? (persist ? 200 : 100) + (int)pc : (int)pc) + (cg1 ? 1000 : 0) + (cl ? 2000 : 0) +
                    (persist && lr ? 4000 : 0);
    if (persist && lr) {
        dda_status_t s = lr_setup(K, st);
        if (s != DDA_OK) return s;
    }
    PcgGraph*& G = reinterpret_cast<PcgGraph*&>(K->graph_engine);
    if (G && G->pc != key) {
        pcg_graph_free(G);
        G = nullptr;
    }
    if (!G) {
        const int need_rows = (K->n + 10 * WPB - 1) / (10 * WPB);
        const GSpmvVariant& gv = gspmv_variant();
        int g_spmv = occ_grid(scaled ? (const void*)gv.scaled : (const void*)gv.plain, gv.minb);
        if (g_spmv > need_rows) g_spmv = need_rows > 0 ? need_rows : 1;
        const int need_vec = ((K->n + 4) / 5 + WPB - 1) / WPB;
        int g_vec = occ_grid(scaled ? (const void*)k_s_update : (const void*)k_g_update, 8);
        if (g_vec > need_vec) g_vec = need_vec > 0 ? need_vec : 1;
        int Gmax = g_spmv > g_vec ? g_spmv : g_vec;
        if (ilu_grid() > Gmax) Gmax = ilu_grid();
        int g_persist = 0;
        if (persist) {   // every CTA must be co-resident (cooperative launch)
            int per_sm = 0;
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, persist_kernel, DDA_THREADS, 0);
            if (per_sm > kSpLoopMinb) per_sm = kSpLoopMinb;
            if (per_sm < 1) per_sm = 1;   // (checked above)
            g_persist = cl ? kClCtas : device_sms() * per_sm;
            // small (L2-resident) systems are barrier-latency bound: no more CTAs than ten-row groups
            // need (DDA_PERSIST_CTAS overrides, tuning aid)
            const int cap = env_int("DDA_PERSIST_CTAS", need_rows > 0 ? need_rows : 1);
            if (cap > 0 && g_persist > cap) g_persist = cap;
            if (g_persist > Gmax) Gmax = g_persist;
        }
        const size_t bytes = (7 * N + 8 * (size_t)Gmax) * sizeof(double) + sizeof(CallArgs) + sizeof(State) + 64;
        // may reallocate the workspace (and drop any engine holding the old pointers): do it first
        dda_status_t s = ensure_workspace(K, bytes, st);
        if (s != DDA_OK) return s;
        G = new PcgGraph();
        G->pc = key;
        G->G_spmv = g_spmv;
        G->G_vec = g_vec;
        G->G_persist = g_persist;
        G->cluster = cl;
        double* ws = K->ws;
        GArgs& a = G->a;
        a.A = view_of(K);
        a.dinv = K->dinv;
        a.r = ws; a.z = ws + N; a.p0 = ws + 2 * N; a.p1 = ws + 3 * N; a.q = ws + 4 * N; a.t = ws + 5 * N;
        a.w = ws + 6 * N;
        a.part = ws + 7 * N;
        a.Gmax = Gmax;
        char* tail = reinterpret_cast<char*>(a.part + 8 * (size_t)Gmax);
        a.ca = reinterpret_cast<CallArgs*>(tail);
        a.st = reinterpret_cast<State*>(tail + ((sizeof(CallArgs) + 15) / 16) * 16);
        a.pc = (int)pc;
        a.out = reinterpret_cast<int*>(reinterpret_cast<char*>(K->scratch) + 128);
        a.use_cond = 1;
        a.ilu_up = K->ilu_up;
        a.ilu_inv = K->ilu_inv;
        a.ilu_flags_f = K->ilu_flags ? K->ilu_flags + K->n : nullptr;
        a.ilu_flags_b = K->ilu_flags ? K->ilu_flags + 2 * (size_t)K->n : nullptr;
        a.ilu_counters = K->ilu_flags ? K->ilu_flags + 3 * (size_t)K->n + 2 : nullptr;
        a.ilu_order = K->ilu_order;
        a.hist = K->hist;          // (the graph loop bakes it at capture: dda_pcg_set_history drops the engine)
        a.hist_cap = K->hist_cap;
        a.su = K->sc_upper;
        a.lfac = K->lfac;
        a.sfac = K->sfac;
        a.bj_w = K->bj_w;
        a.dinv_fmax = reinterpret_cast<const unsigned long long*>(reinterpret_cast<char*>(K->scratch) + 192);
        if (persist && lr) {
            a.lr = reinterpret_cast<double2*>(K->lr_buf);
            a.lr_off = K->lr_off;
            a.lr_cnt = reinterpret_cast<unsigned*>(reinterpret_cast<char*>(K->lr_buf) + K->lr_bytes);
        }
        G->g_ilu = ilu_grid();
        DDA_CK(cudaMemsetAsync(a.st, 0, sizeof(State), st));       // ticket = 0

        if (!persist) {   // persistent: no graph, k_sp_loop runs the whole loop
            // ---- the loop: a while conditional node whose body is captured from a stream
            DDA_CK(cudaGraphCreate(&G->graph, 0));
            DDA_CK(cudaGraphConditionalHandleCreate(&G->h, G->graph, 1, cudaGraphCondAssignDefault));
            cudaGraphNodeParams cp = {};
            cp.type = cudaGraphNodeTypeConditional;
            cp.conditional.handle = G->h;
            cp.conditional.type = cudaGraphCondTypeWhile;
            cp.conditional.size = 1;
            cudaGraphNode_t cnode;
            DDA_CK(cudaGraphAddNode(&cnode, G->graph, nullptr, 0, &cp));
            cudaGraph_t body = cp.conditional.phGraph_out[0];
            cudaStream_t cs;
            DDA_CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
            DDA_CK(cudaStreamBeginCaptureToGraph(cs, body, nullptr, nullptr, 0, cudaStreamCaptureModeThreadLocal));
            // body = two PCG iterations; kernels chained with programmatic dependent launch
            cudaLaunchAttribute pdl[1];
            pdl[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
            pdl[0].val.programmaticStreamSerializationAllowed = env_int("DDA_PDL", 1) ? 1 : 0;
            // iterations per while-loop pass (tuning aid); the kernels exit early once the loop is done
            int body_iters = env_int("DDA_BODY_ITERS", 2);
            if (body_iters < 1 || body_iters > 16) body_iters = 2;
            G->body_iters = body_iters;
            auto launch = [&](auto kern, int grid, auto... args) {
                cudaLaunchConfig_t cfg = {};
                cfg.gridDim = dim3(grid);
                cfg.blockDim = dim3(DDA_THREADS);
                cfg.stream = cs;
                cfg.attrs = pdl;
                cfg.numAttrs = 1;
                cudaLaunchKernelEx(&cfg, kern, args...);
            };
            for (int rep = 0; rep < body_iters; ++rep) {
                if (scaled) {
                    launch(gspmv_variant().scaled, G->G_spmv, a, G->h);
                    launch(k_s_update, G->G_vec, a, G->h);
                    launch(k_s_check, G->G_vec, a, G->h);
                    continue;
                }
                launch(gspmv_variant().plain, G->G_spmv, a, G->h);
                launch(k_g_update, G->G_vec, a, G->h);
                if (pc == DDA_PC_SSOR_AI) {
                    launch(k_g_ssor_lower<false>, G->G_spmv, a);
                    launch(k_g_ssor_upper<false>, G->G_spmv, a, G->h);
                } else if (pc == DDA_PC_ILU0) {
                    cudaMemsetAsync(a.ilu_flags_f, 0, 2 * (size_t)K->n * sizeof(int), cs);
                    cudaMemsetAsync(a.ilu_counters, 0, 2 * sizeof(int), cs);
                    k_g_ilu_fwd<false><<<G->g_ilu, DDA_THREADS, 0, cs>>>(a);
                    k_g_ilu_bwd<false><<<G->g_ilu, DDA_THREADS, 0, cs>>>(a, G->h);
                }
            }
            cudaError_t ce = cudaStreamEndCapture(cs, nullptr);
            cudaStreamDestroy(cs);
            if (ce != cudaSuccess) { dda_status_t s2 = cuda_fail(ce); pcg_graph_free(G); G = nullptr; return s2; }
            ce = cudaGraphInstantiate(&G->exec, G->graph, 0);
            if (ce != cudaSuccess) { dda_status_t s2 = cuda_fail(ce); pcg_graph_free(G); G = nullptr; return s2; }
        }
    }
    trace("solve: engine ready");
    GArgs& a = G->a;
    CallArgs hca{F, d0, d, tol, omega, maxit};
    DDA_CK(cudaMemcpyAsync(const_cast<CallArgs*>(a.ca), &hca, sizeof hca, cudaMemcpyHostToDevice, st));
    // ---- prelude
    if (d0) {
        k_g_spmv_x<true><<<G->G_spmv, DDA_THREADS, 0, st>>>(a);
        DDA_LAUNCHED();
    }
    if (scaled)
        k_s_init<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
    else
        k_g_init<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
    DDA_LAUNCHED();
    if (pc == DDA_PC_SSOR_AI && !scaled) {
        k_g_ssor_lower<true><<<G->G_spmv, DDA_THREADS, 0, st>>>(a);
        DDA_LAUNCHED();
        k_g_ssor_upper<true><<<G->G_spmv, DDA_THREADS, 0, st>>>(a, G->h);
        DDA_LAUNCHED();
    } else if (pc == DDA_PC_ILU0) {
        DDA_CK(cudaMemsetAsync(a.ilu_flags_f, 0, 2 * (size_t)K->n * sizeof(int), st));
        DDA_CK(cudaMemsetAsync(a.ilu_counters, 0, 2 * sizeof(int), st));
        k_g_ilu_fwd<true><<<G->g_ilu, DDA_THREADS, 0, st>>>(a);
        DDA_LAUNCHED();
        k_g_ilu_bwd<true><<<G->g_ilu, DDA_THREADS, 0, st>>>(a, G->h);
        DDA_LAUNCHED();
    }
    // ---- the device-side loop (its kernel launches are counted below from the iteration count)
    if (G->G_persist) {
        a.lr_discard = env_int("DDA_LR_DISCARD", 1) != 0;
        a.lr_sync = env_int("DDA_LR_SYNC", 0);
        a.trace = g_trace;
        a.trace_iters = g_trace_iters;
        a.hist = K->hist;
        a.hist_cap = K->hist_cap;
        if (G->cluster) {   // one cluster of kClCtas CTAs (co-scheduled by the hardware)
            cudaLaunchConfig_t cfg = {};
            cfg.gridDim = dim3(kClCtas);
            cfg.blockDim = dim3(kClThreads);
            cfg.stream = st;
            cudaLaunchAttribute at[1];
            at[0].id = cudaLaunchAttributeClusterDimension;
            at[0].val.clusterDim.x = kClCtas;
            at[0].val.clusterDim.y = 1;
            at[0].val.clusterDim.z = 1;
            cfg.attrs = at;
            cfg.numAttrs = 1;
            DDA_CK(cudaLaunchKernelEx(&cfg, k_sp_cg1_cl, a));
        } else {
            if (a.lr_cnt) {   // the push form's ready flags / step counters start at zero in every launch
                const int ngrp = (K->n + 9) / 10, W = G->G_persist * WPB;
                const int nc = a.lr_sync == 1 ? (ngrp + W - 1) / W : ngrp;
                DDA_CK(cudaMemsetAsync(a.lr_cnt, 0, sizeof(unsigned) * (size_t)nc, st));
                // tag mode: every entry starts with tag 0, the parity of no iteration of this launch
                // before the first (iteration k writes tag (k + 1) & 1)
                if (a.lr_sync == 3) DDA_CK(cudaMemsetAsync(a.lr, 0, K->lr_bytes, st));
            }
            void* kargs[] = {reinterpret_cast<void*>(&a)};
            DDA_CK(cudaLaunchCooperativeKernel(persist_kernel, dim3(G->G_persist),
                                               dim3(DDA_THREADS), kargs, 0, st));
        }
        DDA_LAUNCHED();
    } else {
        DDA_CK(cudaGraphLaunch(G->exec, st));
    }
    // ---- epilogue: [d = S^T x], true residual
    if (scaled) {
        k_s_final<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
        DDA_LAUNCHED();
    }
    k_g_spmv_x<false><<<G->G_spmv, DDA_THREADS, 0, st>>>(a);
    DDA_LAUNCHED();
    k_g_resid<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
    DDA_LAUNCHED();
    struct { int it, status; double rel; int checks, pad; } hres;
    DDA_CK(cudaMemcpyAsync(&hres, a.out, sizeof hres, cudaMemcpyDeviceToHost, st));
    trace("solve: all issued");
    DDA_CK(cudaStreamSynchronize(st));
    trace("solve: final sync");
    // loop body: k_g_spmv + k_g_update (+ 2 SSOR-AI halves or 2 ILU sweeps) per iteration, body_iters
    // iterations per pass; the body runs ceil(max(iterations, 1) / body_iters) times (once, as a no-op
    // pass, when the setup already decided the result); every kernel of a pass is launched
    const int per_it = (pc == DDA_PC_SSOR_AI || pc == DDA_PC_ILU0) ? 4 : (scaled ? 3 : 2);
    const int its = hres.it > 0 ? hres.it : 1;
    if (!G->G_persist) note_launch(per_it * G->body_iters * ((its + G->body_iters - 1) / G->body_iters));
    K->last_checks = scaled ? hres.checks : 0;
    if (iters) *iters = hres.it;
    if (rel_res) *rel_res = hres.rel;
    return (dda_status_t)hres.status;
}

}  // namespace dda

// Internal tuning hook (not part of include/dda.h): runs the setup of a BJ solve,
// then times `reps` direct launches of each loop-body kernel (outside the graph).
// ms[0] = k_g_spmv (fused, k >= 1), ms[1] = k_g_update.
extern "C" int dda__time_pcg_phases_ex(dda_matrix_t K, const double* F, double* d, int reps, float* ms, int scaled) {
    using namespace dda;
    cudaStream_t st = 0;
    int it = 0;
    double rr = 0;
    if (!K->dinv_valid && bj_setup(K, st, nullptr) != DDA_OK) return -1;
    // reps < 0: build the engine with a zero-iteration solve (the loop body never runs inside the
    // graph), then time |reps| phase pairs launched directly (compute-sanitizer triage)
    const int maxit0 = reps < 0 ? 0 : 3;
    if (reps < 0) reps = -reps;
    if (pcg_graph_solve(K, F, nullptr, d, 1e-10, maxit0, DDA_PC_BJ, 1.0, &it, &rr, st, scaled != 0) < 0) return -2;
    PcgGraph* G = reinterpret_cast<PcgGraph*>(K->graph_engine);
    GArgs a = G->a;
    a.use_cond = 0;
    // re-run the setup so the state is "in the loop"
    CallArgs hca{F, nullptr, d, 1e-300, 1.0, 1 << 30};
    cudaMemcpy(const_cast<CallArgs*>(a.ca), &hca, sizeof hca, cudaMemcpyHostToDevice);
    if (scaled)
        k_s_init<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
    else
        k_g_init<<<G->G_vec, DDA_THREADS, 0, st>>>(a);
    int one = 1;
    cudaMemcpy(&a.st->k, &one, sizeof(int), cudaMemcpyHostToDevice);
    cudaEvent_t e0, e1, e2;
    cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventCreate(&e2);
    float t_spmv = 0, t_upd = 0;
    for (int r = 0; r < reps; ++r) {
        cudaMemcpy(&a.st->k, &one, sizeof(int), cudaMemcpyHostToDevice);   // stay on the fused path
        cudaEventRecord(e0, st);
        if (scaled)
            gspmv_variant().scaled<<<G->G_spmv, DDA_THREADS, 0, st>>>(a, 0);
        else
            gspmv_variant().plain<<<G->G_spmv, DDA_THREADS, 0, st>>>(a, 0);
        cudaEventRecord(e1, st);
        if (scaled)
            k_s_update<<<G->G_vec, DDA_THREADS, 0, st>>>(a, 0);
        else
            k_g_update<<<G->G_vec, DDA_THREADS, 0, st>>>(a, 0);
        cudaEventRecord(e2, st);
        cudaEventSynchronize(e2);
        float x, y;
        cudaEventElapsedTime(&x, e0, e1);
        cudaEventElapsedTime(&y, e1, e2);
        t_spmv += x; t_upd += y;
    }
    ms[0] = t_spmv / reps;
    ms[1] = t_upd / reps;
    cudaEventDestroy(e0); cudaEventDestroy(e1); cudaEventDestroy(e2);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

extern "C" int dda__time_pcg_phases(dda_matrix_t K, const double* F, double* d, int reps, float* ms) {
    return dda__time_pcg_phases_ex(K, F, d, reps, ms, 0);
}

// Internal query (not in include/dda.h): exact stopping tests (k_s_check passes) of the last
// scaled-engine solve on K (bench.py's algorithmic byte count).
extern "C" int dda__last_checks(dda_matrix_t K) { return K ? K->last_checks : -1; }

// Internal debugging hook (not in include/dda.h): copies the scaled-engine arrays to host
// buffers (any may be NULL): su [nnzb][36] tiled, lfac / sfac [n][24] packed lower.
extern "C" int dda__scaled_export(dda_matrix_t K, double* su, double* lfac, double* sfac) {
    using namespace dda;
    if (!K) return -1;
    if (!K->dinv_valid && bj_setup(K, 0, nullptr) != DDA_OK) return -2;
    if (scaled_setup(K, 0) != DDA_OK) return -3;
    if (cudaDeviceSynchronize() != cudaSuccess) return -4;
    if (su && K->nnzb) cudaMemcpy(su, K->sc_upper, sizeof(double) * kBlk * K->nnzb, cudaMemcpyDeviceToHost);
    if (lfac) cudaMemcpy(lfac, K->lfac, sizeof(double) * kDinv * K->n, cudaMemcpyDeviceToHost);
    if (sfac) cudaMemcpy(sfac, K->sfac, sizeof(double) * kDinv * K->n, cudaMemcpyDeviceToHost);
    return cudaGetLastError() == cudaSuccess ? 0 : -5;
}

// Internal testing hook (not in include/dda.h): the scaled engine's loop, 1 = persistent cooperative
// kernel, 0 = CUDA-graph while loop, -1 = DDA_SCALED_LOOP / default.  Engines cached on a matrix
// are keyed by the loop kind, so the next solve rebuilds as needed.
extern "C" void dda__set_scaled_loop(int v) { dda::g_scaled_loop = v; }
// Internal hook: k_sp_loop timeline buffer (device, [iters][G][4] u64: phase A start, phase A end,
// sigma known, phase B end), null = off.  Returns the persistent grid size of the cached engine
// (0 if none yet).
extern "C" int dda__set_loop_trace(dda_matrix_t K, unsigned long long* buf, int iters) {
    dda::g_trace = buf;
    dda::g_trace_iters = iters;
    dda::PcgGraph* G = K ? reinterpret_cast<dda::PcgGraph*>(K->graph_engine) : nullptr;
    return G ? G->G_persist : 0;
}

// Internal query: the scaled engine's loop driver the next solve uses (1 persistent, 0 graph).
extern "C" int dda__get_scaled_loop() {
    if (dda::g_scaled_loop < 0) {
        const char* e = getenv("DDA_SCALED_LOOP");
        return (e && (e[0] == 'g' || e[0] == '0')) ? 0 : 1;
    }
    return dda::g_scaled_loop;
}

// Internal timing hook (experiment): ms[0..3] = k_x_ks<LDG=1,3>, k_x_ks<0,3>, k_x_ks<1,4>, k_x_ks<0,4>
// (bare Ks products at 3 and 4 CTAs/SM) and ms[4] = the fused scaled k_g_spmv, averaged over reps.
extern "C" int dda__time_ks_variants(dda_matrix_t K, const double* F, double* d, int reps, float* ms) {
    using namespace dda;
    cudaStream_t st = 0;
    float dummy[2];
    if (dda__time_pcg_phases_ex(K, F, d, 1, dummy, 1) != 0) return -1;
    PcgGraph* G = reinterpret_cast<PcgGraph*>(K->graph_engine);
    GArgs a = G->a;
    a.use_cond = 0;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int g3 = device_sms() * 3, g4 = device_sms() * 4;
    for (int v = 0; v < 5; ++v) {
        float tot = 0;
        for (int r = 0; r < reps + 1; ++r) {
            cudaEventRecord(e0, st);
            if (v == 0) k_x_ks<true, 3><<<g3, DDA_THREADS, 0, st>>>(a);
            if (v == 1) k_x_ks<false, 3><<<g3, DDA_THREADS, 0, st>>>(a);
            if (v == 2) k_x_ks<true, 4><<<g4, DDA_THREADS, 0, st>>>(a);
            if (v == 3) k_x_ks<false, 4><<<g4, DDA_THREADS, 0, st>>>(a);
            if (v == 4) gspmv_variant().scaled<<<G->G_spmv, DDA_THREADS, 0, st>>>(a, 0);
            cudaEventRecord(e1, st);
            cudaEventSynchronize(e1);
            float x;
            cudaEventElapsedTime(&x, e0, e1);
            if (r) tot += x;
        }
        ms[v] = tot / reps;
    }
    cudaEventDestroy(e0); cudaEventDestroy(e1);
    return cudaGetLastError() == cudaSuccess ? 0 : -3;
}

// Residual history (dda.h): registered per matrix; a change drops the cached engine, whose CUDA graph
// bakes the pointer
extern "C" dda_status_t dda_pcg_set_history(dda_matrix_t K, double* buf, int32_t cap) {
    if (!K || cap < 0 || (buf == nullptr) != (cap == 0)) return DDA_ERR_ARG;
    if (K->hist != buf || K->hist_cap != cap) {
        if (K->graph_engine) {
            cudaDeviceSynchronize();
            dda::pcg_graph_free(K->graph_engine);
            K->graph_engine = nullptr;
        }
        K->hist = buf;
        K->hist_cap = cap;
    }
    return DDA_OK;
}
