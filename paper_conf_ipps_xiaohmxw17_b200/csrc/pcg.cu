// A5/A6 — the PCG solve of K d = F as ONE persistent cooperative kernel
// (§IV.A; textbook PCG, Saad Alg. 9.1, reading Z1/Z2/Z19).
//
// Per iteration k (block-Jacobi):
//   phase A  p^(k) = z + beta p^(k-1) formed on the fly for every gathered
//            neighbour and written by the owner of each row (the textbook
//            "phase C" fused into the SpMV, ping-pong p buffers), q = K p^(k),
//            CTA partial of p^T q
//   -- grid barrier --  sigma = fixed-order sum of the partials (every CTA)
//   phase B  alpha = rho/sigma; d += alpha p; r -= alpha q; z = D^{-1} r;
//            partials of r^T r and r^T z
//   -- grid barrier --  convergence test ||r|| <= tol ||F||, beta = rho'/rho
// Two grid barriers per iteration.  SSOR-AI inserts its two half-passes
// (lower on t = D^{-1} r, upper on w) after B, with a barrier after each.  Every CTA evaluates the scalars
// itself from the same partials in the same order, so all CTAs take the same
// branch and the result is bitwise reproducible for a given launch
// configuration.  The host reads the outcome once, after the kernel.
#include <cooperative_groups.h>

#include <cmath>
#include <cstdlib>

#include "precond_dev.cuh"

namespace cg = cooperative_groups;

namespace dda {
namespace {

constexpr int WPB = DDA_THREADS / 32;

struct PcgOut {
    int iters;
    int status;
    double rel_res;
    double rr;
    double FF;
};

struct PcgArgs {
    BsrView A;
    const double* __restrict__ dinv;
    const double* __restrict__ F;
    const double* d0;      // may be null; may alias d
    double* d;
    double* r;
    double* z;
    double* p;             // p buffer 0 (p^(k) lives in buffer k % 2)
    double* p1;            // p buffer 1
    double* q;
    double* t;
    double* w;
    double* part;          // [4][G] CTA partials
    PcgOut* out;
    int pc;
    double omega;
    double tol;
    int maxit;
};

// deterministic CTA reduction of NV values -> part[k*G + blockIdx.x]
template <int NV>
__device__ __forceinline__ void cta_partials(double (&v)[NV], double* part, int G, double (*red)[4]) {
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
#pragma unroll
    for (int k = 0; k < NV; ++k) v[k] = warp_sum(v[k]);
    if (lane == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) red[wib][k] = v[k];
    }
    cta_barrier();
    if (threadIdx.x < NV) {
        double s = 0.0;
        for (int w = 0; w < WPB; ++w) s += red[w][threadIdx.x];
        part[threadIdx.x * G + blockIdx.x] = s;
    }
    cta_barrier();
}

// fixed-order sum of part[k*G .. k*G+G) for k < NV, identical in every CTA
template <int NV>
__device__ __forceinline__ void grid_sums(const double* part, int G, double (&out)[NV], double* bc) {
    const int lane = threadIdx.x & 31;
    if ((threadIdx.x >> 5) == 0) {
#pragma unroll
        for (int k = 0; k < NV; ++k) {
            double s = 0.0;
            for (int j = lane; j < G; j += 32) s += ld_cg(part + k * G + j);
            s = warp_sum(s);
            if (lane == 0) bc[k] = s;
        }
    }
    cta_barrier();
#pragma unroll
    for (int k = 0; k < NV; ++k) out[k] = bc[k];
    cta_barrier();
}

// ---------------------------------------------------------------- phases
// Each phase is a separate non-inlined function so that the persistent kernel
// keeps one copy of each row loop and a small register footprint (40 registers:
// 6 CTAs x 8 warps per SM), instead of the union of all phases' live ranges.

__device__ __forceinline__ int warp_id_global() { return blockIdx.x * WPB + (threadIdx.x >> 5); }

// q = K x (all rows); returns this lane's share of x^T q when `dot`
__device__ __noinline__ double ph_spmv(const PcgArgs& P, const double* x, bool dot) {
    const int lane = threadIdx.x & 31;
    double acc = 0.0;
    for_rows<SPMV_FULL>(P.A, warp_id_global(), gridDim.x * WPB, XCg{x}, lane,
                        [&](int i, bool ok, double y0, double y1) {
                            if (ok && is_out_lane(lane)) {
                                const size_t o = 6 * (size_t)i + 2 * (q_of(lane) / 3);
                                *reinterpret_cast<double2*>(P.q + o) = make_double2(y0, y1);
                                if (dot) {
                                    const double2 xv = ld_cg2(x + o);
                                    acc += xv.x * y0 + xv.y * y1;
                                }
                            }
                        });
    return acc;
}

// x_j = z_j + beta * p_j formed on the fly (phase C fused into the next SpMV)
struct XFused {
    const double* z;
    const double* p;
    double beta;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        const size_t o = 6 * (size_t)vec + 2 * pair;
        const double2 zz = ld_cg2(z + o), pp = ld_cg2(p + o);
        return make_double2(fma(beta, pp.x, zz.x), fma(beta, pp.y, zz.y));
    }
};

// p_new = z + beta p_old (own rows, written), q = K p_new; returns this lane's share of p_new^T q
__device__ __noinline__ double ph_spmv_fused(const PcgArgs& P, const double* pold, double* pnew, double beta) {
    const int lane = threadIdx.x & 31;
    const XFused xf{P.z, pold, beta};
    double acc = 0.0;
    for_rows<SPMV_FULL>(P.A, warp_id_global(), gridDim.x * WPB, xf, lane,
                        [&](int i, bool ok, double y0, double y1) {
                            const int q = q_of(lane);
                            if (ok && is_out_lane(lane)) {
                                const size_t o = 6 * (size_t)i + 2 * (q / 3);
                                *reinterpret_cast<double2*>(P.q + o) = make_double2(y0, y1);
                                const double2 pv = xf(i, q / 3);
                                *reinterpret_cast<double2*>(pnew + o) = pv;
                                acc += pv.x * y0 + pv.y * y1;
                            }
                        });
    return acc;
}

// setup: d = d0 (or 0), r = F - q (or F), t/z/p = M^{-1} r pieces; partials (F^T F, r^T r, r^T z)
__device__ __noinline__ double3 ph_init(const PcgArgs& P) {
    const int lane = threadIdx.x & 31;
    const int n = P.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool use_dinv = (P.pc == DDA_PC_BJ || P.pc == DDA_PC_SSOR_AI);
    double FF = 0.0, rr = 0.0, rz = 0.0;
    for (int grp = warp_id_global(); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0, fv = 0.0;
        if (R.valid) {
            fv = P.F[R.idx];
            const double dv = P.d0 ? ld_cg(P.d0 + R.idx) : 0.0;
            if (P.d != P.d0) P.d[R.idx] = dv;
            rv = P.d0 ? fv - ld_cg(P.q + R.idx) : fv;
            P.r[R.idx] = rv;
        }
        FF += fv * fv;
        rr += rv * rv;
        const double tz = use_dinv ? bj_lane(P.dinv, R, rv) : rv;
        if (R.valid) {
            if (P.pc == DDA_PC_SSOR_AI) {
                P.t[R.idx] = tz;
            } else {
                P.z[R.idx] = tz;
                P.p[R.idx] = tz;
                rz += rv * tz;
            }
        }
    }
    return make_double3(FF, rr, rz);
}

// phase B: d += alpha p; r -= alpha q; z = D^{-1} r (BJ) / t = D^{-1} r (SSOR) / z = r; partials (r^T r, r^T z)
__device__ __noinline__ double2 ph_update(const PcgArgs& P, const double* pk, double alpha) {
    const int lane = threadIdx.x & 31;
    const int n = P.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    const bool use_dinv = (P.pc == DDA_PC_BJ || P.pc == DDA_PC_SSOR_AI);
    double rr = 0.0, rz = 0.0;
    for (int grp = warp_id_global(); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        double rv = 0.0;
        if (R.valid) {
            const double pv = ld_cg(pk + R.idx);
            P.d[R.idx] = ld_cg(P.d + R.idx) + alpha * pv;
            rv = ld_cg(P.r + R.idx) - alpha * ld_cg(P.q + R.idx);
            P.r[R.idx] = rv;
        }
        rr += rv * rv;
        const double tz = use_dinv ? bj_lane(P.dinv, R, rv) : rv;
        if (R.valid) {
            if (P.pc == DDA_PC_SSOR_AI) {
                P.t[R.idx] = tz;
            } else {
                P.z[R.idx] = tz;
                rz += rv * tz;
            }
        }
    }
    return make_double2(rr, rz);
}

// phase C (unfused variant): p = z + beta p
__device__ __noinline__ void ph_p(const PcgArgs& P, double beta) {
    const int lane = threadIdx.x & 31;
    const int n = P.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    for (int grp = warp_id_global(); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) P.p[R.idx] = fma(beta, ld_cg(P.p + R.idx), ld_cg(P.z + R.idx));
    }
}

// SSOR-AI lower half pass: w = D^{-1} (r - omega L t)
__device__ __noinline__ void ph_ssor_lower(const PcgArgs& P) {
    const int lane = threadIdx.x & 31;
    for_rows<SPMV_LOWER_T>(P.A, warp_id_global(), gridDim.x * WPB, XCg{P.t}, lane,
                           [&](int i, bool ok, double y0, double y1) {
                               ssor_lower_row(P.dinv, i, ok, y0, y1, P.r, P.omega, P.w, lane);
                           });
}

// SSOR-AI upper half pass: z = w - omega D^{-1} U w (and p = z at setup); returns r^T z share
__device__ __noinline__ double ph_ssor_upper(const PcgArgs& P, bool init) {
    const int lane = threadIdx.x & 31;
    double rz = 0.0;
    for_rows<SPMV_UPPER>(P.A, warp_id_global(), gridDim.x * WPB, XCg{P.w}, lane,
                         [&](int i, bool ok, double y0, double y1) {
                             const double zz = ssor_upper_row(P.dinv, i, ok, y0, y1, P.w, P.omega, lane);
                             if (ok && q_of(lane) < 6) {
                                 const size_t idx = 6 * (size_t)i + q_of(lane);
                                 P.z[idx] = zz;
                                 if (init) P.p[idx] = zz;
                                 rz += ld_cg(P.r + idx) * zz;
                             }
                         });
    return rz;
}

// true residual share: sum (F - q)^2 with q = K d
__device__ __noinline__ double ph_resid(const PcgArgs& P) {
    const int lane = threadIdx.x & 31;
    const int n = P.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    double acc = 0.0;
    for (int grp = warp_id_global(); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) {
            const double e = P.F[R.idx] - ld_cg(P.q + R.idx);
            acc += e * e;
        }
    }
    return acc;
}

__device__ __noinline__ void ph_zero_d(const PcgArgs& P) {
    const int lane = threadIdx.x & 31;
    const int n = P.A.n, ngrp = (n + 4) / 5, W = gridDim.x * WPB;
    for (int grp = warp_id_global(); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        if (R.valid) P.d[R.idx] = 0.0;
    }
}

template <int MINB, bool FUSED>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_pcg(const __grid_constant__ PcgArgs P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ double red[WPB][4];
    __shared__ double bc[4];
    const int G = gridDim.x;

    // ------------------------------------------------------------ setup: r = F - K d0
    if (P.d0) {
        ph_spmv(P, P.d0, false);
        grid.sync();
    }
    {
        const double3 v3 = ph_init(P);
        double v[3] = {v3.x, v3.y, v3.z};
        cta_partials<3>(v, P.part, G, red);
    }
    grid.sync();
    double FF, rr, rho;
    {
        double s[3];
        grid_sums<3>(P.part, G, s, bc);
        FF = s[0]; rr = s[1]; rho = s[2];
    }
    const double bnorm = sqrt(FF);
    int status = DDA_ERR_NO_CONVERGENCE;
    int iters = 0;
    bool skip_final = false;
    if (FF == 0.0) {                                    // reading Z2: d = 0, iters = 0, rel_res = 0
        ph_zero_d(P);
        status = DDA_OK;
        skip_final = true;
    } else if (sqrt(rr) <= P.tol * bnorm) {
        status = DDA_OK;
    } else {
        if (P.pc == DDA_PC_SSOR_AI) {
            grid.sync();                                // t visible; part[2G..] free again
            ph_ssor_lower(P);
            grid.sync();
            double v[1] = {ph_ssor_upper(P, true)};
            cta_partials<1>(v, P.part + 2 * G, G, red);
            grid.sync();
            double s[1];
            grid_sums<1>(P.part + 2 * G, G, s, bc);
            rho = s[0];
        }
        if (!(rho > 0.0) || !isfinite(rho)) {
            status = DDA_ERR_BREAKDOWN;
        } else {
            double beta = 0.0;
            for (int k = 0; k < P.maxit; ++k) {
                double* pk = (FUSED && (k & 1)) ? P.p1 : P.p;
                // ---- phase A: p^(k) = z + beta p^(k-1) (k > 0), q = K p^(k), partial p^T q
                {
                    double v[1] = {(k == 0 || !FUSED) ? ph_spmv(P, FUSED ? P.p : P.p, true)
                                                      : ph_spmv_fused(P, (k & 1) ? P.p : P.p1, pk, beta)};
                    cta_partials<1>(v, P.part, G, red);
                }
                grid.sync();
                double sigma;
                {
                    double s[1];
                    grid_sums<1>(P.part, G, s, bc);
                    sigma = s[0];
                }
                if (!(sigma > 0.0) || !isfinite(sigma)) { status = DDA_ERR_BREAKDOWN; break; }
                const double alpha = rho / sigma;
                // ---- phase B: d += alpha p; r -= alpha q; z = M^{-1} r (BJ / none) or t = D^{-1} r
                {
                    const double2 v2 = ph_update(P, pk, alpha);
                    double v[2] = {v2.x, v2.y};
                    cta_partials<2>(v, P.part + G, G, red);
                }
                grid.sync();
                double rz;
                {
                    double s[2];
                    grid_sums<2>(P.part + G, G, s, bc);
                    rr = s[0]; rz = s[1];
                }
                iters = k + 1;
                if (sqrt(rr) <= P.tol * bnorm) { status = DDA_OK; break; }
                if (P.pc == DDA_PC_SSOR_AI) {
                    ph_ssor_lower(P);
                    grid.sync();
                    double v[1] = {ph_ssor_upper(P, false)};
                    cta_partials<1>(v, P.part + 2 * G, G, red);
                    grid.sync();
                    double s[1];
                    grid_sums<1>(P.part + 2 * G, G, s, bc);
                    rz = s[0];
                }
                if (!(rz > 0.0) || !isfinite(rz)) { status = DDA_ERR_BREAKDOWN; break; }
                beta = rz / rho;
                rho = rz;
                if (!FUSED) {   // phase C: p = z + beta p (else fused into the next phase A)
                    ph_p(P, beta);
                    grid.sync();
                }
            }
        }
    }

    // ------------------------------------------------------------ true residual ||F - K d|| / ||F||
    double rel = 0.0;
    if (!skip_final) {
        grid.sync();
        ph_spmv(P, P.d, false);
        grid.sync();
        double v[1] = {ph_resid(P)};
        cta_partials<1>(v, P.part + 3 * G, G, red);
        grid.sync();
        double s[1];
        grid_sums<1>(P.part + 3 * G, G, s, bc);
        rel = sqrt(s[0]) / bnorm;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        P.out->iters = iters;
        P.out->status = status;
        P.out->rel_res = rel;
        P.out->rr = rr;
        P.out->FF = FF;
    }
}

typedef void (*PcgKernel)(const PcgArgs);
// occupancy variants (tuning aid, DDA_PCG_VARIANT): min CTAs of 256 threads per SM
const PcgKernel kPcgVariants[] = {k_pcg<5, true>, k_pcg<5, false>, k_pcg<6, true>, k_pcg<6, false>};

PcgKernel pcg_kernel() {
    static int v = -1;
    if (v < 0) {
        const char* e = getenv("DDA_PCG_VARIANT");
        v = e ? atoi(e) : 0;
        if (v < 0 || v > 3) v = 0;
    }
    return kPcgVariants[v];
}

int pcg_grid() {
    static int cached_dev = -1, cached = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev != cached_dev) {
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, pcg_kernel(), DDA_THREADS, 0);
        cached = device_sms() * (per_sm > 0 ? per_sm : 1);
        cached_dev = dev;
    }
    return cached;
}

}  // namespace

dda_status_t pcg_solve(dda_matrix* K, const double* F, const double* d0, double* d, double tol, int32_t maxit,
                       dda_precond_t pc, double omega, int32_t* iters, double* rel_res, cudaStream_t st) {
    if (iters) *iters = 0;
    if (rel_res) *rel_res = 0.0;
    if (!K || !F || !d || !(tol > 0.0) || maxit < 0) return DDA_ERR_ARG;
    if (pc != DDA_PC_NONE && pc != DDA_PC_BJ && pc != DDA_PC_SSOR_AI) return DDA_ERR_ARG;
    if ((pc == DDA_PC_BJ || pc == DDA_PC_SSOR_AI) && !K->dinv_valid) {
        dda_status_t s = bj_setup(K, st, nullptr);
        if (s != DDA_OK) return s;
    }
    const size_t N = 6 * (size_t)K->n;
    int G = pcg_grid();
    {   // fewer CTAs when the rows are few: grid barriers and partial sums scale with the CTA count
        static int cap = -1;
        if (cap < 0) {
            const char* e = getenv("DDA_PCG_GRID");
            cap = e ? atoi(e) : 0;
        }
        if (cap > 0 && cap < G) G = cap;
    }
    const int need = (K->n + 3 * WPB - 1) / (3 * WPB);
    if (need < G) G = need > 0 ? need : 1;
    const size_t bytes = (7 * N + 4 * (size_t)G) * sizeof(double);
    {
        dda_status_t s = ensure_workspace(K, bytes, st);
        if (s != DDA_OK) return s;
    }
    PcgArgs a;
    a.A = view_of(K);
    a.dinv = K->dinv;
    a.F = F;
    a.d0 = d0;
    a.d = d;
    a.r = K->ws;
    a.z = K->ws + N;
    a.p = K->ws + 2 * N;
    a.q = K->ws + 3 * N;
    a.t = K->ws + 4 * N;
    a.w = K->ws + 5 * N;
    a.p1 = K->ws + 6 * N;
    a.part = K->ws + 7 * N;
    a.out = reinterpret_cast<PcgOut*>(reinterpret_cast<char*>(K->scratch) + 64);
    a.pc = (int)pc;
    a.omega = omega;
    a.tol = tol;
    a.maxit = maxit;
    void* args[] = {&a};
    DDA_CK(cudaLaunchCooperativeKernel((const void*)pcg_kernel(), dim3(G), dim3(DDA_THREADS), args, 0, st));
    note_launch();
    PcgOut h;
    DDA_CK(cudaMemcpyAsync(&h, a.out, sizeof h, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    if (iters) *iters = h.iters;
    if (rel_res) *rel_res = h.rel_res;
    return (dda_status_t)h.status;
}

}  // namespace dda

using namespace dda;

// Engine choice: block-Jacobi and SSOR-AI run the scaled engine (pcg_graph.cu: PCG on S K S^T,
// same iterates, no D / D^{-1} in the loop) in one persistent cooperative kernel at every size: at
// 10k blocks (L2-resident, barrier-latency bound, grid capped to the rows) 9.8 us per iteration vs
// 15.0 for the unscaled persistent kernel; at 30k 15.8 vs 28.4; at 1M 304 vs 456.  ILU(0) and the
// unpreconditioned solve run the unscaled engines: the CUDA-graph while loop (ILU, and "none" from
// 64k blocks) or the persistent kernel on K ("none" below 64k).
// DDA_PCG_ENGINE=graph|persistent|scaled overrides.
static int g_forced_engine = -2;
// Internal testing hook (not in include/dda.h): -1 = automatic, 0 = graph, 1 = persistent, 2 = scaled.
extern "C" void dda__set_pcg_engine(int e) { g_forced_engine = e; }

static int pcg_engine(const dda_matrix* K, dda_precond_t pc) {   // 0 = graph, 1 = persistent, 2 = scaled
    int& forced = g_forced_engine;
    if (forced == -2) {
        const char* v = getenv("DDA_PCG_ENGINE");
        forced = !v ? -1 : ((v[0] == 'p' || v[0] == '1') ? 1 : ((v[0] == 's' || v[0] == '2') ? 2 : 0));
    }
    if (pc == DDA_PC_ILU0) return 0;   // the sync-free ILU sweeps exist in the graph engine only
    if (forced == 2) return (pc == DDA_PC_BJ || pc == DDA_PC_SSOR_AI) ? 2 : 0;
    if (forced >= 0) return forced;
    if (pc == DDA_PC_BJ || pc == DDA_PC_SSOR_AI) return 2;   // scaled engine at every size
    return (pc != DDA_PC_SSOR_AI && K->n < 65536) ? 1 : 0;
}

// Internal query (not in include/dda.h): the engine dda_pcg_solve would use (bench.py's byte accounting).
extern "C" int dda__pcg_engine(dda_matrix_t K, int pc) { return K ? pcg_engine(K, (dda_precond_t)pc) : -1; }

extern "C" dda_status_t dda_pcg_solve(dda_matrix_t K, const double* F, const double* d0, double* d, double tol,
                                      int32_t maxit, dda_precond_t pc, double omega, int32_t* iters,
                                      double* rel_res, void* stream) {
    DDA_NVTX("dda_pcg_solve");
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (!K) return DDA_ERR_ARG;
    if (K->rperm) return dda::ro_pcg(K, F, d0, d, tol, maxit, pc, omega, iters, rel_res, st);
    return dda::pcg_entry(K, F, d0, d, tol, maxit, pc, omega, iters, rel_res, st);
}

dda_status_t dda::pcg_entry(dda_matrix* K, const double* F, const double* d0, double* d, double tol, int32_t maxit,
                            dda_precond_t pc, double omega, int32_t* iters, double* rel_res, cudaStream_t st) {
    if (!K) return DDA_ERR_ARG;
    const int engine = pcg_engine(K, pc);
    if (engine == 1) return pcg_solve(K, F, d0, d, tol, maxit, pc, omega, iters, rel_res, st);
    if (iters) *iters = 0;
    if (rel_res) *rel_res = 0.0;
    if (!K || !F || !d || !(tol > 0.0) || maxit < 0) return DDA_ERR_ARG;
    if (pc != DDA_PC_NONE && pc != DDA_PC_BJ && pc != DDA_PC_SSOR_AI && pc != DDA_PC_ILU0) return DDA_ERR_ARG;
    if ((pc == DDA_PC_BJ || pc == DDA_PC_SSOR_AI) && !K->dinv_valid) {
        dda_status_t s = bj_setup(K, st, nullptr);
        if (s != DDA_OK) return s;
    }
    if (pc == DDA_PC_ILU0 && !K->ilu_valid) {
        dda_status_t s = ilu_setup(K, st, nullptr);
        if (s != DDA_OK) return s;
    }
    return pcg_graph_solve(K, F, d0, d, tol, maxit, pc, omega, iters, rel_res, st, engine == 2);
}

extern "C" dda_status_t dda_solve_host(int32_t n, const double* kdiag, int64_t m, const int32_t* bi,
                                       const int32_t* bj, const double* pen, const double* e, const double* g,
                                       const double* F, const double* d0, double* d, double tol, int32_t maxit,
                                       dda_precond_t pc, double omega, int32_t* iters, double* rel_res,
                                       void* stream) {
    DDA_NVTX("dda_solve_host");
    if (n <= 0 || m < 0 || !kdiag || !F || !d) return DDA_ERR_ARG;
    if (m > 0 && (!bi || !bj || !pen || !e || !g)) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const size_t N = 6 * (size_t)n;
    // one allocation, every sub-buffer 256-byte aligned (e, g need 16 B for the vector loads)
    auto up = [](size_t b) { return (b + 255) & ~(size_t)255; };
    const size_t sz[9] = {sizeof(double) * 36 * (size_t)n, sizeof(double) * N, sizeof(double) * N,
                          sizeof(double) * N, sizeof(double) * (size_t)m, sizeof(double) * 6 * (size_t)m,
                          sizeof(double) * 6 * (size_t)m, sizeof(int32_t) * (size_t)m, sizeof(int32_t) * (size_t)m};
    size_t off[10] = {0};
    for (int k = 0; k < 9; ++k) off[k + 1] = off[k] + up(sz[k] ? sz[k] : 1);
    char* buf = nullptr;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&buf), off[9], st));
    struct Free {
        char* b; cudaStream_t s;
        ~Free() { cudaStreamSynchronize(s); dev_free_on(b, s); }
    } fr{buf, st};
    double* dk = reinterpret_cast<double*>(buf + off[0]);
    double* dF = reinterpret_cast<double*>(buf + off[1]);
    double* dd0 = reinterpret_cast<double*>(buf + off[2]);
    double* dd = reinterpret_cast<double*>(buf + off[3]);
    double* dpen = reinterpret_cast<double*>(buf + off[4]);
    double* de = reinterpret_cast<double*>(buf + off[5]);
    double* dg = reinterpret_cast<double*>(buf + off[6]);
    int32_t* dbi = reinterpret_cast<int32_t*>(buf + off[7]);
    int32_t* dbj = reinterpret_cast<int32_t*>(buf + off[8]);
    // The key arrays (bi, bj, pen) go first on the caller's stream; e, g, kdiag (needed only by the
    // value step of the assembly) and F, d0 (needed by the solve) follow on a second stream, so their
    // transfer overlaps the key sorts.  The caller's stream waits on two events before using them.
    struct Aux {
        cudaStream_t cs = nullptr;
        cudaEvent_t vals = nullptr, rhs = nullptr, start = nullptr;
        ~Aux() {
            if (cs) { cudaStreamSynchronize(cs); cudaStreamDestroy(cs); }
            if (vals) cudaEventDestroy(vals);
            if (rhs) cudaEventDestroy(rhs);
            if (start) cudaEventDestroy(start);
        }
    } aux;
    DDA_CK(cudaStreamCreateWithFlags(&aux.cs, cudaStreamNonBlocking));
    DDA_CK(cudaEventCreateWithFlags(&aux.vals, cudaEventDisableTiming));
    DDA_CK(cudaEventCreateWithFlags(&aux.rhs, cudaEventDisableTiming));
    DDA_CK(cudaEventCreateWithFlags(&aux.start, cudaEventDisableTiming));
    DDA_CK(cudaEventRecord(aux.start, st));                 // the buffer is allocated stream-ordered on st
    DDA_CK(cudaStreamWaitEvent(aux.cs, aux.start, 0));
    if (m > 0) {
        DDA_CK(cudaMemcpyAsync(dbi, bi, sizeof(int32_t) * m, cudaMemcpyHostToDevice, st));
        DDA_CK(cudaMemcpyAsync(dbj, bj, sizeof(int32_t) * m, cudaMemcpyHostToDevice, st));
        DDA_CK(cudaMemcpyAsync(dpen, pen, sizeof(double) * m, cudaMemcpyHostToDevice, st));
        DDA_CK(cudaMemcpyAsync(de, e, sizeof(double) * 6 * m, cudaMemcpyHostToDevice, aux.cs));
        DDA_CK(cudaMemcpyAsync(dg, g, sizeof(double) * 6 * m, cudaMemcpyHostToDevice, aux.cs));
    }
    DDA_CK(cudaMemcpyAsync(dk, kdiag, sizeof(double) * 36 * (size_t)n, cudaMemcpyHostToDevice, aux.cs));
    DDA_CK(cudaEventRecord(aux.vals, aux.cs));
    DDA_CK(cudaMemcpyAsync(dF, F, sizeof(double) * N, cudaMemcpyHostToDevice, aux.cs));
    if (d0) DDA_CK(cudaMemcpyAsync(dd0, d0, sizeof(double) * N, cudaMemcpyHostToDevice, aux.cs));
    DDA_CK(cudaEventRecord(aux.rhs, aux.cs));
    dda_matrix_t K = nullptr;
    dda_status_t s = build_matrix_impl(n, dk, m, dbi, dbj, dpen, de, dg, st, aux.vals, &K);
    if (s != DDA_OK) return s;
    DDA_CK(cudaStreamWaitEvent(st, aux.rhs, 0));
    s = dda_pcg_solve(K, dF, d0 ? dd0 : nullptr, dd, tol, maxit, pc, omega, iters, rel_res, stream);
    if (s == DDA_OK || s == DDA_ERR_NO_CONVERGENCE || s == DDA_ERR_BREAKDOWN) {
        cudaError_t ce = cudaMemcpyAsync(d, dd, sizeof(double) * N, cudaMemcpyDeviceToHost, st);
        if (ce == cudaSuccess) ce = cudaStreamSynchronize(st);
        if (ce != cudaSuccess) s = cuda_fail(ce);
    }
    dda_matrix_free(K);
    return s;
}

// Streamed end-to-end batch (dda.h): system k+1's inputs go host->device on a copy stream into the
// free one of two input slots while system k is assembled and solved on the caller's stream; system
// k's d goes device->host on the copy stream behind its solve.  Events order the reuse: a slot is
// refilled only after the solve that read it (in_free), a result buffer is rewritten only after
// its device->host copy (out_free).
extern "C" dda_status_t dda_solve_host_batch(int32_t nsys, dda_host_system* sys, double tol, int32_t maxit,
                                             dda_precond_t pc, double omega, void* stream) {
    DDA_NVTX("dda_solve_host_batch");
    if (nsys < 0 || (nsys > 0 && !sys)) return DDA_ERR_ARG;
    int32_t nmax = 0;
    int64_t mmax = 0;
    for (int k = 0; k < nsys; ++k) {
        dda_host_system& S = sys[k];
        S.iters = 0;
        S.rel_res = 0.0;
        S.status = DDA_ERR_ARG;
        if (S.n_blocks <= 0 || S.n_springs < 0 || !S.kdiag || !S.F || !S.d) return DDA_ERR_ARG;
        if (S.n_springs > 0 && (!S.bi || !S.bj || !S.pen || !S.e || !S.g)) return DDA_ERR_ARG;
        nmax = S.n_blocks > nmax ? S.n_blocks : nmax;
        mmax = S.n_springs > mmax ? S.n_springs : mmax;
    }
    if (nsys == 0) return DDA_OK;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const size_t Nmax = 6 * (size_t)nmax;
    auto up = [](size_t b) { return (b + 255) & ~(size_t)255; };
    // slot layout: kdiag, F, d0, pen, e, g, bi, bj (every sub-buffer 256-byte aligned)
    const size_t sz[8] = {sizeof(double) * 36 * (size_t)nmax, sizeof(double) * Nmax, sizeof(double) * Nmax,
                          sizeof(double) * (size_t)mmax, sizeof(double) * 6 * (size_t)mmax,
                          sizeof(double) * 6 * (size_t)mmax, sizeof(int32_t) * (size_t)mmax,
                          sizeof(int32_t) * (size_t)mmax};
    size_t off[9] = {0};
    for (int q = 0; q < 8; ++q) off[q + 1] = off[q] + up(sz[q] ? sz[q] : 1);
    const size_t slot_bytes = off[8], res_bytes = up(sizeof(double) * Nmax);
    char* buf = nullptr;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&buf), 2 * slot_bytes + 2 * res_bytes, st));
    struct Res {
        char* b; cudaStream_t s; cudaStream_t cs = nullptr;
        cudaEvent_t ev[11] = {};
        ~Res() {
            if (cs) { cudaStreamSynchronize(cs); cudaStreamDestroy(cs); }
            cudaStreamSynchronize(s);
            for (cudaEvent_t e : ev) if (e) cudaEventDestroy(e);
            dev_free_on(b, s);
        }
    } res{buf, st};
    DDA_CK(cudaStreamCreateWithFlags(&res.cs, cudaStreamNonBlocking));
    for (cudaEvent_t& e : res.ev) DDA_CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    // per slot: keys (bi, bj, pen) landed / values (e, g, kdiag) landed / right-hand side (F, d0) landed;
    // the slot's inputs no longer read; the result buffer copied out
    cudaEvent_t start = res.ev[0], *keys_ready = res.ev + 1, *vals_ready = res.ev + 3, *rhs_ready = res.ev + 5,
                *in_free = res.ev + 7, *out_free = res.ev + 9;
    cudaStream_t cs = res.cs;
    DDA_CK(cudaEventRecord(start, st));                     // the buffer is allocated stream-ordered on st
    DDA_CK(cudaStreamWaitEvent(cs, start, 0));
    auto slot = [&](int k, int q) { return buf + (size_t)(k & 1) * slot_bytes + off[q]; };
    auto result = [&](int k) { return reinterpret_cast<double*>(buf + 2 * slot_bytes + (size_t)(k & 1) * res_bytes); };
    // copy order = use order: the key arrays first, so the assembly's key sorts start while the
    // 96 B / spring of e, g are still in flight (matters for the first system; later ones were copied
    // during the previous solve)
    auto copy_in = [&](int k) -> cudaError_t {
        const dda_host_system& S = sys[k];
        const size_t N = 6 * (size_t)S.n_blocks, m = (size_t)S.n_springs;
        cudaError_t e = k >= 2 ? cudaStreamWaitEvent(cs, in_free[k & 1], 0) : cudaSuccess;
        if (m > 0) {
            if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 6), S.bi, sizeof(int32_t) * m, cudaMemcpyHostToDevice, cs);
            if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 7), S.bj, sizeof(int32_t) * m, cudaMemcpyHostToDevice, cs);
            if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 3), S.pen, sizeof(double) * m, cudaMemcpyHostToDevice, cs);
        }
        if (e == cudaSuccess) e = cudaEventRecord(keys_ready[k & 1], cs);
        if (m > 0) {
            if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 4), S.e, sizeof(double) * 6 * m, cudaMemcpyHostToDevice, cs);
            if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 5), S.g, sizeof(double) * 6 * m, cudaMemcpyHostToDevice, cs);
        }
        if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 0), S.kdiag, sizeof(double) * 6 * N, cudaMemcpyHostToDevice, cs);
        if (e == cudaSuccess) e = cudaEventRecord(vals_ready[k & 1], cs);
        if (e == cudaSuccess) e = cudaMemcpyAsync(slot(k, 1), S.F, sizeof(double) * N, cudaMemcpyHostToDevice, cs);
        if (e == cudaSuccess && S.d0) e = cudaMemcpyAsync(slot(k, 2), S.d0, sizeof(double) * N, cudaMemcpyHostToDevice, cs);
        if (e == cudaSuccess) e = cudaEventRecord(rhs_ready[k & 1], cs);
        return e;
    };
    DDA_CK(copy_in(0));
    for (int k = 0; k < nsys; ++k) {
        dda_host_system& S = sys[k];
        if (k + 1 < nsys) DDA_CK(copy_in(k + 1));          // overlaps this system's assembly and solve
        DDA_CK(cudaStreamWaitEvent(st, keys_ready[k & 1], 0));
        if (k >= 2) DDA_CK(cudaStreamWaitEvent(st, out_free[k & 1], 0));
        const double* dk = reinterpret_cast<const double*>(slot(k, 0));
        dda_matrix_t K = nullptr;
        dda_status_t s = build_matrix_impl(S.n_blocks, dk, S.n_springs, reinterpret_cast<const int32_t*>(slot(k, 6)),
                                           reinterpret_cast<const int32_t*>(slot(k, 7)),
                                           reinterpret_cast<const double*>(slot(k, 3)),
                                           reinterpret_cast<const double*>(slot(k, 4)),
                                           reinterpret_cast<const double*>(slot(k, 5)), st, vals_ready[k & 1], &K);
        if (s != DDA_OK) { S.status = s; return s; }
        DDA_CK(cudaStreamWaitEvent(st, rhs_ready[k & 1], 0));
        s = dda_pcg_solve(K, reinterpret_cast<const double*>(slot(k, 1)),
                          S.d0 ? reinterpret_cast<const double*>(slot(k, 2)) : nullptr, result(k), tol, maxit, pc,
                          omega, &S.iters, &S.rel_res, stream);
        S.status = s;
        const bool solved = s == DDA_OK || s == DDA_ERR_NO_CONVERGENCE || s == DDA_ERR_BREAKDOWN;
        DDA_CK(cudaEventRecord(in_free[k & 1], st));        // the slot's inputs are no longer read
        if (solved) {
            DDA_CK(cudaStreamWaitEvent(cs, in_free[k & 1], 0));
            DDA_CK(cudaMemcpyAsync(S.d, result(k), sizeof(double) * 6 * (size_t)S.n_blocks, cudaMemcpyDeviceToHost, cs));
        }
        DDA_CK(cudaEventRecord(out_free[k & 1], cs));
        matrix_free_impl(K, &st);
        if (!solved) return s;
    }
    DDA_CK(cudaStreamSynchronize(cs));
    return DDA_OK;
}
