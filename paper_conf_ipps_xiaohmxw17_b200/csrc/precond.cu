// A3 — block-Jacobi construction (Table I "construction time" P:174) and
// standalone preconditioner application (A3/A7) for testing.
//
// BJ construction: per diagonal block, Cholesky D = L L^T (6 square roots),
// L^{-1} by forward substitution, D^{-1} = L^{-T} L^{-1}, stored as the packed
// upper triangle (21 doubles padded to 24 = 192 B).  One thread per block with
// everything in registers; ~250 flops against 288 B read + 192 B written, so
// the kernel is HBM-bound.  A non-positive or non-finite
// pivot reports DDA_ERR_NOT_SPD with the smallest offending block index.
#include <climits>

#include "precond_dev.cuh"

namespace dda {
namespace {

__global__ void __launch_bounds__(128) k_bj_inv(int32_t n, const double* __restrict__ diag, double* __restrict__ dinv,
                                                double* __restrict__ full, double* __restrict__ lfac,
                                                double* __restrict__ sfac, double* __restrict__ wlow,
                                                int* __restrict__ bad, unsigned long long* __restrict__ fnorm_max) {
    double fmax_local = 0.0;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double* D = diag + (size_t)kBlk * i;
        double A[6][6];
#pragma unroll
        for (int q = 0; q < 9; ++q) {
            const double4 v = ld_chunk(D + 4 * q);
            const int R = q / 3, C = q % 3;
            A[2 * R][2 * C] = v.x; A[2 * R][2 * C + 1] = v.y;
            A[2 * R + 1][2 * C] = v.z; A[2 * R + 1][2 * C + 1] = v.w;
        }
        double L[6][6];
        bool ok = true;
#pragma unroll
        for (int j = 0; j < 6; ++j) {
            double d = A[j][j];
#pragma unroll
            for (int k = 0; k < j; ++k) d -= L[j][k] * L[j][k];
            ok = ok && (d > 0.0) && isfinite(d);
            const double ljj = sqrt(d > 0.0 ? d : 1.0);
            L[j][j] = ljj;
            const double inv = 1.0 / ljj;
#pragma unroll
            for (int r = j + 1; r < 6; ++r) {
                double s = A[r][j];
#pragma unroll
                for (int k = 0; k < j; ++k) s -= L[r][k] * L[j][k];
                L[r][j] = s * inv;
            }
        }
        if (!ok) atomicMin(bad, (int)i);
        // Li = L^{-1} (lower triangular)
        double Li[6][6];
#pragma unroll
        for (int c = 0; c < 6; ++c) {
#pragma unroll
            for (int r = 0; r < 6; ++r) {
                if (r < c) { Li[r][c] = 0.0; continue; }
                double s = (r == c) ? 1.0 : 0.0;
#pragma unroll
                for (int k = c; k < r; ++k) s -= L[r][k] * Li[k][c];
                Li[r][c] = s / L[r][r];
            }
        }
        double* out = dinv + (size_t)kDinv * i;
        double P[24];
#pragma unroll
        for (int r = 0; r < 6; ++r)
#pragma unroll
            for (int c = r; c < 6; ++c) {
                double s = 0.0;
#pragma unroll
                for (int k = c; k < 6; ++k) s += Li[k][r] * Li[k][c];
                P[pk_off(r, c)] = s;
            }
        P[21] = P[22] = P[23] = 0.0;
        if (fnorm_max) {   // ||D_i^{-1}||_F >= 1 / lambda_min(D_i): the scaled engine's stopping-test bound
            double f2 = 0.0;
#pragma unroll
            for (int r = 0; r < 6; ++r)
#pragma unroll
                for (int c = r; c < 6; ++c) f2 += (r == c ? 1.0 : 2.0) * P[pk_off(r, c)] * P[pk_off(r, c)];
            fmax_local = fmax(fmax_local, ok ? sqrt(f2) : 0.0);
            if (wlow) {   // per-block lower bound of lambda_min(D_i) = 1 / ||D_i^{-1}||_2 (scaled engine)
                double ninf = 0.0;
#pragma unroll
                for (int r = 0; r < 6; ++r) {
                    double s = 0.0;
#pragma unroll
                    for (int c = 0; c < 6; ++c) s += fabs(P[r <= c ? pk_off(r, c) : pk_off(c, r)]);
                    ninf = fmax(ninf, s);
                }
                const double nb = fmin(sqrt(f2), ninf);
                wlow[i] = (ok && nb > 0.0 && isfinite(nb)) ? 1.0 / nb : 0.0;
            }
        }
#pragma unroll
        for (int q = 0; q < 12; ++q) reinterpret_cast<double2*>(out)[q] = make_double2(P[2 * q], P[2 * q + 1]);
        if (lfac) {   // packed lower triangles of L and S = L^{-1} for the scaled BJ engine (pcg_graph.cu)
            double PL[24], PS[24];
#pragma unroll
            for (int r = 0; r < 6; ++r)
#pragma unroll
                for (int c = 0; c <= r; ++c) {
                    PL[lo_off(r, c)] = L[r][c];
                    PS[lo_off(r, c)] = Li[r][c];
                }
            PL[21] = PL[22] = PL[23] = PS[21] = PS[22] = PS[23] = 0.0;
            double* lo = lfac + (size_t)kDinv * i;
            double* so = sfac + (size_t)kDinv * i;
#pragma unroll
            for (int q = 0; q < 12; ++q) {
                reinterpret_cast<double2*>(lo)[q] = make_double2(PL[2 * q], PL[2 * q + 1]);
                reinterpret_cast<double2*>(so)[q] = make_double2(PS[2 * q], PS[2 * q + 1]);
            }
        }
        if (full) {
#pragma unroll
            for (int r = 0; r < 6; ++r)
#pragma unroll
                for (int c = 0; c < 6; ++c) full[36 * i + 6 * r + c] = P[r <= c ? pk_off(r, c) : pk_off(c, r)];
        }
    }
    if (fnorm_max) {   // one atomic per warp (positive doubles order like their bit patterns)
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) fmax_local = fmax(fmax_local, __shfl_xor_sync(0xffffffffu, fmax_local, o));
        if ((threadIdx.x & 31) == 0 && fmax_local > 0.0)
            atomicMax(fnorm_max, (unsigned long long)__double_as_longlong(fmax_local));
    }
}

__global__ void __launch_bounds__(DDA_THREADS) k_bj_apply(int32_t n, const double* __restrict__ dinv,
                                                          const double* __restrict__ r, double* __restrict__ z) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    const int ngrp = (n + 4) / 5;
    for (int grp = blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5); grp < ngrp; grp += W) {
        const Row5 R = row5(grp, lane, n);
        const double v = R.valid ? r[R.idx] : 0.0;
        const double zz = bj_lane(dinv, R, v);
        if (R.valid) z[R.idx] = zz;
    }
}

__global__ void __launch_bounds__(DDA_THREADS) k_ssor_lower(BsrView A, const double* __restrict__ dinv, double omega,
                                                            const double* r, const double* t, double* w) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    for_rows<SPMV_LOWER_T>(A, blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5), W, XCg{t}, lane,
                           [&](int i, bool ok, double y0, double y1) {
                               ssor_lower_row(dinv, i, ok, y0, y1, r, omega, w, lane);
                           });
}

__global__ void __launch_bounds__(DDA_THREADS) k_ssor_upper(BsrView A, const double* __restrict__ dinv, double omega,
                                                            const double* w, double* z) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    for_rows<SPMV_UPPER>(A, blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5), W, XCg{w}, lane,
                         [&](int i, bool ok, double y0, double y1) {
                             const double zz = ssor_upper_row(dinv, i, ok, y0, y1, w, omega, lane);
                             if (ok && q_of(lane) < 6) z[6 * (size_t)i + q_of(lane)] = zz;
                         });
}

int grid_rows(int rows_per_warp, int n) {
    const int warps = (n + rows_per_warp - 1) / rows_per_warp;
    int g = (warps + DDA_THREADS / 32 - 1) / (DDA_THREADS / 32);
    const int cap = device_sms() * 8;
    return g < 1 ? 1 : (g > cap ? cap : g);
}

}  // namespace

static dda_status_t bj_setup_n(dda_matrix* K, int32_t nrows, cudaStream_t st, int32_t* bad_block, double* full) {
    if (bad_block) *bad_block = -1;
    int* bad = reinterpret_cast<int*>(K->scratch);
    const int big = INT_MAX;
    DDA_CK(cudaMemcpyAsync(bad, &big, sizeof(int), cudaMemcpyHostToDevice, st));
    int g = (nrows + 127) / 128;
    const int cap = device_sms() * 16;
    if (g > cap) g = cap;
    if (!K->lfac) {
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->lfac), sizeof(double) * kDinv * (size_t)K->n, st));
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->sfac), sizeof(double) * kDinv * (size_t)K->n, st));
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->bj_w), sizeof(double) * (size_t)K->n, st));
    }
    K->scaled_valid = false;
    unsigned long long* fmax = reinterpret_cast<unsigned long long*>(reinterpret_cast<char*>(K->scratch) + 192);
    DDA_CK(cudaMemsetAsync(fmax, 0, sizeof(unsigned long long), st));
    k_bj_inv<<<g, 128, 0, st>>>(nrows, K->diag, K->dinv, full, K->lfac, K->sfac, K->bj_w, bad, fmax);
    DDA_LAUNCHED();
    int hbad = 0;
    DDA_CK(cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, st));
    trace("bj_setup: issued");
    DDA_CK(cudaStreamSynchronize(st));
    trace("bj_setup: sync");
    if (hbad != INT_MAX) {
        if (bad_block) *bad_block = hbad;
        K->dinv_valid = false;
        return DDA_ERR_NOT_SPD;
    }
    K->dinv_valid = nrows == K->n;
    return DDA_OK;
}

dda_status_t bj_setup(dda_matrix* K, cudaStream_t st, int32_t* bad_block, double* full) {
    return bj_setup_n(K, K->n, st, bad_block, full);
}
dda_status_t bj_setup(dda_matrix* K, cudaStream_t st, int32_t* bad_block) { return bj_setup(K, st, bad_block, nullptr); }
// block-Jacobi inverses of the first nrows blocks only (the own rows of a partition)
dda_status_t bj_setup_rows(dda_matrix* K, int32_t nrows, cudaStream_t st, int32_t* bad_block) {
    return bj_setup_n(K, nrows, st, bad_block, nullptr);
}

}  // namespace dda

using namespace dda;

extern "C" dda_status_t dda_bj_setup(dda_matrix_t K, double* dinv_full, int32_t* bad_block, void* stream) {
    DDA_NVTX("dda_bj_setup");
    if (!K) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    if (K->rperm) return ro_bj_setup(K, dinv_full, bad_block, st);
    return bj_setup(K, st, bad_block, dinv_full);
}

extern "C" dda_status_t dda_precond_apply(dda_matrix_t K, dda_precond_t pc, double omega, const double* r, double* z,
                                          void* stream) {
    DDA_NVTX("dda_precond_apply");
    if (!K || !r || !z || r == z) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    return K->rperm ? ro_precond(K, pc, omega, r, z, st) : dda::precond_apply(K, pc, omega, r, z, st);
}

dda_status_t dda::precond_apply(dda_matrix* K, dda_precond_t pc, double omega, const double* r, double* z,
                                cudaStream_t st) {
    const size_t N = 6 * (size_t)K->n;
    if (pc == DDA_PC_NONE) {
        DDA_CK(cudaMemcpyAsync(z, r, N * sizeof(double), cudaMemcpyDeviceToDevice, st));
        DDA_CK(cudaStreamSynchronize(st));
        return DDA_OK;
    }
    if (pc == DDA_PC_ILU0) {
        if (!K->ilu_valid) {
            dda_status_t s = ilu_setup(K, st, nullptr);
            if (s != DDA_OK) return s;
        }
        dda_status_t ws = ensure_workspace(K, 2 * N * sizeof(double), st);
        if (ws != DDA_OK) return ws;
        dda_status_t s = ilu_apply(K, r, z, K->ws, K->ws + N, st);
        if (s != DDA_OK) return s;
        DDA_CK(cudaStreamSynchronize(st));
        return DDA_OK;
    }
    if (pc != DDA_PC_BJ && pc != DDA_PC_SSOR_AI) return DDA_ERR_ARG;
    if (!K->dinv_valid) {
        dda_status_t s = bj_setup(K, st, nullptr);
        if (s != DDA_OK) return s;
    }
    if (pc == DDA_PC_BJ) {
        k_bj_apply<<<grid_rows(5, K->n), DDA_THREADS, 0, st>>>(K->n, K->dinv, r, z);
        DDA_LAUNCHED();
    } else {
        {
            dda_status_t ws = ensure_workspace(K, 2 * N * sizeof(double), st);
            if (ws != DDA_OK) return ws;
        }
        double* t = K->ws;
        double* w = K->ws + N;
        k_bj_apply<<<grid_rows(5, K->n), DDA_THREADS, 0, st>>>(K->n, K->dinv, r, t);
        DDA_LAUNCHED();
        k_ssor_lower<<<grid_rows(3, K->n), DDA_THREADS, 0, st>>>(view_of(K), K->dinv, omega, r, t, w);
        DDA_LAUNCHED();
        k_ssor_upper<<<grid_rows(3, K->n), DDA_THREADS, 0, st>>>(view_of(K), K->dinv, omega, w, z);
        DDA_LAUNCHED();
    }
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}
