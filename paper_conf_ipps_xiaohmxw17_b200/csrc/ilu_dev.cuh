// A8 device routines shared by ilu.cu and the CUDA-graph PCG engine (see ilu.cu).
#pragma once
#include "precond_dev.cuh"

namespace dda {

__device__ __forceinline__ int ld_acquire(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
    asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void wait_ready(const int* flags, int k) {
    while (ld_acquire(flags + k) == 0) __nanosleep(32);
}
// next row in the schedule `order` (a topological order of the dependency DAG,
// levels ascending): rows are handed out in that order, so every dependency of a
// row was handed out earlier to a running warp (no deadlock) and the in-flight
// window covers whole wavefronts.  Returns n when the schedule is exhausted.
__device__ __forceinline__ int next_row(int* counter, const int* __restrict__ order, int n, int lane) {
    int r = n;
    if (lane == 0) {
        const int c = atomicAdd(counter, 1);
        r = c < n ? __ldg(order + c) : n;
    }
    return __shfl_sync(0xffffffffu, r, 0);
}

// ------------------------------------------------------------------ triangular sweeps

// One warp, one row: acc(pair) = sum over the row's block list of forward
// (chunk * x) or transposed (chunk^T * x) products; the three 9-lane groups take
// blocks g, g+3, ...; result in lanes 0..5 (one DOF each).
template <bool LOWER>
__device__ __forceinline__ double row_sum(const BsrView& A, const double* __restrict__ vals, int i,
                                          const double* x, const int* flags, int lane) {
    const unsigned full = 0xffffffffu;
    const int g = grp_of(lane), q = q_of(lane), R = q / 3, C = q - 3 * R;
    const int b0 = LOWER ? A.low_ptr[i] : A.row_ptr[i];
    const int nb = (LOWER ? A.low_ptr[i + 1] : A.row_ptr[i + 1]) - b0;
    const int* deps = LOWER ? A.low_row : A.col_idx;
    // first round of matrix chunks is independent of the dependencies: load it before waiting
    double4 a_pre = make_double4(0.0, 0.0, 0.0, 0.0);
    if (lane < 27 && g < nb)
        a_pre = ld_chunk(vals + (size_t)kBlk * (LOWER ? A.low_to_up[b0 + g] : b0 + g) + 4 * (LOWER ? 3 * C + R : q));
    // the dependencies are polled in parallel, one lane each (a sequential poll costs one L2 round
    // trip per dependency even when all are ready)
    for (int b = lane; b < nb; b += 32) wait_ready(flags, deps[b0 + b]);
    __syncwarp();
    double f0 = 0.0, f1 = 0.0;
    for (int b = g; b < nb + 2; b += 3) {       // every lane iterates equally (nb + 2 >= g)
        const bool act = lane < 27 && b < nb;
        int blk = 0, vec = 0;
        if (act) {
            if (LOWER) {
                blk = A.low_to_up[b0 + b];
                vec = A.low_row[b0 + b];
            } else {
                blk = b0 + b;
                vec = A.col_idx[b0 + b];
            }
            const double4 a = (b == g) ? a_pre : ld_chunk(vals + (size_t)kBlk * blk + 4 * (LOWER ? 3 * C + R : q));
            const double2 xv = __ldcg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * C));
            const double m01 = LOWER ? a.z : a.y, m10 = LOWER ? a.y : a.z;
            f0 = fma(a.x, xv.x, fma(m01, xv.y, f0));
            f1 = fma(m10, xv.x, fma(a.w, xv.y, f1));
        }
    }
    // sum over groups into lanes 0..8, then over C into lanes 0,3,6
    const int s1 = (lane + 9) & 31, s2 = (lane + 18) & 31;
    double a0 = __shfl_sync(full, f0, s1), a1 = __shfl_sync(full, f1, s1);
    double c0 = __shfl_sync(full, f0, s2), c1 = __shfl_sync(full, f1, s2);
    f0 = (f0 + a0) + c0;
    f1 = (f1 + a1) + c1;
    const int n1 = (lane + 1) & 31, n2 = (lane + 2) & 31;
    a0 = __shfl_sync(full, f0, n1); a1 = __shfl_sync(full, f1, n1);
    c0 = __shfl_sync(full, f0, n2); c1 = __shfl_sync(full, f1, n2);
    const double y0 = (f0 + a0) + c0, y1 = (f1 + a1) + c1;
    const int a = lane < 6 ? lane : 0;
    const double lo = __shfl_sync(full, y0, 3 * (a >> 1)), hi = __shfl_sync(full, y1, 3 * (a >> 1));
    return (a & 1) ? hi : lo;
}

// row a = lane (lanes 0..5) of the tiled pivot inverse U_ii^{-1}: independent of the dependencies,
// so it is loaded before the warp waits for them (off the critical path of the sweep)
struct PivRow {
    double v[6];
};
__device__ __forceinline__ PivRow pivot_row(const double* __restrict__ Finv, int i, int lane) {
    const int a = lane < 6 ? lane : 0;
    PivRow p;
#pragma unroll
    for (int c = 0; c < 6; ++c) p.v[c] = __ldg(Finv + (size_t)kBlk * i + tile_off(a, c));
    return p;
}
// w_a = sum_c Finv_i[a][c] v_c, v on lanes 0..5
__device__ __forceinline__ double pivot_apply(const PivRow& F, double v) {
    double s = 0.0;
#pragma unroll
    for (int c = 0; c < 6; ++c) {
        const double vc = __shfl_sync(0xffffffffu, v, c);
        s = fma(F.v[c], vc, s);
    }
    return s;
}

// forward sweep: y = r - (strict lower) yh, yh = U_ii^{-1} y   (rows in forward-level order)
__device__ __forceinline__ void ilu_forward_rows(const BsrView& A, const double* Fup, const double* Finv, const double* r, double* y,
                                 double* yh, int* flags, int* counter, const int* order) {
    const int lane = threadIdx.x & 31;
    for (int i = next_row(counter, order, A.n, lane); i < A.n; i = next_row(counter, order, A.n, lane)) {
        const PivRow F = pivot_row(Finv, i, lane);
        const double ri = (lane < 6) ? r[6 * (size_t)i + lane] : 0.0;
        const double s = row_sum<true>(A, Fup, i, yh, flags, lane);
        const double yi = (lane < 6) ? ri - s : 0.0;
        const double hi = pivot_apply(F, yi);
        if (lane < 6) {
            y[6 * (size_t)i + lane] = yi;
            yh[6 * (size_t)i + lane] = hi;
        }
        __syncwarp();                       // the six stores of the row precede the release (st.release.gpu
        if (lane == 0) {                    // orders this thread's earlier writes; the warp's via __syncwarp
            __threadfence();                // plus this fence, which makes them visible at gpu scope)
            st_release(flags + i, 1);
        }
    }
}

// backward sweep: z = U_ii^{-1} (y - (strict upper) z)   (rows in backward-level order); returns r^T z share
__device__ __forceinline__ double ilu_backward_rows(const BsrView& A, const double* Fup, const double* Finv, const double* y,
                                    double* z, const double* r, double* p_init, int* flags, int* counter,
                                    const int* order) {
    const int lane = threadIdx.x & 31;
    double rz = 0.0;
    for (int i = next_row(counter, order, A.n, lane); i < A.n; i = next_row(counter, order, A.n, lane)) {
        const PivRow F = pivot_row(Finv, i, lane);
        const double yi = (lane < 6) ? y[6 * (size_t)i + lane] : 0.0;
        const double s = row_sum<false>(A, Fup, i, z, flags, lane);
        const double t = (lane < 6) ? yi - s : 0.0;
        const double zi = pivot_apply(F, t);
        if (lane < 6) {
            z[6 * (size_t)i + lane] = zi;
            if (p_init) p_init[6 * (size_t)i + lane] = zi;
            rz += r[6 * (size_t)i + lane] * zi;
        }
        __syncwarp();
        if (lane == 0) {
            __threadfence();
            st_release(flags + i, 1);
        }
    }
    return rz;
}


}  // namespace dda
