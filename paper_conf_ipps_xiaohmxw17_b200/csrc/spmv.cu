// A4 — dda_spmv: standalone symmetric BSR6 SpMV launch (§IV.B).
//
// Grid = (#SMs x resident CTAs) persistent CTAs; warp w handles block rows
// w, w + W, w + 2W, ... so the whole grid sweeps the rows in increasing order
// and the transposed block V_ki needed by row i was streamed from HBM by the
// warp of row k a short time earlier (one course of the slope ~ 1-3 MB of
// traffic ago): it is re-read from the 126 MB L2, not from HBM.
#include <cstdlib>

#include "spmv_col.cuh"

namespace dda {
namespace {

struct XLdg {
    const double* __restrict__ x;
    using Raw = double2;
    __device__ __forceinline__ Raw raw(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
    __device__ __forceinline__ double2 cook(const Raw& r) const { return r; }
    __device__ __forceinline__ double2 operator()(int vec, int pair) const { return raw(vec, pair); }
};

template <int MODE, int MINB>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_spmv(BsrView A, const double* __restrict__ x,
                                                            double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    auto st = [&](int i, bool ok, double y0, double y1) {
        if (ok && is_out_lane(lane))
            *reinterpret_cast<double2*>(y + 6 * (size_t)i + 2 * (q_of(lane) / 3)) = make_double2(y0, y1);
    };
    for_rows<MODE>(A, blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5), W, XLdg{x}, lane, st);
}

// column-pair map (spmv_col.cuh), 10 rows per warp; V4: block list decoded one block ahead
template <int MODE, int MINB, int V = 4>
__global__ void __launch_bounds__(DDA_THREADS, MINB) k_spmv3(BsrView A, const double* __restrict__ x,
                                                             double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    auto st = [&](int i, bool ok, double y0, double y1) {
        if (ok) *reinterpret_cast<double2*>(y + 6 * (size_t)i + 2 * ccol_of(lane)) = make_double2(y0, y1);
    };
    for_rows_c<MODE, V>(A, blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5), W, XLdg{x}, lane, st);
}

// kernel variants for tuning (DDA_SPMV_VARIANT).  Default: the column-pair map with look-ahead
// decode and two blocks in flight per lane (v5) at 3 CTAs/SM (no spills): 0.237 ms at 1M blocks =
// 83% of the measured HBM copy peak.  v4 (one block in flight) at 4 CTAs/SM: 0.252 ms; v3 (decode
// inside the loop) at 5 CTAs/SM: 0.269 ms; the 9-lane group map (g9-b6): 0.272 ms.
typedef void (*SpmvKernel)(BsrView, const double*, double*);
struct Variant { SpmvKernel k; const char* name; int rows_per_warp; };
const Variant kVariants[] = {
    {k_spmv3<SPMV_FULL, 3, 5>, "c5-b3", 10}, {k_spmv<SPMV_FULL, 6>, "g9-b6", 3}, {k_spmv3<SPMV_FULL, 4, 4>, "c4-b4", 10},
    {k_spmv3<SPMV_FULL, 5, 3>, "c3-b5", 10}, {k_spmv3<SPMV_FULL, 2, 5>, "c5-b2", 10},
};
constexpr int kNumVariants = sizeof(kVariants) / sizeof(kVariants[0]);

int variant() {
    static int v = -2;
    if (v == -2) {
        const char* e = getenv("DDA_SPMV_VARIANT");
        v = e ? atoi(e) : 0;
        if (v < 0 || v >= kNumVariants) v = 0;
    }
    return v;
}

int spmv_grid(SpmvKernel k) {
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k, DDA_THREADS, 0);
    return device_sms() * (per_sm > 0 ? per_sm : 1);
}

// Full-storage BSR6 expansion (configs[3] comparison): row i lists the lower blocks
// V_ki^T (k < i, ascending), D_i, then the upper blocks V_ij, all stored explicitly.
__global__ void k_full_ptr(int32_t n, const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ low_ptr,
                           int32_t* __restrict__ fptr) {
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i <= n; i += gridDim.x * blockDim.x)
        fptr[i] = row_ptr[i] + low_ptr[i] + i;
}

// one thread per (output block, entry chunk q)
__global__ void k_full_fill(int32_t n, BsrView A, const int32_t* __restrict__ fptr, int32_t* __restrict__ fcol,
                            double* __restrict__ fval) {
    const int64_t total = (int64_t)fptr[n] * 9;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t ob = t / 9;
        const int q = (int)(t - 9 * ob);
        // row of ob: binary search in fptr
        int lo = 0, hi = n - 1;
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (fptr[mid] <= ob) lo = mid; else hi = mid - 1;
        }
        const int i = lo;
        const int k = (int)(ob - fptr[i]);
        const int nl = A.low_ptr[i + 1] - A.low_ptr[i];
        const double* src;
        int col;
        bool tr = false;
        if (k < nl) {
            const int tt = A.low_ptr[i] + k;
            src = A.upper + (size_t)kBlk * A.low_to_up[tt];
            col = A.low_row[tt];
            tr = true;
        } else if (k == nl) {
            src = A.diag + (size_t)kBlk * i;
            col = i;
        } else {
            const int u = A.row_ptr[i] + (k - nl - 1);
            src = A.upper + (size_t)kBlk * u;
            col = A.col_idx[u];
        }
        if (q == 0) fcol[ob] = col;
        const int R = q / 3, C = q % 3;
        double4 v;
        if (!tr) {
            v = *reinterpret_cast<const double4*>(src + 4 * q);
        } else {                                   // chunk (R,C) of V^T = transpose of chunk (C,R) of V
            const double4 c = *reinterpret_cast<const double4*>(src + 4 * (3 * C + R));
            v = make_double4(c.x, c.z, c.y, c.w);
        }
        *reinterpret_cast<double4*>(fval + (size_t)kBlk * ob + 4 * q) = v;
    }
}

}  // namespace

dda_status_t spmv(dda_matrix* K, const double* x, double* y, cudaStream_t s) {
    const char* te = getenv("DDA_SPMV_TMA");
    if (te && te[0] == '1') return spmv_tma(K, x, y, s);
    const Variant& V = kVariants[variant()];
    const SpmvKernel k = V.k;
    int g = spmv_grid(k);
    const int rpb = V.rows_per_warp * (DDA_THREADS / 32);
    const int need = (K->n + rpb - 1) / rpb;
    if (need < g) g = need > 0 ? need : 1;
    k<<<g, DDA_THREADS, 0, s>>>(view_of(K), x, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

}  // namespace dda

// configs[3]: full-storage BSR6 SpMV (every off-diagonal block stored twice), built on first use
dda_status_t dda::spmv_full(dda_matrix* K, const double* x, double* y, cudaStream_t st) {
    if (!K->full_ptr) {
        // allocate into locals and publish only when all three exist (a partial expansion must not
        // be taken for a built one on the next call)
        const size_t nb = (size_t)K->n + 2 * (size_t)K->nnzb;
        int32_t *fp = nullptr, *fc = nullptr;
        double* fv = nullptr;
        cudaError_t e = dev_alloc(reinterpret_cast<void**>(&fp), ((size_t)K->n + 1) * sizeof(int32_t), st);
        if (e == cudaSuccess) e = dev_alloc(reinterpret_cast<void**>(&fc), nb * sizeof(int32_t), st);
        if (e == cudaSuccess) e = dev_alloc(reinterpret_cast<void**>(&fv), nb * kBlk * sizeof(double), st);
        if (e != cudaSuccess) {
            if (fp) dev_free_on(fp, st);
            if (fc) dev_free_on(fc, st);
            return cuda_fail(e);
        }
        k_full_ptr<<<(K->n + 256) / 256, 256, 0, st>>>(K->n, K->row_ptr, K->low_ptr, fp);
        DDA_LAUNCHED();
        k_full_fill<<<device_sms() * 8, 256, 0, st>>>(K->n, view_of(K), fp, fc, fv);
        DDA_LAUNCHED();
        K->full_ptr = fp;
        K->full_col = fc;
        K->full_val = fv;
    }
    BsrView F = view_of(K);
    F.row_ptr = K->full_ptr;
    F.col_idx = K->full_col;
    F.upper = K->full_val;
    const SpmvKernel k = k_spmv<SPMV_UPPER, 6>;
    int g = spmv_grid(k);
    const int need = (K->n + 3 * (DDA_THREADS / 32) - 1) / (3 * (DDA_THREADS / 32));
    if (need < g) g = need > 0 ? need : 1;
    k<<<g, DDA_THREADS, 0, st>>>(F, x, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

extern "C" dda_status_t dda_spmv_full(dda_matrix_t K, const double* x, double* y, void* stream) {
    DDA_NVTX("dda_spmv_full");
    if (!K || !x || !y || x == y) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    return K->rperm ? dda::ro_spmv(K, x, y, st, true) : dda::spmv_full(K, x, y, st);
}

extern "C" dda_status_t dda_spmv(dda_matrix_t K, const double* x, double* y, void* stream) {
    DDA_NVTX("dda_spmv");
    if (!K || !x || !y || x == y) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    return K->rperm ? dda::ro_spmv(K, x, y, st, false) : dda::spmv(K, x, y, st);
}
