// A4 — dda_spmv: standalone symmetric BSR6 SpMV launch (§IV.B).
//
// Grid = (#SMs x resident CTAs) persistent CTAs; warp w handles block rows
// w, w + W, w + 2W, ... so the whole grid sweeps the rows in increasing order
// and the transposed block V_ki needed by row i was streamed from HBM by the
// warp of row k a short time earlier (one course of the slope ~ 1-3 MB of
// traffic ago): it is re-read from the 126 MB L2, not from HBM.
#include "spmv_warp.cuh"

namespace dda {
namespace {

struct XLdg {
    const double* __restrict__ x;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
};

template <int MODE>
__global__ void __launch_bounds__(DDA_THREADS) k_spmv(BsrView A, const double* __restrict__ x,
                                                      double* __restrict__ y) {
    const int lane = threadIdx.x & 31;
    const int W = gridDim.x * (DDA_THREADS / 32);
    for (int i = blockIdx.x * (DDA_THREADS / 32) + (threadIdx.x >> 5); i < A.n; i += W) {
        double y0, y1;
        spmv_row<MODE>(A, i, XLdg{x}, lane, y0, y1);
        if (lane < 9 && (lane % 3) == 0)
            *reinterpret_cast<double2*>(y + 6 * (size_t)i + 2 * (lane / 3)) = make_double2(y0, y1);
    }
}

int spmv_grid() {
    static int cached_dev = -1, cached = 0;
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev != cached_dev) {
        int per_sm = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_spmv<SPMV_FULL>, DDA_THREADS, 0);
        cached = device_sms() * (per_sm > 0 ? per_sm : 1);
        cached_dev = dev;
    }
    return cached;
}

}  // namespace

dda_status_t spmv(dda_matrix* K, const double* x, double* y, cudaStream_t s) {
    int g = spmv_grid();
    const int need = (K->n + DDA_THREADS / 32 - 1) / (DDA_THREADS / 32);
    if (need < g) g = need > 0 ? need : 1;
    k_spmv<SPMV_FULL><<<g, DDA_THREADS, 0, s>>>(view_of(K), x, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

}  // namespace dda

extern "C" dda_status_t dda_spmv(dda_matrix_t K, const double* x, double* y, void* stream) {
    if (!K || !x || !y || x == y) return DDA_ERR_ARG;
    return dda::spmv(K, x, y, reinterpret_cast<cudaStream_t>(stream));
}
