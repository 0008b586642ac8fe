// A4 — dda_spmv: standalone symmetric BSR6 SpMV launch (§IV.B).
//
// Grid = (#SMs x resident CTAs) persistent CTAs; warp w handles block rows
// w, w + W, w + 2W, ... so the whole grid sweeps the rows in increasing order
// and the transposed block V_ki needed by row i was streamed from HBM by the
// warp of row k a short time earlier (one course of the slope ~ 1-3 MB of
// traffic ago): it is re-read from the 126 MB L2, not from HBM.
#include <cstdlib>

#include "spmv_warp.cuh"

namespace dda {
namespace {

struct XLdg {
    const double* __restrict__ x;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
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

// occupancy variants for tuning (DDA_SPMV_VARIANT): min CTAs per SM of 256 threads
typedef void (*SpmvKernel)(BsrView, const double*, double*);
struct Variant { SpmvKernel k; const char* name; };
const Variant kVariants[] = {
    {k_spmv<SPMV_FULL, 6>, "b6"}, {k_spmv<SPMV_FULL, 4>, "b4"}, {k_spmv<SPMV_FULL, 8>, "b8"},
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

}  // namespace

dda_status_t spmv(dda_matrix* K, const double* x, double* y, cudaStream_t s) {
    const SpmvKernel k = kVariants[variant()].k;
    int g = spmv_grid(k);
    const int need = (K->n + 3 * (DDA_THREADS / 32) - 1) / (3 * (DDA_THREADS / 32));
    if (need < g) g = need > 0 ? need : 1;
    k<<<g, DDA_THREADS, 0, s>>>(view_of(K), x, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

}  // namespace dda

extern "C" dda_status_t dda_spmv(dda_matrix_t K, const double* x, double* y, void* stream) {
    if (!K || !x || !y || x == y) return DDA_ERR_ARG;
    return dda::spmv(K, x, y, reinterpret_cast<cudaStream_t>(stream));
}
