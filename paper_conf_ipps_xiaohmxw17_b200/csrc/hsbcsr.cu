// NEXT-2 ablation — the paper's own SpMV, HSBCSR two-stage (§IV.B), built on
// B200 for the comparison P:222 reports (2.8x over cuSPARSE on the K40), next to dda_spmv.
//
// Storage (Fig. 6): d-data (diagonal blocks) and nd-data-up (upper off-diagonal blocks)
// in the "half slice" layout: the 6x6 blocks are cut into six slices by local row r; slice r holds
// row r (6 doubles) of every block in block order (row, then column), and each slice is padded to
// a multiple of 32 doubles (reading Z13).  Element (block b, row r, column c) sits at
// slice_stride * r + 6 b + c.  Indices: row-up-i / row-low-i / row-low-p are the
// matrix's row_ptr[1..] / low_ptr[1..] / low_to_up (the paper's packed rc is not needed: the
// block's row and column come from urow / col_idx).
//
// Two stages:
//   stage 1: every upper block b = (i, j) is applied to both vectors: up-res[b] = V_b x_j and
//            low-res[b] = V_b^T x_i (12 doubles written per block).  Six threads per block, thread
//            c owns column c and walks the slices: low-res[b][c] = sum_r V[r][c] x_i[r] accumulates
//            in its registers ("added up in the registers directly"); the products V[r][c] x_j[c]
//            are reduced over c in shared memory, thread r summing row r (Fig. 8).  Consecutive
//            threads read consecutive doubles of a slice (coalesced); x is read through the
//            read-only path (the paper's texture reads).
//   stage 2: y_i = D_i x_i + sum_{u in row i} up-res[u] + sum_{t in lower row i} low-res[row-low-p[t]]:
//            one thread per scalar row (i, r) (the paper's groups of 48 = 8 rows x 6 threads).
// Not atomic, deterministic; it moves the 96 B of up-res / low-res per block through memory twice
// (written, read), which the single-pass kernel of spmv_col.cuh avoids.
#include <vector>

#include "dda_internal.cuh"

struct dda_hsbcsr {
    dda_matrix* K = nullptr;
    int64_t dstride = 0, ustride = 0;   // slice lengths (doubles), multiples of 32
    double* ddata = nullptr;            // [6][dstride]
    double* ndup = nullptr;             // [6][ustride]
    double* upres = nullptr;            // [nnzb][6]
    double* lowres = nullptr;           // [nnzb][6]
};

namespace dda {
namespace {

constexpr int HS_BLOCKS = 32;           // upper blocks per CTA in stage 1 (6 threads each)

// tiled block layout (dda_internal.cuh) -> half-slice layout
__global__ void k_hs_slice(int64_t nb, int64_t stride, const double* __restrict__ tiled, double* __restrict__ sl) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nb * 36; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t b = t / 36;
        const int rc = (int)(t - 36 * b), r = rc / 6, c = rc - 6 * r;
        sl[stride * r + 6 * b + c] = tiled[36 * b + tile_off(r, c)];
    }
}

__global__ void __launch_bounds__(6 * HS_BLOCKS) k_hs_stage1(int64_t nnzb, int64_t stride,
                                                            const double* __restrict__ nd,
                                                            const int32_t* __restrict__ urow,
                                                            const int32_t* __restrict__ col,
                                                            const double* __restrict__ x, double* __restrict__ upres,
                                                            double* __restrict__ lowres) {
    __shared__ double prod[HS_BLOCKS][6][7];            // [block][row r][column c] (+1 pad: banks)
    const int lb = threadIdx.x / 6, c = threadIdx.x - 6 * lb;
    for (int64_t b0 = (int64_t)blockIdx.x * HS_BLOCKS; b0 < nnzb; b0 += (int64_t)gridDim.x * HS_BLOCKS) {
        const int64_t b = b0 + lb;
        const bool ok = b < nnzb;
        if (ok) {
            const int64_t i = urow[b], j = col[b];
            const double xjc = __ldg(x + 6 * j + c);
            double lr = 0.0;
#pragma unroll
            for (int r = 0; r < 6; ++r) {
                const double v = __ldg(nd + stride * r + 6 * b + c);
                lr = fma(v, __ldg(x + 6 * i + r), lr);
                prod[lb][r][c] = v * xjc;
            }
            lowres[6 * b + c] = lr;
        }
        __syncthreads();
        if (ok) {                                       // thread r = c reduces row r of the block
            const int r = c;
            double s = prod[lb][r][0];
#pragma unroll
            for (int k = 1; k < 6; ++k) s += prod[lb][r][k];
            upres[6 * b + r] = s;
        }
        __syncthreads();
    }
}

__global__ void k_hs_stage2(int32_t n, int64_t dstride, const double* __restrict__ dd,
                            const int32_t* __restrict__ row_ptr, const int32_t* __restrict__ low_ptr,
                            const int32_t* __restrict__ low_to_up, const double* __restrict__ x,
                            const double* __restrict__ upres, const double* __restrict__ lowres,
                            double* __restrict__ y) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < 6 * (int64_t)n;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t i = t / 6;
        const int r = (int)(t - 6 * i);
        double s = 0.0;
#pragma unroll
        for (int c = 0; c < 6; ++c) s = fma(__ldg(dd + dstride * r + 6 * i + c), __ldg(x + 6 * i + c), s);
        for (int32_t u = row_ptr[i]; u < row_ptr[i + 1]; ++u) s += upres[6 * (int64_t)u + r];
        for (int32_t q = low_ptr[i]; q < low_ptr[i + 1]; ++q) s += lowres[6 * (int64_t)low_to_up[q] + r];
        y[t] = s;
    }
}

inline int hgrid(int64_t items, int tpb) {
    int64_t g = (items + tpb - 1) / tpb;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 16;
    return (int)(g < cap ? g : cap);
}

}  // namespace
}  // namespace dda

extern "C" void dda_hsbcsr_free(dda_hsbcsr_t H) {
    if (!H) return;
    cudaDeviceSynchronize();
    for (void* p : {(void*)H->ddata, (void*)H->ndup, (void*)H->upres, (void*)H->lowres})
        if (p) dda::dev_free(p);
    delete H;
}

extern "C" dda_status_t dda_hsbcsr_build(dda_matrix_t K, void* stream, dda_hsbcsr_t* out) {
    DDA_NVTX("dda_hsbcsr_build");
    using namespace dda;
    if (!out) return DDA_ERR_ARG;
    *out = nullptr;
    if (!K || K->rperm) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    dda_hsbcsr* H = new dda_hsbcsr();
    H->K = K;
    H->dstride = ((6 * (int64_t)K->n + 31) / 32) * 32;
    H->ustride = ((6 * K->nnzb + 31) / 32) * 32;
    const size_t z = (size_t)(K->nnzb > 0 ? K->nnzb : 1);
    cudaError_t e = dev_alloc(reinterpret_cast<void**>(&H->ddata), 6 * H->dstride * sizeof(double), st);
    if (e == cudaSuccess) e = dev_alloc(reinterpret_cast<void**>(&H->ndup), 6 * (H->ustride > 0 ? H->ustride : 32) * sizeof(double), st);
    if (e == cudaSuccess) e = dev_alloc(reinterpret_cast<void**>(&H->upres), 6 * z * sizeof(double), st);
    if (e == cudaSuccess) e = dev_alloc(reinterpret_cast<void**>(&H->lowres), 6 * z * sizeof(double), st);
    if (e != cudaSuccess) {
        dda_hsbcsr_free(H);
        return cuda_fail(e);
    }
    cudaMemsetAsync(H->ddata, 0, 6 * H->dstride * sizeof(double), st);   // padding
    k_hs_slice<<<hgrid(36 * (int64_t)K->n, 256), 256, 0, st>>>(K->n, H->dstride, K->diag, H->ddata);
    note_launch();
    if (K->nnzb > 0) {
        cudaMemsetAsync(H->ndup, 0, 6 * H->ustride * sizeof(double), st);
        k_hs_slice<<<hgrid(36 * K->nnzb, 256), 256, 0, st>>>(K->nnzb, H->ustride, K->upper, H->ndup);
        note_launch();
    }
    e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
        dda_hsbcsr_free(H);
        return cuda_fail(e);
    }
    *out = H;
    return DDA_OK;
}

extern "C" dda_status_t dda_hsbcsr_spmv(dda_hsbcsr_t H, const double* x, double* y, void* stream) {
    DDA_NVTX("dda_hsbcsr_spmv");
    using namespace dda;
    if (!H || !x || !y || x == y) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    dda_matrix* K = H->K;
    if (K->nnzb > 0) {
        k_hs_stage1<<<hgrid(K->nnzb, HS_BLOCKS), 6 * HS_BLOCKS, 0, st>>>(K->nnzb, H->ustride, H->ndup, K->urow,
                                                                         K->col_idx, x, H->upres, H->lowres);
        DDA_LAUNCHED();
    }
    k_hs_stage2<<<hgrid(6 * (int64_t)K->n, 256), 256, 0, st>>>(K->n, H->dstride, H->ddata, K->row_ptr, K->low_ptr,
                                                               K->low_to_up, x, H->upres, H->lowres, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

extern "C" dda_status_t dda_hsbcsr_export(dda_hsbcsr_t H, double* d_data, double* nd_data_up, int64_t* strides) {
    if (!H) return DDA_ERR_ARG;
    if (strides) { strides[0] = H->dstride; strides[1] = H->ustride; }
    if (cudaDeviceSynchronize() != cudaSuccess) return DDA_ERR_CUDA;
    if (d_data && cudaMemcpy(d_data, H->ddata, 6 * H->dstride * sizeof(double), cudaMemcpyDeviceToHost) != cudaSuccess)
        return DDA_ERR_CUDA;
    if (nd_data_up && H->ustride > 0 &&
        cudaMemcpy(nd_data_up, H->ndup, 6 * H->ustride * sizeof(double), cudaMemcpyDeviceToHost) != cudaSuccess)
        return DDA_ERR_CUDA;
    return DDA_OK;
}
