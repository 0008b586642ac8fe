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
#include <nccl.h>

#include <cmath>
#include <cstring>
#include <vector>

#include "precond_dev.cuh"
#include "spmv_col.cuh"

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
    __syncthreads();
    if (threadIdx.x == 0) {
        double s = 0.0;
        for (int w = 0; w < WPB; ++w) s += red[w];
        part[k * slot_stride + blockIdx.x] = s;
    }
    __syncthreads();
}

__global__ void k_pack(int n_send, const int* __restrict__ idx, const double* __restrict__ x, double* __restrict__ buf) {
    for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < 6 * n_send; t += gridDim.x * blockDim.x)
        buf[t] = x[6 * (size_t)idx[t / 6] + t % 6];
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
        __syncthreads();
        for (int h = blockDim.x / 2; h > 0; h >>= 1) {
            if (threadIdx.x < h) red[threadIdx.x] += red[threadIdx.x + h];
            __syncthreads();
        }
        if (threadIdx.x == 0) out[k] = red[0];
        __syncthreads();
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
    int G_spmv = 0, G_vec = 0, G_spmv2 = 0;
};

struct dda_comm {
    bool loopback = false;
    int nranks = 1, rank = 0;    // NCCL: world; loopback: nranks = partitions, rank unused
    ncclComm_t nccl = nullptr;
    std::vector<DistPart> parts;
};

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

extern "C" void dda_comm_free(dda_comm_t c) {
    if (!c) return;
    cudaDeviceSynchronize();
    for (DistPart& p : c->parts) {
        void* ptrs[] = {p.send_idx, p.sendbuf, p.x, p.q, p.r, p.z, p.part, p.scal, p.red, p.dst,
                        (void*)p.scal_ptrs};
        for (void* v : ptrs)
            if (v) dev_free(v);
    }
    if (c->nccl) ncclCommDestroy(c->nccl);
    delete c;
}

extern "C" dda_status_t dda_dist_attach(dda_comm_t c, int32_t part, dda_matrix_t K, int32_t n_own,
                                        const int32_t* send_counts, const int32_t* send_idx,
                                        const int32_t* recv_counts, void* stream) {
    if (!c || !K || !send_counts || !recv_counts) return DDA_ERR_ARG;
    const int P = c->nranks;
    const int slot = c->loopback ? part : 0;
    if (slot < 0 || slot >= (int)c->parts.size() || n_own < 1 || n_own > K->n) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    DistPart& D = c->parts[slot];
    if (D.K) {                                   // re-attach (e.g. a rebuilt matrix): release the old buffers
        cudaStreamSynchronize(st);
        void* ptrs[] = {D.send_idx, D.sendbuf, D.x, D.q, D.r, D.z, D.part, D.scal, D.red, D.dst,
                        (void*)D.scal_ptrs};
        for (void* v : ptrs)
            if (v) dev_free(v);
        D = DistPart();
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
    int Gm = D.G_spmv > D.G_vec ? D.G_spmv : D.G_vec;
    if (D.G_spmv2 > Gm) Gm = D.G_spmv2;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.send_idx), (D.n_send + 1) * sizeof(int), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.sendbuf), (6 * (size_t)D.n_send + 1) * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.x), nl6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.q), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.r), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.z), no6 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.part), 3 * (size_t)Gm * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.scal), 8 * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.red), 8 * sizeof(double), st));
    DDA_CK(dev_alloc(&D.dst, sizeof(DState), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&D.scal_ptrs), (P + 1) * sizeof(double*), st));
    if (D.n_send)
        DDA_CK(cudaMemcpyAsync(D.send_idx, send_idx, D.n_send * sizeof(int), cudaMemcpyHostToDevice, st));
    DDA_CK(cudaMemsetAsync(D.x, 0, nl6 * sizeof(double), st));
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

namespace {

// fill x[n_own:] of every local partition from the peers' own rows
dda_status_t halo_exchange(dda_comm* c, cudaStream_t st) {
    const int P = c->nranks;
    for (DistPart& D : c->parts) {
        if (D.n_send) {
            k_pack<<<(6 * D.n_send + 255) / 256 < 1024 ? (6 * D.n_send + 255) / 256 : 1024, 256, 0, st>>>(
                D.n_send, D.send_idx, D.x, D.sendbuf);
            DDA_LAUNCHED();
        }
    }
    if (c->loopback) {
        for (int p = 0; p < P; ++p)
            for (int q = 0; q < P; ++q) {
                if (p == q) continue;
                DistPart& S = c->parts[p];
                DistPart& R = c->parts[q];
                if (S.send_counts[q] != R.recv_counts[p]) return DDA_ERR_ARG;
                if (!S.send_counts[q]) continue;
                DDA_CK(cudaMemcpyAsync(R.x + 6 * ((size_t)R.n_own + R.recv_off[p]), S.sendbuf + 6 * (size_t)S.send_off[q],
                                       6 * sizeof(double) * S.send_counts[q], cudaMemcpyDeviceToDevice, st));
            }
        return DDA_OK;
    }
    DistPart& D = c->parts[0];
    DDA_NCCL(ncclGroupStart());
    for (int q = 0; q < P; ++q) {
        if (q == c->rank) continue;
        if (D.send_counts[q])
            DDA_NCCL(ncclSend(D.sendbuf + 6 * (size_t)D.send_off[q], 6 * (size_t)D.send_counts[q], ncclDouble, q,
                              c->nccl, st));
        if (D.recv_counts[q])
            DDA_NCCL(ncclRecv(D.x + 6 * ((size_t)D.n_own + D.recv_off[q]), 6 * (size_t)D.recv_counts[q], ncclDouble, q,
                              c->nccl, st));
    }
    DDA_NCCL(ncclGroupEnd());
    return DDA_OK;
}

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
    if (c->nranks > 1) DDA_NCCL(ncclAllReduce(D.scal, D.scal, nv, ncclDouble, ncclSum, c->nccl, st));
    DDA_CK(cudaMemcpyAsync(out, D.scal, nv * sizeof(double), cudaMemcpyDeviceToHost, st));
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

extern "C" dda_status_t dda_pcg_solve_dist(dda_comm_t c, const double* const* F, const double* const* d0,
                                           double* const* d, double tol, int32_t maxit, dda_precond_t pc,
                                           int32_t* iters, double* rel_res, void* stream) {
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
