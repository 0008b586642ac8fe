// A1/A2 — global stiffness matrix building and canonical export (§III.C).
//
// The paper resolves the write conflicts of assembly with sort + scan (Fig. 4,
// P:106): each contact computes its sub-matrix into array D, D is sorted by
// block number into SD, boundary flags di mark segment heads, a scan of di
// gives segment ids sd1 and ends sd2, and each sub-matrix is the sum of its
// segment; "all the sort and scan steps act on the block number and index; the
// data of a sub-matrix are moved only for assembly in the final step".
//
// B200 version, same steps, no atomics, no materialised D:
//   keys   (min(i,j), max(i,j)) packed into 64 bits; values = spring ids
//   sort   stable LSD radix sort of (key, s)           [the paper's ref [31]]
//   heads  di[t] = key[t] != key[t-1]; inclusive scan  [ref [30]] -> unique block ids
//   CSR    row_ptr by lower-bound fill over the sorted unique rows; col_idx
//   values one thread per (block, row r): the 6 entries of row r summed over
//          the segment in increasing spring index, products (p*e[r])*g[c]
//          rounded as written (__dmul_rn/__dadd_rn: bit-identical to the
//          definition, reading Z8)
//   diag   the 2m (spring, side) endpoint records stably sorted by block;
//          D_i = Kd_i (upper triangle) + the segment in spring order, mirrored
//   T-map  stable sort of the unique blocks by (col, row): low_ptr / low_row /
//          low_to_up = the paper's row-low-i / row-low-p
// The sort permutations are kept for value-only re-assembly (dda_update_values).
#include <cub/cub.cuh>

#include <climits>
#include <cmath>
#include <cstring>
#include <vector>

#include "dda_internal.cuh"

namespace dda {
namespace {

constexpr int TPB = 256;

inline int grid_for(int64_t items) {
    int64_t g = (items + TPB - 1) / TPB;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 32;
    return (int)(g < cap ? g : cap);
}

inline int bits_for(uint64_t maxval) {
    int b = 1;
    while (b < 64 && (maxval >> b) != 0) ++b;
    return b;
}

__global__ void k_keys(int32_t n, int64_t m, const int32_t* __restrict__ bi, const int32_t* __restrict__ bj,
                       const double* __restrict__ pen, uint64_t* __restrict__ key, int32_t* __restrict__ val,
                       uint8_t* __restrict__ orient, int* __restrict__ err) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < m; s += (int64_t)gridDim.x * blockDim.x) {
        const int32_t i = bi[s], j = bj[s];
        const double p = pen[s];
        const bool bad = i < 0 || i >= n || j < 0 || j >= n || i == j || !(p >= 0.0) || isinf(p);
        if (bad) atomicOr(err, 1);
        const uint64_t a = (uint64_t)(bad ? 0 : (i < j ? i : j));
        const uint64_t b = (uint64_t)(bad ? 0 : (i < j ? j : i));
        key[s] = a * (uint64_t)n + b;
        val[s] = (int32_t)s;
        orient[s] = (i < j) ? 1 : 0;
    }
}

__global__ void k_heads(int64_t m, const uint64_t* __restrict__ key, int32_t* __restrict__ flag) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x)
        flag[t] = (t == 0 || key[t] != key[t - 1]) ? 1 : 0;
}

// unique blocks: segment start, block row, block column
__global__ void k_unique(int32_t n, int64_t m, const uint64_t* __restrict__ key, const int32_t* __restrict__ uid,
                         int32_t* __restrict__ seg, int32_t* __restrict__ urow, int32_t* __restrict__ col) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x) {
        if (t == 0 || key[t] != key[t - 1]) {
            const int32_t u = uid[t] - 1;
            seg[u] = (int32_t)t;
            urow[u] = (int32_t)(key[t] / (uint64_t)n);
            col[u] = (int32_t)(key[t] % (uint64_t)n);
        }
    }
}

// ptr[v] = lower bound of v in the sorted array sk[0..cnt), v = 0..n
__global__ void k_bounds(int32_t n, int64_t cnt, const int32_t* __restrict__ sk, int32_t* __restrict__ ptr) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t <= cnt; t += (int64_t)gridDim.x * blockDim.x) {
        const int32_t prev = (t == 0) ? -1 : sk[t - 1];
        const int32_t cur = (t == cnt) ? n : sk[t];
        for (int32_t v = prev + 1; v <= cur; ++v) ptr[v] = (int32_t)t;
    }
}

// V_u: sum over the segment, in increasing spring index, of
//   (p*e[r])*g[c]  if i < j   (K_ij)      or      (p*e[c])*g[r]  if i > j   (K_ij^T)
// One thread per unique block with its 36 entries in registers: every spring of the
// segment is read once (pen, e row, g row: five 32 B sectors), instead of once per
// (block, row) thread.
__global__ void __launch_bounds__(128) k_offdiag(int64_t nnzb, const int32_t* __restrict__ seg,
                                                 const int32_t* __restrict__ perm, const uint8_t* __restrict__ orient,
                                                 const double* __restrict__ pen, const double* __restrict__ e,
                                                 const double* __restrict__ g, double* __restrict__ upper) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < nnzb; u += (int64_t)gridDim.x * blockDim.x) {
        double acc[6][6];
#pragma unroll
        for (int r = 0; r < 6; ++r)
#pragma unroll
            for (int c = 0; c < 6; ++c) acc[r][c] = 0.0;
        const int32_t t1 = seg[u + 1];
        for (int32_t t = seg[u]; t < t1; ++t) {
            const int64_t s = perm[t];
            const double p = pen[s];
            double es[6], gs[6];
#pragma unroll
            for (int k = 0; k < 3; ++k) {
                const double2 a = *reinterpret_cast<const double2*>(e + 6 * s + 2 * k);
                const double2 b = *reinterpret_cast<const double2*>(g + 6 * s + 2 * k);
                es[2 * k] = a.x; es[2 * k + 1] = a.y; gs[2 * k] = b.x; gs[2 * k + 1] = b.y;
            }
            if (orient[s]) {
#pragma unroll
                for (int r = 0; r < 6; ++r) {
                    const double pr = __dmul_rn(p, es[r]);
#pragma unroll
                    for (int c = 0; c < 6; ++c) acc[r][c] = __dadd_rn(acc[r][c], __dmul_rn(pr, gs[c]));
                }
            } else {
#pragma unroll
                for (int c = 0; c < 6; ++c) {
                    const double pc = __dmul_rn(p, es[c]);
#pragma unroll
                    for (int r = 0; r < 6; ++r) acc[r][c] = __dadd_rn(acc[r][c], __dmul_rn(pc, gs[r]));
                }
            }
        }
        double* B = upper + (size_t)kBlk * u;
#pragma unroll
        for (int q = 0; q < 9; ++q) {
            const int R = q / 3, C = q % 3;
            *reinterpret_cast<double4*>(B + 4 * q) =
                make_double4(acc[2 * R][2 * C], acc[2 * R][2 * C + 1], acc[2 * R + 1][2 * C], acc[2 * R + 1][2 * C + 1]);
        }
    }
}

// D_i: Kd_i's upper triangle, then the block's endpoint records in spring order
// (p*w[r])*w[c] for r <= c, mirrored.  One thread per block, 21 accumulators.
__global__ void __launch_bounds__(128) k_diag(int32_t n, const int32_t* __restrict__ dstart,
                                              const int32_t* __restrict__ dperm, const double* __restrict__ pen,
                                              const double* __restrict__ e, const double* __restrict__ g,
                                              const double* __restrict__ kdiag, double* __restrict__ diag) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double acc[6][6];
#pragma unroll
        for (int r = 0; r < 6; ++r)
#pragma unroll
            for (int c = 0; c < 6; ++c) acc[r][c] = (c >= r) ? kdiag[36 * i + 6 * r + c] : 0.0;
        const int32_t t1 = dstart[i + 1];
        for (int32_t t = dstart[i]; t < t1; ++t) {
            const int32_t v = dperm[t];
            const int64_t s = v >> 1;
            const double* wp = ((v & 1) ? g : e) + 6 * s;
            double w[6];
#pragma unroll
            for (int k = 0; k < 3; ++k) {
                const double2 a = *reinterpret_cast<const double2*>(wp + 2 * k);
                w[2 * k] = a.x; w[2 * k + 1] = a.y;
            }
            const double p = pen[s];
#pragma unroll
            for (int r = 0; r < 6; ++r) {
                const double pr = __dmul_rn(p, w[r]);
#pragma unroll
                for (int c = r; c < 6; ++c) acc[r][c] = __dadd_rn(acc[r][c], __dmul_rn(pr, w[c]));
            }
        }
        double* D = diag + (size_t)kBlk * i;
#pragma unroll
        for (int q = 0; q < 9; ++q) {
            const int R = q / 3, C = q % 3;
            double m[2][2];
#pragma unroll
            for (int a = 0; a < 2; ++a)
#pragma unroll
                for (int b = 0; b < 2; ++b) {
                    const int r = 2 * R + a, c = 2 * C + b;
                    m[a][b] = r <= c ? acc[r][c] : acc[c][r];
                }
            *reinterpret_cast<double4*>(D + 4 * q) = make_double4(m[0][0], m[0][1], m[1][0], m[1][1]);
        }
    }
}

__global__ void k_dkeys(int64_t m, const int32_t* __restrict__ bi, const int32_t* __restrict__ bj,
                        int32_t* __restrict__ dkey, int32_t* __restrict__ dval) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < m; s += (int64_t)gridDim.x * blockDim.x) {
        dkey[2 * s] = bi[s];
        dkey[2 * s + 1] = bj[s];
        dval[2 * s] = (int32_t)(2 * s);
        dval[2 * s + 1] = (int32_t)(2 * s + 1);
    }
}

__global__ void k_tkeys(int32_t n, int64_t nnzb, const int32_t* __restrict__ urow, const int32_t* __restrict__ col,
                        uint64_t* __restrict__ tkey, int32_t* __restrict__ tval) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < nnzb; u += (int64_t)gridDim.x * blockDim.x) {
        tkey[u] = (uint64_t)col[u] * (uint64_t)n + (uint64_t)urow[u];
        tval[u] = (int32_t)u;
    }
}

__global__ void k_tfill(int32_t n, int64_t nnzb, const uint64_t* __restrict__ tkey, int32_t* __restrict__ low_row,
                        int32_t* __restrict__ tcol) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nnzb; t += (int64_t)gridDim.x * blockDim.x) {
        low_row[t] = (int32_t)(tkey[t] % (uint64_t)n);
        tcol[t] = (int32_t)(tkey[t] / (uint64_t)n);
    }
}

// RAII for stream-ordered temporaries
struct Tmp {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit Tmp(cudaStream_t st) : s(st) {}
    template <class T>
    cudaError_t get(T** p, size_t count) {
        void* q = nullptr;
        cudaError_t e = dev_alloc(&q, count ? count * sizeof(T) : 16, s);
        if (e == cudaSuccess) ptrs.push_back(q);
        *p = reinterpret_cast<T*>(q);
        return e;
    }
    ~Tmp() {
        for (void* p : ptrs) dev_free_on(p, s);
    }
};

template <class T>
cudaError_t dmalloc(T** p, size_t count, cudaStream_t st) {
    return dev_alloc(reinterpret_cast<void**>(p), count ? count * sizeof(T) : 16, st);
}

}  // namespace

dda_status_t run_values(dda_matrix* K, const double* kdiag, const double* pen, const double* e, const double* g,
                        cudaStream_t st) {
    if (K->nnzb > 0) {
        const int gb = (int)((K->nnzb + 127) / 128);
        k_offdiag<<<gb, 128, 0, st>>>(K->nnzb, K->seg, K->perm, K->orient, pen, e, g, K->upper);
        DDA_LAUNCHED();
    }
    k_diag<<<(K->n + 127) / 128, 128, 0, st>>>(K->n, K->dstart, K->dperm, pen, e, g, kdiag, K->diag);
    DDA_LAUNCHED();
    K->dinv_valid = false;
    K->scaled_valid = false;
    K->ilu_valid = false;
    if (K->full_ptr) {                 // the full-storage copy holds the old values
        cudaStreamSynchronize(st);
        dev_free(K->full_ptr); dev_free(K->full_col); dev_free(K->full_val);
        K->full_ptr = nullptr; K->full_col = nullptr; K->full_val = nullptr;
    }
    return DDA_OK;
}

dda_status_t cuda_fail(cudaError_t e);

}  // namespace dda

using namespace dda;

extern "C" void dda_matrix_free(dda_matrix_t K) { dda::matrix_free_impl(K, nullptr); }

// sync == nullptr: device-wide synchronisation first (the ABI's rule: no stream may still use the
// arrays); else only that stream, the one every use of K was ordered on (dda_solve_host_batch, whose
// copy stream keeps running)
void dda::matrix_free_impl(dda_matrix_t K, cudaStream_t* sync) {
    if (!K) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(K->device);
    trace("free: enter");
    if (sync) cudaStreamSynchronize(*sync);
    else cudaDeviceSynchronize();
    trace("free: synchronized");
    if (K->graph_engine) pcg_graph_free(K->graph_engine);
    trace("free: engine freed");
    void* ptrs[] = {K->row_ptr, K->col_idx, K->low_ptr, K->low_row, K->low_to_up, K->urow, K->diag, K->upper,
                    K->perm, K->seg, K->dperm, K->dstart, K->orient, K->dinv, K->ws, K->scratch,
                    K->ilu_up, K->ilu_inv, K->ilu_flags, K->ilu_order, K->full_ptr, K->full_col, K->full_val,
                    K->lfac, K->sfac, K->bj_w, K->sc_upper, K->rperm, K->rinv, K->rtmp, K->tma_tiles, K->lr_off, K->lr_buf};
    for (void* p : ptrs)
        if (p) dev_free(p);
    cudaSetDevice(prev);
    delete K;
}

extern "C" dda_status_t dda_build_matrix(int32_t n, const double* kdiag, int64_t m, const int32_t* bi,
                                         const int32_t* bj, const double* pen, const double* e, const double* g,
                                         void* stream, dda_matrix_t* out) {
    DDA_NVTX("dda_build_matrix");
    return dda::build_matrix_impl(n, kdiag, m, bi, bj, pen, e, g, reinterpret_cast<cudaStream_t>(stream), nullptr,
                                  out);
}

// values_ready (may be null): the stream waits for it before the first use of kdiag / e / g, so the
// host->device copies of those arrays can overlap the key sorts (dda_solve_host)
dda_status_t dda::build_matrix_impl(int32_t n, const double* kdiag, int64_t m, const int32_t* bi, const int32_t* bj,
                                    const double* pen, const double* e, const double* g, cudaStream_t stream,
                                    cudaEvent_t values_ready, dda_matrix_t* out) {
    if (!out) return DDA_ERR_ARG;
    *out = nullptr;
    if (n <= 0 || m < 0 || !kdiag) return DDA_ERR_ARG;
    if (m > 0 && (!bi || !bj || !pen || !e || !g)) return DDA_ERR_ARG;
    if (m > (int64_t)INT_MAX / 2 || (int64_t)n > (int64_t)INT_MAX / 36) return DDA_ERR_ARG;
    if (m > 0 && ((reinterpret_cast<uintptr_t>(e) | reinterpret_cast<uintptr_t>(g)) & 15)) return DDA_ERR_ARG;
    cudaStream_t st = stream;

    dda_matrix* K = new dda_matrix();
    DDA_CK(cudaGetDevice(&K->device));
    K->n = n;
    K->m = m;
    struct Guard {
        dda_matrix* K;
        bool keep = false;
        ~Guard() { if (!keep) dda_matrix_free(K); }
    } guard{K};

    trace("build: enter");
    Tmp tmp(st);
    int* err = nullptr;
    DDA_CK(tmp.get(&err, 1));
    DDA_CK(cudaMemsetAsync(err, 0, sizeof(int), st));

    // ---- (1) keys, (2) stable radix sort by (min,max)
    uint64_t *key = nullptr, *skey = nullptr;
    int32_t *val = nullptr, *flag = nullptr, *uid = nullptr;
    DDA_CK(tmp.get(&key, m));
    DDA_CK(tmp.get(&skey, m));
    DDA_CK(tmp.get(&val, m));
    DDA_CK(tmp.get(&flag, m));
    DDA_CK(tmp.get(&uid, m));
    DDA_CK(dmalloc(&K->perm, m, st));
    DDA_CK(dmalloc(&K->orient, m, st));
    int32_t nnzb = 0;
    if (m > 0) {
        k_keys<<<grid_for(m), TPB, 0, st>>>(n, m, bi, bj, pen, key, val, K->orient, err);
        DDA_LAUNCHED();
        const int kbits = bits_for((uint64_t)n * (uint64_t)n - 1);
        size_t tb = 0;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, key, skey, val, K->perm, (int)m, 0, kbits, st));
        void* tsort = nullptr;
        DDA_CK(tmp.get(reinterpret_cast<char**>(&tsort), tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(tsort, tb, key, skey, val, K->perm, (int)m, 0, kbits, st));
        note_launch(2 + (kbits + 7) / 8);   // onesweep: histogram + exclusive sum + one pass per 8 bits
        // ---- (3) boundary flags + scan
        k_heads<<<grid_for(m), TPB, 0, st>>>(m, skey, flag);
        DDA_LAUNCHED();
        size_t ts = 0;
        DDA_CK(cub::DeviceScan::InclusiveSum(nullptr, ts, flag, uid, (int)m, st));
        void* tscan = nullptr;
        DDA_CK(tmp.get(reinterpret_cast<char**>(&tscan), ts));
        DDA_CK(cub::DeviceScan::InclusiveSum(tscan, ts, flag, uid, (int)m, st));
        note_launch(2);
        DDA_CK(cudaMemcpyAsync(&nnzb, uid + (m - 1), sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    }
    int herr = 0;
    DDA_CK(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, st));
    trace("build: keys+sort+scan issued");
    DDA_CK(cudaStreamSynchronize(st));
    trace("build: nnzb sync");
    if (herr) return DDA_ERR_ARG;
    K->nnzb = nnzb;

    // ---- (4) structure: segments, unique blocks, row_ptr
    DDA_CK(dmalloc(&K->row_ptr, (size_t)n + 1, st));
    DDA_CK(dmalloc(&K->col_idx, nnzb, st));
    DDA_CK(dmalloc(&K->urow, nnzb, st));
    DDA_CK(dmalloc(&K->seg, (size_t)nnzb + 1, st));
    DDA_CK(dmalloc(&K->low_ptr, (size_t)n + 1, st));
    DDA_CK(dmalloc(&K->low_row, nnzb, st));
    DDA_CK(dmalloc(&K->low_to_up, nnzb, st));
    DDA_CK(dmalloc(&K->diag, (size_t)n * kBlk, st));
    DDA_CK(dmalloc(&K->upper, (size_t)nnzb * kBlk, st));
    DDA_CK(dmalloc(&K->dperm, (size_t)2 * m, st));
    DDA_CK(dmalloc(&K->dstart, (size_t)n + 1, st));
    DDA_CK(dmalloc(&K->dinv, (size_t)n * kDinv, st));
    DDA_CK(dmalloc(reinterpret_cast<char**>(&K->scratch), 256, st));
    trace("build: allocations");
    if (m > 0) {
        k_unique<<<grid_for(m), TPB, 0, st>>>(n, m, skey, uid, K->seg, K->urow, K->col_idx);
        DDA_LAUNCHED();
        const int32_t mm = (int32_t)m;
        DDA_CK(cudaMemcpyAsync(K->seg + nnzb, &mm, sizeof(int32_t), cudaMemcpyHostToDevice, st));
    }
    k_bounds<<<grid_for((int64_t)nnzb + 1), TPB, 0, st>>>(n, nnzb, K->urow, K->row_ptr);
    DDA_LAUNCHED();

    // ---- (5) diagonal endpoint records, stably sorted by block
    {
        int32_t *dkey = nullptr, *dskey = nullptr, *dval = nullptr;
        DDA_CK(tmp.get(&dkey, (size_t)2 * m));
        DDA_CK(tmp.get(&dskey, (size_t)2 * m));
        DDA_CK(tmp.get(&dval, (size_t)2 * m));
        if (m > 0) {
            k_dkeys<<<grid_for(m), TPB, 0, st>>>(m, bi, bj, dkey, dval);
            DDA_LAUNCHED();
            const int dbits = bits_for((uint64_t)(n - 1));
            size_t tb = 0;
            DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, dkey, dskey, dval, K->dperm, (int)(2 * m), 0, dbits, st));
            void* tsort = nullptr;
            DDA_CK(tmp.get(reinterpret_cast<char**>(&tsort), tb));
            DDA_CK(cub::DeviceRadixSort::SortPairs(tsort, tb, dkey, dskey, dval, K->dperm, (int)(2 * m), 0, dbits, st));
            note_launch(2 + (dbits + 7) / 8);
        }
        k_bounds<<<grid_for(2 * m + 1), TPB, 0, st>>>(n, 2 * m, dskey, K->dstart);
        DDA_LAUNCHED();
    }

    trace("build: structure issued");
    // ---- values (the final step that moves data)
    if (values_ready) DDA_CK(cudaStreamWaitEvent(st, values_ready, 0));
    {
        dda_status_t sv = run_values(K, kdiag, pen, e, g, st);
        if (sv != DDA_OK) return sv;
    }

    trace("build: values issued");
    // ---- (6) transpose map: stable sort of the unique blocks by (col, row)
    if (nnzb > 0) {
        uint64_t *tkey = nullptr, *tskey = nullptr;
        int32_t *tval = nullptr, *tcol = nullptr;
        DDA_CK(tmp.get(&tkey, nnzb));
        DDA_CK(tmp.get(&tskey, nnzb));
        DDA_CK(tmp.get(&tval, nnzb));
        DDA_CK(tmp.get(&tcol, nnzb));
        k_tkeys<<<grid_for(nnzb), TPB, 0, st>>>(n, nnzb, K->urow, K->col_idx, tkey, tval);
        DDA_LAUNCHED();
        const int kbits = bits_for((uint64_t)n * (uint64_t)n - 1);
        size_t tb = 0;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, tkey, tskey, tval, K->low_to_up, nnzb, 0, kbits, st));
        void* tsort = nullptr;
        DDA_CK(tmp.get(reinterpret_cast<char**>(&tsort), tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(tsort, tb, tkey, tskey, tval, K->low_to_up, nnzb, 0, kbits, st));
        note_launch(2 + (kbits + 7) / 8);   // onesweep: histogram + exclusive sum + one pass per 8 bits
        k_tfill<<<grid_for(nnzb), TPB, 0, st>>>(n, nnzb, tskey, K->low_row, tcol);
        DDA_LAUNCHED();
        k_bounds<<<grid_for((int64_t)nnzb + 1), TPB, 0, st>>>(n, nnzb, tcol, K->low_ptr);
        DDA_LAUNCHED();
    } else {
        DDA_CK(cudaMemsetAsync(K->low_ptr, 0, sizeof(int32_t) * ((size_t)n + 1), st));
    }
    trace("build: all issued");
    DDA_CK(cudaStreamSynchronize(st));   // temporaries are released stream-ordered by ~Tmp
    trace("build: final sync");
    guard.keep = true;
    *out = K;
    return DDA_OK;
}

extern "C" dda_status_t dda_update_values(dda_matrix_t K, const double* kdiag, int64_t m, const double* pen,
                                          const double* e, const double* g, void* stream) {
    DDA_NVTX("dda_update_values");
    if (!K || !kdiag || m != K->m) return DDA_ERR_ARG;
    if (m > 0 && (!pen || !e || !g)) return DDA_ERR_ARG;
    if (m > 0 && ((reinterpret_cast<uintptr_t>(e) | reinterpret_cast<uintptr_t>(g)) & 15)) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    return K->rperm ? ro_update_values(K, kdiag, pen, e, g, st) : run_values(K, kdiag, pen, e, g, st);
}

extern "C" dda_status_t dda_matrix_info(dda_matrix_t K, int32_t* n, int64_t* nnzb) {
    if (!K) return DDA_ERR_ARG;
    if (n) *n = K->n;
    if (nnzb) *nnzb = K->nnzb;
    return DDA_OK;
}

extern "C" dda_status_t dda_matrix_export(dda_matrix_t K, int32_t* row_ptr, int32_t* col_idx, int32_t* low_ptr,
                                          int32_t* low_row, int32_t* low_to_up, double* diag, double* upper) {
    if (!K) return DDA_ERR_ARG;
    if (K->rperm) return ro_export(K, row_ptr, col_idx, low_ptr, low_row, low_to_up, diag, upper);
    return export_internal(K, row_ptr, col_idx, low_ptr, low_row, low_to_up, diag, upper);
}

dda_status_t dda::export_internal(dda_matrix* K, int32_t* row_ptr, int32_t* col_idx, int32_t* low_ptr,
                                  int32_t* low_row, int32_t* low_to_up, double* diag, double* upper) {
    const size_t n1 = (size_t)K->n + 1, z = (size_t)K->nnzb;
    DDA_CK(cudaDeviceSynchronize());
    if (row_ptr) DDA_CK(cudaMemcpy(row_ptr, K->row_ptr, n1 * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (col_idx && z) DDA_CK(cudaMemcpy(col_idx, K->col_idx, z * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (low_ptr) DDA_CK(cudaMemcpy(low_ptr, K->low_ptr, n1 * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (low_row && z) DDA_CK(cudaMemcpy(low_row, K->low_row, z * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (low_to_up && z) DDA_CK(cudaMemcpy(low_to_up, K->low_to_up, z * sizeof(int32_t), cudaMemcpyDeviceToHost));
    auto untile = [](const std::vector<double>& t, double* out, size_t nb) {
        for (size_t b = 0; b < nb; ++b)
            for (int r = 0; r < 6; ++r)
                for (int c = 0; c < 6; ++c) out[36 * b + 6 * r + c] = t[36 * b + tile_off(r, c)];
    };
    if (diag) {
        std::vector<double> t((size_t)K->n * kBlk);
        DDA_CK(cudaMemcpy(t.data(), K->diag, t.size() * sizeof(double), cudaMemcpyDeviceToHost));
        untile(t, diag, (size_t)K->n);
    }
    if (upper && z) {
        std::vector<double> t(z * kBlk);
        DDA_CK(cudaMemcpy(t.data(), K->upper, t.size() * sizeof(double), cudaMemcpyDeviceToHost));
        untile(t, upper, z);
    }
    return DDA_OK;
}
