// §8(b)/(e) — dda_build_matrix_dist: the partition-local assembly of the block-row partitioned
// solve, on the device (beyond the paper: multi-GPU is its future work; the assembly it
// wraps is the paper's, §III.C).
//
// Partition p owns the contiguous global block rows [b_p, b_{p+1}).  From the caller's springs
// (the global list, or any list containing every spring that touches an own row) it builds:
//   selection  the springs with an endpoint in the own range, in spring order (flag + stable
//              compaction, cub::DeviceSelect)                                    — P:104 (a contact
//              between i and j contributes to rows i and j, so these are all the own rows' terms)
//   halo       the remote endpoints of those springs, sorted and unique (radix sort + unique):
//              ascending global id = grouped by owning partition, so each peer's slice of the
//              halo is contiguous and is received in place
//   numbering  own row g -> g - b_p; halo row h -> n_own + rank of h in the halo (binary search)
//   matrix     dda_build_matrix (A1) on the local springs and diagonal terms (halo rows: zero
//              diagonal terms; they are only read as x values), so the own rows of the local
//              matrix are bit-identical to the global rows (same springs, same summation order)
//   plan       per spring with a remote endpoint h owned by q and own endpoint a: the key
//              (q << 32) | (a - b_p); sorted and unique -> the own rows each peer q needs, in q's
//              halo order (ascending global id); the receive counts are the halo's owner counts
// and attaches the matrix and plan to the communicator (dda_dist_attach).  Integer work only
// (ids, flags, sorts); the values are the unchanged A1 assembly.
#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>

#include <climits>
#include <vector>

#include "dda_internal.cuh"

namespace dda {
namespace {

constexpr int TPB = 256;

inline int grid_of(int64_t items) {
    int64_t g = (items + TPB - 1) / TPB;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 32;
    return (int)(g < cap ? g : cap);
}

__device__ __forceinline__ bool own(int32_t g, int32_t r0, int32_t r1) { return g >= r0 && g < r1; }

// keep[s] = spring s touches an own row; err on an id outside [0, n) or a self contact
__global__ void k_dsel(int64_t m, int32_t n, int32_t r0, int32_t r1, const int32_t* __restrict__ bi,
                       const int32_t* __restrict__ bj, uint8_t* __restrict__ keep, int* __restrict__ err) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < m; s += (int64_t)gridDim.x * blockDim.x) {
        const int32_t i = bi[s], j = bj[s];
        if (i < 0 || i >= n || j < 0 || j >= n || i == j) atomicOr(err, 1);
        keep[s] = own(i, r0, r1) || own(j, r0, r1);
    }
}

// owner partition of global row g (bounds [P+1], ascending)
__device__ __forceinline__ int owner_of(const int32_t* __restrict__ bounds, int P, int32_t g) {
    int lo = 0, hi = P;                  // bounds[lo] <= g < bounds[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (bounds[mid] <= g) lo = mid; else hi = mid;
    }
    return lo;
}

// per selected spring: its remote endpoint (INT_MAX if both own) and the send key
// (owner(remote) << 32 | own endpoint - r0), UINT64_MAX if none
__global__ void k_dremote(int ms, const int32_t* __restrict__ sel, const int32_t* __restrict__ bi,
                          const int32_t* __restrict__ bj, int32_t r0, int32_t r1, const int32_t* __restrict__ bounds,
                          int P, int32_t* __restrict__ rem, uint64_t* __restrict__ skey) {
    for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < ms; k += gridDim.x * blockDim.x) {
        const int32_t s = sel[k], i = bi[s], j = bj[s];
        const bool oi = own(i, r0, r1), oj = own(j, r0, r1);
        int32_t h = INT_MAX;
        uint64_t key = ~0ull;
        if (!(oi && oj)) {
            h = oi ? j : i;
            const int32_t a = oi ? i : j;
            key = ((uint64_t)owner_of(bounds, P, h) << 32) | (uint32_t)(a - r0);
        }
        rem[k] = h;
        skey[k] = key;
    }
}

// the local springs: ids renumbered, penalty and vectors gathered in selection (= spring) order
__global__ void k_dlocal(int ms, const int32_t* __restrict__ sel, const int32_t* __restrict__ bi,
                         const int32_t* __restrict__ bj, const double* __restrict__ pen,
                         const double* __restrict__ e, const double* __restrict__ g, int32_t r0, int32_t r1,
                         const int32_t* __restrict__ halo, int nh, int32_t* __restrict__ lbi,
                         int32_t* __restrict__ lbj, double* __restrict__ lpen, double* __restrict__ le,
                         double* __restrict__ lg) {
    const int32_t n_own = r1 - r0;
    auto loc = [&](int32_t x) -> int32_t {
        if (own(x, r0, r1)) return x - r0;
        int lo = 0, hi = nh;             // first halo[t] >= x (x is in the halo)
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            if (halo[mid] < x) lo = mid + 1; else hi = mid;
        }
        return n_own + lo;
    };
    for (int k = blockIdx.x * blockDim.x + threadIdx.x; k < ms; k += gridDim.x * blockDim.x) {
        const int32_t s = sel[k];
        lbi[k] = loc(bi[s]);
        lbj[k] = loc(bj[s]);
        lpen[k] = pen[s];
        const double2* es = reinterpret_cast<const double2*>(e + 6 * (size_t)s);
        const double2* gs = reinterpret_cast<const double2*>(g + 6 * (size_t)s);
        double2* ed = reinterpret_cast<double2*>(le + 6 * (size_t)k);
        double2* gd = reinterpret_cast<double2*>(lg + 6 * (size_t)k);
#pragma unroll
        for (int t = 0; t < 3; ++t) {
            ed[t] = es[t];
            gd[t] = gs[t];
        }
    }
}

struct Scratch {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit Scratch(cudaStream_t st) : s(st) {}
    template <class T>
    cudaError_t get(T** p, size_t count) {
        void* q = nullptr;
        cudaError_t e = dev_alloc(&q, (count ? count : 1) * sizeof(T), s);
        if (e == cudaSuccess) ptrs.push_back(q);
        *p = reinterpret_cast<T*>(q);
        return e;
    }
    ~Scratch() {
        for (void* p : ptrs) dev_free_on(p, s);
    }
};

}  // namespace
}  // namespace dda

extern "C" dda_status_t dda_build_matrix_dist(dda_comm_t c, int32_t part, int32_t n_global, const int32_t* bounds,
                                              const double* kdiag_own, int64_t m, const int32_t* bi,
                                              const int32_t* bj, const double* pen, const double* e,
                                              const double* g, void* stream, dda_matrix_t* out) {
    DDA_NVTX("dda_build_matrix_dist");
    using namespace dda;
    if (!out) return DDA_ERR_ARG;
    *out = nullptr;
    if (!c || !bounds || !kdiag_own || n_global <= 0 || m < 0) return DDA_ERR_ARG;
    if (m > 0 && (!bi || !bj || !pen || !e || !g)) return DDA_ERR_ARG;
    if (m > (int64_t)INT_MAX / 2) return DDA_ERR_ARG;
    if (m > 0 && ((reinterpret_cast<uintptr_t>(e) | reinterpret_cast<uintptr_t>(g)) & 15)) return DDA_ERR_ARG;
    const int P = comm_nparts(c);
    const int me = comm_part_index(c, part);
    if (me < 0) return DDA_ERR_ARG;
    if (bounds[0] != 0 || bounds[P] != n_global) return DDA_ERR_ARG;
    for (int q = 0; q < P; ++q)
        if (bounds[q + 1] <= bounds[q]) return DDA_ERR_ARG;
    const int32_t r0 = bounds[me], r1 = bounds[me + 1], n_own = r1 - r0;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    Scratch tmp(st);

    // ---- selection: springs touching an own row, in spring order
    int *err = nullptr, *nsel = nullptr;
    int32_t *dbounds = nullptr, *sel = nullptr;
    uint8_t* keep = nullptr;
    DDA_CK(tmp.get(&err, 1));
    DDA_CK(tmp.get(&nsel, 1));
    DDA_CK(tmp.get(&dbounds, P + 1));
    DDA_CK(tmp.get(&keep, m));
    DDA_CK(tmp.get(&sel, m));
    DDA_CK(cudaMemsetAsync(err, 0, sizeof(int), st));
    DDA_CK(cudaMemcpyAsync(dbounds, bounds, (P + 1) * sizeof(int32_t), cudaMemcpyHostToDevice, st));
    int ms = 0;
    if (m > 0) {
        k_dsel<<<grid_of(m), TPB, 0, st>>>(m, n_global, r0, r1, bi, bj, keep, err);
        DDA_LAUNCHED();
        thrust::counting_iterator<int32_t> ids(0);
        size_t tb = 0;
        DDA_CK(cub::DeviceSelect::Flagged(nullptr, tb, ids, keep, sel, nsel, (int)m, st));
        void* ts = nullptr;
        DDA_CK(tmp.get(reinterpret_cast<char**>(&ts), tb));
        DDA_CK(cub::DeviceSelect::Flagged(ts, tb, ids, keep, sel, nsel, (int)m, st));
        note_launch(2);
        int herr = 0;
        DDA_CK(cudaMemcpyAsync(&ms, nsel, sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaMemcpyAsync(&herr, err, sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
        if (herr) return DDA_ERR_ARG;
    }

    // ---- remote endpoints -> halo (sorted unique); send keys -> plan (sorted unique)
    int32_t *rem = nullptr, *srem = nullptr, *halo = nullptr;
    uint64_t *skey = nullptr, *sskey = nullptr, *ukey = nullptr;
    int *nh_d = nullptr, *nk_d = nullptr;
    DDA_CK(tmp.get(&rem, ms));
    DDA_CK(tmp.get(&srem, ms));
    DDA_CK(tmp.get(&halo, ms));
    DDA_CK(tmp.get(&skey, ms));
    DDA_CK(tmp.get(&sskey, ms));
    DDA_CK(tmp.get(&ukey, ms));
    DDA_CK(tmp.get(&nh_d, 1));
    DDA_CK(tmp.get(&nk_d, 1));
    int nh = 0, nk = 0;
    if (ms > 0) {
        k_dremote<<<grid_of(ms), TPB, 0, st>>>(ms, sel, bi, bj, r0, r1, dbounds, P, rem, skey);
        DDA_LAUNCHED();
        size_t t1 = 0, t2 = 0, t3 = 0, t4 = 0;
        DDA_CK(cub::DeviceRadixSort::SortKeys(nullptr, t1, rem, srem, ms, 0, 32, st));
        DDA_CK(cub::DeviceSelect::Unique(nullptr, t2, srem, halo, nh_d, ms, st));
        DDA_CK(cub::DeviceRadixSort::SortKeys(nullptr, t3, skey, sskey, ms, 0, 64, st));
        DDA_CK(cub::DeviceSelect::Unique(nullptr, t4, sskey, ukey, nk_d, ms, st));
        size_t tb = t1;
        for (size_t t : {t2, t3, t4}) tb = t > tb ? t : tb;
        void* ts = nullptr;
        DDA_CK(tmp.get(reinterpret_cast<char**>(&ts), tb));
        DDA_CK(cub::DeviceRadixSort::SortKeys(ts, t1, rem, srem, ms, 0, 32, st));
        DDA_CK(cub::DeviceSelect::Unique(ts, t2, srem, halo, nh_d, ms, st));
        DDA_CK(cub::DeviceRadixSort::SortKeys(ts, t3, skey, sskey, ms, 0, 64, st));
        DDA_CK(cub::DeviceSelect::Unique(ts, t4, sskey, ukey, nk_d, ms, st));
        note_launch(8);
        DDA_CK(cudaMemcpyAsync(&nh, nh_d, sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaMemcpyAsync(&nk, nk_d, sizeof(int), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
    }
    std::vector<int32_t> hhalo(nh > 0 ? nh : 1);
    std::vector<uint64_t> hkey(nk > 0 ? nk : 1);
    if (nh) DDA_CK(cudaMemcpyAsync(hhalo.data(), halo, nh * sizeof(int32_t), cudaMemcpyDeviceToHost, st));
    if (nk) DDA_CK(cudaMemcpyAsync(hkey.data(), ukey, nk * sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
    // the sentinels (INT_MAX: both endpoints own; ~0: no remote endpoint) sort last
    DDA_CK(cudaStreamSynchronize(st));
    if (nh && hhalo[nh - 1] == INT_MAX) --nh;
    if (nk && hkey[nk - 1] == ~0ull) --nk;
    const int32_t n_local = n_own + nh;

    // ---- local springs and diagonal terms, then the A1 assembly
    int32_t *lbi = nullptr, *lbj = nullptr;
    double *lpen = nullptr, *le = nullptr, *lg = nullptr, *lkd = nullptr;
    DDA_CK(tmp.get(&lbi, ms));
    DDA_CK(tmp.get(&lbj, ms));
    DDA_CK(tmp.get(&lpen, ms));
    DDA_CK(tmp.get(&le, 6 * (size_t)ms));
    DDA_CK(tmp.get(&lg, 6 * (size_t)ms));
    DDA_CK(tmp.get(&lkd, (size_t)kBlk * n_local));
    if (ms > 0) {
        k_dlocal<<<grid_of(ms), TPB, 0, st>>>(ms, sel, bi, bj, pen, e, g, r0, r1, halo, nh, lbi, lbj, lpen, le, lg);
        DDA_LAUNCHED();
    }
    DDA_CK(cudaMemcpyAsync(lkd, kdiag_own, (size_t)kBlk * n_own * sizeof(double), cudaMemcpyDeviceToDevice, st));
    if (nh) DDA_CK(cudaMemsetAsync(lkd + (size_t)kBlk * n_own, 0, (size_t)kBlk * nh * sizeof(double), st));
    dda_matrix_t K = nullptr;
    dda_status_t s = build_matrix_impl(n_local, lkd, ms, lbi, lbj, lpen, le, lg, st, nullptr, &K);
    if (s != DDA_OK) return s;

    // ---- exchange plan (host, small: about one slope course per cut) and attach
    std::vector<int32_t> send_counts(P, 0), recv_counts(P, 0), send_idx(nk > 0 ? nk : 1);
    for (int t = 0; t < nk; ++t) {
        send_counts[(int)(hkey[t] >> 32)] += 1;
        send_idx[t] = (int32_t)(uint32_t)(hkey[t] & 0xffffffffu);
    }
    for (int t = 0, q = 0; t < nh; ++t) {
        while (hhalo[t] >= bounds[q + 1]) ++q;
        recv_counts[q] += 1;
    }
    s = dda_dist_attach(c, part, K, n_own, send_counts.data(), send_idx.data(), recv_counts.data(), stream);
    if (s != DDA_OK) {
        dda_matrix_free(K);
        return s;
    }
    *out = K;
    return DDA_OK;
}
