// NEXT-4 — interpenetration check and the open-close state switch (§III.A, third
// classification; §III.D; loop 3 of §I), closing the open-close loop around the
// solve with value-only re-assembly (NEXT-1) and a warm-started PCG.
//
// What is computed (reading N4; the oracle's O-11 / O-12 are the definition): the
// contacts are the records of a classified set (VE, VV1, VV2) whose springs are 2k (normal) and
// 2k+1 (shear) of dda_contact_springs.  Per contact, with the signed gap dn0 = n.(P - Q1):
//     un = e_n.d_i + g_n.d_j,  us = e_s.d_i + g_s.d_j,  dn = dn0 + un
//     closed' = dn <= (closed ? open_tol : 0);  lock' = closed' && !(p_s |us| > tan_phi (-p_n dn))
//     p1 = closed' - closed,  p2 = lock' - lock          (the paper's switch integers)
//     category: VE / VV1: C1 p1 != 0, C2 p1 == 0 & p2 != 0, C3 no switch & closed';
//               VV2:      C4 p1 != 0, C5 p1 == 0 & p2 != 0;  else 0
// and the closed normal springs load F with -p_n dn0 [e_n; g_n] (the gap term of their energy).
//
// B200 mapping:
//   * check: one thread per contact, the category computed without branches (the paper's §III.D
//     restructuring: every path computes the same expressions, selects write the result), all
//     products and sums rounded as written (__dmul_rn / __dadd_rn) so states are bit-exact;
//     then the categories are stored class by class (stable 3-bit radix sort, "data
//     classification") and counted;
//   * gap load: write conflicts (several contacts per block) resolved as the paper's assembly does
//     (P:106): the 2 endpoint records of every contact are sorted once by block (stable radix
//     sort), and one thread per block sums its segment in contact order — deterministic, no
//     atomics, bit-identical to the oracle's sequential sum;
//   * loop: penalties from the states -> dda_update_values (cached structure and sort) -> F + gap
//     load -> dda_pcg_solve warm-started from the previous d -> check; the host reads the six
//     category counts once per open-close iteration.
#include <cub/cub.cuh>

#include <cmath>
#include <vector>

#include "dda_internal.cuh"

namespace dda {
namespace {

constexpr int OT = 256;

inline int ogrid(int64_t items) {
    int64_t g = (items + OT - 1) / OT;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 32;
    return (int)(g < cap ? g : cap);
}

// signed gap of record k and (when state != null) the initial state; endpoint keys for the sort
__global__ void k_oc_init(int64_t m, const int32_t* __restrict__ vptr, const double* __restrict__ vxy,
                          const int32_t* __restrict__ ci, const int32_t* __restrict__ cv,
                          const int32_t* __restrict__ cj, const int32_t* __restrict__ ce, double* __restrict__ gap,
                          int32_t* __restrict__ state, uint32_t* __restrict__ ekey, int32_t* __restrict__ eval) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = cv[k], j = cj[k], q = ce[k];
        const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
        const double dx = __dsub_rn(vxy[2 * (size_t)q2], vxy[2 * (size_t)q]);
        const double dy = __dsub_rn(vxy[2 * (size_t)q2 + 1], vxy[2 * (size_t)q + 1]);
        const double len = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        const double ux = __ddiv_rn(dx, len), uy = __ddiv_rn(dy, len);
        const double nx = uy, ny = -ux;
        const double g0 = __dadd_rn(__dmul_rn(nx, __dsub_rn(vxy[2 * (size_t)v], vxy[2 * (size_t)q])),
                                    __dmul_rn(ny, __dsub_rn(vxy[2 * (size_t)v + 1], vxy[2 * (size_t)q + 1])));
        gap[k] = g0;
        if (state) state[k] = g0 <= 0.0 ? 2 : 0;
        ekey[2 * k] = (uint32_t)ci[k];
        ekey[2 * k + 1] = (uint32_t)j;
        eval[2 * k] = (int32_t)(2 * k);
        eval[2 * k + 1] = (int32_t)(2 * k + 1);
    }
}

// estart[b] = first position of block b in the sorted endpoint keys (lower bound), b = 0..n
__global__ void k_oc_bounds(int32_t n, int64_t m2, const uint32_t* __restrict__ skey, int32_t* __restrict__ estart) {
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b <= n; b += (int64_t)gridDim.x * blockDim.x) {
        int64_t lo = 0, hi = m2;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (skey[mid] < (uint32_t)b) lo = mid + 1; else hi = mid;
        }
        estart[b] = (int32_t)lo;
    }
}

// penalties of the states: normal p_n if closed, shear p_s if lock (0 otherwise)
__global__ void k_oc_pen(int64_t m, const int32_t* __restrict__ state, double p_n, double ps, double* __restrict__ pen) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t s = state[k];
        pen[2 * k] = s >= 1 ? p_n : 0.0;
        pen[2 * k + 1] = s == 2 ? ps : 0.0;
    }
}

// out[b] = (F ? F[b] : 0) + sum over b's endpoint records, in contact order, of f e_n (vertex side)
// or f g_n (edge side), f = -(pen[2k] * gap[k]) — one thread per block (P:106's segment sum)
__global__ void k_oc_loads(int32_t n, const int32_t* __restrict__ estart, const int32_t* __restrict__ eperm,
                           const double* __restrict__ gap, const double* __restrict__ pen,
                           const double* __restrict__ e, const double* __restrict__ g, const double* __restrict__ F,
                           double* __restrict__ out) {
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < n; b += (int64_t)gridDim.x * blockDim.x) {
        double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
        for (int32_t t = estart[b]; t < estart[b + 1]; ++t) {
            const int32_t rec = eperm[t];
            const int64_t k = rec >> 1;
            const double f = -__dmul_rn(pen[2 * k], gap[k]);
            const double* vec = ((rec & 1) ? g : e) + 12 * k;          // the normal spring's e_n or g_n
#pragma unroll
            for (int r = 0; r < 6; ++r) acc[r] = __dadd_rn(acc[r], __dmul_rn(f, vec[r]));
        }
#pragma unroll
        for (int r = 0; r < 6; ++r) out[6 * b + r] = F ? __dadd_rn(F[6 * b + r], acc[r]) : acc[r];
    }
}

// the interpenetration check of O-11, branch-restructured (§III.D): key = category, val = k
__global__ void k_oc_check(int64_t m, const int32_t* __restrict__ ci, const int32_t* __restrict__ cj,
                           const int32_t* __restrict__ cls, const double* __restrict__ gap,
                           const double* __restrict__ d, const double* __restrict__ e, const double* __restrict__ g,
                           double p_n, double ps, double tan_phi, double open_tol, int32_t* __restrict__ state,
                           double* __restrict__ pen, int32_t* __restrict__ cat, uint32_t* __restrict__ ckey,
                           int32_t* __restrict__ cval) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const double* di = d + 6 * (size_t)ci[k];
        const double* dj = d + 6 * (size_t)cj[k];
        const double *en = e + 12 * k, *es = e + 12 * k + 6, *gn = g + 12 * k, *gs = g + 12 * k + 6;
        double un = 0.0, us = 0.0;
#pragma unroll
        for (int r = 0; r < 6; ++r) un = __dadd_rn(un, __dmul_rn(en[r], di[r]));
#pragma unroll
        for (int r = 0; r < 6; ++r) un = __dadd_rn(un, __dmul_rn(gn[r], dj[r]));
#pragma unroll
        for (int r = 0; r < 6; ++r) us = __dadd_rn(us, __dmul_rn(es[r], di[r]));
#pragma unroll
        for (int r = 0; r < 6; ++r) us = __dadd_rn(us, __dmul_rn(gs[r], dj[r]));
        const double dn = __dadd_rn(gap[k], un);
        const int old = state[k];
        const int was_closed = old >= 1, was_lock = old == 2;
        const int closed = dn <= (was_closed ? open_tol : 0.0);
        const double fn = -__dmul_rn(p_n, dn);
        const double fs = __dmul_rn(ps, fabs(us));
        const int lock = closed & !(fs > __dmul_rn(tan_phi, fn));
        const int p1 = closed - was_closed, p2 = lock - was_lock;
        // category without branches: a1 = switched open/closed, a2 = switched slide/lock only,
        // a3 = no switch and in contact (VE / VV1 only); h = VV2 shifts C1/C2 to C4/C5
        const int h = cls[k] == 2;
        const int a1 = p1 != 0;
        const int a2 = (!a1) & (p2 != 0);
        const int a3 = (!a1) & (!a2) & closed & (!h);
        const int c = a1 * (1 + 3 * h) + a2 * (2 + 3 * h) + a3 * 3;
        cat[k] = c;
        state[k] = closed * (1 + lock);
        pen[2 * k] = closed ? p_n : 0.0;
        pen[2 * k + 1] = lock ? ps : 0.0;
        ckey[k] = (uint32_t)c;
        cval[k] = (int32_t)k;
    }
}

// start[c] of each category c = 0..5 in the sorted keys (start[6] = m)
__global__ void k_oc_cat_bounds(int64_t m, const uint32_t* __restrict__ skey, int64_t* __restrict__ start) {
    for (int c = threadIdx.x; c <= 6; c += blockDim.x) {
        int64_t lo = 0, hi = m;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (skey[mid] < (uint32_t)c) lo = mid + 1; else hi = mid;
        }
        start[c] = lo;
    }
}

struct OTmp {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit OTmp(cudaStream_t st) : s(st) {}
    template <class T>
    cudaError_t get(T** p, size_t count) {
        void* q = nullptr;
        cudaError_t e = dev_alloc(&q, (count ? count : 1) * sizeof(T), s);
        if (e == cudaSuccess) ptrs.push_back(q);
        *p = reinterpret_cast<T*>(q);
        return e;
    }
    ~OTmp() {
        for (void* p : ptrs) dev_free_on(p, s);
    }
};

dda_status_t oc_init(dda_contacts_t C, int32_t* state, cudaStream_t st) {
    const int64_t m = C->count;
    if (!C->gap) {
        OTmp tmp(st);
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&C->gap), (m ? m : 1) * sizeof(double), st));
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&C->eperm), (2 * m + 1) * sizeof(int32_t), st));
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&C->estart), ((size_t)C->n + 1) * sizeof(int32_t), st));
        uint32_t *ekey = nullptr, *skey = nullptr;
        int32_t* eval = nullptr;
        DDA_CK(tmp.get(&ekey, 2 * m));
        DDA_CK(tmp.get(&skey, 2 * m));
        DDA_CK(tmp.get(&eval, 2 * m));
        if (m > 0) {
            k_oc_init<<<ogrid(m), OT, 0, st>>>(m, C->vptr, C->vxy, C->ci, C->cv, C->cj, C->ce, C->gap, state, ekey,
                                               eval);
            DDA_LAUNCHED();
            int bits = 1;
            while (bits < 32 && ((uint32_t)C->n >> bits) != 0) ++bits;
            size_t tb = 0;
            DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, ekey, skey, eval, C->eperm, (int)(2 * m), 0, bits, st));
            char* ts = nullptr;
            DDA_CK(tmp.get(&ts, tb));
            DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, ekey, skey, eval, C->eperm, (int)(2 * m), 0, bits, st));
            note_launch(4);
        }
        k_oc_bounds<<<ogrid((int64_t)C->n + 1), OT, 0, st>>>(C->n, 2 * m, skey, C->estart);
        DDA_LAUNCHED();
    } else if (state && m > 0) {      // gaps cached: only the initial states
        uint32_t* ekey = nullptr;
        int32_t* eval = nullptr;
        OTmp tmp(st);
        double* gap2 = nullptr;
        DDA_CK(tmp.get(&ekey, 2 * m));
        DDA_CK(tmp.get(&eval, 2 * m));
        DDA_CK(tmp.get(&gap2, m));
        k_oc_init<<<ogrid(m), OT, 0, st>>>(m, C->vptr, C->vxy, C->ci, C->cv, C->cj, C->ce, gap2, state, ekey, eval);
        DDA_LAUNCHED();
    }
    return DDA_OK;
}

dda_status_t oc_check(dda_contacts_t C, const double* d, const double* e, const double* g, double p_n,
                      double shear_ratio, double tan_phi, double open_tol, int32_t* state, double* pen, int32_t* cat,
                      int32_t* cat_order, int64_t* counts, cudaStream_t st) {
    const int64_t m = C->count;
    OTmp tmp(st);
    uint32_t *ckey = nullptr, *skey = nullptr;
    int32_t *cval = nullptr, *sval = nullptr, *catb = cat;
    int64_t* start = nullptr;
    DDA_CK(tmp.get(&ckey, m));
    DDA_CK(tmp.get(&skey, m));
    DDA_CK(tmp.get(&cval, m));
    DDA_CK(tmp.get(&start, 8));
    if (!cat_order) DDA_CK(tmp.get(&sval, m));
    if (!catb) DDA_CK(tmp.get(&catb, m));
    int64_t hs[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (m > 0) {
        const double ps = shear_ratio * p_n;                   // the oracle's shear_ratio * p_n
        k_oc_check<<<ogrid(m), OT, 0, st>>>(m, C->ci, C->cj, C->ctype, C->gap, d, e, g, p_n, ps, tan_phi, open_tol,
                                            state, pen, catb, ckey, cval);
        DDA_LAUNCHED();
        size_t tb = 0;
        int32_t* order = cat_order ? cat_order : sval;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, ckey, skey, cval, order, (int)m, 0, 3, st));
        char* ts = nullptr;
        DDA_CK(tmp.get(&ts, tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, ckey, skey, cval, order, (int)m, 0, 3, st));
        note_launch(2);
        k_oc_cat_bounds<<<1, 32, 0, st>>>(m, skey, start);
        DDA_LAUNCHED();
        DDA_CK(cudaMemcpyAsync(hs, start, 7 * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    }
    DDA_CK(cudaStreamSynchronize(st));
    for (int c = 0; c < 6; ++c) counts[c] = m > 0 ? hs[c + 1] - hs[c] : 0;
    return DDA_OK;
}

bool oc_ready(dda_contacts_t C) { return C && C->classified && C->gap; }

}  // namespace
}  // namespace dda

extern "C" dda_status_t dda_contact_init(dda_contacts_t C, int32_t* state, void* stream) {
    if (!C || !C->classified) return DDA_ERR_ARG;
    return dda::oc_init(C, state, reinterpret_cast<cudaStream_t>(stream));
}

extern "C" dda_status_t dda_contact_loads(dda_contacts_t C, const double* e, const double* g, const double* pen,
                                          const double* F, double* out, void* stream) {
    DDA_NVTX("dda_contact_loads");
    using namespace dda;
    if (!oc_ready(C) || !out || (C->count > 0 && (!e || !g || !pen))) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    k_oc_loads<<<ogrid(C->n), OT, 0, st>>>(C->n, C->estart, C->eperm, C->gap, pen, e, g, F, out);
    DDA_LAUNCHED();
    return DDA_OK;
}

extern "C" dda_status_t dda_contact_check(dda_contacts_t C, const double* d, const double* e, const double* g,
                                          double p_n, double shear_ratio, double tan_phi, double open_tol,
                                          int32_t* state, double* pen, int32_t* cat, int32_t* cat_order,
                                          int64_t* counts, void* stream) {
    DDA_NVTX("dda_contact_check");
    using namespace dda;
    if (!oc_ready(C) || !counts || !(p_n >= 0.0) || !(shear_ratio >= 0.0) || !(tan_phi >= 0.0) ||
        !(open_tol >= 0.0) || !isfinite(p_n) || !isfinite(shear_ratio) || !isfinite(tan_phi) || !isfinite(open_tol))
        return DDA_ERR_ARG;
    if (C->count > 0 && (!d || !e || !g || !state || !pen)) return DDA_ERR_ARG;
    return oc_check(C, d, e, g, p_n, shear_ratio, tan_phi, open_tol, state, pen, cat, cat_order, counts,
                    reinterpret_cast<cudaStream_t>(stream));
}

extern "C" dda_status_t dda_open_close(dda_matrix_t K, dda_contacts_t C, const double* kdiag, const double* F,
                                       const double* e, const double* g, double p_n, double shear_ratio,
                                       double tan_phi, double open_tol, double tol, int32_t maxit, int32_t max_oc,
                                       int32_t* state, double* pen, double* d, int32_t* oc_iters,
                                       int32_t* pcg_iters, int32_t* converged, double* rel_res, void* stream) {
    DDA_NVTX("dda_open_close");
    using namespace dda;
    if (oc_iters) *oc_iters = 0;
    if (pcg_iters) *pcg_iters = 0;
    if (converged) *converged = 0;
    if (!K || !oc_ready(C) || !kdiag || !F || !state || !pen || !d || max_oc < 1) return DDA_ERR_ARG;
    if (C->count > 0 && (!e || !g)) return DDA_ERR_ARG;
    if (K->n != C->n || K->m != 2 * C->count) return DDA_ERR_ARG;
    if (!(p_n >= 0.0) || !(shear_ratio >= 0.0) || !(tan_phi >= 0.0) || !(open_tol >= 0.0)) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    OTmp tmp(st);
    double* Feff = nullptr;
    DDA_CK(tmp.get(&Feff, 6 * (size_t)K->n));
    const int64_t m = C->count;
    if (m > 0) {
        k_oc_pen<<<ogrid(m), OT, 0, st>>>(m, state, p_n, shear_ratio * p_n, pen);
        DDA_LAUNCHED();
    }
    int64_t counts[6];
    int total = 0;
    for (int it = 0; it < max_oc; ++it) {
        dda_status_t s = dda_update_values(K, kdiag, 2 * m, pen, e, g, stream);
        if (s != DDA_OK) return s;
        k_oc_loads<<<ogrid(C->n), OT, 0, st>>>(C->n, C->estart, C->eperm, C->gap, pen, e, g, F, Feff);
        DDA_LAUNCHED();
        int32_t its = 0;
        double rr = 0.0;
        s = dda_pcg_solve(K, Feff, d, d, tol, maxit, DDA_PC_BJ, 1.0, &its, &rr, stream);
        total += its;
        if (pcg_iters) *pcg_iters = total;
        if (rel_res) *rel_res = rr;
        if (s != DDA_OK) return s;
        s = oc_check(C, d, e, g, p_n, shear_ratio, tan_phi, open_tol, state, pen, nullptr, nullptr, counts, st);
        if (s != DDA_OK) return s;
        if (oc_iters) *oc_iters = it + 1;
        if (counts[1] + counts[2] + counts[4] + counts[5] == 0) {
            if (converged) *converged = 1;
            return DDA_OK;
        }
    }
    return DDA_OK;
}

// ---- contact transfer (NEXT-3; reading N3-4; the oracle's O-13): the previous step's records
// sorted by their (v, e) key (radix sort), then a binary search per current record ("sorted search")
namespace dda {
namespace {

__global__ void k_tr_keys(int64_t m, const int32_t* __restrict__ v, const int32_t* __restrict__ e,
                          uint64_t* __restrict__ key, int32_t* __restrict__ idx) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        key[k] = ((uint64_t)(uint32_t)v[k] << 32) | (uint32_t)e[k];
        idx[k] = (int32_t)k;
    }
}

__global__ void k_tr_search(int64_t m, const int32_t* __restrict__ v, const int32_t* __restrict__ e, int64_t mp,
                            const uint64_t* __restrict__ skey, const int32_t* __restrict__ sidx,
                            const int32_t* __restrict__ pstate, int32_t* __restrict__ state,
                            unsigned long long* __restrict__ matched) {
    unsigned long long cnt = 0;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const uint64_t key = ((uint64_t)(uint32_t)v[k] << 32) | (uint32_t)e[k];
        int64_t lo = 0, hi = mp;
        while (lo < hi) {
            const int64_t mid = (lo + hi) >> 1;
            if (skey[mid] < key) lo = mid + 1; else hi = mid;
        }
        if (lo < mp && skey[lo] == key) {
            state[k] = pstate[sidx[lo]];
            ++cnt;
        }
    }
    if (cnt) atomicAdd(matched, cnt);   // a count (integer): order-independent
}

}  // namespace
}  // namespace dda

extern "C" dda_status_t dda_contact_transfer(dda_contacts_t prev, const int32_t* prev_state, dda_contacts_t cur,
                                             int32_t* state, int64_t* matched, void* stream) {
    DDA_NVTX("dda_contact_transfer");
    using namespace dda;
    if (!prev || !cur || (prev->count > 0 && !prev_state) || (cur->count > 0 && !state)) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const int64_t mp = prev->count, m = cur->count;
    OTmp tmp(st);
    uint64_t *key = nullptr, *skey = nullptr;
    int32_t *idx = nullptr, *sidx = nullptr;
    unsigned long long* cnt = nullptr;
    DDA_CK(tmp.get(&key, mp));
    DDA_CK(tmp.get(&skey, mp));
    DDA_CK(tmp.get(&idx, mp));
    DDA_CK(tmp.get(&sidx, mp));
    DDA_CK(tmp.get(&cnt, 1));
    DDA_CK(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long), st));
    if (mp > 0 && m > 0) {
        k_tr_keys<<<ogrid(mp), OT, 0, st>>>(mp, prev->cv, prev->ce, key, idx);
        DDA_LAUNCHED();
        size_t tb = 0;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, key, skey, idx, sidx, (int)mp, 0, 64, st));
        char* ts = nullptr;
        DDA_CK(tmp.get(&ts, tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, key, skey, idx, sidx, (int)mp, 0, 64, st));
        note_launch(4);
        k_tr_search<<<ogrid(m), OT, 0, st>>>(m, cur->cv, cur->ce, mp, skey, sidx, prev_state, state, cnt);
        DDA_LAUNCHED();
    }
    unsigned long long h = 0;
    DDA_CK(cudaMemcpyAsync(&h, cnt, sizeof h, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    if (matched) *matched = (int64_t)h;
    return DDA_OK;
}
