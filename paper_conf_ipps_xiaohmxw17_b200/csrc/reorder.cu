// NEXT-2 — ordering-robust symmetric SpMV: a bandwidth-reducing
// block order.  The symmetric kernel re-reads each transposed block V_ki from L2
// shortly after the warp of row k streamed it from HBM; that reuse needs rows
// that share a block to be close in the processing order (PAPER.md P:180-216
// applies both uses of every stored block).  DDA's block numbering comes from
// the input geometry and can be arbitrary; with a random numbering the kernel
// falls from ~72% to ~44% of HBM (profiles/r01_studies.md).
//
// dda_rcm_order computes the reverse Cuthill-McKee order of the block contact
// graph (vertices = blocks, edges = block pairs coupled by a spring): per
// connected component, BFS from a pseudo-peripheral vertex (repeated BFS to the
// farthest lowest-degree vertex), neighbours visited in increasing degree
// (ties by id), the whole sequence reversed.  Host C++, O(n + m log d); run
// once per contact structure (like a triangular-solve analysis phase).
//
// dda_build_matrix_reordered applies it INSIDE the library: the matrix is
// assembled in the RCM numbering and every entry point that takes or returns block-indexed data
// (vectors, diagonal terms, D^{-1}, the export) permutes at the boundary, so the caller keeps its
// own numbering.  The permutations are device gathers / scatters of 48 B (vectors) or 288 B
// (blocks) per row; a PCG solve permutes F and d once, not per iteration.
#include <algorithm>
#include <cstdint>
#include <numeric>
#include <vector>

#include "dda_internal.cuh"

namespace {

struct Graph {
    std::vector<int64_t> ptr;
    std::vector<int32_t> adj;
};

Graph build_graph(int32_t n, int64_t m, const int32_t* bi, const int32_t* bj) {
    std::vector<int64_t> deg(n + 1, 0);
    for (int64_t s = 0; s < m; ++s) { ++deg[bi[s] + 1]; ++deg[bj[s] + 1]; }
    for (int32_t v = 0; v < n; ++v) deg[v + 1] += deg[v];
    std::vector<int32_t> tmp(deg[n]);
    std::vector<int64_t> fill(deg.begin(), deg.end() - 1);
    for (int64_t s = 0; s < m; ++s) { tmp[fill[bi[s]]++] = bj[s]; tmp[fill[bj[s]]++] = bi[s]; }
    Graph G;
    G.ptr.assign(n + 1, 0);
    for (int32_t v = 0; v < n; ++v) {            // sort + dedup each neighbour list
        auto b = tmp.begin() + deg[v], e = tmp.begin() + deg[v + 1];
        std::sort(b, e);
        G.ptr[v + 1] = G.ptr[v] + (std::unique(b, e) - b);
    }
    G.adj.resize(G.ptr[n]);
    for (int32_t v = 0; v < n; ++v) {
        const int64_t cnt = G.ptr[v + 1] - G.ptr[v];
        std::copy(tmp.begin() + deg[v], tmp.begin() + deg[v] + cnt, G.adj.begin() + G.ptr[v]);
    }
    return G;
}

// BFS from root over unvisited vertices of its component; returns the vertices in BFS order
// (neighbours in increasing degree, then id) and the last level's lowest-degree vertex.
int32_t bfs(const Graph& G, int32_t root, std::vector<int32_t>& level, std::vector<int32_t>& order,
            std::vector<int32_t>& nb) {
    order.clear();
    order.push_back(root);
    level[root] = 0;
    for (size_t h = 0; h < order.size(); ++h) {
        const int32_t v = order[h];
        nb.clear();
        for (int64_t t = G.ptr[v]; t < G.ptr[v + 1]; ++t)
            if (level[G.adj[t]] < 0) nb.push_back(G.adj[t]);
        std::sort(nb.begin(), nb.end(), [&](int32_t a, int32_t b) {
            const int64_t da = G.ptr[a + 1] - G.ptr[a], db = G.ptr[b + 1] - G.ptr[b];
            return da != db ? da < db : a < b;
        });
        for (int32_t w : nb) {
            level[w] = level[v] + 1;
            order.push_back(w);
        }
    }
    const int32_t last = level[order.back()];
    int32_t best = order.back();
    for (auto it = order.rbegin(); it != order.rend() && level[*it] == last; ++it) {
        const int64_t d = G.ptr[*it + 1] - G.ptr[*it], db = G.ptr[best + 1] - G.ptr[best];
        if (d < db || (d == db && *it < best)) best = *it;
    }
    return best;
}

}  // namespace

extern "C" dda_status_t dda_rcm_order(int32_t n, int64_t m, const int32_t* bi, const int32_t* bj, int32_t* perm) {
    DDA_NVTX("dda_rcm_order");
    if (n <= 0 || m < 0 || !perm || (m > 0 && (!bi || !bj))) return DDA_ERR_ARG;
    for (int64_t s = 0; s < m; ++s)
        if (bi[s] < 0 || bi[s] >= n || bj[s] < 0 || bj[s] >= n || bi[s] == bj[s]) return DDA_ERR_ARG;
    const Graph G = build_graph(n, m, bi, bj);
    std::vector<int32_t> level(n, -1), order, nb, out;
    out.reserve(n);
    for (int32_t start = 0; start < n; ++start) {
        if (level[start] >= 0) continue;
        // pseudo-peripheral root: lowest-degree vertex of the component, then repeat
        // BFS from the farthest lowest-degree vertex while the eccentricity grows
        int32_t root = start;
        bfs(G, start, level, order, nb);
        for (int32_t v : order) {
            const int64_t d = G.ptr[v + 1] - G.ptr[v], dr = G.ptr[root + 1] - G.ptr[root];
            if (d < dr || (d == dr && v < root)) root = v;
        }
        int32_t ecc = -1;
        for (int it = 0; it < 8; ++it) {
            for (int32_t v : order) level[v] = -1;
            const int32_t far = bfs(G, root, level, order, nb);
            const int32_t e = level[order.back()];
            if (e <= ecc) break;
            ecc = e;
            if (it + 1 < 8) {
                for (int32_t v : order) level[v] = -1;
                root = far;
                bfs(G, root, level, order, nb);
            }
        }
        out.insert(out.end(), order.begin(), order.end());
    }
    // reverse Cuthill-McKee: perm[new] = old
    for (int32_t k = 0; k < n; ++k) perm[k] = out[n - 1 - k];
    return DDA_OK;
}

namespace dda {
namespace {

// out[w*new + c] = in[w*perm[new] + c] (gather into the internal order) or, with scatter,
// out[w*perm[new] + c] = in[w*new + c]; w doubles per row
template <bool SCATTER>
__global__ void k_permute(int32_t n, int w, const int32_t* __restrict__ perm, const double* __restrict__ in,
                          double* __restrict__ out) {
    const int64_t total = (int64_t)n * w;
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = t / w, c = t - r * w;
        const int64_t u = perm[r];
        if (SCATTER) out[u * w + c] = in[t];
        else out[t] = in[u * w + c];
    }
}

__global__ void k_map_ids(int64_t m, const int32_t* __restrict__ inv, const int32_t* __restrict__ src,
                          int32_t* __restrict__ dst, int32_t n, int* __restrict__ err) {
    for (int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; s < m; s += (int64_t)gridDim.x * blockDim.x) {
        const int32_t v = src[s];
        if (v < 0 || v >= n) { atomicOr(err, 1); dst[s] = 0; }
        else dst[s] = inv[v];
    }
}

inline int pgrid(int64_t items) {
    int64_t g = (items + 255) / 256;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 16;
    return (int)(g < cap ? g : cap);
}

dda_status_t gather(dda_matrix* K, int w, const double* in, double* out, cudaStream_t st) {
    k_permute<false><<<pgrid((int64_t)K->n * w), 256, 0, st>>>(K->n, w, K->rperm, in, out);
    DDA_LAUNCHED();
    return DDA_OK;
}
dda_status_t scatter(dda_matrix* K, int w, const double* in, double* out, cudaStream_t st) {
    k_permute<true><<<pgrid((int64_t)K->n * w), 256, 0, st>>>(K->n, w, K->rperm, in, out);
    DDA_LAUNCHED();
    return DDA_OK;
}

dda_status_t ensure_rtmp(dda_matrix* K, cudaStream_t st) {
    if (!K->rtmp) DDA_CK(dev_alloc(reinterpret_cast<void**>(&K->rtmp), 3 * 6 * (size_t)K->n * sizeof(double), st));
    return DDA_OK;
}

}  // namespace

dda_status_t ro_spmv(dda_matrix* K, const double* x, double* y, cudaStream_t st, bool full) {
    dda_status_t s = ensure_rtmp(K, st);
    if (s != DDA_OK) return s;
    double *tx = K->rtmp, *ty = K->rtmp + 6 * (size_t)K->n;
    if ((s = gather(K, 6, x, tx, st)) != DDA_OK) return s;
    s = full ? spmv_full(K, tx, ty, st) : spmv(K, tx, ty, st);
    if (s != DDA_OK) return s;
    return scatter(K, 6, ty, y, st);
}

dda_status_t ro_pcg(dda_matrix* K, const double* F, const double* d0, double* d, double tol, int32_t maxit,
                    dda_precond_t pc, double omega, int32_t* iters, double* rel_res, cudaStream_t st) {
    if (iters) *iters = 0;
    if (rel_res) *rel_res = 0.0;
    if (!F || !d) return DDA_ERR_ARG;
    dda_status_t s = ensure_rtmp(K, st);
    if (s != DDA_OK) return s;
    const size_t N = 6 * (size_t)K->n;
    double *tF = K->rtmp, *td = K->rtmp + N, *td0 = K->rtmp + 2 * N;
    if ((s = gather(K, 6, F, tF, st)) != DDA_OK) return s;
    if (d0 && (s = gather(K, 6, d0, td0, st)) != DDA_OK) return s;
    const dda_status_t r = pcg_entry(K, tF, d0 ? td0 : nullptr, td, tol, maxit, pc, omega, iters, rel_res, st);
    if (r != DDA_OK && r != DDA_ERR_NO_CONVERGENCE && r != DDA_ERR_BREAKDOWN) return r;
    if ((s = scatter(K, 6, td, d, st)) != DDA_OK) return s;
    DDA_CK(cudaStreamSynchronize(st));
    return r;
}

dda_status_t ro_precond(dda_matrix* K, dda_precond_t pc, double omega, const double* r, double* z, cudaStream_t st) {
    dda_status_t s = ensure_rtmp(K, st);
    if (s != DDA_OK) return s;
    double *tr = K->rtmp, *tz = K->rtmp + 6 * (size_t)K->n;
    if ((s = gather(K, 6, r, tr, st)) != DDA_OK) return s;
    if ((s = precond_apply(K, pc, omega, tr, tz, st)) != DDA_OK) return s;
    if ((s = scatter(K, 6, tz, z, st)) != DDA_OK) return s;
    DDA_CK(cudaStreamSynchronize(st));
    return DDA_OK;
}

dda_status_t ro_bj_setup(dda_matrix* K, double* dinv_full, int32_t* bad_block, cudaStream_t st) {
    double* tmp = nullptr;
    if (dinv_full) DDA_CK(dev_alloc(reinterpret_cast<void**>(&tmp), (size_t)kBlk * K->n * sizeof(double), st));
    int32_t bad = -1;
    dda_status_t s = bj_setup(K, st, &bad, tmp);
    if (bad_block) {
        *bad_block = -1;
        if (bad >= 0) DDA_CK(cudaMemcpy(bad_block, K->rperm + bad, sizeof(int32_t), cudaMemcpyDeviceToHost));
    }
    if (s == DDA_OK && tmp) s = scatter(K, kBlk, tmp, dinv_full, st);
    if (tmp) {
        cudaStreamSynchronize(st);
        dev_free_on(tmp, st);
    }
    return s;
}

dda_status_t ro_update_values(dda_matrix* K, const double* kdiag, const double* pen, const double* e, const double* g,
                              cudaStream_t st) {
    double* kd = nullptr;
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&kd), (size_t)kBlk * K->n * sizeof(double), st));
    dda_status_t s = gather(K, kBlk, kdiag, kd, st);
    if (s == DDA_OK) s = run_values(K, kd, pen, e, g, st);
    dev_free_on(kd, st);
    return s;
}

// the canonical export (A2) in the caller's numbering: internal block (a, b) is the caller's
// (perm[a], perm[b]), stored at (min, max) and transposed when perm[a] > perm[b]; then the CSR and
// the lower (CSC) arrays are rebuilt by sorting, exactly as A2 defines them
dda_status_t ro_export(dda_matrix* K, int32_t* row_ptr, int32_t* col_idx, int32_t* low_ptr, int32_t* low_row,
                       int32_t* low_to_up, double* diag, double* upper) {
    const int32_t n = K->n;
    const size_t z = (size_t)K->nnzb;
    std::vector<int32_t> rp(n + 1), ci(z ? z : 1), perm(n);
    std::vector<double> dg((size_t)n * kBlk), up(z ? z * kBlk : 1);
    dda_status_t s = export_internal(K, rp.data(), ci.data(), nullptr, nullptr, nullptr, dg.data(), up.data());
    if (s != DDA_OK) return s;
    DDA_CK(cudaMemcpy(perm.data(), K->rperm, n * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (diag)
        for (int32_t a = 0; a < n; ++a) std::copy(&dg[(size_t)kBlk * a], &dg[(size_t)kBlk * a] + kBlk, diag + (size_t)kBlk * perm[a]);
    struct Ent { int32_t r, c; int64_t src; bool tr; };
    std::vector<Ent> ent(z);
    for (int32_t a = 0; a < n; ++a)
        for (int32_t u = rp[a]; u < rp[a + 1]; ++u) {
            const int32_t pa = perm[a], pb = perm[ci[u]];
            ent[u] = pa < pb ? Ent{pa, pb, u, false} : Ent{pb, pa, u, true};
        }
    std::sort(ent.begin(), ent.end(), [](const Ent& x, const Ent& y) { return x.r != y.r ? x.r < y.r : x.c < y.c; });
    if (row_ptr) {
        std::fill(row_ptr, row_ptr + n + 1, 0);
        for (const Ent& x : ent) ++row_ptr[x.r + 1];
        for (int32_t v = 0; v < n; ++v) row_ptr[v + 1] += row_ptr[v];
    }
    if (col_idx)
        for (size_t u = 0; u < z; ++u) col_idx[u] = ent[u].c;
    if (upper)
        for (size_t u = 0; u < z; ++u) {
            const double* B = &up[(size_t)kBlk * ent[u].src];
            for (int r = 0; r < 6; ++r)
                for (int c = 0; c < 6; ++c) upper[kBlk * u + 6 * r + c] = ent[u].tr ? B[6 * c + r] : B[6 * r + c];
        }
    if (low_ptr || low_row || low_to_up) {
        std::vector<int64_t> ord(z);
        std::iota(ord.begin(), ord.end(), 0);
        std::stable_sort(ord.begin(), ord.end(), [&](int64_t x, int64_t y) {
            return ent[x].c != ent[y].c ? ent[x].c < ent[y].c : ent[x].r < ent[y].r;
        });
        if (low_ptr) {
            std::fill(low_ptr, low_ptr + n + 1, 0);
            for (const Ent& x : ent) ++low_ptr[x.c + 1];
            for (int32_t v = 0; v < n; ++v) low_ptr[v + 1] += low_ptr[v];
        }
        for (size_t t = 0; t < z; ++t) {
            if (low_row) low_row[t] = ent[ord[t]].r;
            if (low_to_up) low_to_up[t] = (int32_t)ord[t];
        }
    }
    return DDA_OK;
}

}  // namespace dda

extern "C" dda_status_t dda_build_matrix_reordered(int32_t n, const double* kdiag, int64_t m, const int32_t* bi,
                                                   const int32_t* bj, const double* pen, const double* e,
                                                   const double* g, void* stream, dda_matrix_t* out) {
    DDA_NVTX("dda_build_matrix_reordered");
    using namespace dda;
    if (!out) return DDA_ERR_ARG;
    *out = nullptr;
    if (n <= 0 || m < 0 || !kdiag || (m > 0 && (!bi || !bj))) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    // the RCM order of the contact graph (host; once per contact structure)
    std::vector<int32_t> hbi(m > 0 ? m : 1), hbj(m > 0 ? m : 1), perm(n), inv(n);
    if (m > 0) {
        DDA_CK(cudaMemcpyAsync(hbi.data(), bi, m * sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaMemcpyAsync(hbj.data(), bj, m * sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        DDA_CK(cudaStreamSynchronize(st));
    }
    dda_status_t s = dda_rcm_order(n, m, hbi.data(), hbj.data(), perm.data());
    if (s != DDA_OK) return s;
    for (int32_t k = 0; k < n; ++k) inv[perm[k]] = k;
    int32_t *dperm = nullptr, *dinv = nullptr, *lbi = nullptr, *lbj = nullptr;
    double* lkd = nullptr;
    int* err = nullptr;
    auto release = [&]() {
        for (void* p : {(void*)lbi, (void*)lbj, (void*)lkd, (void*)err}) if (p) dev_free_on(p, st);
    };
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&dperm), n * sizeof(int32_t), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&dinv), n * sizeof(int32_t), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&lbi), (m > 0 ? m : 1) * sizeof(int32_t), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&lbj), (m > 0 ? m : 1) * sizeof(int32_t), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&lkd), (size_t)kBlk * n * sizeof(double), st));
    DDA_CK(dev_alloc(reinterpret_cast<void**>(&err), sizeof(int), st));
    DDA_CK(cudaMemsetAsync(err, 0, sizeof(int), st));
    DDA_CK(cudaMemcpyAsync(dperm, perm.data(), n * sizeof(int32_t), cudaMemcpyHostToDevice, st));
    DDA_CK(cudaMemcpyAsync(dinv, inv.data(), n * sizeof(int32_t), cudaMemcpyHostToDevice, st));
    if (m > 0) {
        k_map_ids<<<pgrid(m), 256, 0, st>>>(m, dinv, bi, lbi, n, err);
        DDA_LAUNCHED();
        k_map_ids<<<pgrid(m), 256, 0, st>>>(m, dinv, bj, lbj, n, err);
        DDA_LAUNCHED();
    }
    k_permute<false><<<pgrid((int64_t)n * kBlk), 256, 0, st>>>(n, kBlk, dperm, kdiag, lkd);
    DDA_LAUNCHED();
    dda_matrix_t K = nullptr;
    s = build_matrix_impl(n, lkd, m, lbi, lbj, pen, e, g, st, nullptr, &K);
    release();
    if (s != DDA_OK) {
        dev_free_on(dperm, st);
        dev_free_on(dinv, st);
        return s;
    }
    K->rperm = dperm;
    K->rinv = dinv;
    *out = K;
    return DDA_OK;
}
