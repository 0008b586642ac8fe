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
#include <algorithm>
#include <cstdint>
#include <vector>

#include "dda.h"

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
