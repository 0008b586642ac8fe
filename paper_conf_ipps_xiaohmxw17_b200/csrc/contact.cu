// NEXT-3 — contact detection on the GPU (§III.B, §III.A) and the springs of
// its vertex-edge contacts (the input of the assembly).
//
// What is computed (reading N3; the oracle's O-8 / O-9 are the definition): blocks are
// polygons with counter-clockwise vertices; for every vertex v of a block i and every edge e of
// another block j,
//     d = Q2 - Q1, w = P - Q1, L2 = d.d, tn = w.d, t = clamp(tn / L2, 0, 1), C = Q1 + t d,
//     dist2 = |P - C|^2,
// (v, e) is a contact iff dist2 < d0^2, typed VE if 0 < tn < L2 and VV otherwise.  The
// products and sums are rounded as written (__dmul_rn / __dadd_rn, no FMA contraction), so every
// decision, t and dist2 are bit-identical to the oracle's.  Records come out in increasing (v, e).
//
// B200 design (the paper's broad phase is an n x n/2 all-pairs matrix in m x m tiles, P:86 — O(n^2),
// prior art for its 4k-block cases; here a sort-based uniform grid keeps it O(n) at 1M blocks):
//   1. per-block AABBs and their global extent (one pass, order-preserving u64 atomics);
//   2. cell = floor((min corner - origin) / h) with h >= max block extent + d0, so two blocks within
//      d0 of each other sit in the same or adjacent cells; CUB radix sort of (cell key, block);
//   3. broad phase: each block scans the 3x3 neighbouring cells for blocks j > i whose AABBs, one of
//      them grown by d0, overlap — count, scan, fill (deterministic: sorted cells, fixed scan order);
//   4. narrow phase: one thread per candidate pair tests i's vertices against j's edges and j's
//      vertices against i's edges — count, scan, fill;
//   5. canonical order: radix sort by the 64-bit key (v << 32) | e, then a gather.
// Springs: one thread per VE record (a scan gives its two spring slots): normal and shear springs,
// e = T_i(P)^T n, g = -((1 - t) T_j(Q1)^T n + t T_j(Q2)^T n) with Shi's first-order T.
#include <cub/cub.cuh>

#include <climits>
#include <cmath>
#include <cstring>
#include <vector>

#include "dda_internal.cuh"

namespace dda {
namespace {

constexpr int CT = 256;

inline int cgrid(int64_t items) {
    int64_t g = (items + CT - 1) / CT;
    if (g < 1) g = 1;
    const int64_t cap = (int64_t)device_sms() * 32;
    return (int)(g < cap ? g : cap);
}

// order-preserving map of a double to u64 (atomicMin / atomicMax of doubles of any sign)
__device__ __forceinline__ unsigned long long ord(double x) {
    const unsigned long long b = (unsigned long long)__double_as_longlong(x);
    return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__host__ inline double unord(unsigned long long u) {
    const unsigned long long b = (u >> 63) ? (u & 0x7fffffffffffffffull) : ~u;
    double x;
    memcpy(&x, &b, sizeof x);
    return x;
}

// ext[0..4] = ord(min x), ord(min y), ord(max x), ord(max y), ord(max block extent); err on bad polygons
__global__ void k_boxes(int32_t n, const int32_t* __restrict__ vptr, const double* __restrict__ vxy,
                        double4* __restrict__ box, unsigned long long* __restrict__ ext, int* __restrict__ err) {
    unsigned long long mnx = ~0ull, mny = ~0ull, mxx = 0, mxy = 0, mxe = 0;
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < n; b += (int64_t)gridDim.x * blockDim.x) {
        const int32_t a = vptr[b], z = vptr[b + 1];
        if (z - a < 3) { atomicOr(err, 1); continue; }
        double x0 = INFINITY, y0 = INFINITY, x1 = -INFINITY, y1 = -INFINITY;
        for (int32_t v = a; v < z; ++v) {
            const double2 p = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)v);
            if (!isfinite(p.x) || !isfinite(p.y)) atomicOr(err, 1);
            x0 = fmin(x0, p.x); y0 = fmin(y0, p.y); x1 = fmax(x1, p.x); y1 = fmax(y1, p.y);
        }
        box[b] = make_double4(x0, y0, x1, y1);
        mnx = min(mnx, ord(x0)); mny = min(mny, ord(y0)); mxx = max(mxx, ord(x1)); mxy = max(mxy, ord(y1));
        mxe = max(mxe, ord(fmax(x1 - x0, y1 - y0)));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mnx = min(mnx, __shfl_xor_sync(0xffffffffu, mnx, o));
        mny = min(mny, __shfl_xor_sync(0xffffffffu, mny, o));
        mxx = max(mxx, __shfl_xor_sync(0xffffffffu, mxx, o));
        mxy = max(mxy, __shfl_xor_sync(0xffffffffu, mxy, o));
        mxe = max(mxe, __shfl_xor_sync(0xffffffffu, mxe, o));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicMin(ext + 0, mnx); atomicMin(ext + 1, mny);
        atomicMax(ext + 2, mxx); atomicMax(ext + 3, mxy); atomicMax(ext + 4, mxe);
    }
}

struct Grid {
    double ox, oy, h;
    int64_t nx, ny;
};

__device__ __forceinline__ int64_t cell_x(const Grid& G, double x) {
    int64_t c = (int64_t)floor((x - G.ox) / G.h);
    return c < 0 ? 0 : (c >= G.nx ? G.nx - 1 : c);
}
__device__ __forceinline__ int64_t cell_y(const Grid& G, double y) {
    int64_t c = (int64_t)floor((y - G.oy) / G.h);
    return c < 0 ? 0 : (c >= G.ny ? G.ny - 1 : c);
}

__global__ void k_cellkeys(int32_t n, Grid G, const double4* __restrict__ box, uint64_t* __restrict__ key,
                           int32_t* __restrict__ id) {
    for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < n; b += (int64_t)gridDim.x * blockDim.x) {
        const double4 B = box[b];
        key[b] = (uint64_t)(cell_y(G, B.y) * G.nx + cell_x(G, B.x));
        id[b] = (int32_t)b;
    }
}

// cstart[c] = first sorted position with key >= c, c = 0..ncell
__global__ void k_cellstart(int32_t n, int64_t ncell, const uint64_t* __restrict__ skey, int32_t* __restrict__ cstart) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t <= n; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t prev = (t == 0) ? -1 : (int64_t)skey[t - 1];
        const int64_t cur = (t == n) ? ncell : (int64_t)skey[t];
        for (int64_t c = prev + 1; c <= cur; ++c) cstart[c] = (int32_t)t;
    }
}

__device__ __forceinline__ bool near_boxes(const double4& A, const double4& B, double d0) {
    return A.x - d0 <= B.z && B.x <= A.z + d0 && A.y - d0 <= B.w && B.y <= A.w + d0;
}

// broad phase: candidate pairs (i, j), j > i, in the 3x3 cells around i's cell.  FILL = false counts.
template <bool FILL>
__global__ void k_broad(int32_t n, Grid G, double d0, const double4* __restrict__ box,
                        const int32_t* __restrict__ cstart, const int32_t* __restrict__ sid,
                        int32_t* __restrict__ cnt, const int64_t* __restrict__ off, int2* __restrict__ pairs) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double4 A = box[i];
        const int64_t cx = cell_x(G, A.x), cy = cell_y(G, A.y);
        int32_t c = 0;
        int64_t o = FILL ? off[i] : 0;
        for (int64_t yy = cy - 1; yy <= cy + 1; ++yy) {
            if (yy < 0 || yy >= G.ny) continue;
            for (int64_t xx = cx - 1; xx <= cx + 1; ++xx) {
                if (xx < 0 || xx >= G.nx) continue;
                const int64_t cell = yy * G.nx + xx;
                for (int32_t t = cstart[cell]; t < cstart[cell + 1]; ++t) {
                    const int32_t j = sid[t];
                    if (j <= i || !near_boxes(A, box[j], d0)) continue;
                    if (FILL) pairs[o++] = make_int2((int32_t)i, j);
                    else ++c;
                }
            }
        }
        if (!FILL) cnt[i] = c;
    }
}

// the oracle's O-8 test for vertex P against edge (Q1 -> Q2), rounded as written
struct VE {
    bool hit;
    int type;
    double t, dist2;
};
__device__ __forceinline__ VE ve_test(double px, double py, double q1x, double q1y, double q2x, double q2y, double r2) {
    const double dx = __dsub_rn(q2x, q1x), dy = __dsub_rn(q2y, q1y);
    const double wx = __dsub_rn(px, q1x), wy = __dsub_rn(py, q1y);
    const double L2 = __dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy));
    const double tn = __dadd_rn(__dmul_rn(wx, dx), __dmul_rn(wy, dy));
    double t = __ddiv_rn(tn, L2);
    if (t < 0.0) t = 0.0;
    if (t > 1.0) t = 1.0;
    const double cx = __dadd_rn(q1x, __dmul_rn(t, dx)), cy = __dadd_rn(q1y, __dmul_rn(t, dy));
    const double ex = __dsub_rn(px, cx), ey = __dsub_rn(py, cy);
    VE r;
    r.dist2 = __dadd_rn(__dmul_rn(ex, ex), __dmul_rn(ey, ey));
    r.hit = r.dist2 < r2;
    r.type = (tn > 0.0 && tn < L2) ? 0 : 1;
    r.t = t;
    return r;
}

// narrow phase over one pair: vertices of `a` against edges of `b`, then of `b` against `a`
template <bool FILL>
__global__ void k_narrow(int64_t npairs, const int2* __restrict__ pairs, const int32_t* __restrict__ vptr,
                         const double* __restrict__ vxy, double r2, int32_t* __restrict__ cnt,
                         const int64_t* __restrict__ off, uint64_t* __restrict__ key, int32_t* __restrict__ ci,
                         int32_t* __restrict__ cv, int32_t* __restrict__ cj, int32_t* __restrict__ ce,
                         int32_t* __restrict__ ctype, double* __restrict__ ct, double* __restrict__ cd2) {
    for (int64_t p = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < npairs; p += (int64_t)gridDim.x * blockDim.x) {
        const int2 pr = pairs[p];
        int32_t c = 0;
        int64_t o = FILL ? off[p] : 0;
#pragma unroll 1
        for (int side = 0; side < 2; ++side) {
            const int32_t i = side ? pr.y : pr.x, j = side ? pr.x : pr.y;
            const int32_t va = vptr[i], vz = vptr[i + 1], ea = vptr[j], ez = vptr[j + 1];
            for (int32_t v = va; v < vz; ++v) {
                const double2 P = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)v);
                for (int32_t e = ea; e < ez; ++e) {
                    const int32_t e2 = (e + 1 < ez) ? e + 1 : ea;
                    const double2 Q1 = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)e);
                    const double2 Q2 = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)e2);
                    const VE r = ve_test(P.x, P.y, Q1.x, Q1.y, Q2.x, Q2.y, r2);
                    if (!r.hit) continue;
                    if (FILL) {
                        key[o] = ((uint64_t)(uint32_t)v << 32) | (uint32_t)e;
                        ci[o] = i; cv[o] = v; cj[o] = j; ce[o] = e; ctype[o] = r.type; ct[o] = r.t; cd2[o] = r.dist2;
                        ++o;
                    } else {
                        ++c;
                    }
                }
            }
        }
        if (!FILL) cnt[p] = c;
    }
}

template <class T>
__global__ void k_gather(int64_t m, const int32_t* __restrict__ idx, const T* __restrict__ src, T* __restrict__ dst) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x)
        dst[t] = src[idx[t]];
}

__global__ void k_iota(int64_t m, int32_t* __restrict__ v) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x)
        v[t] = (int32_t)t;
}

__global__ void k_isve(int64_t m, const int32_t* __restrict__ ctype, int32_t* __restrict__ f) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x)
        f[t] = ctype[t] == 0 ? 1 : 0;
}

// Angle judgment and VV1 / VV2 split (reading N3-2, the oracle's O-10): key = class + 1 (0 abandoned,
// 1 VE, 2 VV1, 3 VV2), every product and sum rounded as written (__dmul_rn / __dadd_rn / __dsub_rn)
__global__ void k_classify(int64_t m, const int32_t* __restrict__ vptr, const double* __restrict__ vxy,
                           const int32_t* __restrict__ ci, const int32_t* __restrict__ cv,
                           const int32_t* __restrict__ cj, const int32_t* __restrict__ ce,
                           const int32_t* __restrict__ ctype, double s2, uint32_t* __restrict__ key,
                           int32_t* __restrict__ idx) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t i = ci[k], v = cv[k], j = cj[k], q = ce[k];
        const int32_t vp = (v > vptr[i]) ? v - 1 : vptr[i + 1] - 1;
        const int32_t vn = (v + 1 < vptr[i + 1]) ? v + 1 : vptr[i];
        const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
        const double2 P = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)v);
        const double2 Pa = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)vp);
        const double2 Pb = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)vn);
        const double2 Q1 = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)q);
        const double2 Q2 = *reinterpret_cast<const double2*>(vxy + 2 * (size_t)q2);
        const double ax = __dsub_rn(Pa.x, P.x), ay = __dsub_rn(Pa.y, P.y);
        const double bx = __dsub_rn(Pb.x, P.x), by = __dsub_rn(Pb.y, P.y);
        const double dx = __dsub_rn(Q2.x, Q1.x), dy = __dsub_rn(Q2.y, Q1.y);
        const double Nx = dy, Ny = -dx;
        const double NN = __dadd_rn(__dmul_rn(Nx, Nx), __dmul_rn(Ny, Ny));
        const double aa = __dadd_rn(__dmul_rn(ax, ax), __dmul_rn(ay, ay));
        const double bb = __dadd_rn(__dmul_rn(bx, bx), __dmul_rn(by, by));
        const double lim = __dmul_rn(s2, NN);
        const bool convex = __dsub_rn(__dmul_rn(ax, by), __dmul_rn(ay, bx)) < 0.0;
        const double fa = __dadd_rn(__dmul_rn(Nx, ax), __dmul_rn(Ny, ay));
        const double fb = __dadd_rn(__dmul_rn(Nx, bx), __dmul_rn(Ny, by));
        const bool out_a = fa >= 0.0 || __dmul_rn(fa, fa) <= __dmul_rn(lim, aa);
        const bool out_b = fb >= 0.0 || __dmul_rn(fb, fb) <= __dmul_rn(lim, bb);
        uint32_t c;
        if (!(convex && out_a && out_b)) {
            c = 0;
        } else if (ctype[k] == 0) {
            c = 1;
        } else {
            const double xa = __dsub_rn(__dmul_rn(dx, ay), __dmul_rn(dy, ax));
            const double xb = __dsub_rn(__dmul_rn(dx, by), __dmul_rn(dy, bx));
            const bool par = __dmul_rn(xa, xa) <= __dmul_rn(lim, aa) || __dmul_rn(xb, xb) <= __dmul_rn(lim, bb);
            c = par ? 2 : 3;
        }
        key[k] = c;
        idx[k] = (int32_t)k;
    }
}

// start[c] = first position of key c in the sorted keys (c = 0..3; start[4] = m), set by the heads
__global__ void k_class_bounds(int64_t m, const uint32_t* __restrict__ skey, int64_t* __restrict__ start) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t c = skey[t];
        const uint32_t p = t > 0 ? skey[t - 1] : 0u;
        if (t == 0) for (uint32_t z = 0; z <= c; ++z) start[z] = 0;
        else for (uint32_t z = p + 1; z <= c; ++z) start[z] = t;
        if (t == m - 1) for (uint32_t z = c + 1; z <= 4; ++z) start[z] = m;
    }
}

__global__ void k_class_type(int64_t m, const uint32_t* __restrict__ skey, int32_t* __restrict__ type) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < m; t += (int64_t)gridDim.x * blockDim.x)
        type[t] = (int32_t)skey[t] - 1;
}

// T(P)^T u for Shi's first-order T at offset (x, y) from the centroid, rounded as the oracle writes it
__device__ __forceinline__ void tt_times(double x, double y, double ux, double uy, double* o) {
    o[0] = ux;
    o[1] = uy;
    o[2] = __dadd_rn(__dmul_rn(-y, ux), __dmul_rn(x, uy));
    o[3] = __dmul_rn(x, ux);
    o[4] = __dmul_rn(y, uy);
    o[5] = __dadd_rn(__dmul_rn(__dmul_rn(0.5, y), ux), __dmul_rn(__dmul_rn(0.5, x), uy));
}

__global__ void k_springs(int64_t m, const int32_t* __restrict__ slot, const int32_t* __restrict__ vptr,
                          const double* __restrict__ vxy, const double* __restrict__ cxy,
                          const int32_t* __restrict__ ci, const int32_t* __restrict__ cv,
                          const int32_t* __restrict__ cj, const int32_t* __restrict__ ce,
                          const int32_t* __restrict__ ctype, const double* __restrict__ ct, double p_n, double ps,
                          int32_t* __restrict__ bi, int32_t* __restrict__ bj, double* __restrict__ pen,
                          double* __restrict__ e, double* __restrict__ g, int all) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < m; k += (int64_t)gridDim.x * blockDim.x) {
        if (!all && ctype[k] != 0) continue;
        const int32_t i = ci[k], j = cj[k], v = cv[k], q = ce[k];
        const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
        const double dx = __dsub_rn(vxy[2 * (size_t)q2], vxy[2 * (size_t)q]);
        const double dy = __dsub_rn(vxy[2 * (size_t)q2 + 1], vxy[2 * (size_t)q + 1]);
        const double len = __dsqrt_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)));
        const double ux = __ddiv_rn(dx, len), uy = __ddiv_rn(dy, len);
        const double t = ct[k];
        const double pix = __dsub_rn(vxy[2 * (size_t)v], cxy[2 * (size_t)i]);
        const double piy = __dsub_rn(vxy[2 * (size_t)v + 1], cxy[2 * (size_t)i + 1]);
        const double q1x = __dsub_rn(vxy[2 * (size_t)q], cxy[2 * (size_t)j]);
        const double q1y = __dsub_rn(vxy[2 * (size_t)q + 1], cxy[2 * (size_t)j + 1]);
        const double q2x = __dsub_rn(vxy[2 * (size_t)q2], cxy[2 * (size_t)j]);
        const double q2y = __dsub_rn(vxy[2 * (size_t)q2 + 1], cxy[2 * (size_t)j + 1]);
        const double omt = __dsub_rn(1.0, t);
        const int64_t s0 = 2 * (all ? k : (int64_t)slot[k]);
#pragma unroll
        for (int sp = 0; sp < 2; ++sp) {
            const double nx = sp == 0 ? uy : ux, ny = sp == 0 ? -ux : uy;
            double a[6], b1[6], b2[6];
            tt_times(pix, piy, nx, ny, a);
            tt_times(q1x, q1y, nx, ny, b1);
            tt_times(q2x, q2y, nx, ny, b2);
            const int64_t s = s0 + sp;
            bi[s] = i;
            bj[s] = j;
            pen[s] = sp == 0 ? p_n : ps;
#pragma unroll
            for (int r = 0; r < 6; ++r) {
                e[6 * s + r] = a[r];
                g[6 * s + r] = -__dadd_rn(__dmul_rn(omt, b1[r]), __dmul_rn(t, b2[r]));
            }
        }
    }
}

struct CTmp {
    cudaStream_t s;
    std::vector<void*> ptrs;
    explicit CTmp(cudaStream_t st) : s(st) {}
    template <class T>
    cudaError_t get(T** p, size_t count) {
        void* q = nullptr;
        cudaError_t e = dev_alloc(&q, count ? count * sizeof(T) : 16, s);
        if (e == cudaSuccess) ptrs.push_back(q);
        *p = reinterpret_cast<T*>(q);
        return e;
    }
    ~CTmp() {
        for (void* p : ptrs) dev_free_on(p, s);
    }
};

// exclusive scan of int32 counts into int64 offsets (+ total), stream-ordered, total read back
cudaError_t scan_counts(const int32_t* cnt, int64_t items, int64_t* off, int64_t* total, CTmp& tmp) {
    if (items == 0) { *total = 0; return cudaSuccess; }
    size_t tb = 0;
    cudaError_t e = cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, off, items + 1, tmp.s);
    if (e != cudaSuccess) return e;
    void* ts = nullptr;
    e = tmp.get(reinterpret_cast<char**>(&ts), tb);
    if (e != cudaSuccess) return e;
    // cnt has items entries; the scan over items + 1 reads one past: the caller allocates cnt[items] = 0
    e = cub::DeviceScan::ExclusiveSum(ts, tb, cnt, off, items + 1, tmp.s);
    if (e != cudaSuccess) return e;
    e = cudaMemcpyAsync(total, off + items, sizeof(int64_t), cudaMemcpyDeviceToHost, tmp.s);
    if (e != cudaSuccess) return e;
    return cudaStreamSynchronize(tmp.s);
}

}  // namespace
}  // namespace dda

using namespace dda;

extern "C" void dda_contacts_free(dda_contacts_t C) {
    if (!C) return;
    int prev = 0;
    cudaGetDevice(&prev);
    cudaSetDevice(C->device);
    cudaDeviceSynchronize();
    void* ptrs[] = {C->ci, C->cv, C->cj, C->ce, C->ctype, C->ct, C->cd2, C->gap, C->eperm, C->estart};
    for (void* p : ptrs)
        if (p) dev_free(p);
    cudaSetDevice(prev);
    delete C;
}

extern "C" dda_status_t dda_detect_contacts(int32_t n, const int32_t* vptr, const double* vxy, double d0,
                                            void* stream, dda_contacts_t* out) {
    DDA_NVTX("dda_detect_contacts");
    if (!out) return DDA_ERR_ARG;
    *out = nullptr;
    if (n <= 0 || !vptr || !vxy || !(d0 > 0.0) || !isfinite(d0)) return DDA_ERR_ARG;
    if (reinterpret_cast<uintptr_t>(vxy) & 15) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    dda_contacts* C = new dda_contacts();
    struct Guard {
        dda_contacts* C;
        bool keep = false;
        ~Guard() { if (!keep) dda_contacts_free(C); }
    } guard{C};
    DDA_CK(cudaGetDevice(&C->device));
    C->n = n;
    C->vptr = vptr;
    C->vxy = vxy;
    CTmp tmp(st);

    // ---- 1. boxes and extent
    double4* box = nullptr;
    unsigned long long* ext = nullptr;
    int* err = nullptr;
    DDA_CK(tmp.get(&box, n));
    DDA_CK(tmp.get(&ext, 5));
    DDA_CK(tmp.get(&err, 1));
    const unsigned long long init[5] = {~0ull, ~0ull, 0ull, 0ull, 0ull};
    DDA_CK(cudaMemcpyAsync(ext, init, sizeof init, cudaMemcpyHostToDevice, st));
    DDA_CK(cudaMemsetAsync(err, 0, sizeof(int), st));
    k_boxes<<<cgrid(n), CT, 0, st>>>(n, vptr, vxy, box, ext, err);
    DDA_LAUNCHED();
    unsigned long long hext[5];
    int herr = 0;
    DDA_CK(cudaMemcpyAsync(hext, ext, sizeof hext, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaMemcpyAsync(&herr, err, sizeof herr, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    if (herr) return DDA_ERR_ARG;
    Grid G;
    G.ox = unord(hext[0]);
    G.oy = unord(hext[1]);
    const double wx = unord(hext[2]) - G.ox, wy = unord(hext[3]) - G.oy;
    G.h = (unord(hext[4]) + d0) * (1.0 + 1e-9);   // margin: near blocks stay in adjacent cells after rounding
    // cells only affect speed (h >= max extent + d0 keeps near blocks in adjacent cells): coarsen the
    // grid until it has at most ~2 cells per block
    for (;;) {
        G.nx = (int64_t)floor(wx / G.h) + 1;
        G.ny = (int64_t)floor(wy / G.h) + 1;
        if (G.nx * G.ny <= 2 * (int64_t)n + 64) break;
        G.h *= 1.25;
    }
    const int64_t ncell = G.nx * G.ny;

    // ---- 2. cell keys, sort, cell starts
    uint64_t *key = nullptr, *skey = nullptr;
    int32_t *id = nullptr, *sid = nullptr, *cstart = nullptr;
    DDA_CK(tmp.get(&key, n));
    DDA_CK(tmp.get(&skey, n));
    DDA_CK(tmp.get(&id, n));
    DDA_CK(tmp.get(&sid, n));
    DDA_CK(tmp.get(&cstart, ncell + 1));
    k_cellkeys<<<cgrid(n), CT, 0, st>>>(n, G, box, key, id);
    DDA_LAUNCHED();
    int kbits = 1;
    while (kbits < 63 && ((uint64_t)ncell >> kbits) != 0) ++kbits;
    {
        size_t tb = 0;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, key, skey, id, sid, n, 0, kbits, st));
        char* ts = nullptr;
        DDA_CK(tmp.get(&ts, tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, key, skey, id, sid, n, 0, kbits, st));
    }
    k_cellstart<<<cgrid((int64_t)n + 1), CT, 0, st>>>(n, ncell, skey, cstart);
    DDA_LAUNCHED();

    // ---- 3. broad phase
    int32_t* cnt = nullptr;
    int64_t* off = nullptr;
    DDA_CK(tmp.get(&cnt, (size_t)n + 1));
    DDA_CK(tmp.get(&off, (size_t)n + 1));
    DDA_CK(cudaMemsetAsync(cnt + n, 0, sizeof(int32_t), st));
    k_broad<false><<<cgrid(n), CT, 0, st>>>(n, G, d0, box, cstart, sid, cnt, nullptr, nullptr);
    DDA_LAUNCHED();
    int64_t npairs = 0;
    DDA_CK(scan_counts(cnt, n, off, &npairs, tmp));
    if (npairs > (int64_t)INT_MAX) return DDA_ERR_OOM;
    int2* pairs = nullptr;
    DDA_CK(tmp.get(&pairs, npairs));
    if (npairs > 0) {
        k_broad<true><<<cgrid(n), CT, 0, st>>>(n, G, d0, box, cstart, sid, nullptr, off, pairs);
        DDA_LAUNCHED();
    }
    C->n_pairs = npairs;

    // ---- 4. narrow phase
    const double r2 = d0 * d0;                               // the oracle's d0 * d0
    int32_t* pcnt = nullptr;
    int64_t* poff = nullptr;
    DDA_CK(tmp.get(&pcnt, (size_t)npairs + 1));
    DDA_CK(tmp.get(&poff, (size_t)npairs + 1));
    DDA_CK(cudaMemsetAsync(pcnt + npairs, 0, sizeof(int32_t), st));
    int64_t m = 0;
    if (npairs > 0) {
        k_narrow<false><<<cgrid(npairs), CT, 0, st>>>(npairs, pairs, vptr, vxy, r2, pcnt, nullptr, nullptr, nullptr,
                                                      nullptr, nullptr, nullptr, nullptr, nullptr, nullptr);
        DDA_LAUNCHED();
        DDA_CK(scan_counts(pcnt, npairs, poff, &m, tmp));
    }
    if (m > (int64_t)INT_MAX) return DDA_ERR_OOM;
    C->count = m;
    uint64_t *rkey = nullptr, *rskey = nullptr;
    int32_t *ri = nullptr, *rv = nullptr, *rj = nullptr, *re = nullptr, *rt = nullptr, *ord_ = nullptr, *sord = nullptr;
    double *rtt = nullptr, *rd2 = nullptr;
    DDA_CK(tmp.get(&rkey, m)); DDA_CK(tmp.get(&rskey, m));
    DDA_CK(tmp.get(&ri, m)); DDA_CK(tmp.get(&rv, m)); DDA_CK(tmp.get(&rj, m)); DDA_CK(tmp.get(&re, m));
    DDA_CK(tmp.get(&rt, m)); DDA_CK(tmp.get(&rtt, m)); DDA_CK(tmp.get(&rd2, m));
    DDA_CK(tmp.get(&ord_, m)); DDA_CK(tmp.get(&sord, m));
    auto owned = [&](auto** p) { return dev_alloc(reinterpret_cast<void**>(p), m ? m * sizeof(**p) : 16, st); };
    DDA_CK(owned(&C->ci)); DDA_CK(owned(&C->cv)); DDA_CK(owned(&C->cj)); DDA_CK(owned(&C->ce));
    DDA_CK(owned(&C->ctype)); DDA_CK(owned(&C->ct)); DDA_CK(owned(&C->cd2));
    if (m > 0) {
        k_narrow<true><<<cgrid(npairs), CT, 0, st>>>(npairs, pairs, vptr, vxy, r2, nullptr, poff, rkey, ri, rv, rj,
                                                     re, rt, rtt, rd2);
        DDA_LAUNCHED();
        // ---- 5. canonical order: increasing (v, e)
        k_iota<<<cgrid(m), CT, 0, st>>>(m, ord_);
        DDA_LAUNCHED();
        size_t tb = 0;
        DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, rkey, rskey, ord_, sord, (int)m, 0, 64, st));
        char* ts = nullptr;
        DDA_CK(tmp.get(&ts, tb));
        DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, rkey, rskey, ord_, sord, (int)m, 0, 64, st));
        k_gather<int32_t><<<cgrid(m), CT, 0, st>>>(m, sord, ri, C->ci);
        k_gather<int32_t><<<cgrid(m), CT, 0, st>>>(m, sord, rv, C->cv);
        k_gather<int32_t><<<cgrid(m), CT, 0, st>>>(m, sord, rj, C->cj);
        k_gather<int32_t><<<cgrid(m), CT, 0, st>>>(m, sord, re, C->ce);
        k_gather<int32_t><<<cgrid(m), CT, 0, st>>>(m, sord, rt, C->ctype);
        k_gather<double><<<cgrid(m), CT, 0, st>>>(m, sord, rtt, C->ct);
        k_gather<double><<<cgrid(m), CT, 0, st>>>(m, sord, rd2, C->cd2);
        note_launch(6);
        DDA_LAUNCHED();
        // VE count
        int32_t* f = nullptr;
        int64_t* foff = nullptr;
        DDA_CK(tmp.get(&f, (size_t)m + 1));
        DDA_CK(tmp.get(&foff, (size_t)m + 1));
        DDA_CK(cudaMemsetAsync(f + m, 0, sizeof(int32_t), st));
        k_isve<<<cgrid(m), CT, 0, st>>>(m, C->ctype, f);
        DDA_LAUNCHED();
        DDA_CK(scan_counts(f, m, foff, &C->n_ve, tmp));
    }
    DDA_CK(cudaStreamSynchronize(st));
    guard.keep = true;
    *out = C;
    return DDA_OK;
}

extern "C" dda_status_t dda_contacts_info(dda_contacts_t C, int64_t* count, int64_t* n_ve, int64_t* n_pairs) {
    if (!C) return DDA_ERR_ARG;
    if (count) *count = C->count;
    if (n_ve) *n_ve = C->n_ve;
    if (n_pairs) *n_pairs = C->n_pairs;
    return DDA_OK;
}

extern "C" dda_status_t dda_contacts_export(dda_contacts_t C, int32_t* i, int32_t* v, int32_t* j, int32_t* e,
                                            int32_t* type, double* t, double* dist2) {
    if (!C) return DDA_ERR_ARG;
    const size_t m = (size_t)C->count;
    if (m == 0) return DDA_OK;
    DDA_CK(cudaDeviceSynchronize());
    if (i) DDA_CK(cudaMemcpy(i, C->ci, m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (v) DDA_CK(cudaMemcpy(v, C->cv, m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (j) DDA_CK(cudaMemcpy(j, C->cj, m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (e) DDA_CK(cudaMemcpy(e, C->ce, m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (type) DDA_CK(cudaMemcpy(type, C->ctype, m * sizeof(int32_t), cudaMemcpyDeviceToHost));
    if (t) DDA_CK(cudaMemcpy(t, C->ct, m * sizeof(double), cudaMemcpyDeviceToHost));
    if (dist2) DDA_CK(cudaMemcpy(dist2, C->cd2, m * sizeof(double), cudaMemcpyDeviceToHost));
    return DDA_OK;
}

extern "C" dda_status_t dda_contact_springs(dda_contacts_t C, const double* cxy, double p_n, double shear_ratio,
                                            int32_t* bi, int32_t* bj, double* pen, double* e, double* g,
                                            void* stream) {
    DDA_NVTX("dda_contact_springs");
    if (!C || !cxy || !(p_n >= 0.0) || !(shear_ratio >= 0.0) || !isfinite(p_n) || !isfinite(shear_ratio))
        return DDA_ERR_ARG;
    const int64_t m = C->count;
    if ((C->classified ? m : C->n_ve) == 0) return DDA_OK;
    if (!bi || !bj || !pen || !e || !g) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const double ps = shear_ratio * p_n;                     // the oracle's shear_ratio * p_n
    if (C->classified) {                                     // every record (VE, VV1, VV2), slot = record
        k_springs<<<cgrid(m), CT, 0, st>>>(m, nullptr, C->vptr, C->vxy, cxy, C->ci, C->cv, C->cj, C->ce, C->ctype,
                                           C->ct, p_n, ps, bi, bj, pen, e, g, 1);
        DDA_LAUNCHED();
        return DDA_OK;
    }
    CTmp tmp(st);
    int32_t *f = nullptr, *slot = nullptr;
    DDA_CK(tmp.get(&f, (size_t)m + 1));
    DDA_CK(tmp.get(&slot, (size_t)m + 1));
    DDA_CK(cudaMemsetAsync(f + m, 0, sizeof(int32_t), st));
    k_isve<<<cgrid(m), CT, 0, st>>>(m, C->ctype, f);
    DDA_LAUNCHED();
    {   // int32 exclusive scan: VE slot of each record
        size_t tb = 0;
        DDA_CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, f, slot, (int)m, st));
        char* ts = nullptr;
        DDA_CK(tmp.get(&ts, tb));
        DDA_CK(cub::DeviceScan::ExclusiveSum(ts, tb, f, slot, (int)m, st));
    }
    k_springs<<<cgrid(m), CT, 0, st>>>(m, slot, C->vptr, C->vxy, cxy, C->ci, C->cv, C->cj, C->ce, C->ctype, C->ct,
                                       p_n, ps, bi, bj, pen, e, g, 0);
    DDA_LAUNCHED();
    return DDA_OK;
}

// Second classification: the angle judgment abandons records, the rest is stored
// class by class in successive arrays (VE, VV1, VV2; increasing (v, e) within a class) — a stable
// 2-bit radix sort of the class keys ("scan and radix sort methods are used to classify or abandon
// data") and one gather per field.
extern "C" dda_status_t dda_classify_contacts(dda_contacts_t C, double sin_tol, void* stream) {
    DDA_NVTX("dda_classify_contacts");
    if (!C || !(sin_tol >= 0.0) || !(sin_tol < 1.0) || C->classified) return DDA_ERR_ARG;
    cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
    const int64_t m = C->count;
    C->classified = true;
    if (m == 0) return DDA_OK;
    CTmp tmp(st);
    uint32_t *key = nullptr, *skey = nullptr;
    int32_t *idx = nullptr, *sidx = nullptr;
    int64_t* start = nullptr;
    DDA_CK(tmp.get(&key, m)); DDA_CK(tmp.get(&skey, m));
    DDA_CK(tmp.get(&idx, m)); DDA_CK(tmp.get(&sidx, m));
    DDA_CK(tmp.get(&start, 5));
    const double s2 = sin_tol * sin_tol;                     // the oracle's sin_tol * sin_tol
    k_classify<<<cgrid(m), CT, 0, st>>>(m, C->vptr, C->vxy, C->ci, C->cv, C->cj, C->ce, C->ctype, s2, key, idx);
    DDA_LAUNCHED();
    size_t tb = 0;
    DDA_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, key, skey, idx, sidx, (int)m, 0, 2, st));
    char* ts = nullptr;
    DDA_CK(tmp.get(&ts, tb));
    DDA_CK(cub::DeviceRadixSort::SortPairs(ts, tb, key, skey, idx, sidx, (int)m, 0, 2, st));
    note_launch(2);
    k_class_bounds<<<cgrid(m), CT, 0, st>>>(m, skey, start);
    DDA_LAUNCHED();
    int64_t hs[5];
    DDA_CK(cudaMemcpyAsync(hs, start, sizeof hs, cudaMemcpyDeviceToHost, st));
    DDA_CK(cudaStreamSynchronize(st));
    const int64_t kept = m - hs[1];
    const int32_t* keep_idx = sidx + hs[1];
    int32_t *ni = nullptr, *nv = nullptr, *nj = nullptr, *ne = nullptr, *nt = nullptr;
    double *ntt = nullptr, *nd2 = nullptr;
    auto owned = [&](auto** p) { return dev_alloc(reinterpret_cast<void**>(p), kept ? kept * sizeof(**p) : 16, st); };
    DDA_CK(owned(&ni)); DDA_CK(owned(&nv)); DDA_CK(owned(&nj)); DDA_CK(owned(&ne)); DDA_CK(owned(&nt));
    DDA_CK(owned(&ntt)); DDA_CK(owned(&nd2));
    if (kept > 0) {
        k_gather<int32_t><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->ci, ni);
        k_gather<int32_t><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->cv, nv);
        k_gather<int32_t><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->cj, nj);
        k_gather<int32_t><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->ce, ne);
        k_gather<double><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->ct, ntt);
        k_gather<double><<<cgrid(kept), CT, 0, st>>>(kept, keep_idx, C->cd2, nd2);
        k_class_type<<<cgrid(kept), CT, 0, st>>>(kept, skey + hs[1], nt);
        note_launch(6);
        DDA_LAUNCHED();
    }
    void* old[] = {C->ci, C->cv, C->cj, C->ce, C->ctype, C->ct, C->cd2};
    for (void* p : old) dev_free_on(p, st);
    C->ci = ni; C->cv = nv; C->cj = nj; C->ce = ne; C->ctype = nt; C->ct = ntt; C->cd2 = nd2;
    C->count = kept;
    C->n_ve = hs[2] - hs[1];
    C->n_vv1 = hs[3] - hs[2];
    C->n_vv2 = hs[4] - hs[3];
    return DDA_OK;
}

extern "C" dda_status_t dda_contacts_classes(dda_contacts_t C, int64_t* n_ve, int64_t* n_vv1, int64_t* n_vv2,
                                             int32_t* classified) {
    if (!C) return DDA_ERR_ARG;
    if (n_ve) *n_ve = C->n_ve;
    if (n_vv1) *n_vv1 = C->n_vv1;
    if (n_vv2) *n_vv2 = C->n_vv2;
    if (classified) *classified = C->classified ? 1 : 0;
    return DDA_OK;
}
