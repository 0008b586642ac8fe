// A4 ablation — the symmetric BSR6 SpMV with its block stream staged through shared memory by the
// TMA unit (cp.async.bulk + mbarrier): the north_star's "staged through shared memory or TMA" and the
// paper's own staging (§IV.B), measured on B200 against the default LSU kernel.
// Internal: DDA_SPMV_TMA=1 routes dda_spmv here (tests check it is bit-identical).
//
// Same product, thread map and per-lane summation order as the column-pair kernel (spmv_col.cuh, v5),
// so y is bit-identical.  A CTA (4 warps) takes a tile of 40 consecutive block rows. Before its warps
// start, one elected thread arms an mbarrier with the byte count and issues 1-D bulk copies:
//   D   the tile's diagonal blocks                       (contiguous: rows r0..r1-1)
//   A   the tile's upper blocks = its forward blocks      (contiguous: row_ptr[r0] .. row_ptr[r1])
//   B   optionally (TT_CAPB_ > 0) the upper blocks its rows use TRANSPOSED that lie below A (one course
//       down on the slope numbering: a contiguous range found once per matrix by k_tma_tiles)
// The warps then read those blocks from shared memory; x gathers, the index decode and blocks
// outside the staged ranges come from global memory as before.
//
// Measured at 1M blocks (tools/spmv_ab.py, profiles/r02_spmv_tma.json), against 0.237 ms for the
// LSU kernel:
//   * D + A + B staged, 2 CTAs/SM: 0.509 ms;
//   * D + A staged, 4 CTAs/SM: 0.320 ms (this configuration);
//   * A only staged: 0.436 ms.
// The bulk copies do not shorten what bounds the kernel: the per-row chains of index decode -> x gather
// -> FMA, which need warps in flight.  The staged tiles cost those warps, because shared memory caps a
// tile pipeline at 16 warps/SM against the LSU kernel's 24 with two blocks of loads in flight per lane.
// Kept as the measured ablation; the default dda_spmv stays on the LSU path.
#include <cstdlib>

#include "spmv_col.cuh"

namespace dda {
namespace {

constexpr int TT_ROWS = 40;                  // block rows per tile (4 warps x 10)
constexpr int TT_WARPS = TT_ROWS / 10;
constexpr int TT_CAPA = 128;                 // staged forward blocks per tile (more: read from global)
#ifndef TT_CAPB_
#define TT_CAPB_ 0
#endif
constexpr int TT_CAPB = TT_CAPB_;            // staged transposed-source blocks per tile (0: none)
#ifndef TT_STAGE_D
#define TT_STAGE_D 1
#endif
constexpr int TT_DROWS = TT_STAGE_D ? TT_ROWS : 0;   // diagonal blocks staged (else read from global)
constexpr size_t TT_SMEM = sizeof(double) * kBlk * (TT_DROWS + TT_CAPA + TT_CAPB);

// tile t: {u0, u1, v0, v1} = staged forward range [u0, u1) (u1 - u0 <= CAPA) and transposed-source
// range [v0, v1) (v1 - v0 <= CAPB, else empty): the min / max of low_to_up over the tile's lower
// entries that lie below u0 (the ones inside [u0, u1) are already in A).  One warp per tile.
__global__ void k_tma_tiles(BsrView A, int ntiles, int4* __restrict__ tiles) {
    const int lane = threadIdx.x & 31;
    for (int t = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); t < ntiles; t += gridDim.x * (blockDim.x / 32)) {
        const int r0 = t * TT_ROWS, r1 = min(A.n, r0 + TT_ROWS);
        const int u0 = A.row_ptr[r0], u1full = A.row_ptr[r1];
        const int u1 = min(u1full, u0 + TT_CAPA);
        const int l0 = A.low_ptr[r0], l1 = A.low_ptr[r1];
        int vmin = INT_MAX, vmax = -1;
        for (int q = l0 + lane; q < l1; q += 32) {
            const int u = A.low_to_up[q];
            if (u < u0) { vmin = min(vmin, u); vmax = max(vmax, u); }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            vmin = min(vmin, __shfl_xor_sync(0xffffffffu, vmin, o));
            vmax = max(vmax, __shfl_xor_sync(0xffffffffu, vmax, o));
        }
        int v0 = 0, v1 = 0;
        if (TT_CAPB > 0 && vmax >= vmin && vmax + 1 - vmin <= TT_CAPB) { v0 = vmin; v1 = vmax + 1; }
        if (lane == 0) tiles[t] = make_int4(u0, u1, v0, v1);
    }
}

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ double4 lds_chunk(uint32_t a) {
    double4 v;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%4];\n\tld.shared.v2.f64 {%2, %3}, [%4+16];"
                 : "=d"(v.x), "=d"(v.y), "=d"(v.z), "=d"(v.w) : "r"(a));
    return v;
}

struct XLdgT {
    const double* __restrict__ x;
    __device__ __forceinline__ double2 operator()(int vec, int pair) const {
        return __ldg(reinterpret_cast<const double2*>(x + 6 * (size_t)vec + 2 * pair));
    }
};

struct TileView {
    uint32_t sD, sA, sB;   // shared addresses of the staged ranges
    int r0, u0, u1, v0, v1;
};

// chunk data of one block for lane C: from shared memory when staged, else from global
struct TData {
    double4 c0, c1, c2;
    double2 x;
    bool tr;
};
__device__ __forceinline__ TData tdata_load(const BsrView& A, const TileView& T, const CEnt& e, bool valid,
                                            const XLdgT& xl, int C) {
    TData d;
    d.tr = e.vec < 0;
    const int q0 = d.tr ? 3 * C : C, qs = d.tr ? 1 : 3;
    d.x = xl(d.tr ? ~e.vec : e.vec, C);
    uint32_t s = 0;
    bool staged = false;
    if (e.blk < 0) {                                   // diagonal block of a tile row
        staged = TT_STAGE_D != 0;
        s = T.sD + (uint32_t)((~e.blk - T.r0) * kBlk * 8);
    } else if (e.blk >= T.u0 && e.blk < T.u1) {
        staged = true;
        s = T.sA + (uint32_t)((e.blk - T.u0) * kBlk * 8);
    } else if (e.blk >= T.v0 && e.blk < T.v1) {
        staged = true;
        s = T.sB + (uint32_t)((e.blk - T.v0) * kBlk * 8);
    }
    if (valid && staged) {
        d.c0 = lds_chunk(s + 32 * q0);
        d.c1 = lds_chunk(s + 32 * (q0 + qs));
        d.c2 = lds_chunk(s + 32 * (q0 + 2 * qs));
    } else {
        const double* blk = e.blk >= 0 ? A.upper + (size_t)kBlk * e.blk : A.diag + (size_t)kBlk * ~e.blk;
        const bool g = valid && !staged;
        d.c0 = ld_chunk_if(blk + 4 * q0, g);
        d.c1 = ld_chunk_if(blk + 4 * (q0 + qs), g);
        d.c2 = ld_chunk_if(blk + 4 * (q0 + 2 * qs), g);
    }
    return d;
}

// spmv_row_c5 (SPMV_FULL) with the block source of tdata_load
__device__ __forceinline__ void row_tma(const BsrView& A, const TileView& T, int i, bool ok, const RowBounds& rb,
                                        const XLdgT& xl, int lane, double& y0, double& y1) {
    const unsigned full = 0xffffffffu;
    const int h = cgrp_of(lane);
    const int C = ccol_of(lane);
    const int nb = (ok && lane < 30) ? 1 + rb.nu + rb.nl : 0;
    const int nbmax = __reduce_max_sync(full, nb);
    double acc[6] = {0.0, 0.0, 0.0, 0.0, 0.0, 0.0};
    CEnt e1 = cent_decode<SPMV_FULL>(A, i, rb, 0, nb);
    TData d0 = tdata_load(A, T, e1, 0 < nb, xl, C);
    e1 = cent_decode<SPMV_FULL>(A, i, rb, 1, nb);
    for (int b = 0; b < nbmax; ++b) {
        const CEnt e2 = cent_decode<SPMV_FULL>(A, i, rb, b + 2, nb);
        const TData d1 = tdata_load(A, T, e1, b + 1 < nb, xl, C);
        const double4 cs[3] = {d0.c0, d0.c1, d0.c2};
        const double2 xv = d0.x;
#pragma unroll
        for (int k = 0; k < 3; ++k) {
            const double4 c = cs[k];
            const double m01 = d0.tr ? c.z : c.y;
            const double m10 = d0.tr ? c.y : c.z;
            acc[2 * k] = fma(c.x, xv.x, fma(m01, xv.y, acc[2 * k]));
            acc[2 * k + 1] = fma(m10, xv.x, fma(c.w, xv.y, acc[2 * k + 1]));
        }
        d0 = d1;
        e1 = e2;
    }
    const int c1 = C == 2 ? 0 : C + 1, c2 = C == 0 ? 2 : C - 1;
    const int s1 = lane < 30 ? 3 * h + c1 : lane, s2 = lane < 30 ? 3 * h + c2 : lane;
    const double2 v1 = pick_pair(acc, c2);
    const double r1x = __shfl_sync(full, v1.x, s1), r1y = __shfl_sync(full, v1.y, s1);
    const double2 v2 = pick_pair(acc, c1);
    const double r2x = __shfl_sync(full, v2.x, s2), r2y = __shfl_sync(full, v2.y, s2);
    const double2 own = pick_pair(acc, C);
    y0 = (own.x + r1x) + r2x;
    y1 = (own.y + r1y) + r2y;
}

__global__ void __launch_bounds__(32 * TT_WARPS, TT_CAPB > 0 ? 2 : (TT_STAGE_D ? 4 : 6)) k_spmv_tma(BsrView A, const int4* __restrict__ tiles, int ntiles,
                                                               const double* __restrict__ x, double* __restrict__ y) {
    extern __shared__ __align__(128) double smem[];
    __shared__ __align__(8) unsigned long long bar;
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const uint32_t sbar = smem_addr(&bar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(sbar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    TileView T;
    T.sD = smem_addr(smem);
    T.sA = T.sD + TT_DROWS * kBlk * 8;
    T.sB = T.sA + TT_CAPA * kBlk * 8;
    const XLdgT xl{x};
    uint32_t phase = 0;
    for (int t = blockIdx.x; t < ntiles; t += gridDim.x) {
        const int4 td = __ldg(tiles + t);
        T.r0 = t * TT_ROWS;
        const int r1 = min(A.n, T.r0 + TT_ROWS);
        T.u0 = td.x; T.u1 = td.y; T.v0 = td.z; T.v1 = td.w;
        if (threadIdx.x == 0) {
            // the previous tile's shared-memory reads (generic proxy) precede these async-proxy writes
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            const uint32_t bD = TT_STAGE_D ? (uint32_t)(r1 - T.r0) * kBlk * 8 : 0u, bA = (uint32_t)(T.u1 - T.u0) * kBlk * 8,
                           bB = (uint32_t)(T.v1 - T.v0) * kBlk * 8;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(sbar), "r"(bD + bA + bB)
                         : "memory");
            if (bD) bulk_g2s(T.sD, A.diag + (size_t)kBlk * T.r0, bD, sbar);
            if (bA) bulk_g2s(T.sA, A.upper + (size_t)kBlk * T.u0, bA, sbar);
            if (bB) bulk_g2s(T.sB, A.upper + (size_t)kBlk * T.v0, bB, sbar);
        }
        const int i = T.r0 + 10 * w + cgrp_of(lane);
        const bool ok = lane < 30 && i < r1;
        const RowBounds rb = row_bounds<SPMV_FULL>(A, i, ok);     // overlaps the copies
        {   // wait for the tile's bytes (phase parity)
            uint32_t done = 0;
            while (!done) {
                asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
                             " selp.u32 %0, 1, 0, p;\n}"
                             : "=r"(done) : "r"(sbar), "r"(phase) : "memory");
            }
        }
        phase ^= 1;
        double y0, y1;
        row_tma(A, T, ok ? i : A.n, ok, rb, xl, lane, y0, y1);
        if (ok) *reinterpret_cast<double2*>(y + 6 * (size_t)i + 2 * ccol_of(lane)) = make_double2(y0, y1);
        __syncthreads();   // every read of this tile's shared copy is done before the next copies
    }
}

}  // namespace

// (tuning aid / A/B: DDA_SPMV_TMA=1 routes dda_spmv here)
dda_status_t spmv_tma(dda_matrix* K, const double* x, double* y, cudaStream_t st) {
    const int ntiles = (K->n + TT_ROWS - 1) / TT_ROWS;
    if (!K->tma_tiles) {
        int4* tl = nullptr;
        DDA_CK(dev_alloc(reinterpret_cast<void**>(&tl), sizeof(int4) * (size_t)(ntiles > 0 ? ntiles : 1), st));
        k_tma_tiles<<<(ntiles + 7) / 8, 256, 0, st>>>(view_of(K), ntiles, tl);
        DDA_LAUNCHED();
        K->tma_tiles = tl;
    }
    static bool attr = false;
    if (!attr) {
        DDA_CK(cudaFuncSetAttribute(k_spmv_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TT_SMEM));
        attr = true;
    }
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_spmv_tma, 32 * TT_WARPS, TT_SMEM);
    int g = device_sms() * (per_sm > 0 ? per_sm : 1);
    if (g > ntiles) g = ntiles > 0 ? ntiles : 1;
    k_spmv_tma<<<g, 32 * TT_WARPS, TT_SMEM, st>>>(view_of(K), reinterpret_cast<const int4*>(K->tma_tiles), ntiles,
                                                  x, y);
    DDA_LAUNCHED();
    return DDA_OK;
}

}  // namespace dda
