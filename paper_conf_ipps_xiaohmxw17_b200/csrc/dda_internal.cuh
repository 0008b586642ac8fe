// Internal definitions of the B200 DDA solver library (not part of the ABI).
//
// Device layout:
//  * every 6x6 block (diagonal D_i and upper V_ij) is 36 doubles = 288 B, stored
//    "2x2-tiled": chunk q = 3R + C (R, C in 0..2) holds the 2x2 sub-block
//    rows 2R..2R+1, cols 2C..2C+1 as [a(2R,2C), a(2R,2C+1), a(2R+1,2C), a(2R+1,2C+1)];
//    one chunk is 32 B = one 256-bit load, so a block is 9 lanes x 32 B;
//  * blocks are 32 B aligned (cudaMalloc base + 288 B stride);
//  * block-Jacobi inverses are packed upper triangles, 21 doubles padded to 24;
//  * index arrays are int32 (row_ptr / low_ptr [n+1], col_idx / low_row / low_to_up [nnzb]).
#pragma once

#include <cuda_runtime.h>
#include <cstdint>
#include <cstddef>

#include "dda.h"

// NVTX ranges on the C ABI entry points (SURVEY §5 tracing): header-only NVTX v3, a no-op unless a
// tool (nsys, ncu --nvtx) injects itself, so the ranges cost nothing in normal runs
#include <nvtx3/nvToolsExt.h>

#ifndef DDA_THREADS
#define DDA_THREADS 256
#endif

namespace dda {

constexpr int kBlk = 36;       // doubles per 6x6 block
constexpr int kDinv = 24;      // doubles per packed inverse (21 used)

// offset of element (r, c) in the 2x2-tiled block layout
__host__ __device__ __forceinline__ int tile_off(int r, int c) {
    return 4 * (3 * (r >> 1) + (c >> 1)) + 2 * (r & 1) + (c & 1);
}
// offset of (r, c), r <= c, in the packed upper triangle (row-major)
__host__ __device__ __forceinline__ int pk_off(int r, int c) {
    return r * 6 - (r * (r - 1)) / 2 + (c - r);
}

// offset of (r, c), c <= r, in the packed lower triangle (row-major): Cholesky factors L, L^{-1}
__host__ __device__ __forceinline__ int lo_off(int r, int c) { return (r * (r + 1)) / 2 + c; }

// ------------------------------------------------------------------ host-side bookkeeping
void note_launch(int k = 1);               // counts kernel launches (dda_launch_count)
void trace(const char* what);              // DDA_TRACE=1: host wall-clock trace to stderr (diagnostics)
dda_status_t cuda_fail(cudaError_t e);      // records the message, maps to a status
int device_sms();
// the library's caching device allocator (alloc.cu): repeated builds in the open-close loop
// reuse freed blocks without CUDA calls; frees are stream-ordered (event per block)
cudaError_t dev_alloc(void** p, size_t bytes, cudaStream_t st);
void dev_free_on(void* p, cudaStream_t st);
void dev_free(void* p);   // on the legacy default stream

#define DDA_CK(call)                                   \
    do {                                               \
        cudaError_t _e = (call);                       \
        if (_e != cudaSuccess) return dda::cuda_fail(_e); \
    } while (0)

#define DDA_LAUNCHED()                                 \
    do {                                               \
        dda::note_launch();                            \
        cudaError_t _e = cudaGetLastError();           \
        if (_e != cudaSuccess) return dda::cuda_fail(_e); \
    } while (0)

struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};
#define DDA_NVTX(name) ::dda::NvtxRange dda_nvtx_range_(name)

// ------------------------------------------------------------------ device-side load helpers

// 256-bit read-only load of one 2x2 chunk (ld.global.nc.v4.f64 -> LDG.E.ENL2.256)
__device__ __forceinline__ double4 ld_chunk(const double* p) {
    double4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f64 {%0,%1,%2,%3}, [%4];"
                 : "=d"(v.x), "=d"(v.y), "=d"(v.z), "=d"(v.w) : "l"(p));
    return v;
}
// predicated variant: no memory access (and zeros) when !pred
__device__ __forceinline__ double4 ld_chunk_if(const double* p, bool pred) {
    double4 v = make_double4(0.0, 0.0, 0.0, 0.0);
    asm volatile("{\n .reg .pred q;\n setp.ne.b32 q, %5, 0;\n"
                 " @q ld.global.nc.L1::no_allocate.v4.f64 {%0,%1,%2,%3}, [%4];\n}"
                 : "+d"(v.x), "+d"(v.y), "+d"(v.z), "+d"(v.w) : "l"(p), "r"((int)pred));
    return v;
}
// Loads of vectors written earlier in the same persistent kernel.  They are only
// read after a grid barrier (cooperative_groups grid.sync: a gpu-scope fence,
// which also invalidates L1), so plain weak loads are coherent; they must not
// use the read-only .nc path.  DDA_VEC_CG selects L2-only (.cg) loads instead.
#ifdef DDA_VEC_CG
__device__ __forceinline__ double2 ld_cg2(const double* p) { return __ldcg(reinterpret_cast<const double2*>(p)); }
__device__ __forceinline__ double ld_cg(const double* p) { return __ldcg(p); }
#else
__device__ __forceinline__ double2 ld_cg2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ double ld_cg(const double* p) { return *p; }
#endif

// CTA barrier after lane-divergent code (if (lane == 0) ..., tree steps): __syncthreads() is the
// .aligned bar.sync, which every thread of a warp must reach converged; __syncwarp() reconverges
// first (compute-sanitizer synccheck flagged the bare barrier as divergent)
__device__ __forceinline__ void cta_barrier() {
    __syncwarp();
    __syncthreads();
}
// the same with the NON-aligned barrier.sync, defined for threads of a warp that arrive separately:
// used in the last-CTA reductions of the CUDA-graph loop kernels, where synccheck reported the
// aligned form as divergent under programmatic dependent launch (and the persistent loops keep the
// aligned one: the non-aligned form measured slower there)
__device__ __forceinline__ void cta_barrier_na() {
    __syncwarp();
    asm volatile("barrier.sync 0;" ::: "memory");
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

}  // namespace dda

// ------------------------------------------------------------------ the opaque handle
struct dda_matrix {
    int device = 0;
    int32_t n = 0;
    int64_t nnzb = 0;
    int64_t m = 0;
    // structure (device)
    int32_t* row_ptr = nullptr;
    int32_t* col_idx = nullptr;
    int32_t* low_ptr = nullptr;
    int32_t* low_row = nullptr;
    int32_t* low_to_up = nullptr;
    int32_t* urow = nullptr;        // [nnzb] block row of each upper block
    double* diag = nullptr;         // [n][36] tiled
    double* upper = nullptr;        // [nnzb][36] tiled
    // cached assembly permutation for value-only re-assembly (NEXT-1)
    int32_t* perm = nullptr;        // [m] spring ids sorted stably by (min,max)
    int32_t* seg = nullptr;         // [nnzb+1] segment starts into perm
    int32_t* dperm = nullptr;       // [2m] endpoint records 2s+side sorted stably by block
    int32_t* dstart = nullptr;      // [n+1]
    uint8_t* orient = nullptr;      // [m] 1 if bi[s] < bj[s]
    // preconditioners
    double* dinv = nullptr;         // [n][24] packed D_i^{-1}
    bool dinv_valid = false;
    double* lfac = nullptr;         // [n][24] packed lower Cholesky factor L_i of D_i (D_i = L_i L_i^T)
    double* sfac = nullptr;         // [n][24] packed lower S_i = L_i^{-1}
    double* bj_w = nullptr;         // [n] w_i <= lambda_min(D_i): 1 / min(||D_i^{-1}||_F, ||D_i^{-1}||_inf)
    double* sc_upper = nullptr;     // [nnzb][36] tiled: S_i V_ij S_j^T (scaled BJ engine)
    bool scaled_valid = false;
    double* ilu_up = nullptr;       // [nnzb][36] tiled: U_ij of the block IC(0) = ILU(0) factor
    double* ilu_inv = nullptr;      // [n][36] tiled: U_ii^{-1}
    int* ilu_flags = nullptr;       // [3n + 8]: factor / forward / backward ready flags, counters
    int* ilu_order = nullptr;       // [2n]: forward-level schedule, backward-level schedule
    int ilu_levels_f = 0, ilu_levels_b = 0;
    bool ilu_valid = false;
    // PCG workspace
    double* ws = nullptr;
    size_t ws_bytes = 0;
    void* scratch = nullptr;        // small device scratch (result struct, flags)
    void* graph_engine = nullptr;   // cached CUDA-graph PCG engine (pcg_graph.cu)
    void* tma_tiles = nullptr;      // spmv_tma.cu tile descriptors (int4 per 40-row tile), built on first use
    int32_t* full_ptr = nullptr;    // full-storage BSR6 copy for the configs[3] comparison (dda_spmv_full)
    int32_t* full_col = nullptr;
    double* full_val = nullptr;
    int64_t graph_iters = 0;        // loop-body launches issued inside graphs (launch accounting)
    int last_checks = 0;            // scaled engine: exact stopping tests in the last solve
    double* hist = nullptr;         // residual history (dda_pcg_set_history): [hist_cap][2] device doubles
    int hist_cap = 0;
    // NEXT-2 internal block order (dda_build_matrix_reordered): the arrays above are in the internal
    // (RCM) numbering; rperm[new] = user id, rinv[user] = new; vectors are permuted at the ABI
    int32_t* rperm = nullptr;
    int32_t* rinv = nullptr;
    double* rtmp = nullptr;         // [3][6n] permuted vector scratch
    // push-form phase A of the persistent BJ loop (pcg_graph.cu, phase_a_lr): structure-only map
    int32_t* lr_off = nullptr;      // [nnzb] entry of upper block u in lr_buf, 16 B units
    void* lr_buf = nullptr;         // 48 nnzb + 128 ceil(n/10) + 128 bytes of entries, then counters
    size_t lr_bytes = 0;            // bytes of entries (the counters follow)
};

// contact records of dda_detect_contacts (contact.cu) and the open-close state (openclose.cu)
struct dda_contacts {
    int device = 0;
    int32_t n = 0;
    int64_t count = 0, n_ve = 0, n_pairs = 0;
    bool classified = false;         // dda_classify_contacts ran: ctype = class (0 VE, 1 VV1, 2 VV2)
    int64_t n_vv1 = 0, n_vv2 = 0;
    const int32_t* vptr = nullptr;   // caller's geometry (must outlive dda_contact_springs)
    const double* vxy = nullptr;
    int32_t *ci = nullptr, *cv = nullptr, *cj = nullptr, *ce = nullptr, *ctype = nullptr;
    double *ct = nullptr, *cd2 = nullptr;
    // NEXT-4 (dda_contact_init): signed gaps and the contact endpoints sorted by block
    double* gap = nullptr;           // [count] n.(P - Q1)
    int32_t* eperm = nullptr;        // [2 count] endpoint records 2k + side, stably sorted by block
    int32_t* estart = nullptr;       // [n + 1] segment starts into eperm
};

namespace dda {
dda_status_t ensure_workspace(dda_matrix* K, size_t bytes, cudaStream_t st);
dda_status_t bj_setup(dda_matrix* K, cudaStream_t s, int32_t* bad_block);
dda_status_t spmv(dda_matrix* K, const double* x, double* y, cudaStream_t s);
dda_status_t spmv_tma(dda_matrix* K, const double* x, double* y, cudaStream_t s);
void pcg_graph_free(void* g);
dda_status_t scaled_setup(dda_matrix* K, cudaStream_t st);
void matrix_free_impl(dda_matrix_t K, cudaStream_t* sync);
dda_status_t build_matrix_impl(int32_t n, const double* kdiag, int64_t m, const int32_t* bi, const int32_t* bj,
                               const double* pen, const double* e, const double* g, cudaStream_t stream,
                               cudaEvent_t values_ready, dda_matrix_t* out);   // S_i V_ij S_j^T (needs lfac / sfac of every row)
dda_status_t ilu_setup(dda_matrix* K, cudaStream_t st, int32_t* bad_block);
dda_status_t bj_setup(dda_matrix* K, cudaStream_t st, int32_t* bad_block, double* full);
dda_status_t run_values(dda_matrix* K, const double* kdiag, const double* pen, const double* e, const double* g,
                        cudaStream_t st);
dda_status_t spmv_full(dda_matrix* K, const double* x, double* y, cudaStream_t st);
dda_status_t precond_apply(dda_matrix* K, dda_precond_t pc, double omega, const double* r, double* z, cudaStream_t st);
dda_status_t pcg_entry(dda_matrix* K, const double* F, const double* d0, double* d, double tol, int32_t maxit,
                       dda_precond_t pc, double omega, int32_t* iters, double* rel_res, cudaStream_t st);
dda_status_t export_internal(dda_matrix* K, int32_t* row_ptr, int32_t* col_idx, int32_t* low_ptr, int32_t* low_row,
                             int32_t* low_to_up, double* diag, double* upper);
// reordered matrices (reorder.cu): the same operations in the caller's numbering
dda_status_t ro_spmv(dda_matrix* K, const double* x, double* y, cudaStream_t st, bool full);
dda_status_t ro_pcg(dda_matrix* K, const double* F, const double* d0, double* d, double tol, int32_t maxit,
                    dda_precond_t pc, double omega, int32_t* iters, double* rel_res, cudaStream_t st);
dda_status_t ro_precond(dda_matrix* K, dda_precond_t pc, double omega, const double* r, double* z, cudaStream_t st);
dda_status_t ro_bj_setup(dda_matrix* K, double* dinv_full, int32_t* bad_block, cudaStream_t st);
dda_status_t ro_update_values(dda_matrix* K, const double* kdiag, const double* pen, const double* e, const double* g,
                              cudaStream_t st);
dda_status_t ro_export(dda_matrix* K, int32_t* row_ptr, int32_t* col_idx, int32_t* low_ptr, int32_t* low_row,
                       int32_t* low_to_up, double* diag, double* upper);
dda_status_t ilu_apply(dda_matrix* K, const double* r, double* z, double* y, double* yh, cudaStream_t st);
int ilu_grid();
int comm_nparts(const dda_comm* c);                 // partitions of the communicator (NCCL: ranks)
int comm_part_index(const dda_comm* c, int part);   // global partition index of local slot `part`, -1 if invalid
dda_status_t pcg_graph_solve(dda_matrix* K, const double* F, const double* d0, double* d, double tol,
                             int32_t maxit, dda_precond_t pc, double omega, int32_t* iters, double* rel_res,
                             cudaStream_t st, bool scaled);
}  // namespace dda
