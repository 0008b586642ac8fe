/*
 * dda.h — C ABI of the B200-native DDA equation-solving hot path.
 *
 * The path is the open-close inner-loop solve K·d = F of 2-D Discontinuous
 * Deformation Analysis (§IV): K is the global
 * stiffness matrix, "naturally blocky and symmetric", each entry a 6x6
 * sub-matrix, all diagonal sub-matrices nonzero, a_ij != 0 only if blocks i and
 * j are in contact, and "only the upper entry of A is computed and stored"
 * (P:102).  K is solved by preconditioned conjugate gradients with
 * block-Jacobi, SSOR approximate inverse or ILU(0).
 *
 * Conventions (every entry point):
 *  - Block ids are 0-based int32; the DOFs of block b are (u0, v0, r0, ex, ey,
 *    gxy) at global indices 6b..6b+5 (reading Z11).  Values are IEEE fp64.
 *  - "device" pointers are CUDA device (or managed) memory owned by the caller
 *    and valid for the duration of the call; "host" pointers are host memory
 *    (pinned memory gives the fastest copies).  No pointer is retained.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *    stream).  Work is stream-ordered; calls documented as "synchronising"
 *    wait for the stream before returning.
 *  - Every status is returned, never thrown; there is no global error state.
 *    dda_status_string() names a status.
 *  - A dda_matrix_t is an opaque handle owning device arrays; it is bound to the
 *    device that was current when it was built and must be released with
 *    dda_matrix_free().  Handles are not thread-safe: do not use one handle
 *    from two host threads at once.
 */
#ifndef DDA_H
#define DDA_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dda_matrix *dda_matrix_t;

typedef enum {
    DDA_OK = 0,
    DDA_ERR_ARG = 1,             /* invalid argument (sizes, null pointers, ids, tol, maxit, penalties) */
    DDA_ERR_CUDA = 2,            /* a CUDA runtime call failed (message via dda_last_cuda_error) */
    DDA_ERR_OOM = 3,             /* device allocation failed */
    DDA_ERR_NOT_SPD = 4,         /* a (pivot) diagonal block is not symmetric positive definite */
    DDA_ERR_BREAKDOWN = 5,       /* PCG breakdown: p^T K p <= 0, r^T z <= 0 or not finite (Z19) */
    DDA_ERR_NO_CONVERGENCE = 6,  /* maxit reached before ||r|| <= tol ||F|| */
    DDA_ERR_NCCL = 7             /* reserved for the distributed solver */
} dda_status_t;

typedef enum {
    DDA_PC_NONE = 0,     /* plain CG */
    DDA_PC_BJ = 1,       /* block Jacobi: z_i = D_i^{-1} r_i (Table I) */
    DDA_PC_SSOR_AI = 2,  /* SSOR approximate inverse (ref [36]; reading Z14) */
    DDA_PC_ILU0 = 3      /* block ILU(0) = IC(0) for symmetric K (reading Z15); sync-free sweeps */
} dda_precond_t;

/*
 * A1 — Assembly (§III.C; Fig. 4 steps: per-contact sub-matrix →
 * sort by block number → boundary flags → scan → segment sums).
 *
 * Builds K from per-block diagonal terms and m contact springs.  Spring s =
 * (bi[s], bj[s], pen[s], e[s][6], g[s][6]) couples vertex block i = bi[s] and
 * edge block j = bj[s] and contributes
 *      a_ii += p e e^T,   a_jj += p g g^T,   a_ij += p e g^T  (a_ji = a_ij^T).
 * The stored off-diagonal block is (min(i,j), max(i,j)); it receives p e g^T
 * if i < j and its transpose if i > j (reading Z7).  Every entry is the sum,
 * in increasing spring index, of the products (p*e[r])*g[c] rounded as
 * written (no FMA contraction), so values are bit-identical to the
 * definition (reading Z8); the diagonal starts from kdiag's upper triangle
 * (the lower triangle of kdiag is ignored, reading Z9).  A spring with p = 0
 * still creates its block (reading Z10).  m = 0 is valid (K block diagonal).
 *
 *  n_blocks     number of blocks n > 0 (6n unknowns)
 *  kdiag        device, [n][6][6] row-major: elastic + inertia + fixed-point
 *               terms of each block; upper triangle read
 *  n_springs    m >= 0
 *  bi, bj       device, [m] int32 block ids in [0, n), bi[s] != bj[s]
 *  pen          device, [m] penalties, finite and >= 0
 *  e, g         device, [m][6] spring vectors of block bi / bj (16-byte aligned)
 *  stream       cudaStream_t
 *  out          receives the new handle (NULL on failure)
 * Errors: DDA_ERR_ARG for n <= 0, m < 0, a NULL pointer with m > 0, an id out
 * of range, bi == bj, or a negative / non-finite penalty (the id and penalty
 * checks run on the device and are reported after the call synchronises the
 * stream once to size the output).  DDA_ERR_OOM / DDA_ERR_CUDA otherwise.
 * Synchronising.
 */
dda_status_t dda_build_matrix(int32_t n_blocks, const double *kdiag, int64_t n_springs,
                              const int32_t *bi, const int32_t *bj, const double *pen,
                              const double *e, const double *g, void *stream, dda_matrix_t *out);

/*
 * A1 (inner-loop variant, NEXT-1) — value-only re-assembly.  Same springs
 * (same count, same (bi, bj) sequence) with new penalties / vectors / diagonal
 * terms: reuses the cached sort permutation and structure (contacts are fixed
 * within a time step; only states and penalties change in the open-close loop,
 * P:27).  The caller guarantees bi/bj are unchanged (not checked
 * beyond the count).  Invalidates preconditioner state.  Stream-ordered.
 */
dda_status_t dda_update_values(dda_matrix_t K, const double *kdiag, int64_t n_springs,
                               const double *pen, const double *e, const double *g, void *stream);

/* Sizes of a built matrix: n and the number of stored upper off-diagonal blocks. */
dda_status_t dda_matrix_info(dda_matrix_t K, int32_t *n_blocks, int64_t *nnzb_upper);

/*
 * A2 — Canonical export.  Host buffers, each may be NULL:
 *  row_ptr   [n+1]   upper CSR offsets; the paper's row-up-i[i] = row_ptr[i+1]
 *  col_idx   [nnzb]  strictly increasing within a row, every entry > its row
 *  low_ptr   [n+1]   CSR offsets of the virtual lower part; row-low-i[i] = low_ptr[i+1]
 *  low_row   [nnzb]  for lower position t in row i: the k < i with (k,i) stored, ascending
 *  low_to_up [nnzb]  row-low-p: position of block (k,i) in the upper storage
 *  diag      [n][36] row-major D_i
 *  upper     [nnzb][36] row-major V_ij, in row_ptr order
 * Internal device layouts are private.  Synchronising.
 */
dda_status_t dda_matrix_export(dda_matrix_t K, int32_t *row_ptr, int32_t *col_idx, int32_t *low_ptr,
                               int32_t *low_row, int32_t *low_to_up, double *diag, double *upper);

/*
 * A4 — Symmetric block SpMV  y = K x  (§IV.B), from the upper
 * storage only: y_i = D_i x_i + sum_{j>i} V_ij x_j + sum_{k<i} V_ki^T x_k.
 * Atomic-free and deterministic (bitwise run-to-run).
 *  x, y   device, [6n]; must not alias.   Stream-ordered.
 */
dda_status_t dda_spmv(dda_matrix_t K, const double *x, double *y, void *stream);

/*
 * configs[3] comparison — the same product from FULL-storage BSR6: on first use
 * the library expands K (every off-diagonal block stored in both rows, the
 * representation "most of the proposed SpMV methods need to recover")
 * and then runs the same warp kernel with every block forward.  Reads
 * (1 + 2u) blocks per row instead of (1 + u).  x, y device [6n], no alias.
 */
dda_status_t dda_spmv_full(dda_matrix_t K, const double *x, double *y, void *stream);

/*
 * A3 — Block-Jacobi setup (Table I "construction" P:174): D_i^{-1} for
 * every diagonal block by 6x6 Cholesky.  Called implicitly by dda_pcg_solve;
 * exposed for testing.  If dinv (device, [n][36] row-major) is non-NULL the
 * inverses are also written there.  DDA_ERR_NOT_SPD if some D_i is not SPD;
 * *bad_block (host, may be NULL) receives its index (-1 otherwise).
 * Synchronising.
 */
dda_status_t dda_bj_setup(dda_matrix_t K, double *dinv, int32_t *bad_block, void *stream);

/*
 * A7/A8 — Preconditioner application z = M^{-1} r (device [6n] each) for
 * testing the preconditioners in isolation.  Sets the preconditioner up first
 * if needed (block-Jacobi inverses; for DDA_PC_ILU0 the block IC(0) factor
 * U_ij = A_ij - sum_k U_ki^T U_kk^{-1} U_kj on the stored pattern, which may
 * return DDA_ERR_NOT_SPD for a non-SPD pivot).  omega is used by
 * DDA_PC_SSOR_AI only.  Synchronising.
 */
dda_status_t dda_precond_apply(dda_matrix_t K, dda_precond_t pc, double omega, const double *r, double *z,
                               void *stream);

/*
 * A5/A6 — PCG solve of K d = F, warm-started from d0
 * ("the equation solution of the previous step is the initial value").
 *  F       device [6n]
 *  d0      device [6n] initial guess, or NULL for zero; may alias d
 *  d       device [6n] solution
 *  tol     > 0: stop when ||r_k||_2 <= tol ||F||_2 on the recursive residual (reading Z1)
 *  maxit   >= 0 (the paper's DDA policy is 200)
 *  pc      preconditioner;  omega: SSOR-AI relaxation (1.0 default, ignored otherwise)
 *  iters   host out: iterations performed
 *  rel_res host out: TRUE relative residual ||F - K d||_2 / ||F||_2 (one extra SpMV)
 * The whole iteration runs on the device; the host reads the result once at the end.
 * Block-Jacobi and SSOR-AI run PCG on the block-scaled S K S^T (S = blockdiag(L_i^{-1}),
 * same iterates, reading Z25) in ONE persistent cooperative kernel, whose CTAs must all be
 * co-resident.  When the occupancy query finds no room for it, the solve falls back before
 * writing any state (block-Jacobi: the CUDA-graph while loop with the same phases as kernels;
 * SSOR-AI: the unscaled graph engine); a cooperative launch that still fails returns
 * DDA_ERR_CUDA (DDA_SCALED_LOOP=graph selects the graph loop for block-Jacobi explicitly).
 * ILU(0) and the unpreconditioned solve run a CUDA-graph device-side while loop.  Returns DDA_OK,
 * DDA_ERR_NO_CONVERGENCE (d, iters, rel_res still filled), DDA_ERR_BREAKDOWN
 * (d = last iterate), DDA_ERR_NOT_SPD (preconditioner setup).  F = 0 gives
 * d = 0, iters = 0, rel_res = 0, DDA_OK (reading Z2).  Synchronising.
 */
dda_status_t dda_pcg_solve(dda_matrix_t K, const double *F, const double *d0, double *d, double tol,
                           int32_t maxit, dda_precond_t pc, double omega, int32_t *iters, double *rel_res,
                           void *stream);

/*
 * Optional residual history: registers a DEVICE buffer of 2*cap doubles that the
 * following dda_pcg_solve calls on K fill, one pair per iteration k (0-based, k < min(iters, cap)):
 *   hist[2k]     rho_{k+1} = r_{k+1}^T M^{-1} r_{k+1}, the PCG inner product of the new residual
 *                (block-Jacobi: |L^{-1} r|^2, L the block Cholesky factors);
 *   hist[2k + 1] |r_{k+1}|^2 when the exact stopping test (reading Z1) was evaluated at that
 *                iteration, else NaN.
 * Written by the block-Jacobi scaled engine (the default BJ path: persistent two-phase or
 * single-reduction loop, or its CUDA-graph loop); other preconditioners leave the buffer untouched.
 * buf = NULL with cap = 0 unregisters.  The buffer must stay valid while registered.  Registering
 * or changing it rebuilds the cached solver engine on the next solve.  DDA_ERR_ARG: K NULL, cap < 0,
 * or buf / cap inconsistent.
 */
dda_status_t dda_pcg_set_history(dda_matrix_t K, double *buf, int32_t cap);

/*
 * End-to-end entry with HOST buffers (the benchmark's e2e leg): copies the
 * inputs host→device, assembles, sets up the preconditioner, solves, copies d
 * device→host and frees everything.  Arguments as dda_build_matrix and
 * dda_pcg_solve, all host pointers; d0 may be NULL.  Synchronising.
 */
dda_status_t dda_solve_host(int32_t n_blocks, const double *kdiag, int64_t n_springs, const int32_t *bi,
                            const int32_t *bj, const double *pen, const double *e, const double *g,
                            const double *F, const double *d0, double *d, double tol, int32_t maxit,
                            dda_precond_t pc, double omega, int32_t *iters, double *rel_res, void *stream);

/*
 * Streamed end-to-end entry: nsys independent host systems solved in order (a
 * time-stepping driver's loop 1 of PAPER.md Fig. 1, one system per step) with
 * the host->device copy of system k+1 and the device->host copy of system k's d
 * overlapping the assembly and solve of system k (a second, copy stream; two
 * device input slots sized for the largest system).  Per system the work is
 * exactly dda_solve_host's.  Host buffers should be pinned (pageable buffers
 * work but their copies do not overlap) and must not change until the call
 * returns.  Fields marked out are written per system; the call returns DDA_OK
 * unless an argument or CUDA error stops the batch (then the systems before the
 * failing one are complete and its status field holds the error).  d0 may be
 * NULL.  Synchronising.
 */
typedef struct {
    int32_t n_blocks;
    int64_t n_springs;
    const double *kdiag;          /* [n_blocks][36] */
    const int32_t *bi, *bj;       /* [n_springs] */
    const double *pen;            /* [n_springs] */
    const double *e, *g;          /* [n_springs][6] */
    const double *F;              /* [6 n_blocks] */
    const double *d0;             /* [6 n_blocks] or NULL */
    double *d;                    /* out: [6 n_blocks] */
    int32_t iters;                /* out */
    double rel_res;               /* out: TRUE relative residual */
    dda_status_t status;          /* out: as dda_pcg_solve */
} dda_host_system;

dda_status_t dda_solve_host_batch(int32_t nsys, dda_host_system *sys, double tol, int32_t maxit, dda_precond_t pc,
                                  double omega, void *stream);

/*
 * (e) — Multi-GPU block-row partitioned PCG (beyond the paper: multi-GPU is its
 * future work).  A partition is an ordinary dda_matrix_t built on the
 * partition's LOCAL numbering: own rows 0..n_own-1 (a contiguous range of
 * global rows, same order) followed by halo rows grouped by owning peer
 * (ascending peer, global order within a peer); it is assembled from every
 * spring that touches an own row, so its own rows are exact global rows.
 * dda_build_matrix_dist (below) builds a partition and attaches it in one call; dda_dist_attach
 * takes a partition built elsewhere.
 *
 * Transports: NCCL (dda_comm_init: one partition per process / GPU; rank 0
 * creates the 128-byte id with dda_comm_unique_id and the caller broadcasts it)
 * or LOOPBACK (dda_comm_init_loopback: all partitions in this process on the
 * current GPU — the same partitioned algorithm, exchanges by device copy).
 *
 * dda_dist_attach: partition `part` (0 for NCCL; 0..nparts-1 for loopback) is
 * matrix K with n_own own rows; send_counts[q] own rows go to peer q, listed
 * (local ids, host) in send_idx concatenated by peer, in the peer's halo order;
 * recv_counts[q] halo rows come from q (sum = K's rows - n_own).  Host arrays
 * [nranks].  K must outlive the communicator's use of it.
 *
 * dda_pcg_solve_dist: F[p], d0[p] (entry or whole array may be NULL), d[p]:
 * device [6 n_own] per local partition (one entry for NCCL).  Same stop rule,
 * statuses and reported TRUE residual as dda_pcg_solve; DDA_PC_BJ or
 * DDA_PC_NONE (SSOR-AI and ILU(0) are single-GPU only).  Block-Jacobi runs the
 * scaled engine per partition (PCG on S K S^T, reading Z25; S of the halo rows is
 * exchanged once per solve).  The loop depends on the transport: NCCL runs v4
 * (per iteration one halo of p overlapped with the interior rows and one 6-double
 * allreduce); LOOPBACK runs v6 (every partition in ONE persistent cooperative
 * kernel, halo rows read from their owners, fixed-order sums); IPC runs v7 (one
 * persistent kernel per rank, see dda_comm_init_ipc).  DDA_DIST_VERSION = 7 / 5 /
 * 4 / 3 selects the loopback per-rank kernels, the peer-load per-iteration
 * launches, the halo-copy launches or the round-1 loop; DDA_DIST_SCALED=0 the
 * unscaled loop (also the unpreconditioned solve).  Synchronising.
 * dda_spmv_dist: y = K x over own rows (x, y device [6 n_own] per partition).
 */
typedef struct dda_comm *dda_comm_t;
dda_status_t dda_comm_unique_id(void *id128);
dda_status_t dda_comm_init(int32_t nranks, int32_t rank, const void *id128, dda_comm_t *out);
dda_status_t dda_comm_init_loopback(int32_t nparts, dda_comm_t *out);

/*
 * IPC transport (one partition per process; the processes may share a GPU or sit on NVLink-connected
 * GPUs): no NCCL.  Each rank's partition buffers that peers read in place (halo send rows, r~ and the
 * PCG direction vectors, the send lists) are exported as CUDA IPC handles; rank 0 also exports the
 * arrival counter and slot sets the collectives use.  Sequence: dda_comm_init_ipc, build or attach the
 * rank's partition (dda_build_matrix_dist / dda_dist_attach), dda_comm_ipc_export (blob NULL: *bytes =
 * the blob size), exchange the blobs between the processes by any means (the caller's), then
 * dda_comm_ipc_import with all blobs in rank order, each `bytes` long.  dda_pcg_solve_dist (BJ) then
 * runs v7: one persistent cooperative kernel per rank, halo rows read from the owners' mapped arrays,
 * every reduction a fixed-order one-shot sum through rank 0's slot sets, every wait bounded
 * (DDA_ERR_CUDA if a peer never arrives).  nranks <= 8.  DDA_ERR_ARG: a blob from another rank count,
 * a send list that does not match this rank's receive list, re-import, or no partition attached.
 * Beyond the paper (multi-GPU is its future work).
 */
dda_status_t dda_comm_init_ipc(int32_t nranks, int32_t rank, dda_comm_t *out);
dda_status_t dda_comm_ipc_export(dda_comm_t c, void *blob, int64_t *bytes);
dda_status_t dda_comm_ipc_import(dda_comm_t c, const void *blobs, int64_t bytes);
dda_status_t dda_dist_attach(dda_comm_t c, int32_t part, dda_matrix_t K, int32_t n_own, const int32_t *send_counts,
                             const int32_t *send_idx, const int32_t *recv_counts, void *stream);
dda_status_t dda_spmv_dist(dda_comm_t c, const double *const *x_own, double *const *y_own, void *stream);

/*
 * dda_build_matrix_dist — the partition-local assembly on the device (§8(b); A1 per partition,
 * P:100-110, with P:104's "a contact contributes to rows i and j" deciding which springs a
 * partition needs).  Partition `part` (0 for NCCL, 0..nparts-1 for loopback) owns the global
 * block rows [row_bounds[me], row_bounds[me+1]) with me = its partition index (the NCCL rank, or
 * `part`).  The call:
 *   1. selects, in spring order, the springs with an endpoint in the own range;
 *   2. forms the halo = their remote endpoints, sorted and unique (ascending global id, hence
 *      grouped by owning partition);
 *   3. numbers own row g as g - row_bounds[me] and halo row h as n_own + (rank of h in the halo);
 *   4. assembles the local matrix with dda_build_matrix (halo rows get zero diagonal terms; the
 *      own rows are then bit-identical to the global rows);
 *   5. derives the exchange plan (the own rows each peer needs, ascending; the halo rows each
 *      peer sends) and attaches matrix and plan to the communicator (dda_dist_attach).
 *  n_global     global block count; row_bounds: host [nparts+1], 0 = b_0 < b_1 < ... = n_global,
 *               identical on every partition
 *  kdiag_own    device [n_own][6][6] diagonal terms of the own rows (global rows b_me..b_me+1-1)
 *  n_springs, bi, bj, pen, e, g   device, GLOBAL block ids: the whole spring list, or any list
 *               that contains every spring touching an own row (others are skipped)
 *  out          receives the local matrix (caller-owned: dda_matrix_free after the last
 *               distributed call that uses it; re-building a partition re-attaches)
 * F / d of the partition are the global vectors' own-row slices [6 b_me, 6 b_me+1).  Errors:
 * DDA_ERR_ARG for a bad partition index or bounds, ids out of [0, n_global) or bi == bj (checked
 * on the device), or anything dda_build_matrix rejects.  Synchronising (sizes are read back).
 * dda_dist_info reports a partition's n_own, n_halo and exchange plan (host arrays [nparts],
 * send_idx [sum send_counts]; any may be NULL).
 */
dda_status_t dda_build_matrix_dist(dda_comm_t c, int32_t part, int32_t n_global, const int32_t *row_bounds,
                                   const double *kdiag_own, int64_t n_springs, const int32_t *bi, const int32_t *bj,
                                   const double *pen, const double *e, const double *g, void *stream,
                                   dda_matrix_t *out);
dda_status_t dda_dist_info(dda_comm_t c, int32_t part, int32_t *n_own, int32_t *n_halo, int32_t *send_counts,
                           int32_t *recv_counts, int32_t *send_idx);
dda_status_t dda_pcg_solve_dist(dda_comm_t c, const double *const *F, const double *const *d0, double *const *d,
                                double tol, int32_t maxit, dda_precond_t pc, int32_t *iters, double *rel_res,
                                void *stream);
void dda_comm_free(dda_comm_t c);

/*
 * NEXT-2 — ordering-robust SpMV: reverse Cuthill-McKee order of the block
 * contact graph (blocks joined by a spring), host arrays, O(n + m log d).  The
 * symmetric SpMV re-reads each transposed block from L2 soon after its first
 * use; a random block numbering breaks that reuse (P:180 applies both uses of
 * every stored block).  perm[new] = old block id; renumber kdiag / springs / F
 * with it before dda_build_matrix and map d back (partition.py's peers use the
 * same convention).  DDA_ERR_ARG for bad ids.
 */
dda_status_t dda_rcm_order(int32_t n_blocks, int64_t n_springs, const int32_t *bi, const int32_t *bj,
                           int32_t *perm);

/*
 * NEXT-2 — the same order applied INSIDE the library: arguments and errors as dda_build_matrix
 * (bi, bj device, caller's numbering).  The matrix is assembled in the RCM numbering of the contact
 * graph (computed on the host from a copy of bi, bj: once per contact structure); every entry point
 * keeps the caller's numbering by permuting at the boundary: dda_spmv / dda_spmv_full / dda_pcg_solve
 * / dda_precond_apply (vectors gathered in and scattered out: 48 B per row each way, once per call —
 * a PCG solve permutes F, d0 and d, not its iterations), dda_update_values (kdiag gathered),
 * dda_bj_setup (D^{-1} and the failing block id in the caller's numbering), dda_matrix_export (the
 * canonical arrays of the caller's numbering, rebuilt on the host; values bit-identical to
 * dda_build_matrix's).  Block-Jacobi (and plain CG) do not depend on the order; SSOR-AI's triangular
 * split and ILU(0)'s incomplete factor are those of the internal order.  Not accepted by
 * dda_dist_attach.  Synchronising.
 */
dda_status_t dda_build_matrix_reordered(int32_t n_blocks, const double *kdiag, int64_t n_springs, const int32_t *bi,
                                        const int32_t *bj, const double *pen, const double *e, const double *g,
                                        void *stream, dda_matrix_t *out);

/*
 * NEXT-2 ablation — the paper's HSBCSR two-stage SpMV (§IV.B; Figs. 6-9), for the
 * comparison of P:222 (2.8x over cuSPARSE on the K40) next to dda_spmv on B200.
 * dda_hsbcsr_build copies K (not a reordered one) into the half-slice layout: d-data [6][dstride]
 * and nd-data-up [6][ustride], where slice r holds row r (6 doubles) of every diagonal / upper block
 * in block order and each slice is padded to a multiple of 32 doubles (reading Z13), so entry
 * (block b, row r, column c) is at stride * r + 6 b + c.  dda_hsbcsr_spmv computes y = K x in two
 * stages: (1) per upper block b = (i, j), up-res[b] = V_b x_j and low-res[b] = V_b^T x_i; (2) per row,
 * D_i x_i + the up-res of its row + the low-res of its lower row through row-low-p (= low_to_up).
 * x, y device [6n], no alias; stream-ordered; same tolerance as dda_spmv.  dda_hsbcsr_export copies
 * the two slice arrays to host buffers (either may be NULL) and the two strides (host int64 [2]).
 * The handle reads K's index arrays: K must outlive it.
 */
typedef struct dda_hsbcsr *dda_hsbcsr_t;
dda_status_t dda_hsbcsr_build(dda_matrix_t K, void *stream, dda_hsbcsr_t *out);
dda_status_t dda_hsbcsr_spmv(dda_hsbcsr_t H, const double *x, double *y, void *stream);
dda_status_t dda_hsbcsr_export(dda_hsbcsr_t H, double *d_data, double *nd_data_up, int64_t *strides);
void dda_hsbcsr_free(dda_hsbcsr_t H);

/*
 * NEXT-3 — contact detection on the GPU (§III.B): the narrow phase's distance
 * judgment and its VE / VV classification, and the springs of the VE contacts that feed
 * dda_build_matrix (P:96 contact edge ratio).
 *
 * Geometry (device, caller-owned, valid until dda_contacts_free): block b is the polygon of vertices
 * vptr[b] .. vptr[b+1]-1 of vxy [V][2] (x, y interleaved, 16 B aligned), counter-clockwise, >= 3
 * vertices; edge e of block b runs from vertex e to the next vertex of b (cyclically).
 * dda_detect_contacts records every (vertex v of block i, edge e of block j != i) with
 *     d = Q2 - Q1, w = P - Q1, L2 = d.d, tn = w.d, t = clamp(tn / L2, 0, 1), C = Q1 + t d,
 *     dist2 = |P - C|^2 < d0^2      (each product and sum rounded as written),
 * typed VE (0) if 0 < tn < L2 and VV (1) otherwise (reading N3), in increasing (v, e).
 * The contact arrays are library-owned device memory (dda_contacts_t).  DDA_ERR_ARG: n <= 0, null
 * or misaligned pointers, d0 not positive and finite, a polygon with < 3 vertices or a non-finite
 * coordinate.  The call synchronises the stream (counts are read back).
 */
typedef struct dda_contacts *dda_contacts_t;
dda_status_t dda_detect_contacts(int32_t n_blocks, const int32_t *vptr, const double *vxy, double d0,
                                 void *stream, dda_contacts_t *out);
/* count = records, n_ve = VE records (each yields 2 springs), n_pairs = broad-phase candidate pairs */
dda_status_t dda_contacts_info(dda_contacts_t C, int64_t *count, int64_t *n_ve, int64_t *n_pairs);
/* host buffers of `count` entries (any may be NULL): i, v, j, e, type, t, dist2 */
dda_status_t dda_contacts_export(dda_contacts_t C, int32_t *i, int32_t *v, int32_t *j, int32_t *e,
                                 int32_t *type, double *t, double *dist2);
/*
 * Springs of the VE records, in record order, each a normal then a shear spring (every contact
 * "lock"; the open-close state switch is NEXT-4, out of scope): with u = d/|d| the edge tangent and
 * nrm = (u.y, -u.x) the outward normal of the counter-clockwise edge,
 *     e = T_i(P)^T n,  g = -((1 - t) T_j(Q1)^T n + t T_j(Q2)^T n),  n = nrm (normal) or u (shear),
 * T Shi's first-order displacement matrix at the offset from the block centroid cxy [n][2] (device),
 * penalties p_n and shear_ratio * p_n.  Outputs (device, caller-owned, 2 * n_ve entries; e, g
 * [2 n_ve][6] 16 B aligned) are exactly dda_build_matrix's spring inputs (bi = vertex block i,
 * bj = edge block j).  Stream-ordered, no synchronisation.
 */
dda_status_t dda_contact_springs(dda_contacts_t C, const double *cxy, double p_n, double shear_ratio,
                                 int32_t *bi, int32_t *bj, double *pen, double *e, double *g, void *stream);
/*
 * Second classification (§III.A; §III.B): the angle judgment and the VV1 / VV2 split
 * (reading N3-2; the oracle's O-10).  For record (vertex P = v of block i, edge
 * Q1 -> Q2 of block j) with a = P_prev - P, b = P_next - P (P's two edges), d = Q2 - Q1,
 * N = (d.y, -d.x) and s2 = sin_tol^2:
 *     keep iff  a.x b.y - a.y b.x < 0  (P convex)  and, for x in {a, b},
 *               N.x >= 0 or (N.x)^2 <= (s2 |N|^2) |x|^2   (no edge of P enters e's inner side by
 *                                                          more than asin(sin_tol))
 *     a kept VE record stays VE (class 0); a kept VV record is VV1 (class 1) if d is parallel to
 *     a or b within the tolerance ((d x a)^2 <= (s2 |d|^2) |a|^2, or with b), else VV2 (class 2).
 * Every product and sum is rounded as written.  The kept records are then stored class by class
 * (VE, VV1, VV2; increasing (v, e) within a class) by a stable radix sort on the class: the set is
 * replaced in place, `type` of dda_contacts_export becomes the class, dda_contacts_info's count and
 * n_ve the kept records, and dda_contact_springs then emits a normal and a shear spring for EVERY
 * record (VV1 / VV2 at the record's edge with t = 0 or 1), 2 * count springs.  sin_tol in [0, 1);
 * a set can be classified once (DDA_ERR_ARG otherwise).  Synchronising (class counts are read
 * back).  dda_contacts_classes reports the class counts and whether the set is classified.
 */
dda_status_t dda_classify_contacts(dda_contacts_t C, double sin_tol, void *stream);
dda_status_t dda_contacts_classes(dda_contacts_t C, int64_t *n_ve, int64_t *n_vv1, int64_t *n_vv2,
                                  int32_t *classified);
void dda_contacts_free(dda_contacts_t C);

/*
 * NEXT-4 — interpenetration check and open-close state switch (§III.A, third classification:
 * the switch integers p1, p2 and the categories C1-C5; §III.D, branch-restructured
 * kernels; P:27 loop 3).  Reading N4 (the oracle's O-11 / O-12).  The contacts are
 * the records of a CLASSIFIED set (dda_classify_contacts); contact k owns springs 2k (normal,
 * e_n, g_n) and 2k+1 (shear) of dda_contact_springs, passed back as e, g (device [2 count][6]).
 * States (device int32 [count]): 0 open, 1 slide, 2 lock.
 *
 * dda_contact_init: the signed gaps dn0 = n.(P - Q1) of every record (n the outward unit normal
 *   of its edge) and the contact endpoints sorted by block (cached in C); if state != NULL, the
 *   initial states: lock if dn0 <= 0 (touching / penetrating), else open.  Stream-ordered.
 * dda_contact_loads: out (device [6n]) = F (device [6n], or NULL for 0) + the gap load of the
 *   closed normal springs, F_i += f e_n, F_j += f g_n with f = -(pen[2k] dn0_k), summed per block in
 *   contact order (deterministic; pen device [2 count]).  Stream-ordered.
 * dda_contact_check: for the solution d (device [6n]):
 *     un = e_n.d_i + g_n.d_j, us = e_s.d_i + g_s.d_j, dn = dn0 + un,
 *     closed' = dn <= (closed ? open_tol : 0), lock' = closed' and not (p_s |us| > tan_phi (-p_n dn))
 *     p1 = closed' - closed, p2 = lock' - lock;
 *     VE / VV1: C1 p1 != 0; C2 p1 == 0 & p2 != 0; C3 p1 == p2 == 0 & closed'.
 *     VV2: C4 p1 != 0; C5 p1 == 0 & p2 != 0.  Otherwise category 0.
 *   state is updated in place; pen (device [2 count]) receives the next assembly's penalties
 *   (normal p_n if closed', shear shear_ratio p_n if lock', else 0); cat (device [count], may be
 *   NULL) the categories; cat_order (device [count], may be NULL) the contact ids grouped by
 *   category (stable); counts (host [6]) the number per category 0..5.  Products and sums are
 *   rounded as written, so states are bit-identical to the oracle's for the same d.  Synchronising.
 * dda_open_close: loop 3 — with the penalties of `state`: dda_update_values(K, kdiag, pen, e, g);
 *   F_eff = F + gap load; dda_pcg_solve(K, F_eff, d0 = d, d) with block-Jacobi (warm start);
 *   dda_contact_check; until no contact switches (no C1, C2, C4, C5) or max_oc iterations.  K must
 *   have been built from this set's springs (K's n = the contacts' n, 2 count springs); d (device
 *   [6n]) is the warm start in and the solution out; state in/out; pen out.  oc_iters, pcg_iters
 *   (total), converged (1 / 0) and rel_res (last solve) are host outputs.  DDA_ERR_ARG for a set
 *   that is not classified and initialised (dda_contact_init).  Synchronising.
 */
/*
 * NEXT-3 contact transfer (§III.B; reading N3-4, the oracle's O-13): for every record k of the
 * current set `cur`, state[k] (device int32 [cur count]) becomes prev_state[j] (device, [prev count])
 * of the previous step's record j with the same (vertex v, edge e) pair, and keeps its value (e.g.
 * the initial state of dda_contact_init) when there is none.  The previous records are radix-sorted
 * by (v, e) and searched ("sorted search").  matched (host, may be NULL): records transferred.
 * Synchronising.
 */
dda_status_t dda_contact_transfer(dda_contacts_t prev, const int32_t *prev_state, dda_contacts_t cur, int32_t *state,
                                  int64_t *matched, void *stream);
dda_status_t dda_contact_init(dda_contacts_t C, int32_t *state, void *stream);
dda_status_t dda_contact_loads(dda_contacts_t C, const double *e, const double *g, const double *pen, const double *F,
                               double *out, void *stream);
dda_status_t dda_contact_check(dda_contacts_t C, const double *d, const double *e, const double *g, double p_n,
                               double shear_ratio, double tan_phi, double open_tol, int32_t *state, double *pen,
                               int32_t *cat, int32_t *cat_order, int64_t *counts, void *stream);
dda_status_t dda_open_close(dda_matrix_t K, dda_contacts_t C, const double *kdiag, const double *F, const double *e,
                            const double *g, double p_n, double shear_ratio, double tan_phi, double open_tol,
                            double tol, int32_t maxit, int32_t max_oc, int32_t *state, double *pen, double *d,
                            int32_t *oc_iters, int32_t *pcg_iters, int32_t *converged, double *rel_res, void *stream);

/* Number of kernel launches the library has issued in this process (for the
 * benchmark's gpu_launches count). */
int64_t dda_launch_count(void);

/* Device memory.  The library allocates its own arrays (matrix, preconditioners,
 * PCG workspace, assembly temporaries) from a caching allocator: blocks freed by
 * dda_matrix_free stay cached and are handed back, stream-ordered, to the next
 * build of a similar size (the open-close loop rebuilds K every loop).
 * dda_memory_release returns every cached block to the driver (it synchronises
 * each device that holds some); dda_memory_cached reports the cached bytes.
 * Caller-owned buffers are never touched by either. */
void dda_memory_release(void);
int64_t dda_memory_cached(void);

void dda_matrix_free(dda_matrix_t K);
const char *dda_status_string(dda_status_t s);
/* Text of the last CUDA error seen by this thread ("" if none). */
const char *dda_last_cuda_error(void);

#ifdef __cplusplus
}
#endif
#endif /* DDA_H */
