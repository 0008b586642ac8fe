/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, single-threaded, obviously-correct CPU implementation of what
 * the hot path computes: assembly of the upper-symmetric 6x6-block stiffness
 * matrix from contact springs, its full expansion, SpMV, 6x6 block inverses,
 * textbook PCG and the three preconditioners of the paper's study.  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load it.  It shares no code, header, helper or table with
 * the CUDA path (paper_conf_ipps_xiaohmxw17_b200/csrc) and imports nothing from
 * it.  Compiled with -ffp-contract=off so products and sums round exactly as
 * written (ambiguity Z8/Z25 in DESIGN.md).
 *
 * Citations: "P:<line>" is /root/reference/PAPER.md.  Every function is pinned
 * by tests/test_oracle_*.py against something other than itself (scipy /
 * numpy library routines, closed forms, brute force, special cases); see the
 * "pins" column of DESIGN.md §4.  Parity unpinned: nothing (the paper's own
 * printed timings — Tables I–III — need its datasets and are not reproduced).
 */
#include <math.h>
#ifdef _OPENMP
#include <omp.h>
#endif
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { ORC_OK = 0, ORC_ERR_ARG = 1, ORC_ERR_OOM = 3, ORC_ERR_NOT_SPD = 4,
       ORC_ERR_BREAKDOWN = 5, ORC_ERR_NO_CONVERGENCE = 6 };
enum { ORC_PC_NONE = 0, ORC_PC_BJ = 1, ORC_PC_SSOR_AI = 2, ORC_PC_ILU0 = 3 };

typedef struct orc_matrix {
    int32_t n;            /* block rows */
    int64_t nnzb;         /* stored upper off-diagonal blocks */
    int32_t *row_ptr;     /* [n+1]  upper CSR; row-up-i[i] == row_ptr[i+1] */
    int32_t *col_idx;     /* [nnzb] */
    int32_t *low_ptr;     /* [n+1]  CSR of the (virtual) lower part, row-low-i */
    int32_t *low_row;     /* [nnzb] block column of each lower entry (= its upper row) */
    int32_t *low_to_up;   /* [nnzb] row-low-p: lower position -> upper position */
    double  *diag;        /* [n][36] diagonal sub-matrices (d-data) */
    double  *upper;       /* [nnzb][36] upper sub-matrices (nd-data-up) */
    /* O-2: full scalar CSR with both triangles, built on demand */
    int64_t  fnnz;
    int64_t *frow;        /* [6n+1] */
    int32_t *fcol;
    double  *fval;
    /* O-6: block ILU(0) factors on the full block pattern, built on demand */
    int64_t *bptr;        /* [n+1] full block pattern (both triangles + diagonal) */
    int32_t *bcol;
    int64_t *bdiagpos;    /* [n] position of the diagonal block in each row */
    double  *bval;        /* [nblocks][36] L (strict lower, unit diag implied) and U */
    double  *bdinv;       /* [n][36] inverse of each U_ii */
} orc_matrix;

static int cmp_u64(const void *a, const void *b) {
    uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
    return (x > y) - (x < y);
}

static int64_t find_key(const uint64_t *keys, int64_t cnt, uint64_t k) {
    int64_t lo = 0, hi = cnt - 1;
    while (lo <= hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (keys[mid] == k) return mid;
        if (keys[mid] < k) lo = mid + 1; else hi = mid - 1;
    }
    return -1;
}

void orc_free(orc_matrix *M) {
    if (!M) return;
    free(M->row_ptr); free(M->col_idx); free(M->low_ptr); free(M->low_row); free(M->low_to_up);
    free(M->diag); free(M->upper);
    free(M->frow); free(M->fcol); free(M->fval);
    free(M->bptr); free(M->bcol); free(M->bdiagpos); free(M->bval); free(M->bdinv);
    free(M);
}

/*
 * O-1  Assembly by definition ("only the upper entry of A is computed
 * and stored"; "this contact couple will contribute to sub-matrix a_ii,
 * a_jj, a_ij, and a_ji"; P:106 sum of each segment).
 *
 * Spring s = (i, j, p, e, g) contributes p*e*e^T to a_ii, p*g*g^T to a_jj and
 * K_ij = p*e*g^T to a_ij (a_ji = K_ij^T).  The stored block is (a,b) =
 * (min,max)(i,j); if i > j the stored block receives K_ij^T.  Each entry is
 * the sum, in increasing spring index, of (p*e[r])*g[c] (or the transposed
 * placement) starting from +0.0; the diagonal starts from Kd's upper triangle
 * and only r <= c is accumulated, then mirrored (ambiguities Z7, Z8, Z9).
 */
int orc_assemble(int32_t n, const double *kdiag, int64_t m,
                 const int32_t *bi, const int32_t *bj, const double *pen,
                 const double *e, const double *g, orc_matrix **out) {
    *out = NULL;
    if (n <= 0 || m < 0 || !kdiag) return ORC_ERR_ARG;
    if (m > 0 && (!bi || !bj || !pen || !e || !g)) return ORC_ERR_ARG;
    for (int64_t s = 0; s < m; ++s) {
        if (bi[s] < 0 || bi[s] >= n || bj[s] < 0 || bj[s] >= n || bi[s] == bj[s]) return ORC_ERR_ARG;
        if (!(pen[s] >= 0.0) || isinf(pen[s])) return ORC_ERR_ARG;
    }
    orc_matrix *M = (orc_matrix *)calloc(1, sizeof(orc_matrix));
    if (!M) return ORC_ERR_OOM;
    M->n = n;

    /* the set of unordered pairs {i,j}, as keys a*n+b with a<b, sorted */
    uint64_t *keys = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(m > 0 ? m : 1));
    if (!keys) { orc_free(M); return ORC_ERR_OOM; }
    for (int64_t s = 0; s < m; ++s) {
        uint64_t a = (uint64_t)(bi[s] < bj[s] ? bi[s] : bj[s]);
        uint64_t b = (uint64_t)(bi[s] < bj[s] ? bj[s] : bi[s]);
        keys[s] = a * (uint64_t)n + b;
    }
    qsort(keys, (size_t)m, sizeof(uint64_t), cmp_u64);
    int64_t nnzb = 0;
    for (int64_t s = 0; s < m; ++s)
        if (s == 0 || keys[s] != keys[s - 1]) keys[nnzb++] = keys[s];
    M->nnzb = nnzb;

    M->row_ptr = (int32_t *)calloc((size_t)n + 1, sizeof(int32_t));
    M->col_idx = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnzb ? nnzb : 1));
    M->low_ptr = (int32_t *)calloc((size_t)n + 1, sizeof(int32_t));
    M->low_row = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnzb ? nnzb : 1));
    M->low_to_up = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nnzb ? nnzb : 1));
    M->diag = (double *)malloc(sizeof(double) * 36 * (size_t)n);
    M->upper = (double *)calloc((size_t)(nnzb ? nnzb : 1) * 36, sizeof(double));
    if (!M->row_ptr || !M->col_idx || !M->low_ptr || !M->low_row || !M->low_to_up || !M->diag || !M->upper) {
        free(keys); orc_free(M); return ORC_ERR_OOM;
    }
    /* upper CSR (row-up-i) */
    for (int64_t u = 0; u < nnzb; ++u) {
        int32_t a = (int32_t)(keys[u] / (uint64_t)n);
        M->col_idx[u] = (int32_t)(keys[u] % (uint64_t)n);
        M->row_ptr[a + 1] += 1;
    }
    for (int32_t i = 0; i < n; ++i) M->row_ptr[i + 1] += M->row_ptr[i];

    /* upper values: springs in increasing s */
    for (int64_t s = 0; s < m; ++s) {
        int32_t i = bi[s], j = bj[s];
        uint64_t a = (uint64_t)(i < j ? i : j), b = (uint64_t)(i < j ? j : i);
        int64_t u = find_key(keys, nnzb, a * (uint64_t)n + b);
        double *B = M->upper + 36 * u;
        const double p = pen[s];
        const double *es = e + 6 * s, *gs = g + 6 * s;
        for (int r = 0; r < 6; ++r)
            for (int c = 0; c < 6; ++c) {
                double C = (i < j) ? (p * es[r]) * gs[c]     /* K_ij[r][c]           */
                                   : (p * es[c]) * gs[r];    /* K_ij^T[r][c] = K_ij[c][r] */
                B[6 * r + c] = B[6 * r + c] + C;
            }
    }
    /* diagonal: Kd upper triangle first, then springs in s order; mirror (Z9) */
    for (int32_t i = 0; i < n; ++i)
        for (int r = 0; r < 6; ++r)
            for (int c = r; c < 6; ++c) M->diag[36 * i + 6 * r + c] = kdiag[36 * i + 6 * r + c];
    for (int64_t s = 0; s < m; ++s) {
        const double p = pen[s];
        const double *es = e + 6 * s, *gs = g + 6 * s;
        double *Di = M->diag + 36 * (int64_t)bi[s], *Dj = M->diag + 36 * (int64_t)bj[s];
        for (int r = 0; r < 6; ++r)
            for (int c = r; c < 6; ++c) {
                Di[6 * r + c] = Di[6 * r + c] + (p * es[r]) * es[c];
                Dj[6 * r + c] = Dj[6 * r + c] + (p * gs[r]) * gs[c];
            }
    }
    for (int32_t i = 0; i < n; ++i)
        for (int r = 0; r < 6; ++r)
            for (int c = 0; c < r; ++c) M->diag[36 * i + 6 * r + c] = M->diag[36 * i + 6 * c + r];

    /* transpose map (row-low-i, row-low-p): counting transpose, rows ascending */
    for (int64_t u = 0; u < nnzb; ++u) M->low_ptr[M->col_idx[u] + 1] += 1;
    for (int32_t i = 0; i < n; ++i) M->low_ptr[i + 1] += M->low_ptr[i];
    int32_t *fill = (int32_t *)calloc((size_t)n, sizeof(int32_t));
    if (!fill) { free(keys); orc_free(M); return ORC_ERR_OOM; }
    for (int32_t a = 0; a < n; ++a)
        for (int32_t u = M->row_ptr[a]; u < M->row_ptr[a + 1]; ++u) {
            int32_t col = M->col_idx[u];
            int32_t pos = M->low_ptr[col] + fill[col]++;
            M->low_row[pos] = a;
            M->low_to_up[pos] = u;
        }
    free(fill);
    free(keys);
    *out = M;
    return ORC_OK;
}

void orc_info(const orc_matrix *M, int32_t *n, int64_t *nnzb) { *n = M->n; *nnzb = M->nnzb; }

void orc_export(const orc_matrix *M, int32_t *row_ptr, int32_t *col_idx, int32_t *low_ptr,
                int32_t *low_row, int32_t *low_to_up, double *diag, double *upper) {
    size_t n1 = (size_t)M->n + 1, z = (size_t)M->nnzb;
    if (row_ptr) memcpy(row_ptr, M->row_ptr, n1 * sizeof(int32_t));
    if (col_idx) memcpy(col_idx, M->col_idx, z * sizeof(int32_t));
    if (low_ptr) memcpy(low_ptr, M->low_ptr, n1 * sizeof(int32_t));
    if (low_row) memcpy(low_row, M->low_row, z * sizeof(int32_t));
    if (low_to_up) memcpy(low_to_up, M->low_to_up, z * sizeof(int32_t));
    if (diag) memcpy(diag, M->diag, (size_t)M->n * 36 * sizeof(double));
    if (upper) memcpy(upper, M->upper, z * 36 * sizeof(double));
}

/*
 * O-2  Full expansion: the scalar 6n x 6n CSR with both triangles (the matrix
 * the paper says most SpMV methods must "recover").  Block row i lists,
 * in increasing block column: the lower blocks V_ki^T (k<i), D_i, then the
 * upper blocks V_ij (j>i); every stored block contributes all 36 entries.
 */
int orc_expand(orc_matrix *M) {
    if (M->frow) return ORC_OK;
    const int32_t n = M->n;
    M->fnnz = 36 * ((int64_t)n + 2 * M->nnzb);
    M->frow = (int64_t *)malloc(sizeof(int64_t) * ((size_t)6 * n + 1));
    M->fcol = (int32_t *)malloc(sizeof(int32_t) * (size_t)M->fnnz);
    M->fval = (double *)malloc(sizeof(double) * (size_t)M->fnnz);
    if (!M->frow || !M->fcol || !M->fval) return ORC_ERR_OOM;
    int64_t pos = 0;
    for (int32_t i = 0; i < n; ++i)
        for (int r = 0; r < 6; ++r) {
            M->frow[6 * (int64_t)i + r] = pos;
            for (int32_t t = M->low_ptr[i]; t < M->low_ptr[i + 1]; ++t) {
                const int32_t k = M->low_row[t];
                const double *B = M->upper + 36 * (int64_t)M->low_to_up[t];
                for (int c = 0; c < 6; ++c) { M->fcol[pos] = 6 * k + c; M->fval[pos++] = B[6 * c + r]; }
            }
            for (int c = 0; c < 6; ++c) { M->fcol[pos] = 6 * i + c; M->fval[pos++] = M->diag[36 * (int64_t)i + 6 * r + c]; }
            for (int32_t u = M->row_ptr[i]; u < M->row_ptr[i + 1]; ++u) {
                const int32_t j = M->col_idx[u];
                const double *B = M->upper + 36 * (int64_t)u;
                for (int c = 0; c < 6; ++c) { M->fcol[pos] = 6 * j + c; M->fval[pos++] = B[6 * r + c]; }
            }
        }
    M->frow[6 * (int64_t)n] = pos;
    return ORC_OK;
}

int64_t orc_full_nnz(orc_matrix *M) { return orc_expand(M) == ORC_OK ? M->fnnz : -1; }

void orc_full_export(const orc_matrix *M, int64_t *frow, int32_t *fcol, double *fval) {
    memcpy(frow, M->frow, sizeof(int64_t) * ((size_t)6 * M->n + 1));
    memcpy(fcol, M->fcol, sizeof(int32_t) * (size_t)M->fnnz);
    memcpy(fval, M->fval, sizeof(double) * (size_t)M->fnnz);
}

/* O-3  y = A_full x, each row summed in column order (P:180 defines the product). */
int orc_spmv(orc_matrix *M, const double *x, double *y) {
    if (orc_expand(M) != ORC_OK) return ORC_ERR_OOM;
    const int64_t N = 6 * (int64_t)M->n;
    for (int64_t row = 0; row < N; ++row) {
        double s = 0.0;
        for (int64_t t = M->frow[row]; t < M->frow[row + 1]; ++t) s += M->fval[t] * x[M->fcol[t]];
        y[row] = s;
    }
    return ORC_OK;
}

/* O-3, timing variant ("a second, clearly labelled number is an OpenMP all-cores oracle
 * SpMV"): the same row loop as orc_spmv split over OpenMP threads — every row is summed in the same
 * order, so y is bitwise equal to orc_spmv's.  *threads = the thread count used. */
int orc_spmv_par(orc_matrix *M, const double *x, double *y, int32_t *threads) {
    if (orc_expand(M) != ORC_OK) return ORC_ERR_OOM;
    const int64_t N = 6 * (int64_t)M->n;
#ifdef _OPENMP
    *threads = omp_get_max_threads();
#pragma omp parallel for schedule(static)
#else
    *threads = 1;
#endif
    for (int64_t row = 0; row < N; ++row) {
        double s = 0.0;
        for (int64_t t = M->frow[row]; t < M->frow[row + 1]; ++t) s += M->fval[t] * x[M->fcol[t]];
        y[row] = s;
    }
    return ORC_OK;
}

/* O-3 on selected scalar rows only, straight from the block storage in the same
 * column order as O-2 (so it equals orc_spmv bit for bit without the 36(n+2nnzb)
 * expansion); used to check the full-size GPU result on sampled rows. */
void orc_spmv_rows(const orc_matrix *M, const int64_t *rows, int64_t k, const double *x, double *y) {
    for (int64_t q = 0; q < k; ++q) {
        const int32_t i = (int32_t)(rows[q] / 6);
        const int r = (int)(rows[q] % 6);
        double s = 0.0;
        for (int32_t t = M->low_ptr[i]; t < M->low_ptr[i + 1]; ++t) {
            const int32_t kk = M->low_row[t];
            const double *B = M->upper + 36 * (int64_t)M->low_to_up[t];
            for (int c = 0; c < 6; ++c) s += B[6 * c + r] * x[6 * (int64_t)kk + c];
        }
        for (int c = 0; c < 6; ++c) s += M->diag[36 * (int64_t)i + 6 * r + c] * x[6 * (int64_t)i + c];
        for (int32_t u = M->row_ptr[i]; u < M->row_ptr[i + 1]; ++u) {
            const int32_t j = M->col_idx[u];
            const double *B = M->upper + 36 * (int64_t)u;
            for (int c = 0; c < 6; ++c) s += B[6 * r + c] * x[6 * (int64_t)j + c];
        }
        y[q] = s;
    }
}

/*
 * O-4  Block inverse of one SPD 6x6 matrix: Cholesky A = L L^T (row by row),
 * L^{-1} by forward substitution, A^{-1} = L^{-T} L^{-1}.  Returns nonzero if
 * a pivot is <= 0 or not finite.  Block-Jacobi is "construction" of these
 * inverses (Table I) and "implementation" z_i = D_i^{-1} r_i.
 */
static int chol_inv6(const double *A, double *Ainv) {
    double L[36] = {0}, Li[36] = {0};
    for (int j = 0; j < 6; ++j) {
        double d = A[6 * j + j];
        for (int k = 0; k < j; ++k) d -= L[6 * j + k] * L[6 * j + k];
        if (!(d > 0.0) || !isfinite(d)) return 1;
        L[6 * j + j] = sqrt(d);
        for (int i = j + 1; i < 6; ++i) {
            double s = A[6 * i + j];
            for (int k = 0; k < j; ++k) s -= L[6 * i + k] * L[6 * j + k];
            L[6 * i + j] = s / L[6 * j + j];
        }
    }
    for (int c = 0; c < 6; ++c)          /* solve L * Li[:,c] = e_c */
        for (int i = 0; i < 6; ++i) {
            double s = (i == c) ? 1.0 : 0.0;
            for (int k = 0; k < i; ++k) s -= L[6 * i + k] * Li[6 * k + c];
            Li[6 * i + c] = s / L[6 * i + i];
        }
    for (int i = 0; i < 6; ++i)
        for (int j = 0; j < 6; ++j) {
            double s = 0.0;
            for (int k = 0; k < 6; ++k) s += Li[6 * k + i] * Li[6 * k + j];
            Ainv[6 * i + j] = s;
        }
    return 0;
}

int orc_bj_inv(const orc_matrix *M, double *dinv, int32_t *bad_block) {
    if (bad_block) *bad_block = -1;
    for (int32_t i = 0; i < M->n; ++i)
        if (chol_inv6(M->diag + 36 * (int64_t)i, dinv + 36 * (int64_t)i)) {
            if (bad_block) *bad_block = i;
            return ORC_ERR_NOT_SPD;
        }
    return ORC_OK;
}

static void bj_apply(int32_t n, const double *dinv, const double *r, double *z) {
    for (int64_t i = 0; i < n; ++i)
        for (int a = 0; a < 6; ++a) {
            double s = 0.0;
            for (int c = 0; c < 6; ++c) s += dinv[36 * i + 6 * a + c] * r[6 * i + c];
            z[6 * i + a] = s;
        }
}

/*
 * O-6  SSOR approximate inverse (after ref [36]; reading Z14):
 *   z = (I - w D^{-1} U) D^{-1} (I - w L D^{-1}) r,   L = U^T,
 * the symmetric Gauss-Seidel inverse (D + wU)^{-1} D (D + wL)^{-1} with each
 * triangular inverse truncated to first order, built from the full matrix
 * split A = L + D + U by block column (<, ==, > the block row).
 */
int orc_ssor_ai_apply(orc_matrix *M, const double *dinv, double omega, const double *r, double *z) {
    if (orc_expand(M) != ORC_OK) return ORC_ERR_OOM;
    const int32_t n = M->n;
    const int64_t N = 6 * (int64_t)n;
    double *t = (double *)malloc(sizeof(double) * (size_t)N);
    double *s = (double *)calloc((size_t)N, sizeof(double));
    double *w = (double *)malloc(sizeof(double) * (size_t)N);
    if (!t || !s || !w) { free(t); free(s); free(w); return ORC_ERR_OOM; }
    bj_apply(n, dinv, r, t);                                   /* t = D^{-1} r        */
    for (int64_t row = 0; row < N; ++row) {                    /* s = r - w L t       */
        double acc = 0.0;
        for (int64_t q = M->frow[row]; q < M->frow[row + 1]; ++q)
            if (M->fcol[q] / 6 < row / 6) acc += M->fval[q] * t[M->fcol[q]];
        s[row] = r[row] - omega * acc;
    }
    bj_apply(n, dinv, s, w);                                   /* w = D^{-1} s        */
    for (int64_t row = 0; row < N; ++row) {                    /* t = U w             */
        double acc = 0.0;
        for (int64_t q = M->frow[row]; q < M->frow[row + 1]; ++q)
            if (M->fcol[q] / 6 > row / 6) acc += M->fval[q] * w[M->fcol[q]];
        t[row] = acc;
    }
    bj_apply(n, dinv, t, s);                                   /* s = D^{-1} U w      */
    for (int64_t row = 0; row < N; ++row) z[row] = w[row] - omega * s[row];
    free(t); free(s); free(w);
    return ORC_OK;
}

/* 6x6 inverse by Gauss-Jordan with partial pivoting (a library-grade primitive). */
static int gj_inv6(const double *A, double *Ainv) {
    double a[6][12];
    for (int i = 0; i < 6; ++i)
        for (int j = 0; j < 12; ++j) a[i][j] = (j < 6) ? A[6 * i + j] : (j - 6 == i ? 1.0 : 0.0);
    for (int c = 0; c < 6; ++c) {
        int p = c;
        for (int i = c + 1; i < 6; ++i) if (fabs(a[i][c]) > fabs(a[p][c])) p = i;
        if (!(fabs(a[p][c]) > 0.0) || !isfinite(a[p][c])) return 1;
        if (p != c) for (int j = 0; j < 12; ++j) { double tmp = a[c][j]; a[c][j] = a[p][j]; a[p][j] = tmp; }
        double piv = a[c][c];
        for (int j = 0; j < 12; ++j) a[c][j] /= piv;
        for (int i = 0; i < 6; ++i)
            if (i != c) { double f = a[i][c]; for (int j = 0; j < 12; ++j) a[i][j] -= f * a[c][j]; }
    }
    for (int i = 0; i < 6; ++i) for (int j = 0; j < 6; ++j) Ainv[6 * i + j] = a[i][j + 6];
    return 0;
}

static void mm6(const double *A, const double *B, double *C) {   /* C = A B */
    for (int i = 0; i < 6; ++i)
        for (int j = 0; j < 6; ++j) {
            double s = 0.0;
            for (int k = 0; k < 6; ++k) s += A[6 * i + k] * B[6 * k + j];
            C[6 * i + j] = s;
        }
}

static int64_t bfind(const orc_matrix *M, int32_t row, int32_t col) {
    int64_t lo = M->bptr[row], hi = M->bptr[row + 1] - 1;
    while (lo <= hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (M->bcol[mid] == col) return mid;
        if (M->bcol[mid] < col) lo = mid + 1; else hi = mid - 1;
    }
    return -1;
}

/*
 * O-6  Block ILU(0) without pivoting on the full block pattern ("ILU
 * ... provided by cuSPARSE"; reading Z15), Saad's IKJ variant in block form:
 *   for i: for k < i in row i (ascending): A_ik <- A_ik A_kk^{-1};
 *          for j > k in row i with (k,j) in the pattern: A_ij <- A_ij - A_ik A_kj.
 * Uses both triangles and no symmetric shortcut (deliberately different code
 * from the GPU's upper-only incomplete-Cholesky form).
 */
int orc_ilu0_factor(orc_matrix *M) {
    const int32_t n = M->n;
    free(M->bptr); free(M->bcol); free(M->bdiagpos); free(M->bval); free(M->bdinv);
    const int64_t nb = (int64_t)n + 2 * M->nnzb;
    M->bptr = (int64_t *)malloc(sizeof(int64_t) * ((size_t)n + 1));
    M->bcol = (int32_t *)malloc(sizeof(int32_t) * (size_t)nb);
    M->bdiagpos = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
    M->bval = (double *)malloc(sizeof(double) * 36 * (size_t)nb);
    M->bdinv = (double *)malloc(sizeof(double) * 36 * (size_t)n);
    if (!M->bptr || !M->bcol || !M->bdiagpos || !M->bval || !M->bdinv) return ORC_ERR_OOM;
    int64_t pos = 0;
    for (int32_t i = 0; i < n; ++i) {
        M->bptr[i] = pos;
        for (int32_t t = M->low_ptr[i]; t < M->low_ptr[i + 1]; ++t) {
            const double *B = M->upper + 36 * (int64_t)M->low_to_up[t];
            M->bcol[pos] = M->low_row[t];
            for (int r = 0; r < 6; ++r) for (int c = 0; c < 6; ++c) M->bval[36 * pos + 6 * r + c] = B[6 * c + r];
            ++pos;
        }
        M->bdiagpos[i] = pos;
        M->bcol[pos] = i;
        memcpy(M->bval + 36 * pos, M->diag + 36 * (int64_t)i, 36 * sizeof(double));
        ++pos;
        for (int32_t u = M->row_ptr[i]; u < M->row_ptr[i + 1]; ++u) {
            M->bcol[pos] = M->col_idx[u];
            memcpy(M->bval + 36 * pos, M->upper + 36 * (int64_t)u, 36 * sizeof(double));
            ++pos;
        }
    }
    M->bptr[n] = pos;
    double T[36];
    for (int32_t i = 0; i < n; ++i) {
        for (int64_t q = M->bptr[i]; q < M->bdiagpos[i]; ++q) {
            const int32_t k = M->bcol[q];
            mm6(M->bval + 36 * q, M->bdinv + 36 * (int64_t)k, T);      /* A_ik <- A_ik A_kk^{-1} */
            memcpy(M->bval + 36 * q, T, sizeof T);
            for (int64_t qj = q + 1; qj < M->bptr[i + 1]; ++qj) {
                const int64_t kj = bfind(M, k, M->bcol[qj]);
                if (kj < 0) continue;
                mm6(M->bval + 36 * q, M->bval + 36 * kj, T);             /* A_ij -= A_ik A_kj */
                for (int z = 0; z < 36; ++z) M->bval[36 * qj + z] -= T[z];
            }
        }
        if (gj_inv6(M->bval + 36 * M->bdiagpos[i], M->bdinv + 36 * (int64_t)i)) return ORC_ERR_NOT_SPD;
    }
    return ORC_OK;
}

/* O-6  ILU(0) apply: forward y_i = r_i - sum_{k<i} L_ik y_k, then
 * backward z_i = U_ii^{-1} (y_i - sum_{j>i} U_ij z_j). */
void orc_ilu0_apply(const orc_matrix *M, const double *r, double *z) {
    const int32_t n = M->n;
    for (int32_t i = 0; i < n; ++i) {
        double y[6];
        for (int a = 0; a < 6; ++a) y[a] = r[6 * (int64_t)i + a];
        for (int64_t q = M->bptr[i]; q < M->bdiagpos[i]; ++q) {
            const double *B = M->bval + 36 * q;
            const double *yk = z + 6 * (int64_t)M->bcol[q];
            for (int a = 0; a < 6; ++a) for (int c = 0; c < 6; ++c) y[a] -= B[6 * a + c] * yk[c];
        }
        for (int a = 0; a < 6; ++a) z[6 * (int64_t)i + a] = y[a];
    }
    for (int32_t i = n - 1; i >= 0; --i) {
        double y[6];
        for (int a = 0; a < 6; ++a) y[a] = z[6 * (int64_t)i + a];
        for (int64_t q = M->bdiagpos[i] + 1; q < M->bptr[i + 1]; ++q) {
            const double *B = M->bval + 36 * q;
            const double *zj = z + 6 * (int64_t)M->bcol[q];
            for (int a = 0; a < 6; ++a) for (int c = 0; c < 6; ++c) y[a] -= B[6 * a + c] * zj[c];
        }
        const double *Ui = M->bdinv + 36 * (int64_t)i;
        for (int a = 0; a < 6; ++a) {
            double s = 0.0;
            for (int c = 0; c < 6; ++c) s += Ui[6 * a + c] * y[c];
            z[6 * (int64_t)i + a] = s;
        }
    }
}

static double dot(int64_t N, const double *a, const double *b) {
    double s = 0.0;
    for (int64_t i = 0; i < N; ++i) s += a[i] * b[i];
    return s;
}

/*
 * O-5  Textbook preconditioned CG (Saad, Iterative Methods, Alg. 9.1; the
 * paper gives no pseudo-code: P:54).  Warm start from d0.
 * Stop when ||r_k||_2 <= tol * ||F||_2 on the recursive residual (reading Z1);
 * the true residual ||F - K d|| / ||F|| is reported.  F = 0 -> d = 0 (Z2).
 * Breakdown when sigma = p^T K p <= 0 or rho' <= 0 or either is not finite
 * (Z19).  If `trace` is non-NULL, d after iteration k is stored at
 * trace[k*6n] (k = 0 is d0), for the K-norm monotonicity pin (Z18).
 */
int orc_pcg(orc_matrix *M, const double *F, const double *d0, double *d, double tol, int32_t maxit,
            int32_t precond, double omega, int32_t *iters, double *rel_res, double *trace) {
    const int32_t n = M->n;
    const int64_t N = 6 * (int64_t)n;
    *iters = 0; *rel_res = 0.0;
    if (!(tol > 0.0) || maxit < 0) return ORC_ERR_ARG;
    if (orc_expand(M) != ORC_OK) return ORC_ERR_OOM;
    double *r = (double *)malloc(sizeof(double) * (size_t)N);
    double *z = (double *)malloc(sizeof(double) * (size_t)N);
    double *p = (double *)malloc(sizeof(double) * (size_t)N);
    double *q = (double *)malloc(sizeof(double) * (size_t)N);
    double *dinv = (double *)malloc(sizeof(double) * 36 * (size_t)n);
    if (!r || !z || !p || !q || !dinv) { free(r); free(z); free(p); free(q); free(dinv); return ORC_ERR_OOM; }
    int st = ORC_OK;
#define ORC_FAIL(code) do { st = (code); goto done; } while (0)
    if (precond == ORC_PC_BJ || precond == ORC_PC_SSOR_AI) {
        if (orc_bj_inv(M, dinv, NULL)) ORC_FAIL(ORC_ERR_NOT_SPD);
    } else if (precond == ORC_PC_ILU0) {
        int fs = orc_ilu0_factor(M);
        if (fs) ORC_FAIL(fs);
    } else if (precond != ORC_PC_NONE) ORC_FAIL(ORC_ERR_ARG);

    const double b = sqrt(dot(N, F, F));
    if (b == 0.0) {                                                  /* Z2 */
        for (int64_t k = 0; k < N; ++k) d[k] = 0.0;
        if (trace) memcpy(trace, d, sizeof(double) * (size_t)N);
        goto done;
    }
    if (d != d0) memcpy(d, d0, sizeof(double) * (size_t)N);
    if (trace) memcpy(trace, d, sizeof(double) * (size_t)N);
    orc_spmv(M, d, q);
    for (int64_t k = 0; k < N; ++k) r[k] = F[k] - q[k];              /* r = F - K d0 */
    if (sqrt(dot(N, r, r)) <= tol * b) goto final;
#define APPLY_M(src, dst) do { \
        if (precond == ORC_PC_BJ) bj_apply(n, dinv, src, dst); \
        else if (precond == ORC_PC_SSOR_AI) orc_ssor_ai_apply(M, dinv, omega, src, dst); \
        else if (precond == ORC_PC_ILU0) orc_ilu0_apply(M, src, dst); \
        else memcpy(dst, src, sizeof(double) * (size_t)N); } while (0)
    APPLY_M(r, z);                                                   /* z = M^{-1} r */
    memcpy(p, z, sizeof(double) * (size_t)N);                        /* p = z        */
    double rho = dot(N, r, z);
    if (!(rho > 0.0) || !isfinite(rho)) ORC_FAIL(ORC_ERR_BREAKDOWN);
    st = ORC_ERR_NO_CONVERGENCE;
    for (int32_t k = 0; k < maxit; ++k) {
        orc_spmv(M, p, q);                                           /* q = K p      */
        const double sigma = dot(N, p, q);
        if (!(sigma > 0.0) || !isfinite(sigma)) { st = ORC_ERR_BREAKDOWN; break; }
        const double alpha = rho / sigma;
        for (int64_t t = 0; t < N; ++t) d[t] += alpha * p[t];
        for (int64_t t = 0; t < N; ++t) r[t] -= alpha * q[t];
        *iters = k + 1;
        if (trace) memcpy(trace + (size_t)(k + 1) * (size_t)N, d, sizeof(double) * (size_t)N);
        if (sqrt(dot(N, r, r)) <= tol * b) { st = ORC_OK; break; }
        APPLY_M(r, z);
        const double rho1 = dot(N, r, z);
        if (!(rho1 > 0.0) || !isfinite(rho1)) { st = ORC_ERR_BREAKDOWN; break; }
        const double beta = rho1 / rho;
        for (int64_t t = 0; t < N; ++t) p[t] = z[t] + beta * p[t];
        rho = rho1;
    }
#undef APPLY_M
final:
    orc_spmv(M, d, q);
    for (int64_t k = 0; k < N; ++k) r[k] = F[k] - q[k];
    *rel_res = sqrt(dot(N, r, r)) / b;
done:
#undef ORC_FAIL
    free(r); free(z); free(p); free(q); free(dinv);
    return st;
}

/*
 * O-7  Dense LDL^T without pivoting of the assembled 6n x 6n matrix, then
 * L y = b, D w = y, L^T x = w.  Tiny sizes only (the configs[0] check "vs
 * dense LDL^T").  Returns ORC_ERR_NOT_SPD if a pivot is <= 0.
 */
int orc_ldlt_solve(orc_matrix *M, const double *b, double *x) {
    if (orc_expand(M) != ORC_OK) return ORC_ERR_OOM;
    const int64_t N = 6 * (int64_t)M->n;
    double *A = (double *)calloc((size_t)(N * N), sizeof(double));
    double *D = (double *)malloc(sizeof(double) * (size_t)N);
    if (!A || !D) { free(A); free(D); return ORC_ERR_OOM; }
    for (int64_t row = 0; row < N; ++row)
        for (int64_t t = M->frow[row]; t < M->frow[row + 1]; ++t) A[row * N + M->fcol[t]] = M->fval[t];
    /* L stored in the strict lower triangle of A */
    for (int64_t j = 0; j < N; ++j) {
        double dj = A[j * N + j];
        for (int64_t k = 0; k < j; ++k) dj -= A[j * N + k] * A[j * N + k] * D[k];
        if (!(dj > 0.0) || !isfinite(dj)) { free(A); free(D); return ORC_ERR_NOT_SPD; }
        D[j] = dj;
        for (int64_t i = j + 1; i < N; ++i) {
            double s = A[i * N + j];
            for (int64_t k = 0; k < j; ++k) s -= A[i * N + k] * A[j * N + k] * D[k];
            A[i * N + j] = s / dj;
        }
    }
    for (int64_t i = 0; i < N; ++i) {
        double s = b[i];
        for (int64_t k = 0; k < i; ++k) s -= A[i * N + k] * x[k];
        x[i] = s;
    }
    for (int64_t i = 0; i < N; ++i) x[i] /= D[i];
    for (int64_t i = N - 1; i >= 0; --i) {
        double s = x[i];
        for (int64_t k = i + 1; k < N; ++k) s -= A[k * N + i] * x[k];
        x[i] = s;
    }
    free(A); free(D);
    return ORC_OK;
}

/*
 * O-8 (NEXT-3)  Contact detection: the narrow phase's distance judgment and its VE / VV
 * classification (§III.B; §III.A).  Plain definition, all pairs, no
 * broad phase.  Blocks are polygons: block b owns vertices vptr[b] .. vptr[b+1]-1 of vxy[V][2],
 * counter-clockwise; edge e of block b runs from vertex e to the next vertex of b (cyclically).
 * For every vertex v (of block i) in [v_begin, v_end) and every edge e of every block j != i:
 *     d = Q2 - Q1,  w = P - Q1,  L2 = d.d,  tn = w.d,  t = clamp(tn / L2, 0, 1),
 *     C = Q1 + t d,  dist2 = |P - C|^2          (each product and sum rounded as written)
 * (v, e) is a contact iff dist2 < d0^2; its type is VE (0) if 0 < tn < L2 (the nearest point of
 * the edge is interior) and VV (1) otherwise (the nearest point is the vertex Q1 or Q2).
 * Records come out in increasing (v, e), i.e. increasing (i, v, j, e).  At most `cap` are
 * written; the return value is the total count (or -1 on bad arguments).
 */
int64_t orc_detect_contacts(int32_t n, const int32_t *vptr, const double *vxy, double d0, int32_t v_begin,
                            int32_t v_end, int64_t cap, int32_t *ci, int32_t *cv, int32_t *cj, int32_t *ce,
                            int32_t *ctype, double *ct, double *cd2) {
    if (n <= 0 || !vptr || !vxy || !(d0 > 0.0)) return -1;
    const double r2 = d0 * d0;
    int64_t cnt = 0;
    int32_t i = 0;
    for (int32_t v = v_begin; v < v_end; ++v) {
        while (!(vptr[i] <= v && v < vptr[i + 1])) ++i;      /* block of vertex v (v ascending) */
        const double px = vxy[2 * v], py = vxy[2 * v + 1];
        for (int32_t j = 0; j < n; ++j) {
            if (j == i) continue;
            const int32_t a = vptr[j], b = vptr[j + 1];
            for (int32_t e = a; e < b; ++e) {
                const int32_t e2 = (e + 1 < b) ? e + 1 : a;
                const double q1x = vxy[2 * e], q1y = vxy[2 * e + 1];
                const double dx = vxy[2 * e2] - q1x, dy = vxy[2 * e2 + 1] - q1y;
                const double wx = px - q1x, wy = py - q1y;
                const double L2 = dx * dx + dy * dy;
                const double tn = wx * dx + wy * dy;
                double t = tn / L2;
                if (t < 0.0) t = 0.0;
                if (t > 1.0) t = 1.0;
                const double cx = q1x + t * dx, cy = q1y + t * dy;
                const double ex = px - cx, ey = py - cy;
                const double dist2 = ex * ex + ey * ey;
                if (dist2 < r2) {
                    if (cnt < cap) {
                        ci[cnt] = i; cv[cnt] = v; cj[cnt] = j; ce[cnt] = e;
                        ctype[cnt] = (tn > 0.0 && tn < L2) ? 0 : 1;
                        ct[cnt] = t; cd2[cnt] = dist2;
                    }
                    ++cnt;
                }
            }
        }
    }
    return cnt;
}

/* T(P)^T u for Shi's first-order displacement function at offset (x, y) from the block centroid
 * (rows of T: [1, 0, -y, x, 0, y/2] and [0, 1, x, 0, y, x/2]; external, Shi 1988). */
static void tt_times(double x, double y, double ux, double uy, double *o) {
    o[0] = ux;
    o[1] = uy;
    o[2] = -y * ux + x * uy;
    o[3] = x * ux;
    o[4] = y * uy;
    o[5] = 0.5 * y * ux + 0.5 * x * uy;
}

/*
 * O-9 (NEXT-3)  Springs of the VE contacts (the input of O-1): for each record with type
 * VE, in record order, a normal spring then a shear spring (every contact "lock"; the open-close
 * state switch is NEXT-4).  With u = d / |d| the edge tangent and nrm = (u.y, -u.x) the outward
 * normal of the counter-clockwise edge, P the vertex of block i, Q1, Q2 the edge of block j and
 * t the record's edge ratio:
 *     e = T_i(P)^T n,   g = -((1 - t) T_j(Q1)^T n + t T_j(Q2)^T n),   n = nrm (normal) or u (shear)
 * penalties p_n and shear_ratio * p_n.  Writes 2 * (#VE) springs; returns that count.
 */
int64_t orc_contact_springs(int32_t n, const int32_t *vptr, const double *vxy, const double *cxy, int64_t nc,
                            const int32_t *ci, const int32_t *cv, const int32_t *cj, const int32_t *ce,
                            const int32_t *ctype, const double *ct, double p_n, double shear_ratio,
                            int32_t *bi, int32_t *bj, double *pen, double *e, double *g) {
    int64_t s = 0;
    (void)n;
    for (int64_t k = 0; k < nc; ++k) {
        if (ctype[k] != 0) continue;
        const int32_t i = ci[k], j = cj[k], v = cv[k], q = ce[k];
        const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
        const double dx = vxy[2 * q2] - vxy[2 * q], dy = vxy[2 * q2 + 1] - vxy[2 * q + 1];
        const double len = sqrt(dx * dx + dy * dy);
        const double ux = dx / len, uy = dy / len;
        const double t = ct[k];
        const double pix = vxy[2 * v] - cxy[2 * i], piy = vxy[2 * v + 1] - cxy[2 * i + 1];
        const double q1x = vxy[2 * q] - cxy[2 * j], q1y = vxy[2 * q + 1] - cxy[2 * j + 1];
        const double q2x = vxy[2 * q2] - cxy[2 * j], q2y = vxy[2 * q2 + 1] - cxy[2 * j + 1];
        for (int sp = 0; sp < 2; ++sp) {
            const double nx = sp == 0 ? uy : ux, ny = sp == 0 ? -ux : uy;
            double a[6], b1[6], b2[6];
            tt_times(pix, piy, nx, ny, a);
            tt_times(q1x, q1y, nx, ny, b1);
            tt_times(q2x, q2y, nx, ny, b2);
            bi[s] = i;
            bj[s] = j;
            pen[s] = sp == 0 ? p_n : shear_ratio * p_n;
            for (int r = 0; r < 6; ++r) {
                e[6 * s + r] = a[r];
                g[6 * s + r] = -((1.0 - t) * b1[r] + t * b2[r]);
            }
            ++s;
        }
    }
    return s;
}

/*
 * O-10 (NEXT-3)  The angle judgment and the VV1 / VV2 split (§III.A, second
 * classification: "some data of VE and VV are abandoned if they cannot fulfill the contact angle
 * condition; the other data of VV will be divided into VV1 and VV2; the contacts with parallel
 * edges are classified as VV1 or as VV2 otherwise"; §III.B).  The paper gives no formula; the
 * reading (N3-2) after Shi's contact rules (external) is, for record k = (vertex P =
 * v of block i, edge e = Q1 -> Q2 of block j), with P_prev / P_next the neighbours of v in block i:
 *     a = P_prev - P,  b = P_next - P         (the two edges of block i at P, pointing away)
 *     d = Q2 - Q1,     N = (d.y, -d.x)        (outward normal of the counter-clockwise edge)
 *     s2 = sin_tol * sin_tol,  NN = N.N
 *     convex:  a.x b.y - a.y b.x < 0          (P is a convex corner of block i)
 *     out(x):  N.x >= 0  or  (N.x)^2 <= (s2 NN) |x|^2      (edge x of P does not point into the
 *                                                          inner side of e by more than the
 *                                                          tolerance angle asin(sin_tol))
 * the record passes the angle judgment iff convex and out(a) and out(b); a passing VE record stays
 * VE (class 0); a passing VV record is VV1 (class 1) if one of P's edges is parallel to e within
 * the tolerance, (d x a)^2 <= (s2 NN) |a|^2 or (d x b)^2 <= (s2 NN) |b|^2, else VV2 (class 2);
 * a failing record is abandoned (class -1).  Every product and sum is rounded as written.
 */
int orc_classify_contacts(int32_t n, const int32_t *vptr, const double *vxy, int64_t nc, const int32_t *ci,
                          const int32_t *cv, const int32_t *cj, const int32_t *ce, const int32_t *ctype,
                          double sin_tol, int32_t *cls) {
    if (n <= 0 || !vptr || !vxy || !(sin_tol >= 0.0) || !(sin_tol < 1.0)) return ORC_ERR_ARG;
    const double s2 = sin_tol * sin_tol;
    for (int64_t k = 0; k < nc; ++k) {
        const int32_t i = ci[k], v = cv[k], j = cj[k], q = ce[k];
        const int32_t vp = (v > vptr[i]) ? v - 1 : vptr[i + 1] - 1;
        const int32_t vn = (v + 1 < vptr[i + 1]) ? v + 1 : vptr[i];
        const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
        const double px = vxy[2 * v], py = vxy[2 * v + 1];
        const double ax = vxy[2 * vp] - px, ay = vxy[2 * vp + 1] - py;
        const double bx = vxy[2 * vn] - px, by = vxy[2 * vn + 1] - py;
        const double dx = vxy[2 * q2] - vxy[2 * q], dy = vxy[2 * q2 + 1] - vxy[2 * q + 1];
        const double Nx = dy, Ny = -dx;
        const double NN = Nx * Nx + Ny * Ny;
        const double aa = ax * ax + ay * ay, bb = bx * bx + by * by;
        const double lim = s2 * NN;
        const int convex = (ax * by - ay * bx) < 0.0;
        const double fa = Nx * ax + Ny * ay, fb = Nx * bx + Ny * by;
        const int out_a = fa >= 0.0 || fa * fa <= lim * aa;
        const int out_b = fb >= 0.0 || fb * fb <= lim * bb;
        if (!(convex && out_a && out_b)) {
            cls[k] = -1;
        } else if (ctype[k] == 0) {
            cls[k] = 0;
        } else {
            const double xa = dx * ay - dy * ax, xb = dx * by - dy * bx;
            const int par = xa * xa <= lim * aa || xb * xb <= lim * bb;
            cls[k] = par ? 1 : 2;
        }
    }
    return ORC_OK;
}

/* signed distance of record k's vertex from its edge line, n.(P - Q1), n = (u.y, -u.x), as O-11 */
static double contact_gap(const int32_t *vptr, const double *vxy, int32_t v, int32_t j, int32_t q) {
    const int32_t q2 = (q + 1 < vptr[j + 1]) ? q + 1 : vptr[j];
    const double dx = vxy[2 * q2] - vxy[2 * q], dy = vxy[2 * q2 + 1] - vxy[2 * q + 1];
    const double len = sqrt(dx * dx + dy * dy);
    const double ux = dx / len, uy = dy / len;
    const double nx = uy, ny = -ux;
    return nx * (vxy[2 * v] - vxy[2 * q]) + ny * (vxy[2 * v + 1] - vxy[2 * q + 1]);
}

/*
 * O-11 (NEXT-4)  Interpenetration check and open-close state switch of one open-close iteration
 * (§III.A, third classification; §III.D; loop 3 of §I).  The paper
 * names the switch integers p1, p2 in {-1, 0, 1} and the categories C1-C5 but gives no formulas;
 * the reading (N4) after Shi's open-close rules (external):
 * contact k is record k of a classified set (class 0 VE, 1 VV1, 2 VV2) whose springs are 2k (normal,
 * vectors e_n, g_n) and 2k+1 (shear, e_s, g_s) of O-9; d is the solution of K d = F.  With u the
 * unit tangent of the record's edge (u = d/|d|, as O-9) and n = (u.y, -u.x) its outward normal:
 *     dn0 = n.x (P.x - Q1.x) + n.y (P.y - Q1.y)        signed distance of the vertex (> 0 outside)
 *     un  = sum_r e_n[r] d_i[r] + sum_r g_n[r] d_j[r]   relative normal displacement (r = 0..5 in
 *     us  = sum_r e_s[r] d_i[r] + sum_r g_s[r] d_j[r]   order, e before g, from +0.0)
 *     dn  = dn0 + un
 *     closed = dn <= (was closed ? open_tol : 0)  (an open contact closes when it touches; a closed
 *              one opens only when its vertex separates by more than the tension tolerance)
 *     fn = -p_n dn;   fs = (shear_ratio p_n) |us|
 *     lock   = closed and not (fs > tan_phi fn)         (Mohr-Coulomb, no cohesion)
 *     state' = 0 open / 1 slide / 2 lock;   p1 = closed' - closed;   p2 = lock' - lock
 * Categories: VE and VV1: C1 |p1| > 0; C2 p1 = 0 and |p2| > 0; C3 p1 = p2 = 0 and closed'
 * ("some other condition" read as: the contact stays in contact); VV2: C4 |p1| > 0; C5 p1 = 0 and
 * |p2| > 0; otherwise 0 (abandoned: nothing to re-check).  Penalties of the next assembly: normal
 * p_n if closed' else 0, shear shear_ratio p_n if lock' else 0 (an open contact keeps its springs
 * with p = 0, reading Z10, so the spring list and the matrix structure do not change).
 * state[k] is read (previous) and overwritten (new); cat[k] receives 0..5; pen [2 nc].
 */
int orc_contact_check(int32_t n, const int32_t *vptr, const double *vxy, int64_t nc, const int32_t *ci,
                      const int32_t *cv, const int32_t *cj, const int32_t *ce, const int32_t *cls, const double *d,
                      const double *e, const double *g, double p_n, double shear_ratio, double tan_phi,
                      double open_tol, int32_t *state, double *pen, int32_t *cat) {
    if (n <= 0 || !(p_n >= 0.0) || !(shear_ratio >= 0.0) || !(tan_phi >= 0.0) || !(open_tol >= 0.0))
        return ORC_ERR_ARG;
    const double ps = shear_ratio * p_n;
    for (int64_t k = 0; k < nc; ++k) {
        const int32_t i = ci[k], v = cv[k], j = cj[k], q = ce[k];
        const double dn0 = contact_gap(vptr, vxy, v, j, q);
        const double *en = e + 12 * k, *es = e + 12 * k + 6, *gn = g + 12 * k, *gs = g + 12 * k + 6;
        double un = 0.0, us = 0.0;
        for (int r = 0; r < 6; ++r) un = un + en[r] * d[6 * (int64_t)i + r];
        for (int r = 0; r < 6; ++r) un = un + gn[r] * d[6 * (int64_t)j + r];
        for (int r = 0; r < 6; ++r) us = us + es[r] * d[6 * (int64_t)i + r];
        for (int r = 0; r < 6; ++r) us = us + gs[r] * d[6 * (int64_t)j + r];
        const double dn = dn0 + un;
        const int old = state[k];
        const int closed = dn <= (old >= 1 ? open_tol : 0.0);
        const double fn = -p_n * dn;
        const double fs = ps * fabs(us);
        const int lock = closed && !(fs > tan_phi * fn);
        const int p1 = closed - (old >= 1);
        const int p2 = lock - (old == 2);
        int c = 0;
        if (cls[k] == 2) {
            if (p1 != 0) c = 4;
            else if (p2 != 0) c = 5;
        } else {
            if (p1 != 0) c = 1;
            else if (p2 != 0) c = 2;
            else if (closed) c = 3;
        }
        cat[k] = c;
        state[k] = closed ? (lock ? 2 : 1) : 0;
        pen[2 * k] = closed ? p_n : 0.0;
        pen[2 * k + 1] = lock ? ps : 0.0;
    }
    return ORC_OK;
}

/*
 * O-12 (NEXT-4)  Contact initialisation and the gap load of the open-close loop (reading N4).
 * The normal spring of a closed contact stores the energy p_n (dn0 + un)^2 / 2 (un = e_n.d_i +
 * g_n.d_j, dn0 = the signed gap of O-11): its stiffness p_n [e_n; g_n][e_n; g_n]^T is assembled by
 * O-1 from the spring list, and its load is
 *     F_i += f e_n,   F_j += f g_n,    f = -(pen[2k] * dn0_k)
 * summed into Fc (zeroed here) for k = 0, 1, ... in that order, each product f * e[r] rounded and
 * then added (Fc[b] is the plain sequential sum over the contacts touching b, in contact order).
 * Initial states (when state0 != NULL): lock (2) if dn0 <= 0 (touching or penetrating), else open.
 */
int orc_contact_loads(int32_t n, const int32_t *vptr, const double *vxy, int64_t nc, const int32_t *ci,
                      const int32_t *cv, const int32_t *cj, const int32_t *ce, const double *e, const double *g,
                      const double *pen, double *Fc, int32_t *state0) {
    if (n <= 0) return ORC_ERR_ARG;
    for (int64_t t = 0; t < 6 * (int64_t)n; ++t) Fc[t] = 0.0;
    for (int64_t k = 0; k < nc; ++k) {
        const double dn0 = contact_gap(vptr, vxy, cv[k], cj[k], ce[k]);
        if (state0) state0[k] = dn0 <= 0.0 ? 2 : 0;
        if (!pen) continue;
        const double f = -(pen[2 * k] * dn0);
        const int64_t i = ci[k], j = cj[k];
        for (int r = 0; r < 6; ++r) Fc[6 * i + r] = Fc[6 * i + r] + f * e[12 * k + r];
        for (int r = 0; r < 6; ++r) Fc[6 * j + r] = Fc[6 * j + r] + f * g[12 * k + r];
    }
    return ORC_OK;
}

/*
 * O-13 (NEXT-3)  Contact transfer (§III.B: "each contact of the previous step will
 * search the contacts of the current step; if their contact data are the same, then the contact
 * status parameter ... of the previous step [is] transferred to the current step").  Reading N3-4:
 * the contact data of a record are its (vertex v, edge e) pair (global vertex / edge ids, stable
 * across steps); the transferred parameter is the open-close state.  For every current record k:
 * state[k] = prev_state[j] for the previous record j with the same (v, e), else init[k] (the
 * gap-based initial state of O-12).  Plain search over the previous records.  Returns the number of
 * matched records.
 */
int64_t orc_contact_transfer(int64_t n_prev, const int32_t *pv, const int32_t *pe, const int32_t *pstate,
                             int64_t n_cur, const int32_t *cv, const int32_t *ce, const int32_t *init,
                             int32_t *state) {
    int64_t matched = 0;
    for (int64_t k = 0; k < n_cur; ++k) {
        int32_t s = init[k];
        for (int64_t j = 0; j < n_prev; ++j)
            if (pv[j] == cv[k] && pe[j] == ce[k]) { s = pstate[j]; ++matched; break; }
        state[k] = s;
    }
    return matched;
}
