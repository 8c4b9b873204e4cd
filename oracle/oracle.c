/*
 * oracle/oracle.c -- plain, slow, obviously-correct CPU oracle for MergePath-SpMM.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_ispass_shangndk23_b200/) never links, imports or calls it, and this
 * file shares no code, header, table or helper with the CUDA path.
 *
 * Paper: Shan, Gurevin, Nye, Ding, Khan, "MergePath-SpMM: Parallel Sparse
 * Matrix-Matrix Algorithm for Graph Neural Network Acceleration", ISPASS 2023.
 * Citations "P:<line>" refer to the extracted paper text, with the
 * section / algorithm named beside each.
 *
 * Precision: every floating-point accumulation is fp64 (the paper never states its
 * precision; reading R15).  fp32 x fp32 products are exact in
 * fp64, so O1 is the exact row-wise product up to the rounding of one fp64 sum.
 *
 * Functions (all plain loops; OpenMP only splits independent output rows):
 *   O1 oracle_csr_spmm_f64   C = A*B, row-wise product              (sec. II)
 *   O2 (same call)           Bnd = |A|*|B|, used by the tolerance    (north star)
 *   O3 oracle_dense_spmm_f64 dense brute force                       (textbook)
 *   O4 oracle_plan / oracle_merge_coord / oracle_partition           (Alg. 1)
 *      oracle_merge_coord64 / oracle_partition64: the same, int64 RP  (NEXT-4)
 *   O5 oracle_merge_walk     explicit merge of row ends and nnz      (Fig. 3 text)
 *   O6 oracle_alg2_emulate   serial Alg. 2 with write counters       (Alg. 2)
 *   O7 oracle_shard          merge-path shard bounds + tail rows     (north star stage 4)
 *   O9 oracle_xw_f64         the combination X*W (+ ReLU) of a GCN layer (NEXT-3)
 *
 * Parity pins for every function live in tests/test_oracle_pins.py (see DESIGN.md
 * "Oracle pins").  No function here is "parity unpinned".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define ORACLE_ABI 1

int oracle_abi_version(void) { return ORACLE_ABI; }

int oracle_num_threads(void)
{
#ifdef _OPENMP
    extern int omp_get_max_threads(void);
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ------------------------------------------------------------------------- */
/* O1 + O2: the row-wise product, P:41-43 (sec. II):                          */
/*     C[i,:] = sum_j A[i,j] * XW[j,:]                                        */
/* over the CSR entries of row i, RP[i] <= j < RP[i+1] (CSR: P:88).           */
/* Duplicated column indices are separate entries and are both summed.        */
/* rows == NULL -> all m rows, output row r at C + r*ldc.                     */
/* rows != NULL -> nrows listed rows, output row t at C + t*ldc.              */
/* bnd (may be NULL) receives sum_j |A[i,j]| * |XW[j,k]| in the same layout.  */
/* ------------------------------------------------------------------------- */
int oracle_csr_spmm_f64(int64_t m, const int32_t *RP, const int32_t *CP, const float *AV,
                        const float *XW, int64_t ldb, int32_t K,
                        const int64_t *rows, int64_t nrows,
                        double *C, double *bnd, int64_t ldc)
{
    int64_t count = rows ? nrows : m;
    if (count < 0 || K < 0) return 1;
    int64_t t;
#pragma omp parallel for schedule(dynamic, 256)
    for (t = 0; t < count; ++t) {
        int64_t i = rows ? rows[t] : t;
        double *c = C + t * ldc;
        double *b = bnd ? bnd + t * ldc : NULL;
        for (int32_t k = 0; k < K; ++k) {
            c[k] = 0.0;
            if (b) b[k] = 0.0;
        }
        if (i < 0 || i >= m) continue;
        for (int64_t j = RP[i]; j < RP[i + 1]; ++j) {
            double a = (double)AV[j];
            const float *xw = XW + (int64_t)CP[j] * ldb;
            for (int32_t k = 0; k < K; ++k) {
                c[k] += a * (double)xw[k];
                if (b) b[k] += fabs(a) * fabs((double)xw[k]);
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O3: dense brute force.  Materialise A as an m x n dense fp64 matrix,       */
/* summing duplicate entries, then the textbook triple loop C = A * XW.       */
/* Only for tiny inputs (the caller keeps m*n small).                         */
/* ------------------------------------------------------------------------- */
int oracle_dense_spmm_f64(int64_t m, int64_t n, const int32_t *RP, const int32_t *CP,
                          const float *AV, const float *XW, int64_t ldb, int32_t K,
                          double *C, int64_t ldc)
{
    if (m < 0 || n < 0 || K < 0) return 1;
    double *D = (double *)calloc((size_t)(m * n > 0 ? m * n : 1), sizeof(double));
    if (!D) return 2;
    for (int64_t i = 0; i < m; ++i)
        for (int64_t j = RP[i]; j < RP[i + 1]; ++j)
            D[i * n + CP[j]] += (double)AV[j];
    for (int64_t i = 0; i < m; ++i)
        for (int32_t k = 0; k < K; ++k) {
            double s = 0.0;
            for (int64_t c = 0; c < n; ++c)
                s += D[i * n + c] * (double)XW[c * ldb + k];
            C[i * ldc + k] = s;
        }
    free(D);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O4: Alg. 1.                                                      */
/*                                                                            */
/* Line 2: merge_items = total_nodes + number_of_nonzeros.                    */
/* Line 3: items per thread.  The printed formula is (M + P)/P     */
/*   reading R1 takes ceil(M/P) = (M + P - 1)/P (Merrill [18]).               */
/* sec. III-C: the number of threads is merge_items / cost, and   */
/*   when that is below a threshold the threshold is used (reading R13).      */
/* ------------------------------------------------------------------------- */
int oracle_plan(int64_t m, int64_t nnz, int64_t cost, int64_t min_parts,
                int64_t *num_parts, int64_t *items_per_part)
{
    if (m < 0 || nnz < 0 || cost < 1 || min_parts < 1) return 1;
    int64_t merge_items = m + nnz;                        /* Alg. 1 line 2 */
    int64_t threads = (merge_items + cost - 1) / cost;
    if (threads < min_parts) threads = min_parts;
    *num_parts = threads;
    *items_per_part = (merge_items + threads - 1) / threads; /* line 3, reading R1 */
    return 0;
}

/* Alg. 1 lines 6-7, BINARYSEARCH(cost, RP, nnz, total_nodes).                */
/* The paper's rule "first point on the diagonal where RP[i] > j" (with */
/* the strict comparison the Fig. 3 example uses; reading R4) is, in    */
/* 0-based coordinates (x = i - 1, y = j + 1), the point                      */
/*     x = max{ x in [max(0, d - nnz), min(d, m)] : x + RP[x] <= d },         */
/*     y = d - x,                                                             */
/* i.e. the row end of row x-1 is taken before nnz y when RP[x] == y          */
/* (reading R5).  Written as the plain bisection over that x range.           */
int oracle_merge_coord(const int32_t *RP, int64_t m, int64_t nnz, int64_t d,
                       int64_t *x_out, int64_t *y_out)
{
    if (d < 0 || d > m + nnz) return 1;
    int64_t lo = d - nnz > 0 ? d - nnz : 0;   /* lowest x on the diagonal  */
    int64_t hi = d < m ? d : m;               /* highest x on the diagonal */
    /* invariant: lo satisfies lo + RP[lo] <= d (RP[lo] <= nnz and d-lo <= ...)*/
    while (lo < hi) {
        int64_t mid = lo + (hi - lo + 1) / 2;
        if (mid + (int64_t)RP[mid] <= d) lo = mid;
        else hi = mid - 1;
    }
    *x_out = lo;
    *y_out = d - lo;
    return 0;
}

/* Alg. 1 lines 4-7 for every thread p = 0..P: diagonal                       */
/*   d_p = diag_begin + min(p * L, diag_end - diag_begin)                     */
/* (line 4 with the thread index p, lines 5 as the start of thread p+1,       */
/* reading R2).  Writes P+1 coordinates.                                      */
int oracle_partition(const int32_t *RP, int64_t m, int64_t nnz, int64_t diag_begin,
                     int64_t diag_end, int64_t P, int64_t L, int32_t *cx, int32_t *cy)
{
    if (P < 1 || L < 0 || diag_begin < 0 || diag_end < diag_begin || diag_end > m + nnz)
        return 1;
    for (int64_t p = 0; p <= P; ++p) {
        int64_t off = p * L;
        if (off > diag_end - diag_begin) off = diag_end - diag_begin;
        int64_t x, y;
        oracle_merge_coord(RP, m, nnz, diag_begin + off, &x, &y);
        cx[p] = (int32_t)x;
        cy[p] = (int32_t)y;
    }
    return 0;
}

/* O4 with 64-bit row offsets (NEXT-4: graphs with m + nnz >= 2^31).  The same */
/* closed form as oracle_merge_coord / oracle_partition, on int64 RP; rows     */
/* stay < 2^31 so x is returned as int32, y as int64.                          */
int oracle_merge_coord64(const int64_t *RP, int64_t m, int64_t nnz, int64_t d,
                         int64_t *x_out, int64_t *y_out)
{
    if (d < 0 || d > m + nnz) return 1;
    int64_t lo = d - nnz > 0 ? d - nnz : 0;
    int64_t hi = d < m ? d : m;
    while (lo < hi) {
        int64_t mid = lo + (hi - lo + 1) / 2;
        if (mid + RP[mid] <= d) lo = mid;
        else hi = mid - 1;
    }
    *x_out = lo;
    *y_out = d - lo;
    return 0;
}

int oracle_partition64(const int64_t *RP, int64_t m, int64_t nnz, int64_t diag_begin,
                       int64_t diag_end, int64_t P, int64_t L, int32_t *cx, int64_t *cy)
{
    if (P < 1 || L < 0 || diag_begin < 0 || diag_end < diag_begin || diag_end > m + nnz)
        return 1;
    for (int64_t p = 0; p <= P; ++p) {
        int64_t off = p * L;
        if (off > diag_end - diag_begin) off = diag_end - diag_begin;
        int64_t x, y;
        oracle_merge_coord64(RP, m, nnz, diag_begin + off, &x, &y);
        cx[p] = (int32_t)x;
        cy[p] = y;
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O5: the explicit merge walk of Fig. 3: start at (0,0); each      */
/* merge item either moves along x (processing a row end) or along y          */
/* (processing a non-zero).  A row end is taken as soon as all of its         */
/* non-zeros have been consumed (RP[x+1] <= y), else the next non-zero.       */
/* Records the coordinate after every item: xs/ys have M+1 entries.           */
/* ------------------------------------------------------------------------- */
int oracle_merge_walk(const int32_t *RP, int64_t m, int64_t nnz, int32_t *xs, int32_t *ys)
{
    int64_t x = 0, y = 0, M = m + nnz;
    xs[0] = 0;
    ys[0] = 0;
    for (int64_t d = 1; d <= M; ++d) {
        if (x < m && (int64_t)RP[x + 1] <= y) x += 1;   /* row end of row x */
        else y += 1;                                     /* non-zero y       */
        xs[d] = (int32_t)x;
        ys[d] = (int32_t)y;
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O6: Alg. 2, serial fp64 emulation, reconstructed from the text */
/* of sec. III-B (the listing at P:104-119 is garbled; reading R8).           */
/* C is read-modify-written: the caller prefills it (zeros for the result,    */
/* garbage to see which rows are touched only by "atomic" updates).           */
/* n_atomic counts the atomic row updates (lines 5, 9, 13), n_regular the     */
/* plain complete-row stores (line 15): the write statistic of Fig. 5.        */
/* ------------------------------------------------------------------------- */
static void row_partial_sum(const int32_t *CP, const float *AV, const float *XW, int64_t ldb,
                            int32_t K, int64_t j0, int64_t j1, double *T)
{
    for (int32_t k = 0; k < K; ++k) T[k] = 0.0;
    for (int64_t j = j0; j < j1; ++j)
        for (int32_t k = 0; k < K; ++k)
            T[k] += (double)AV[j] * (double)XW[(int64_t)CP[j] * ldb + k];
}

int oracle_alg2_emulate(int64_t m, const int32_t *RP, const int32_t *CP, const float *AV,
                        const float *XW, int64_t ldb, int32_t K,
                        const int32_t *cx, const int32_t *cy, int64_t P,
                        double *C, int64_t ldc, int64_t *n_atomic, int64_t *n_regular)
{
    double *T = (double *)malloc(sizeof(double) * (size_t)(K > 0 ? K : 1));
    if (!T) return 2;
    int64_t na = 0, nr = 0;
    for (int64_t p = 0; p < P; ++p) {
        int64_t start_row = cx[p], start_y = cy[p];
        int64_t end_row = cx[p + 1], end_y = cy[p + 1];
        /* sec. III-B: the start row is partial iff the start coordinate's */
        /* non-zero id differs from the row offset of the start row; same for end.*/
        int start_partial = start_row < m && start_y != RP[start_row];
        int end_partial = end_row < m && end_y != RP[end_row];
        if (start_partial) {                                   /* line 2  */
            if (start_row == end_row) {                        /* line 3  */
                row_partial_sum(CP, AV, XW, ldb, K, start_y, end_y, T);  /* line 4 */
                for (int32_t k = 0; k < K; ++k) C[start_row * ldc + k] += T[k]; /* 5 */
                na += 1;
                continue;                                      /* line 6  */
            }
            row_partial_sum(CP, AV, XW, ldb, K, start_y, RP[start_row + 1], T); /* 8 */
            for (int32_t k = 0; k < K; ++k) C[start_row * ldc + k] += T[k];  /* line 9 */
            na += 1;
            start_row += 1;                                    /* line 10 */
        }
        if (end_partial) {                                     /* line 11 */
            row_partial_sum(CP, AV, XW, ldb, K, RP[end_row], end_y, T);      /* 12 */
            for (int32_t k = 0; k < K; ++k) C[end_row * ldc + k] += T[k];    /* 13 */
            na += 1;
        }
        for (int64_t r = start_row; r < end_row; ++r) {        /* line 14, [start,end) */
            row_partial_sum(CP, AV, XW, ldb, K, RP[r], RP[r + 1], T);       /* 15 */
            for (int32_t k = 0; k < K; ++k) C[r * ldc + k] = T[k];
            nr += 1;
        }
    }
    free(T);
    if (n_atomic) *n_atomic = na;
    if (n_regular) *n_regular = nr;
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O7: merge-path sharding over G devices (north-star stage 4; not in the     */
/* paper).  Shard g covers diagonals [D_g, D_{g+1}), D_g = min(g*ceil(M/G),M) */
/* (Alg. 1 lines 3-4 applied with G "threads"); (X_g, Y_g) by O4.  Shard g   */
/* consumes the row ends of rows X_g .. X_{g+1}-1, so it owns those rows.     */
/* Its tail row is X_{g+1} when that row is cut (Y_{g+1} > RP[X_{g+1}]), else */
/* -1.                                                                        */
/* ------------------------------------------------------------------------- */
int oracle_shard(const int32_t *RP, int64_t m, int64_t nnz, int32_t G,
                 int32_t *X, int32_t *Y, int32_t *tail_rows)
{
    if (G < 1) return 1;
    int64_t M = m + nnz;
    int64_t per = (M + G - 1) / G;
    for (int32_t g = 0; g <= G; ++g) {
        int64_t d = (int64_t)g * per;
        if (d > M) d = M;
        int64_t x, y;
        oracle_merge_coord(RP, m, nnz, d, &x, &y);
        X[g] = (int32_t)x;
        Y[g] = (int32_t)y;
    }
    for (int32_t g = 0; g < G; ++g) {
        int64_t r = X[g + 1];
        tail_rows[g] = (r < m && (int64_t)Y[g + 1] > (int64_t)RP[r]) ? (int32_t)r : -1;
    }
    return 0;
}

/* Oracle for one shard's local output: rows [X_g, X_{g+1}) summed over the   */
/* shard's non-zeros only, and the shard's tail vector (row X_{g+1}'s sum     */
/* over non-zeros [max(Y_g, RP[X_{g+1}]), Y_{g+1})).  Plain sums, fp64.       */
int oracle_shard_local(int64_t m, const int32_t *RP, const int32_t *CP, const float *AV,
                       const float *XW, int64_t ldb, int32_t K,
                       int64_t Xg, int64_t Yg, int64_t Xg1, int64_t Yg1,
                       double *C_local, int64_t ldc, double *tail)
{
    for (int64_t r = Xg; r < Xg1; ++r) {
        int64_t j0 = RP[r] > Yg ? RP[r] : Yg;
        int64_t j1 = RP[r + 1] < Yg1 ? RP[r + 1] : Yg1;
        row_partial_sum(CP, AV, XW, ldb, K, j0, j1 > j0 ? j1 : j0, C_local + (r - Xg) * ldc);
    }
    for (int32_t k = 0; k < K; ++k) tail[k] = 0.0;
    if (Xg1 < m && Yg1 > RP[Xg1]) {
        int64_t j0 = RP[Xg1] > Yg ? RP[Xg1] : Yg;
        row_partial_sum(CP, AV, XW, ldb, K, j0, Yg1, tail);
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O9: the GCN layer's combination and activation around the aggregation,     */
/* P:37-39 (sec. II): H' = sigma(A * (X * W)) with sigma = ReLU.  This is the */
/* X * W (combination) half and the activation, in fp64:                      */
/*     out[i, j] = sum_{f < F} X[i, f] * W[f, j]      (relu: max(out, 0))     */
/* X: n x F row-major (ldx), W: F x N row-major (ldw) -- W itself, not its    */
/* transpose -- out: n x N (ldo).  Inputs are fp32 (bf16 values are exact in  */
/* fp32); products are exact in fp64.  OpenMP over output rows only.         */
/* ------------------------------------------------------------------------- */
int oracle_xw_f64(int64_t n, int64_t F, int32_t N, const float *X, int64_t ldx,
                  const float *W, int64_t ldw, int32_t relu, double *out, int64_t ldo)
{
    if (n < 0 || F < 0 || N < 0) return 1;
    int64_t i;
#pragma omp parallel for schedule(static)
    for (i = 0; i < n; ++i) {
        double *o = out + i * ldo;
        for (int32_t j = 0; j < N; ++j) o[j] = 0.0;
        for (int64_t f = 0; f < F; ++f) {
            const double x = (double)X[i * ldx + f];
            const float *w = W + f * ldw;
            for (int32_t j = 0; j < N; ++j) o[j] += x * (double)w[j];
        }
        if (relu)
            for (int32_t j = 0; j < N; ++j) o[j] = o[j] > 0.0 ? o[j] : 0.0;
    }
    return 0;
}
