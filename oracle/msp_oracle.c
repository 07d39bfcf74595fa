/*
 * msp_oracle.c -- plain, slow, obviously correct CPU oracle for the three
 * CSR operations of Dalton, Baxter, Merrill, Olson, Garland, "Optimizing
 * Sparse Matrix Operations on GPUs using Merge Path" (IPDPS 2015).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.  It
 * shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_daltonbmog15_b200/csrc) and never includes its headers.
 *
 * Citations "P:n" are lines of PAPER.md (the paper text); readings of the
 * paper that it leaves open are numbered Z1..Z24 as in DESIGN.md §2.
 *
 * Build: gcc -O2 -ffp-contract=off -fPIC -shared (no FMA contraction, no
 * SIMD intrinsics), so each addition and multiplication rounds once, in the
 * order written here.
 *
 * Value type: dt == 0 -> float32 arrays, dt == 1 -> float64 arrays.
 *
 * Parity pins (tests/test_oracle_*.py, all -m "not gpu"): the paper's worked
 * example, dense brute force with integer values,
 * identities (A*I = A, A+0 = A, A+B = B+A, (A+B)x = Ax+Bx, (AB)x = A(Bx)),
 * Poisson closed forms (nnz, Nprods, row sums, A*A value set), scipy as a
 * third opinion on positive matrices.  No function here is "parity unpinned".
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

static double ld(const void *p, int dt, int64_t i)
{
    return dt ? ((const double *)p)[i] : (double)((const float *)p)[i];
}

static void st(void *p, int dt, int64_t i, double v)
{
    if (dt) ((double *)p)[i] = v;
    else ((float *)p)[i] = (float)v; /* one round-to-nearest-even, Z4 */
}

/* ------------------------------------------------------------------------
 * SpMV  y = A x   (scalar CSR)
 *
 * For each row i: acc = 0.0 (fp64); for j = rp[i] .. rp[i+1]-1 ascending,
 * acc += v[j] * x[c[j]]; y[i] = (T) acc.  fp32 inputs accumulate in fp64 and
 * round once on store (Z4).  An empty row gives +0.0 (Z6).  s[i] =
 * sum_j |v_j| |x_c_j| in fp64 is the tolerance scale (BJ:5).
 * `rows` selects a subset (nsel entries); rows == NULL means all m rows and
 * y/s are indexed by row; otherwise y/s are indexed by position in `rows`.
 * --------------------------------------------------------------------- */
void oracle_spmv(int32_t m, const int32_t *rp, const int32_t *col, const void *val,
                 const void *x, int dt, int64_t nsel, const int32_t *rows,
                 void *y, double *s)
{
    int64_t cnt = rows ? nsel : (int64_t)m;
    for (int64_t q = 0; q < cnt; ++q) {
        int64_t i = rows ? rows[q] : q;
        double acc = 0.0, sc = 0.0;
        for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
            double a = ld(val, dt, j);
            double xv = ld(x, dt, col[j]);
            acc += a * xv;
            sc += fabs(a) * fabs(xv);
        }
        st(y, dt, q, acc);
        if (s) s[q] = sc;
    }
}

/* ------------------------------------------------------------------------
 * SpAdd  C = A + B   (union of sorted (row,col) tuples P:538-550;
 * tuple order = Algorithm 1; sequential row-wise form P:504-508).
 *
 * For each row: two-pointer walk over A.col and B.col.  The smaller column is
 * emitted first; on a tie A's entry is emitted first (Alg. 1, Z3).  Adjacent
 * emitted entries with equal column are then summed left to right in the
 * value type T (Z2: for well-formed inputs this is exactly one (T)(a + b)).
 * The structure is the symbolic union; a cancellation a + b == 0 stays as an
 * explicit 0 (Z1).  Entries present in one input only are copied bit for bit.
 *
 * Counting pass: colC == NULL -> only rpC is written.  Returns nnzC.
 * rpC has m+1 entries written as int64 (caller checks the int32 range).
 * --------------------------------------------------------------------- */
static int64_t spadd_row(int64_t i, const int32_t *rpA, const int32_t *colA, const void *valA,
                         const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                         int32_t *colC, void *valC, int64_t out)
{
    int64_t a = rpA[i], ae = rpA[i + 1], b = rpB[i], be = rpB[i + 1];
    int64_t start = out;
    int32_t last_col = 0;
    double last_val = 0.0;
    int have = 0;
    while (a < ae || b < be) {
        int32_t c;
        double v;
        /* Alg. 1: take A when colA <= colB */
        if (b >= be || (a < ae && colA[a] <= colB[b])) {
            c = colA[a];
            v = ld(valA, dt, a);
            ++a;
        } else {
            c = colB[b];
            v = ld(valB, dt, b);
            ++b;
        }
        if (have && c == last_col) {
            /* duplicate key: reduce in T (single rounding per add) */
            if (dt) last_val = last_val + v;
            else last_val = (double)((float)last_val + (float)v);
        } else {
            if (have) {
                if (colC) { colC[out] = last_col; st(valC, dt, out, last_val); }
                ++out;
            }
            last_col = c;
            last_val = v;
            have = 1;
        }
    }
    if (have) {
        if (colC) { colC[out] = last_col; st(valC, dt, out, last_val); }
        ++out;
    }
    return out - start;
}

int64_t oracle_spadd(int32_t m, const int32_t *rpA, const int32_t *colA, const void *valA,
                     const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                     int64_t *rpC, int32_t *colC, void *valC)
{
    int64_t out = 0;
    rpC[0] = 0;
    for (int64_t i = 0; i < m; ++i) {
        out += spadd_row(i, rpA, colA, valA, rpB, colB, valB, dt, colC, valC, out);
        rpC[i + 1] = out;
    }
    return out;
}

/* Row subset: rows[q] -> entries written at offC[q] .. offC[q+1]; offC must be
 * the exclusive prefix of the counts (obtain with colC == NULL first). */
void oracle_spadd_rows(int64_t nsel, const int32_t *rows,
                       const int32_t *rpA, const int32_t *colA, const void *valA,
                       const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                       int64_t *offC, int32_t *colC, void *valC)
{
    int64_t out = 0;
    offC[0] = 0;
    for (int64_t q = 0; q < nsel; ++q) {
        out += spadd_row(rows[q], rpA, colA, valA, rpB, colB, valB, dt, colC, valC, out);
        offC[q + 1] = out;
    }
}

/* ------------------------------------------------------------------------
 * SpGEMM  C = A B   (Gustavson's sequential algorithm with an O(n)
 * dense accumulator, P:244-250 and ref [12]).
 *
 * Per row i of A: for each a_ik (k ascending), for each b_kj (j ascending):
 *   first touch of j in row i (mark[j] != i): mark, acc[j] = a*b,
 *     abs[j] = |a||b|, append j to `touched`;
 *   otherwise acc[j] += a*b, abs[j] += |a||b|.
 * All arithmetic in fp64 (fp32 products are exact in fp64, Z4).  Sort the
 * touched list ascending and emit (j, (T) acc[j]).  Membership is decided by
 * `mark` only, never by acc != 0, so structural zeros are kept (Z1).
 * nprods = sum over A's nonzeros of nnz(B row colA[j]).
 * --------------------------------------------------------------------- */
static int cmp_i32(const void *p, const void *q)
{
    int32_t a = *(const int32_t *)p, b = *(const int32_t *)q;
    return (a > b) - (a < b);
}

typedef struct {
    int64_t *mark;
    double *acc, *absacc;
    int32_t *touched;
} gus_ws;

static int gus_alloc(gus_ws *w, int32_t n)
{
    size_t nn = n > 0 ? (size_t)n : 1;
    w->mark = (int64_t *)malloc(nn * sizeof(int64_t));
    w->acc = (double *)malloc(nn * sizeof(double));
    w->absacc = (double *)malloc(nn * sizeof(double));
    w->touched = (int32_t *)malloc(nn * sizeof(int32_t));
    if (!w->mark || !w->acc || !w->absacc || !w->touched) return -1;
    for (size_t j = 0; j < nn; ++j) w->mark[j] = -1;
    return 0;
}

static void gus_free(gus_ws *w)
{
    free(w->mark); free(w->acc); free(w->absacc); free(w->touched);
}

/* one row; returns its nnz; writes entries at out.. when colC != NULL */
static int64_t gus_row(gus_ws *w, int64_t i, int64_t tag,
                       const int32_t *rpA, const int32_t *colA, const void *valA,
                       const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                       int32_t *colC, void *valC, double *scaleC, int64_t out, int64_t *nprods)
{
    int64_t nt = 0;
    for (int64_t ja = rpA[i]; ja < rpA[i + 1]; ++ja) {
        int32_t k = colA[ja];
        double a = ld(valA, dt, ja);
        for (int64_t jb = rpB[k]; jb < rpB[k + 1]; ++jb) {
            int32_t j = colB[jb];
            double b = ld(valB, dt, jb);
            double p = a * b;
            ++*nprods;
            if (w->mark[j] != tag) {
                w->mark[j] = tag;
                w->acc[j] = p;
                w->absacc[j] = fabs(a) * fabs(b);
                w->touched[nt++] = j;
            } else {
                w->acc[j] += p;
                w->absacc[j] += fabs(a) * fabs(b);
            }
        }
    }
    if (colC) {
        qsort(w->touched, (size_t)nt, sizeof(int32_t), cmp_i32);
        for (int64_t t = 0; t < nt; ++t) {
            int32_t j = w->touched[t];
            colC[out + t] = j;
            st(valC, dt, out + t, w->acc[j]);
            if (scaleC) scaleC[out + t] = w->absacc[j];
        }
    }
    return nt;
}

/* Full product.  colC == NULL -> symbolic count only.  Returns nnzC, or -1 on
 * allocation failure.  rpC is int64[m+1]. */
int64_t oracle_spgemm(int32_t m, int32_t n,
                      const int32_t *rpA, const int32_t *colA, const void *valA,
                      const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                      int64_t *rpC, int32_t *colC, void *valC, double *scaleC, int64_t *nprods)
{
    gus_ws w;
    if (gus_alloc(&w, n)) { gus_free(&w); return -1; }
    int64_t out = 0, np = 0;
    rpC[0] = 0;
    for (int64_t i = 0; i < m; ++i) {
        out += gus_row(&w, i, i, rpA, colA, valA, rpB, colB, valB, dt, colC, valC, scaleC, out, &np);
        rpC[i + 1] = out;
    }
    if (nprods) *nprods = np;
    gus_free(&w);
    return out;
}

/* Row subset (for sampled checks at full size).  offC is int64[nsel+1]: when
 * colC == NULL it receives the prefix of the per-row counts; when colC is
 * given, offC must hold that prefix already. Returns total entries or -1. */
int64_t oracle_spgemm_rows(int64_t nsel, const int32_t *rows, int32_t n,
                           const int32_t *rpA, const int32_t *colA, const void *valA,
                           const int32_t *rpB, const int32_t *colB, const void *valB, int dt,
                           int64_t *offC, int32_t *colC, void *valC, double *scaleC)
{
    gus_ws w;
    if (gus_alloc(&w, n)) { gus_free(&w); return -1; }
    int64_t out = 0, np = 0;
    offC[0] = 0;
    for (int64_t q = 0; q < nsel; ++q) {
        out += gus_row(&w, rows[q], q, rpA, colA, valA, rpB, colB, valB, dt, colC, valC, scaleC, out, &np);
        offC[q + 1] = out;
    }
    gus_free(&w);
    return out;
}

/* Nprods only: sum_j nnz(B row colA[j]). */
int64_t oracle_nprods(int64_t nnzA, const int32_t *colA, const int32_t *rpB)
{
    int64_t s = 0;
    for (int64_t j = 0; j < nnzA; ++j) s += (int64_t)rpB[colA[j] + 1] - rpB[colA[j]];
    return s;
}

/* ------------------------------------------------------------------------
 * Multi-GPU row split: rank r owns rows
 * [R_r, R_{r+1}) with R_r = lower_bound(rp, ceil(r * nnz / P)), R_0 = 0,
 * R_P = m.  Plain linear scan (the oracle is allowed to be slow).
 * --------------------------------------------------------------------- */
void oracle_row_split(int32_t m, const int32_t *rp, int32_t P, int32_t *starts)
{
    int64_t nnz = rp[m];
    starts[0] = 0;
    for (int32_t r = 1; r < P; ++r) {
        int64_t target = (r * nnz + P - 1) / P;
        int32_t i = 0;
        while (i < m && rp[i] < target) ++i;
        starts[r] = i;
    }
    starts[P] = m;
}

/* ---------------------------------------------------------------- set ops
 * Set operations on sorted key lists with duplicates (§8(f) f1):
 * each key carries a rank inside its run of equal keys, and the i-th copy of
 * a key in A matches the i-th copy in B ("key-rank pairs").  So for
 * a key with cA copies in A and cB in B the result holds
 *   union         max(cA, cB) copies: the min(cA, cB) matched from A, the rest
 *                 from the longer side;
 *   intersection  min(cA, cB) copies, from A;
 *   difference    max(cA - cB, 0) copies: A's copies of rank >= cB;
 *   sym. diff.    |cA - cB| copies from the longer side,
 * in ascending key order (the sequential two-pointer walk of Algorithm 1,
 * A first on ties).  Keys are unsigned 64-bit; values are opaque
 * 64-bit payloads that travel with their key (A's on a matched pair).
 * op: 0 union, 1 intersection, 2 difference (A - B), 3 symmetric difference.
 * C / Cv may be NULL (count only).  Returns the result size. */
int64_t oracle_set_op(int op, const uint64_t *A, const uint64_t *Av, int64_t nA,
                      const uint64_t *B, const uint64_t *Bv, int64_t nB, uint64_t *C, uint64_t *Cv)
{
    int64_t i = 0, j = 0, n = 0;
#define EMIT(K, V)                 \
    do {                           \
        if (C) C[n] = (K);         \
        if (Cv) Cv[n] = (V);       \
        ++n;                       \
    } while (0)
    while (i < nA || j < nB) {
        if (j >= nB || (i < nA && A[i] < B[j])) {           /* A only */
            if (op == 0 || op == 2 || op == 3) EMIT(A[i], Av ? Av[i] : 0);
            ++i;
        } else if (i >= nA || B[j] < A[i]) {                /* B only */
            if (op == 0 || op == 3) EMIT(B[j], Bv ? Bv[j] : 0);
            ++j;
        } else {                                            /* matched pair, same rank */
            if (op == 0 || op == 1) EMIT(A[i], Av ? Av[i] : 0);
            ++i;
            ++j;
        }
    }
#undef EMIT
    return n;
}
