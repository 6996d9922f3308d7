/*
 * sw_oracle.c — TEST INFRASTRUCTURE ONLY.  The plain, slow, obviously-correct CPU oracle
 * for the hot path.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  It shares no code, header, table or
 * helper with the CUDA path (paper_conf_ipps_hainscobr11_b200/csrc).
 *
 * What it computes (§II, Eq.(1); dependencies of Fig.1, L14):
 *
 *   E[i][j] = max( E[i][j-1] - sigma , H[i][j-1] - rho )
 *   F[i][j] = max( F[i-1][j] - sigma , H[i-1][j] - rho )
 *   H[i][j] = max( 0 , E[i][j] , F[i][j] , H[i-1][j-1] + w(q_i, d_j) )
 *   boundary: H[0][j] = H[i][0] = 0 ; E[i][0] = F[0][j] = -inf   (reading c4)
 *   score(q, d) = max over all H[i][j]  ("The optimal alignment score is given by the
 *                 maximum score in table H", L12), which is >= 0 because of the clamp.
 *
 * Rows i = 1..m index the query q, columns j = 1..n the database sequence d (reading c1);
 * w = matrix[q_i * A + d_j] (row = query symbol, reading c5).  Score-only evaluation in
 * linear space ("when only the optimal score is required, the space complexity is
 * linear", L14): one row of H and F plus a scalar E, swept row by row in the order of
 * Eq.(1).  int32 arithmetic (reading c11); -inf is INT32_MIN/4 so that "-inf - sigma"
 * cannot wrap for any accepted sigma.
 *
 * Pinned (tests/test_oracle_pins.py) against: the full m x n tables written out in
 * Python; brute-force enumeration of every local alignment; the cubic
 * Waterman-Smith-Beyer general-gap DP; Durbin et al. Fig.2.5 (score 28); LCS, longest
 * common substring and ungapped Kadane special cases; invariants.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define ORACLE_NEG_INF (INT32_MIN / 4)

static inline int32_t max2(int32_t a, int32_t b) { return a > b ? a : b; }

/* Eq.(1) for one (q, d) pair.  H and F are caller scratch of n+1 int32 each. */
static int32_t sw_pair(const uint8_t* q, int32_t m, const uint8_t* d, int64_t n,
                       const int8_t* W, int32_t A, int32_t rho, int32_t sigma,
                       int32_t* H, int32_t* F) {
    int32_t best = 0;
    for (int64_t j = 0; j <= n; ++j) { H[j] = 0; F[j] = ORACLE_NEG_INF; }  /* row 0 */
    for (int32_t i = 1; i <= m; ++i) {
        const int8_t* wrow = W + (int64_t)q[i - 1] * A;
        int32_t E = ORACLE_NEG_INF;   /* E[i][0] */
        int32_t Hdiag = H[0];         /* H[i-1][0] = 0 */
        H[0] = 0;                     /* H[i][0] */
        for (int64_t j = 1; j <= n; ++j) {
            /* here H[j] still holds H[i-1][j] and H[j-1] already holds H[i][j-1] */
            E = max2(E - sigma, H[j - 1] - rho);                 /* E[i][j] */
            F[j] = max2(F[j] - sigma, H[j] - rho);              /* F[i][j] */
            int32_t h = Hdiag + (int32_t)wrow[d[j - 1]];        /* H[i-1][j-1] + w(q_i, d_j) */
            h = max2(h, E);
            h = max2(h, F[j]);
            h = max2(h, 0);
            Hdiag = H[j];                                        /* H[i-1][j] is the next diag */
            H[j] = h;                                            /* H[i][j] */
            best = max2(best, h);
        }
    }
    return best;
}

typedef struct { int64_t len; int64_t idx; } len_idx;
static int cmp_desc(const void* a, const void* b) {
    const len_idx* x = (const len_idx*)a; const len_idx* y = (const len_idx*)b;
    if (x->len != y->len) return x->len > y->len ? -1 : 1;
    return x->idx < y->idx ? -1 : (x->idx > y->idx);
}

/* Scores of query q against every sequence of a CSR database; out[k] for sequence k.
 * threads <= 0 means "OpenMP default".  Returns 0, or -1 on bad arguments / OOM. */
int sw_oracle_scores(const uint8_t* q, int32_t m, const int8_t* W, int32_t A,
                     int32_t rho, int32_t sigma, const uint8_t* res, const int64_t* off,
                     int64_t N, int32_t threads, int32_t* out) {
    if (!q || !W || !off || !out || m < 0 || A <= 0 || rho < 0 || sigma < 0 || N < 0) return -1;
    if (N == 0) return 0;
    len_idx* order = (len_idx*)malloc(sizeof(len_idx) * (size_t)N);
    if (!order) return -1;
    int64_t maxn = 0;
    for (int64_t k = 0; k < N; ++k) {
        order[k].len = off[k + 1] - off[k];
        order[k].idx = k;
        if (order[k].len > maxn) maxn = order[k].len;
    }
    qsort(order, (size_t)N, sizeof(len_idx), cmp_desc);   /* longest first: load balance only */
    int failed = 0;
#ifdef _OPENMP
    if (threads > 0) omp_set_num_threads(threads);
#endif
#pragma omp parallel
    {
        int32_t* H = (int32_t*)malloc(sizeof(int32_t) * (size_t)(maxn + 1));
        int32_t* F = (int32_t*)malloc(sizeof(int32_t) * (size_t)(maxn + 1));
        if (!H || !F) {
#pragma omp atomic write
            failed = 1;
        } else {
#pragma omp for schedule(dynamic, 1)
            for (int64_t t = 0; t < N; ++t) {
                int64_t k = order[t].idx;
                out[k] = sw_pair(q, m, res + off[k], off[k + 1] - off[k], W, A, rho, sigma, H, F);
            }
        }
        free(H); free(F);
    }
    free(order);
    return failed ? -1 : 0;
}

/* Single pair, for tests. */
int32_t sw_oracle_pair(const uint8_t* q, int32_t m, const uint8_t* d, int64_t n,
                       const int8_t* W, int32_t A, int32_t rho, int32_t sigma) {
    int32_t* H = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n + 1));
    int32_t* F = (int32_t*)malloc(sizeof(int32_t) * (size_t)(n + 1));
    int32_t s = (H && F) ? sw_pair(q, m, d, n, W, A, rho, sigma, H, F) : -1;
    free(H); free(F);
    return s;
}

int sw_oracle_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
