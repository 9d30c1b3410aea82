/*
 * ted_dense.c -- fp64 CPU oracle of Algorithm 1 (TED), plain C + OpenMP.
 * TEST INFRASTRUCTURE ONLY: loaded by tests/ and bench.py's cpu_baseline /
 * --impl reference legs through oracle/dense.py; never by the product path.
 * Shares no code, header or constant with paper_conf_date_sunbg021_b200/.
 *
 * It is the same literal algorithm as oracle/ted.py, written in C so that the
 * oracle finishes the bench-size batches (N = 16384, K = 2 GiB fp64) in
 * seconds.  Steps, in the paper's order (Alg. 1):
 *   l.1  K <- K_VV            oracle_gram(): K_ij = exp(-gamma sum_k (x_ik-x_jk)^2)
 *   l.3  x = argmax_v ||K_v||^2 / (k(v,v)+mu)   column norms, then scores,
 *                              then the lowest-index max over unselected v
 *   l.4  X = X u x
 *   l.5  K = K - K_x K_x^T / (k(x,x)+mu)   (whole matrix, reading A7)
 * OpenMP only splits independent columns (l.3) / rows (l.1, l.5); each sum
 * runs sequentially in its index, as written.  No blocking or fusion.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Alg. 1 l.1 with the RBF reading A1: K is N x N row-major fp64. */
void oracle_gram(const float* X, int64_t N, int32_t d, double gamma, double* K) {
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
        for (int64_t j = 0; j < N; ++j) {
            double s = 0.0;
            for (int32_t k = 0; k < d; ++k) {
                double diff = (double)X[i * d + k] - (double)X[j * d + k];
                s += diff * diff;
            }
            K[i * N + j] = exp(-gamma * s);
        }
    }
}

/* Alg. 1 l.3: score_v = ||K_v||^2 / (k(v,v) + mu) for every column v. */
static void oracle_scores(const double* K, int64_t N, double mu, double* score) {
    #pragma omp parallel
    {
#ifdef _OPENMP
        int nt = omp_get_num_threads(), tid = omp_get_thread_num();
#else
        int nt = 1, tid = 0;
#endif
        int64_t j0 = N * tid / nt, j1 = N * (tid + 1) / nt;
        for (int64_t j = j0; j < j1; ++j) score[j] = 0.0;
        for (int64_t i = 0; i < N; ++i) {           /* sum over rows, in order */
            const double* row = K + i * N;
            for (int64_t j = j0; j < j1; ++j) score[j] += row[j] * row[j];
        }
        for (int64_t j = j0; j < j1; ++j) score[j] = score[j] / (K[j * N + j] + mu);
    }
}

/* Alg. 1 l.5: K = K - K_x K_x^T / (k(x,x) + mu), with K_x copied first. */
static void oracle_deflate(double* K, int64_t N, int64_t s, double mu, double* Kx) {
    for (int64_t i = 0; i < N; ++i) Kx[i] = K[i * N + s];
    const double c = Kx[s] + mu;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
        double* row = K + i * N;
        const double a = Kx[i];
        for (int64_t j = 0; j < N; ++j) row[j] = row[j] - a * Kx[j] / c;
    }
}

/*
 * Alg. 1 on a K already built (consumed in place).  forced (nullable) gives
 * s_t per step (teacher forcing); the oracle still reports its own argmax.
 * Outputs per step t (arrays of length m): idx = s_t taken, score = fp64
 * score of s_t, argmax = own lowest-index argmax over unselected,
 * max_score = its score, gap = (top1-top2)/top1 over unselected (inf if
 * only one point is left).  Returns 0, or -1 on bad input / a forced index
 * selected twice.
 */
int oracle_ted_on_matrix(double* K, int64_t N, double mu, int32_t m,
                         const int64_t* forced, int64_t* idx, double* score_out,
                         int64_t* argmax_out, double* max_out, double* gap_out) {
    if (N < 1 || m < 1 || m > N || !(mu > 0)) return -1;
    double* score = (double*)malloc(sizeof(double) * N);
    double* Kx = (double*)malloc(sizeof(double) * N);
    unsigned char* sel = (unsigned char*)calloc((size_t)N, 1);
    if (!score || !Kx || !sel) { free(score); free(Kx); free(sel); return -1; }
    int rc = 0;
    for (int32_t t = 0; t < m; ++t) {
        oracle_scores(K, N, mu, score);
        int64_t best = -1; double top1 = -INFINITY, top2 = -INFINITY;
        for (int64_t v = 0; v < N; ++v) {                  /* reading A4, A5 */
            if (sel[v]) continue;
            if (score[v] > top1) { top2 = top1; top1 = score[v]; best = v; }
            else if (score[v] > top2) { top2 = score[v]; }
        }
        int64_t s = forced ? forced[t] : best;
        if (s < 0 || s >= N || sel[s]) { rc = -1; break; }
        idx[t] = s;
        score_out[t] = score[s];
        argmax_out[t] = best;
        max_out[t] = top1;
        gap_out[t] = (N - t >= 2) ? (top1 > 0 ? (top1 - top2) / top1 : 0.0) : INFINITY;
        sel[s] = 1;                                       /* l.4 */
        oracle_deflate(K, N, s, mu, Kx);                  /* l.5 */
    }
    free(score); free(Kx); free(sel);
    return rc;
}

/* TED(V, mu, m) from feature rows: l.1 then l.2-7.  K is caller scratch N*N. */
int oracle_ted(const float* X, int64_t N, int32_t d, double gamma, double mu,
               int32_t m, const int64_t* forced, double* K, int64_t* idx,
               double* score_out, int64_t* argmax_out, double* max_out,
               double* gap_out) {
    oracle_gram(X, N, d, gamma, K);
    return oracle_ted_on_matrix(K, N, mu, m, forced, idx, score_out, argmax_out,
                                max_out, gap_out);
}
