/*
 * ted_matfree.c -- O2: matrix-free fp64 CPU oracle of Algorithm 1 (TED),
 * plain C + OpenMP.  TEST INFRASTRUCTURE ONLY: loaded by tests/ and bench.py's
 * cpu_baseline / --impl reference legs through oracle/matfree.py; never by the
 * product path.  Shares no code, header or constant with
 * paper_conf_date_sunbg021_b200/.
 *
 * Why a second C oracle: the dense one (ted_dense.c) holds K in fp64, 8 N^2
 * bytes -- 34 GB at N = 65536.  This one holds O(N m) numbers and recomputes
 * rows of K from the features, so it runs Alg. 1 at any N.
 *
 * What it computes.  Alg. 1 deflates K once per pick
 * (l.5: K <- K - K_x K_x^T / (k(x,x) + mu)).  After the picks S the deflated
 * matrix has the closed form (pin C2, checked against the literal deflation
 * in tests/test_oracle_pins.py)
 *
 *     K^(S) = K - L L^T,   L = [l_1 ... l_t] (N x t),
 *     l_t   = K^(S_{t-1})_{:,s_t} / sqrt(K^(S_{t-1})_{s_t s_t} + mu)
 *           = (K_{:,s_t} - L L_{s_t}^T) / sqrt(K_{s_t s_t} - |L_{s_t}|^2 + mu)
 *
 * (l.5 itself: K - K_x K_x^T / c = K - l l^T with l = K_x / sqrt(c)).  The
 * l.3 quantities of every column v then follow from K (never stored) and L:
 *
 *     ||K^(S)_{:v}||^2 = g_v - 2 L_v . A_v + L_v^T C L_v,
 *         g_v = ||K_{:v}||^2,  A = K L (N x t),  C = L^T L (t x t)
 *     K^(S)_{vv}       = K_vv - |L_v|^2
 *     score_v          = ||K^(S)_{:v}||^2 / (K^(S)_{vv} + mu)
 *
 * Per step (in the paper's order): l.3 scores of all v and the lowest-index
 * argmax over unselected v (readings A4, A5), l.4 X = X u x, l.5 as the new
 * factor column l and its mat-vec K l (rows of K recomputed from X, fp64,
 * direct-difference RBF as reading A1; or the test-only linear kernel).
 * OpenMP splits independent rows; every sum runs sequentially in its index.
 * Cost: (m + 1) passes over the N^2 kernel values, memory (2 m + 4) N doubles.
 * When the caller grants cache_bytes >= 8 N^2 (host RAM permitting), the
 * values k(x_i, x_j) computed in the first pass are kept and re-read by the
 * later passes instead of being recomputed -- the same numbers, so the result
 * is bitwise the same; it only trades memory for the m recomputations.  With
 * between 4 N (N + 1) and 8 N^2 bytes only the upper triangle j >= i is kept
 * (K is symmetric) and the mat-vec K l runs over it once: row i adds
 * K_ij l_j (j >= i) in order and scatters K_ij l_i into a per-thread copy of
 * the result for j > i; the copies are added in thread order (a fixed order
 * for a fixed thread count; the sums differ from the row order only in
 * rounding).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

int matfree_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* k(x_i, x_j) in fp64 (reading A1: exp(-gamma sum_k (x_ik - x_jk)^2); linear: x_i . x_j) */
static double kij(const double* X, int32_t d, int64_t i, int64_t j, double gamma, int linear) {
    const double* a = X + i * d;
    const double* b = X + j * d;
    double s = 0.0;
    if (linear) {
        for (int32_t k = 0; k < d; ++k) s += a[k] * b[k];
        return s;
    }
    for (int32_t k = 0; k < d; ++k) {
        const double diff = a[k] - b[k];
        s += diff * diff;
    }
    return exp(-gamma * s);
}

/*
 * TED(V, mu, m) on feature rows X (N x d fp32).  forced (nullable): s_t per
 * step (teacher forcing); the oracle still reports its own argmax.  Outputs
 * (length m): idx = s_t taken, score = fp64 score of s_t, argmax = own
 * lowest-index argmax over unselected, max_score = its score, gap =
 * (top1 - top2) / top1 over unselected (INFINITY when one point is left).
 * all_scores (nullable, m x N): every score of every step (-INFINITY for
 * selected points).  Returns 0, or -1 on bad input / a forced index selected
 * twice / allocation failure.
 */
int matfree_ted(const float* Xf, int64_t N, int32_t d, double gamma, int32_t linear, double mu, int32_t m,
                const int64_t* forced, int64_t* idx, double* score_out, int64_t* argmax_out, double* max_out,
                double* gap_out, double* all_scores, int64_t cache_bytes) {
    if (N < 1 || d < 1 || m < 1 || m > N || !(mu > 0)) return -1;
    double* Kc = NULL;                                             /* optional cache of the N^2 values */
    double* Ku = NULL;                                             /* or of the upper triangle, row-packed */
    double* qt = NULL;                                             /* per-thread scatter targets (Ku) */
    int nthr = matfree_num_threads();
    if (cache_bytes > 0 && (double)N * (double)N * 8.0 <= (double)cache_bytes)
        Kc = (double*)malloc(sizeof(double) * (size_t)N * (size_t)N);
    else if (cache_bytes > 0 && (double)N * (double)(N + 1) * 4.0 + 8.0 * nthr * N <= (double)cache_bytes) {
        Ku = (double*)malloc(sizeof(double) * (size_t)N * (size_t)(N + 1) / 2);
        qt = Ku ? (double*)malloc(sizeof(double) * (size_t)nthr * (size_t)N) : NULL;
        if (!qt) { free(Ku); Ku = NULL; }
    }
    double* X = (double*)malloc(sizeof(double) * (size_t)N * d);
    double* L = (double*)calloc((size_t)N * m, sizeof(double));    /* column t at L + t N */
    double* A = (double*)calloc((size_t)N * m, sizeof(double));    /* A = K L, same layout */
    double* C = (double*)calloc((size_t)m * m, sizeof(double));    /* C = L^T L */
    double* g = (double*)malloc(sizeof(double) * (size_t)N);
    double* kd = (double*)malloc(sizeof(double) * (size_t)N);      /* K_vv */
    double* score = (double*)malloc(sizeof(double) * (size_t)N);
    unsigned char* sel = (unsigned char*)calloc((size_t)N, 1);
    int rc = 0;
    if (!X || !L || !A || !C || !g || !kd || !score || !sel) { rc = -1; goto done; }
    for (int64_t q = 0; q < N * d; ++q) X[q] = (double)Xf[q];

    /* Alg. 1 l.1 (implicitly): g_v = ||K_:v||^2 and K_vv.  Column v of K equals
     * row v exactly (the direct-difference form is symmetric in its operands). */
    #pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < N; ++v) {
        double s = 0.0;
        double* up = Ku ? Ku + (size_t)v * N - (size_t)v * (v - 1) / 2 - (size_t)v : NULL;   /* up[j], j >= v */
        for (int64_t i = 0; i < N; ++i) {
            const double k = kij(X, d, v, i, gamma, linear);
            if (Kc) Kc[(size_t)v * N + i] = k;
            if (up && i >= v) up[i] = k;
            s += k * k;
        }
        g[v] = s;
        kd[v] = kij(X, d, v, v, gamma, linear);
    }

    for (int32_t t = 0; t < m; ++t) {
        /* l.3: score_v = ||K^(S)_:v||^2 / (K^(S)_vv + mu) for every v */
        #pragma omp parallel for schedule(static)
        for (int64_t v = 0; v < N; ++v) {
            double la = 0.0, lcl = 0.0, ll = 0.0;
            for (int32_t a = 0; a < t; ++a) {
                const double lva = L[(size_t)a * N + v];
                la += lva * A[(size_t)a * N + v];
                ll += lva * lva;
                double cl = 0.0;
                for (int32_t b = 0; b < t; ++b) cl += C[(size_t)a * m + b] * L[(size_t)b * N + v];
                lcl += lva * cl;
            }
            const double n2 = g[v] - 2.0 * la + lcl;
            score[v] = n2 / (kd[v] - ll + mu);
        }
        int64_t best = -1;
        double top1 = -INFINITY, top2 = -INFINITY;
        for (int64_t v = 0; v < N; ++v) {                  /* readings A4, A5 */
            if (sel[v]) continue;
            if (score[v] > top1) { top2 = top1; top1 = score[v]; best = v; }
            else if (score[v] > top2) { top2 = score[v]; }
        }
        if (all_scores)
            for (int64_t v = 0; v < N; ++v) all_scores[(size_t)t * N + v] = sel[v] ? -INFINITY : score[v];
        const int64_t s = forced ? forced[t] : best;
        if (s < 0 || s >= N || sel[s]) { rc = -1; goto done; }
        idx[t] = s;
        score_out[t] = score[s];
        argmax_out[t] = best;
        max_out[t] = top1;
        gap_out[t] = (N - t >= 2) ? (top1 > 0 ? (top1 - top2) / top1 : 0.0) : INFINITY;
        sel[s] = 1;                                        /* l.4 */
        if (t + 1 == m) break;                             /* the last l.5 cannot change X */

        /* l.5: l = (K_:s - L L_s^T) / sqrt(K_ss - |L_s|^2 + mu) */
        double ls2 = 0.0;
        for (int32_t a = 0; a < t; ++a) ls2 += L[(size_t)a * N + s] * L[(size_t)a * N + s];
        const double rt = sqrt(kd[s] - ls2 + mu);
        double* l = L + (size_t)t * N;
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < N; ++i) {
            double v = Kc ? Kc[(size_t)i * N + s]
                     : Ku ? Ku[(size_t)(i < s ? i : s) * N - (size_t)(i < s ? i : s) * ((i < s ? i : s) - 1) / 2
                               - (size_t)(i < s ? i : s) + (size_t)(i < s ? s : i)]
                          : kij(X, d, i, s, gamma, linear);
            for (int32_t a = 0; a < t; ++a) v -= L[(size_t)a * N + i] * L[(size_t)a * N + s];
            l[i] = v / rt;
        }
        /* A gains K l (rows of K recomputed); C gains L^T l */
        double* Al = A + (size_t)t * N;
        if (Ku) {                                          /* upper triangle: row sums + scattered columns */
            memset(qt, 0, sizeof(double) * (size_t)nthr * (size_t)N);
            #pragma omp parallel num_threads(nthr)
            {
#ifdef _OPENMP
                double* q = qt + (size_t)omp_get_thread_num() * N;
#else
                double* q = qt;
#endif
                #pragma omp for schedule(static, 16)
                for (int64_t i = 0; i < N; ++i) {
                    const double* up = Ku + (size_t)i * N - (size_t)i * (i - 1) / 2 - (size_t)i;
                    const double li = l[i];
                    double acc = 0.0;
                    for (int64_t j = i; j < N; ++j) {
                        acc += up[j] * l[j];
                        if (j > i) q[j] += up[j] * li;
                    }
                    Al[i] = acc;
                }
            }
            #pragma omp parallel for schedule(static)
            for (int64_t i = 0; i < N; ++i) {
                double a = Al[i];
                for (int th = 0; th < nthr; ++th) a += qt[(size_t)th * N + i];
                Al[i] = a;
            }
        } else {
            #pragma omp parallel for schedule(static)
            for (int64_t i = 0; i < N; ++i) {
                double acc = 0.0;
                if (Kc) {
                    const double* row = Kc + (size_t)i * N;
                    for (int64_t j = 0; j < N; ++j) acc += row[j] * l[j];
                } else {
                    for (int64_t j = 0; j < N; ++j) acc += kij(X, d, i, j, gamma, linear) * l[j];
                }
                Al[i] = acc;
            }
        }
        for (int32_t a = 0; a <= t; ++a) {
            double c = 0.0;
            for (int64_t i = 0; i < N; ++i) c += L[(size_t)a * N + i] * l[i];
            C[(size_t)a * m + t] = c;
            C[(size_t)t * m + a] = c;
        }
    }
done:
    free(Kc); free(Ku); free(qt); free(X); free(L); free(A); free(C); free(g); free(kd); free(score); free(sel);
    return rc;
}
