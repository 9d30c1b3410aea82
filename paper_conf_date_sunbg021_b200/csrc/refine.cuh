// refine.cuh -- K4: near-tie refinement of the greedy pick (SURVEY.md Sec.
// 2.3 K4, Sec. 8(c) "numerics vs the 1e-6 gap rule").
//
// The fp32 path's scores carry ~1e-6 relative error (mostly from the fp32
// Gram entries), so two candidates whose exact scores differ by less than a
// few 1e-6 may be ordered wrongly.  Every finalize kernel therefore also
// emits its CTA's top-2 keys; after a TED one check kernel finds the steps
// whose second-best fp32 score is within tau of the best and lists all
// candidates within tau.  For such a step the host recomputes the
// candidates' scores in fp64 from the features -- the closed form of the
// deflation after the selected set S (pin C2):
//
//   K^(S)_:c = K_:c - K_:S (K_SS + mu I)^-1 K_Sc,
//   score_c = ||K^(S)_:c||^2 / (K^(S)_cc + mu)
//
// and takes the exact argmax (ties: lowest index).  If it differs from the
// GPU's pick, the TED is re-run with the corrected prefix forced.
//
// Completeness.  Each score unit (a CTA, a fin unit of 32 rows, a cluster
// warp) reports only its best two keys.  The candidate list of a step is
// complete -- it holds EVERY unselected point whose fp32 score is within tau
// of the best -- exactly when no unit's second key lies in the window (then
// that unit has no third one either) and at most kMaxCand keys do.  The GPU's
// own pick, the maximum of all unit keys, is then always on the list.  A step
// whose list may be incomplete is flagged kFlagFull: the host re-scores ALL
// unselected points in fp64 (refine_all_* below: the same closed form, every
// candidate) and takes that argmax, so the decision never depends on which
// candidates a unit happened to report.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "kernels.cuh"

namespace bted {
namespace rf {

constexpr float kTau = 2e-5f;          // near-tie window, relative (>= 8x the measured fp32 error)
constexpr int kMaxCand = 32;
constexpr unsigned long long kForced = 1ull << 63;   // key flag of a forced (preset) pick
constexpr int kFlagNear = 1;           // near tie, complete candidate list
constexpr int kFlagFull = 2;           // near tie, list may be incomplete: re-score every unselected point

__device__ __forceinline__ float key_score(unsigned long long k) {
    return __uint_as_float((uint32_t)(k >> 32) - 1u);
}

// Per step t (one CTA each): reduce the score units' (top1, top2) keys; flag a
// near tie and list the candidates within tau of the best (kFlagNear), or flag
// kFlagFull when the list may be incomplete (see the header).
__global__ void __launch_bounds__(256)
neartie_check_kernel(const unsigned long long* __restrict__ top2, int nC, const unsigned long long* __restrict__ keys,
                     float tau, int* __restrict__ flags, uint32_t* __restrict__ cand, int* __restrict__ ncand,
                     int* __restrict__ nflag) {
    // (gridDim.y > 1: one independent TED per y, m = gridDim.x steps each, arrays back to back)
    {
        const int64_t y = blockIdx.y, m = gridDim.x;
        top2 += y * m * nC * 2;
        keys += y * m;
        flags += y * m;
        cand += y * m * kMaxCand;
        ncand += y * m;
        nflag += y;
    }
    __shared__ unsigned long long red[8];
    __shared__ int cnt, over;
    const int t = blockIdx.x, tid = threadIdx.x;
    const unsigned long long kt = keys[t];
    if (kt & kForced) { if (tid == 0) { flags[t] = 0; ncand[t] = 0; } return; }
    const unsigned long long* p = top2 + (int64_t)t * nC * 2;
    unsigned long long m1 = 0ull;
    for (int q = tid; q < 2 * nC; q += 256) m1 = p[q] > m1 ? p[q] : m1;
    m1 = warp_max_u64(m1);
    if ((tid & 31) == 0) red[tid >> 5] = m1;
    if (tid == 0) { cnt = 0; over = 0; }
    __syncthreads();
    unsigned long long best = 0ull;
    for (int q = 0; q < 8; ++q) best = red[q] > best ? red[q] : best;
    __syncthreads();
    unsigned long long m2 = 0ull;
    for (int q = tid; q < 2 * nC; q += 256) if (p[q] != best && p[q] > m2) m2 = p[q];
    m2 = warp_max_u64(m2);
    if ((tid & 31) == 0) red[tid >> 5] = m2;
    __syncthreads();
    unsigned long long second = 0ull;
    for (int q = 0; q < 8; ++q) second = red[q] > second ? red[q] : second;
    const float s1 = key_score(best);
    const float lim = s1 * (1.f - tau);
    const bool near = second != 0ull && key_score(second) >= lim;
    if (near) {
        for (int q = tid; q < 2 * nC; q += 256) {
            const unsigned long long k = p[q];
            if (k != 0ull && key_score(k) >= lim) {
                if (q & 1) over = 1;                    // a unit's SECOND key in the window: it may hold a third
                const int pos = atomicAdd(&cnt, 1);
                if (pos < kMaxCand) cand[(int64_t)t * kMaxCand + pos] = key_index(k);
            }
        }
    }
    __syncthreads();
    if (tid == 0) {
        const bool full = near && (over || cnt > kMaxCand);
        flags[t] = near ? (full ? kFlagFull : kFlagNear) : 0;
        ncand[t] = near ? min(cnt, kMaxCand) : 0;
        if (near) atomicAdd(nflag, 1);
    }
}

// Row-shard K4 (bted_shard_nearties): per step t, this band's candidates within
// tau of the GLOBAL pick keys[t] (already all-reduced), from the band's per-CTA
// top-2 keys; a forced (preset) step lists none.  ncand[t] = -1 when the band's
// list may be incomplete (a CTA's second key in the window, or > kMaxCand).
// One CTA per step.
__global__ void __launch_bounds__(256)
shard_neartie_kernel(const unsigned long long* __restrict__ top2, int nC, const unsigned long long* __restrict__ keys,
                     float tau, uint32_t* __restrict__ cand, int* __restrict__ ncand) {
    __shared__ int cnt, over;
    const int t = blockIdx.x, tid = threadIdx.x;
    const unsigned long long kt = keys[t];
    if (tid == 0) { cnt = 0; over = 0; }
    __syncthreads();
    if (!(kt & kForced) && kt != 0ull) {
        const float lim = key_score(kt) * (1.f - tau);
        const unsigned long long* p = top2 + (int64_t)t * nC * 2;
        for (int q = tid; q < 2 * nC; q += 256) {
            const unsigned long long k = p[q];
            if (k != 0ull && key_score(k) >= lim) {
                if (q & 1) over = 1;
                const int pos = atomicAdd(&cnt, 1);
                if (pos < kMaxCand) cand[(int64_t)t * kMaxCand + pos] = key_index(k);
            }
        }
    }
    __syncthreads();
    if (tid == 0) ncand[t] = (over || cnt > kMaxCand) ? -1 : cnt;
}

// G[j][i] = k(x_i, x_{cols[j]}) in fp64 (direct difference; reading A1), i < N.
__global__ void refine_cols_kernel(const float* __restrict__ X, int32_t N, int32_t d, double gamma, int32_t linear,
                                   const uint32_t* __restrict__ cols, double* __restrict__ G) {
    const int j = blockIdx.y;
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= N) return;
    const uint32_t c = cols[j];
    double a = 0.0;
    for (int k = 0; k < d; ++k) {
        const double xi = (double)X[(int64_t)i * d + k], xc = (double)X[(int64_t)c * d + k];
        if (linear) a = __fma_rn(xi, xc, a);
        else { const double df = xi - xc; a = __fma_rn(df, df, a); }
    }
    G[(int64_t)j * N + i] = linear ? a : exp(-gamma * a);
}

// One CTA: A = K_SS + mu I (t x t) -> Cholesky L L^T -> W[:, c] = A^-1 K_Sc for
// the nc candidates.  cols = [S (t) | C (nc)], G from refine_cols_kernel.
// (A lives in dynamic shared memory when the launch provides t*t doubles of it:
// the right-looking factorisation's ~3t barriers then cost no global round trips)
__global__ void __launch_bounds__(256)
refine_solve_kernel(const double* __restrict__ G, int32_t N, const uint32_t* __restrict__ cols, int t, int nc,
                    double mu, double* __restrict__ Ag, double* __restrict__ W, int a_in_smem) {
    extern __shared__ double As[];
    double* A = a_in_smem ? As : Ag;
    const int tid = threadIdx.x;
    for (int e = tid; e < t * t; e += 256) {
        const int a = e / t, b = e % t;
        A[e] = G[(int64_t)a * N + cols[b]] + (a == b ? mu : 0.0);
    }
    __syncthreads();
    for (int k = 0; k < t; ++k) {                       // right-looking Cholesky, lower triangle
        const double dkk = sqrt(A[k * t + k]);          // (every thread; two barriers per column)
        __syncthreads();                                // all have read A[k][k] before it changes
        if (tid == 0) A[k * t + k] = dkk;
        for (int i = k + 1 + tid; i < t; i += 256) A[i * t + k] /= dkk;
        __syncthreads();
        for (int e = tid; e < (t - k - 1) * (t - k - 1); e += 256) {
            const int i = k + 1 + e / (t - k - 1), j = k + 1 + e % (t - k - 1);
            if (j <= i) A[i * t + j] -= A[i * t + k] * A[j * t + k];
        }
        __syncthreads();
    }
    if (a_in_smem == 2) {                               // all candidates at once, right-looking, in smem
        double* B = As + (size_t)t * t;                 // [nc][t]: K_Sc -> y -> w
        for (int e = tid; e < nc * t; e += 256) {
            const int c = e / t, i = e % t;
            B[e] = G[(int64_t)i * N + cols[t + c]];
        }
        __syncthreads();
        for (int i = 0; i < t; ++i) {                   // L y = b
            const double lii = A[i * t + i];
            for (int c = tid; c < nc; c += 256) B[c * t + i] /= lii;
            __syncthreads();
            for (int e = tid; e < nc * (t - i - 1); e += 256) {
                const int c = e / (t - i - 1), j = i + 1 + e % (t - i - 1);
                B[c * t + j] -= A[j * t + i] * B[c * t + i];
            }
            __syncthreads();
        }
        for (int i = t - 1; i >= 0; --i) {              // L^T w = y
            const double lii = A[i * t + i];
            for (int c = tid; c < nc; c += 256) B[c * t + i] /= lii;
            __syncthreads();
            for (int e = tid; e < nc * i; e += 256) {
                const int c = e / i, j = e % i;
                B[c * t + j] -= A[i * t + j] * B[c * t + i];
            }
            __syncthreads();
        }
        for (int e = tid; e < nc * t; e += 256) W[e] = B[e];
        return;
    }
    for (int c = tid; c < nc; c += 256) {               // W[:, c] = L^-T L^-1 K_Sc
        double* w = W + (int64_t)c * t;
        for (int i = 0; i < t; ++i) {                   // forward
            double v = G[(int64_t)i * N + cols[t + c]];
            for (int k = 0; k < i; ++k) v -= A[i * t + k] * w[k];
            w[i] = v / A[i * t + i];
        }
        for (int i = t - 1; i >= 0; --i) {              // backward
            double v = w[i];
            for (int k = i + 1; k < t; ++k) v -= A[k * t + i] * w[k];
            w[i] = v / A[i * t + i];
        }
    }
}

// r_ic = K_ic - sum_k K_{i,S_k} W[k][c]: per-CTA partial sums of r_ic^2 and the
// residual at the candidate's own row.  One thread per (row, candidate): grid
// (ceil(N / 256), nc); the candidate's W column is broadcast from shared memory.
__global__ void __launch_bounds__(256)
refine_resid2_kernel(const double* __restrict__ G, int32_t N, const uint32_t* __restrict__ cols, int t,
                     const double* __restrict__ W, double* __restrict__ part, double* __restrict__ diag) {
    extern __shared__ double wc[];                      // [t]
    __shared__ double red[8];
    const int c = blockIdx.y, tid = threadIdx.x;
    for (int k = tid; k < t; k += 256) wc[k] = W[(int64_t)c * t + k];
    __syncthreads();
    const int i = blockIdx.x * 256 + tid;
    double r2 = 0.0;
    if (i < N) {
        double r = G[(int64_t)(t + c) * N + i];
        for (int k = 0; k < t; ++k) r -= G[(int64_t)k * N + i] * wc[k];
        r2 = r * r;
        if ((uint32_t)i == cols[t + c]) diag[c] = r;
    }
    for (int off = 16; off > 0; off >>= 1) r2 += __shfl_xor_sync(0xffffffffu, r2, off);
    if ((tid & 31) == 0) red[tid >> 5] = r2;
    __syncthreads();
    if (tid == 0) {
        double v = 0.0;
        for (int w = 0; w < 8; ++w) v += red[w];
        part[(int64_t)blockIdx.x * kMaxCand + c] = v;
    }
}

// exact scores of the candidates and their argmax (ties: lowest index)
__global__ void refine_pick_kernel(const double* __restrict__ part, int nblocks, const double* __restrict__ diag,
                                   const uint32_t* __restrict__ cols, int t, int nc, double mu,
                                   double* __restrict__ out_score, uint32_t* __restrict__ out_idx) {
    if (threadIdx.x != 0) return;
    double bs = -1.0;
    uint32_t bi = 0xFFFFFFFFu;
    for (int c = 0; c < nc; ++c) {
        double n = 0.0;
        for (int b = 0; b < nblocks; ++b) n += part[(int64_t)b * kMaxCand + c];
        const double sc = n / (diag[c] + mu);
        const uint32_t idx = cols[t + c];
        out_score[c] = sc;
        if (sc > bs || (sc == bs && idx < bi)) { bs = sc; bi = idx; }
    }
    out_idx[0] = bi;
    out_score[kMaxCand] = bs;
}

// ------------------------------------------------------------------ full re-scoring (kFlagFull)
// Exact fp64 scores of EVERY point after the picks S (|S| = t), the closed form
// of pin C2 for all candidates at once:
//   W = (K_SS + mu I)^-1 K_S:            (t x N; Cholesky of K_SS + mu I)
//   r_ic = K_ic - sum_k K_{i,S_k} W_kc,   score_c = sum_i r_ic^2 / (r_cc + mu)
// K_ic recomputed from the features in fp64 (as refine_cols_kernel).  Every
// candidate's sum runs in a fixed order, so exact duplicates score bitwise
// equal and tie to the lowest index.  Cost ~N^2 (t + d) fp64 FMAs: a rare path.

// one CTA: Ag (t x t, global) <- Cholesky factor (lower) of K_SS + mu I, G = K_:S [t][N]
__global__ void __launch_bounds__(256)
refine_chol_kernel(const double* __restrict__ G, int32_t N, const uint32_t* __restrict__ S, int t, double mu,
                   double* __restrict__ A) {
    const int tid = threadIdx.x;
    for (int e = tid; e < t * t; e += 256) {
        const int a = e / t, b = e % t;
        A[e] = G[(int64_t)a * N + S[b]] + (a == b ? mu : 0.0);
    }
    __syncthreads();
    for (int k = 0; k < t; ++k) {                       // right-looking, lower triangle
        const double dkk = sqrt(A[k * t + k]);
        __syncthreads();
        if (tid == 0) A[k * t + k] = dkk;
        for (int i = k + 1 + tid; i < t; i += 256) A[i * t + k] /= dkk;
        __syncthreads();
        for (int e = tid; e < (t - k - 1) * (t - k - 1); e += 256) {
            const int i = k + 1 + e / (t - k - 1), j = k + 1 + e % (t - k - 1);
            if (j <= i) A[i * t + j] -= A[i * t + k] * A[j * t + k];
        }
        __syncthreads();
    }
}

// one thread per column c: Wt[:, c] = L^-T L^-1 K_{S,c}  (Wt is t x N, c contiguous)
__global__ void __launch_bounds__(256)
refine_solve_all_kernel(const double* __restrict__ G, int32_t N, int t, const double* __restrict__ A,
                        double* __restrict__ Wt) {
    const int c = blockIdx.x * 256 + threadIdx.x;
    if (c >= N) return;
    for (int i = 0; i < t; ++i) {                       // forward: L y = K_Sc
        double v = G[(int64_t)i * N + c];
        for (int k = 0; k < i; ++k) v -= __ldg(&A[i * t + k]) * Wt[(int64_t)k * N + c];
        Wt[(int64_t)i * N + c] = v / __ldg(&A[i * t + i]);
    }
    for (int i = t - 1; i >= 0; --i) {                  // backward: L^T w = y
        double v = Wt[(int64_t)i * N + c];
        for (int k = i + 1; k < t; ++k) v -= __ldg(&A[k * t + i]) * Wt[(int64_t)k * N + c];
        Wt[(int64_t)i * N + c] = v / __ldg(&A[i * t + i]);
    }
}

constexpr int kAllCand = 16;            // candidates per CTA of refine_all_scores_kernel
constexpr int kAllMaxD = 64;

// CTA b: candidates c = 16b .. 16b+15 over all rows i (fixed order per
// candidate: thread-strided rows, then a fixed warp/CTA tree).  score[c] =
// fp64 exact score, or -1 for selected / padding candidates.
__global__ void __launch_bounds__(256)
refine_all_scores_kernel(const float* __restrict__ X, int32_t N, int32_t d, double gamma, int32_t linear,
                         const double* __restrict__ G, int t, const double* __restrict__ Wt,
                         const uint8_t* __restrict__ selmask, double mu, double* __restrict__ score) {
    extern __shared__ double wsm[];                     // [t][kAllCand]
    __shared__ float xc[kAllCand][kAllMaxD];
    __shared__ double red[8][kAllCand];
    __shared__ double rcc[kAllCand];
    const int tid = threadIdx.x, c0 = blockIdx.x * kAllCand;
    for (int e = tid; e < t * kAllCand; e += 256) {
        const int k = e / kAllCand, c = e % kAllCand;
        wsm[e] = c0 + c < N ? Wt[(int64_t)k * N + c0 + c] : 0.0;
    }
    for (int e = tid; e < kAllCand * d; e += 256) {
        const int c = e / d, k = e % d;
        xc[c][k] = c0 + c < N ? X[(int64_t)(c0 + c) * d + k] : 0.f;
    }
    if (tid < kAllCand) rcc[tid] = 0.0;
    __syncthreads();
    double ss[kAllCand];
#pragma unroll
    for (int c = 0; c < kAllCand; ++c) ss[c] = 0.0;
    for (int i = tid; i < N; i += 256) {
        double kv[kAllCand];
#pragma unroll
        for (int c = 0; c < kAllCand; ++c) kv[c] = 0.0;
        for (int k = 0; k < d; ++k) {
            const double xi = (double)X[(int64_t)i * d + k];
#pragma unroll
            for (int c = 0; c < kAllCand; ++c) {
                if (linear) kv[c] = __fma_rn(xi, (double)xc[c][k], kv[c]);
                else { const double df = xi - (double)xc[c][k]; kv[c] = __fma_rn(df, df, kv[c]); }
            }
        }
        if (!linear) {
#pragma unroll
            for (int c = 0; c < kAllCand; ++c) kv[c] = exp(-gamma * kv[c]);
        }
        for (int k = 0; k < t; ++k) {
            const double g = G[(int64_t)k * N + i];
#pragma unroll
            for (int c = 0; c < kAllCand; ++c) kv[c] = __fma_rn(-g, wsm[k * kAllCand + c], kv[c]);
        }
#pragma unroll
        for (int c = 0; c < kAllCand; ++c) {
            ss[c] = __fma_rn(kv[c], kv[c], ss[c]);
            if (i == c0 + c) rcc[c] = kv[c];            // r_cc: the candidate's own row
        }
    }
#pragma unroll
    for (int c = 0; c < kAllCand; ++c) {
        double v = ss[c];
        for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
        if ((tid & 31) == 0) red[tid >> 5][c] = v;
    }
    __syncthreads();
    if (tid < kAllCand) {
        const int c = c0 + tid;
        if (c < N) {
            double n = 0.0;
            for (int w = 0; w < 8; ++w) n += red[w][tid];
            score[c] = selmask[c] ? -1.0 : n / (rcc[tid] + mu);
        }
    }
}

// one CTA: the exact argmax of score[0..N) (score >= 0; ties: lowest index)
__global__ void __launch_bounds__(1024)
refine_all_pick_kernel(const double* __restrict__ score, int32_t N, double* __restrict__ out_score,
                       uint32_t* __restrict__ out_idx) {
    __shared__ double bs[32];
    __shared__ uint32_t bi[32];
    double b = -1.0;
    uint32_t ib = 0xFFFFFFFFu;
    for (int c = threadIdx.x; c < N; c += 1024) {       // ascending c per thread: strict > keeps the lowest
        const double v = score[c];
        if (v > b) { b = v; ib = (uint32_t)c; }
    }
    for (int off = 16; off > 0; off >>= 1) {
        const double ob = __shfl_xor_sync(0xffffffffu, b, off);
        const uint32_t oi = __shfl_xor_sync(0xffffffffu, ib, off);
        if (ob > b || (ob == b && oi < ib)) { b = ob; ib = oi; }
    }
    if ((threadIdx.x & 31) == 0) { bs[threadIdx.x >> 5] = b; bi[threadIdx.x >> 5] = ib; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < 32; ++w)
            if (bs[w] > b || (bs[w] == b && bi[w] < ib)) { b = bs[w]; ib = bi[w]; }
        *out_score = b;
        *out_idx = ib;
    }
}

}  // namespace rf
}  // namespace bted
