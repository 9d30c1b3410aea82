// implicit.cuh -- implicit deflation on the packed
// read-only Gram matrix.
//
// Algorithm 1 deflates K <- K - K_:s K_s: / (K_ss + mu)
// every step.  Written as K^(t) = K - L L^T with L = [l_1 .. l_t] (N x t),
// l_t = K^(t-1)_:s / sqrt(K^(t-1)_ss + mu), the same selections follow from
// K itself (never rewritten) plus the factor L:
//
//   R = K - L L^T (implicit),  l = R_:s / sqrt(R_ss + mu)
//   l_i   = (K_is - sum_k L_ik L_sk) / sqrt(c)                     (kernel A)
//   q     = K l  (one pass over the packed tiles, READ ONLY: 2 N^2 B) (kernel B)
//   (R l)_v = q_v - sum_k L_vk h_k,  h = L^T l,  |l|^2
//   n_v  <- n_v - 2 l_v (R l)_v + l_v^2 |l|^2      (= ||R'_:v||^2)   (kernel C)
//   r_vv <- r_vv - l_v^2,   score_v = n_v / (r_vv + mu)
//
// Every accumulation is fp64 (K stays the fp32 Gram of K1p), so the
// recurrence's cancellation costs nothing at the 1e-5 parity tolerance.  A
// step moves 2 N^2 bytes (packed K, read once) + O(N m) instead of the
// literal deflation's 4 N^2 (packed) / 8 N^2 (dense).  Sums run in orders
// that depend on N only (canonical trees as in packed.cuh, fp64), so exact
// duplicate points still tie to the lowest index.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "kernels.cuh"
#include "packed.cuh"

namespace bted {
namespace im {

using pk::T;
using pk::kGroups;
using pk::tile_ij;
using pk::tile_offset;
using pk::num_tiles;
using pk::packed_index;
constexpr int kThreads = 256;
constexpr int kMaxM = 256;           // factor columns held per step (m <= kMaxM)

__device__ __forceinline__ double warp_sum64(double v) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

// fp32 -> fp64 with integer ops (the F2F.F64.F32 pipe is the tile pass's
// bottleneck on B200).  Exact for zeros and normal numbers: exponent rebias
// (+896) and mantissa shift; subnormal inputs (|x| < 2^-126) take the
// hardware conversion (the caller checks per warp).
__device__ __forceinline__ double f2d_int(float x) {
    const uint32_t u = __float_as_uint(x), t = u & 0x7FFFFFFFu, sgn = u & 0x80000000u;
    const uint32_t hi = t ? (((t >> 3) + 0x38000000u) | sgn) : sgn;
    return __hiloint2double((int)hi, (int)(u << 29));
}
__device__ __forceinline__ bool is_subnormal(float x) {
    const uint32_t t = __float_as_uint(x) & 0x7FFFFFFFu;
    return t != 0u && t < 0x00800000u;
}

// ------------------------------------------------------------------ tile pass (fp64 partials)
// kNorm: row/col partials of K_ij^2 (the initial ||K_:v||^2);  else of K_ij w_j
// (rows) and K_ij w_i (columns): q = K w.  One CTA (256 threads) per stored
// tile; warp w: rows 16w..16w+15, half-warp h: rows 16w+8h..+7, lane hl:
// columns 8hl..8hl+7.  Canonical per-128 tree: groups of 4 consecutive terms
// (sequential), then the 32-leaf butterfly.
constexpr size_t tile_pass_smem_bytes = (size_t)(T * (kGroups + 1) + kGroups * T + T) * sizeof(double);

template <bool kNorm>
__global__ void __launch_bounds__(kThreads)
tile_pass_kernel(const float* __restrict__ K, int nT, const double* __restrict__ w, double* __restrict__ P64,
                 const double* __restrict__ Hpart, int nHpart, int nh, int hstride, double* __restrict__ h) {
    // group sums: rows [r][q] (row stride 33: conflict-free tree reads), columns
    // [q][c][hl] (group q, lane hl, its column 8hl+c).  Then threads 0..127 run the
    // canonical 32-leaf tree of one row each, threads 128..255 of one column each.
    constexpr int kRS = kGroups + 1;
    extern __shared__ double dsm[];                    // dynamic: tile_pass_smem_bytes
    double* rgs = dsm;                                 // [T][kRS]     33 KiB
    double* cgs = rgs + T * kRS;                       // [kGroups*T]  32 KiB
    double* wi = cgs + kGroups * T;                    // [T] w on the tile's rows
    const int tid = threadIdx.x, w_ = tid / 32, l = tid % 32;
    const int hw = l >> 4, hl = l & 15, c8 = 8 * hl;
    const int nTiles = (int)num_tiles(nT);
    const int64_t NP = (int64_t)nT * T;
    // kernel A left per-CTA partials of h = L^T l and |l|^2: CTAs k, k + grid, ...
    // reduce column k (thread-strided sequential sums, then a fixed tree)
    if (!kNorm) {
        for (int col = blockIdx.x; col < nh; col += gridDim.x) {
            double a = 0.0;
            for (int b = tid; b < nHpart; b += kThreads) a = __dadd_rn(a, Hpart[(int64_t)b * hstride + col]);
            a = warp_sum64(a);
            if (l == 0) cgs[w_] = a;
            __syncthreads();
            if (tid == 0) {
                double v = 0.0;
                for (int q = 0; q < kThreads / 32; ++q) v = __dadd_rn(v, cgs[q]);
                h[col] = v;
            }
            __syncthreads();
        }
    }
    const int64_t k = blockIdx.x;
    int I, J;
    tile_ij(k, nT, I, J);
    (void)nTiles;
    double wc[8];
    if (!kNorm) {
        if (tid < T) wi[tid] = w[(int64_t)I * T + tid];
#pragma unroll
        for (int c = 0; c < 8; ++c) wc[c] = w[(int64_t)J * T + c8 + c];
        __syncthreads();
    }
    const float* gin = K + k * (int64_t)(T * T);
    double cg[8];
#pragma unroll
    for (int r0 = 0; r0 < 8; r0 += 4) {
        f8 kv[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) kv[u] = ld8_stream(gin + (16 * w_ + 8 * hw + r0 + u) * T + c8);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int rr = r0 + u;
            const int r = 16 * w_ + 8 * hw + rr;
            double kd[8];
            bool sub = false;
#pragma unroll
            for (int c = 0; c < 8; ++c) sub |= is_subnormal(kv[u].v[c]);
            if (__any_sync(0xffffffffu, sub)) {
#pragma unroll
                for (int c = 0; c < 8; ++c) kd[c] = (double)kv[u].v[c];
            } else {
#pragma unroll
                for (int c = 0; c < 8; ++c) kd[c] = f2d_int(kv[u].v[c]);
            }
            // row terms K_ij * (K_ij | w_j): two groups of 4 consecutive columns
            const double* f = kNorm ? kd : wc;
            double ga = __dmul_rn(kd[0], f[0]);
            ga = __fma_rn(kd[1], f[1], ga); ga = __fma_rn(kd[2], f[2], ga); ga = __fma_rn(kd[3], f[3], ga);
            double gb = __dmul_rn(kd[4], f[4]);
            gb = __fma_rn(kd[5], f[5], gb); gb = __fma_rn(kd[6], f[6], gb); gb = __fma_rn(kd[7], f[7], gb);
            rgs[r * kRS + 2 * hl] = ga;
            rgs[r * kRS + 2 * hl + 1] = gb;
            if (I != J) {
                // column terms K_ij * (K_ij | w_i): groups of 4 consecutive rows
                const double wr = kNorm ? 0.0 : wi[r];
#pragma unroll
                for (int c = 0; c < 8; ++c) {
                    const double g = kNorm ? kd[c] : wr;
                    cg[c] = (rr & 3) == 0 ? __dmul_rn(kd[c], g) : __fma_rn(kd[c], g, cg[c]);
                }
                if ((rr & 3) == 3) {
#pragma unroll
                    for (int c = 0; c < 8; ++c) cgs[(r >> 2) * T + c * 16 + hl] = cg[c];
                }
            }
        }
    }
    __syncthreads();
    double hh[kGroups];
    if (tid < T) {                                      // row tid: P[J][I*T + tid]
#pragma unroll
        for (int q = 0; q < kGroups; ++q) hh[q] = rgs[tid * kRS + q];
    } else if (I != J) {                                // column: P[I][J*T + 8(c&15) + (c>>4)]
#pragma unroll
        for (int q = 0; q < kGroups; ++q) hh[q] = cgs[q * T + (tid - T)];
    }
    if (tid < T || I != J) {
#pragma unroll
        for (int off = 16; off > 0; off >>= 1)
#pragma unroll
            for (int q = 0; q < off; ++q) hh[q] = __dadd_rn(hh[q], hh[q + off]);
        if (tid < T) P64[(int64_t)J * NP + (int64_t)I * T + tid] = hh[0];
        else {
            const int c = tid - T;
            P64[(int64_t)I * NP + (int64_t)J * T + 8 * (c & 15) + (c >> 4)] = hh[0];
        }
    }
}

// ------------------------------------------------------------------ kernel A: the new factor column
// l_i = (K_is - sum_{k<tp} L_ik L_sk) / sqrt(r_ss + mu) for every row i (0 on
// padding), L[:, tp] = l, ell = l; per-CTA partials of h_k = sum_i L_ik l_i
// (k < tp) and of |l|^2 (slot tp), reduced by the tile pass.  A warp takes
// kRowsPerWarp rows; lane j holds factor columns j, j+32, ... (kMaxM / 32).
constexpr int kRowsPerWarp = 4;
constexpr int kEllRows = (kThreads / 32) * kRowsPerWarp;      // 32 rows per CTA
__global__ void __launch_bounds__(kThreads)
ell_kernel(const float* __restrict__ K, int nT, int32_t N, double* __restrict__ L, int32_t ldL, int32_t tp,
           const double* __restrict__ rdiag, float mu, const unsigned long long* __restrict__ keys, int32_t t,
           double* __restrict__ ell, double* __restrict__ Hpart, uint8_t* __restrict__ sel) {
    constexpr int kC = kMaxM / 32;
    __shared__ double part[kThreads / 32][kMaxM + 1];
    const int tid = threadIdx.x, w = tid / 32, l = tid % 32;
    const uint32_t s = key_index(keys[t - 1]);
    if (blockIdx.x == 0 && tid == 0) sel[s] = 1;
    const double rc = __dsqrt_rn(__dadd_rn(rdiag[s], (double)mu));
    double ls[kC], hacc[kC], lsq = 0.0;
#pragma unroll
    for (int c = 0; c < kC; ++c) {
        const int q = l + 32 * c;
        ls[c] = q < tp ? L[(int64_t)s * ldL + q] : 0.0;
        hacc[c] = 0.0;
    }
    for (int rr = 0; rr < kRowsPerWarp; ++rr) {
        const int i = blockIdx.x * kEllRows + w * kRowsPerWarp + rr;
        const double* Li = L + (int64_t)i * ldL;
        double li_q[kC];
        double dot = 0.0;
#pragma unroll
        for (int c = 0; c < kC; ++c) {
            const int q = l + 32 * c;
            li_q[c] = q < tp ? Li[q] : 0.0;
            dot = __fma_rn(li_q[c], ls[c], dot);
        }
        dot = warp_sum64(dot);
        double li = 0.0;
        if (i < N) li = __ddiv_rn(__dsub_rn((double)K[packed_index(i, (int)s, nT)], dot), rc);
        if (l == 0) {
            L[(int64_t)i * ldL + tp] = li;
            ell[i] = li;
        }
#pragma unroll
        for (int c = 0; c < kC; ++c) hacc[c] = __fma_rn(li_q[c], li, hacc[c]);
        lsq = __fma_rn(li, li, lsq);
    }
#pragma unroll
    for (int c = 0; c < kC; ++c) {
        const int q = l + 32 * c;
        if (q < tp) part[w][q] = hacc[c];
    }
    if (l == 0) part[w][tp] = lsq;
    __syncthreads();
    for (int q = tid; q <= tp; q += kThreads) {
        double a = 0.0;
        for (int ww = 0; ww < kThreads / 32; ++ww) a = __dadd_rn(a, part[ww][q]);
        Hpart[(int64_t)blockIdx.x * (ldL + 1) + q] = a;
    }
}

// ------------------------------------------------------------------ kernel C: scores
// t == 0 (after the norm pass): n_v = q_v (= ||K_:v||^2), r_vv = K_vv.
// t >= 1: (R l)_v = q_v - sum_{k<tp} L_vk h_k; n_v -= 2 l_v (R l)_v - l_v^2 |l|^2;
// r_vv -= l_v^2.  Score n_v / (r_vv + mu) rounded to fp32, masked, packed key.
constexpr int kFinRows = 32;
__global__ void __launch_bounds__(kThreads)
fin64_kernel(const double* __restrict__ P64, int nT, int32_t N, const float* __restrict__ K, float mu,
             const double* __restrict__ L, int32_t ldL, int32_t tp, const double* __restrict__ h,
             double* __restrict__ nv, double* __restrict__ rdiag, const uint8_t* __restrict__ sel,
             const unsigned long long* __restrict__ keys, int32_t t, unsigned long long* __restrict__ key_out,
             int* __restrict__ err, unsigned long long* __restrict__ top2) {
    __shared__ double part[8][kFinRows];
    __shared__ double hs[kMaxM + 1];
    const int lane = threadIdx.x % 32, w = threadIdx.x / 32;
    const int64_t NP = (int64_t)nT * T;
    const int i = blockIdx.x * kFinRows + lane;
    if (t > 0)
        for (int q = threadIdx.x; q <= tp; q += kThreads) hs[q] = h[q];
    const int per = (nT + 7) / 8;
    const int j0 = min(nT, w * per), j1 = min(nT, j0 + per);
    const double* src = P64 + i;
    double acc = 0.0;
    int J = j0;
    for (; J + 8 <= j1; J += 8) {
        double v[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) v[q] = src[(int64_t)(J + q) * NP];
#pragma unroll
        for (int q = 0; q < 8; ++q) acc = __dadd_rn(acc, v[q]);
    }
    for (; J < j1; ++J) acc = __dadd_rn(acc, src[(int64_t)J * NP]);
    part[w][lane] = acc;
    __syncthreads();
    if (w != 0) return;
    unsigned long long key = 0ull;
    if (i < N) {
        double q = part[0][lane];
#pragma unroll
        for (int u = 1; u < 8; ++u) q = __dadd_rn(q, part[u][lane]);
        const uint32_t s = t > 0 ? key_index(keys[t - 1]) : 0xFFFFFFFFu;
        double n, r;
        if (t == 0) {
            const int B = i / T, rr = i % T;
            n = q;
            r = (double)K[tile_offset(B, B, nT) * (T * T) + (int64_t)rr * T + rr];
        } else {
            const double* Li = L + (int64_t)i * ldL;
            double rl = q;
            for (int k = 0; k < tp; ++k) rl = __fma_rn(-Li[k], hs[k], rl);
            const double lv = Li[tp];
            n = nv[i];
            n = __fma_rn(-2.0 * lv, rl, n);
            n = __fma_rn(__dmul_rn(lv, lv), hs[tp], n);
            r = __fma_rn(-lv, lv, rdiag[i]);
        }
        nv[i] = n;
        rdiag[i] = r;
        const bool masked = sel[i] != 0 || (uint32_t)i == s;
        const float sc = (float)(__ddiv_rn(n > 0.0 ? n : 0.0, __dadd_rn(r, (double)mu)));
        if (!(__dadd_rn(r, (double)mu) > 0.0) || !(sc >= 0.f) || !(sc <= 3.402823466e38f)) {
            if (!masked) atomicOr(err, 1);
        } else if (!masked) {
            key = pack_key(sc, (uint32_t)i);
        }
    }
    const unsigned long long k1 = warp_max_u64(key);
    if (top2) {                                        // the CTA's best two keys (K4 near-tie check)
        const unsigned long long k2 = warp_max_u64(key == k1 ? 0ull : key);
        if (lane == 0) {
            top2[((int64_t)t * gridDim.x + blockIdx.x) * 2] = k1;
            top2[((int64_t)t * gridDim.x + blockIdx.x) * 2 + 1] = k2;
        }
    }
    if (lane == 0 && k1) atomicMax(key_out, k1);
}

}  // namespace im
}  // namespace bted
