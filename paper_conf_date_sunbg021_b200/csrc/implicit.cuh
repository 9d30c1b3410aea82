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

__device__ __forceinline__ void st_f64_hint(double* p, double v, uint64_t policy) {
    asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;" :: "l"(p), "d"(v), "l"(policy) : "memory");
}
// ------------------------------------------------------------------ tile pass (fp64 partials)
// kNorm: row/col partials of K_ij^2 (the initial ||K_:v||^2);  else of K_ij w_j
// (rows) and K_ij w_i (columns): q = K w.
//
// Persistent: 2 CTAs per SM, each a TMA ring of kStages 16 KiB chunks (32
// rows of a 64 KiB tile) fed by one producer lane (cp.async.bulk +
// mbarrier), so HBM streams independently of the fp64 arithmetic.  Eight
// consumer warps: in chunk c warp w owns tile rows 32c + 4w .. +3, lane l
// columns 4l .. 4l+3 (conflict-free LDS.128).
//
// Canonical per-128 tree (the SAME for rows and columns, so exact duplicate
// points get bitwise-equal norms and tie to the lowest index): groups of 4
// consecutive terms summed sequentially (mul, fma, fma, fma), then the
// 32-leaf butterfly h[q] += h[q + 16], += h[q + 8], ..., += h[q + 1].
//   rows:    group q = lane q  ->  a reduce-scatter shuffle butterfly
//            (xor 16 keeps rows {0,1}/{2,3}, xor 8 one row, then xor 4/2/1);
//   columns: group q = 8c + w  ->  levels 16 and 8 pair chunks (c, c+2) and
//            (0, 1) in registers, levels 4/2/1 pair warps through smem.
//
// fp32 -> fp64: the norm pass (once per TED) converts with F2F (exact for
// every value) and raises *kflag if any K entry is not a positive normal
// number (zero, subnormal, negative: linear kernel, underflowed RBF).  The
// per-step pass then uses 2 integer ops per element (exponent rebias +
// mantissa shift, exact for positive normals) unless *kflag is set.
constexpr int kChunkRows = 32;
constexpr int kChunkFloats = kChunkRows * T;                  // 4096
constexpr uint32_t kChunkBytes = kChunkFloats * 4;            // 16 KiB
constexpr int kStages = 5;                                    // 80 KiB ring per CTA (2 CTAs per SM)
constexpr int kTPWarps = 8;                                   // consumer warps
constexpr int kTPThreads = (kTPWarps + 1) * 32;               // + 1 producer warp
constexpr int kTPBlocksPerSM = 2;
constexpr int kChunks = T / kChunkRows;
struct TPSmem {
    float ring[kStages][kChunkFloats];
    double colstage[2][kTPWarps][T];                          // double-buffered per tile
    double red[kTPWarps];
    double wrow[kTPWarps][16];
    uint64_t full[kStages], empty[kStages];
};
constexpr size_t tile_pass_smem_bytes = sizeof(TPSmem);

__device__ __forceinline__ void tp_sync() {                   // named barrier 1: the 8 consumer warps
    asm volatile("bar.sync 1, %0;" :: "n"(kTPWarps * 32) : "memory");
}
// exact for a positive normal fp32 (the per-step fast path)
__device__ __forceinline__ double f2d_pos(float x) {
    const uint32_t u = __float_as_uint(x);
    return __hiloint2double((int)((u >> 3) + 0x38000000u), (int)(u << 29));
}
__device__ __forceinline__ bool not_pos_normal(float x) {
    return __float_as_uint(x) - 0x00800000u >= 0x7F000000u;
}

template <bool kNorm, bool kExact>
__device__ __forceinline__ void tp_consume(TPSmem& S, int nT, const double* __restrict__ w,
                                           double* __restrict__ P64, int* __restrict__ kflag) {
    const int tid = threadIdx.x, wq = tid / 32, l = tid % 32;
    const int64_t nTiles = num_tiles(nT);
    const int64_t NP = (int64_t)nT * T;
    const uint64_t keep = pk::policy_evict_last();            // partials are re-read by fin64 from L2
    bool odd_value = false;
    int n = 0, tile_it = 0;
    for (int64_t k = blockIdx.x; k < nTiles; k += gridDim.x, ++tile_it) {
        int I, J;
        tile_ij(k, nT, I, J);
        const bool offdiag = I != J;
        double wc[4];                                         // w on the lane's 4 columns
        if (!kNorm) {
#pragma unroll
            for (int x = 0; x < 4; ++x) wc[x] = w[(int64_t)J * T + 4 * l + x];
            // w on the warp's 16 rows of the tile (row 32c + 4w + r at [4c + r]); warp-private
            __syncwarp();
            if (l < 16) S.wrow[wq][l] = w[(int64_t)I * T + kChunkRows * (l >> 2) + 4 * wq + (l & 3)];
            __syncwarp();
        }
        double hold[2][4];
#pragma unroll
        for (int c = 0; c < kChunks; ++c, ++n) {
            const int st = n % kStages;
            pk::mbar_wait(&S.full[st], (uint32_t)(n / kStages) & 1u);
            // per row: load from the stage, convert, the row group (4 consecutive
            // columns) and the running column groups (4 rows: mul for row 0, then fma)
            double g[4], cg[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const float4 kv = *reinterpret_cast<const float4*>(&S.ring[st][(4 * wq + r) * T + 4 * l]);
                const float f32[4] = {kv.x, kv.y, kv.z, kv.w};
                double kd[4];
#pragma unroll
                for (int x = 0; x < 4; ++x) {
                    kd[x] = kExact ? (double)f32[x] : f2d_pos(f32[x]);
                    if (kNorm) odd_value |= not_pos_normal(f32[x]);
                }
                const double* f = kNorm ? kd : wc;
                double a = __dmul_rn(kd[0], f[0]);
                a = __fma_rn(kd[1], f[1], a);
                a = __fma_rn(kd[2], f[2], a);
                g[r] = __fma_rn(kd[3], f[3], a);
                // (diagonal tiles compute the column groups too and drop them: no per-row branch)
                const double wi = kNorm ? 0.0 : S.wrow[wq][4 * c + r];
#pragma unroll
                for (int x = 0; x < 4; ++x)
                    cg[x] = r == 0 ? __dmul_rn(kd[x], kNorm ? kd[x] : wi)
                                   : __fma_rn(kd[x], kNorm ? kd[x] : wi, cg[x]);
            }
            __syncwarp();
            if (l == 0) pk::mbar_arrive(&S.empty[st]);
            // row butterfly as a reduce-scatter: lanes < 16 keep rows 0,1, lanes >= 16 rows 2,3
            const bool up = l >= 16;
            const double s0 = __shfl_xor_sync(0xffffffffu, up ? g[0] : g[2], 16);
            const double s1 = __shfl_xor_sync(0xffffffffu, up ? g[1] : g[3], 16);
            const double h0 = __dadd_rn(up ? g[2] : g[0], s0);
            const double h1 = __dadd_rn(up ? g[3] : g[1], s1);
            const bool odd = (l & 8) != 0;                    // lanes 8..15 / 24..31 keep the odd row
            double hr = __dadd_rn(odd ? h1 : h0, __shfl_xor_sync(0xffffffffu, odd ? h0 : h1, 8));
            hr = __dadd_rn(hr, __shfl_xor_sync(0xffffffffu, hr, 4));
            hr = __dadd_rn(hr, __shfl_xor_sync(0xffffffffu, hr, 2));
            hr = __dadd_rn(hr, __shfl_xor_sync(0xffffffffu, hr, 1));
            if ((l & 7) == 0)                                  // row 32c + 4w + l/8: P[J][I*T + row]
                st_f64_hint(&P64[(int64_t)J * NP + (int64_t)I * T + kChunkRows * c + 4 * wq + (l >> 3)], hr, keep);
#pragma unroll
            for (int x = 0; x < 4; ++x) {
                if (c < 2) hold[c][x] = cg[x];                                      // groups w, 8 + w
                else hold[c - 2][x] = __dadd_rn(hold[c - 2][x], cg[x]);             // level 16
            }
        }
        if (offdiag) {
            const int buf = tile_it & 1;
#pragma unroll
            for (int x = 0; x < 4; ++x) S.colstage[buf][wq][4 * l + x] = __dadd_rn(hold[0][x], hold[1][x]);  // level 8
            tp_sync();
            if (tid < T) {                                   // levels 4, 2, 1 over the 8 warps
                double v[kTPWarps];
#pragma unroll
                for (int q = 0; q < kTPWarps; ++q) v[q] = S.colstage[buf][q][tid];
#pragma unroll
                for (int q = 0; q < 4; ++q) v[q] = __dadd_rn(v[q], v[q + 4]);
                v[0] = __dadd_rn(v[0], v[2]);
                v[1] = __dadd_rn(v[1], v[3]);
                st_f64_hint(&P64[(int64_t)I * NP + (int64_t)J * T + tid], __dadd_rn(v[0], v[1]), keep);
            }
        }
    }
    if (kNorm && odd_value) atomicOr(kflag, 1);
}

template <bool kNorm>
__global__ void __launch_bounds__(kTPThreads, kTPBlocksPerSM)
tile_pass_kernel(const float* __restrict__ K, int nT, const double* __restrict__ w, double* __restrict__ P64,
                 const double* __restrict__ Hpart, int nHpart, int nh, int hstride, double* __restrict__ h,
                 int* __restrict__ kflag) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    TPSmem& S = *reinterpret_cast<TPSmem*>(smem_raw);
    const int tid = threadIdx.x, wq = tid / 32, l = tid % 32;
    const int64_t nTiles = num_tiles(nT);
    if (tid == 0) {
        for (int q = 0; q < kStages; ++q) { pk::mbar_init(&S.full[q], 1); pk::mbar_init(&S.empty[q], kTPWarps); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (wq == kTPWarps) {
        // ---------------- producer: one lane streams this CTA's tiles, 4 chunks each
        if (l == 0) {
            const uint64_t pol = pk::policy_evict_first();    // K is read once per step
            int n = 0;
            for (int64_t k = blockIdx.x; k < nTiles; k += gridDim.x) {
                const float* src = K + k * (int64_t)(T * T);
                for (int c = 0; c < kChunks; ++c, ++n) {
                    const int st = n % kStages;
                    pk::mbar_wait(&S.empty[st], ((uint32_t)(n / kStages) & 1u) ^ 1u);
                    pk::mbar_expect_tx(&S.full[st], kChunkBytes);
                    pk::bulk_g2s_hint(S.ring[st], src + c * kChunkFloats, kChunkBytes, &S.full[st], pol);
                }
            }
        }
        return;
    }

    // ---------------- consumers
    if (kNorm) {
        tp_consume<true, true>(S, nT, w, P64, kflag);
        return;
    }
    // kernel A left per-CTA partials of h = L^T l and |l|^2: CTAs k, k + grid, ...
    // reduce column k (thread-strided sequential sums, then a fixed tree)
    for (int col = blockIdx.x; col < nh; col += gridDim.x) {
        double a = 0.0;
        for (int b = tid; b < nHpart; b += kTPWarps * 32) a = __dadd_rn(a, Hpart[(int64_t)b * hstride + col]);
        a = warp_sum64(a);
        if (l == 0) S.red[wq] = a;
        tp_sync();
        if (tid == 0) {
            double v = 0.0;
            for (int q = 0; q < kTPWarps; ++q) v = __dadd_rn(v, S.red[q]);
            h[col] = v;
        }
        tp_sync();
    }
    if (*kflag) tp_consume<false, true>(S, nT, w, P64, kflag);
    else tp_consume<false, false>(S, nT, w, P64, kflag);
}

// ------------------------------------------------------------------ kernel A: the new factor column
// L is column-major: Lc[k * ldL + i] (factor column k, row i), ldL = NPa, so
// every per-row sum over k reads coalesced.  For every row i:
//   l_i = (K_is - sum_{k<tp} L_ik L_sk) / sqrt(r_ss + mu)    (0 on padding)
// written to Lc[tp][i] and ell[i]; per-CTA partials of h_k = sum_i L_ik l_i
// (k < tp) and of |l|^2 (slot tp) go to Hpart (reduced by the tile pass).
// CTA = 64 rows x 4 k-phases (k = g, g+4, ...); the 4 phase sums are added in
// a fixed order, so a row's l_i depends on its own data only.
constexpr int kEllRows = 64;
__global__ void __launch_bounds__(kThreads)
ell_kernel(const float* __restrict__ K, int nT, int32_t N, double* __restrict__ Lc, int64_t ldL, int32_t tp,
           const double* __restrict__ rdiag, float mu, const unsigned long long* __restrict__ keys, int32_t t,
           double* __restrict__ ell, double* __restrict__ Hpart, int32_t hstride, uint8_t* __restrict__ sel) {
    __shared__ double Ls[kMaxM];
    __shared__ double part[4][kEllRows];
    __shared__ double lrow[kEllRows];
    const int tid = threadIdx.x, r = tid % kEllRows, g = tid / kEllRows, wq = tid / 32, l = tid % 32;
    const uint32_t s = key_index(keys[t - 1]);
    if (blockIdx.x == 0 && tid == 0) sel[s] = 1;
    const double rc = __dsqrt_rn(__dadd_rn(rdiag[s], (double)mu));
    for (int k = tid; k < tp; k += kThreads) Ls[k] = Lc[(int64_t)k * ldL + s];
    __syncthreads();
    const int64_t i0 = (int64_t)blockIdx.x * kEllRows;
    const int64_t i = i0 + r;
    double acc = 0.0;
    int k = g;
    for (; k + 12 < tp; k += 16) {                           // 4 independent loads in flight
        const double a0 = Lc[(int64_t)k * ldL + i], a1 = Lc[(int64_t)(k + 4) * ldL + i];
        const double a2 = Lc[(int64_t)(k + 8) * ldL + i], a3 = Lc[(int64_t)(k + 12) * ldL + i];
        acc = __fma_rn(a0, Ls[k], acc);
        acc = __fma_rn(a1, Ls[k + 4], acc);
        acc = __fma_rn(a2, Ls[k + 8], acc);
        acc = __fma_rn(a3, Ls[k + 12], acc);
    }
    for (; k < tp; k += 4) acc = __fma_rn(Lc[(int64_t)k * ldL + i], Ls[k], acc);
    part[g][r] = acc;
    __syncthreads();
    if (g == 0) {
        const double dot = __dadd_rn(__dadd_rn(__dadd_rn(part[0][r], part[1][r]), part[2][r]), part[3][r]);
        double li = 0.0;
        if (i < N) li = __ddiv_rn(__dsub_rn((double)K[packed_index((int)i, (int)s, nT)], dot), rc);
        Lc[(int64_t)tp * ldL + i] = li;
        ell[i] = li;
        lrow[r] = li;
    }
    __syncthreads();
    // h partials: warp wq takes k = wq, wq + 8, ...; slot tp = |l|^2
    for (int kk = wq; kk <= tp; kk += kThreads / 32) {
        double v;
        if (kk < tp) {
            v = __dmul_rn(Lc[(int64_t)kk * ldL + i0 + l], lrow[l]);
            v = __fma_rn(Lc[(int64_t)kk * ldL + i0 + 32 + l], lrow[32 + l], v);
        } else {
            v = __dmul_rn(lrow[l], lrow[l]);
            v = __fma_rn(lrow[32 + l], lrow[32 + l], v);
        }
        v = warp_sum64(v);
        if (l == 0) Hpart[(int64_t)blockIdx.x * hstride + kk] = v;
    }
}

// ------------------------------------------------------------------ kernel C: scores
// t == 0 (after the norm pass): n_v = q_v (= ||K_:v||^2), r_vv = K_vv.
// t >= 1: (R l)_v = q_v - sum_{k<tp} L_vk h_k; n_v -= 2 l_v (R l)_v - l_v^2 |l|^2;
// r_vv -= l_v^2.  Score n_v / (r_vv + mu) rounded to fp32, masked, packed key.
// CTA = 32 rows (lanes) x 8 warps; warp w sums the J-range and the k-range
// w of its rows, the 8 partial sums are added in warp order.
constexpr int kFinRows = 32;
__global__ void __launch_bounds__(kThreads)
fin64_kernel(const double* __restrict__ P64, int nT, int32_t N, const float* __restrict__ K, float mu,
             const double* __restrict__ Lc, int64_t ldL, int32_t tp, const double* __restrict__ h,
             double* __restrict__ nv, double* __restrict__ rdiag, const uint8_t* __restrict__ sel,
             const unsigned long long* __restrict__ keys, int32_t t, unsigned long long* __restrict__ key_out,
             int* __restrict__ err, unsigned long long* __restrict__ top2) {
    __shared__ double part[8][kFinRows];
    __shared__ double lpart[8][kFinRows];
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
    double la = 0.0;                                       // sum_{k in range w} L_ik h_k
    if (t > 0) {
        const int kper = (tp + 7) / 8;
        const int k0 = min(tp, w * kper), k1 = min(tp, k0 + kper);
        int k = k0;
        for (; k + 4 <= k1; k += 4) {
            double a[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) a[q] = Lc[(int64_t)(k + q) * ldL + i];
#pragma unroll
            for (int q = 0; q < 4; ++q) la = __fma_rn(a[q], hs[k + q], la);
        }
        for (; k < k1; ++k) la = __fma_rn(Lc[(int64_t)k * ldL + i], hs[k], la);
    }
    lpart[w][lane] = la;
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
            double lh = lpart[0][lane];
#pragma unroll
            for (int u = 1; u < 8; ++u) lh = __dadd_rn(lh, lpart[u][lane]);
            const double rl = __dsub_rn(q, lh);
            const double lv = Lc[(int64_t)tp * ldL + i];
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
