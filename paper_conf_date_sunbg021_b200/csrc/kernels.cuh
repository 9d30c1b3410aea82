// kernels.cuh -- sm_100a kernels of the TED hot path (Algorithm 1).
//
// Layout in HBM:
//   K    fp32, rows x ld row-major, ld = round_up(N, 32) (128-byte rows);
//        columns [N, ld) are kept exactly 0 so no kernel needs a column mask.
//   XT   fp32, d x ld (feature-major copy of X, zero padded) for K1.
//   keys u64 [m]: keys[t] = packed argmax of step t (see pack_key).
//   sel  u8 [rows]: 1 once a row has been selected (reading A4).
//
// Bit-symmetry: K1 computes K_ij with the direct-difference form and K2
// updates with the product first, v = fma(-(a_i*p_j), 1/c, k_ij); both are
// invariant under i <-> j, so K stays bitwise symmetric and the row norm of
// row v IS the column norm ||K_v||^2 of Alg. 1 l.3.  Every row's reduction
// order depends on N only (never on the grid or on which shard owns it).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bted {

constexpr int kWarp = 32;

// key = ((bits(score) + 1) << 32) | (0xFFFFFFFF - idx): a u64 max picks the
// largest score and, among equal scores, the LOWEST index (reading A5).
// score >= 0 always (a sum of squares over a positive denominator), so its
// IEEE bits order like the value.  0 means "no candidate".
__device__ __forceinline__ unsigned long long pack_key(float score, uint32_t idx) {
    return ((unsigned long long)(__float_as_uint(score) + 1u) << 32) |
           (unsigned long long)(0xFFFFFFFFu - idx);
}
__device__ __forceinline__ uint32_t key_index(unsigned long long key) {
    return 0xFFFFFFFFu - (uint32_t)(key & 0xFFFFFFFFull);
}

__device__ __forceinline__ float4 ld_stream(const float* p) {
    float4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ float4 ld_keep(const float* p) {
    float4 r;
    asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ void st_stream(float* p, float4 v) {
    asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};"
                 :: "l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
}

// One element of Alg. 1 l.5: k - (a*p)/c, product first (bit-symmetric).
__device__ __forceinline__ float deflate1(float k, float a, float p, float inv_c) {
    return __fmaf_rn(-__fmul_rn(a, p), inv_c, k);
}

__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long v) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
        unsigned long long o = __shfl_xor_sync(0xffffffffu, v, off);
        v = o > v ? o : v;
    }
    return v;
}
// xor butterfly: every lane ends with the bitwise-same sum (each level adds
// two values commutatively), in an order fixed by the lane layout.
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
    return v;
}

// Score of Alg. 1 l.3 from a row norm g and the new diagonal entry:
// g / (k(v,v) + mu).  Flags a NaN / non-positive denominator.
__device__ __forceinline__ unsigned long long score_key(float g, float diag, float mu, uint32_t idx,
                                                        bool masked, int* err) {
    const float den = __fadd_rn(diag, mu);
    const float sc = __fdiv_rn(g, den);
    if (!(den > 0.f) || !(sc >= 0.f) || !(sc <= 3.402823466e38f)) {
        if (!masked) atomicOr(err, 1);
        return 0ull;
    }
    return masked ? 0ull : pack_key(sc, idx);
}

// CTA-wide max of one key per thread, then one atomicMax into *dst.  With
// top2 (K4 near-tie check, refine.cuh) the CTA's two best keys are also
// written to top2[0..1] (keys are distinct: they carry the row index); key2 is
// a thread's second-best key when it scored several rows (else 0).
__device__ __forceinline__ void top2_merge(unsigned long long& b1, unsigned long long& b2, unsigned long long c1,
                                           unsigned long long c2) {
    const unsigned long long hi = b1 > c1 ? b1 : c1, lo = b1 > c1 ? c1 : b1;
    const unsigned long long s2 = b2 > c2 ? b2 : c2;
    b1 = hi;
    b2 = lo > s2 ? lo : s2;
}
template <int kThreads>
__device__ __forceinline__ void cta_key_max_to(unsigned long long key, unsigned long long* dst,
                                               unsigned long long* top2 = nullptr,
                                               unsigned long long key2 = 0ull) {
    __shared__ unsigned long long red[kThreads / kWarp][2];
    unsigned long long b1 = key, b2 = key2;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
        const unsigned long long c1 = __shfl_xor_sync(0xffffffffu, b1, off);
        const unsigned long long c2 = __shfl_xor_sync(0xffffffffu, b2, off);
        top2_merge(b1, b2, c1, c2);
    }
    const int w = threadIdx.x / kWarp, l = threadIdx.x % kWarp;
    if (l == 0) { red[w][0] = b1; red[w][1] = b2; }
    __syncthreads();
    if (w == 0) {
        unsigned long long v1 = l < kThreads / kWarp ? red[l][0] : 0ull;
        unsigned long long v2 = l < kThreads / kWarp ? red[l][1] : 0ull;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
            const unsigned long long c1 = __shfl_xor_sync(0xffffffffu, v1, off);
            const unsigned long long c2 = __shfl_xor_sync(0xffffffffu, v2, off);
            top2_merge(v1, v2, c1, c2);
        }
        if (l == 0 && v1 != 0ull) atomicMax(dst, v1);
        if (l == 0 && top2) { top2[0] = v1; top2[1] = v2; }
    }
}

// ---------------------------------------------------------------------------
// K0: XT[k][j] = X[j][k] for j < N, 0 for N <= j < ld.
__global__ void transpose_pad_kernel(const float* __restrict__ X, int32_t N, int32_t d,
                                     float* __restrict__ XT, int64_t ld) {
    int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= ld) return;
    for (int k = 0; k < d; ++k) XT[(int64_t)k * ld + j] = j < N ? X[j * (int64_t)d + k] : 0.f;
}

// ---------------------------------------------------------------------------
// K1: Alg. 1 l.1 (K <- K_VV) + l.3 at t = 1 (row norms, scores, first key).
// CTA = 256 threads owns kRows consecutive rows of the band; thread t covers
// the float4 column groups t, t+256, ...  X_i of the CTA's rows sit in smem
// (broadcast reads), X_j come from XT as float4 (L2-resident, 4 MiB max).
template <int kRows, int kThreads>
__global__ void __launch_bounds__(kThreads)
gram_rownorm_kernel(const float* __restrict__ XT, int64_t ld, int32_t d, int32_t N,
                    int32_t row0, int32_t nrows, float gamma, int32_t linear,
                    float* __restrict__ K, float mu,
                    unsigned long long* __restrict__ key_out, int* __restrict__ err,
                    unsigned long long* __restrict__ top2 = nullptr) {
    extern __shared__ float xi[];                       // [kRows][d]
    __shared__ float red[kThreads / kWarp][kRows];
    const int lrow0 = blockIdx.x * kRows;               // local row of this CTA
    for (int e = threadIdx.x; e < kRows * d; e += kThreads) {
        const int r = e / d, k = e % d;
        const int lr = lrow0 + r;
        xi[r * d + k] = lr < nrows ? XT[(int64_t)k * ld + row0 + lr] : 0.f;
    }
    __syncthreads();
    float norm[kRows];
#pragma unroll
    for (int r = 0; r < kRows; ++r) norm[r] = 0.f;
    const float ng = -gamma;
    const int64_t nvec = ld >> 2;
    for (int64_t v = threadIdx.x; v < nvec; v += kThreads) {
        const int64_t j0 = v << 2;
        float acc[kRows][4];
#pragma unroll
        for (int r = 0; r < kRows; ++r) acc[r][0] = acc[r][1] = acc[r][2] = acc[r][3] = 0.f;
        for (int k = 0; k < d; ++k) {
            const float4 xj = *reinterpret_cast<const float4*>(XT + (int64_t)k * ld + j0);
#pragma unroll
            for (int r = 0; r < kRows; ++r) {
                const float x = xi[r * d + k];
                if (linear) {
                    acc[r][0] = __fmaf_rn(x, xj.x, acc[r][0]);
                    acc[r][1] = __fmaf_rn(x, xj.y, acc[r][1]);
                    acc[r][2] = __fmaf_rn(x, xj.z, acc[r][2]);
                    acc[r][3] = __fmaf_rn(x, xj.w, acc[r][3]);
                } else {
                    float df;
                    df = __fsub_rn(x, xj.x); acc[r][0] = __fmaf_rn(df, df, acc[r][0]);
                    df = __fsub_rn(x, xj.y); acc[r][1] = __fmaf_rn(df, df, acc[r][1]);
                    df = __fsub_rn(x, xj.z); acc[r][2] = __fmaf_rn(df, df, acc[r][2]);
                    df = __fsub_rn(x, xj.w); acc[r][3] = __fmaf_rn(df, df, acc[r][3]);
                }
            }
        }
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
            const int lr = lrow0 + r;
            if (lr >= nrows) continue;
            float4 o;
            float* oc = &o.x;
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const float val = linear ? acc[r][c] : expf(__fmul_rn(ng, acc[r][c]));
                oc[c] = (j0 + c < N) ? val : 0.f;
                norm[r] = __fmaf_rn(oc[c], oc[c], norm[r]);
            }
            st_stream(K + (int64_t)lr * ld + j0, o);
        }
    }
    // row norms: warp butterfly, then warps in order
    const int w = threadIdx.x / kWarp, l = threadIdx.x % kWarp;
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
        const float s = warp_sum(norm[r]);
        if (l == 0) red[w][r] = s;
    }
    __syncthreads();
    unsigned long long key = 0ull;
    if (threadIdx.x < kRows) {
        const int r = threadIdx.x, lr = lrow0 + r;
        if (lr < nrows) {
            float g = 0.f;
            for (int ww = 0; ww < kThreads / kWarp; ++ww) g = __fadd_rn(g, red[ww][r]);
            // diagonal entry of the fresh K: recompute exactly as the sweep did
            float diag;
            {
                float a = 0.f;
                for (int k = 0; k < d; ++k) {
                    const float x = xi[r * d + k];
                    if (linear) a = __fmaf_rn(x, x, a);
                    else { const float df = __fsub_rn(x, x); a = __fmaf_rn(df, df, a); }
                }
                diag = linear ? a : expf(__fmul_rn(ng, a));
            }
            key = score_key(g, diag, mu, (uint32_t)(row0 + lr), false, err);
        }
    }
    // (top2 at step 0 is laid out like K2's: CTA b of K1 covers K2's CTAs 2b, 2b+1)
    if (top2 && threadIdx.x == 0) top2[4 * (int64_t)blockIdx.x + 2] = top2[4 * (int64_t)blockIdx.x + 3] = 0ull;
    cta_key_max_to<kThreads>(key, key_out, top2 ? top2 + 4 * (int64_t)blockIdx.x : nullptr);
}

// ---------------------------------------------------------------------------
// 256-bit global accesses (sm_100: LDG.E.256 / STG.E.256).  A lane moves 8
// consecutive fp32 per instruction; K streams with L1 no-allocate loads and
// evict-first (.cs) stores, the pivot row with plain cached loads (L2-hot).
struct f8 { float v[8]; };
__device__ __forceinline__ f8 ld8_stream(const float* p) {
    f8 r;
    asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]), "=f"(r.v[4]), "=f"(r.v[5]),
                   "=f"(r.v[6]), "=f"(r.v[7]) : "l"(p));
    return r;
}
__device__ __forceinline__ f8 ld8_keep(const float* p) {
    f8 r;
    asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]), "=f"(r.v[4]), "=f"(r.v[5]),
                   "=f"(r.v[6]), "=f"(r.v[7]) : "l"(p));
    return r;
}
__device__ __forceinline__ void st8_stream(float* p, const f8& r) {
    asm volatile("st.global.cs.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
                 :: "l"(p), "f"(r.v[0]), "f"(r.v[1]), "f"(r.v[2]), "f"(r.v[3]), "f"(r.v[4]), "f"(r.v[5]),
                    "f"(r.v[6]), "f"(r.v[7]) : "memory");
}

// ---------------------------------------------------------------------------
// K2: Alg. 1 l.5 at step t (pivot s_t = keys[t-1]) fused with l.3 of step
// t+1: K_out = K_in - K_in[:,s] K_in[s,:] / (K_in[s,s] + mu), new row norms,
// scores, and the packed argmax into keys[t].  One warp owns kRows rows at a
// time; lane l covers the 8-float column groups l, l+32, ... (kUnroll groups
// in flight per row, 256-bit loads).  The pivot row p (= column s by
// symmetry) is read through L2 once per kRows rows.  Ping-pong buffers
// (K_in != K_out) make the pivot row read-only during the sweep.
// Chosen by scripts/k2_variants.cu (profiles/r1/k2_variants.txt).
template <int kRows, int kUnroll, int kThreads>
__global__ void __launch_bounds__(kThreads)
deflate_rescore_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int64_t ld,
                       int32_t row0, int32_t nrows, const float* __restrict__ pivot_ext,
                       unsigned long long* __restrict__ keys, int32_t t, float mu,
                       uint8_t* __restrict__ sel, int* __restrict__ err,
                       unsigned long long* __restrict__ top2 = nullptr) {
    constexpr int kWarps = kThreads / kWarp;
    const uint32_t s = key_index(keys[t - 1]);
    const float* __restrict__ p = pivot_ext ? pivot_ext : Kin + (int64_t)((int32_t)s - row0) * ld;
    const float inv_c = __frcp_rn(__fadd_rn(p[s], mu));   // 1 / (k(x,x) + mu)
    if (blockIdx.x == 0 && threadIdx.x == 0 && (int32_t)s >= row0 && (int32_t)s < row0 + nrows)
        sel[(int32_t)s - row0] = 1;
    const int w = threadIdx.x / kWarp, l = threadIdx.x % kWarp;
    const int lrow0 = (blockIdx.x * kWarps + w) * kRows;
    const int64_t nvec = ld >> 3;

    float a[kRows], acc[kRows];
    const float* kin[kRows];
    float* kout[kRows];
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
        const int lr = min(lrow0 + r, nrows - 1);       // clamp: duplicate work is discarded
        a[r] = p[row0 + lr];                            // K_in[i, s] = K_in[s, i]
        kin[r] = Kin + (int64_t)lr * ld;
        kout[r] = Kout + (int64_t)lr * ld;
        acc[r] = 0.f;
    }
    const bool any = lrow0 < nrows;
    if (any) {
        int64_t v = l;
        for (; v + (kUnroll - 1) * kWarp < nvec; v += kUnroll * kWarp) {
            f8 pv[kUnroll], kv[kUnroll][kRows];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                pv[u] = ld8_keep(p + ((v + u * kWarp) << 3));
#pragma unroll
                for (int r = 0; r < kRows; ++r) kv[u][r] = ld8_stream(kin[r] + ((v + u * kWarp) << 3));
            }
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
#pragma unroll
                for (int r = 0; r < kRows; ++r) {
                    f8 o;
#pragma unroll
                    for (int c = 0; c < 8; ++c) {
                        o.v[c] = deflate1(kv[u][r].v[c], a[r], pv[u].v[c], inv_c);
                        acc[r] = __fmaf_rn(o.v[c], o.v[c], acc[r]);
                    }
                    if (lrow0 + r < nrows) st8_stream(kout[r] + ((v + u * kWarp) << 3), o);
                }
            }
        }
        for (; v < nvec; v += kWarp) {                  // ragged tail of the row
            const f8 pv = ld8_keep(p + (v << 3));
#pragma unroll
            for (int r = 0; r < kRows; ++r) {
                const f8 kv = ld8_stream(kin[r] + (v << 3));
                f8 o;
#pragma unroll
                for (int c = 0; c < 8; ++c) {
                    o.v[c] = deflate1(kv.v[c], a[r], pv.v[c], inv_c);
                    acc[r] = __fmaf_rn(o.v[c], o.v[c], acc[r]);
                }
                if (lrow0 + r < nrows) st8_stream(kout[r] + (v << 3), o);
            }
        }
    }
    unsigned long long key = 0ull;
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
        const float g = warp_sum(acc[r]);
        if (l == r && any && lrow0 + r < nrows) {
            const int lr = lrow0 + r;
            const int32_t i = row0 + lr;
            // new diagonal entry, computed by the same instruction the sweep used
            const float diag = deflate1(Kin[(int64_t)lr * ld + i], a[r], p[i], inv_c);
            const bool masked = sel[lr] != 0 || (uint32_t)i == s;
            key = score_key(g, diag, mu, (uint32_t)i, masked, err);
        }
    }
    cta_key_max_to<kThreads>(key, keys + t, top2 ? top2 + ((int64_t)t * gridDim.x + blockIdx.x) * 2 : nullptr);
}

// ---------------------------------------------------------------------------
// col[lr] = K[lr][s_t] for the band's rows, s_t = keys[t] (sharded pivot exchange).
__global__ void pivot_column_kernel(const float* __restrict__ K, int64_t ld, int32_t nrows,
                                    const unsigned long long* __restrict__ keys, int32_t t,
                                    float* __restrict__ col) {
    const uint32_t s = key_index(keys[t]);
    for (int lr = blockIdx.x * blockDim.x + threadIdx.x; lr < nrows; lr += gridDim.x * blockDim.x)
        col[lr] = K[(int64_t)lr * ld + s];
}

}  // namespace bted
