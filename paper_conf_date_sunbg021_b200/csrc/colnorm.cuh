// colnorm.cuh -- the north_star's literal norm exchange for the row-sharded TED
// ("norm_mode = 1"): every shard deflates its band of K
// (Alg. 1 l.5) and accumulates PARTIAL COLUMN norms
//   c_j = sum_{i in band} K'_ij^2          for every column j of the band,
// the caller all-reduces c (sum over shards, N floats), and each shard scores
// its own indices from the global column norm ||K'_j||^2 (Alg. 1 l.3,
// "K_v ... v's corresponding column").  The default symmetric
// mode (kernels.cuh) uses the band's row norms instead -- the same numbers by
// bit-symmetry, without the N-float all-reduce; this mode is the ablation.
//
// Layout: the dense band (rows x ld fp32, kernels.cuh).  A CTA owns one
// 256-column strip (lane l: 8 consecutive columns, 256-bit accesses) of one
// chunk of kColChunk rows; warp w walks rows w, w+8, ... of the chunk and keeps
// its 8 column sums in registers.  The 8 warps combine in a fixed order and
// write partial[chunk][j]; colnorm_reduce sums the chunks in order, so the
// local column norms are deterministic (independent of the grid schedule).
#pragma once
#include "kernels.cuh"

namespace bted {

constexpr int kColChunk = 512;     // rows per partial-sum chunk
constexpr int kColThreads = 256;   // 8 warps x 32 lanes x 8 columns = 256-column strip

// kDeflate: K_out = K_in - K_in[:,s] K_in[s,:] / (K_in[s,s] + mu) with s =
// keys[t-1] (the same deflate1 instruction as kernels.cuh, so the band is
// bitwise the band of the symmetric mode) and column partials of K_out;
// otherwise (t = 0) only the column partials of K_in.
template <bool kDeflate>
__global__ void __launch_bounds__(kColThreads)
deflate_colnorm_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int64_t ld,
                       int32_t row0, int32_t nrows, const float* __restrict__ pivot,
                       const unsigned long long* __restrict__ keys, int32_t t, float mu,
                       uint8_t* __restrict__ sel, float* __restrict__ partial) {
    constexpr int kWarps = kColThreads / kWarp;
    __shared__ float red[kWarps][kWarp * 8 + 1];
    const int w = threadIdx.x / kWarp, l = threadIdx.x % kWarp;
    const int64_t j0 = (int64_t)blockIdx.x * (kWarp * 8) + l * 8;   // first column of this lane
    const bool live = j0 < ld;                                       // ld % 32 == 0: whole groups
    const int c0 = blockIdx.y * kColChunk;
    const int c1 = min(nrows, c0 + kColChunk);

    float inv_c = 0.f;
    f8 pv;
#pragma unroll
    for (int c = 0; c < 8; ++c) pv.v[c] = 0.f;
    if (kDeflate) {
        const uint32_t s = key_index(keys[t - 1]);
        inv_c = __frcp_rn(__fadd_rn(pivot[s], mu));
        if (live) pv = ld8_keep(pivot + j0);
        if (blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0 && (int32_t)s >= row0 &&
            (int32_t)s < row0 + nrows)
            sel[(int32_t)s - row0] = 1;
    }
    float acc[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) acc[c] = 0.f;
    if (live) {
        int lr = c0 + w;
        constexpr int kU = 4;                                       // rows in flight per warp
        for (; lr + (kU - 1) * kWarps < c1; lr += kU * kWarps) {
            f8 kv[kU];
#pragma unroll
            for (int u = 0; u < kU; ++u) kv[u] = ld8_stream(Kin + (int64_t)(lr + u * kWarps) * ld + j0);
#pragma unroll
            for (int u = 0; u < kU; ++u) {
                if (kDeflate) {
                    const float a = pivot[row0 + lr + u * kWarps];  // K_in[i, s] = K_in[s, i]
#pragma unroll
                    for (int c = 0; c < 8; ++c) kv[u].v[c] = deflate1(kv[u].v[c], a, pv.v[c], inv_c);
                    st8_stream(Kout + (int64_t)(lr + u * kWarps) * ld + j0, kv[u]);
                }
#pragma unroll
                for (int c = 0; c < 8; ++c) acc[c] = __fmaf_rn(kv[u].v[c], kv[u].v[c], acc[c]);
            }
        }
        for (; lr < c1; lr += kWarps) {
            f8 kv = ld8_stream(Kin + (int64_t)lr * ld + j0);
            if (kDeflate) {
                const float a = pivot[row0 + lr];
#pragma unroll
                for (int c = 0; c < 8; ++c) kv.v[c] = deflate1(kv.v[c], a, pv.v[c], inv_c);
                st8_stream(Kout + (int64_t)lr * ld + j0, kv);
            }
#pragma unroll
            for (int c = 0; c < 8; ++c) acc[c] = __fmaf_rn(kv.v[c], kv.v[c], acc[c]);
        }
    }
#pragma unroll
    for (int c = 0; c < 8; ++c) red[w][l * 8 + c] = acc[c];
    __syncthreads();
    // thread x sums column x of the strip over the 8 warps in order
    const int64_t j = (int64_t)blockIdx.x * (kWarp * 8) + threadIdx.x;
    if (j < ld) {
        float g = 0.f;
#pragma unroll
        for (int ww = 0; ww < kWarps; ++ww) g = __fadd_rn(g, red[ww][threadIdx.x]);
        partial[(int64_t)blockIdx.y * ld + j] = g;
    }
}

// colnorm[j] = sum over chunks (in order) of partial[chunk][j].
__global__ void colnorm_reduce_kernel(const float* __restrict__ partial, int32_t nchunks, int64_t ld,
                                      float* __restrict__ colnorm) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < ld; j += (int64_t)gridDim.x * blockDim.x) {
        float g = 0.f;
        for (int c = 0; c < nchunks; ++c) g = __fadd_rn(g, partial[(int64_t)c * ld + j]);
        colnorm[j] = g;
    }
}

// Scores of the band's own indices i = row0 + lr from the all-reduced column
// norms: score_i = colnorm[i] / (K[lr][i] + mu), unselected only; packed
// argmax into keys[t] (the caller then all-reduces it with MAX).
__global__ void __launch_bounds__(256)
colnorm_scores_kernel(const float* __restrict__ K, int64_t ld, int32_t row0, int32_t nrows,
                      const float* __restrict__ colnorm, float mu, const uint8_t* __restrict__ sel,
                      unsigned long long* __restrict__ keys, int32_t t, int* __restrict__ err,
                      unsigned long long* __restrict__ top2 = nullptr) {
    unsigned long long best = 0ull, second = 0ull;           // this thread's two best keys (K4)
    for (int lr = blockIdx.x * blockDim.x + threadIdx.x; lr < nrows; lr += gridDim.x * blockDim.x) {
        const int32_t i = row0 + lr;
        const unsigned long long k =
            score_key(colnorm[i], K[(int64_t)lr * ld + i], mu, (uint32_t)i, sel[lr] != 0, err);
        second = k > best ? best : (k > second ? k : second);
        best = k > best ? k : best;
    }
    // top2 (K4): this CTA's two best keys at top2[2 * blockIdx.x], the layout
    // bted_shard_nearties reads (one slot pair per CTA of the step)
    cta_key_max_to<256>(best, keys + t, top2 ? top2 + 2 * (int64_t)blockIdx.x : nullptr, second);
}

}  // namespace bted
