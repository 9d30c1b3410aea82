// sample.cuh -- device side of Algorithm 2 l.2 (batch draws), the gather of
// a batch's features, and l.5 (union of the batch winners).  PAPER.md:156.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bted {

// splitmix64 output function (reading A10).
__host__ __device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
constexpr uint64_t kBatchStride = 0xD1B54A32D192ED03ull;

// Xb[j][:] = X[idx[j]][:]   (X_b = X[V_b]; one thread per element)
__global__ void gather_rows_kernel(const float* __restrict__ X, int32_t d, const uint32_t* __restrict__ idx,
                                   int64_t M, float* __restrict__ Xb) {
    const int64_t total = M * d;
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
         e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = e / d;
        const int32_t k = (int32_t)(e - j * d);
        Xb[e] = X[(int64_t)idx[j] * d + k];
    }
}

// winners[t] = pool_idx[ key_index(keys[t]) ], t < m  (positions -> pool rows)
__global__ void map_winners_kernel(const unsigned long long* __restrict__ keys, int32_t m,
                                   const uint32_t* __restrict__ pool_idx, int64_t* __restrict__ out) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < m) {
        const uint32_t pos = 0xFFFFFFFFu - (uint32_t)(keys[t] & 0xFFFFFFFFull);
        out[t] = (int64_t)pool_idx[pos];
    }
}

// the same for nb batches at once (blockIdx.y = batch): keys [nb][m], pool_idx [nb][M], out [nb][m]
__global__ void map_winners_batched_kernel(const unsigned long long* __restrict__ keys, int32_t m,
                                           const uint32_t* __restrict__ pool_idx, int64_t M,
                                           int64_t* __restrict__ out) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t b = blockIdx.y;
    if (t < m) {
        const uint32_t pos = 0xFFFFFFFFu - (uint32_t)(keys[b * m + t] & 0xFFFFFFFFull);
        out[b * m + t] = (int64_t)pool_idx[b * M + pos];
    }
}

// negative entries are padding: they map to 0xFFFFFFFF, which sorts last;
// an entry >= N (a bad device-side winner list) is dropped and flags kBadWinner
constexpr int kBadWinner = 16;
__global__ void i64_to_u32_kernel(const int64_t* __restrict__ in, int64_t n, int64_t N, uint32_t* __restrict__ out,
                                  int* __restrict__ err) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        const int64_t v = in[j];
        if (v >= N) atomicOr(err, kBadWinner);
        out[j] = (v < 0 || v >= N) ? 0xFFFFFFFFu : (uint32_t)v;
    }
}

// Alg. 2 l.5 for up to kUnionMax winners in ONE CTA (replaces the radix sort + unique
// + drop-padding launches): X_U = sorted unique(winners), negative entries are padding,
// entries >= N flag kBadWinner and are dropped.  Bitonic sort in shared memory, then a
// block-wide scan compacts the first occurrence of every index.
constexpr int kUnionMax = 4096;
constexpr int kUnionThreads = 1024;
__global__ void __launch_bounds__(kUnionThreads)
union_small_kernel(const int64_t* __restrict__ w, int n, int64_t N, uint32_t* __restrict__ out,
                   int* __restrict__ count, int* __restrict__ err) {
    __shared__ uint32_t key[kUnionMax];
    __shared__ int wsum[kUnionThreads / 32];
    const int tid = threadIdx.x;
    int np = 1;
    while (np < n) np <<= 1;
    for (int i = tid; i < np; i += kUnionThreads) {
        uint32_t k = 0xFFFFFFFFu;
        if (i < n) {
            const int64_t v = w[i];
            if (v >= N) atomicOr(err, 16);                  // kBadWinner
            if (v >= 0 && v < N) k = (uint32_t)v;
        }
        key[i] = k;
    }
    __syncthreads();
    for (int size = 2; size <= np; size <<= 1)
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int q = tid; q < np; q += kUnionThreads) {
                const int p = q ^ stride;
                if (p > q) {
                    const bool up = (q & size) == 0;
                    const uint32_t a = key[q], c = key[p];
                    if ((a > c) == up) { key[q] = c; key[p] = a; }
                }
            }
            __syncthreads();
        }
    // each thread owns 4 consecutive slots: keep = first occurrence and not padding
    uint32_t kv[4];
    int keep[4], cnt = 0;
#pragma unroll
    for (int x = 0; x < 4; ++x) {
        const int i = 4 * tid + x;
        kv[x] = i < np ? key[i] : 0xFFFFFFFFu;
        keep[x] = i < np && kv[x] != 0xFFFFFFFFu && (i == 0 || key[i - 1] != kv[x]);
        cnt += keep[x];
    }
    // exclusive scan of cnt over the block (warp shuffles, then the warp totals in order)
    const int lane = tid & 31, wi = tid >> 5;
    int incl = cnt;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
        const int o = __shfl_up_sync(0xffffffffu, incl, off);
        if (lane >= off) incl += o;
    }
    if (lane == 31) wsum[wi] = incl;
    __syncthreads();
    int base = 0, total = 0;
    for (int q = 0; q < kUnionThreads / 32; ++q) {
        if (q < wi) base += wsum[q];
        total += wsum[q];
    }
    int pos = base + incl - cnt;
#pragma unroll
    for (int x = 0; x < 4; ++x)
        if (keep[x]) out[pos++] = kv[x];
    if (tid == 0) *count = total;
}

// drop the padding value from the end of the unique list
__global__ void drop_pad_kernel(const uint32_t* __restrict__ uniq, int* __restrict__ count) {
    const int c = *count;
    if (c > 0 && uniq[c - 1] == 0xFFFFFFFFu) *count = c - 1;
}

__global__ void u32_to_i64_kernel(const uint32_t* __restrict__ in, int64_t n, int64_t* __restrict__ out) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
        out[j] = (int64_t)in[j];
}

// *bad = 1 if any of X[0..n) is NaN or +-inf (input validation on the device:
// a host scan of a 2^20 x 16 pool costs ~10 ms, this ~10 us)
__global__ void finite_check_kernel(const float* __restrict__ X, int64_t n, int* __restrict__ bad) {
    bool ok = true;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        ok &= isfinite(X[i]);
    if (__syncthreads_or(!ok) && threadIdx.x == 0) *bad = 1;
}

// ---------------------------------------------------------------------------
// Batch draws by radix SELECT instead of a full sort (all batches at once).
// V_b = the M smallest key_b(i); key order = (hash32, i).  hash32 is computed on
// the fly, nothing of size P is stored.  Two radix levels of 12 bits each:
//   sel_hist (lvl 0)  histogram of hash32 bits 31..20 per batch
//   sel_thresh        the bin b0* holding the M-th smallest key, count before it
//   sel_hist (lvl 1)  histogram of bits 19..8 of the keys inside bin b0*
//   sel_thresh        the sub-bin b1* holding it, count before it (cumulative)
//   sel_collect       keys whose top 24 bits are (b0*, b1*): the candidates
//   sel_finish        sort the candidates (bitonic, smem): the M-th smallest key k*
//   sel_count / sel_scan / sel_write   ordered compaction of {i : key_b(i) <= k*}:
//                each V_b comes out in ascending index order, no sort.
// The candidate bin holds ~P/2^24 keys (<= 128 on average for P < 2^31), far
// below kCandCap.  Should it ever overflow, sel_finish sets kSampleOverflow in
// the error word and the compaction kernels write nothing (kstar never read).
constexpr int kSelBins = 4096;
constexpr int kCandCap = 4096;
constexpr int kSampleOverflow = 8;     // error-word bit of a sampler candidate overflow

__device__ __forceinline__ uint64_t batch_hash_seed(uint64_t seed, int32_t b) {
    return splitmix64(seed + (uint64_t)b * kBatchStride);
}
__device__ __forceinline__ uint32_t hash32_of(uint64_t hb, uint64_t i) {
    return (uint32_t)(splitmix64(hb + i) >> 32);
}
// warp-aggregated atomic increment; every lane of the warp must call it
__device__ __forceinline__ unsigned warp_agg_inc(unsigned* ctr, bool pred) {
    const unsigned m = __ballot_sync(0xffffffffu, pred);
    const int lane = threadIdx.x & 31;
    unsigned base = 0;
    if (m) {
        const int leader = __ffs(m) - 1;
        if (lane == leader) base = atomicAdd(ctr, (unsigned)__popc(m));
        base = __shfl_sync(0xffffffffu, base, leader);
    }
    return base + (unsigned)__popc(m & ((1u << lane) - 1u));
}

// level 0 (bstar == nullptr): histogram of h >> 20; level 1: histogram of
// (h >> 8) & 0xFFF over the keys with h >> 20 == bstar[k]
__global__ void sel_hist_kernel(uint64_t P, uint64_t seed, int32_t b_begin, int32_t b_step,
                                const int* __restrict__ bstar, unsigned* __restrict__ hist) {
    __shared__ unsigned h[kSelBins];
    const int k = blockIdx.y;
    const uint64_t hb = batch_hash_seed(seed, b_begin + k * b_step);
    const unsigned b0 = bstar ? (unsigned)bstar[k] : 0u;
    for (int q = threadIdx.x; q < kSelBins; q += blockDim.x) h[q] = 0u;
    __syncthreads();
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t x = hash32_of(hb, i);
        if (!bstar) atomicAdd(&h[x >> 20], 1u);
        else if ((x >> 20) == b0) atomicAdd(&h[(x >> 8) & 0xFFFu], 1u);
    }
    __syncthreads();
    for (int q = threadIdx.x; q < kSelBins; q += blockDim.x)
        if (h[q]) atomicAdd(&hist[(int64_t)k * kSelBins + q], h[q]);
}

// one CTA (1024 threads) per batch: inclusive scan of the 4096 bins, first bin
// whose cumulative count reaches the rank M - below_in[k] (below_in nullable = 0);
// below_out[k] = below_in[k] + the count of the bins before it
__global__ void __launch_bounds__(1024)
sel_thresh_kernel(const unsigned* __restrict__ hist, int64_t M, const int* __restrict__ below_in,
                  int* __restrict__ bstar, int* __restrict__ below_out) {
    __shared__ unsigned part[1024];
    const int k = blockIdx.x, tid = threadIdx.x;
    const unsigned* hk = hist + (int64_t)k * kSelBins;
    const unsigned base = below_in ? (unsigned)below_in[k] : 0u;
    const unsigned need = (unsigned)M - base;
    unsigned v[4], s = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) { v[q] = hk[4 * tid + q]; s += v[q]; }
    part[tid] = s;
    __syncthreads();
    for (int off = 1; off < 1024; off <<= 1) {           // Hillis-Steele inclusive scan
        const unsigned a = tid >= off ? part[tid - off] : 0u;
        __syncthreads();
        part[tid] += a;
        __syncthreads();
    }
    unsigned c = tid ? part[tid - 1] : 0u;                // count before this thread's 4 bins
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        if (c < need && c + v[q] >= need) { bstar[k] = 4 * tid + q; below_out[k] = (int)(base + c); }
        c += v[q];
    }
}

// the candidates: keys whose top 24 hash bits are (b0*, b1*)
__global__ void sel_collect_kernel(uint64_t P, uint64_t seed, int32_t b_begin, int32_t b_step,
                                   const int* __restrict__ bstar0, const int* __restrict__ bstar1,
                                   uint64_t* __restrict__ cand, unsigned* __restrict__ ncand) {
    const int k = blockIdx.y;
    const uint64_t hb = batch_hash_seed(seed, b_begin + k * b_step);
    const unsigned top = ((unsigned)bstar0[k] << 12) | (unsigned)bstar1[k];
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    const uint64_t first = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint64_t iters = (P + stride - 1) / stride;      // uniform per warp: ballots stay converged
    for (uint64_t it = 0; it < iters; ++it) {
        const uint64_t i = first + it * stride;
        const bool in = i < P;
        const uint32_t h = in ? hash32_of(hb, i) : 0xFFFFFFFFu;
        const bool is_cand = in && (h >> 8) == top;
        const unsigned pc = warp_agg_inc(ncand + k, is_cand);
        if (is_cand && pc < (unsigned)kCandCap) cand[(int64_t)k * kCandCap + pc] = ((uint64_t)h << 32) | i;
    }
}

// one CTA (1024 threads) per batch: bitonic sort of the candidates in smem, then
// kstar[k] = the M-th smallest key of the batch (rank M - below[k] among them)
__global__ void __launch_bounds__(1024)
sel_finish_kernel(int64_t M, const int* __restrict__ below, const uint64_t* __restrict__ cand,
                  const unsigned* __restrict__ ncand, int* __restrict__ err, uint64_t* __restrict__ kstar) {
    __shared__ uint64_t s[kCandCap];
    const int k = blockIdx.x, tid = threadIdx.x;
    const unsigned n = ncand[k];
    const int need = (int)M - below[k];
    if (n > (unsigned)kCandCap || need < 1 || need > (int)n) {
        if (tid == 0) { atomicOr(err, kSampleOverflow); kstar[k] = 0ull; }
        return;
    }
    int np = 1;
    while (np < (int)n) np <<= 1;
    for (int q = tid; q < np; q += 1024) s[q] = q < (int)n ? cand[(int64_t)k * kCandCap + q] : ~0ull;
    __syncthreads();
    for (int size = 2; size <= np; size <<= 1)
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int q = tid; q < np; q += 1024) {
                const int p = q ^ stride;
                if (p > q) {
                    const bool up = (q & size) == 0;
                    const uint64_t a = s[q], c = s[p];
                    if ((a > c) == up) { s[q] = c; s[p] = a; }
                }
            }
            __syncthreads();
        }
    if (tid == 0) kstar[k] = s[need - 1];
}

// ---------------------------------------------------------------------------
// Ordered compaction: V_b = {i : key_b(i) <= kstar[b]} written in ascending i
// (no sort).  A CTA owns the index chunk [c*kCmpChunk, (c+1)*kCmpChunk).
constexpr int kCmpThreads = 256;
constexpr int kCmpChunk = kCmpThreads * 16;

__device__ __forceinline__ bool sel_pred(uint64_t hb, uint64_t i, uint64_t P, uint64_t kstar) {
    return i < P && ((((uint64_t)hash32_of(hb, i)) << 32) | i) <= kstar;
}

__global__ void __launch_bounds__(kCmpThreads)
sel_count_kernel(uint64_t P, uint64_t seed, int32_t b_begin, int32_t b_step, const uint64_t* __restrict__ kstar,
                 unsigned* __restrict__ cnt, const int* __restrict__ err) {
    __shared__ unsigned red[kCmpThreads / 32];
    const int k = blockIdx.y, G = gridDim.x;
    if (*err & kSampleOverflow) { if (threadIdx.x == 0) cnt[(int64_t)k * G + blockIdx.x] = 0u; return; }
    const uint64_t hb = batch_hash_seed(seed, b_begin + k * b_step), ks = kstar[k];
    const uint64_t base = (uint64_t)blockIdx.x * kCmpChunk;
    unsigned c = 0;
#pragma unroll 4
    for (int q = 0; q < kCmpChunk / kCmpThreads; ++q) c += sel_pred(hb, base + q * kCmpThreads + threadIdx.x, P, ks);
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) c += __shfl_xor_sync(0xffffffffu, c, off);
    if (threadIdx.x % 32 == 0) red[threadIdx.x / 32] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned t = 0;
        for (int w = 0; w < kCmpThreads / 32; ++w) t += red[w];
        cnt[(int64_t)k * G + blockIdx.x] = t;
    }
}

// per batch (one CTA of 1024 threads): exclusive scan of the G chunk counts, in place
__global__ void __launch_bounds__(1024) sel_scan_kernel(unsigned* __restrict__ cnt, int G) {
    __shared__ unsigned part[1024];
    unsigned* c = cnt + (int64_t)blockIdx.x * G;
    unsigned carry = 0;
    for (int b0 = 0; b0 < G; b0 += 1024) {
        const int q = b0 + threadIdx.x;
        const unsigned v = q < G ? c[q] : 0u;
        part[threadIdx.x] = v;
        __syncthreads();
        for (int off = 1; off < 1024; off <<= 1) {
            const unsigned a = threadIdx.x >= off ? part[threadIdx.x - off] : 0u;
            __syncthreads();
            part[threadIdx.x] += a;
            __syncthreads();
        }
        if (q < G) c[q] = carry + part[threadIdx.x] - v;
        const unsigned tot = part[1023];
        __syncthreads();
        carry += tot;
    }
}

__global__ void __launch_bounds__(kCmpThreads)
sel_write_kernel(uint64_t P, uint64_t seed, int32_t b_begin, int32_t b_step, const uint64_t* __restrict__ kstar,
                 const unsigned* __restrict__ off, int64_t M, uint32_t* __restrict__ out, const int* __restrict__ err) {
    __shared__ unsigned wcount[kCmpThreads / 32];
    const int k = blockIdx.y, G = gridDim.x, w = threadIdx.x / 32, l = threadIdx.x % 32;
    if (*err & kSampleOverflow) return;
    const uint64_t hb = batch_hash_seed(seed, b_begin + k * b_step), ks = kstar[k];
    const uint64_t base = (uint64_t)blockIdx.x * kCmpChunk;
    unsigned pos = off[(int64_t)k * G + blockIdx.x];
    uint32_t* o = out + (int64_t)k * M;
    for (int q = 0; q < kCmpChunk / kCmpThreads; ++q) {
        const uint64_t i = base + q * kCmpThreads + threadIdx.x;
        const bool p = sel_pred(hb, i, P, ks);
        const unsigned m = __ballot_sync(0xffffffffu, p);
        if (l == 0) wcount[w] = __popc(m);
        __syncthreads();
        unsigned before = 0, tot = 0;
#pragma unroll
        for (int ww = 0; ww < kCmpThreads / 32; ++ww) {
            before += ww < w ? wcount[ww] : 0u;
            tot += wcount[ww];
        }
        const unsigned at = pos + before + __popc(m & ((1u << l) - 1u));
        if (p && at < (unsigned)M) o[at] = (uint32_t)i;
        pos += tot;
        __syncthreads();
    }
}

}  // namespace bted
