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

// key_b(i) = (splitmix64(h_b + i) & 0xFFFFFFFF00000000) | i
__global__ void batch_keys_kernel(uint64_t P, uint64_t hb, uint64_t* __restrict__ keys) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P;
         i += (uint64_t)gridDim.x * blockDim.x)
        keys[i] = (splitmix64(hb + i) & 0xFFFFFFFF00000000ull) | i;
}

// the M smallest keys (sorted by key) -> their indices (low halves)
__global__ void low_half_kernel(const uint64_t* __restrict__ sorted, int64_t M, uint32_t* __restrict__ idx) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < M; j += (int64_t)gridDim.x * blockDim.x)
        idx[j] = (uint32_t)(sorted[j] & 0xFFFFFFFFull);
}

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

// negative entries are padding: they map to 0xFFFFFFFF, which sorts last
__global__ void i64_to_u32_kernel(const int64_t* __restrict__ in, int64_t n, uint32_t* __restrict__ out) {
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
        out[j] = in[j] < 0 ? 0xFFFFFFFFu : (uint32_t)in[j];
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

}  // namespace bted
