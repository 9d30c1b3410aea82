// xchg.cuh -- peer-memory exchanges of the in-library multi-GPU row-band TED
// (bted_select, num_devices = P > 1, BTED_FLAG_DENSE; SURVEY.md 8(e) mode 2).
//
// Each device owns a band of rows of the dense K (Alg. 1).
// Per step the bands exchange: the argmax key (max over the P band keys), the
// pivot column s (= row s by bit-symmetry; each band holds its slice) and, in
// the literal norm mode, the partial column norms (sum over the P bands).  A
// device publishes a value by finishing its producer kernel and bumping its
// release counter (im::publish_kernel); the consumer kernels below wait on all
// P counters and then read the peers' buffers directly (NVLink loads), reducing
// in rank order -- so every device computes bitwise the same result.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "implicit.cuh"

namespace bted {
namespace xg {

using im::kMaxDev;

struct Peers {
    const void* buf[kMaxDev];                 // device p's published buffer
    const unsigned long long* flag[kMaxDev];  // device p's release counter
    int P;
    unsigned long long expect;
    unsigned long long timeout_ns;
    __device__ __forceinline__ void wait(int* err) const {
        im::PeerQ q{};
        q.P = P;
        q.expect = expect;
        q.timeout_ns = timeout_ns;
        for (int p = 0; p < P; ++p) q.flag[p] = flag[p];
        im::wait_peers(q, err);
    }
};

// keys[t] = max over the P devices' keys[t] (their band maxima; forced keys win)
__global__ void keymax_kernel(Peers pk, int32_t t, unsigned long long* __restrict__ keys, int* __restrict__ err) {
    pk.wait(err);
    if (threadIdx.x == 0) {
        unsigned long long m = 0ull;
        for (int p = 0; p < pk.P; ++p) {
            const unsigned long long v = __ldcv(static_cast<const unsigned long long*>(pk.buf[p]) + t);
            m = v > m ? v : m;
        }
        keys[t] = m;
    }
}

// pivot[j] = K[s, j] from the bands' column slices: band q holds rows
// [q Bw, min(N, (q+1) Bw)) and published K[those rows, s]; entries >= N are 0
__global__ void gather_pivot_kernel(Peers pk, int64_t Bw, int64_t N, int64_t W, float* __restrict__ pivot,
                                    int* __restrict__ err) {
    pk.wait(err);
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < W; j += (int64_t)gridDim.x * blockDim.x) {
        float v = 0.f;
        if (j < N) {
            const int q = (int)(j / Bw);
            v = __ldcv(static_cast<const float*>(pk.buf[q]) + (j - (int64_t)q * Bw));
        }
        pivot[j] = v;
    }
}

// out[j] = sum over the P bands of their partial column norms, in rank order
__global__ void sum_colnorm_kernel(Peers pk, int64_t n, float* __restrict__ out, int* __restrict__ err) {
    pk.wait(err);
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        float a = __ldcv(static_cast<const float*>(pk.buf[0]) + j);
        for (int p = 1; p < pk.P; ++p) a = __fadd_rn(a, __ldcv(static_cast<const float*>(pk.buf[p]) + j));
        out[j] = a;
    }
}

}  // namespace xg
}  // namespace bted
