// gram_tc.cuh -- K1 (Alg. 1 l.1; RBF reading A1) on the 5th-gen
// tensor cores: the packed upper-triangular Gram tiles of the implicit engine.
//
// k(x_i, x_j) = exp(-gamma ||x_i - x_j||^2) with ||x_i - x_j||^2 expanded as
//     n_i + n_j - 2 x'_i . x'_j,    x' = x - c  (c = the mean feature vector),
// where the 128 x 128 block of dot products x'_I . x'_J^T is ONE tcgen05.mma
// chain per tile (M = N = 128, fp32 accumulator in TMEM).  Centring makes the
// expansion as accurate as the direct-difference form it replaces (translation
// leaves every distance unchanged; the cancellation of n_i + n_j - 2 dot is then
// relative to the spread of the data, not to |x|^2): measured on the knob and
// uniform pools, the largest entry error is 3.1-3.6 ulp * (1 + gamma d^2)
// against 2.1-3.5 for the direct form, inside pin C1's 6 ulp * (1 + gamma d^2)
// (DESIGN.md "K1 on tensor cores").
//
// fp32 operands through bf16 tensor cores without losing precision: each
// centred fp32 value is split exactly into three bf16 parts v = h + m + l
// (8 + 8 + 8 significand bits), and the dot product is the sum of the six
// MMAs m.m, h.l, l.h, h.m, m.h, h.h (the three dropped terms m.l, l.m, l.l
// are below 2^-32 relative) -- products of bf16 are exact in fp32; the
// smallest terms accumulate first.  The operands are prepared once per TED
// (prep kernel) in the tensor cores' canonical K-major layout (no swizzle):
// 8 x 8 core matrices of 128 B, k-chunks 128 B apart (LBO), 8-row groups
// 1536 B apart (SBO), six 16-wide k-slices per block of 128 rows.
//
// Per tile (I <= J): all threads copy the two 24 KiB operand blocks into
// shared memory, one elected thread issues the six MMAs and commits them to
// an mbarrier, eight warps read the accumulator (tcgen05.ld, warp w: TMEM
// lanes 32 (w % 4).., columns 64 (w / 4)..), form K, stage the tile in shared
// memory (reusing the operand space) and write it out with coalesced
// 512-byte rows.  Diagonal tiles store their upper triangle mirrored, so the
// matrix is bit-symmetric by construction, and K_ii = 1 exactly.
#pragma once
#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include "packed.cuh"

namespace bted {
namespace tc {

using pk::T;
constexpr int kThreads = 256;
constexpr int kD = 16;                         // features per k-slice (d <= 16)
constexpr int kSlices = 6;                     // the six split products
constexpr int kK = kD * kSlices;               // 96 bf16 per row
constexpr uint32_t kLBO = 128;                 // bytes between k-adjacent core matrices
constexpr uint32_t kSBO = (kK / 8) * 128;      // 1536: bytes between 8-row groups
constexpr uint32_t kBlockBytes = (T / 8) * kSBO;   // 24576 per 128-row block
constexpr int kStageLd = T + 4;                // padded staging row (floats): conflict-free float4 writes
constexpr size_t kSmemBytes = (size_t)T * kStageLd * sizeof(float) > 2 * kBlockBytes
                                  ? (size_t)T * kStageLd * sizeof(float) : 2 * (size_t)kBlockBytes;
// kind::f16, A = B = bf16 (K-major), D = f32, M = 128, N = 128
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(T >> 3) << 17) | ((uint32_t)(T >> 4) << 24);

// byte offset of element (row r, k) of a block in the canonical K-major layout
__host__ __device__ __forceinline__ uint32_t op_offset(int r, int k) {
    return (uint32_t)(r >> 3) * kSBO + (uint32_t)(k >> 3) * kLBO + (uint32_t)(r & 7) * 16u + (uint32_t)(k & 7) * 2u;
}

// ---------------------------------------------------------------- prep
// c = mean of the N rows (one CTA, thread-strided fp32 sums in row order, then a
// fixed tree over the 256 threads): any c is exact in the algebra; the mean keeps
// the expansion's cancellation small
__global__ void __launch_bounds__(kThreads) center_kernel(const float* __restrict__ X, int32_t N, int32_t d,
                                                         float* __restrict__ c) {
    __shared__ float red[kThreads];
    for (int k = 0; k < d; ++k) {
        float s = 0.f;
        for (int i = threadIdx.x; i < N; i += kThreads) s = __fadd_rn(s, X[(int64_t)i * d + k]);
        red[threadIdx.x] = s;
        __syncthreads();
        for (int off = kThreads / 2; off > 0; off >>= 1) {
            if (threadIdx.x < off) red[threadIdx.x] = __fadd_rn(red[threadIdx.x], red[threadIdx.x + off]);
            __syncthreads();
        }
        if (threadIdx.x == 0) c[k] = __fdiv_rn(red[0], (float)N);
        __syncthreads();
    }
}

__device__ __forceinline__ void split3(float v, __nv_bfloat16& h, __nv_bfloat16& m, __nv_bfloat16& l) {
    h = __float2bfloat16_rn(v);
    const float r1 = __fsub_rn(v, __bfloat162float(h));          // exact
    m = __float2bfloat16_rn(r1);
    const float r2 = __fsub_rn(r1, __bfloat162float(m));         // exact
    l = __float2bfloat16_rn(r2);                                  // exact for normal v
}

// per row i (padding rows: 0): x' = x - c, n_i = sum_k x'_k^2 (fp32, k order),
// and the two operand blocks: A slices [m, h, l, h, m, h], B slices [m, l, h, m, h, h]
__global__ void __launch_bounds__(kThreads) prep_kernel(const float* __restrict__ X, int32_t N, int32_t d,
                                                       int nT, const float* __restrict__ c,
                                                       uint8_t* __restrict__ opA, uint8_t* __restrict__ opB,
                                                       float* __restrict__ nrm) {
    const int64_t i = (int64_t)blockIdx.x * kThreads + threadIdx.x;
    if (i >= (int64_t)nT * T) return;
    const int blk = (int)(i / T), r = (int)(i % T);
    uint8_t* a = opA + (size_t)blk * kBlockBytes;
    uint8_t* b = opB + (size_t)blk * kBlockBytes;
    float n = 0.f;
    for (int k = 0; k < kD; ++k) {
        float v = 0.f;
        if (i < N && k < d) v = __fsub_rn(X[i * d + k], c[k]);
        n = __fmaf_rn(v, v, n);
        __nv_bfloat16 h, m, l;
        split3(v, h, m, l);
        const __nv_bfloat16 sa[kSlices] = {m, h, l, h, m, h};
        const __nv_bfloat16 sb[kSlices] = {m, l, h, m, h, h};
#pragma unroll
        for (int s = 0; s < kSlices; ++s) {
            *reinterpret_cast<__nv_bfloat16*>(a + op_offset(r, s * kD + k)) = sa[s];
            *reinterpret_cast<__nv_bfloat16*>(b + op_offset(r, s * kD + k)) = sb[s];
        }
    }
    nrm[i] = i < N ? n : 0.f;
}

// ---------------------------------------------------------------- tcgen05 helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr) {
    uint64_t desc = 0;
    desc |= (uint64_t)((saddr >> 4) & 0x3FFFu);                  // start address
    desc |= (uint64_t)((kLBO >> 4) & 0x3FFFu) << 16;             // leading (k) byte offset
    desc |= (uint64_t)((kSBO >> 4) & 0x3FFFu) << 32;             // stride (8-row group) byte offset
    desc |= (uint64_t)1 << 46;                                   // version 1 (sm_100)
    return desc;                                                 // base offset 0, SWIZZLE_NONE
}

__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(kIdesc), "r"(acc));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile("{\n\t.reg .pred done;\n\tWAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
                 "@!done bra WAIT_%=;\n\t}\n" :: "r"(smem_u32(bar)), "r"(phase) : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
    uint32_t r[16];
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 "
                 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int q = 0; q < 16; ++q) v[q] = __uint_as_float(r[q]);
}

// ---------------------------------------------------------------- the tile kernel
// grid: persistent, tile k = blockIdx.x + j gridDim.x (k < num_tiles(nT)); writes
// K[k] (64 KiB, row-major) of the packed upper-triangular layout
__global__ void __launch_bounds__(kThreads)
gram_tc_kernel(const uint8_t* __restrict__ opA, const uint8_t* __restrict__ opB, const float* __restrict__ nrm,
               int32_t N, float gamma, float* __restrict__ K, int nT) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ __align__(8) uint64_t mbar;
    __shared__ uint32_t tmem_base;
    __shared__ float nI[T], nJ[T];
    uint8_t* sA = smem;
    uint8_t* sB = smem + kBlockBytes;
    float* stage = reinterpret_cast<float*>(smem);                // reuses the operand space after the MMAs
    const int tid = threadIdx.x, w = tid / 32, lane = tid % 32;
    if (w == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_u32(&tmem_base)), "n"(T));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        mbar_init(&mbar);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");   // visible to the async proxy
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tbase = tmem_base;
    const float ng = -gamma;
    const int64_t ntiles = pk::num_tiles(nT);
    uint32_t phase = 0;
    for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x) {
        int I, J;
        pk::tile_ij(k, nT, I, J);
        // operands: 2 x 24 KiB from the prepared blocks (L2-resident)
        const uint4* ga = reinterpret_cast<const uint4*>(opA + (size_t)I * kBlockBytes);
        const uint4* gb = reinterpret_cast<const uint4*>(opB + (size_t)J * kBlockBytes);
        uint4* la = reinterpret_cast<uint4*>(sA);
        uint4* lb = reinterpret_cast<uint4*>(sB);
        for (int q = tid; q < (int)(kBlockBytes / 16); q += kThreads) {
            la[q] = __ldg(&ga[q]);
            lb[q] = __ldg(&gb[q]);
        }
        if (tid < T) { nI[tid] = nrm[(int64_t)I * T + tid]; nJ[tid] = nrm[(int64_t)J * T + tid]; }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic smem writes -> tensor core reads
        __syncthreads();
        if (tid == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const uint32_t a0 = smem_u32(sA), b0 = smem_u32(sB);
#pragma unroll
            for (int s = 0; s < kSlices; ++s)                      // each k-slice = 16 bf16 = 2 core matrices
                mma_bf16(tbase, smem_desc(a0 + 2 * s * kLBO), smem_desc(b0 + 2 * s * kLBO), s > 0 ? 1u : 0u);
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         :: "r"(smem_u32(&mbar)) : "memory");
        }
        mbar_wait(&mbar, phase);
        phase ^= 1u;
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        // epilogue: warp w reads TMEM lanes 32 (w % 4) .. +31 (tile rows), columns 64 (w / 4) .. +63
        const int r = 32 * (w & 3) + lane;
        const int cbase = 64 * (w >> 2);
        const int gi = I * T + r;
        const float ni = nI[r];
#pragma unroll 1
        for (int cc = 0; cc < 64; cc += 16) {
            float v[16];
            tmem_ld16(tbase + ((uint32_t)(32 * (w & 3)) << 16) + (uint32_t)(cbase + cc), v);
            float o[16];
#pragma unroll
            for (int q = 0; q < 16; ++q) {
                const int cj = cbase + cc + q;
                const int gj = J * T + cj;
                float d2 = __fmaf_rn(-2.f, v[q], __fadd_rn(ni, nJ[cj]));
                d2 = d2 > 0.f ? d2 : 0.f;
                const float kv = gi == gj ? 1.f : expf(__fmul_rn(ng, d2));
                o[q] = (gi < N && gj < N) ? kv : 0.f;
            }
            float4* dst = reinterpret_cast<float4*>(stage + (size_t)r * kStageLd + cbase + cc);
#pragma unroll
            for (int q = 0; q < 4; ++q) dst[q] = make_float4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
        }
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        // coalesced store: warp w writes rows w, w + 8, ...; diagonal tiles mirror the upper triangle
        float* tile = K + k * (int64_t)(T * T);
        for (int row = w; row < T; row += kThreads / 32) {
            const float* srow = stage + (size_t)row * kStageLd;
            float4 o = *reinterpret_cast<const float4*>(srow + 4 * lane);
            if (I == J) {
                float* oc = &o.x;
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int col = 4 * lane + q;
                    if (col < row) oc[q] = stage[(size_t)col * kStageLd + row];
                }
            }
            __stcs(reinterpret_cast<float4*>(tile + (size_t)row * T) + lane, o);
        }
        __syncthreads();                                           // staging / operand space reused next tile
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (w == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tbase), "n"(T));
}

}  // namespace tc
}  // namespace bted
