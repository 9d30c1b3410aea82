// gram_tc.cuh -- K1 (Alg. 1 l.1; RBF reading A1) on the 5th-gen
// tensor cores: the packed upper-triangular Gram tiles of the implicit engine.
//
// k(x_i, x_j) = exp(-gamma ||x_i - x_j||^2) with ||x_i - x_j||^2 expanded as
//     n_i + n_j - 2 x'_i . x'_j,    x' = x - c  (c = the mean feature vector),
// where the 128 x 128 blocks of dot products x'_I . x'_J^T are tcgen05.mma
// chains per tile (M = N = 128, fp32 accumulators in TMEM).  Centring makes the
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
// products h.l, l.h, m.m, h.m, m.h, h.h (the three dropped terms m.l, l.m, l.l
// are below 2^-32 relative) -- products of bf16 are exact in fp32; the smallest
// terms accumulate first.  ONE accumulator D = x'_I . x'_J^T, bit-symmetric by
// construction: each cross term sits in a single MMA instruction with both of
// its halves ([h | l] . [l | h] puts h_r l_c and l_r h_c in the same K = 16
// reduction, features 0-7 or 8-15), so under r <-> c every instruction reduces
// the same multiset of 16 products, and the tensor core's K = 16 reduction is a
// symmetric function of its products (measured on B200: D == D^T bitwise, the
// result independent of the operand's position in the tile and of the tile's
// orientation, exact duplicate rows bitwise equal -- scripts/tc_sym_probe.cu).
// The operands are prepared once per TED (prep kernel) in the tensor cores'
// canonical K-major layout (no swizzle): 8 x 8 core matrices of 128 B, 8-row
// groups 1536 B apart (SBO), twelve 8-wide k-chunks per row,
//     0 h0-7  1 l0-7  2 h8-15  3 l8-15  4 m0-7  5 m8-15
//     6 h0-7  7 m0-7  8 h8-15  9 m8-15  10 h0-7  11 h8-15,
// and every MMA addresses its two k-chunks (A and B) through the descriptor's
// start and leading byte offset (LBO), so one copy of the block serves both
// operand arrangements.
//
// Per tile (I <= J): the two 24 KiB operand blocks arrive by TMA bulk copies
// (mbarrier), one thread issues the six MMAs and commits them to an mbarrier,
// eight warps read the accumulator (tcgen05.ld), form K and store it; the
// next tile's copies overlap the epilogue.  The same K function (kval2) serves
// the recomputing tile pass (rc_pass.cuh), so the stored Gram and the
// recomputed one are the same numbers.
#pragma once
#include <cstdint>
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include "packed.cuh"

namespace bted {
namespace tc {

using pk::T;
constexpr int kThreads = 256;
constexpr int kD = 16;                         // features per k-slice (d <= 16)
constexpr int kSlices = 6;                     // the six MMAs (K = 16 each)
constexpr int kK = kD * kSlices;               // 96 bf16 per row (12 k-chunks of 8)
constexpr uint32_t kChunk = 128;               // bytes of one 8 x 8 core matrix (k-chunk)
constexpr uint32_t kSBO = (kK / 8) * 128;      // 1536: bytes between 8-row groups
constexpr uint32_t kBlockBytes = (T / 8) * kSBO;   // 24576 per 128-row block

// kind::f16, A = B = bf16 (K-major), D = f32, M = 128, N = 128
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(T >> 3) << 17) | ((uint32_t)(T >> 4) << 24);

// byte offset of element (row r, k) of a block in the canonical K-major layout
__host__ __device__ __forceinline__ uint32_t op_offset(int r, int k) {
    return (uint32_t)(r >> 3) * kSBO + (uint32_t)(k >> 3) * kChunk + (uint32_t)(r & 7) * 16u + (uint32_t)(k & 7) * 2u;
}
// MMA s: A = k-chunks (a0, a0 + 1), B = k-chunks (b0, b0 + blbo) of the block above
//   s = 0, 1: [h | l] . [l | h]   2: [m] . [m]   3, 4: [h | m] . [m | h]   5: [h] . [h]
__host__ __device__ __forceinline__ uint32_t mma_a0(int s) { return s == 0 ? 0u : s == 1 ? 2u : s == 2 ? 4u : s == 3 ? 6u : s == 4 ? 8u : 10u; }
__host__ __device__ __forceinline__ uint32_t mma_b0(int s) { return s == 0 ? 1u : s == 1 ? 3u : s == 2 ? 4u : s == 3 ? 7u : s == 4 ? 9u : 10u; }
__host__ __device__ __forceinline__ uint32_t mma_blbo(int s) { return s == 0 || s == 1 ? 5u : s == 3 ? 3u : s == 4 ? 2u : 1u; }

// ---------------------------------------------------------------- prep
// c = mean of the N rows (fixed-order partial sums: deterministic): any c is exact
// in the algebra; the mean keeps the expansion's cancellation small
constexpr int kCenterThreads = 256;
constexpr int kCenterBlocks = 64;
// pass 1: CTA b sums rows b*256 + tid, + 64*256, ... (in order) per thread, then a
// fixed tree over its threads -> part[b][k]
__global__ void __launch_bounds__(kCenterThreads) center_part_kernel(const float* __restrict__ X, int32_t N, int32_t d,
                                                                    float* __restrict__ part) {
    __shared__ float red[kCenterThreads / 32][kD];
    float s[kD];
#pragma unroll
    for (int k = 0; k < kD; ++k) s[k] = 0.f;
    for (int64_t i = (int64_t)blockIdx.x * kCenterThreads + threadIdx.x; i < N;
         i += (int64_t)kCenterBlocks * kCenterThreads) {
#pragma unroll
        for (int k = 0; k < kD; ++k)
            if (k < d) s[k] = __fadd_rn(s[k], X[i * d + k]);
    }
    const int w = threadIdx.x / 32, l = threadIdx.x % 32;
#pragma unroll
    for (int k = 0; k < kD; ++k) {
        float v = s[k];
        for (int off = 16; off > 0; off >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, off));
        if (l == 0) red[w][k] = v;
    }
    __syncthreads();
    if (threadIdx.x < kD) {
        float t = 0.f;
        for (int q = 0; q < kCenterThreads / 32; ++q) t = __fadd_rn(t, red[q][threadIdx.x]);
        part[blockIdx.x * kD + threadIdx.x] = t;
    }
}
// pass 2: c_k = (sum of the 64 partials in order) / N
__global__ void center_kernel(const float* __restrict__ part, int32_t N, int32_t d, float* __restrict__ c) {
    const int k = threadIdx.x;
    if (k >= d) return;
    float t = 0.f;
    for (int b = 0; b < kCenterBlocks; ++b) t = __fadd_rn(t, part[b * kD + k]);
    c[k] = __fdiv_rn(t, (float)N);
}

__device__ __forceinline__ void split3(float v, __nv_bfloat16& h, __nv_bfloat16& m, __nv_bfloat16& l) {
    h = __float2bfloat16_rn(v);
    const float r1 = __fsub_rn(v, __bfloat162float(h));          // exact
    m = __float2bfloat16_rn(r1);
    const float r2 = __fsub_rn(r1, __bfloat162float(m));         // exact
    l = __float2bfloat16_rn(r2);                                  // exact for normal v
}

// per row i (padding rows: 0): x' = x - c and its operand row (the twelve k-chunks above)
// opP (optional): a second copy with the rows of every block permuted for the
// recomputing pass (rc_pass.cuh): tile row r = 16a + 4qd + r' sits at row (TMEM lane)
// 32qd + 4a + r', so that a TMEM lane quarter holds every fourth 4-row group.
__host__ __device__ __forceinline__ int rc_lane_of_row(int r) { return 32 * ((r & 15) >> 2) + 4 * (r >> 4) + (r & 3); }
__host__ __device__ __forceinline__ int rc_row_of_lane(int L) { return 16 * ((L & 31) >> 2) + 4 * (L >> 5) + (L & 3); }
__global__ void __launch_bounds__(kThreads) prep_kernel(const float* __restrict__ X, int32_t N, int32_t d,
                                                       int nT, const float* __restrict__ c,
                                                       uint8_t* __restrict__ opA, uint8_t* __restrict__ opP = nullptr) {
    const int64_t i = (int64_t)blockIdx.x * kThreads + threadIdx.x;
    if (i >= (int64_t)nT * T) return;
    const int blk = (int)(i / T), r = (int)(i % T);
    uint8_t* a = opA + (size_t)blk * kBlockBytes;
    __nv_bfloat16 h[kD], m[kD], l[kD];
#pragma unroll
    for (int k = 0; k < kD; ++k) {
        float v = 0.f;
        if (i < N && k < d) v = __fsub_rn(X[i * d + k], c[k]);
        split3(v, h[k], m[k], l[k]);
    }
    // k-chunk q of a row = 8 bf16 = one 16-byte core-matrix row
    uint8_t* ap = opP ? opP + (size_t)blk * kBlockBytes : nullptr;
    const int rp = rc_lane_of_row(r);
    auto put = [&](int q, const __nv_bfloat16* v) {
        uint4 u;
        __nv_bfloat16* e = reinterpret_cast<__nv_bfloat16*>(&u);
#pragma unroll
        for (int x = 0; x < 8; ++x) e[x] = v[x];
        *reinterpret_cast<uint4*>(a + op_offset(r, 8 * q)) = u;
        if (ap) *reinterpret_cast<uint4*>(ap + op_offset(rp, 8 * q)) = u;
    };
    put(0, h); put(1, l); put(2, h + 8); put(3, l + 8); put(4, m); put(5, m + 8);
    put(6, h); put(7, m); put(8, h + 8); put(9, m + 8); put(10, h); put(11, h + 8);
}

// ---------------------------------------------------------------- tcgen05 helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
// paired fp32 arithmetic (one instruction for two IEEE round-to-nearest operations)
__device__ __forceinline__ unsigned long long f2pack(float lo, float hi) {
    return ((unsigned long long)__float_as_uint(hi) << 32) | __float_as_uint(lo);
}
__device__ __forceinline__ float f2lo(unsigned long long v) { return __uint_as_float((uint32_t)v); }
__device__ __forceinline__ float f2hi(unsigned long long v) { return __uint_as_float((uint32_t)(v >> 32)); }
__device__ __forceinline__ unsigned long long f2add(unsigned long long a, unsigned long long b) {
    unsigned long long d;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ unsigned long long f2sub(unsigned long long a, unsigned long long b) {
    unsigned long long d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ unsigned long long f2mul(unsigned long long a, unsigned long long b) {
    unsigned long long d;
    asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
// 2^x on the SFU (MUFU.EX2); the rounding of the scaled argument -g log2(e) d2 adds a
// relative error ~ g d2 ulp, inside pin C1's (1 + g d2) factor
__device__ __forceinline__ float ex2_approx(float x) {
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t lbo) {
    uint64_t desc = 0;
    desc |= (uint64_t)((saddr >> 4) & 0x3FFFu);                  // start address
    desc |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;              // leading (k) byte offset
    desc |= (uint64_t)((kSBO >> 4) & 0x3FFFu) << 32;             // stride (8-row group) byte offset
    desc |= (uint64_t)1 << 46;                                   // version 1 (sm_100)
    return desc;                                                 // base offset 0, SWIZZLE_NONE
}

__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(kIdesc), "r"(acc));
}


// tcgen05.ld of 16 consecutive columns without the wait (several loads share one
// tcgen05.wait::ld); the registers are valid only after tmem_wait_ld()
__device__ __forceinline__ void tmem_ld16_async(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 "
                 "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

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

// ---------------------------------------------------------------- the dot products
// D = x'_I . x'_J^T in TMEM columns [tD, tD + 128) (one accumulator, bit-symmetric:
// see the header).  The squared norms are D's own diagonal, n_r = D_rr, so that
// d2 = (n_r + n_c) - 2 D_rc is exactly 0 for identical points (K = 1, like the
// direct form).
// Accuracy guard: the expansion's rounding is relative to the centred norms, so the
// tensor-core Gram is used only when gamma * max_r n_r <= kGuard (the median-gamma
// knob and uniform pools: ~1-2); otherwise (badly scaled data, a huge gamma) the
// direct-difference kernel writes the Gram instead -- both kernels are launched and
// each reads the decision from *nmax_bits (max n_r, as non-negative float bits).
constexpr float kGuard = 4.f;
__device__ __forceinline__ bool tc_ok(const int* nmax_bits, float gamma) {
    return __fmul_rn(gamma, __int_as_float(*nmax_bits)) <= kGuard;
}
__device__ __forceinline__ void issue_gram_mmas(uint32_t tD, uint32_t aI, uint32_t aJ) {
#pragma unroll
    for (int s = 0; s < kSlices; ++s)
        mma_bf16(tD, smem_desc(aI + kChunk * mma_a0(s), kChunk), smem_desc(aJ + kChunk * mma_b0(s), kChunk * mma_blbo(s)),
                 s > 0 ? 1u : 0u);
}
// K for two columns from their dot products D and t = n_r + n_c (f32x2: one instruction per
// pair; the same IEEE operations per element as the scalar form, so symmetric inputs give
// symmetric K):  d2 = t - 2 D (one rounding, fma),  K = 2^(-gamma log2(e) max(d2, 0)).
// Every Gram entry of the tensor-core path -- stored (gram_tc_kernel) or recomputed in a
// tile pass (rc_pass.cuh) -- is this function of (D_rc, n_r + n_c).
__device__ __forceinline__ unsigned long long f2fma(unsigned long long a, unsigned long long b, unsigned long long c) {
    unsigned long long d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}
__device__ __forceinline__ void kval2(float D0, float D1, unsigned long long t2, unsigned long long g2, float& k0,
                                      float& k1) {
    const unsigned long long d2 = f2fma(f2pack(-2.f, -2.f), f2pack(D0, D1), t2);
    const unsigned long long y = f2mul(g2, f2pack(fmaxf(f2lo(d2), 0.f), fmaxf(f2hi(d2), 0.f)));
    k0 = ex2_approx(f2lo(y));
    k1 = ex2_approx(f2hi(y));
}

template <int kCols = T>
__device__ __forceinline__ void tmem_alloc(uint32_t* dst) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                 :: "r"(smem_u32(dst)), "n"(kCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
template <int kCols = T>
__device__ __forceinline__ void tmem_free(uint32_t base) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(base), "n"(kCols));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_u32(bar)) : "memory");
}

// n_r = D_rr for every row of every block (one CTA per block I: the diagonal tile's D)
__global__ void __launch_bounds__(kThreads)
gram_tc_norm_kernel(const uint8_t* __restrict__ opA, float* __restrict__ nrm, int* __restrict__ nmax_bits) {
    extern __shared__ __align__(1024) uint8_t smem[];            // [A_I]
    __shared__ __align__(8) uint64_t ldbar, mmabar;
    __shared__ uint32_t tmem_base;
    const int tid = threadIdx.x, w = tid / 32, lane = tid % 32, I = blockIdx.x;
    if (w == 0) tmem_alloc(&tmem_base);
    if (tid == 0) {
        pk::mbar_init(&ldbar, 1);
        pk::mbar_init(&mmabar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tbase = tmem_base;
    if (tid == 0) {
        pk::mbar_expect_tx(&ldbar, kBlockBytes);
        pk::bulk_g2s(smem, opA + (size_t)I * kBlockBytes, kBlockBytes, &ldbar);
    }
    pk::mbar_wait(&ldbar, 0);
    if (tid == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t a = smem_u32(smem);
        issue_gram_mmas(tbase, a, a);
        mma_commit(&mmabar);
    }
    pk::mbar_wait(&mmabar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (w < 4) {                                               // lane r = 32 w + lane needs column r
        const int r = 32 * w + lane;
        float d0[16], d1[16];
        const uint32_t lb = (uint32_t)(32 * w) << 16;
        tmem_ld16(tbase + lb + (uint32_t)(32 * w), d0);
        tmem_ld16(tbase + lb + (uint32_t)(32 * w + 16), d1);
        float n = 0.f;
#pragma unroll
        for (int q = 0; q < 16; ++q) {
            if (lane == q) n = d0[q];
            if (lane == 16 + q) n = d1[q];
        }
        nrm[(int64_t)I * T + r] = n;
        atomicMax(nmax_bits, __float_as_int(fmaxf(n, 0.f)));
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (w == 0) tmem_free(tbase);
}

// ---------------------------------------------------------------- the tile kernel
// Persistent, two CTAs (256 threads each) per SM: CTA b owns the contiguous tile
// range [b per, (b+1) per) of the packed upper triangle (row-major over I <= J), so
// consecutive tiles share the row block I (its operand block is reloaded only when
// I changes).  As soon as a tile's MMAs completed, the operand copies of the next
// tile are issued (cp.async.bulk), overlapping this tile's epilogue; the next
// tile's MMAs (into the other of two TMEM accumulators) are issued half-way through
// this tile's epilogue.  Epilogue, in two column halves: warp w reads TMEM lanes 32 (w % 4)
// .. +31 (tile rows) and 32 of the columns 64 (w / 4) .. +63 of D, forms K
// into a padded staging buffer (128 rows x 64 columns), and the CTA writes the half
// tile with coalesced 128-byte row segments; tiles on the ragged edge zero the
// padding.  The other CTA on the SM computes while this one stores.
constexpr int kTcThreads = 256;
constexpr int kStageCols = 64;
constexpr int kStageLd = kStageCols + 4;                         // conflict-free float4 staging rows
constexpr size_t kStageBytes = (size_t)T * kStageLd * sizeof(float);
constexpr size_t kTileSmemBytes = 2 * (size_t)kBlockBytes + kStageBytes;   // 48 KiB + 34 KiB

__global__ void __launch_bounds__(kTcThreads, 2)
gram_tc_kernel(const uint8_t* __restrict__ opA, const float* __restrict__ nrm,
               int32_t N, float gamma, float* __restrict__ K, int nT, const int* __restrict__ nmax_bits) {
    if (!tc_ok(nmax_bits, gamma)) return;                         // the direct-form kernel writes K
    extern __shared__ __align__(1024) uint8_t smem[];            // [A_I | A_J | stage]
    __shared__ __align__(8) uint64_t ldbar;
    __shared__ __align__(8) uint64_t mmabar;
    __shared__ uint32_t tmem_base;
    __shared__ __align__(16) float nIs[2][T];
    __shared__ __align__(16) float nJs[2][T];
    float* stage = reinterpret_cast<float*>(smem + 2 * kBlockBytes);
    const int tid = threadIdx.x, w = tid / 32, lane = tid % 32;
    const int64_t ntiles = pk::num_tiles(nT);
    const int64_t per = (ntiles + gridDim.x - 1) / gridDim.x;
    const int64_t k0 = (int64_t)blockIdx.x * per, k1 = k0 + per < ntiles ? k0 + per : ntiles;
    if (w == 0) tmem_alloc<2 * T>(&tmem_base);
    if (tid == 0) {
        pk::mbar_init(&ldbar, 1);
        pk::mbar_init(&mmabar, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tbase = tmem_base;
    const float ngl2e = __fmul_rn(-gamma, 1.4426950408889634f);   // exp(-g d2) = 2^(-g log2(e) d2)
    int I = 0, J = 0, loadedI = -1;
    if (k0 < k1) pk::tile_ij(k0, nT, I, J);
    // thread 0: the copies of tile (I, J); norms into slot b
    auto issue = [&](int I_, int J_, int b) {
        const bool newI = I_ != loadedI;
        pk::mbar_expect_tx(&ldbar, (newI ? kBlockBytes : 0u) + kBlockBytes + 2u * T * 4u);
        if (newI) pk::bulk_g2s(smem, opA + (size_t)I_ * kBlockBytes, kBlockBytes, &ldbar);
        pk::bulk_g2s(smem + kBlockBytes, opA + (size_t)J_ * kBlockBytes, kBlockBytes, &ldbar);
        pk::bulk_g2s(nIs[b], nrm + (int64_t)I_ * T, T * 4u, &ldbar);
        pk::bulk_g2s(nJs[b], nrm + (int64_t)J_ * T, T * 4u, &ldbar);
        loadedI = I_;
    };
    uint32_t ldph = 0u, mph = 0u;
    auto mma = [&](int b) {
        pk::mbar_wait(&ldbar, ldph);
        ldph ^= 1u;
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        issue_gram_mmas(tbase + (uint32_t)(b * T), smem_u32(smem), smem_u32(smem + kBlockBytes));
        mma_commit(&mmabar);
    };
    if (tid == 0 && k0 < k1) { issue(I, J, 0); mma(0); }
    const int q4 = w & 3, hh = w >> 2;                             // TMEM lane quarter, column half
    const int r = 32 * q4 + lane;
    const uint32_t lb = (uint32_t)(32 * q4) << 16;
    for (int64_t k = k0; k < k1; ++k) {
        const int b = (int)((k - k0) & 1);
        pk::mbar_wait(&mmabar, mph);
        mph ^= 1u;
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        int In = I, Jn = J + 1;                                    // the next tile of the range
        if (Jn == nT) { ++In; Jn = In; }
        if (tid == 0 && k + 1 < k1) issue(In, Jn, b ^ 1);          // operands free after MMA(k)
        const float ni = nIs[b][r];
        const float* nj = nJs[b];
        const bool edge = (I + 1) * T > N || (J + 1) * T > N;
        const bool rowv = I * T + r < N;
        float* tile = K + k * (int64_t)(T * T);
        const uint32_t tD = tbase + (uint32_t)(b * T) + lb;
        const unsigned long long g2 = f2pack(ngl2e, ngl2e);
#pragma unroll 1
        for (int half = 0; half < 2; ++half) {
            // part 1: 32 columns per warp, TMEM -> K values -> staging columns 32 hh .. +31
            {
                const int c0 = 64 * hh + 32 * half;                // tile column
                float* srow = stage + (size_t)r * kStageLd + 32 * hh;
#pragma unroll
                for (int cc = 0; cc < 32; cc += 16) {
                    uint32_t du[16];
                    tmem_ld16_async(tD + (uint32_t)(c0 + cc), du);
                    tmem_wait_ld();
                    float o[16];
#pragma unroll
                    for (int q = 0; q < 16; q += 2) {
                        const float2 njq = *reinterpret_cast<const float2*>(&nj[c0 + cc + q]);
                        kval2(__uint_as_float(du[q]), __uint_as_float(du[q + 1]),
                              f2add(f2pack(ni, ni), f2pack(njq.x, njq.y)), g2, o[q], o[q + 1]);
                    }
                    if (edge) {
#pragma unroll
                        for (int q = 0; q < 16; ++q)
                            if (!rowv || J * T + c0 + cc + q >= N) o[q] = 0.f;
                    }
                    float4* dst = reinterpret_cast<float4*>(srow + cc);
#pragma unroll
                    for (int q = 0; q < 4; ++q)
                        dst[q] = make_float4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
                }
            }
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
            __syncthreads();                                       // staging half complete
            if (half == 0 && tid == 0 && k + 1 < k1) mma(b ^ 1);   // MMA(k+1): the other accumulator
            // part 2: rows in pairs per warp instruction: lanes 0-15 row 2i, 16-31 row 2i+1;
            // lane group g = lane % 16: segment g / 8 (tile columns 64 (g / 8) + 32 half ..), 16 B each
#pragma unroll 2
            for (int row0 = 2 * w; row0 < T; row0 += 2 * (kTcThreads / 32)) {
                const int row = row0 + (lane >> 4), g = lane & 15, seg = g >> 3, e = (g & 7) * 4;
                const float4 v = *reinterpret_cast<const float4*>(stage + (size_t)row * kStageLd + 32 * seg + e);
                __stcs(reinterpret_cast<float4*>(tile + (size_t)row * T + 64 * seg + 32 * half + e), v);
            }
            __syncthreads();                                       // the staging half is reused
        }
        I = In;
        J = Jn;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (w == 0) tmem_free<2 * T>(tbase);
}

// ---------------------------------------------------------------- the tile kernel, warp-specialised
// Same tiles, same K values (the same kval2 on the same accumulator), restructured so
// the epilogue never waits on a copy or an MMA issue:
//   * a PRODUCER warp (warp 8, one lane) issues the operand copies (cp.async.bulk) and the
//     six MMAs of every tile: MMA(t) into TMEM accumulator t % 2 once the epilogue has
//     released it (acc_free) and tile t's operands have landed; then the copies of tile
//     t + 1 into operand slot (t + 1) % 2 (A_J and the norms are double-buffered; the A_I
//     block is reloaded, after MMA(t) completed, only when the row block changes);
//   * eight EPILOGUE warps read the accumulator (tcgen05.ld), form K (kval2) into two
//     16 KiB boxes [128 rows][32 floats] per half tile in the 128-byte swizzled layout the
//     tensor map names (16-byte chunk c of row r at chunk c ^ (r % 8): conflict-free for a
//     warp writing 32 consecutive rows), and one thread stores the boxes with
//     cp.async.bulk.tensor (TMA); a box is rewritten only after its bulk group READ it.
// tmap: K as a 2-D fp32 tensor [tiles * 128 rows][128 columns], box 32 x 128, SWIZZLE_128B.
constexpr int kBoxCols = 32;
constexpr size_t kBoxBytes = (size_t)T * kBoxCols * sizeof(float);          // 16 KiB
constexpr int kWsThreads = kTcThreads + 32;                                  // + the producer warp
constexpr size_t kTmaSmemBytes = 3 * (size_t)kBlockBytes + 2 * kBoxBytes;    // A_I, A_J x 2, 2 boxes: 104 KiB

__device__ __forceinline__ void tma_store_2d(const void* tmap, const void* src, int c0, int c1) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                 :: "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(smem_u32(src)) : "memory");
}
__device__ __forceinline__ void epi_sync() {                   // named barrier 1: the 8 epilogue warps
    asm volatile("bar.sync 1, %0;" :: "n"(kTcThreads) : "memory");
}

__global__ void __launch_bounds__(kWsThreads, 2)
gram_tc_tma_kernel(const uint8_t* __restrict__ opA, const float* __restrict__ nrm, int32_t N, float gamma, int nT,
                   const int* __restrict__ nmax_bits, const __grid_constant__ CUtensorMap tmap) {
    if (!tc_ok(nmax_bits, gamma)) return;                         // the direct-form kernel writes K
    extern __shared__ __align__(1024) uint8_t smem[];            // [A_I | A_J 0 | A_J 1 | box 0 | box 1]
    __shared__ __align__(8) uint64_t ldbar[2], mmabar[2], freebar[2];
    __shared__ uint32_t tmem_base;
    __shared__ __align__(16) float nIs[2][T];
    __shared__ __align__(16) float nJs[2][T];
    uint8_t* const aI = smem;
    uint8_t* const box = smem + 3 * kBlockBytes;
    const int tid = threadIdx.x, w = tid / 32, lane = tid % 32;
    const int64_t ntiles = pk::num_tiles(nT);
    const int64_t per = (ntiles + gridDim.x - 1) / gridDim.x;
    const int64_t k0 = (int64_t)blockIdx.x * per, k1 = k0 + per < ntiles ? k0 + per : ntiles;
    const int cnt = k0 < k1 ? (int)(k1 - k0) : 0;
    if (w == 0) tmem_alloc<2 * T>(&tmem_base);
    if (tid == 0) {
        for (int q = 0; q < 2; ++q) {
            pk::mbar_init(&ldbar[q], 1);
            pk::mbar_init(&mmabar[q], 1);
            pk::mbar_init(&freebar[q], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tbase = tmem_base;

    if (w == kTcThreads / 32) {                                   // ---- producer warp
        if (lane == 0 && cnt > 0) {
            int I = 0, J = 0, loadedI = -1;
            pk::tile_ij(k0, nT, I, J);
            // copies of tile (I_, J_) into operand slot s (A_I only when the row block changes)
            auto load = [&](int I_, int J_, int s) {
                const bool newI = I_ != loadedI;
                pk::mbar_expect_tx(&ldbar[s], (newI ? kBlockBytes : 0u) + kBlockBytes + 2u * T * 4u);
                if (newI) pk::bulk_g2s(aI, opA + (size_t)I_ * kBlockBytes, kBlockBytes, &ldbar[s]);
                pk::bulk_g2s(smem + (1 + s) * kBlockBytes, opA + (size_t)J_ * kBlockBytes, kBlockBytes, &ldbar[s]);
                pk::bulk_g2s(nIs[s], nrm + (int64_t)I_ * T, T * 4u, &ldbar[s]);
                pk::bulk_g2s(nJs[s], nrm + (int64_t)J_ * T, T * 4u, &ldbar[s]);
                loadedI = I_;
            };
            load(I, J, 0);
            for (int it = 0; it < cnt; ++it) {
                const int s = it & 1;
                // MMA(it): accumulator s released by epilogue(it - 2), operands of tile it landed
                if (it >= 2) pk::mbar_wait(&freebar[s], (uint32_t)((it - 2) >> 1) & 1u);
                pk::mbar_wait(&ldbar[s], (uint32_t)(it >> 1) & 1u);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                issue_gram_mmas(tbase + (uint32_t)(s * T), smem_u32(aI), smem_u32(smem + (1 + s) * kBlockBytes));
                mma_commit(&mmabar[s]);
                if (it + 1 < cnt) {                               // copies of tile it + 1 into slot s ^ 1
                    int In = I, Jn = J + 1;
                    if (Jn == nT) { ++In; Jn = In; }
                    // slot s ^ 1 (A_J, norms) was last read by epilogue(it - 1); A_I by MMA(it)
                    if (it >= 1) pk::mbar_wait(&freebar[s ^ 1], (uint32_t)((it - 1) >> 1) & 1u);
                    if (In != loadedI) pk::mbar_wait(&mmabar[s], (uint32_t)(it >> 1) & 1u);
                    load(In, Jn, s ^ 1);
                    I = In;
                    J = Jn;
                }
            }
        }
    } else {                                                      // ---- epilogue warps
        const float ngl2e = __fmul_rn(-gamma, 1.4426950408889634f);   // exp(-g d2) = 2^(-g log2(e) d2)
        const unsigned long long g2 = f2pack(ngl2e, ngl2e);
        const int q4 = w & 3, hh = w >> 2;                         // TMEM lane quarter, box (column half)
        const int r = 32 * q4 + lane;
        const uint32_t lb = (uint32_t)(32 * q4) << 16;
        uint8_t* const myrow = box + hh * kBoxBytes + (size_t)r * (kBoxCols * 4);
        int I = 0, J = 0;
        if (cnt > 0) pk::tile_ij(k0, nT, I, J);
        for (int it = 0; it < cnt; ++it) {
            const int s = it & 1;
            const int64_t k = k0 + it;
            pk::mbar_wait(&mmabar[s], (uint32_t)(it >> 1) & 1u);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            const float ni = nIs[s][r];
            const float* nj = nJs[s];
            const bool edge = (I + 1) * T > N || (J + 1) * T > N;
            const bool rowv = I * T + r < N;
            const uint32_t tD = tbase + (uint32_t)(s * T) + lb;
#pragma unroll 1
            for (int half = 0; half < 2; ++half) {
                // the boxes are free once the previous half's stores have read them
                if (tid == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                epi_sync();
                const int c0 = 64 * hh + 32 * half;                // tile column of box hh's column 0
#pragma unroll
                for (int cc = 0; cc < 32; cc += 16) {
                    uint32_t du[16];
                    tmem_ld16_async(tD + (uint32_t)(c0 + cc), du);
                    tmem_wait_ld();
                    float o[16];
#pragma unroll
                    for (int q = 0; q < 16; q += 2) {
                        const float2 njq = *reinterpret_cast<const float2*>(&nj[c0 + cc + q]);
                        kval2(__uint_as_float(du[q]), __uint_as_float(du[q + 1]),
                              f2add(f2pack(ni, ni), f2pack(njq.x, njq.y)), g2, o[q], o[q + 1]);
                    }
                    if (edge) {
#pragma unroll
                        for (int q = 0; q < 16; ++q)
                            if (!rowv || J * T + c0 + cc + q >= N) o[q] = 0.f;
                    }
#pragma unroll
                    for (int q = 0; q < 4; ++q) {                  // 16-byte chunk cc/4 + q, swizzled
                        const int ch = (cc >> 2) + q;
                        *reinterpret_cast<float4*>(myrow + ((ch ^ (r & 7)) << 4)) =
                            make_float4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
                    }
                }
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic writes -> async proxy
                asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
                epi_sync();                                        // both boxes complete
                if (tid == 0) {
                    if (half == 1) pk::mbar_arrive(&freebar[s]);   // accumulator s and norm slot s read
                    const int row = (int)(k * T);
                    tma_store_2d(&tmap, box, 32 * half, row);
                    tma_store_2d(&tmap, box + kBoxBytes, 64 + 32 * half, row);
                    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                }
            }
            if (++J == nT) { ++I; J = I; }
        }
        if (tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (w == 0) tmem_free<2 * T>(tbase);
}

}  // namespace tc
}  // namespace bted
