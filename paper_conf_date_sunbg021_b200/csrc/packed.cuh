// packed.cuh -- packed-symmetric TED kernels.
//
// K is stored once: only the upper-triangular T x T tiles (I <= J) of the
// N x N matrix, each tile contiguous (row-major, 64 KiB at T = 128), tiles in
// row-major order over the upper triangle.  Padding rows/columns (>= N) are
// exactly 0.  A step of Alg. 1 then streams 4 N^2 bytes
// (+ the diagonal tiles' duplicated halves) instead of 8 N^2:
//
//   K2p: tile (I,J) <- tile - p_I p_J^T / (k(s,s)+mu)  (product first, as dense)
//        row partials    P[J][i] = sum_{j in J} K_ij^2     (i in block I)
//        column partials P[I][j] = sum_{i in I} K_ij^2     (j in block J, I < J)
//   fin: ||K_v||^2 = sum_J P[J][v] in J order, because block (I,J), J < I, is
//        the transpose of the stored tile (J,I); score and masked argmax.
//
// Every element value is bitwise the same as in the dense layout (same
// operands, same instruction).  Row and column partials use ONE canonical
// 128-term summation tree (groups of 4 consecutive terms, then a
// 32-leaf butterfly), so a row's norm does not depend on whether its
// partials came from rows or columns of stored tiles: exact duplicate points
// get bitwise-equal scores and tie to the lowest index (reading A5).
//
// K2p is a TMA pipeline: one producer warp streams tiles into a 3-stage
// shared-memory ring with cp.async.bulk (mbarrier complete_tx), eight
// consumer warps update them and write the new tile with 128-bit streaming
// stores.  Pivot segments (row s of K_in restricted to a tile's row/column
// block) are read straight from K_in: no pivot-extraction kernel.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "kernels.cuh"

namespace bted {
namespace pk {

constexpr int T = 128;                 // tile edge
constexpr int kConsumers = 256;        // 8 consumer warps
constexpr int kTileBytes = T * T * 4;  // 64 KiB
constexpr int kGroups = T / 4;         // 32 groups of 4 rows per tile

__host__ __device__ __forceinline__ int64_t tile_offset(int I, int J, int nT) {
    // tiles of rows 0..I-1 precede row I: sum_{i<I} (nT - i)
    return (int64_t)I * nT - (int64_t)I * (I - 1) / 2 + (J - I);
}
__host__ __device__ __forceinline__ int64_t num_tiles(int nT) { return (int64_t)nT * (nT + 1) / 2; }

// tile linear index -> (I, J) (row-major over the upper triangle)
__device__ __forceinline__ void tile_ij(int64_t k, int nT, int& I, int& J) {
    double a = 2.0 * nT + 1.0;
    int i = (int)((a - sqrt(a * a - 8.0 * (double)k)) * 0.5);
    if (i < 0) i = 0;
    if (i > nT - 1) i = nT - 1;
    while (i > 0 && tile_offset(i, i, nT) > k) --i;
    while (i < nT - 1 && tile_offset(i + 1, i + 1, nT) <= k) ++i;
    I = i;
    J = i + (int)(k - tile_offset(i, i, nT));
}

// element (i, j) of the symmetric matrix in packed storage
__device__ __forceinline__ int64_t packed_index(int i, int j, int nT) {
    const int I = i / T, J = j / T;
    return I <= J ? tile_offset(I, J, nT) * (T * T) + (int64_t)(i % T) * T + (j % T)
                  : tile_offset(J, I, nT) * (T * T) + (int64_t)(j % T) * T + (i % T);
}

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n}"
        :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
// same, with an L2 eviction-priority policy (createpolicy) for streamed data
__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy) : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ float ld_hint(const float* p, uint64_t policy) {
    float v;
    asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(policy));
    return v;
}
__device__ __forceinline__ float4 ld4_hint(const float* p, uint64_t policy) {
    float4 v;
    asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(policy));
    return v;
}

__device__ __forceinline__ void consumer_sync() {       // named barrier 1: the 256 consumer threads
    asm volatile("bar.sync 1, %0;" :: "n"(kConsumers) : "memory");
}

// ------------------------------------------------------------------ f32x2 (sm_100 FADD2 / FFMA2)
__device__ __forceinline__ unsigned long long pack2(float lo, float hi) {
    return ((unsigned long long)__float_as_uint(hi) << 32) | (unsigned long long)__float_as_uint(lo);
}
__device__ __forceinline__ void unpack2(unsigned long long v, float& lo, float& hi) {
    lo = __uint_as_float((unsigned)(v & 0xFFFFFFFFull));
    hi = __uint_as_float((unsigned)(v >> 32));
}
__device__ __forceinline__ unsigned long long sub2(unsigned long long a, unsigned long long b) {
    unsigned long long d;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
    return d;
}
__device__ __forceinline__ unsigned long long fma2(unsigned long long a, unsigned long long b, unsigned long long c) {
    unsigned long long d;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
    return d;
}

// ------------------------------------------------------------------ canonical sums
// group of 4 consecutive terms: ((v0^2 + v1^2) + v2^2) + v3^2 with fused steps
__device__ __forceinline__ float group4(float v0, float v1, float v2, float v3) {
    float g = __fmul_rn(v0, v0);
    g = __fmaf_rn(v1, v1, g);
    g = __fmaf_rn(v2, v2, g);
    return __fmaf_rn(v3, v3, g);
}
// 32-leaf butterfly over groups held by smem column (stride T): same tree as warp_sum
__device__ __forceinline__ float tree32_smem(const float* g, int stride) {
    float h[kGroups];
#pragma unroll
    for (int q = 0; q < kGroups; ++q) h[q] = g[q * stride];
#pragma unroll
    for (int off = 16; off > 0; off >>= 1)
#pragma unroll
        for (int q = 0; q < off; ++q) h[q] = __fadd_rn(h[q], h[q + off]);
    return h[0];
}

// Per-lane state while a warp walks its 16 rows of a tile (lane l owns columns 4l..4l+3).
struct RowWalk {
    float cg[4];     // running group-of-4-rows sums for the lane's 4 columns
    float rowsum;    // lane l < 16: partial of row 16w + l
};

// one row (index rr within the warp's 16) of new values o -> partials
__device__ __forceinline__ void walk_row(RowWalk& a, int rr, int l, const float4& o, float (*colg)[T], int w,
                                         bool want_cols) {
    float rp = group4(o.x, o.y, o.z, o.w);
    rp = warp_sum(rp);                                   // butterfly over the 32 groups of the row
    if (l == rr) a.rowsum = rp;
    if (want_cols) {
        if ((rr & 3) == 0) {
            a.cg[0] = __fmul_rn(o.x, o.x); a.cg[1] = __fmul_rn(o.y, o.y);
            a.cg[2] = __fmul_rn(o.z, o.z); a.cg[3] = __fmul_rn(o.w, o.w);
        } else {
            a.cg[0] = __fmaf_rn(o.x, o.x, a.cg[0]); a.cg[1] = __fmaf_rn(o.y, o.y, a.cg[1]);
            a.cg[2] = __fmaf_rn(o.z, o.z, a.cg[2]); a.cg[3] = __fmaf_rn(o.w, o.w, a.cg[3]);
        }
        if ((rr & 3) == 3) {                            // group (16w + rr) / 4 complete
            const int q = 4 * w + (rr >> 2);
            *reinterpret_cast<float4*>(&colg[q][4 * l]) = make_float4(a.cg[0], a.cg[1], a.cg[2], a.cg[3]);
        }
    }
}

// After all 8 warps walked the tile (and colg is complete, consumer_sync
// done by the caller): write row partials and the column tree.
__device__ __forceinline__ void write_partials(float* P, int64_t NP, int I, int J, int w, int l, const RowWalk& a,
                                               float (*colg)[T], int tid) {
    if (l < 16) P[(int64_t)J * NP + (int64_t)I * T + 16 * w + l] = a.rowsum;
    if (I != J && tid < T) P[(int64_t)I * NP + (int64_t)J * T + tid] = tree32_smem(&colg[0][tid], T);
}

// ------------------------------------------------------------------ K1p: Gram tiles
// Alg. 1 l.1 on the upper-triangular tiles (+ the partials of the first l.3).
// One CTA (256 threads) per tile in a persistent loop.  Lane l keeps the
// features of its 4 columns in registers (kD <= 32); the rows' features
// are smem broadcasts.
// ------------------------------------------------------------------ fin: scores + argmax
// Alg. 1 l.3 from the partials: g_i = sum_J P[J][i], score = g / (k(i,i) + mu)
// with the new diagonal read back from the diagonal tile, masked (selected /
// the pivot / padding), packed key -> atomicMax(key_out).  The sum runs in a
// fixed order that depends on nT only (the same for every row: exact
// duplicates still tie): 8 contiguous J ranges, each summed sequentially,
// then the 8 range sums in order.  CTA = 32 rows x 8 ranges (lane = row, so
// every load is a coalesced 128-byte row of P); all of a thread's loads are
// issued before its adds.
constexpr int kFinThreads = 256;
constexpr int kFinRows = 32;
__global__ void __launch_bounds__(kFinThreads)
finalize_packed_kernel(const float* __restrict__ P, int nT, int32_t N, const float* __restrict__ K, float mu,
                       const uint8_t* __restrict__ sel, const unsigned long long* __restrict__ keys, int32_t t,
                       unsigned long long* __restrict__ key_out, int* __restrict__ err,
                       unsigned long long* __restrict__ top2) {
    __shared__ float part[8][kFinRows];
    const int lane = threadIdx.x % 32, w = threadIdx.x / 32;
    const int64_t NP = (int64_t)nT * T;
    const int i = blockIdx.x * kFinRows + lane;            // row (< nT*T by construction)
    const uint32_t s = t > 0 ? key_index(keys[t - 1]) : 0xFFFFFFFFu;
    // warp 0 fetches the row's new diagonal entry and mask up front (off the critical path)
    float diag = 0.f;
    bool sl = true;
    if (w == 0 && i < N) {
        const int B = i / T, r = i % T;
        diag = K[tile_offset(B, B, nT) * (T * T) + (int64_t)r * T + r];
        sl = sel[i] != 0;
    }
    const int per = (nT + 7) / 8;
    const int j0 = min(nT, w * per), j1 = min(nT, j0 + per);
    const float* src = P + i;
    float acc = 0.f;
    int J = j0;
    for (; J + 16 <= j1; J += 16) {
        float v[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) v[q] = src[(int64_t)(J + q) * NP];
#pragma unroll
        for (int q = 0; q < 16; ++q) acc = __fadd_rn(acc, v[q]);
    }
    for (; J < j1; ++J) acc = __fadd_rn(acc, src[(int64_t)J * NP]);
    part[w][lane] = acc;
    __syncthreads();
    if (w == 0) {
        unsigned long long key = 0ull;
        if (i < N) {
            float g = part[0][lane];
#pragma unroll
            for (int q = 1; q < 8; ++q) g = __fadd_rn(g, part[q][lane]);
            const bool masked = sl || (uint32_t)i == s;
            key = score_key(g, diag, mu, (uint32_t)i, masked, err);
        }
        const unsigned long long k1 = warp_max_u64(key);
        if (top2) {                                    // the CTA's best two keys (K4 near-tie check)
            const unsigned long long k2 = warp_max_u64(key == k1 ? 0ull : key);
            if (lane == 0) {
                top2[((int64_t)t * gridDim.x + blockIdx.x) * 2] = k1;
                top2[((int64_t)t * gridDim.x + blockIdx.x) * 2 + 1] = k2;
            }
        }
        if (lane == 0 && k1) atomicMax(key_out, k1);
    }
}

// ------------------------------------------------------------------ K2p: TMA deflate
// kSub rows of a tile per pipeline stage (kSub x 128 fp32), kStagesOf(kSub)
// stages in a ~192 KiB ring.  kHints: evict-first policy on the streamed
// tiles and evict-last on the pivot segments (reused by every tile of a
// block row/column), pivot segments prefetched one tile ahead.
__host__ __device__ constexpr int kStagesOf(int sub) { return (192 * 1024) / (sub * T * 4); }
__host__ __device__ constexpr size_t k2p_smem_bytes(int sub) {
    return (size_t)kStagesOf(sub) * sub * T * 4 + 2 * (size_t)kGroups * T * 4 + 2 * kStagesOf(sub) * 8;
}

template <int kSub, bool kHints>
__global__ void __launch_bounds__(kConsumers + kWarp, 1)
deflate_packed_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int nT, int32_t N,
                      float* __restrict__ P, const unsigned long long* __restrict__ keys, int32_t t, float mu,
                      uint8_t* __restrict__ sel) {
    constexpr int kS = kStagesOf(kSub);
    constexpr int kStageFloats = kSub * T;
    constexpr int kSubs = T / kSub;             // stages per tile
    constexpr int kRW = kSub / 8;               // rows per warp per stage
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    float* stage = reinterpret_cast<float*>(smem_raw);                       // [kS][kSub*T]
    float (*colg)[kGroups][T] = reinterpret_cast<float (*)[kGroups][T]>(smem_raw + (size_t)kS * kStageFloats * 4);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)kS * kStageFloats * 4 + 2 * kGroups * T * 4);
    uint64_t* empty = full + kS;

    const int tid = threadIdx.x;
    const int64_t ntiles = num_tiles(nT);
    if (tid == 0) {
        for (int q = 0; q < kS; ++q) { mbar_init(full + q, 1); mbar_init(empty + q, kConsumers / kWarp); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (tid >= kConsumers) {
        // ---------------- producer warp: one elected lane streams the tiles, kSub rows per stage
        if (tid == kConsumers) {
            const uint64_t pol = policy_evict_first();    // K streams through L2 once per step
            int n = 0;
            for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x) {
                const float* src = Kin + k * (int64_t)(T * T);
                for (int sb = 0; sb < kSubs; ++sb, ++n) {
                    const int st = n % kS;
                    const uint32_t ph = (uint32_t)(n / kS) & 1u;
                    mbar_wait(empty + st, ph ^ 1u);
                    mbar_expect_tx(full + st, kStageFloats * 4);
                    if (kHints) bulk_g2s_hint(stage + st * kStageFloats, src + sb * kStageFloats, kStageFloats * 4,
                                              full + st, pol);
                    else bulk_g2s(stage + st * kStageFloats, src + sb * kStageFloats, kStageFloats * 4, full + st);
                }
            }
        }
        return;
    }

    // ---------------- consumers
    const int w = tid / kWarp, l = tid % kWarp;
    const int64_t NP = (int64_t)nT * T;
    const uint32_t s = key_index(keys[t - 1]);
    const int S = (int)(s / T), rs = (int)(s % T);
    const float inv_c = __frcp_rn(__fadd_rn(Kin[packed_index((int)s, (int)s, nT)], mu));   // 1/(k(s,s)+mu)
    if (blockIdx.x == 0 && tid == 0 && (int32_t)s < N) sel[s] = 1;
    // K_in[s, B*T + c]: a contiguous row segment of tile (S,B) if S <= B, else a column of tile (B,S)
    const uint64_t keep = kHints ? policy_evict_last() : 0ull;
    auto ldf = [&](const float* p) -> float { return kHints ? ld_hint(p, keep) : __ldg(p); };
    auto seg = [&](int B, int c) -> float {
        return S <= B ? ldf(Kin + tile_offset(S, B, nT) * (T * T) + (int64_t)rs * T + c)
                      : ldf(Kin + tile_offset(B, S, nT) * (T * T) + (int64_t)c * T + rs);
    };
    // the warp's 16 rows of a tile: row(l) for l < 16
    auto my_row = [&](int q) { return (q / kRW) * kSub + w * kRW + (q % kRW); };
    auto load_segs = [&](int64_t k, float& pr, float4& pc) {
        int I, J;
        tile_ij(k, nT, I, J);
        pr = l < 16 ? seg(I, my_row(l)) : 0.f;                 // a_i for the warp's 16 rows
        if (S <= J) {
            const float* p = Kin + tile_offset(S, J, nT) * (T * T) + (int64_t)rs * T + 4 * l;
            pc = kHints ? ld4_hint(p, keep) : __ldg(reinterpret_cast<const float4*>(p));
        } else {
            pc.x = seg(J, 4 * l); pc.y = seg(J, 4 * l + 1); pc.z = seg(J, 4 * l + 2); pc.w = seg(J, 4 * l + 3);
        }
    };
    float pr_next = 0.f;
    float4 pc_next = make_float4(0.f, 0.f, 0.f, 0.f);
    if ((int64_t)blockIdx.x < ntiles) load_segs(blockIdx.x, pr_next, pc_next);
    int n = 0, tcount = 0;
    for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x, ++tcount) {
        int I, J;
        tile_ij(k, nT, I, J);
        float (*cg)[T] = colg[tcount & 1];
        const float pr_l = pr_next;
        const float4 pc = pc_next;
        if (k + gridDim.x < ntiles) load_segs(k + gridDim.x, pr_next, pc_next);   // next tile's segments
        float* gout = Kout + k * (int64_t)(T * T);
        RowWalk a;
        a.rowsum = 0.f;
        for (int sb = 0; sb < kSubs; ++sb, ++n) {
            const int st = n % kS;
            const uint32_t ph = (uint32_t)(n / kS) & 1u;
            mbar_wait(full + st, ph);
            const float* sm = stage + st * kStageFloats;
#pragma unroll
            for (int rr = 0; rr < kRW; ++rr) {
                const int q = sb * kRW + rr;                       // the warp's q-th row of the tile
                const int r = sb * kSub + w * kRW + rr;            // row within the tile
                const float ai = __shfl_sync(0xffffffffu, pr_l, q);
                const float4 kv = *reinterpret_cast<const float4*>(sm + (w * kRW + rr) * T + 4 * l);
                float4 o;
                o.x = deflate1(kv.x, ai, pc.x, inv_c);
                o.y = deflate1(kv.y, ai, pc.y, inv_c);
                o.z = deflate1(kv.z, ai, pc.z, inv_c);
                o.w = deflate1(kv.w, ai, pc.w, inv_c);
                st_stream(gout + r * T + 4 * l, o);
                // partials: row sum via the canonical tree; column groups of 4 rows
                float rp = group4(o.x, o.y, o.z, o.w);
                rp = warp_sum(rp);
                if (l == q) a.rowsum = rp;
                if (I != J) {
                    if ((r & 3) == 0) {
                        a.cg[0] = __fmul_rn(o.x, o.x); a.cg[1] = __fmul_rn(o.y, o.y);
                        a.cg[2] = __fmul_rn(o.z, o.z); a.cg[3] = __fmul_rn(o.w, o.w);
                    } else {
                        a.cg[0] = __fmaf_rn(o.x, o.x, a.cg[0]); a.cg[1] = __fmaf_rn(o.y, o.y, a.cg[1]);
                        a.cg[2] = __fmaf_rn(o.z, o.z, a.cg[2]); a.cg[3] = __fmaf_rn(o.w, o.w, a.cg[3]);
                    }
                    if ((r & 3) == 3)
                        *reinterpret_cast<float4*>(&cg[r >> 2][4 * l]) =
                            make_float4(a.cg[0], a.cg[1], a.cg[2], a.cg[3]);
                }
            }
            __syncwarp();
            if (l == 0) mbar_arrive(empty + st);   // this warp is done reading the stage
        }
        consumer_sync();                           // colg of this tile complete
        if (l < 16) P[(int64_t)J * NP + (int64_t)I * T + my_row(l)] = a.rowsum;
        if (I != J && tid < T) P[(int64_t)I * NP + (int64_t)J * T + tid] = tree32_smem(&cg[0][tid], T);
    }
}

// 256-bit-store variant: a half-warp covers one row (lane: 8 consecutive
// columns), rows split so each half-warp walks whole groups of 4 rows.
template <int kSub, bool kHints>
__global__ void __launch_bounds__(kConsumers + kWarp, 1)
deflate_packed_v8_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int nT, int32_t N,
                      float* __restrict__ P, const unsigned long long* __restrict__ keys, int32_t t, float mu,
                      uint8_t* __restrict__ sel) {
    constexpr int kS = kStagesOf(kSub);
    constexpr int kStageFloats = kSub * T;
    constexpr int kSubs = T / kSub;             // stages per tile
    constexpr int kRW = kSub / 8;               // rows per warp per stage
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    float* stage = reinterpret_cast<float*>(smem_raw);                       // [kS][kSub*T]
    float (*colg)[kGroups][T] = reinterpret_cast<float (*)[kGroups][T]>(smem_raw + (size_t)kS * kStageFloats * 4);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)kS * kStageFloats * 4 + 2 * kGroups * T * 4);
    uint64_t* empty = full + kS;

    const int tid = threadIdx.x;
    const int64_t ntiles = num_tiles(nT);
    if (tid == 0) {
        for (int q = 0; q < kS; ++q) { mbar_init(full + q, 1); mbar_init(empty + q, kConsumers / kWarp); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (tid >= kConsumers) {
        // ---------------- producer warp: one elected lane streams the tiles, kSub rows per stage
        if (tid == kConsumers) {
            const uint64_t pol = policy_evict_first();    // K streams through L2 once per step
            int n = 0;
            for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x) {
                const float* src = Kin + k * (int64_t)(T * T);
                for (int sb = 0; sb < kSubs; ++sb, ++n) {
                    const int st = n % kS;
                    const uint32_t ph = (uint32_t)(n / kS) & 1u;
                    mbar_wait(empty + st, ph ^ 1u);
                    mbar_expect_tx(full + st, kStageFloats * 4);
                    if (kHints) bulk_g2s_hint(stage + st * kStageFloats, src + sb * kStageFloats, kStageFloats * 4,
                                              full + st, pol);
                    else bulk_g2s(stage + st * kStageFloats, src + sb * kStageFloats, kStageFloats * 4, full + st);
                }
            }
        }
        return;
    }

    // ---------------- consumers
    const int w = tid / kWarp, l = tid % kWarp;
    const int64_t NP = (int64_t)nT * T;
    const uint32_t s = key_index(keys[t - 1]);
    const int S = (int)(s / T), rs = (int)(s % T);
    const float inv_c = __frcp_rn(__fadd_rn(Kin[packed_index((int)s, (int)s, nT)], mu));   // 1/(k(s,s)+mu)
    if (blockIdx.x == 0 && tid == 0 && (int32_t)s < N) sel[s] = 1;
    // K_in[s, B*T + c]: a contiguous row segment of tile (S,B) if S <= B, else a column of tile (B,S)
    const uint64_t keep = kHints ? policy_evict_last() : 0ull;
    auto ldf = [&](const float* p) -> float { return kHints ? ld_hint(p, keep) : __ldg(p); };
    auto seg = [&](int B, int c) -> float {
        return S <= B ? ldf(Kin + tile_offset(S, B, nT) * (T * T) + (int64_t)rs * T + c)
                      : ldf(Kin + tile_offset(B, S, nT) * (T * T) + (int64_t)c * T + rs);
    };
    // the warp's 16 rows of a tile: row(l) for l < 16
    auto my_row = [&](int q) { return (q / kRW) * kSub + w * kRW + (q % kRW); };
    const int c8 = 8 * (l & 15);
    auto load_segs = [&](int64_t k, float& pr, float4& pa, float4& pb) {
        int I, J;
        tile_ij(k, nT, I, J);
        pr = l < 16 ? seg(I, my_row(l)) : 0.f;                 // a_i for the warp's 16 rows
        if (S <= J) {
            const float* p = Kin + tile_offset(S, J, nT) * (T * T) + (int64_t)rs * T + c8;
            pa = __ldg(reinterpret_cast<const float4*>(p));
            pb = __ldg(reinterpret_cast<const float4*>(p + 4));
        } else {
            pa.x = seg(J, c8); pa.y = seg(J, c8 + 1); pa.z = seg(J, c8 + 2); pa.w = seg(J, c8 + 3);
            pb.x = seg(J, c8 + 4); pb.y = seg(J, c8 + 5); pb.z = seg(J, c8 + 6); pb.w = seg(J, c8 + 7);
        }
    };
    float pr_next = 0.f;
    float4 pa_next = make_float4(0.f, 0.f, 0.f, 0.f), pb_next = pa_next;
    if ((int64_t)blockIdx.x < ntiles) load_segs(blockIdx.x, pr_next, pa_next, pb_next);
    int n = 0, tcount = 0;
    for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x, ++tcount) {
        int I, J;
        tile_ij(k, nT, I, J);
        float (*cgs)[T] = colg[tcount & 1];
        const float pr_l = pr_next;
        const float4 pc0 = pa_next, pc1 = pb_next;
        if (k + gridDim.x < ntiles) load_segs(k + gridDim.x, pr_next, pa_next, pb_next);   // next tile's segments
        float* gout = Kout + k * (int64_t)(T * T);
        float rowsum = 0.f;                         // lane l < 16: partial of the warp's row l
        float cg[8];
        const int hw = l >> 4, hl = l & 15;         // half-warp: rows, lane: 8 columns 8hl..8hl+7
        for (int sb = 0; sb < kSubs; ++sb, ++n) {
            const int st = n % kS;
            const uint32_t ph = (uint32_t)(n / kS) & 1u;
            mbar_wait(full + st, ph);
            const float* sm = stage + st * kStageFloats;
#pragma unroll
            for (int rr = 0; rr < kRW / 2; ++rr) {
                const int lrow = hw * (kRW / 2) + rr;              // row of the warp within the stage
                const int q = sb * kRW + lrow;                     // the warp's q-th row of the tile
                const int r = sb * kSub + w * kRW + lrow;          // row within the tile
                const float ai = __shfl_sync(0xffffffffu, pr_l, q);
                const float4 k0 = *reinterpret_cast<const float4*>(sm + (w * kRW + lrow) * T + 8 * hl);
                const float4 k1 = *reinterpret_cast<const float4*>(sm + (w * kRW + lrow) * T + 8 * hl + 4);
                f8 o;
                o.v[0] = deflate1(k0.x, ai, pc0.x, inv_c); o.v[1] = deflate1(k0.y, ai, pc0.y, inv_c);
                o.v[2] = deflate1(k0.z, ai, pc0.z, inv_c); o.v[3] = deflate1(k0.w, ai, pc0.w, inv_c);
                o.v[4] = deflate1(k1.x, ai, pc1.x, inv_c); o.v[5] = deflate1(k1.y, ai, pc1.y, inv_c);
                o.v[6] = deflate1(k1.z, ai, pc1.z, inv_c); o.v[7] = deflate1(k1.w, ai, pc1.w, inv_c);
                st8_stream(gout + r * T + 8 * hl, o);
                // canonical row tree: groups (8hl..+3), (8hl+4..+7) = groups 2hl, 2hl+1;
                // levels 16,8,4,2 are xor 8,4,2,1 within the half-warp, level 1 is a + b
                float ga = group4(o.v[0], o.v[1], o.v[2], o.v[3]);
                float gb = group4(o.v[4], o.v[5], o.v[6], o.v[7]);
#pragma unroll
                for (int off = 8; off > 0; off >>= 1) {
                    ga = __fadd_rn(ga, __shfl_xor_sync(0xffffffffu, ga, off));
                    gb = __fadd_rn(gb, __shfl_xor_sync(0xffffffffu, gb, off));
                }
                const float rp = __fadd_rn(ga, gb);
                // row q's sum lives in half hw; lane q (< 16) keeps it
                const float rq0 = __shfl_sync(0xffffffffu, rp, 0);    // half 0's row
                const float rq1 = __shfl_sync(0xffffffffu, rp, 16);   // half 1's row
                const int q0 = sb * kRW + rr, q1 = sb * kRW + kRW / 2 + rr;
                if (l == q0) rowsum = rq0;
                if (l == q1) rowsum = rq1;
                if (I != J) {
                    if ((r & 3) == 0) {
#pragma unroll
                        for (int c = 0; c < 8; ++c) cg[c] = __fmul_rn(o.v[c], o.v[c]);
                    } else {
#pragma unroll
                        for (int c = 0; c < 8; ++c) cg[c] = __fmaf_rn(o.v[c], o.v[c], cg[c]);
                    }
                    if ((r & 3) == 3) {
                        *reinterpret_cast<float4*>(&cgs[r >> 2][8 * hl]) = make_float4(cg[0], cg[1], cg[2], cg[3]);
                        *reinterpret_cast<float4*>(&cgs[r >> 2][8 * hl + 4]) = make_float4(cg[4], cg[5], cg[6], cg[7]);
                    }
                }
            }
            __syncwarp();
            if (l == 0) mbar_arrive(empty + st);   // this warp is done reading the stage
        }
        consumer_sync();                           // colg of this tile complete
        if (l < 16) P[(int64_t)J * NP + (int64_t)I * T + my_row(l)] = rowsum;
        if (I != J && tid < T) P[(int64_t)I * NP + (int64_t)J * T + tid] = tree32_smem(&cgs[0][tid], T);
    }
}

// L2-priority variants for the LDG kernel: K streams evict-first, the
// partials (nT * NP floats, read by the finalize kernel) are kept evict-last.
__device__ __forceinline__ f8 ld8_evict_first(const float* p) {
    f8 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]), "=f"(r.v[4]), "=f"(r.v[5]),
                   "=f"(r.v[6]), "=f"(r.v[7]) : "l"(p));
    return r;
}
__device__ __forceinline__ void st_keep(float* p, float v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" :: "l"(p), "f"(v), "l"(pol) : "memory");
}

template <int kD>
__global__ void __launch_bounds__(kConsumers, (kD <= 16 ? 3 : 1))
gram_packed_kernel(const float* __restrict__ X, int32_t N, int32_t d, float gamma, int32_t linear,
                   float* __restrict__ K, int nT, float* __restrict__ P) {

    __shared__ __align__(16) float xi[T][kD];
    __shared__ __align__(16) float xj[T][kD];
    __shared__ __align__(16) float colg[kGroups][T];
    const int tid = threadIdx.x, w = tid / kWarp, l = tid % kWarp;
    const int64_t ntiles = num_tiles(nT);
    const int64_t NP = (int64_t)nT * T;
    const float ng = -gamma;
    {
        const int64_t k = blockIdx.x;                    // one tile per CTA
        int I, J;
        tile_ij(k, nT, I, J);
        for (int q = tid; q < T * kD; q += kConsumers) {
            const int r = q / kD, c = q % kD;
            const int gi = I * T + r, gj = J * T + r;
            xi[r][c] = (gi < N && c < d) ? X[(int64_t)gi * d + c] : 0.f;   // zero features add (0-0)^2 = 0
            xj[r][c] = (gj < N && c < d) ? X[(int64_t)gj * d + c] : 0.f;
        }
        consumer_sync();
        // column features as f32x2 pairs (columns 4l,4l+1 | 4l+2,4l+3): the
        // distance loop runs on FADD2/FFMA2 (IEEE RN per half: bitwise the
        // same as the scalar __fsub_rn / __fmaf_rn sequence)
        unsigned long long y01[kD], y23[kD];
#pragma unroll
        for (int q = 0; q < kD; ++q) {
            y01[q] = pack2(xj[4 * l + 0][q], xj[4 * l + 1][q]);
            y23[q] = pack2(xj[4 * l + 2][q], xj[4 * l + 3][q]);
        }
        float* tile = K + k * (int64_t)(T * T);
        RowWalk a;
        a.rowsum = 0.f;
        for (int rr = 0; rr < 16; rr += 2) {
            // two rows at once: four independent FFMA2 chains (ILP at 2 CTAs / SM)
            const int r = 16 * w + rr;
            unsigned long long a01[2] = {0ull, 0ull}, a23[2] = {0ull, 0ull};
#pragma unroll
            for (int q = 0; q < kD; q += 4) {
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    const float4 xv = *reinterpret_cast<const float4*>(&xi[r + h][q]);
                    const float xs[4] = {xv.x, xv.y, xv.z, xv.w};
#pragma unroll
                    for (int qq = 0; qq < 4; ++qq) {
                        const unsigned long long xx = pack2(xs[qq], xs[qq]);
                        if (linear) {
                            a01[h] = fma2(xx, y01[q + qq], a01[h]);
                            a23[h] = fma2(xx, y23[q + qq], a23[h]);
                        } else {
                            const unsigned long long d01 = sub2(xx, y01[q + qq]), d23 = sub2(xx, y23[q + qq]);
                            a01[h] = fma2(d01, d01, a01[h]);
                            a23[h] = fma2(d23, d23, a23[h]);
                        }
                    }
                }
            }
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                float acc[4];
                unpack2(a01[h], acc[0], acc[1]);
                unpack2(a23[h], acc[2], acc[3]);
                float4 o;
                float* oc = &o.x;
                const bool rv = I * T + r + h < N;
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    const bool cv = J * T + 4 * l + c < N;
                    const float val = linear ? acc[c] : expf(__fmul_rn(ng, acc[c]));
                    oc[c] = (rv && cv) ? val : 0.f;
                }
                st_stream(tile + (r + h) * T + 4 * l, o);
                walk_row(a, rr + h, l, o, colg, w, I != J);
            }
        }
        consumer_sync();
        write_partials(P, NP, I, J, w, l, a, colg, tid);
    }
    (void)ntiles;
}


// ------------------------------------------------------------------ K1i: Gram tiles only
// Alg. 1 l.1 for the implicit engine, whose fp64 norm pass recomputes the
// first scores: the same tiles, bitwise the same values as K1p (same FADD2 /
// FFMA2 sequence over the features in order, same expf), without the fp32
// partials.  Row features are staged as duplicated pairs (x, x), so one
// LDS.128 feeds two features of a row with no packing; each warp runs kH rows
// at once (2 kH independent FFMA2 chains per lane).  At N = 16384 (B200, warm
// ncu): 369 us with kH = 2 at 3 CTAs/SM, 388 us with kH = 4 at 2 CTAs/SM,
// vs 412 us for K1p with its fp32 partials.
template <int kD, bool kLinear, int kH = 4>
__global__ void __launch_bounds__(kConsumers, kH == 4 ? 2 : 3)
gram_tile_kernel(const float* __restrict__ X, int32_t N, int32_t d, float gamma, float* __restrict__ K, int nT,
                 int sr = 0, int sp = 1, const int* __restrict__ = nullptr) {
    __shared__ __align__(16) unsigned long long xi2[T][kD];     // (x, x) pairs of the tile's rows
    __shared__ __align__(16) float xj[T][kD];
    const int tid = threadIdx.x, w = tid / kWarp, l = tid % kWarp;
    const float ng = -gamma;
    int I, J;
    tile_ij((int64_t)sr + (int64_t)sp * blockIdx.x, nT, I, J);     // (tile shards: every sp-th tile)
    for (int q = tid; q < T * kD; q += kConsumers) {
        const int r = q / kD, c = q % kD;
        const int gi = I * T + r, gj = J * T + r;
        const float xv = (gi < N && c < d) ? X[(int64_t)gi * d + c] : 0.f;   // zero features add (0-0)^2 = 0
        xi2[r][c] = pack2(xv, xv);
        xj[r][c] = (gj < N && c < d) ? X[(int64_t)gj * d + c] : 0.f;
    }
    __syncthreads();
    unsigned long long y01[kD], y23[kD];
#pragma unroll
    for (int q = 0; q < kD; ++q) {
        y01[q] = pack2(xj[4 * l + 0][q], xj[4 * l + 1][q]);
        y23[q] = pack2(xj[4 * l + 2][q], xj[4 * l + 3][q]);
    }
    float* tile = K + (int64_t)blockIdx.x * (T * T);
    bool cv[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) cv[c] = J * T + 4 * l + c < N;
#pragma unroll 1
    for (int rr = 0; rr < 16; rr += kH) {
        const int r = 16 * w + rr;
        unsigned long long a01[kH], a23[kH];
#pragma unroll
        for (int h = 0; h < kH; ++h) a01[h] = a23[h] = 0ull;
#pragma unroll
        for (int q = 0; q < kD; q += 2) {
#pragma unroll
            for (int h = 0; h < kH; ++h) {
                const ulonglong2 xx = *reinterpret_cast<const ulonglong2*>(&xi2[r + h][q]);
                if (kLinear) {
                    a01[h] = fma2(xx.x, y01[q], a01[h]);
                    a23[h] = fma2(xx.x, y23[q], a23[h]);
                    a01[h] = fma2(xx.y, y01[q + 1], a01[h]);
                    a23[h] = fma2(xx.y, y23[q + 1], a23[h]);
                } else {
                    unsigned long long d01 = sub2(xx.x, y01[q]), d23 = sub2(xx.x, y23[q]);
                    a01[h] = fma2(d01, d01, a01[h]);
                    a23[h] = fma2(d23, d23, a23[h]);
                    d01 = sub2(xx.y, y01[q + 1]);
                    d23 = sub2(xx.y, y23[q + 1]);
                    a01[h] = fma2(d01, d01, a01[h]);
                    a23[h] = fma2(d23, d23, a23[h]);
                }
            }
        }
#pragma unroll
        for (int h = 0; h < kH; ++h) {
            float acc[4];
            unpack2(a01[h], acc[0], acc[1]);
            unpack2(a23[h], acc[2], acc[3]);
            const bool rv = I * T + r + h < N;
            float4 o;
            float* oc = &o.x;
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const float val = kLinear ? acc[c] : expf(__fmul_rn(ng, acc[c]));
                oc[c] = (rv && cv[c]) ? val : 0.f;
            }
            st_stream(tile + (r + h) * T + 4 * l, o);
        }
    }
}

// K1i variant with two columns per lane: warps 2v and 2v+1 cover rows
// 32v .. 32v+31, lane l of warp w the columns 64 (w & 1) + 2l, +1; kH rows
// at once.  Half the column-feature registers of
// gram_tile_kernel (no spills at 4 CTAs/SM), 2 kH independent FFMA2 chains
// per lane, coalesced float2 stores (256 B per warp and row).  Bitwise the
// same values (same operand pairs, same feature order, same expf).
template <int kD, bool kLinear, int kH>
__global__ void __launch_bounds__(kConsumers, 4)
gram_tile2_kernel(const float* __restrict__ X, int32_t N, int32_t d, float gamma, float* __restrict__ K, int nT,
                  int sr = 0, int sp = 1, const int* __restrict__ tc_nmax_bits = nullptr) {
    // (the implicit head launches this kernel after the tensor-core one: it writes K only
    // when the tensor-core kernel's accuracy guard declined, gram_tc.cuh kGuard)
    if (tc_nmax_bits && __fmul_rn(gamma, __int_as_float(*tc_nmax_bits)) <= 4.f) return;
    __shared__ __align__(16) unsigned long long xi2[T][kD];     // (x, x) pairs of the tile's rows
    __shared__ __align__(16) float xj[T][kD + 1];
    const int tid = threadIdx.x, w = tid / kWarp, l = tid % kWarp;
    const float ng = -gamma;
    // tiles kl = blockIdx.x, + gridDim.x, ... of this shard (one per CTA when the grid covers them all)
    const int64_t nloc = (num_tiles(nT) - sr + sp - 1) / sp;
    for (int64_t kl = blockIdx.x; kl < nloc; kl += gridDim.x) {
    int I, J;
    tile_ij((int64_t)sr + (int64_t)sp * kl, nT, I, J);
    for (int q = tid; q < T * kD; q += kConsumers) {
        const int r = q / kD, c = q % kD;
        const int gi = I * T + r, gj = J * T + r;
        const float xv = (gi < N && c < d) ? X[(int64_t)gi * d + c] : 0.f;
        xi2[r][c] = pack2(xv, xv);
        xj[r][c] = (gj < N && c < d) ? X[(int64_t)gj * d + c] : 0.f;
    }
    __syncthreads();
    const int c0 = 64 * (w & 1) + 2 * l;                         // this lane's two columns
    unsigned long long y[kD];
#pragma unroll
    for (int q = 0; q < kD; ++q) y[q] = pack2(xj[c0][q], xj[c0 + 1][q]);
    float* tile = K + kl * (T * T);
    const bool cv0 = J * T + c0 < N, cv1 = J * T + c0 + 1 < N;
    const int rbase = 32 * (w >> 1);                             // warps 2v, 2v+1: rows 32v .. 32v+31
#pragma unroll 1
    for (int rr = 0; rr < 32; rr += kH) {
        const int r = rbase + rr;
        unsigned long long a[kH];
#pragma unroll
        for (int h = 0; h < kH; ++h) a[h] = 0ull;
#pragma unroll
        for (int q = 0; q < kD; q += 2) {
#pragma unroll
            for (int h = 0; h < kH; ++h) {
                const ulonglong2 xx = *reinterpret_cast<const ulonglong2*>(&xi2[r + h][q]);
                if (kLinear) {
                    a[h] = fma2(xx.x, y[q], a[h]);
                    a[h] = fma2(xx.y, y[q + 1], a[h]);
                } else {
                    unsigned long long dd = sub2(xx.x, y[q]);
                    a[h] = fma2(dd, dd, a[h]);
                    dd = sub2(xx.y, y[q + 1]);
                    a[h] = fma2(dd, dd, a[h]);
                }
            }
        }
#pragma unroll
        for (int h = 0; h < kH; ++h) {
            float a0, a1;
            unpack2(a[h], a0, a1);
            const bool rv = I * T + r + h < N;
            const float v0 = kLinear ? a0 : expf(__fmul_rn(ng, a0));
            const float v1 = kLinear ? a1 : expf(__fmul_rn(ng, a1));
            float2 o;
            o.x = (rv && cv0) ? v0 : 0.f;
            o.y = (rv && cv1) ? v1 : 0.f;
            __stcs(reinterpret_cast<float2*>(tile + (r + h) * T + c0), o);
        }
    }
    __syncthreads();                                             // xi2 / xj are refilled for the next tile
    }
}

// ------------------------------------------------------------------ K2p (LDG variant)
// One CTA (256 threads) per tile, non-persistent (the hardware scheduler
// balances 8256+ tiles over the SMs; several CTAs per SM keep many 256-bit
// loads in flight, like the dense K2).  Warp w owns rows 16w..16w+15; half-warp
// h of it rows 16w+8h..+7 (two whole groups of 4 rows); lane hl owns columns
// 8hl..8hl+7.  Same element arithmetic and canonical partial trees as the
// TMA variant (bit-identical outputs).
template <int kU>
__global__ void __launch_bounds__(kConsumers)
deflate_packed_ldg_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int nT, int32_t N,
                          float* __restrict__ P, const unsigned long long* __restrict__ keys, int32_t t, float mu,
                          uint8_t* __restrict__ sel) {
    __shared__ __align__(16) float cgs[kGroups][T];
    const int tid = threadIdx.x, w = tid / kWarp, l = tid % kWarp;
    const int hw = l >> 4, hl = l & 15, c8 = 8 * hl;
    const int64_t k = blockIdx.x;
    int I, J;
    tile_ij(k, nT, I, J);
    const int64_t NP = (int64_t)nT * T;
    const uint32_t s = key_index(keys[t - 1]);
    const int S = (int)(s / T), rs = (int)(s % T);
    if (k == 0 && tid == 0 && (int32_t)s < N) sel[s] = 1;
    const float inv_c = __frcp_rn(__fadd_rn(__ldg(Kin + packed_index((int)s, (int)s, nT)), mu));
    auto seg = [&](int B, int c) -> float {
        return S <= B ? __ldg(Kin + tile_offset(S, B, nT) * (T * T) + (int64_t)rs * T + c)
                      : __ldg(Kin + tile_offset(B, S, nT) * (T * T) + (int64_t)c * T + rs);
    };
    // a_i for the half-warp's 8 rows (lane hl < 8 holds row 16w + 8hw + hl), p_j for the lane's 8 columns
    const float pr_l = hl < 8 ? seg(I, 16 * w + 8 * hw + hl) : 0.f;
    float pc[8];
    if (S <= J) {
        const float* p = Kin + tile_offset(S, J, nT) * (T * T) + (int64_t)rs * T + c8;
        const float4 a = __ldg(reinterpret_cast<const float4*>(p)), b = __ldg(reinterpret_cast<const float4*>(p + 4));
        pc[0] = a.x; pc[1] = a.y; pc[2] = a.z; pc[3] = a.w; pc[4] = b.x; pc[5] = b.y; pc[6] = b.z; pc[7] = b.w;
    } else {
#pragma unroll
        for (int c = 0; c < 8; ++c) pc[c] = seg(J, c8 + c);
    }
    const float* gin = Kin + k * (int64_t)(T * T);
    float* gout = Kout + k * (int64_t)(T * T);
    float rowsum = 0.f;                      // lane q < 16 of the warp: the warp's row q
    float cg[8];
#pragma unroll
    for (int r0 = 0; r0 < 8; r0 += kU) {
        f8 kv[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) kv[u] = ld8_evict_first(gin + (16 * w + 8 * hw + r0 + u) * T + c8);
#pragma unroll
        for (int u = 0; u < kU; ++u) {
            const int rr = r0 + u;                       // row within the half-warp's 8
            const int r = 16 * w + 8 * hw + rr;          // row within the tile
            const float ai = __shfl_sync(0xffffffffu, pr_l, 16 * hw + rr);
            f8 o;
#pragma unroll
            for (int c = 0; c < 8; ++c) o.v[c] = deflate1(kv[u].v[c], ai, pc[c], inv_c);
            st8_stream(gout + r * T + c8, o);
            float ga = group4(o.v[0], o.v[1], o.v[2], o.v[3]);
            float gb = group4(o.v[4], o.v[5], o.v[6], o.v[7]);
#pragma unroll
            for (int off = 8; off > 0; off >>= 1) {
                ga = __fadd_rn(ga, __shfl_xor_sync(0xffffffffu, ga, off));
                gb = __fadd_rn(gb, __shfl_xor_sync(0xffffffffu, gb, off));
            }
            const float rp = __fadd_rn(ga, gb);
            const float rq0 = __shfl_sync(0xffffffffu, rp, 0), rq1 = __shfl_sync(0xffffffffu, rp, 16);
            if (l == rr) rowsum = rq0;
            if (l == 8 + rr) rowsum = rq1;
            if (I != J) {
                if ((rr & 3) == 0) {
#pragma unroll
                    for (int c = 0; c < 8; ++c) cg[c] = __fmul_rn(o.v[c], o.v[c]);
                } else {
#pragma unroll
                    for (int c = 0; c < 8; ++c) cg[c] = __fmaf_rn(o.v[c], o.v[c], cg[c]);
                }
                if ((rr & 3) == 3) {
                    *reinterpret_cast<float4*>(&cgs[r >> 2][c8]) = make_float4(cg[0], cg[1], cg[2], cg[3]);
                    *reinterpret_cast<float4*>(&cgs[r >> 2][c8 + 4]) = make_float4(cg[4], cg[5], cg[6], cg[7]);
                }
            }
        }
    }
    const uint64_t keep = policy_evict_last();
    if (l < 16) st_keep(P + (int64_t)J * NP + (int64_t)I * T + 16 * w + l, rowsum, keep);
    if (I != J) {
        __syncthreads();
        if (tid < T) st_keep(P + (int64_t)I * NP + (int64_t)J * T + tid, tree32_smem(&cgs[0][tid], T), keep);
    }
}

}  // namespace pk
}  // namespace bted
