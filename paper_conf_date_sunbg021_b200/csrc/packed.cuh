// packed.cuh -- packed-symmetric TED kernels.
//
// K is stored once: only the upper-triangular T x T tiles (I <= J) of the
// N x N matrix, each tile contiguous (row-major, 64 KiB at T = 128), tiles in
// row-major order over the upper triangle.  Padding rows/columns (>= N) are
// exactly 0.  A step of Alg. 1 then streams 4 N^2 bytes
// (+ the diagonal tiles' duplicated halves) instead of 8 N^2:
//
//   K2p: tile (I,J) <- tile - p_I p_J^T / (k(s,s)+mu)  (product first, as dense)
//        row partials   P[J][i] = sum_{j in J} K_ij^2      (i in block I)
//        column partials P[I][j] = sum_{i in I} K_ij^2     (j in block J, I < J)
//   and ||K_v||^2 = sum_J P[J][v] in J order (deterministic), because the
//   (I,J) block for J < I is the transpose of the stored (J,I) tile.
//
// Every element value is bitwise the same as in the dense layout (same
// operands, same instruction); only the norm summation order differs.
//
// K2p is a TMA pipeline: one producer warp streams tiles into a 3-stage
// shared-memory ring with cp.async.bulk (mbarrier complete_tx), eight
// consumer warps update them, store the new tile with 128-bit streaming
// stores and reduce the partials.  The block of rows whose partials are
// complete is finished (score + argmax) by the CTA that delivers its last
// partial (a per-block arrival counter), so a step stays ONE kernel.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "kernels.cuh"

namespace bted {
namespace pk {

constexpr int T = 128;                 // tile edge
constexpr int kConsumers = 256;        // 8 consumer warps
constexpr int kStages = 3;
constexpr int kTileBytes = T * T * 4;  // 64 KiB

__host__ __device__ __forceinline__ int64_t tile_offset(int I, int J, int nT) {
    // tiles of rows 0..I-1 precede row I: sum_{i<I} (nT - i)
    return (int64_t)I * nT - (int64_t)I * (I - 1) / 2 + (J - I);
}
__host__ __device__ __forceinline__ int64_t num_tiles(int nT) { return (int64_t)nT * (nT + 1) / 2; }

// tile linear index -> (I, J) (row-major over the upper triangle)
__device__ __forceinline__ void tile_ij(int64_t k, int nT, int& I, int& J) {
    // solve offset(I) <= k < offset(I+1) with offset(I) = I*nT - I(I-1)/2
    double a = 2.0 * nT + 1.0;
    int i = (int)((a - sqrt(a * a - 8.0 * (double)k)) * 0.5);
    if (i < 0) i = 0;
    if (i > nT - 1) i = nT - 1;
    while (i > 0 && tile_offset(i, i, nT) > k) --i;
    while (i < nT - 1 && tile_offset(i + 1, i + 1, nT) <= k) ++i;
    I = i;
    J = i + (int)(k - tile_offset(i, i, nT));
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
__device__ __forceinline__ void consumer_sync() {       // named barrier 1: the 256 consumer threads
    asm volatile("bar.sync 1, %0;" :: "n"(kConsumers) : "memory");
}
__device__ __forceinline__ float4 lds4(const float* p) { return *reinterpret_cast<const float4*>(p); }

// ------------------------------------------------------------------ shared epilogue
// Partials of one finished tile: rowp[r] (row sums over the tile's columns)
// and, for off-diagonal tiles, colp[c].  Written to P, then the arrival
// counters of blocks I and J are bumped; a block whose nT partials are all
// in is finished by this CTA: g_i = sum_J P[J][i], score, masked argmax.
struct Epi {
    float* P;                // [nT][NP] partials
    int64_t NP;              // nT * T
    unsigned int* cnt;       // [nT] arrival counters (this step's parity)
    const float* Kdiag_base; // Kout (diagonal read-back)
    int nT, N;
    float mu;
    const uint8_t* sel;
    uint32_t s;              // pivot of this step (0xFFFFFFFF for the Gram)
    unsigned long long* key_out;
    int* err;
};

__device__ __forceinline__ void finish_block(const Epi& e, int B, int tid, unsigned long long* red) {
    unsigned long long key = 0ull;
    if (tid < T) {
        const int i = B * T + tid;
        if (i < e.N) {
            float g = 0.f;
            for (int J = 0; J < e.nT; ++J) g = __fadd_rn(g, __ldcg(e.P + (int64_t)J * e.NP + i));
            const float* dt = e.Kdiag_base + tile_offset(B, B, e.nT) * (int64_t)(T * T);
            const float diag = __ldcg(dt + tid * T + tid);
            const bool masked = (e.sel && e.sel[i] != 0) || (uint32_t)i == e.s;
            key = score_key(g, diag, e.mu, (uint32_t)i, masked, e.err);
        }
    }
    key = warp_max_u64(key);
    const int w = tid / kWarp, l = tid % kWarp;
    if (l == 0) red[w] = key;
    consumer_sync();
    if (tid == 0) {
        unsigned long long v = 0ull;
        for (int k = 0; k < kConsumers / kWarp; ++k) v = red[k] > v ? red[k] : v;
        if (v) atomicMax(e.key_out, v);
    }
    consumer_sync();
}

// After the tile's partials are stored by the consumers (all 256 threads
// passed consumer_sync): count arrivals, finish completed blocks.
__device__ __forceinline__ void arrive_and_finish(const Epi& e, int I, int J, int tid, int* flag,
                                                  unsigned long long* red) {
    __threadfence();                 // this thread's tile / partial stores are visible GPU-wide
    consumer_sync();
    if (tid == 0) {
        int f = 0;
        if (atomicAdd(e.cnt + I, 1u) == (unsigned)(e.nT - 1)) f |= 1;
        if (I != J && atomicAdd(e.cnt + J, 1u) == (unsigned)(e.nT - 1)) f |= 2;
        if (f) __threadfence();
        *flag = f;
    }
    consumer_sync();
    const int f = *flag;
    if (f & 1) { if (tid == 0) e.cnt[I] = 0u; finish_block(e, I, tid, red); }
    if (f & 2) { if (tid == 0) e.cnt[J] = 0u; finish_block(e, J, tid, red); }
}

// Consumer part common to K1p / K2p: given 16 rows x 4 columns of new
// values per lane (row-by-row), accumulate partials.  Layout: warp w owns
// rows 16w..16w+15 of the tile, lane l owns columns 4l..4l+3.
struct TileAcc {
    float col[4];
    float rowsum;            // lane l < 16: the sum of row 16w + l after the tile
};

__device__ __forceinline__ void store_partials(const Epi& e, int I, int J, int w, int l, const TileAcc& a,
                                               float (*colred)[T]) {
    // row partials of rows 16w + l (l < 16) -> P[J][I*T + 16w + l]
    if (l < 16) e.P[(int64_t)J * e.NP + (int64_t)I * T + 16 * w + l] = a.rowsum;
    if (I != J) {
        colred[w][4 * l + 0] = a.col[0];
        colred[w][4 * l + 1] = a.col[1];
        colred[w][4 * l + 2] = a.col[2];
        colred[w][4 * l + 3] = a.col[3];
    }
    consumer_sync();
    const int tid = w * kWarp + l;
    if (I != J && tid < T) {
        float c = 0.f;
        for (int ww = 0; ww < kConsumers / kWarp; ++ww) c = __fadd_rn(c, colred[ww][tid]);
        e.P[(int64_t)I * e.NP + (int64_t)J * T + tid] = c;
    }
    consumer_sync();
}

// ------------------------------------------------------------------ K1p: Gram tiles
// Alg. 1 l.1 + first l.3 on the upper-triangular tiles.  One CTA (256
// threads) per tile in a persistent loop.  Lane l keeps the features of its
// 4 columns in registers (kD <= 32); the rows' features are smem broadcasts.
template <int kD>
__global__ void __launch_bounds__(kConsumers)
gram_packed_kernel(const float* __restrict__ X, int32_t N, int32_t d, float gamma, int32_t linear,
                   float* __restrict__ K, int nT, float* __restrict__ P, unsigned int* __restrict__ cnt,
                   float mu, unsigned long long* __restrict__ key_out, int* __restrict__ err) {
    __shared__ __align__(16) float xi[T][kD];
    __shared__ __align__(16) float xj[T][kD];
    __shared__ float colred[kConsumers / kWarp][T];
    __shared__ unsigned long long red[kConsumers / kWarp];
    __shared__ int flag;
    const int tid = threadIdx.x, w = tid / kWarp, l = tid % kWarp;
    const int64_t ntiles = num_tiles(nT);
    const float ng = -gamma;
    Epi e{P, (int64_t)nT * T, cnt, K, nT, N, mu, nullptr, 0xFFFFFFFFu, key_out, err};
    for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x) {
        int I, J;
        tile_ij(k, nT, I, J);
        for (int q = tid; q < T * kD; q += kConsumers) {
            const int r = q / kD, c = q % kD;
            const int gi = I * T + r, gj = J * T + r;
            xi[r][c] = (gi < N && c < d) ? X[(int64_t)gi * d + c] : 0.f;   // zero features add (0-0)^2 = 0
            xj[r][c] = (gj < N && c < d) ? X[(int64_t)gj * d + c] : 0.f;
        }
        consumer_sync();
        float y[4][kD];
#pragma unroll
        for (int c = 0; c < 4; ++c)
#pragma unroll
            for (int q = 0; q < kD; q += 4) {
                const float4 v = *reinterpret_cast<const float4*>(&xj[4 * l + c][q]);
                y[c][q] = v.x; y[c][q + 1] = v.y; y[c][q + 2] = v.z; y[c][q + 3] = v.w;
            }
        float* tile = K + k * (int64_t)(T * T);
        TileAcc a;
        a.col[0] = a.col[1] = a.col[2] = a.col[3] = 0.f;
        a.rowsum = 0.f;
        for (int rr = 0; rr < 16; ++rr) {
            const int r = 16 * w + rr;
            float acc[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
            for (int q = 0; q < kD; q += 4) {
                const float4 xv = *reinterpret_cast<const float4*>(&xi[r][q]);
                const float xs[4] = {xv.x, xv.y, xv.z, xv.w};
#pragma unroll
                for (int qq = 0; qq < 4; ++qq) {
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        if (linear) acc[c] = __fmaf_rn(xs[qq], y[c][q + qq], acc[c]);
                        else { const float df = __fsub_rn(xs[qq], y[c][q + qq]); acc[c] = __fmaf_rn(df, df, acc[c]); }
                    }
                }
            }
            float4 o;
            float* oc = &o.x;
            float rp = 0.f;
            const bool rv = I * T + r < N;
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const bool cv = J * T + 4 * l + c < N;
                const float val = linear ? acc[c] : expf(__fmul_rn(ng, acc[c]));
                oc[c] = (rv && cv) ? val : 0.f;
                rp = __fmaf_rn(oc[c], oc[c], rp);
                a.col[c] = __fmaf_rn(oc[c], oc[c], a.col[c]);
            }
            st_stream(tile + r * T + 4 * l, o);
            rp = warp_sum(rp);
            if (l == rr) a.rowsum = rp;
        }
        store_partials(e, I, J, w, l, a, colred);
        arrive_and_finish(e, I, J, tid, &flag, red);
    }
}

// ------------------------------------------------------------------ pivot extraction
// p[j] = K[s][j] for j < nT*T, s = key_index(keys[t]) (the new pivot).
__global__ void packed_pivot_kernel(const float* __restrict__ K, int nT, const unsigned long long* __restrict__ keys,
                                    int32_t t, float* __restrict__ p) {
    const uint32_t s = key_index(keys[t]);
    const int S = (int)(s / T), rs = (int)(s % T);
    const int64_t NP = (int64_t)nT * T;
    for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < NP; j += (int64_t)gridDim.x * blockDim.x) {
        const int J = (int)(j / T), c = (int)(j % T);
        float v;
        if (S <= J) v = K[tile_offset(S, J, nT) * (T * T) + rs * T + c];
        else        v = K[tile_offset(J, S, nT) * (T * T) + c * T + rs];
        p[j] = v;
    }
}

// ------------------------------------------------------------------ K2p: TMA deflate
__global__ void __launch_bounds__(kConsumers + kWarp, 1)
deflate_packed_kernel(const float* __restrict__ Kin, float* __restrict__ Kout, int nT, int32_t N,
                      const float* __restrict__ p, float* __restrict__ P, unsigned int* __restrict__ cnt,
                      unsigned long long* __restrict__ keys, int32_t t, float mu, uint8_t* __restrict__ sel,
                      int* __restrict__ err) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    float* stage = reinterpret_cast<float*>(smem_raw);                       // [kStages][T*T]
    uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + kStages * kTileBytes);
    uint64_t* empty = full + kStages;
    __shared__ float colred[kConsumers / kWarp][T];
    __shared__ unsigned long long red[kConsumers / kWarp];
    __shared__ int flag;

    const int tid = threadIdx.x;
    const int64_t ntiles = num_tiles(nT);
    if (tid == 0) {
        for (int q = 0; q < kStages; ++q) { mbar_init(full + q, 1); mbar_init(empty + q, kConsumers / kWarp); }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();

    if (tid >= kConsumers) {
        // ---------------- producer warp: one elected lane streams the tiles
        if (tid == kConsumers) {
            int n = 0;
            for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x, ++n) {
                const int st = n % kStages;
                const uint32_t ph = (uint32_t)(n / kStages) & 1u;
                mbar_wait(empty + st, ph ^ 1u);
                mbar_expect_tx(full + st, kTileBytes);
                const float* src = Kin + k * (int64_t)(T * T);
                float* dst = stage + st * (T * T);
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    bulk_g2s(dst + q * (T * T / 4), src + q * (T * T / 4), kTileBytes / 4, full + st);
            }
        }
        return;
    }

    // ---------------- consumers
    const int w = tid / kWarp, l = tid % kWarp;
    const uint32_t s = key_index(keys[t - 1]);
    const float inv_c = __frcp_rn(__fadd_rn(p[s], mu));
    if (blockIdx.x == 0 && tid == 0 && (int32_t)s < N) sel[s] = 1;
    Epi e{P, (int64_t)nT * T, cnt, Kout, nT, N, mu, sel, s, keys + t, err};
    int n = 0;
    for (int64_t k = blockIdx.x; k < ntiles; k += gridDim.x, ++n) {
        int I, J;
        tile_ij(k, nT, I, J);
        const int st = n % kStages;
        const uint32_t ph = (uint32_t)(n / kStages) & 1u;
        // pivot segments: rows of block I (one per lane < 16), columns of block J
        const float pr_l = l < 16 ? p[I * T + 16 * w + l] : 0.f;
        const float4 pc = *reinterpret_cast<const float4*>(p + J * T + 4 * l);
        mbar_wait(full + st, ph);
        const float* sm = stage + st * (T * T);
        float* gout = Kout + k * (int64_t)(T * T);
        TileAcc a;
        a.col[0] = a.col[1] = a.col[2] = a.col[3] = 0.f;
        a.rowsum = 0.f;
#pragma unroll 4
        for (int rr = 0; rr < 16; ++rr) {
            const int r = 16 * w + rr;
            const float ai = __shfl_sync(0xffffffffu, pr_l, rr);
            const float4 kv = lds4(sm + r * T + 4 * l);
            float4 o;
            o.x = deflate1(kv.x, ai, pc.x, inv_c);
            o.y = deflate1(kv.y, ai, pc.y, inv_c);
            o.z = deflate1(kv.z, ai, pc.z, inv_c);
            o.w = deflate1(kv.w, ai, pc.w, inv_c);
            st_stream(gout + r * T + 4 * l, o);
            float rp = __fmul_rn(o.x, o.x);
            rp = __fmaf_rn(o.y, o.y, rp);
            rp = __fmaf_rn(o.z, o.z, rp);
            rp = __fmaf_rn(o.w, o.w, rp);
            a.col[0] = __fmaf_rn(o.x, o.x, a.col[0]);
            a.col[1] = __fmaf_rn(o.y, o.y, a.col[1]);
            a.col[2] = __fmaf_rn(o.z, o.z, a.col[2]);
            a.col[3] = __fmaf_rn(o.w, o.w, a.col[3]);
            rp = warp_sum(rp);
            if (l == rr) a.rowsum = rp;
        }
        __syncwarp();
        if (l == 0) mbar_arrive(empty + st);       // this warp is done reading the stage
        store_partials(e, I, J, w, l, a, colred);
        arrive_and_finish(e, I, J, tid, &flag, red);
    }
}

}  // namespace pk
}  // namespace bted
