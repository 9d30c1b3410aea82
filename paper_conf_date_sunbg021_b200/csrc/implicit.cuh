// implicit.cuh -- implicit deflation on the packed
// read-only Gram matrix.
//
// Algorithm 1 deflates K <- K - K_:s K_s: / (K_ss + mu)
// every step.  Written as K^(t) = K - L L^T with L = [l_1 .. l_t] (N x t),
// l_t = K^(t-1)_:s / sqrt(K^(t-1)_ss + mu), the same selections follow from
// K itself (never rewritten) plus the factor L:
//
//   R = K - L L^T (implicit),  l = R_:s / sqrt(c),  c = R_ss + mu
//   l_i   = (K_is - sum_k L_ik L_sk) / sqrt(c)                     (kernel A)
//   h     = L^T l:  h_k = ((K l_k)_s - sum_j G_kj L_sj) / sqrt(c),  G = L^T L
//           |l|^2 = ||R_:s||^2 / c = n_s / c   (O(m^2) from the history;  kernel A)
//   q     = K l  (one pass over the packed tiles, READ ONLY: 2 N^2 B) (kernel B)
//   (R l)_v = q_v - sum_k L_vk h_k
//   n_v  <- n_v - 2 l_v (R l)_v + l_v^2 |l|^2      (= ||R'_:v||^2)   (kernel C)
//   r_vv <- r_vv - l_v^2,   score_v = n_v / (r_vv + mu);   Q[t] = q, G gets h
// (K l_k)_s = (K_:s)^T l_k because K is symmetric: kernel C keeps every q.
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
// mbarrier), so HBM streams independently of the fp64 arithmetic.  Tiles
// are handed out dynamically (an atomic counter per pass, grabbed by the
// producer one tile ahead), so all CTAs finish a pass within about a tile.
// Eight consumer warps: in chunk c warp w owns tile rows 32c + 4w .. +3,
// lane l columns 4l .. 4l+3 (conflict-free LDS.128).
//
// Canonical per-128 tree (the SAME for rows and columns, so exact duplicate
// points get bitwise-equal norms and tie to the lowest index): groups of 4
// consecutive terms summed sequentially (mul, fma, fma, fma), then the
// 32-leaf butterfly h[q] += h[q + 16], += h[q + 8], ..., += h[q + 1].
//   rows:    group q = lane q  ->  levels 16 / 8 in registers after a per-warp
//            shared-memory transpose (rowx), then xor shuffles 4/2/1;
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
constexpr int kWSlots = 3;                                    // tile slots: the producer runs a tile ahead
constexpr int kRowxLd = 40;                                   // row pitch (doubles) of rowx: 64-bit reads of
                                                              // (row l/8, group l%8 + 8k) hit distinct banks
struct TPSmem {
    float ring[kStages][kChunkFloats];
    double colstage[2][kTPWarps][T];                          // double-buffered per tile
    double wslot[kWSlots][2][T];                              // [slot][0: w on block J, 1: w on block I]
    int64_t wtile[kWSlots];                                   // the slot's tile index (-1: end of pass)
    int wI[kWSlots], wJ[kWSlots];                             // ... and its block coordinates (I <= J)
    double red[kTPWarps];
    double rowx[kTPWarps][4][kRowxLd];                        // per-warp row-group transposes
    uint64_t full[kStages], empty[kStages];
    uint64_t wfull[kWSlots], wempty[kWSlots];
    uint64_t cbar[2];                                         // colstage[b] complete (8 warps arrived)
    int grab;
};
constexpr size_t tile_pass_smem_bytes = sizeof(TPSmem);

// Programmatic dependent launch (the split loop's kernels are launched with
// programmatic stream serialization): wait = the previous grid has completed
// and its writes are visible (a no-op for a normal launch); trigger = let the
// next grid launch now.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

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

// partial stores: streaming (.cs), or L2 evict-last (kAbl & 64: tile_pass_kernel's kKeepP, chosen by
// the library when the partial buffer fits well inside L2 -- then they never reach DRAM;
// profiles/r2/partials_l2)
template <int kAbl>
__device__ __forceinline__ void tp_store(double* p, double v, uint64_t keep) {
    if (kAbl & 16) *p = v;
    else if (kAbl & 64) st_f64_hint(p, v, keep);
    else __stcs(p, v);
}
// kAbl (scripts/tp_ablate.cu; the library uses 0 and 64): 1 = no partial stores,
// 8 = no arithmetic at all (LDS + release: the streaming ceiling), 16 = plain
// partial stores (no L2 hint), 64 = L2 evict-last partial stores
//
// Latency hiding: a chunk's row butterfly is finished one chunk later (its
// shuffle chain overlaps the next chunk's DFMA chains), and a tile's column
// tree is handed to warps 0-3 through an mbarrier and finished one chunk into
// the next tile (no CTA-wide barrier per tile).  n / tile_it / col_it carry the
// ring, w-slot and column-buffer phases across calls.
// Sm: the shared-memory struct (TPSmem, or rc_pass.cuh's RCSmem: the same members),
// kSt its ring depth; kSwz: the ring chunks are stored with 16-byte granule g of
// row r at g ^ (r & 7) (written row-per-lane by the recomputing epilogue).
// Row tree of a chunk: the 4 row groups of every lane go through a per-warp shared-memory
// transpose, lane (r, j) = (l / 8, l % 8) adds groups j, j + 16, j + 8, j + 24 of row r in
// registers (levels 16, 8), levels 4 / 2 / 1 are xor shuffles -- the same pairs as the 32-leaf
// butterfly, so bitwise the same sums as a shuffle reduce-scatter, with ~15 fewer instructions per
// chunk (-2.2 % per step on the power-capped N = 65536 config, profiles/r2/partials_l2).
template <bool kNorm, bool kExact, int kAbl = 0, class Sm = TPSmem, int kSt = kStages, bool kSwz = false>
__device__ __forceinline__ void tp_consume(Sm& S, int nT, double* P64, int* __restrict__ kflag, int& n,
                                           int& tile_it, int& col_it) {
    double sink = 0.0;
    const int tid = threadIdx.x, wq = tid / 32, l = tid % 32;
    const int64_t NP = (int64_t)nT * T;
    const uint64_t keep = pk::policy_evict_last();
    bool odd_value = false;
    // pending row tree (the previous chunk's level-8 value) and column tree (the previous
    // off-diagonal tile)
    double hv = 0.0;
    bool rpend = false, cpend = false;
    int cit = 0;
    double* rptr = P64;                                       // the pending chunk's 4 row partials
    double* cptr = P64;                                       // the pending tile's column partials
    int st = n % kSt;                                         // ring slot and phase of chunk n
    uint32_t ph = (uint32_t)(n / kSt) & 1u;
    auto row_finish = [&]() {                                  // levels 4, 2, 1 of the pending chunk
        if (!rpend) return;
        rpend = false;
        double hr = __dadd_rn(hv, __shfl_xor_sync(0xffffffffu, hv, 4));
        hr = __dadd_rn(hr, __shfl_xor_sync(0xffffffffu, hr, 2));
        hr = __dadd_rn(hr, __shfl_xor_sync(0xffffffffu, hr, 1));
        if ((l & 7) == 0) {                                   // row 32c + 4w + l/8: P[J][I*T + row]
            if (kAbl & 1) sink += hr;
            else tp_store<kAbl>(rptr, hr, keep);
        }
    };
    auto col_finish = [&]() {                                  // levels 4, 2, 1 over the 8 warps
        if (!cpend) return;
        cpend = false;
        if (tid < T) {
            const int buf = cit & 1;
            pk::mbar_wait(&S.cbar[buf], (uint32_t)(cit >> 1) & 1u);
            double v[kTPWarps];
#pragma unroll
            for (int q = 0; q < kTPWarps; ++q) v[q] = S.colstage[buf][q][tid];
#pragma unroll
            for (int q = 0; q < 4; ++q) v[q] = __dadd_rn(v[q], v[q + 4]);
            v[0] = __dadd_rn(v[0], v[2]);
            v[1] = __dadd_rn(v[1], v[3]);
            if (kAbl & 1) sink += v[0] + v[1];
            else tp_store<kAbl>(cptr, __dadd_rn(v[0], v[1]), keep);
        }
    };
    for (;; ++tile_it) {
        // the producer publishes the next tile of this CTA (dynamic: grabbed from a
        // counter of the pass) and, unless kNorm, its w slices w_J, w_I (TMA)
        const int ws = tile_it % kWSlots;
        pk::mbar_wait(&S.wfull[ws], (uint32_t)(tile_it / kWSlots) & 1u);
        const int64_t k = S.wtile[ws];
        if (k < 0) {                                          // end of the pass
            __syncwarp();
            if (l == 0) pk::mbar_arrive(&S.wempty[ws]);
            ++tile_it;
            break;
        }
        const int I = S.wI[ws], J = S.wJ[ws];                 // published by the producer with k
        const bool offdiag = I != J;
        double wc[4];                                         // w on the lane's 4 columns
        if (!kNorm) {
#pragma unroll
            for (int x = 0; x < 4; ++x) wc[x] = S.wslot[ws][0][4 * l + x];
        }
        double hold[2][4];
        double* const rowbase = P64 + (int64_t)J * NP + (int64_t)I * T + 4 * wq + (l >> 3);
#pragma unroll
        for (int c = 0; c < kChunks; ++c, ++n) {
            const int stc = st;
            pk::mbar_wait(&S.full[stc], ph);
            if (++st == kSt) { st = 0; ph ^= 1u; }
            if (kAbl & 8) {
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    const float4 kv = *reinterpret_cast<const float4*>(&S.ring[stc][(4 * wq + r) * T + 4 * l]);
                    sink += (double)(kv.x + kv.y + kv.z + kv.w);
                }
                __syncwarp();
                if (l == 0) pk::mbar_arrive(&S.empty[stc]);
                continue;
            }
            // per row: load from the stage, convert, the row group (4 consecutive
            // columns) and the running column groups (4 rows: mul for row 0, then fma)
            double g[4], cg[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const int row = 4 * wq + r;
                const float4 kv = *reinterpret_cast<const float4*>(&S.ring[stc][row * T + 4 * (kSwz ? l ^ (row & 7) : l)]);
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
                const double wi = kNorm ? 0.0 : S.wslot[ws][1][kChunkRows * c + 4 * wq + r];
#pragma unroll
                for (int x = 0; x < 4; ++x)
                    cg[x] = r == 0 ? __dmul_rn(kd[x], kNorm ? kd[x] : wi)
                                   : __fma_rn(kd[x], kNorm ? kd[x] : wi, cg[x]);
            }
            __syncwarp();
            if (l == 0) pk::mbar_arrive(&S.empty[stc]);
            row_finish();                                     // the previous chunk's rows
            {                                                 // this chunk's levels 16 and 8
                double* rx = &S.rowx[wq][0][0];
#pragma unroll
                for (int r = 0; r < 4; ++r) rx[r * kRowxLd + l] = g[r];
                __syncwarp();
                const double* rr = rx + (l >> 3) * kRowxLd + (l & 7);
                hv = __dadd_rn(__dadd_rn(rr[0], rr[16]), __dadd_rn(rr[8], rr[24]));
                __syncwarp();                                 // reads done before the next chunk's writes
            }
            rpend = true;
            rptr = rowbase + kChunkRows * c;
            if (c == 0) col_finish();                          // the previous tile's columns
#pragma unroll
            for (int x = 0; x < 4; ++x) {
                if (c < 2) hold[c][x] = cg[x];                                      // groups w, 8 + w
                else hold[c - 2][x] = __dadd_rn(hold[c - 2][x], cg[x]);             // level 16
            }
        }
        __syncwarp();                                         // this warp is done with the slot
        if (l == 0) pk::mbar_arrive(&S.wempty[ws]);
        if (offdiag && !(kAbl & 8)) {
            const int buf = col_it & 1;
#pragma unroll
            for (int x = 0; x < 4; ++x) S.colstage[buf][wq][4 * l + x] = __dadd_rn(hold[0][x], hold[1][x]);  // level 8
            __syncwarp();
            if (l == 0) pk::mbar_arrive(&S.cbar[buf]);
            cpend = true; cit = col_it;
            cptr = P64 + (int64_t)I * NP + (int64_t)J * T + tid;
            ++col_it;
        }
    }
    row_finish();
    col_finish();
    if (kNorm && odd_value) atomicOr(kflag, 1);
    if ((kAbl & ~64) && sink == 1.2345) P64[0] = sink;
}

// Producer lane: `passes` passes over the tiles, grabbed one at a time from
// tilectr[pass]; per tile: publish {k, w_J, w_I (kW, TMA)} in a slot, then its
// 4 K chunks.  wait_w(pass, I, J) runs before a w copy (the persistent loop
// waits there for the ell units of blocks I and J).  The next grab is issued
// one tile ahead so its latency overlaps the current tile's copies.
//
// L2 reuse across passes (serpentine order): pass p hands the tiles out in
// ascending order when (dir0 + p) is even, descending otherwise, so the next
// pass starts with the tiles the previous one read last (still in L2; K is
// read-only and identical in every pass).  Measured on B200 (resnet18,
// profiles/r1r/l2_sweep.txt): 89.0 -> 85.7 us per step with every load
// evict-first; additionally pinning the last keep_tiles tiles with an
// evict-last (or evict-normal) policy measured no better (32 MiB) or worse
// (>= 64 MiB), and evict-normal loads throughout cost +6 us.  keep_tiles
// defaults to 0 (BTED_L2_KEEP_MB overrides, for experiments).
//
// Tile sharding (sp > 1, the multi-GPU implicit engine): this GPU stores and
// streams only the tiles k = sr + sp * kl (kl = 0, 1, ...), compactly at
// K + kl * T^2; consumers get the global index k (partials land where the
// unsharded pass would put them).
template <bool kW, class WaitW, class Sm = TPSmem, int kSt = kStages>
__device__ __forceinline__ void tp_produce(Sm& S, const float* __restrict__ K, int nT, const double* w,
                                           int passes, int* tilectr, WaitW wait_w, int dir0 = 0,
                                           int keep_tiles = 0, int sr = 0, int sp = 1) {
    const uint64_t pol = pk::policy_evict_first();            // K is read once per step
    const uint64_t pol_keep = pk::policy_evict_last();        // ... except a tail kept for the next pass
    const int64_t nAll = num_tiles(nT);
    const int64_t nTiles = (nAll - sr + sp - 1) / sp;         // tiles stored on this GPU
    int n = 0, ti = 0;
    for (int pass = 0; pass < passes; ++pass) {
        const bool rev = ((dir0 + pass) & 1) != 0;
        int next = atomicAdd(&tilectr[pass], 1);
        for (;; ++ti) {
            const int64_t kh = next;                          // handing order
            if (kh < nTiles) next = atomicAdd(&tilectr[pass], 1);
            const int64_t kl = kh < nTiles && rev ? nTiles - 1 - kh : kh;     // local tile
            const int64_t k = kh < nTiles ? sr + sp * kl : nAll;              // global tile index
            const uint64_t kpol = kh >= nTiles - keep_tiles ? pol_keep : pol;
            const int ws = ti % kWSlots;
            pk::mbar_wait(&S.wempty[ws], ((uint32_t)(ti / kWSlots) & 1u) ^ 1u);
            S.wtile[ws] = k < nAll ? k : -1;
            int I = 0, J = 0;
            if (k < nAll) {                                   // the coordinates once, for every consumer
                tile_ij(k, nT, I, J);
                S.wI[ws] = I;
                S.wJ[ws] = J;
            }
            if (k >= nAll || !kW) {
                pk::mbar_arrive(&S.wfull[ws]);               // release: the tile index
            } else {
                wait_w(pass, I, J);
                pk::mbar_expect_tx(&S.wfull[ws], 2 * T * 8);
                pk::bulk_g2s(S.wslot[ws][0], w + (int64_t)J * T, T * 8, &S.wfull[ws]);
                pk::bulk_g2s(S.wslot[ws][1], w + (int64_t)I * T, T * 8, &S.wfull[ws]);
            }
            if (k >= nAll) { ++ti; break; }
            const float* src = K + kl * (int64_t)(T * T);
            for (int c = 0; c < kChunks; ++c, ++n) {
                const int st = n % kSt;
                pk::mbar_wait(&S.empty[st], ((uint32_t)(n / kSt) & 1u) ^ 1u);
                pk::mbar_expect_tx(&S.full[st], kChunkBytes);
                pk::bulk_g2s_hint(S.ring[st], src + c * kChunkFloats, kChunkBytes, &S.full[st], kpol);
            }
        }
    }
}
struct NoWait { __device__ void operator()(int, int, int) const {} };
struct PdlWait {                                               // once: kernel A of this step complete
    mutable bool done = false;
    __device__ void operator()(int, int, int) const { if (!done) { pdl_wait(); done = true; } }
};

__device__ __forceinline__ void tp_init_barriers(TPSmem& S) {
    if (threadIdx.x == 0) {
        for (int q = 0; q < kStages; ++q) { pk::mbar_init(&S.full[q], 1); pk::mbar_init(&S.empty[q], kTPWarps); }
        for (int q = 0; q < kWSlots; ++q) { pk::mbar_init(&S.wfull[q], 1); pk::mbar_init(&S.wempty[q], kTPWarps); }
        for (int q = 0; q < 2; ++q) pk::mbar_init(&S.cbar[q], kTPWarps);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
}

// Kernel B (norm pass when kNorm): q = K w into per-tile partials P64.
// tilectr: this launch's tile counter (zeroed).
// kKeepP: store the partials with an L2 evict-last hint (they stay in L2 for kernel C and are
// overwritten by the next pass, never written back) -- for partial buffers well inside L2.
template <bool kNorm, bool kKeepP = false>
__global__ void __launch_bounds__(kTPThreads, kTPBlocksPerSM)
tile_pass_kernel(const float* __restrict__ K, int nT, const double* __restrict__ w, double* __restrict__ P64,
                 int* __restrict__ kflag, int* __restrict__ tilectr, int dir, int keep_tiles,
                 int sr = 0, int sp = 1) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    TPSmem& S = *reinterpret_cast<TPSmem*>(smem_raw);
    tp_init_barriers(S);
    if (threadIdx.x / 32 == kTPWarps) {                      // producer warp: one lane streams
        // (PDL: K streams while kernel A finishes; w only once it has completed)
        if (threadIdx.x % 32 == 0) tp_produce<!kNorm>(S, K, nT, w, 1, tilectr, PdlWait{}, dir, keep_tiles, sr, sp);
        return;
    }
    int n = 0, tile_it = 0, col_it = 0;
    constexpr int kSt = kKeepP ? 64 : 0;                      // tp_store: evict-last / streaming
    if (kNorm) {
        tp_consume<true, true, kSt>(S, nT, P64, kflag, n, tile_it, col_it);
        return;
    }
    if (*kflag) tp_consume<false, true, kSt>(S, nT, P64, kflag, n, tile_it, col_it);
    else tp_consume<false, false, kSt>(S, nT, P64, kflag, n, tile_it, col_it);
    pdl_trigger();                                           // kernel C may launch as CTAs drain
}

// ------------------------------------------------------------------ kernel A: the new factor column
// L is column-major: Lc[k * ldL + i] (factor column k, row i), ldL = NPa, so
// every per-row sum over k reads coalesced.  For every row i:
//   l_i = (K_is - sum_{k<tp} L_ik L_sk) / sqrt(r_ss + mu)    (0 on padding)
// written to Lc[tp][i] and ell[i].  Unit = 64 rows x 4 k-phases (k = g, g+4,
// ...) on 256 threads; the 4 phase sums are added in a fixed order, so a
// row's l_i depends on its own data only.
constexpr int kEllRows = 64;
struct EllSmem {
    double Ls[kMaxM];
    double part[4][kEllRows];
};
struct SyncCTA { __device__ void operator()() const { __syncthreads(); } };
struct SyncConsumers { __device__ void operator()() const { tp_sync(); } };

// k(x_i, x_j) recomputed from the features with K1p/K1i's operation sequence
// (fsub, fma over the features in order, then expf(-gamma * d2)): bitwise the
// stored Gram entry (the tile-sharded engine holds only some tiles of K).
struct XKern {
    const float* X = nullptr; int d = 0; float ng = 0.f; int linear = 0;
    __device__ __forceinline__ float operator()(int64_t i, int64_t j) const {
        float a = 0.f;
        for (int q = 0; q < d; ++q) {
            const float xi = X[i * d + q], xj = X[j * d + q];
            if (linear) a = __fmaf_rn(xi, xj, a);
            else { const float df = __fsub_rn(xi, xj); a = __fmaf_rn(df, df, a); }
        }
        return linear ? a : expf(__fmul_rn(ng, a));
    }
};

// this thread's first 16 factor entries L_ik (k = g, g + 4, ...; they do not depend on the pick s)
__device__ __forceinline__ void ell_rows(int unit, const double* Lc, int64_t ldL, int32_t tp, double (&a)[16]) {
    const int r = threadIdx.x % kEllRows, g = threadIdx.x / kEllRows;
    const int64_t i = (int64_t)unit * kEllRows + r;
#pragma unroll
    for (int q = 0; q < 16; ++q) a[q] = (g + 4 * q < tp) ? __ldcg(&Lc[(int64_t)(g + 4 * q) * ldL + i]) : 0.0;
}
// kPre: a[] was loaded by ell_rows already (ell_kernel does it before waiting for the pick)
template <class Sync, bool kPre = false>
__device__ __forceinline__ void ell_unit(int unit, EllSmem& sm, Sync sync, const float* __restrict__ K, int nT,
                                         int32_t N, double* Lc, int64_t ldL, int32_t tp, uint32_t s,
                                         double rc, double* ell, XKern xk, double (&a)[16]) {
    const int tid = threadIdx.x, r = tid % kEllRows, g = tid / kEllRows;
    const int64_t i = (int64_t)unit * kEllRows + r;
    const float kis = (g == 0 && i < N) ? (xk.X ? xk(i, s) : K[packed_index((int)i, (int)s, nT)]) : 0.f;
    for (int k = tid; k < tp; k += kThreads) sm.Ls[k] = __ldcg(&Lc[(int64_t)k * ldL + s]);
    // this thread's L_ik (k = g, g + 4, ...): loaded before the barrier, 16 at a time
    double acc = 0.0;
    int k = g;
    int na = 0;
    if (!kPre) ell_rows(unit, Lc, ldL, tp, a);
    sync();
#pragma unroll
    for (int q = 0; q < 16; ++q)
        if (g + 4 * q < tp) acc = __fma_rn(a[q], sm.Ls[g + 4 * q], acc);
    (void)na;
    for (k = g + 64; k < tp; k += 32) {                       // tp > 64: 8 more at a time
        double b[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) b[q] = (k + 4 * q < tp) ? __ldcg(&Lc[(int64_t)(k + 4 * q) * ldL + i]) : 0.0;
#pragma unroll
        for (int q = 0; q < 8; ++q)
            if (k + 4 * q < tp) acc = __fma_rn(b[q], sm.Ls[k + 4 * q], acc);
    }
    sm.part[g][r] = acc;
    sync();
    if (g == 0) {
        const double dot = __dadd_rn(__dadd_rn(__dadd_rn(sm.part[0][r], sm.part[1][r]), sm.part[2][r]), sm.part[3][r]);
        double li = 0.0;
        if (i < N) li = __ddiv_rn(__dsub_rn((double)kis, dot), rc);
        Lc[(int64_t)tp * ldL + i] = li;
        ell[i] = li;
    }
    sync();                                                  // smem reusable by the next unit
}

// h = L^T l and |l|^2 from the history (no pass over N):
//   h_k = (Q[k][s] - sum_{j<tp} G[k][j] L_sj) / sqrt(c)  (k < tp),  h_tp = n_s / c
// Q[k][v] = (K l_k)_v (kept by kernel C), G = L^T L (m x m, ldG = m; its new
// column / row tp is this h).  One CTA; thread k sums over j in order.
template <class Sync>
__device__ __forceinline__ void h_unit(double* Ls, Sync sync, const double* Lc, int64_t ldL, const double* Qc,
                                       double* G, int32_t ldG, int32_t tp, uint32_t s, double c, double n_s,
                                       double* h) {
    const int tid = threadIdx.x;
    for (int k = tid; k < tp; k += kThreads) Ls[k] = __ldcg(&Lc[(int64_t)k * ldL + s]);
    sync();
    const double rc = __dsqrt_rn(c);
    for (int k = tid; k <= tp; k += kThreads) {
        double hk;
        if (k < tp) {
            double acc = 0.0;
            // G is symmetric by construction (row and column tp are both written with h below), so
            // G[j][k] = G[k][j]: the threads k of one j read consecutive addresses (coalesced);
            // the same values in the same order as a row walk
            for (int j = 0; j < tp; ++j) acc = __fma_rn(__ldcg(&G[(int64_t)j * ldG + k]), Ls[j], acc);
            hk = __ddiv_rn(__dsub_rn(__ldcg(&Qc[(int64_t)k * ldL + s]), acc), rc);
            G[(int64_t)tp * ldG + k] = hk;
        } else {
            hk = __ddiv_rn(n_s, c);
        }
        G[(int64_t)k * ldG + tp] = hk;
        h[k] = hk;
    }
    sync();
}

// grid = nEll units + 1 CTA for h
__global__ void __launch_bounds__(kThreads)
ell_kernel(const float* __restrict__ K, int nT, int32_t N, double* __restrict__ Lc, int64_t ldL, int32_t tp,
           const double* __restrict__ rdiag, const double* __restrict__ nv, float mu,
           const unsigned long long* __restrict__ keys, int32_t t, double* __restrict__ ell, const double* Qc,
           double* G, int32_t ldG, double* h, uint8_t* __restrict__ sel, XKern xk = XKern{}) {
    __shared__ EllSmem sm;
    // the factor rows (written by earlier, completed steps) before waiting for this step's pick
    double a[16];
    const bool hcta = blockIdx.x == gridDim.x - 1;
    if (!hcta) ell_rows(blockIdx.x, Lc, ldL, tp, a);
    pdl_wait();                                              // kernel C of the previous step complete
    pdl_trigger();                                           // the K.l pass may start streaming K now
    const uint32_t s = key_index(keys[t - 1]);
    if (blockIdx.x == 0 && threadIdx.x == 0) sel[s] = 1;
    const double c = __dadd_rn(rdiag[s], (double)mu);
    if (hcta) {
        h_unit(sm.Ls, SyncCTA{}, Lc, ldL, Qc, G, ldG, tp, s, c, nv[s], h);
        return;
    }
    ell_unit<SyncCTA, true>(blockIdx.x, sm, SyncCTA{}, K, nT, N, Lc, ldL, tp, s, __dsqrt_rn(c), ell, xk, a);
}
// ------------------------------------------------------------------ kernel C: scores
// t == 0 (after the norm pass): n_v = q_v (= ||K_:v||^2), r_vv = K_vv.
// t >= 1: (R l)_v = q_v - sum_{k<tp} L_vk h_k; n_v -= 2 l_v (R l)_v - l_v^2 |l|^2;
// r_vv -= l_v^2.  Score n_v / (r_vv + mu) rounded to fp32, masked, packed key.
// Unit = 32 rows (lanes) x 8 warps; warp w sums the J-range and the k-range
// w of its rows, the 8 partial sums are added in warp order.
// In-library multi-GPU exchange (bted_select with num_devices = P > 1): the P
// devices' partial q = K l live in their own memory; every device's score
// kernel waits for all P "published" flags and sums the P partials itself,
// in rank order, through peer (NVLink) loads -- the all-reduce fused into its
// consumer, bitwise identical on every device and independent of P's layout.
constexpr int kMaxDev = 16;
constexpr int kErrPeerTimeout = 32;           // error-word bit: a peer never published (ENCCL)
struct PeerQ {
    const double* q[kMaxDev];                 // device p's partial q of this step
    const unsigned long long* flag[kMaxDev];  // device p's publish counter
    int P;
    unsigned long long expect;                // this step's counter value
    unsigned long long timeout_ns;            // give up (kErrPeerTimeout) after this long
    __device__ __forceinline__ double sum(int64_t i) const {
        double a = __ldcv(&q[0][i]);
        for (int p = 1; p < P; ++p) a = __dadd_rn(a, __ldcv(&q[p][i]));
        return a;
    }
};
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
// thread 0 of the CTA waits until every device published `expect` (timeout ->
// kErrPeerTimeout, after which no later wait of this device blocks), then the
// CTA proceeds
__device__ __forceinline__ void wait_peers(const PeerQ& pq, int* err) {
    if (threadIdx.x == 0) {
        const unsigned long long t0 = globaltimer_ns();
        for (int p = 0; p < pq.P; ++p) {
            while (ld_acquire_sys(pq.flag[p]) < pq.expect) {
                if ((*(volatile int*)err & kErrPeerTimeout) || globaltimer_ns() - t0 > pq.timeout_ns) {
                    atomicOr(err, kErrPeerTimeout);
                    break;
                }
                __nanosleep(64);
            }
        }
    }
    __syncthreads();
}
// after the producers of this stream's step completed: make their writes
// visible system-wide, then publish the step counter
__global__ void publish_kernel(unsigned long long* flag, unsigned long long v) {
    __threadfence_system();
    asm volatile("st.release.sys.global.u64 [%0], %1;" :: "l"(flag), "l"(v) : "memory");
}

constexpr int kFinRows = 32;
struct FinSmem {
    double part[8][kFinRows];
    double lpart[8][kFinRows];
    double hs[kMaxM + 1];
};

struct NoWaitFn { __device__ void operator()() const {} };
struct PdlWaitFn { __device__ void operator()() const { pdl_wait(); pdl_trigger(); } };
template <class Sync, class WaitP = NoWaitFn>
__device__ __forceinline__ void fin_unit(int unit, int nunits, FinSmem& sm, Sync sync, const double* P64,
                                         int nT, int32_t N, const float* __restrict__ K, float mu,
                                         const double* Lc, int64_t ldL, int32_t tp,
                                         const double* h, double* nv,
                                         double* rdiag, const uint8_t* sel, uint32_t s,
                                         int32_t t, unsigned long long* key_out, int* err,
                                         unsigned long long* top2, double* Qc, bool mark_sel = false,
                                         const double* qin = nullptr, const double* rinit = nullptr,
                                         const PeerQ* pq = nullptr, WaitP wait_partials = WaitP{}) {
    const int lane = threadIdx.x % 32, w = threadIdx.x / 32;
    const int64_t NP = (int64_t)nT * T;
    const int i = unit * kFinRows + lane;
    if (t > 0)
        for (int q = threadIdx.x; q <= tp; q += kThreads) sm.hs[q] = __ldcg(&h[q]);
    // sum_{k in range w} L_ik h_k: inputs of this step's kernel A (complete), not of the K.l pass --
    // computed before wait_partials (fin64_kernel: the PDL wait for the pass)
    sync();
    double la = 0.0;
    if (t > 0) {
        const int kper = (tp + 7) / 8;
        const int k0 = min(tp, w * kper), k1 = min(tp, k0 + kper);
        int k = k0;
        for (; k + 8 <= k1; k += 8) {
            double a[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) a[q] = __ldcg(&Lc[(int64_t)(k + q) * ldL + i]);
#pragma unroll
            for (int q = 0; q < 8; ++q) la = __fma_rn(a[q], sm.hs[k + q], la);
        }
        for (; k < k1; ++k) la = __fma_rn(__ldcg(&Lc[(int64_t)k * ldL + i]), sm.hs[k], la);
    }
    sm.lpart[w][lane] = la;
    wait_partials();
    const int per = (nT + 7) / 8;
    const int j0 = min(nT, w * per), j1 = min(nT, j0 + per);
    double acc = 0.0;
    if (pq) {                                              // q = sum of the devices' partials (rank order)
        acc = w == 0 ? pq->sum(i) : 0.0;
    } else if (qin) {                                      // q given (all-reduced over tile shards)
        acc = w == 0 ? __ldcg(&qin[i]) : 0.0;
    } else {
        const double* src = P64 + i;
        int J = j0;
        for (; J + 16 <= j1; J += 16) {
            double v[16];
#pragma unroll
            for (int q = 0; q < 16; ++q) v[q] = __ldcg(&src[(int64_t)(J + q) * NP]);
#pragma unroll
            for (int q = 0; q < 16; ++q) acc = __dadd_rn(acc, v[q]);
        }
        for (; J < j1; ++J) acc = __dadd_rn(acc, __ldcg(&src[(int64_t)J * NP]));
    }
    sm.part[w][lane] = acc;
    sync();
    if (w == 0) {
        unsigned long long key = 0ull;
        if (i < N) {
            double q = sm.part[0][lane];
#pragma unroll
            for (int u = 1; u < 8; ++u) q = __dadd_rn(q, sm.part[u][lane]);
            double n, r;
            if (t == 0) {
                const int B = i / T, rr = i % T;
                n = q;
                r = rinit ? rinit[i] : (double)K[tile_offset(B, B, nT) * (T * T) + (int64_t)rr * T + rr];
            } else {
                double lh = sm.lpart[0][lane];
#pragma unroll
                for (int u = 1; u < 8; ++u) lh = __dadd_rn(lh, sm.lpart[u][lane]);
                const double rl = __dsub_rn(q, lh);
                const double lv = __ldcg(&Lc[(int64_t)tp * ldL + i]);
                Qc[(int64_t)tp * ldL + i] = q;                 // (K l_tp)_i for later h
                n = __ldcg(&nv[i]);
                n = __fma_rn(-2.0 * lv, rl, n);
                n = __fma_rn(__dmul_rn(lv, lv), sm.hs[tp], n);
                r = __fma_rn(-lv, lv, __ldcg(&rdiag[i]));
            }
            nv[i] = n;
            rdiag[i] = r;
            const bool masked = __ldcg(&sel[i]) != 0 || (uint32_t)i == s;
            if (mark_sel && (uint32_t)i == s) const_cast<uint8_t*>(sel)[i] = 1;
            const float sc = (float)(__ddiv_rn(n > 0.0 ? n : 0.0, __dadd_rn(r, (double)mu)));
            if (!(__dadd_rn(r, (double)mu) > 0.0) || !(sc >= 0.f) || !(sc <= 3.402823466e38f)) {
                if (!masked) atomicOr(err, 1);
            } else if (!masked) {
                key = pack_key(sc, (uint32_t)i);
            }
        }
        const unsigned long long k1 = warp_max_u64(key);
        if (top2) {                                        // the unit's best two keys (K4 near-tie check)
            const unsigned long long k2 = warp_max_u64(key == k1 ? 0ull : key);
            if (lane == 0) {
                top2[((int64_t)t * nunits + unit) * 2] = k1;
                top2[((int64_t)t * nunits + unit) * 2 + 1] = k2;
            }
        }
        if (lane == 0 && k1) atomicMax(key_out, k1);
    }
    sync();                                                // smem reusable by the next unit
}

// The same as two fin_units (rows 64v .. 64v+63, top2 entries 2v and 2v+1) in
// one pass: thread (r, g) sums the J-ranges and k-ranges 2g and 2g+1 of row r
// (the 8 ranges of fin_unit, added in the same order: bitwise the same result).
struct Fin2Smem {
    double part[8][2 * kFinRows];
    double lpart[8][2 * kFinRows];
    double hs[kMaxM + 1];
};
template <class Sync>
__device__ __forceinline__ void fin_unit64(int v, int nunits, Fin2Smem& sm, Sync sync, const double* P64, int nT,
                                           int32_t N, const float* __restrict__ K, float mu, const double* Lc,
                                           int64_t ldL, int32_t tp, const double* h, double* nv, double* rdiag,
                                           uint8_t* sel, uint32_t s, int32_t t, unsigned long long* key_out,
                                           int* err, unsigned long long* top2, double* Qc) {
    constexpr int R = 2 * kFinRows;
    const int tid = threadIdx.x, r = tid % R, g = tid / R, lane = tid % 32, w = tid / 32;
    const int64_t NP = (int64_t)nT * T;
    const int i = v * R + r;
    for (int q = tid; q <= tp; q += kThreads) sm.hs[q] = __ldcg(&h[q]);
    const int per = (nT + 7) / 8, kper = (tp + 7) / 8;
#pragma unroll
    for (int hq = 0; hq < 2; ++hq) {
        const int q = 2 * g + hq;
        const int j0 = min(nT, q * per), j1 = min(nT, j0 + per);
        const double* src = P64 + i;
        double acc = 0.0;
        int J = j0;
        for (; J + 16 <= j1; J += 16) {
            double x[16];
#pragma unroll
            for (int u = 0; u < 16; ++u) x[u] = __ldcg(&src[(int64_t)(J + u) * NP]);
#pragma unroll
            for (int u = 0; u < 16; ++u) acc = __dadd_rn(acc, x[u]);
        }
        for (; J < j1; ++J) acc = __dadd_rn(acc, __ldcg(&src[(int64_t)J * NP]));
        sm.part[q][r] = acc;
    }
    sync();
    if (t > 0) {
#pragma unroll
        for (int hq = 0; hq < 2; ++hq) {
            const int q = 2 * g + hq;
            const int k0 = min(tp, q * kper), k1 = min(tp, k0 + kper);
            double la = 0.0;
            int k = k0;
            for (; k + 8 <= k1; k += 8) {
                double x[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) x[u] = __ldcg(&Lc[(int64_t)(k + u) * ldL + i]);
#pragma unroll
                for (int u = 0; u < 8; ++u) la = __fma_rn(x[u], sm.hs[k + u], la);
            }
            for (; k < k1; ++k) la = __fma_rn(__ldcg(&Lc[(int64_t)k * ldL + i]), sm.hs[k], la);
            sm.lpart[q][r] = la;
        }
    }
    sync();
    if (g == 0) {                                          // warps 0, 1: rows 0..31, 32..63
        unsigned long long key = 0ull;
        if (i < N) {
            double q = sm.part[0][r];
#pragma unroll
            for (int u = 1; u < 8; ++u) q = __dadd_rn(q, sm.part[u][r]);
            double n, rr;
            if (t == 0) {
                const int B = i / T, ri = i % T;
                n = q;
                rr = (double)K[tile_offset(B, B, nT) * (T * T) + (int64_t)ri * T + ri];
            } else {
                double lh = sm.lpart[0][r];
#pragma unroll
                for (int u = 1; u < 8; ++u) lh = __dadd_rn(lh, sm.lpart[u][r]);
                const double rl = __dsub_rn(q, lh);
                const double lv = __ldcg(&Lc[(int64_t)tp * ldL + i]);
                Qc[(int64_t)tp * ldL + i] = q;                 // (K l_tp)_i for later h
                n = __ldcg(&nv[i]);
                n = __fma_rn(-2.0 * lv, rl, n);
                n = __fma_rn(__dmul_rn(lv, lv), sm.hs[tp], n);
                rr = __fma_rn(-lv, lv, __ldcg(&rdiag[i]));
            }
            nv[i] = n;
            rdiag[i] = rr;
            const bool masked = __ldcg(&sel[i]) != 0 || (uint32_t)i == s;
            if ((uint32_t)i == s) sel[i] = 1;
            const float sc = (float)(__ddiv_rn(n > 0.0 ? n : 0.0, __dadd_rn(rr, (double)mu)));
            if (!(__dadd_rn(rr, (double)mu) > 0.0) || !(sc >= 0.f) || !(sc <= 3.402823466e38f)) {
                if (!masked) atomicOr(err, 1);
            } else if (!masked) {
                key = pack_key(sc, (uint32_t)i);
            }
        }
        const unsigned long long k1 = warp_max_u64(key);
        const int unit = 2 * v + w;
        if (top2) {
            const unsigned long long k2 = warp_max_u64(key == k1 ? 0ull : key);
            if (lane == 0 && unit < nunits) {
                top2[((int64_t)t * nunits + unit) * 2] = k1;
                top2[((int64_t)t * nunits + unit) * 2 + 1] = k2;
            }
        }
        if (lane == 0 && k1) atomicMax(key_out, k1);
    }
    sync();
}

__global__ void __launch_bounds__(kThreads)
fin64_kernel(const double* __restrict__ P64, int nT, int32_t N, const float* __restrict__ K, float mu,
             const double* __restrict__ Lc, int64_t ldL, int32_t tp, const double* __restrict__ h,
             double* __restrict__ nv, double* __restrict__ rdiag, const uint8_t* __restrict__ sel,
             const unsigned long long* __restrict__ keys, int32_t t, unsigned long long* __restrict__ key_out,
             int* __restrict__ err, unsigned long long* __restrict__ top2, double* __restrict__ Qc,
             const double* __restrict__ qin = nullptr, const double* __restrict__ rinit = nullptr) {
    __shared__ FinSmem sm;
    // keys[t-1], h and L come from kernels that completed before any CTA of this step's K.l pass
    // let this grid launch (the pass triggers only after its own wait for kernel A: tile_pass_kernel
    // when its consumers finish -- at least one CTA has a tile --, rc_pass_kernel right after its
    // producer's wait); only P64 needs the PDL wait for the pass (inside fin_unit, after L h)
    const uint32_t s = t > 0 ? key_index(keys[t - 1]) : 0xFFFFFFFFu;
    fin_unit(blockIdx.x, gridDim.x, sm, SyncCTA{}, P64, nT, N, K, mu, Lc, ldL, tp, h, nv, rdiag, sel, s, t, key_out,
             err, top2, Qc, false, qin, rinit, nullptr, PdlWaitFn{});
}

// fin64 of the in-library multi-GPU engine: waits for the P partial q of this
// step (PeerQ), sums them while scoring
__global__ void __launch_bounds__(kThreads)
fin64_peer_kernel(PeerQ pq, int nT, int32_t N, const float* __restrict__ K, float mu,
                  const double* __restrict__ Lc, int64_t ldL, int32_t tp, const double* __restrict__ h,
                  double* __restrict__ nv, double* __restrict__ rdiag, const uint8_t* __restrict__ sel,
                  const unsigned long long* __restrict__ keys, int32_t t, unsigned long long* __restrict__ key_out,
                  int* __restrict__ err, unsigned long long* __restrict__ top2, double* __restrict__ Qc,
                  const double* __restrict__ rinit) {
    __shared__ FinSmem sm;
    wait_peers(pq, err);
    const uint32_t s = t > 0 ? key_index(keys[t - 1]) : 0xFFFFFFFFu;
    fin_unit(blockIdx.x, gridDim.x, sm, SyncCTA{}, nullptr, nT, N, K, mu, Lc, ldL, tp, h, nv, rdiag, sel, s, t,
             key_out, err, top2, Qc, false, nullptr, rinit, &pq);
}

// ------------------------------------------------------------------ tile-sharded engine (multi-GPU)
// qpart[i] = sum over the blocks J (in order) of the partials P64[J][i] that
// THIS shard's tiles wrote: tile (min(B,J), max(B,J)) of row i's block B,
// stored here iff its index = sr (mod sp).  The shards' qpart are then summed
// by an all-reduce (the order of that sum is the collective's).
__global__ void __launch_bounds__(kThreads)
qpart_kernel(const double* __restrict__ P64, int nT, int sr, int sp, double* __restrict__ qpart) {
    const int64_t NP = (int64_t)nT * T;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < NP; i += (int64_t)gridDim.x * blockDim.x) {
        const int B = (int)(i / T);
        double acc = 0.0;
        for (int J0 = 0; J0 < nT; J0 += 16) {             // 16 loads in flight; non-owned terms are 0
            double v[16];
#pragma unroll
            for (int q = 0; q < 16; ++q) {
                const int J = J0 + q;
                const bool own = J < nT && tile_offset(min(B, J), max(B, J), nT) % sp == sr;
                v[q] = own ? __ldcg(&P64[(int64_t)J * NP + i]) : 0.0;
            }
#pragma unroll
            for (int q = 0; q < 16; ++q) acc = __dadd_rn(acc, v[q]);
        }
        qpart[i] = acc;
    }
}

// rd[i] = k(x_i, x_i) from the features (the diagonal tiles may live on other shards)
__global__ void diag_init_kernel(XKern xk, int32_t N, int64_t NPa, double* __restrict__ rd) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < NPa; i += (int64_t)gridDim.x * blockDim.x)
        rd[i] = i < N ? (double)xk(i, i) : 0.0;
}

// ------------------------------------------------------------------ the whole step loop in one launch
// Steps t = 1 .. m-1 of the implicit engine in ONE persistent cooperative
// kernel (kTPBlocksPerSM CTAs per SM, all co-resident); every dependency is
// a counter in global memory (release: fence + atomic; acquire: ld.acquire):
//   E  ell units (64 rows, static CTA assignment; each publishes unit_flag[u] = t)
//      and h (the last CTA; hdone)
//   T  tiles (dynamic); the producer copies a tile's w slices once the ell
//      units of its two blocks are published; then tdone += 1 per CTA
//   F  64-row fin units (static assignment) once tdone and h are complete,
//      argmax into keys[t]; fin_done += 1 per CTA
//   next E waits for fin_done (keys[t] final).
// The producer never waits for the consumers' phases, only for ring slots and
// published l: the next step's K chunks stream in while F / E run.  Same
// arithmetic, same order as the three-kernel loop.
struct LoopArgs {
    const float* K; int nT; int32_t N; double* Lc; int64_t ldL; int32_t m; float mu;
    double* rd; double* nv; unsigned long long* keys; double* ell; double* Qc; double* G;
    double* h; double* P64; uint8_t* sel; int* err; unsigned long long* top2; const int* kflag;
    unsigned long long* trace;   // debug (BTED_TRACE): per CTA and step, %globaltimer at 7 phase points
    int* sync;     // zeroed: [0] fin_done, [1] ell_done, [2] tdone, [3] hdone, [4, 4+nEll) unit_flag,
                   // then tilectr[m]
    int keep_tiles;  // L2 reuse across passes (tp_produce); pass 0 = step 1 runs descending
};
__host__ __device__ inline int64_t loop_sync_ints(int64_t nEll, int m) { return 4 + nEll + (int64_t)m; }
static_assert(sizeof(EllSmem) <= sizeof(double) * 2 * kTPWarps * T, "ell scratch aliases colstage");
static_assert(sizeof(Fin2Smem) <= sizeof(double) * 2 * kTPWarps * T, "fin scratch aliases colstage");

__device__ __forceinline__ void trace_at(const LoopArgs& a, int32_t t, int k) {
    if (a.trace && threadIdx.x == 0) {
        unsigned long long ns;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ns));
        a.trace[((int64_t)blockIdx.x * a.m + t) * 8 + k] = ns;
    }
}
__device__ __forceinline__ int ld_acquire_s32(const int* p) {
    int v;
    asm volatile("ld.acquire.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// one thread: wait until *p >= target.  A runaway wait (co-residency broken)
// gives up after ~seconds with err bit 4 instead of hanging the GPU.
__device__ __forceinline__ void spin_ge(const int* p, int target, int* err) {
    long long spins = 0;
    while (ld_acquire_s32(p) < target) {
        if ((++spins & 1023) == 0 && (spins > (1ll << 24) || (*(volatile int*)err & 4))) {
            atomicOr(err, 4);
            return;
        }
        __nanosleep(32);
    }
}
// all consumer threads of the CTA: thread 0 waits, then a CTA-scope barrier
__device__ __forceinline__ void cta_wait_ge(const int* p, int target, int* err) {
    if (threadIdx.x == 0) spin_ge(p, target, err);
    tp_sync();
}
__device__ __forceinline__ void publish_add(int* p) {        // after a tp_sync: this CTA's writes, then +1
    if (threadIdx.x == 0) { __threadfence(); atomicAdd(p, 1); }
}

template <bool kExact>
__device__ __forceinline__ void loop_consumers(TPSmem& S, const LoopArgs& a) {
    const int nEll = (int)((a.ldL) / kEllRows);
    const int nFin = (int)((int64_t)a.nT * T / kFinRows);
    const int nFin64 = nFin / 2;
    int* fin_done = a.sync;
    int* ell_done = a.sync + 1;
    int* tdone = a.sync + 2;
    int* hdone = a.sync + 3;
    int* unit_flag = a.sync + 4;
    EllSmem& es = *reinterpret_cast<EllSmem*>(&S.colstage[0][0][0]);
    Fin2Smem& fs = *reinterpret_cast<Fin2Smem*>(&S.colstage[0][0][0]);
    const bool h_cta = blockIdx.x == gridDim.x - 1;
    int n = 0, tile_it = 0, col_it = 0;
    for (int32_t t = 1; t < a.m; ++t) {
        const int32_t tp = t - 1;
        // E: keys[t-1] final (every CTA's fin units of step t-1; the head kernel for t = 1)
        trace_at(a, t, 0);
        if (t > 1) cta_wait_ge(fin_done, (t - 1) * (int)gridDim.x, a.err);
        trace_at(a, t, 1);
        const uint32_t s = key_index(__ldcg(&a.keys[t - 1]));
        const double c = __dadd_rn(__ldcg(&a.rd[s]), (double)a.mu);
        if (h_cta) {
            h_unit(es.Ls, SyncConsumers{}, a.Lc, a.ldL, a.Qc, a.G, a.m, tp, s, c, __ldcg(&a.nv[s]), a.h);
            publish_add(hdone);
        }
        const double rc = __dsqrt_rn(c);
        for (int u = blockIdx.x; u < nEll; u += gridDim.x) {
            double ar[16];
            ell_unit(u, es, SyncConsumers{}, a.K, a.nT, a.N, a.Lc, a.ldL, tp, s, rc, a.ell, XKern{}, ar);
            if (threadIdx.x == 0) {
                __threadfence();
                asm volatile("st.release.gpu.global.s32 [%0], %1;" :: "l"(unit_flag + u), "r"(t) : "memory");
                atomicAdd(ell_done, 1);
            }
        }
        trace_at(a, t, 2);
        // T: tiles (w gated per tile by the producer)
        trace_at(a, t, 3);
        tp_consume<false, kExact>(S, a.nT, a.P64, nullptr, n, tile_it, col_it);
        tp_sync();
        trace_at(a, t, 4);
        publish_add(tdone);                                 // this CTA's partials of the step are stored
        // F: 64-row fin units, static assignment, once every CTA's partials and h are in
        cta_wait_ge(tdone, t * (int)gridDim.x, a.err);
        if (threadIdx.x == 0) spin_ge(hdone, t, a.err);
        tp_sync();
        trace_at(a, t, 5);
        for (int v = blockIdx.x; v < nFin64; v += gridDim.x)
            fin_unit64(v, nFin, fs, SyncConsumers{}, a.P64, a.nT, a.N, a.K, a.mu, a.Lc, a.ldL, tp, a.h, a.nv, a.rd,
                       a.sel, s, t, a.keys + t, a.err, a.top2, a.Qc);
        tp_sync();
        trace_at(a, t, 6);
        publish_add(fin_done);
    }
}

// the producer's gate before the w copies of tile (I, J) of pass `pass`
// (step t = pass + 1): the ell units of blocks I and J are published (all of
// them, once ell_done says so); then order the async-proxy (TMA) reads of l
// after the generic-proxy writes of the ell phase
struct WaitEll {
    const int* ell_done; const int* unit_flag; int nEll; int* err;
    mutable int ready = 0;                                   // the last pass known complete
    __device__ void operator()(int pass, int I, int J) const {
        const int t = pass + 1;
        if (ready == t) return;
        if (ld_acquire_s32(ell_done) >= t * nEll) {
            ready = t;
        } else {
            for (int u : {2 * I, 2 * I + 1, 2 * J, 2 * J + 1})
                if (u < nEll) spin_ge(unit_flag + u, t, err);
        }
        asm volatile("fence.proxy.async.global;" ::: "memory");
    }
};

__global__ void __launch_bounds__(kTPThreads, kTPBlocksPerSM)
ted_loop_kernel(const LoopArgs a) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    TPSmem& S = *reinterpret_cast<TPSmem*>(smem_raw);
    tp_init_barriers(S);
    const int nEll = (int)(a.ldL / kEllRows);
    if (threadIdx.x / 32 == kTPWarps) {
        // producer: every step's tiles back to back (K never changes)
        if (threadIdx.x % 32 == 0)
            tp_produce<true>(S, a.K, a.nT, a.ell, a.m - 1, a.sync + 4 + nEll, WaitEll{a.sync + 1, a.sync + 4, nEll, a.err},
                              1, a.keep_tiles);
        return;
    }
    if (*a.kflag) loop_consumers<true>(S, a);
    else loop_consumers<false>(S, a);
}

}  // namespace im
}  // namespace bted
