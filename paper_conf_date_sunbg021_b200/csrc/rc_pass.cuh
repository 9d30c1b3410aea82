// rc_pass.cuh -- the implicit engine's K.l pass (kernel B of implicit.cuh) with
// the Gram RECOMPUTED on the tensor cores instead of streamed from HBM.
//
// Alg. 1 in the implicit form of implicit.cuh needs, every
// greedy step, q = K l over the whole packed Gram: 2 N^2 bytes of HBM reads
// (84 us at N = 16384, 0.99 of the measured copy bandwidth -- the step's floor
// as long as K is READ).  K is a function of the N x d features (d <= 16), so
// each 128 x 128 tile can instead be rebuilt on chip: the six bf16 MMAs of
// gram_tc.cuh (one TMEM accumulator) and the K epilogue (kval2) -- exactly the
// numbers the tensor-core Gram kernel stores, because the MMA results do not
// depend on where an operand row sits in its tile (scripts/tc_sym_probe.cu) and
// the epilogue is the same function.  The fp64 products and the canonical
// per-128 trees are those of tp_consume (implicit.cuh), pair for pair (pairwise
// sums commute), so this pass writes bitwise the partials of the streaming pass.
//
// One persistent CTA per SM, 16 worker warps + 1 producer warp; four tiles in
// flight (the 512 TMEM columns = four 128-column accumulators).  Worker group s
// (warps 4s .. 4s + 3) takes the tiles i = s (mod 4) of the CTA's contiguous
// range; warp 4s + qd owns TMEM lane quarter qd of its tile, end to end:
//   TMEM -> K (16 columns per step) -> a private transpose through shared
//   memory -> per lane a 4 x 4 block (4 tile rows x 4 columns) -> fp32 -> fp64
//   -> row groups (4 columns, mul + 3 fma) and column groups (4 rows).
// The A operand is stored with its rows permuted (gram_tc.cuh rc_lane_of_row:
// tile row 16a + 4qd + r' in TMEM lane 32qd + 4a + r'), so in the canonical
// 32-leaf trees (levels 16, 8, 4, 2, 1) the levels a warp cannot do alone come
// LAST: row trees -- levels 16 / 8 / 4 across the warp's 8 column steps in
// registers, 2 / 1 across 4 lanes once per tile; column trees -- 16 / 8 / 4
// across the warp's lanes (per column step, through a small per-warp buffer),
// 2 / 1 across the 4 warps of the tile once per tile.  No ring between warps:
// the producer lane (TMA operand blocks, w slices, the six MMAs per tile) and a
// per-tile "accumulator free" barrier are the only hand-offs.
//
// Status (B200, N = 16384, bench config): correct -- bitwise the streaming pass's
// partials (tests/test_gpu_recompute.py) -- but 121 us per pass against 84 us for the
// streaming pass, so it is opt-in (BTED_FLAG_RECOMPUTE).  The pass is issue-bound:
// ~13.4 warp-instruction slots per Gram entry (K: fma/mul/max/ex2 ~ 4.5, fp32 -> fp64
// 2, the two fp64 products 2, transposes, trees and waits the rest) at ~40 % issue
// efficiency, while streaming costs ~12 slots per entry and hides them under the 2 N^2
// bytes of HBM reads.  profiles/notes/recompute_pass.md has the design sequence.
//
// The accuracy guard (gram_tc.cuh tc_ok) is read on the device: when it fails
// the stored Gram is the direct-difference one and the workers read their K
// values from it (global loads) instead of TMEM -- the same numbers as the
// streaming pass either way.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "gram_tc.cuh"
#include "implicit.cuh"

namespace bted {
namespace rc {

using pk::T;
constexpr int kGroups = 3;                                     // worker groups of 4 warps (one tile each)
constexpr int kWorkWarps = 4 * kGroups;                        // 12
constexpr int kSlots = 4;                                      // TMEM accumulators: one more than the groups, so a
                                                               // group's next MMA never waits for the group itself
constexpr int kProdWarp = kWorkWarps;
constexpr int kThreads = (kWorkWarps + 1) * 32;                // 416
constexpr int kTbLd = 20;                                      // transpose buffer pitch (floats): conflict-free
constexpr int kCbLd = 18;                                      // column buffer pitch (doubles): conflict-free

struct RCSmem {
    uint8_t op[2][2][tc::kBlockBytes];                         // 96 KiB: [slot][A (I, row-permuted), B (J)]
    double wst[2][kSlots][2][T];                               // 16 KiB: [buf][tile slot][w_J, w_I]
    double colq[2][kSlots][4][T];                              // 32 KiB: column sums after levels 16/8/4 [buf][s][qd][col]
    float tb[kWorkWarps][32 * kTbLd];                          // 40 KiB: per-warp transpose buffers
    double cb[kWorkWarps][8 * kCbLd];                          // 18 KiB: per-warp column-group buffers
    float ncs[kWorkWarps][T];                                  // 8 KiB: per-warp n_J
    uint64_t opfull[2], mmafull[kSlots], tmfree[kSlots], wfull[2][kSlots];
    uint32_t tmem;
};
constexpr size_t kSmemBytes = sizeof(RCSmem);
static_assert(kSmemBytes <= 232448, "rc_pass: shared memory over the sm_100 per-block limit");

// tile row of TMEM lane (quarter qd, lane) under the A operand's row permutation
__device__ __forceinline__ int rc_row(int qd, int lane) { return tc::rc_row_of_lane(32 * qd + lane); }
__device__ __forceinline__ void group_sync(int g) {            // named barrier 1 + g: the 4 warps of group g
    asm volatile("bar.sync %0, 128;" :: "r"(1 + g) : "memory");
}

// kNorm: the norm pass (row / column partials of K_ij^2), else q = K w.
template <bool kNorm, bool kExact, bool kTc>
__device__ __forceinline__ void rc_work(RCSmem& S, const float* __restrict__ nrm, float gamma, int32_t N,
                                        const float* __restrict__ K, int nT, int64_t k0, int cnt,
                                        double* __restrict__ P64, int* __restrict__ kflag) {
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const int g = warp / 4, qd = warp % 4, a = lane >> 2, b = lane & 3;
    const int Lrow = rc_row(qd, lane);                          // tile row of this lane's TMEM lane
    const int64_t NP = (int64_t)nT * T;
    const float ngl2e = __fmul_rn(-gamma, 1.4426950408889634f);
    const unsigned long long g2 = tc::f2pack(ngl2e, ngl2e);
    float* tb = S.tb[warp];
    double* cb = S.cb[warp];
    float* ncs = S.ncs[warp];
    bool odd_value = false;
    int I = 0, J = 0;
    if (g < cnt) pk::tile_ij(k0 + g, nT, I, J);
    float nr_next = 0.f;
    float4 nj_next = make_float4(0.f, 0.f, 0.f, 0.f);
    if (kTc && g < cnt) {
        nr_next = __ldg(&nrm[(int64_t)I * T + Lrow]);
        nj_next = __ldg(reinterpret_cast<const float4*>(nrm + (int64_t)J * T) + lane);
    }
    for (int it = g; it < cnt; it += kGroups) {
        const int s = it % kSlots, u = it / kSlots;            // TMEM / w slot, its u-th use
        const uint32_t ph = (uint32_t)u & 1u;
        const bool offdiag = I != J;
        const bool edge = (I + 1) * T > N || (J + 1) * T > N;
        const bool rowv = I * T + Lrow < N;
        int In = I, Jn = J;                                     // this group's next tile, it + 3
        for (int q = 0; q < kGroups; ++q) if (++Jn == nT) { ++In; Jn = In; }
        float nr = 0.f;
        if (kTc) {
            nr = nr_next;
            __syncwarp();
            reinterpret_cast<float4*>(ncs)[lane] = nj_next;
            __syncwarp();
            if (it + kGroups < cnt) {
                nr_next = __ldg(&nrm[(int64_t)In * T + Lrow]);
                nj_next = __ldg(reinterpret_cast<const float4*>(nrm + (int64_t)Jn * T) + lane);
            }
        }
        const unsigned long long nr2 = tc::f2pack(nr, nr);
        const double* const wJ = &S.wst[u & 1][s][0][0];
        const double* const wI = &S.wst[u & 1][s][1][0];
        pk::mbar_wait(&S.wfull[u & 1][s], (uint32_t)(u >> 1) & 1u);   // w slices of this tile (q = K w)
        double wi[4];                                           // w_I on this lane's 4 tile rows 16a + 4qd ..
        if (!kNorm) {
            const double2 w01 = *reinterpret_cast<const double2*>(&wI[16 * a + 4 * qd]);
            const double2 w23 = *reinterpret_cast<const double2*>(&wI[16 * a + 4 * qd + 2]);
            wi[0] = w01.x; wi[1] = w01.y; wi[2] = w23.x; wi[3] = w23.y;
        }
        if (kTc) {
            pk::mbar_wait(&S.mmafull[s], ph);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        }
        const uint32_t taddr = S.tmem + (uint32_t)(s * T) + ((uint32_t)(32 * qd) << 16);
        const float* Ktile = K + (k0 + it) * (int64_t)(T * T) + (int64_t)Lrow * T;   // the stored row (!kTc)
        double rt[4][3];                                        // pending row-tree values (levels 16 / 8)
        double* cq = &S.colq[u & 1][s][qd][0];
#pragma unroll
        for (int step = 0; step < 8; ++step) {
            // column step order 0 4 2 6 1 5 3 7: level 16 pairs (i, i + 4), 8 (i, i + 2), 4 (i, i + 1)
            const int i8 = ((step & 1) << 2) | ((step & 2) ? 2 : 0) | ((step & 4) ? 1 : 0);
            const int c0 = 16 * i8;
            float o[16];
            if (kTc) {
                uint32_t uu[16];
                tc::tmem_ld16_async(taddr + (uint32_t)c0, uu);
                float4 nc[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) nc[q] = reinterpret_cast<const float4*>(ncs + c0)[q];
                tc::tmem_wait_ld();
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    tc::kval2(__uint_as_float(uu[4 * q]), __uint_as_float(uu[4 * q + 1]),
                              tc::f2add(nr2, tc::f2pack(nc[q].x, nc[q].y)), g2, o[4 * q], o[4 * q + 1]);
                    tc::kval2(__uint_as_float(uu[4 * q + 2]), __uint_as_float(uu[4 * q + 3]),
                              tc::f2add(nr2, tc::f2pack(nc[q].z, nc[q].w)), g2, o[4 * q + 2], o[4 * q + 3]);
                }
                if (edge) {
#pragma unroll
                    for (int q = 0; q < 16; ++q)
                        if (!rowv || J * T + c0 + q >= N) o[q] = 0.f;
                }
            } else {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const float4 v = __ldg(reinterpret_cast<const float4*>(Ktile + c0) + q);
                    o[4 * q] = v.x; o[4 * q + 1] = v.y; o[4 * q + 2] = v.z; o[4 * q + 3] = v.w;
                }
            }
            // transpose: lane = TMEM lane (row) -> lane (a, b) = rows 4a .. 4a + 3 (TMEM lanes), columns 4b ..
            __syncwarp();
#pragma unroll
            for (int q = 0; q < 4; ++q)
                *reinterpret_cast<float4*>(tb + lane * kTbLd + 4 * q) =
                    make_float4(o[4 * q], o[4 * q + 1], o[4 * q + 2], o[4 * q + 3]);
            __syncwarp();
            double wc[4];
            if (!kNorm) {
                const double2 w01 = *reinterpret_cast<const double2*>(&wJ[c0 + 4 * b]);
                const double2 w23 = *reinterpret_cast<const double2*>(&wJ[c0 + 4 * b + 2]);
                wc[0] = w01.x; wc[1] = w01.y; wc[2] = w23.x; wc[3] = w23.y;
            }
            double gs[4], cg[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const float4 kv = *reinterpret_cast<const float4*>(tb + (4 * a + r) * kTbLd + 4 * b);
                const float f32[4] = {kv.x, kv.y, kv.z, kv.w};
                double kd[4];
#pragma unroll
                for (int x = 0; x < 4; ++x) {
                    kd[x] = kExact ? (double)f32[x] : im::f2d_pos(f32[x]);
                    if (kNorm) odd_value |= im::not_pos_normal(f32[x]);
                }
                const double* f = kNorm ? kd : wc;
                double acc = __dmul_rn(kd[0], f[0]);
                acc = __fma_rn(kd[1], f[1], acc);
                acc = __fma_rn(kd[2], f[2], acc);
                gs[r] = __fma_rn(kd[3], f[3], acc);
#pragma unroll
                for (int x = 0; x < 4; ++x) {
                    const double m = kNorm ? kd[x] : wi[r];
                    cg[x] = r == 0 ? __dmul_rn(kd[x], m) : __fma_rn(kd[x], m, cg[x]);
                }
            }
            // row trees, levels 16 / 8 / 4 over the column steps (group q = 4 i8 + b)
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const double v = gs[r];
                switch (step) {
                    case 0: rt[r][0] = v; break;                                        // i = 0
                    case 1: rt[r][0] = __dadd_rn(rt[r][0], v); break;                   // 4: L16[0]
                    case 2: rt[r][1] = v; break;                                        // 2
                    case 3: rt[r][0] = __dadd_rn(rt[r][0], __dadd_rn(rt[r][1], v)); break;   // 6: L8[0]
                    case 4: rt[r][1] = v; break;                                        // 1
                    case 5: rt[r][1] = __dadd_rn(rt[r][1], v); break;                   // 5: L16[1]
                    case 6: rt[r][2] = v; break;                                        // 3
                    default: rt[r][0] = __dadd_rn(rt[r][0], __dadd_rn(rt[r][1], __dadd_rn(rt[r][2], v)));  // 7
                }
            }
            // column groups q' = 4a + qd of columns c0 + 4b + x: levels 16 / 8 / 4 (a +- 4, 2, 1) in the warp
            *reinterpret_cast<double2*>(cb + a * kCbLd + 4 * b) = make_double2(cg[0], cg[1]);
            *reinterpret_cast<double2*>(cb + a * kCbLd + 4 * b + 2) = make_double2(cg[2], cg[3]);
            __syncwarp();
            {
                const int cc = lane & 15, h = lane >> 4;            // column c0 + cc, a in {h, h+2, h+4, h+6}
                const double v0 = __dadd_rn(cb[h * kCbLd + cc], cb[(h + 4) * kCbLd + cc]);          // level 16
                const double v2 = __dadd_rn(cb[(h + 2) * kCbLd + cc], cb[(h + 6) * kCbLd + cc]);
                const double v = __dadd_rn(v0, v2);                                                // level 8
                const double vv = __dadd_rn(v, __shfl_xor_sync(0xffffffffu, v, 16));              // level 4
                if (h == 0) cq[c0 + cc] = vv;
            }
            __syncwarp();
        }
        if (kTc) {
            asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        }
        // rows: the level-4 values of groups b (4 rows) -> levels 2 (b +- 2), 1 (b +- 1) across the 4 lanes;
        // reduce-scatter: lane b ends with row 4a + b's partial
        {
            const bool hi2 = (b & 2) != 0;
            const double s0 = __shfl_xor_sync(0xffffffffu, hi2 ? rt[0][0] : rt[2][0], 2);
            const double s1 = __shfl_xor_sync(0xffffffffu, hi2 ? rt[1][0] : rt[3][0], 2);
            const double h0 = __dadd_rn(hi2 ? rt[2][0] : rt[0][0], s0);          // row (hi2 ? 2 : 0)
            const double h1 = __dadd_rn(hi2 ? rt[3][0] : rt[1][0], s1);          // row (hi2 ? 3 : 1)
            const bool odd = (b & 1) != 0;
            const double mine = odd ? h1 : h0, other = odd ? h0 : h1;
            const double rsum = __dadd_rn(mine, __shfl_xor_sync(0xffffffffu, other, 1));
            const int row = 16 * a + 4 * qd + (hi2 ? 2 : 0) + (odd ? 1 : 0);
            __stcs(P64 + (int64_t)J * NP + (int64_t)I * T + row, rsum);
        }
        // columns: levels 2 (qd +- 2) and 1 (qd +- 1) over the group's 4 warps
        group_sync(g);
        if (offdiag) {
            const int col = 32 * qd + lane;
            const double* c4 = &S.colq[u & 1][s][0][col];
            const double v0 = __dadd_rn(c4[0], c4[2 * T]), v1 = __dadd_rn(c4[T], c4[3 * T]);
            __stcs(P64 + (int64_t)I * NP + (int64_t)J * T + col, __dadd_rn(v0, v1));
        }
        __syncwarp();
        if (lane == 0) pk::mbar_arrive(&S.tmfree[s]);           // accumulator, w buffer and colq of slot s free
        I = In;
        J = Jn;
    }
    if (kNorm && odd_value) atomicOr(kflag, 1);
}

template <bool kNorm>
__global__ void __launch_bounds__(kThreads, 1)
rc_pass_kernel(const uint8_t* __restrict__ opP, const uint8_t* __restrict__ opA, const float* __restrict__ nrm,
               const int* __restrict__ nmax_bits, float gamma, int32_t N, const float* __restrict__ K, int nT,
               const double* __restrict__ w, double* __restrict__ P64, int* __restrict__ kflag) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    RCSmem& S = *reinterpret_cast<RCSmem*>(smem_raw);
    const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
    const bool tc = tc::tc_ok(nmax_bits, gamma);               // else: read the stored (direct-form) Gram
    if (threadIdx.x == 0) {
        for (int q = 0; q < 2; ++q) pk::mbar_init(&S.opfull[q], 1);
        for (int q = 0; q < kSlots; ++q) {
            pk::mbar_init(&S.mmafull[q], 1);
            pk::mbar_init(&S.tmfree[q], 4);
            pk::mbar_init(&S.wfull[0][q], 1);
            pk::mbar_init(&S.wfull[1][q], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (tc && warp == 0) tc::tmem_alloc<kSlots * T>(&S.tmem);
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

    const int64_t ntiles = pk::num_tiles(nT);
    const int64_t per = (ntiles + gridDim.x - 1) / gridDim.x;
    const int64_t k0 = min((int64_t)blockIdx.x * per, ntiles), k1 = min(k0 + per, ntiles);
    const int cnt = (int)(k1 - k0);

    if (warp == kProdWarp) {
        if (lane != 0) return;
        int sI0 = -1, sI1 = -1;                                // the A block held by operand slot 0 / 1
        auto load = [&](int I, int J, int b) {                 // operand blocks of tile (I, J) into slot b
            int& sI = b ? sI1 : sI0;
            const bool newI = sI != I;
            pk::mbar_expect_tx(&S.opfull[b], (newI ? tc::kBlockBytes : 0u) + tc::kBlockBytes);
            if (newI) pk::bulk_g2s(S.op[b][0], opP + (size_t)I * tc::kBlockBytes, tc::kBlockBytes, &S.opfull[b]);
            pk::bulk_g2s(S.op[b][1], opA + (size_t)J * tc::kBlockBytes, tc::kBlockBytes, &S.opfull[b]);
            sI = I;
        };
        auto next = [&](int& I, int& J) { if (++J == nT) { ++I; J = I; } };
        int I = 0, J = 0;
        if (cnt > 0) pk::tile_ij(k0, nT, I, J);
        int In = I, Jn = J;                                    // tile it + 2
        if (tc) {
            if (cnt > 0) { load(In, Jn, 0); next(In, Jn); }
            if (cnt > 1) { load(In, Jn, 1); next(In, Jn); }
        }
        // w slices of tile t into buffer (t / 4) & 1 of slot t % 4: tiles 0 .. 3 at their own
        // iteration, tile t + 4 right after tile t - 4 released the buffer (a tile of slack)
        int wI_ = I, wJ_ = J;                                  // the tile whose w is issued next
        auto issue_w = [&](int t) {
            const int ss = t % kSlots, bb = (t / kSlots) & 1;
            if (kNorm) {
                pk::mbar_arrive(&S.wfull[bb][ss]);
            } else {
                pk::mbar_expect_tx(&S.wfull[bb][ss], 2 * T * 8);
                pk::bulk_g2s(S.wst[bb][ss][0], w + (int64_t)wJ_ * T, T * 8, &S.wfull[bb][ss]);
                pk::bulk_g2s(S.wst[bb][ss][1], w + (int64_t)wI_ * T, T * 8, &S.wfull[bb][ss]);
            }
            next(wI_, wJ_);
        };
        if (!kNorm && cnt > 0) {
            im::pdl_wait();                                    // l of this step written (previous kernel)
            // this CTA may let kernel C launch only now: worker groups without a tile finish at
            // once, and kernel C reads this step's h and L before its own wait for the partials
            im::pdl_trigger();
        }
        for (int t = 0; t < kSlots && t < cnt; ++t) issue_w(t);
        for (int it = 0; it < cnt; ++it) {
            const int s = it % kSlots, b = it & 1;
            // slot s is free once group s finished tile it - 4 (accumulator read out, w buffer used)
            if (it >= kSlots) pk::mbar_wait(&S.tmfree[s], (uint32_t)((it - kSlots) / kSlots) & 1u);
            if (it + kSlots < cnt) issue_w(it + kSlots);
            if (tc) {
                pk::mbar_wait(&S.opfull[b], (uint32_t)(it >> 1) & 1u);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                tc::issue_gram_mmas(S.tmem + (uint32_t)(s * T), tc::smem_u32(S.op[b][0]), tc::smem_u32(S.op[b][1]));
                tc::mma_commit(&S.mmafull[s]);
                if (it + 2 < cnt) {                            // operand slot b is free once these MMAs completed
                    pk::mbar_wait(&S.mmafull[s], (uint32_t)(it / kSlots) & 1u);
                    load(In, Jn, b);
                    next(In, Jn);
                }
            }
        }
        return;
    }

    if (tc) {
        if (kNorm) rc_work<true, true, true>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
        else if (*kflag) rc_work<false, true, true>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
        else rc_work<false, false, true>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
    } else {
        if (kNorm) rc_work<true, true, false>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
        else if (*kflag) rc_work<false, true, false>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
        else rc_work<false, false, false>(S, nrm, gamma, N, K, nT, k0, cnt, P64, kflag);
    }
    if (tc) {
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        asm volatile("bar.sync 4, %0;" :: "n"(kWorkWarps * 32) : "memory");   // every worker done with TMEM
        if (warp == 0) {
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            tc::tmem_free<kSlots * T>(S.tmem);
        }
    }
}

}  // namespace rc
}  // namespace bted
