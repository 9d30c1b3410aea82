// small.cuh -- whole-TED-in-one-kernel for small candidate sets (SURVEY.md
// Sec. 8(f) N3: the paper's own workload, M = 500 points per batch, B = 10,
// m = 64, and the |X_U| <= B m point merge TED of Alg. 2 l.6, PAPER.md:156,
// 372-374).  At these sizes a per-step kernel launch costs more than the
// step, so one thread-block CLUSTER runs all m steps of one TED with K held
// in the cluster's distributed shared memory:
//
//   CTA r of a cluster of C owns rows [r*R, r*R+R) of K (dense, ld = N
//   rounded to 4) in its own smem.  Per step: every CTA copies the pivot row
//   from its owner's smem (DSMEM), CTA barrier, deflates its rows except
//   the pivot row s itself (k - (a_i p_j)/c with the same instruction as K2
//   -> bitwise the same elements), computes the new row norms, scores and its
//   masked argmax key, writes the key into every CTA's slot (DSMEM), cluster
//   barrier, each CTA reduces the C keys -> next pivot.  1 cluster barrier
//   per step.  Row s may miss its update: after s is picked no later pivot,
//   multiplier a_i = K_is (read from the pivot copy) or unmasked score reads
//   row s (its entries K_sj live on as K_js in the unselected rows j), so its
//   values cannot change any result -- and since the owner does not write row
//   s in the step that reads it remotely, those reads need no cluster barrier
//   before the deflation (they finish before the reader's exchange barrier,
//   which the owner passes before it next writes row s).  With C = 1 there
//   are no remote readers and every row is updated.
//
// Several TEDs (the B batches) run as independent clusters of one launch.
#pragma once
#include <cstdint>
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include "kernels.cuh"

namespace bted {
namespace sm {

namespace cg = cooperative_groups;
constexpr int kThreads = 512;
constexpr int kWarps = kThreads / 32;
constexpr size_t kSmemBudget = 220 * 1024;

__host__ __device__ __forceinline__ int ldk_for(int N) { return (N + 3) / 4 * 4; }
__host__ __device__ __forceinline__ int rows_per(int N, int C) { return (N + C - 1) / C; }
constexpr int kR = 4;                  // rows per warp iteration (independent reduction chains)
constexpr int kLanePerRow = 32 / kR;   // after warp_sum4: lanes [8h, 8h + 8) hold row h's sum
static_assert(kR == 4, "warp_sum4 reduces four rows");

// Sums of four per-lane values over the warp with 6 shuffles instead of 4 x 5:
// the first two levels (offsets 16, 8) each hand half of the still-open rows
// to the partner, the last three are plain butterflies.  Every row sees the
// xor-butterfly tree of warp_sum (offsets 16, 8, 4, 2, 1; fp32 add is
// commutative), so each result is bitwise warp_sum's.  Returns row
// (l >> 4) * 2 + ((l >> 3) & 1)'s sum, i.e. row l / 8.
__device__ __forceinline__ float warp_sum4(const float (&v)[4], int l) {
    const bool up16 = (l & 16) != 0, up8 = (l & 8) != 0;
    // offset 16: lower lanes keep rows 0, 1; upper lanes keep rows 2, 3
    const float s0 = up16 ? v[0] : v[2], s1 = up16 ? v[1] : v[3];
    const float r0 = __shfl_xor_sync(0xffffffffu, s0, 16), r1 = __shfl_xor_sync(0xffffffffu, s1, 16);
    const float a = __fadd_rn(up16 ? v[2] : v[0], r0), b = __fadd_rn(up16 ? v[3] : v[1], r1);
    // offset 8: keep the even row (lower) or the odd row (upper)
    const float r = __shfl_xor_sync(0xffffffffu, up8 ? a : b, 8);
    float c = __fadd_rn(up8 ? b : a, r);
#pragma unroll
    for (int off = 4; off > 0; off >>= 1) c = __fadd_rn(c, __shfl_xor_sync(0xffffffffu, c, off));
    return c;
}
// dynamic smem of one CTA: band + pivot row + key slots + warp keys + sel
__host__ __device__ __forceinline__ size_t smem_core(int N, int C) {
    const size_t R = (size_t)rows_per(N, C), L = (size_t)ldk_for(N);
    return (R * L + L) * sizeof(float) + (2 * 16 + 2 * kWarps) * sizeof(unsigned long long) + ((R + 15) / 16) * 16;
}
// + the features of all N points staged for the Gram phase (odd row stride d|1:
// lanes reading different points hit different banks)
__host__ __device__ __forceinline__ size_t smem_x(int N, int d) { return (size_t)N * (size_t)(d | 1) * sizeof(float); }
__host__ __device__ __forceinline__ size_t smem_bytes(int N, int C) { return smem_core(N, C); }

template <int C>
__global__ void __launch_bounds__(kThreads, 1)
ted_cluster_kernel(const float* __restrict__ Xall, int32_t N, int32_t d, float gamma, int32_t linear,
                   int32_t m, float mu, unsigned long long* __restrict__ keys_all, int* __restrict__ err,
                   int32_t stage_x, unsigned long long* __restrict__ top2_all,
                   const unsigned long long* __restrict__ forced, int32_t nforced) {
    cg::cluster_group cl = cg::this_cluster();
    const int rank = C == 1 ? 0 : (int)cl.block_rank();
    // a cluster of one CTA needs only the CTA barrier (cluster barriers also
    // invalidate L1)
    auto csync = [&]() {
        if constexpr (C == 1) __syncthreads();
        else cl.sync();
    };
    const int inst = blockIdx.x / C;
    const float* __restrict__ X = Xall + (int64_t)inst * N * d;
    unsigned long long* keys_out = keys_all + (int64_t)inst * m;

    extern __shared__ __align__(16) unsigned char smem[];
    const int R = rows_per(N, C), L = ldk_for(N);
    float* Kb = reinterpret_cast<float*>(smem);                 // [R][L]
    float* piv = Kb + (size_t)R * L;                            // [L]
    unsigned long long* kslot = reinterpret_cast<unsigned long long*>(piv + L);   // [2][16]
    unsigned long long* wred = kslot + 32;                      // [2][kWarps] (step parity)
    uint8_t* sel = reinterpret_cast<uint8_t*>(wred + 2 * kWarps);   // [R]

    const int tid = threadIdx.x, w = tid / 32, l = tid % 32;
    const int r0 = rank * R;
    const int nr = max(0, min(R, N - r0));
    const float ng = -gamma;

    // ---------------- l.1: this CTA's rows of K_VV, plus the first l.3
    // Features from smem when they fit next to the band (stage_x), else from
    // global; the same operands in the same order either way (bitwise the same K).
    const float* Xf = X;
    int xs = d;
    if (stage_x) {
        float* Xs = reinterpret_cast<float*>(smem + smem_core(N, C));
        xs = d | 1;
        for (int q = tid; q < N * d; q += kThreads) Xs[(q / d) * xs + q % d] = X[q];
        Xf = Xs;
    }
    for (int q = tid; q < R; q += kThreads) sel[q] = 0;
    __syncthreads();
    // every CTA of the cluster has started (its shared memory exists) before the
    // first remote (DSMEM) write of the key exchange
    if constexpr (C > 1) cl.sync();
    // K4 (top2_all non-null): every warp records its best two keys of each step,
    // top2[inst][t][rank * kWarps + w][0..1] -- the input of the near-tie check
    const int nU = C * kWarps;
    unsigned long long* top2 = top2_all ? top2_all + (int64_t)inst * m * nU * 2 : nullptr;
    unsigned long long second_local = 0ull;
    auto note = [&](unsigned long long k, unsigned long long& b1, unsigned long long& b2) {
        if (k > b1) { b2 = b1; b1 = k; } else if (k > b2) { b2 = k; }
    };
    auto put_top2 = [&](int t, unsigned long long b1, unsigned long long b2) {
        if (top2) {                                            // lanes 0, 8, 16, 24 hold partial top-2s
#pragma unroll
            for (int off = kLanePerRow; off < 32; off <<= 1)
                top2_merge(b1, b2, __shfl_xor_sync(0xffffffffu, b1, off), __shfl_xor_sync(0xffffffffu, b2, off));
        }
        if (top2 && l == 0) {
            unsigned long long* p = top2 + ((int64_t)t * nU + rank * kWarps + w) * 2;
            p[0] = b1;
            p[1] = b2;
        }
    };
    unsigned long long best_local = 0ull;
    for (int base = w; base < nr; base += kWarps * kR) {
        float acc_norm[kR];
#pragma unroll
        for (int h = 0; h < kR; ++h) acc_norm[h] = 0.f;
        for (int j = l; j < L; j += 32) {
#pragma unroll
            for (int h = 0; h < kR; ++h) {
                const int lr = base + h * kWarps;
                if (lr >= nr) continue;
                const int i = r0 + lr;
                float v = 0.f;
                if (j < N) {
                    float a = 0.f;
                    for (int k = 0; k < d; ++k) {
                        const float xi = Xf[i * xs + k], xj = Xf[j * xs + k];
                        if (linear) a = __fmaf_rn(xi, xj, a);
                        else { const float df = __fsub_rn(xi, xj); a = __fmaf_rn(df, df, a); }
                    }
                    v = linear ? a : expf(__fmul_rn(ng, a));
                }
                Kb[(size_t)lr * L + j] = v;
                acc_norm[h] = __fmaf_rn(v, v, acc_norm[h]);
            }
        }
        float g[kR];
#pragma unroll
        for (int h = 0; h < kR; ++h) g[h] = warp_sum(acc_norm[h]);
        __syncwarp();                                      // the diagonal entry was written by another lane
        if (l == 0) {
#pragma unroll
            for (int h = 0; h < kR; ++h) {
                const int lr = base + h * kWarps;
                if (lr >= nr) continue;
                const int i = r0 + lr;
                const unsigned long long k = score_key(g[h], Kb[(size_t)lr * L + i], mu, (uint32_t)i, false, err);
                note(k, best_local, second_local);
            }
        }
    }
    put_top2(0, best_local, second_local);
    // CTA max -> every CTA's slot[0][rank] -> cluster max
    // (one CTA: every warp reduces the kWarps slots itself after ONE barrier;
    // the slots alternate with the step parity, so the next step's writes
    // cannot race this step's reads)
    auto exchange = [&](unsigned long long key, int parity) -> unsigned long long {
        // only the scoring lanes 0, 8, 16, 24 ever hold a key, so two
        // butterfly levels bring the warp's max to lane 0
        static_assert(kWarps <= 32 && (kWarps & (kWarps - 1)) == 0, "exchange levels");
#pragma unroll
        for (int off = kLanePerRow; off < 32; off <<= 1) {
            const unsigned long long o = __shfl_xor_sync(0xffffffffu, key, off);
            key = o > key ? o : key;
        }
        unsigned long long* wr = wred + parity * kWarps;
        if (l == 0) wr[w] = key;
        __syncthreads();
        unsigned long long v = wr[l % kWarps];            // every lane: max of the kWarps slots
#pragma unroll
        for (int off = kWarps / 2; off > 0; off >>= 1) {
            const unsigned long long o = __shfl_xor_sync(0xffffffffu, v, off);
            v = o > v ? o : v;
        }
        if constexpr (C == 1) {
            return v;
        } else {
            if (w == 0 && l < C) {
                unsigned long long* dst = cl.map_shared_rank(kslot, l);
                dst[parity * 16 + rank] = v;
            }
            csync();
            unsigned long long b = 0ull;
            for (int r = 0; r < C; ++r) b = kslot[parity * 16 + r] > b ? kslot[parity * 16 + r] : b;
            return b;
        }
    };
    unsigned long long best = exchange(best_local, 0);
    if (forced && 0 < nforced) best = forced[0];         // K4 re-run: preset (flagged) picks

    for (int t = 1; t < m; ++t) {
        if (rank == 0 && tid == 0) keys_out[t - 1] = best;
        const int s = (int)key_index(best);
        if (best == 0ull) { if (tid == 0) atomicOr(err, 2); break; }
        // pivot row K[s][:] from its owner's shared memory
        const int owner = s / R;
        const float* src = (C == 1 ? Kb : cl.map_shared_rank(Kb, owner)) + (size_t)(s - owner * R) * L;
        for (int j4 = tid; j4 < L / 4; j4 += kThreads)
            reinterpret_cast<float4*>(piv)[j4] = reinterpret_cast<const float4*>(src)[j4];
        if (owner == rank && tid == 0) sel[s - r0] = 1;
        __syncthreads();                             // this CTA's pivot copy and sel[] (row s is never
                                                     // written again, so remote readers need no barrier)
        const float inv_c = __frcp_rn(__fadd_rn(piv[s], mu));
        best_local = 0ull;
        second_local = 0ull;
        for (int base = w; base < nr; base += kWarps * kR) {
            float acc_norm[kR], a[kR];
            bool act[kR];                            // all rows but the pivot row (see the header)
#pragma unroll
            for (int h = 0; h < kR; ++h) {
                const int lr = base + h * kWarps;
                acc_norm[h] = 0.f;
                act[h] = lr < nr && (C == 1 || r0 + lr != s);   // the pivot row: read remotely now
                a[h] = lr < nr ? piv[r0 + lr] : 0.f;   // K[i][s] = K[s][i]
            }
            for (int j4 = l; j4 < L / 4; j4 += 32) {
                const float4 pv = reinterpret_cast<const float4*>(piv)[j4];
#pragma unroll
                for (int h = 0; h < kR; ++h) {
                    const int lr = base + h * kWarps;
                    if (!act[h]) continue;
                    float4* row = reinterpret_cast<float4*>(Kb + (size_t)lr * L);
                    float4 kv = row[j4];
                    kv.x = deflate1(kv.x, a[h], pv.x, inv_c);
                    kv.y = deflate1(kv.y, a[h], pv.y, inv_c);
                    kv.z = deflate1(kv.z, a[h], pv.z, inv_c);
                    kv.w = deflate1(kv.w, a[h], pv.w, inv_c);
                    row[j4] = kv;
                    acc_norm[h] = __fmaf_rn(kv.x, kv.x, acc_norm[h]);
                    acc_norm[h] = __fmaf_rn(kv.y, kv.y, acc_norm[h]);
                    acc_norm[h] = __fmaf_rn(kv.z, kv.z, acc_norm[h]);
                    acc_norm[h] = __fmaf_rn(kv.w, kv.w, acc_norm[h]);
                }
            }
            const float gl = warp_sum4(acc_norm, l);  // row l / 8 of the group (kLanePerRow)
            __syncwarp();                            // the diagonal entry was written by another lane
            if ((l & (kLanePerRow - 1)) == 0) {      // lane 8h scores row h of the group
                const int lr = base + (l / kLanePerRow) * kWarps;
                if (lr < nr) {
                    const int i = r0 + lr;
                    const bool masked = sel[lr] != 0 || i == s;
                    const unsigned long long k = score_key(gl, Kb[(size_t)lr * L + i], mu, (uint32_t)i, masked, err);
                    note(k, best_local, second_local);
                }
            }
        }
        put_top2(t, best_local, second_local);
        best = exchange(best_local, t & 1);
        if (forced && t < nforced) best = forced[t];
    }
    if (rank == 0 && tid == 0) keys_out[m - 1] = best;
    csync();                                         // no CTA exits while others may read its smem
}

// ---------------------------------------------------------------- N <= 128: one small CTA per TED
// The |X_U| <= B m point merge of Alg. 2 l.6 at the bench's B m = 64,
// and any other TED of at most 128 points.  A whole TED is 64 dependent steps of very
// little work each, so the step's latency chain is the cost: the 512-thread cluster
// kernel spends ~1.5 us per step in shuffle trees and CTA barriers.  Here 4 kMax threads
// hold K in registers, thread (q, j) = (tid / kMax, tid % kMax) the kMax/4 entries of
// column j in rows q kMax/4 .. (K is symmetric: a column is a row, and its squared norm is
// the row norm of Alg. 1 l.3).  Per step, three CTA barriers:
//   the four threads of column s publish it to shared memory | every thread deflates
//   its 16 entries with deflate1 (the instruction every engine uses: K stays bitwise
//   symmetric) and writes its partial sum of squares | the kMax threads of quarter 0 add
//   the four partials ((p0 + p1) + (p2 + p3)), score their column, and the two warps'
//   argmax (redux.sync on the score bits, then on the index bits) meet in shared memory.
// Fixed summation orders throughout (partials: four interleaved accumulators, then
// (a0 + a1) + (a2 + a3)), so exact duplicate points have identical columns, norms and
// scores and tie to the lowest index.  The diagonal entry of column j is carried by its
// quarter-0 thread and updated with the same deflate1 operands as the matrix entry.
// K4: every column is a score unit (nU = kMax; top2_all[inst][t][j] = {key, 0}).
// Two sizes: kMax = 64 (256 threads, 16 entries each) and kMax = 128 (512 threads, 32 entries each:
// e.g. the merge of two 64-point batches).  Units (K4) = kMax, one per column.
constexpr int kTinyMaxN = 128;                     // the largest N the tiny kernels take
__host__ __device__ __forceinline__ int tiny_max_for(int N) { return N <= 64 ? 64 : 128; }
__host__ __device__ __forceinline__ size_t tiny_smem_bytes(int N, int d) {
    const int kMax = tiny_max_for(N);
    return 64 + (size_t)(kMax + 4 * kMax + (size_t)N * (size_t)(d | 1)) * sizeof(float);
}
template <int kMax>
__global__ void __launch_bounds__(4 * kMax, 1)
ted_tiny_kernel(const float* __restrict__ Xall, int32_t N, int32_t d, float gamma, int32_t linear, int32_t m,
                float mu, unsigned long long* __restrict__ keys_all, int* __restrict__ err,
                unsigned long long* __restrict__ top2_all, const unsigned long long* __restrict__ forced,
                int32_t nforced) {
    constexpr int kTinyThreads = 4 * kMax, kTinyRows = kMax / 4, kTinyUnits = kMax, kW0 = kMax / 32;
    extern __shared__ __align__(16) unsigned char tsm[];
    unsigned long long* wbest = reinterpret_cast<unsigned long long*>(tsm);     // [kMax / 32] quarter-0 warps' keys
    float* piv = reinterpret_cast<float*>(tsm + 64);                            // [kMax] pivot column
    float* part = piv + kMax;                                                   // [4][kMax] partial norms
    float* Xs = part + 4 * kMax;                                                // [N][d | 1] features
    const int tid = threadIdx.x, j = tid % kMax, q = tid / kMax, l = tid % 32, w = tid / 32;
    const int inst = blockIdx.x;
    const float* X = Xall + (int64_t)inst * N * d;
    unsigned long long* keys_out = keys_all + (int64_t)inst * m;
    unsigned long long* top2 = top2_all ? top2_all + (int64_t)inst * m * kTinyUnits * 2 : nullptr;
    const int xs = d | 1;
    for (int p = tid; p < N * d; p += kTinyThreads) Xs[(p / d) * xs + p % d] = X[p];
    __syncthreads();
    const bool vj = j < N;
    const float ng = -gamma;
    // l.1: K_ij exactly as the cluster kernel forms it (row i, column j; k ascending)
    float c[kTinyRows];
    {
        float a[kTinyRows];
#pragma unroll
        for (int r = 0; r < kTinyRows; ++r) a[r] = 0.f;
        for (int k = 0; k < d; ++k) {
            const float xj = vj ? Xs[j * xs + k] : 0.f;
#pragma unroll
            for (int r = 0; r < kTinyRows; ++r) {
                const int i = q * kTinyRows + r;
                const float xi = i < N ? Xs[i * xs + k] : 0.f;
                if (linear) a[r] = __fmaf_rn(xi, xj, a[r]);
                else { const float df = __fsub_rn(xi, xj); a[r] = __fmaf_rn(df, df, a[r]); }
            }
        }
#pragma unroll
        for (int r = 0; r < kTinyRows; ++r)
            c[r] = (q * kTinyRows + r < N && vj) ? (linear ? a[r] : expf(__fmul_rn(ng, a[r]))) : 0.f;
    }
    float dg = 0.f;                                         // K_jj (quarter-0 threads)
    if (q == 0 && vj) {
        float a = 0.f;
        for (int k = 0; k < d; ++k) {
            const float xj = Xs[j * xs + k];
            if (linear) a = __fmaf_rn(xj, xj, a);
            else { const float df = __fsub_rn(xj, xj); a = __fmaf_rn(df, df, a); }
        }
        dg = linear ? a : expf(__fmul_rn(ng, a));
    }
    bool selj = false;
    auto put_partial = [&]() {
        float a[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int r = 0; r < kTinyRows; ++r) a[r & 3] = __fmaf_rn(c[r], c[r], a[r & 3]);
        part[q * kMax + j] = __fadd_rn(__fadd_rn(a[0], a[1]), __fadd_rn(a[2], a[3]));
    };
    // after the partials' barrier: quarter 0 scores its columns, the CTA's argmax key
    auto argmax = [&](int t) -> unsigned long long {
        if (q == 0) {
            const float n = __fadd_rn(__fadd_rn(part[j], part[kMax + j]),
                                      __fadd_rn(part[2 * kMax + j], part[3 * kMax + j]));
            const unsigned long long key = vj ? score_key(n, dg, mu, (uint32_t)j, selj, err) : 0ull;
            if (top2) {
                unsigned long long* p = top2 + ((int64_t)t * kTinyUnits + j) * 2;
                p[0] = key;
                p[1] = 0ull;
            }
            const uint32_t hi = (uint32_t)(key >> 32);
            const uint32_t mh = __reduce_max_sync(0xffffffffu, hi);
            const uint32_t ml = __reduce_max_sync(0xffffffffu, hi == mh ? (uint32_t)key : 0u);
            if (l == 0) wbest[w] = ((unsigned long long)mh << 32) | ml;
        }
        __syncthreads();
        unsigned long long bb = wbest[0];
#pragma unroll
        for (int q2 = 1; q2 < kW0; ++q2) bb = wbest[q2] > bb ? wbest[q2] : bb;
        return bb;
    };
    put_partial();
    __syncthreads();
    unsigned long long best = argmax(0);
    if (forced && 0 < nforced) best = forced[0];             // K4 re-run: preset (flagged) picks
    for (int t = 1; t < m; ++t) {
        if (tid == 0) keys_out[t - 1] = best;
        if (best == 0ull) { if (tid == 0) atomicOr(err, 2); break; }
        const int s = (int)key_index(best);
        selj |= j == s;
        if (j == s) {                                       // column s, rows 16q ..: publish
#pragma unroll
            for (int r = 0; r < kTinyRows; r += 4)
                *reinterpret_cast<float4*>(&piv[q * kTinyRows + r]) = make_float4(c[r], c[r + 1], c[r + 2], c[r + 3]);
        }
        __syncthreads();
        const float inv_c = __frcp_rn(__fadd_rn(piv[s], mu));   // 1 / (K_ss + mu)
        const float pj = piv[j];                                // K_sj
#pragma unroll
        for (int r = 0; r < kTinyRows; r += 4) {
            const float4 a = *reinterpret_cast<const float4*>(&piv[q * kTinyRows + r]);   // K_is
            c[r] = deflate1(c[r], a.x, pj, inv_c);
            c[r + 1] = deflate1(c[r + 1], a.y, pj, inv_c);
            c[r + 2] = deflate1(c[r + 2], a.z, pj, inv_c);
            c[r + 3] = deflate1(c[r + 3], a.w, pj, inv_c);
        }
        if (q == 0) dg = deflate1(dg, pj, pj, inv_c);
        put_partial();
        __syncthreads();
        best = argmax(t);
        if (forced && t < nforced) best = forced[t];
    }
    if (tid == 0) keys_out[m - 1] = best;
}

}  // namespace sm
}  // namespace bted

