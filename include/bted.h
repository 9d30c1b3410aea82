/*
 * bted.h -- C ABI of the B200-native BTED hot path (libbted.so).
 *
 * Batch Transductive Experimental Design, Sun, Bai, Geng, Yu, "Deep Neural
 * Network Hardware Deployment Optimization via Advanced Active Learning",
 * DATE 2021.  Citations are to /root/reference/PAPER.md (line, section).
 *
 *   TED(V, mu, m)         Algorithm 1, PAPER.md:134-148 (Sec. III-A)
 *   BTED(V, mu, M, m, B)  Algorithm 2, PAPER.md:152-156 (Sec. III-A)
 *
 * Readings of the paper adopted by this library:
 *   k(v1,v2) = exp(-gamma ||v1-v2||^2) (RBF; PAPER.md:130 says "Euclidean
 *   distance", which is ill-posed for TED); the argmax of Alg.1 l.3 runs over
 *   not-yet-selected points; ties go to the lowest index; l.5 deflates the
 *   whole matrix; indices are returned in selection order.
 *
 * Conventions for every entry point:
 *   - All pointers are plain host pointers unless a parameter says "device".
 *     Output buffers are caller-allocated; the library never keeps a caller
 *     pointer after return, except a device X adopted with x_on_device = 1,
 *     which must outlive the context.
 *   - Feature matrices are row-major fp32, N rows x d columns, contiguous.
 *   - Every call returns a bted_status; no C++ exception crosses the ABI.
 *     On error the outputs are unspecified and bted_last_error() returns a
 *     thread-local description.  After a CUDA error the context is poisoned
 *     (BTED_ESTATE on later calls).
 *   - A context is not thread-safe; distinct contexts may be used from
 *     distinct threads.  All work of a context runs on its CUDA stream.
 *   - There is no CPU fallback: without a usable sm_100 device every compute
 *     entry point fails with BTED_ECUDA.
 */
#ifndef BTED_H_
#define BTED_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct bted_ctx bted_ctx;    /* opaque; owns the device memory of one candidate set */

typedef enum {
    BTED_KERNEL_RBF = 0,     /* k(x,y) = exp(-gamma ||x-y||^2)          (reading A1) */
    BTED_KERNEL_LINEAR = 1   /* k(x,y) = x.y  -- test-only (closed-form pin C8)    */
} bted_kernel;

typedef enum {
    BTED_OK = 0,
    BTED_EINVAL = 1,         /* invalid argument (see each call)                    */
    BTED_ENOMEM = 2,         /* device or host allocation failed                    */
    BTED_ECUDA = 3,          /* CUDA runtime error / no usable device               */
    BTED_ENCCL = 4,          /* multi-GPU exchange failed: an NCCL error, or a peer
                                that stopped publishing (flag wait / collective timeout) */
    BTED_ENUMERIC = 5,       /* NaN score or non-positive k(v,v)+mu during a run    */
    BTED_ESTATE = 6          /* context poisoned by an earlier CUDA error           */
} bted_status;

/* flags */
#define BTED_FLAG_NO_GRAPH 1u   /* launch the m-step loop eagerly (debug / profiling) */
#define BTED_FLAG_DENSE    4u   /* literal deflation on a dense K (N x ld, 8 N^2 bytes per step)
                                   instead of the packed upper-triangular tiles (used when
                                   d <= 32; default engine: BTED_FLAG_IMPLICIT below, 2 N^2 bytes
                                   per step).  Also used when d > 32.  Row-shard contexts
                                   (bted_shard_*) are always dense. */
#define BTED_FLAG_NO_SMALL 8u   /* never use the one-kernel cluster TED for small candidate sets
                                   (N <= ~940: K in distributed shared memory)               */
#define BTED_FLAG_TMA     16u   /* packed layout: stream K through the persistent TMA ring
                                   (cp.async.bulk + mbarrier) instead of the default one-CTA-per-
                                   tile 256-bit-load kernel (which measured faster on B200)   */
#define BTED_FLAG_IMPLICIT 32u   /* implicit deflation (N2) -- the DEFAULT engine for packed layouts
                                   with m <= 256 (the flag is accepted and changes nothing): keep
                                   the packed Gram K read-only and carry K^(t) = K - L L^T by its
                                   fp64 factor L; one K.l pass per step (2 N^2 bytes, read only)
                                   + O(N m).  Same selections in exact arithmetic. */
#define BTED_FLAG_LITERAL  64u   /* literal deflation (Alg. 1 l.5 as written): materialise K^(t)
                                   every step in the packed layout (K2p, 4 N^2 bytes per step;
                                   bted_debug_copy_K then returns K^(t)).  Implied by DENSE. */
#define BTED_FLAG_PERSISTENT_LOOP 256u /* implicit engine: all m-1 steps in ONE cooperative persistent
                                   kernel with grid barriers between the phases, instead of the
                                   default three kernels per step (factor column, K.l pass, scores) */
#define BTED_FLAG_NO_REFINE 128u /* disable K4: near ties (fp32 scores within 2e-5 of the best) are
                                   otherwise re-scored exactly in fp64 from the features and the
                                   exact argmax taken (every single-GPU engine, the tile-sharded
                                   engine and the row-shard API's symmetric mode)               */
#define BTED_FLAG_LOOPBACK 512u /* num_devices > 1: run the G (P) device shards / replicas as
                                   logical devices all on `device` (one stream): the
                                   multi-GPU control flow and exchange on one GPU (tests) */
#define BTED_FLAG_NCCL   1024u  /* bted_select with P > 1: exchange through NCCL collectives
                                   (ncclCommInitAll over the P devices, libnccl.so.2 loaded at
                                   run time) instead of the default peer-memory exchange;
                                   NCCL failures and a stalled collective (BTED_NCCL_TIMEOUT_S,
                                   default 300 s; ncclCommGetAsyncError polled) -> BTED_ENCCL */
#define BTED_FLAG_NO_TC_GRAM 2048u /* implicit engine: build the Gram on CUDA cores (direct-difference
                                   form) instead of the tensor cores (centred expansion, bf16x3
                                   tcgen05.mma with the accumulator in TMEM; the default for the
                                   RBF kernel with d <= 16) */
#define BTED_FLAG_RECOMPUTE 4096u /* implicit engine with the tensor-core Gram: every K.l pass rebuilds
                                   the Gram tiles on the tensor cores (rc_pass.cuh) instead of
                                   streaming the stored Gram from HBM; bitwise the same results.
                                   Off by default: on B200 it is issue-bound at ~121 us per pass at
                                   N = 16384 vs 84 us for the HBM-bound streaming pass */
#define BTED_FLAG_TIMING   2u   /* record CUDA events around K1 and the K2 loop of every batch
                                   TED on the ctx stream; read with bted_get_stats()          */

typedef struct {
    float     gamma;         /* RBF bandwidth, > 0 and finite (ignored for LINEAR)      */
    int32_t   device;        /* CUDA device ordinal; -1 = the calling thread's current  */
    int32_t   num_batches;   /* B of Algorithm 2 (bted_run_batches), >= 1              */
    uint64_t  seed;          /* batch sampling seed (Alg. 2 l.2, reading A10)          */
    int32_t   x_on_device;   /* 1: X is a device pointer on `device` (adopted, not copied) */
    uint32_t  flags;         /* BTED_FLAG_*                                           */
    uintptr_t stream;        /* cudaStream_t to run on; 0 = a stream owned by the ctx
                                (num_devices > 1: the stream of `device` only)         */
    int32_t   num_devices;   /* G = P >= 1 GPUs [device, device + G) driven by this ctx
                                (SURVEY 8(e)); 1 = single GPU.  bted_run_batches runs
                                batch b on device b mod G (no exchange until the
                                merge, which runs on `device`); bted_select row- or
                                tile-shards the ONE candidate set over the P GPUs
                                (see "Multi-GPU" below).  X is replicated.          */
    int32_t   norm_mode;     /* bted_select with P > 1 and BTED_FLAG_DENSE (row bands):
                                0 = local row norms (K bit-symmetric: row norm =
                                column norm, no norm exchange), 1 = the literal
                                all-reduce of every band's partial COLUMN norms
                                (north_star wording; an ablation).  Ignored by the
                                default tile-sharded implicit engine.               */
} bted_params;

/* Fill *p with defaults: gamma 1, device -1, num_batches 1, seed 0, host X,
 * flags 0, own stream, num_devices 1, norm_mode 0. */
void bted_default_params(bted_params* p);

/*
 * bted_create -- a candidate set V ("the input un-sampled set V").
 *   X: N x d row-major fp32 features (Def. 1), host pointer (copied
 *      to the device) or, with params->x_on_device, a device pointer (adopted).
 *   N: 1 <= N < 2^31.  d: 1 <= d <= 64.  All X finite.  gamma > 0 for RBF.
 *   Nothing N x N is allocated here (a pool may have 2^20 rows).
 *   Errors: EINVAL (bad sizes, non-finite X or gamma), ENOMEM, ECUDA.
 */
bted_status bted_create(const float* X, int64_t N, int32_t d, bted_kernel kernel,
                        const bted_params* params, bted_ctx** out);

/*
 * bted_select -- TED(V, mu, m), Algorithm 1 on all N rows.
 *   Builds K = K_VV (l.1), then m times: score_v = ||K_v||^2/(k(v,v)+mu) over
 *   unselected v, x = argmax (lowest index on ties), X = X u x, and
 *   K = K - K_x K_x^T/(k(x,x)+mu) (l.3-5; the deflation after the m-th pick is
 *   skipped because it cannot change X).
 *   out_idx   [m] row indices in selection order (host).
 *   out_score [m] nullable: fp32 score of each pick at the step it was taken.
 *   Idempotent: each call restarts from the fresh Gram matrix.  Device memory
 *   on first use at this N: the default implicit engine keeps one packed
 *   upper-triangular K (~N^2/2 fp32) plus O(N m) fp64 state; the literal
 *   engines ping-pong two K buffers (packed ~N^2, dense 2 N^2 fp32).
 *   Errors: EINVAL (m < 1, m > N, mu <= 0 or non-finite), ENOMEM, ECUDA,
 *   ENUMERIC, ESTATE.
 */
bted_status bted_select(bted_ctx* ctx, int32_t m, float mu,
                        int64_t* out_idx, float* out_score);

/*
 * bted_run_batches -- BTED(V, mu, M, m, B), Algorithm 2
 * with V = the ctx's rows (the pool) and B = params.num_batches:
 *   l.1-4  for b in 0..B-1: V_b = bted_sample_batches(P, M, B, seed)[b];
 *          X_b = V_b[TED(X[V_b], mu, m)]
 *   l.5    X_U = sorted unique(X_0 u ... u X_{B-1})
 *   l.6    X = X_U[TED(X[X_U], mu, min(m, |X_U|))]   (fresh Gram of X_U)
 *   M: m <= M <= N (N = pool rows, < 2^32).  All steps run on the device;
 *   only the |X_U| count and the results cross to the host.
 *   out_idx [m] pool row indices of X in selection order; *out_count =
 *   min(m, |X_U|).  out_batch_idx nullable [B*m]: row b = X_b in selection
 *   order.
 *   Errors: as bted_select, plus EINVAL for M < m or M > N.
 */
bted_status bted_run_batches(bted_ctx* pool, int64_t M, int32_t m, float mu,
                             int64_t* out_idx, int32_t* out_count,
                             int64_t* out_batch_idx);

/*
 * bted_batch_teds -- Algorithm 2 lines 1-4 only, for the batches
 * b = b_begin, b_begin + b_step, ... < B (round-robin sharding of the
 * batches over processes/GPUs).  Writes X_b (pool indices, selection order)
 * to out_winners[k*m .. k*m+m-1] for the k-th batch it runs.
 *   out_winners: host pointer, or a device pointer on the ctx's device when
 *   winners_on_device = 1 (e.g. a torch tensor that is then all-gathered).
 */
bted_status bted_batch_teds(bted_ctx* pool, int64_t M, int32_t m, float mu,
                            int32_t b_begin, int32_t b_step,
                            int64_t* out_winners, int32_t winners_on_device);

/*
 * bted_merge -- Algorithm 2 lines 5-6: X_U = sorted unique(winners[0..n)),
 * then TED(X[X_U], mu, min(m, |X_U|)) on a fresh Gram matrix of X_U.
 *   winners: n pool indices (host, or device with winners_on_device = 1);
 *   negative entries are padding and ignored (e.g. the fill of an
 *   all-gather over ranks with unequal batch counts).
 *   out_idx [m] host; *out_count = min(m, |X_U|).
 */
bted_status bted_merge(bted_ctx* pool, const int64_t* winners, int64_t n,
                       int32_t winners_on_device, int32_t m, float mu,
                       int64_t* out_idx, int32_t* out_count);

/*
 * bted_sample_batches -- Algorithm 2 line 2 draws (reading A10): for each b,
 * the M indices i in [0, P) with the smallest
 *   key_b(i) = (splitmix64(splitmix64(seed + b*0xD1B54A32D192ED03) + i)
 *               & 0xFFFFFFFF00000000) | i,
 * in ascending order of i.  Computed on the
 * current CUDA device.  out: host [B*M].  1 <= M <= P < 2^32, B >= 1.
 */
bted_status bted_sample_batches(int64_t P, int64_t M, int32_t B, uint64_t seed,
                                int64_t* out);

/* ---------------- Multi-GPU through one context (params.num_devices = G > 1) -------
 * SURVEY 8(e), PAPER.md:150 ("stimulate the parallelism") and Alg. 2.
 * One process drives GPUs [device, device + G) (BTED_FLAG_LOOPBACK: G logical
 * devices on `device`, one stream -- the same kernels and exchange protocol);
 * X is replicated on every device; peer access is enabled between them (without
 * P2P only BTED_FLAG_NCCL works).
 *   bted_run_batches: batch b of Alg. 2 runs on device b mod G (one host thread
 *     per device, no exchange), the m winners of every batch are copied to
 *     `device` (l.5) and the union + merge TED run there.  Results are bitwise
 *     those of one device.
 *   bted_select: the candidate set is sharded over P = G devices --
 *     default: the implicit engine's packed Gram tiles k = p (mod P) on device p;
 *       per step each device publishes its partial q = K l (a release counter in
 *       its memory) and every device's score kernel sums the P partials in rank
 *       order through peer loads (bitwise the same on every device);
 *     BTED_FLAG_DENSE: row bands of the dense K; per step the pivot column slices
 *       are gathered, the band maxima max-reduced, and with norm_mode = 1 the
 *       bands' partial column norms summed (the literal column-norm exchange);
 *     BTED_FLAG_NCCL: the q exchange through ncclAllReduce (libnccl.so.2 loaded at
 *       run time; ncclCommInitAll over the P devices).
 *     Candidate sets small enough for the one-kernel cluster TED, or with fewer
 *     Gram tiles (rows) than devices, run on `device` alone.
 *   Errors: BTED_ENCCL (the ctx is then poisoned) when an NCCL call or async error
 *   fails, a collective exceeds BTED_NCCL_TIMEOUT_S (default 300 s; the
 *   communicators are aborted), or a device stops publishing its step (the other
 *   devices' waits time out after BTED_PEER_TIMEOUT_MS, default 20000 ms).
 *   bted_batch_teds / bted_merge / bted_shard_* / bted_ishard_* use `device` only.
 */

/* ---------------- row-sharded TED (one oversized batch over P GPUs) -------------
 * A shard context owns rows [row0, row1) of the N x N matrix K of the full
 * candidate set X (X is replicated: N x d).  The per-step exchange is done by
 * the caller between calls (torch.distributed / NCCL), all on the shard's
 * stream, so the loop can be captured in a CUDA graph:
 *   bted_shard_gram(t=0)  -> keys[0] holds this shard's best key
 *   all-reduce(keys[t], MAX)                      (8 bytes)
 *   bted_shard_pivot_column(t) -> col = K[row0:row1, s_t]
 *   all-gather(col) -> pivot (N floats, = row s_t of K by bit-symmetry)
 *   bted_shard_step(t+1, pivot) -> keys[t+1]
 * keys: device u64 [m] owned by the caller, zeroed before t = 0.  A key packs
 * (score bits + 1) << 32 | (0xFFFFFFFF - index); 0 = no candidate.
 */
bted_status bted_shard_create(const float* X, int64_t N, int32_t d, bted_kernel kernel,
                              int64_t row0, int64_t row1, const bted_params* params,
                              bted_ctx** out);
bted_status bted_shard_gram(bted_ctx* shard, float mu, uint64_t* keys_dev);
bted_status bted_shard_step(bted_ctx* shard, int32_t t, float mu, const float* pivot_dev,
                            uint64_t* keys_dev);
bted_status bted_shard_pivot_column(bted_ctx* shard, int32_t t, const uint64_t* keys_dev,
                                    float* col_dev);
/*
 * Literal norm exchange (the north_star's "NCCL allreduce of partial column
 * norms"; SURVEY §8(e) norm_mode 1, an ablation of the default above).  Alg. 1
 * l.3 scores v by ||K_v||^2 of v's COLUMN; here every shard
 * contributes the part of each column inside its band and the caller sums:
 *   bted_shard_gram(t=0, scratch keys)           (K1 on the band; its keys unused)
 *   bted_shard_colnorm(t=0, pivot=NULL)          -> colnorm = band column norms
 *   all-reduce(colnorm, SUM)                     (ld floats)
 *   bted_shard_scores(t=0, colnorm)              -> keys[0] = band's best key
 *   all-reduce(keys[t], MAX); bted_shard_pivot_column(t) ; all-gather(col)
 *   bted_shard_colnorm(t+1, pivot)               (l.5 on the band + column partials)
 *   all-reduce(colnorm, SUM); bted_shard_scores(t+1, colnorm) -> keys[t+1] ...
 * colnorm_dev: device fp32 [ld] owned by the caller (written, not read, by
 *   bted_shard_colnorm; entries >= N are 0).  The band values are bitwise those
 *   of bted_shard_step; the column sums differ from the row norms only in
 *   rounding order.  Errors: EINVAL (t < 0, t > 0 without pivot/keys, bad mu),
 *   ENOMEM, ECUDA, ESTATE.
 */
bted_status bted_shard_colnorm(bted_ctx* shard, int32_t t, float mu, const float* pivot_dev,
                               const uint64_t* keys_dev, float* colnorm_dev);
bted_status bted_shard_scores(bted_ctx* shard, int32_t t, float mu, const float* colnorm_dev,
                              uint64_t* keys_dev);
/* ---------------- tile-sharded implicit TED (one oversized batch over P GPUs) ----
 * The default single-GPU engine (implicit deflation, BTED_FLAG_IMPLICIT) with
 * its one N^2-sized object -- the read-only packed Gram K -- split over P
 * ranks: rank r computes, stores and streams only the upper-triangular tiles
 * k = r (mod P) (about 2 N^2 / P bytes per step per rank instead of 2 N^2).
 * X (N x d) and the O(N m) fp64 state (factor L, Q, G, running norms) are
 * replicated and evolve identically on every rank; the only exchange is the
 * per-step sum of the ranks' partial q = K l vectors (one all-reduce SUM of
 * qlen doubles), after which every rank computes the same scores and argmax
 * (no argmax all-reduce, no pivot broadcast).  Selection = Alg. 1 (PAPER.md
 * 134-148) in exact arithmetic; the q sum order is the collective's.
 *   bted_ishard_head(m, mu, q)          q = this rank's part of ||K_:v||^2
 *   all-reduce(q, SUM)
 *   bted_ishard_fin(0, mu, q, keys)     keys[0]
 *   for t = 1 .. m-1:
 *     bted_ishard_step(t, mu, keys, q)  l_t (from keys[t-1]), q = this rank's part of K l_t
 *     all-reduce(q, SUM)
 *     bted_ishard_fin(t, mu, q, keys)   keys[t]
 * q_dev: device fp64 [bted_ishard_qlen(ctx)] (caller-owned); keys_dev: device
 * u64 [m], zeroed by the caller before the head (packed keys as above).
 * 0 <= rank < nranks, d <= 32, m <= 256, at least nranks tiles.
 * Errors: EINVAL, ENOMEM, ECUDA, ESTATE; bted_shard_check reports ENUMERIC.
 */
bted_status bted_ishard_create(const float* X, int64_t N, int32_t d, bted_kernel kernel, int32_t rank,
                               int32_t nranks, const bted_params* params, bted_ctx** out);
bted_status bted_ishard_head(bted_ctx* shard, int32_t m, float mu, double* q_dev);
bted_status bted_ishard_step(bted_ctx* shard, int32_t t, float mu, const uint64_t* keys_dev, double* q_dev);
bted_status bted_ishard_fin(bted_ctx* shard, int32_t t, float mu, const double* q_dev, uint64_t* keys_dev);
int64_t     bted_ishard_qlen(const bted_ctx* shard);
/* K4 near-tie refinement for the tile-sharded engine (as on one GPU, DESIGN.md
 * "K4"): after the m-step loop, every step whose second-best fp32 score lies
 * within 2e-5 of the best is re-scored exactly in fp64 from the (replicated)
 * features.  *nforced = 0: the selection stands.  Otherwise forced_host[0 ..
 * *nforced) are flagged keys (the earlier picks and the corrected one): re-run
 * the loop with keys_dev preset to them (zeros after) and call again.  Every
 * rank computes the same answer, so all ranks re-run together.  keys_dev:
 * device u64 [m] of the finished loop; forced_host: host u64 [m].
 * Errors: EINVAL, ECUDA, ESTATE. */
bted_status bted_ishard_refine(bted_ctx* shard, int32_t m, float mu, const uint64_t* keys_dev,
                               uint64_t* forced_host, int32_t* nforced);
/*
 * K4 near-tie refinement for the row-sharded TED (both norm modes: the
 * band's top-2 keys come from bted_shard_gram/step, or from bted_shard_scores
 * in the literal mode; steps t < 256): after the loop, bted_shard_nearties lists this band's candidates of
 * every step whose fp32 score lies within 2e-5 of the global pick keys[t]
 * (cand_dev: device u32 [m][32], ncand_dev: device i32 [m]); the caller
 * all-gathers both over the ranks and calls bted_shard_refine with the host
 * copies (cand_all [nranks][m][32], ncand_all [nranks][m]): the first step
 * whose exact fp64 argmax (from the replicated features) differs from the pick
 * gives forced_host[0 .. *nforced) (flagged keys; 0 = the selection stands).
 * Every rank computes the same answer; re-run the loop with keys preset to
 * them (zeros after) and repeat.  Errors: EINVAL, ECUDA, ESTATE.
 */
bted_status bted_shard_nearties(bted_ctx* shard, int32_t m, const uint64_t* keys_dev, uint32_t* cand_dev,
                                int32_t* ncand_dev);
bted_status bted_shard_refine(bted_ctx* shard, int32_t m, float mu, const uint64_t* keys_dev,
                              const uint32_t* cand_all, const int32_t* ncand_all, int32_t nranks,
                              uint64_t* forced_host, int32_t* nforced);
/* Leading dimension (floats) a pivot buffer must have: pivot_dev[N..ld) must be 0. */
int64_t     bted_shard_ld(const bted_ctx* shard);
/* Sticky device error flag of the shard (BTED_ENUMERIC if a NaN score was seen). */
bted_status bted_shard_check(bted_ctx* shard);

/*
 * bted_update -- replace the features of a ctx (same N, d) for the next call:
 * a pool of the same shape (e.g. the next tuning node).  Host X is copied
 * H2D asynchronously on the ctx stream (pinned memory makes it a DMA; the
 * caller keeps X alive until its next call on this ctx returns); a device X
 * (x_on_device = 1) is copied D2D.  Errors: EINVAL, ECUDA, ESTATE.
 */
bted_status bted_update(bted_ctx* ctx, const float* X, int32_t x_on_device);

/*
 * bted_host_alloc / bted_host_free -- page-locked host memory from the
 * library's CUDA runtime, for feature buffers passed to bted_create /
 * bted_update: host->device copies from it run at DMA speed (memory pinned by
 * another runtime instance in the process, e.g. torch's, is copied as
 * pageable).  Errors: EINVAL, ENOMEM, ECUDA.
 */
bted_status bted_host_alloc(size_t bytes, void** out);
void        bted_host_free(void* p);

/* Accumulated device timings of the TEDs run by a ctx (BTED_FLAG_TIMING):
 * k1_ms = transpose + Gram (Alg. 1 l.1 + first l.3), k2_ms = the fused
 * deflate/rescore loop (k2_launches launches of the K2 kernel), measured
 * with CUDA events on the ctx stream.  Merge TEDs are not included. */
typedef struct {
    uint64_t teds;
    uint64_t k2_launches;
    double   k1_ms;
    double   k2_ms;
    uint64_t small_teds;     /* TEDs run whole by the cluster kernel (small N) */
    double   small_ms;       /* their device time                              */
    uint64_t refined_steps;  /* K4: near-tie steps re-scored exactly in fp64   */
    uint64_t corrected_steps;/* K4: of those, steps whose pick changed         */
    uint64_t full_refined_steps; /* K4: of the refined steps, those whose candidate list
                                    could be incomplete (a score unit's second key in the
                                    window, or > 32 candidates): ALL unselected points
                                    were re-scored in fp64                          */
} bted_stats;
bted_status bted_get_stats(bted_ctx* ctx, bted_stats* out);
bted_status bted_reset_stats(bted_ctx* ctx);

/* ---------------- introspection ---------------- */
void        bted_destroy(bted_ctx* ctx);
const char* bted_status_string(bted_status s);
const char* bted_last_error(void);
/* Number of kernels this library launched since load (all contexts). */
uint64_t    bted_kernel_launches(void);
/* Debug: copy the fp32 K of the last TED run by ctx (which = 0: bted_select,
 * 1: the last batch / merge TED) to host as a dense rows x ld matrix (packed
 * storage is unpacked), i.e. K after the m-1 deflations of that run -- or, for
 * the implicit engine (which never rewrites K), the Gram matrix of that run. */
bted_status bted_debug_copy_K(bted_ctx* ctx, int32_t which, float* out, int64_t* ld_out);

#ifdef __cplusplus
}
#endif
#endif /* BTED_H_ */
