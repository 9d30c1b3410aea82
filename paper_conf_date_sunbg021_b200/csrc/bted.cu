// bted.cu -- TED engine (Alg. 1), BTED scheduler (Alg. 2) and the C ABI of
// include/bted.h.  PAPER.md:134-156.  Built into libbted.so for sm_100a.
//
// Per TED (bted_select / every batch of bted_run_batches) the device runs
//   transpose X -> XT, zero keys/sel, K1 gram_rownorm (l.1 + first l.3),
//   then m-1 times K2 deflate_rescore (l.5 + next l.3) on ping-pong K buffers,
// captured once per (X, N, d, m, mu, gamma) into a CUDA graph.  The pivot
// of step t is read ON THE DEVICE from keys[t-1]; the host sees only the
// m packed keys at the end (no per-step host round trip).
#include <cub/cub.cuh>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nccl.h>            // types only: libnccl.so.2 is loaded at run time (BTED_FLAG_NCCL)
#include <nvtx3/nvToolsExt.h> // header-only NVTX ranges (free unless a profiler attaches)

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <cstdio>
#include <list>
#include <mutex>
#include <new>
#include <string>
#include <thread>
#include <chrono>
#include <vector>

#include "../../include/bted.h"
#include "kernels.cuh"
#include "sample.cuh"
#include "packed.cuh"
#include "small.cuh"
#include "implicit.cuh"
#include "refine.cuh"
#include "colnorm.cuh"
#include "xchg.cuh"
#include <cudaTypedefs.h>
#include "gram_tc.cuh"
#include "rc_pass.cuh"

namespace {

// NVTX range for timelines (nsys / ncu --nvtx): the BTED call, its phases, K4
struct Nvtx {
    explicit Nvtx(const char* name) { nvtxRangePushA(name); }
    ~Nvtx() { nvtxRangePop(); }
};

thread_local std::string g_last_error;
std::atomic<uint64_t> g_launches{0};

void set_error(const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_last_error = buf;
}

struct CudaError {
    cudaError_t e;
    const char* what;
};
struct NcclError {            // a failed or stalled collective (BTED_FLAG_NCCL) -> BTED_ENCCL
    std::string what;
};

#define CK(expr)                                                         \
    do {                                                                 \
        cudaError_t _e = (expr);                                         \
        if (_e != cudaSuccess) throw CudaError{_e, #expr};               \
    } while (0)
#define LAUNCHED(n) g_launches.fetch_add((n), std::memory_order_relaxed)

// Kernel attributes (dynamic smem limits, carveouts) are per device: run f once
// per (call site, current device), thread-safe.
template <class F>
void once_per_device(uint64_t& mask, F&& f) {
    static std::mutex mu;
    int dev = 0;
    cudaGetDevice(&dev);
    const uint64_t bit = 1ull << (dev & 63);
    std::lock_guard<std::mutex> lk(mu);
    if (mask & bit) return;
    f();
    mask |= bit;
}

constexpr int kK1Rows = 16, kK1Threads = 256;
constexpr int kK2Rows = 1, kK2Unroll = 4, kK2Threads = 256;
constexpr int kRowsPerK2Cta = (kK2Threads / 32) * kK2Rows;

inline int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }
inline int64_t ld_for(int64_t N) { return round_up(N, 32); }
inline uint32_t fbits(float f) { uint32_t u; std::memcpy(&u, &f, 4); return u; }

template <class T>
void grow(T*& p, size_t& cap, size_t n) {
    if (n <= cap) return;
    if (p) cudaFree(p);
    p = nullptr;
    cap = 0;
    CK(cudaMalloc(&p, sizeof(T) * n));
    cap = n;
}

// ------------------------------------------------------------------ TED engine
struct GraphKey {
    const float* X;
    int64_t N;
    int32_t d, m, kernel, part;   // part 0 = head (transpose, K1), 1 = loop (m-1 x K2)
    int32_t packed;
    uint32_t mu, gamma;
    const void* keys;
    bool operator==(const GraphKey& o) const {
        return X == o.X && N == o.N && d == o.d && m == o.m && kernel == o.kernel && part == o.part &&
               packed == o.packed &&
               mu == o.mu && gamma == o.gamma && keys == o.keys;
    }
};

struct Stats {
    uint64_t teds = 0, k2_launches = 0, small_teds = 0;
    double k1_ms = 0, k2_ms = 0, small_ms = 0;
};

struct Ted {
    cudaStream_t stream = nullptr;
    float* K[2] = {nullptr, nullptr};
    size_t kcap[2] = {0, 0};
    float* XT = nullptr;
    size_t xtcap = 0;
    uint8_t* sel = nullptr;
    size_t selcap = 0;
    unsigned long long* keys = nullptr;
    size_t keyscap = 0;
    int* err = nullptr;
    size_t errcap = 0;
    // packed-symmetric layout (packed.cuh): per-tile norm partials [nT][nT*T]
    float* P = nullptr;
    size_t pcap = 0;
    // implicit deflation (implicit.cuh): fp64 partials, factor L [NPa][m], l, n, r, h
    double* P64 = nullptr; size_t p64cap = 0;
    double* Lf = nullptr; size_t lfcap = 0;
    double* ell = nullptr; size_t ellcap = 0;
    double* nv = nullptr; size_t nvcap = 0;
    double* rd = nullptr; size_t rdcap = 0;
    double* Qc = nullptr; size_t qccap = 0;      // q = K l of every step, [m][NPa] (h from the history)
    double* G = nullptr; size_t gcap = 0;        // L^T L, [m][m]
    double* hv = nullptr; size_t hvcap = 0;
    int* kflag = nullptr; size_t kflagcap = 0;   // K has a non-positive-normal entry (exact conversion)
    int* bar = nullptr; size_t barcap = 0;       // dependency counters of the persistent loop kernel
    int* tctr = nullptr; size_t tctrcap = 0;     // per-pass tile counters of the K.l passes [m]
    uint8_t* opA = nullptr; size_t opAcap = 0;   // K1 on tensor cores (gram_tc.cuh): operand blocks,
    uint8_t* opB = nullptr; size_t opBcap = 0;   //   row norms of the centred features, the centre
    float* xnrm = nullptr; size_t xnrmcap = 0;
    float* xctr = nullptr; size_t xctrcap = 0;
    int* xmax = nullptr; size_t xmaxcap = 0;
    bool gram_tc = true;                         // implicit head: K1 on tensor cores (else CUDA cores)
    bool rc = false;                             // K.l passes recompute the tensor-core Gram (rc_pass.cuh)
    bool rc_on = false;                          //   ... for the TED being enqueued (set by its head)
    float rc_gamma = 0.f;
    bool split = true;                           // implicit: three kernels per step (else BTED_FLAG_PERSISTENT_LOOP)
    bool implicit = false;
    // K4 near-tie refinement (refine.cuh): per-CTA top-2 keys of every step, flags, candidates
    bool refine = true;
    unsigned long long* top2 = nullptr; size_t top2cap = 0;
    int* flags = nullptr; size_t flagscap = 0;
    uint32_t* cand = nullptr; size_t candcap = 0;
    int* ncand = nullptr; size_t ncandcap = 0;
    int* nflag = nullptr; size_t nflagcap = 0;
    int32_t last_nC = 0;

    void reserve_refine(int64_t NP, int32_t m) {
        grow(top2, top2cap, (size_t)m * (size_t)(NP / 32) * 2);
        grow(flags, flagscap, (size_t)m);
        grow(cand, candcap, (size_t)m * bted::rf::kMaxCand);
        grow(ncand, ncandcap, (size_t)m);
        grow(nflag, nflagcap, 1);
        last_nC = (int32_t)(NP / 32);
    }
    std::list<std::pair<GraphKey, cudaGraphExec_t>> graphs;   // LRU
    int64_t last_rows = 0, last_ld = 0;
    int last_buf = 0;
    bool last_packed = false;
    int32_t last_nT = 0;
    // timing (BTED_FLAG_TIMING): events recorded on the stream around the
    // head and loop graphs of each TED, read back at the next host sync.
    bool timing = false;
    bool tma = false;          // packed K2p: TMA-ring variant instead of the LDG one
    struct Slot { cudaEvent_t e[3]; int32_t m; int32_t small; };   // small > 0: one cluster launch of `small` TEDs
    std::vector<Slot> slots;
    size_t used = 0;
    Stats stats;

    void release() {
        for (auto& g : graphs) cudaGraphExecDestroy(g.second);
        graphs.clear();
        for (int b = 0; b < 2; ++b) if (K[b]) cudaFree(K[b]);
        if (XT) cudaFree(XT);
        if (sel) cudaFree(sel);
        if (keys) cudaFree(keys);
        if (err) cudaFree(err);
        if (P) cudaFree(P);
        for (double* q : {P64, Lf, ell, nv, rd, Qc, G, hv}) if (q) cudaFree(q);
        for (void* q : {(void*)opA, (void*)opB, (void*)xnrm, (void*)xctr, (void*)xmax}) if (q) cudaFree(q);
        opA = opB = nullptr; xnrm = xctr = nullptr; xmax = nullptr;
        P64 = Lf = ell = nv = rd = Qc = G = hv = nullptr;
        if (kflag) cudaFree(kflag);
        kflag = nullptr;
        if (bar) cudaFree(bar);
        bar = nullptr;
        if (tctr) cudaFree(tctr);
        tctr = nullptr;
        for (void* q : {(void*)top2, (void*)flags, (void*)cand, (void*)ncand, (void*)nflag}) if (q) cudaFree(q);
        top2 = nullptr; flags = nullptr; cand = nullptr; ncand = nullptr; nflag = nullptr;
        for (auto& sl : slots) for (auto e : sl.e) cudaEventDestroy(e);
        slots.clear();
        K[0] = K[1] = nullptr; XT = nullptr; sel = nullptr; keys = nullptr; err = nullptr;
        P = nullptr;
    }

    // Buffers of the implicit-deflation engine for an N-point TED.
    // ktiles >= 0: store only that many tiles (a tile shard of the multi-GPU engine)
    void reserve_implicit(int64_t N, int32_t m, int64_t ktiles = -1) {
        const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
        const size_t tiles = (size_t)(ktiles >= 0 ? ktiles : bted::pk::num_tiles(nT)) * bted::pk::T * bted::pk::T;
        const size_t NP = (size_t)nT * bted::pk::T, NPa = (NP + 255) / 256 * 256;
        const void* before[19] = {K[0], sel, keys, P64, Lf, ell, nv, rd, Qc, G, hv, kflag, bar, tctr, opA, opB, xnrm, xctr, xmax};
        grow(K[0], kcap[0], tiles);
        grow(sel, selcap, NPa);
        grow(keys, keyscap, (size_t)std::max(m, 1));
        grow(P64, p64cap, (size_t)nT * NP);
        grow(Lf, lfcap, NPa * (size_t)m);
        grow(ell, ellcap, NPa);
        grow(nv, nvcap, NPa);
        grow(rd, rdcap, NPa);
        grow(Qc, qccap, NPa * (size_t)m);
        grow(G, gcap, (size_t)m * (size_t)m);
        grow(hv, hvcap, (size_t)m + 1);
        if (gram_tc) {
            grow(opA, opAcap, (size_t)nT * bted::tc::kBlockBytes);
            if (rc) grow(opB, opBcap, (size_t)nT * bted::tc::kBlockBytes);   // row-permuted copy (rc_pass.cuh)
            grow(xnrm, xnrmcap, NP);
            grow(xctr, xctrcap, (size_t)bted::tc::kD * (1 + bted::tc::kCenterBlocks));
            grow(xmax, xmaxcap, 1);
        }
        grow(kflag, kflagcap, 1);
        grow(bar, barcap, (size_t)bted::im::loop_sync_ints(NPa / bted::im::kEllRows, m));
        grow(tctr, tctrcap, (size_t)std::max(m, 1));
        if (!err) { grow(err, errcap, 1); CK(cudaMemsetAsync(err, 0, sizeof(int), stream)); }
        const void* top2_before = top2;
        reserve_refine((int64_t)NP, m);
        const void* after[19] = {K[0], sel, keys, P64, Lf, ell, nv, rd, Qc, G, hv, kflag, bar, tctr, opA, opB, xnrm, xctr, xmax};
        if (top2 != top2_before) { for (auto& g : graphs) cudaGraphExecDestroy(g.second); graphs.clear(); }
        if (std::memcmp(before, after, sizeof before) != 0) {
            for (auto& g : graphs) cudaGraphExecDestroy(g.second);
            graphs.clear();
        }
    }

    // Buffers of the packed layout for an N-point TED.
    void reserve_packed(int64_t N, int32_t m) {
        const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
        const size_t tiles = (size_t)bted::pk::num_tiles(nT) * bted::pk::T * bted::pk::T;
        const size_t NP = (size_t)nT * bted::pk::T;
        const void* before[5] = {K[0], K[1], sel, keys, P};
        grow(K[0], kcap[0], tiles);
        if (m > 1) grow(K[1], kcap[1], tiles);
        grow(sel, selcap, NP);
        grow(keys, keyscap, (size_t)std::max(m, 1));
        grow(P, pcap, (size_t)nT * NP);
        if (!err) { grow(err, errcap, 1); CK(cudaMemsetAsync(err, 0, sizeof(int), stream)); }
        const void* top2_before = top2;
        reserve_refine((int64_t)NP, m);
        if (top2 != top2_before) { for (auto& g : graphs) cudaGraphExecDestroy(g.second); graphs.clear(); }
        const void* after[5] = {K[0], K[1], sel, keys, P};
        if (std::memcmp(before, after, sizeof before) != 0) {
            for (auto& g : graphs) cudaGraphExecDestroy(g.second);
            graphs.clear();
        }
    }

    // Buffers for a band of `rows` rows of an N x N problem.
    // Any reallocation invalidates the captured graphs (they hold raw pointers).
    void reserve(int64_t rows, int64_t N, int32_t d, int32_t m) {
        const int64_t ld = ld_for(N);
        const void* before[5] = {K[0], K[1], XT, sel, keys};
        grow(K[0], kcap[0], (size_t)(rows * ld));
        if (m > 1) grow(K[1], kcap[1], (size_t)(rows * ld));
        grow(XT, xtcap, (size_t)(d * ld));
        grow(sel, selcap, (size_t)rows);
        grow(keys, keyscap, (size_t)std::max(m, 1));
        if (!err) { grow(err, errcap, 1); CK(cudaMemsetAsync(err, 0, sizeof(int), stream)); }
        const void* after[5] = {K[0], K[1], XT, sel, keys};
        if (std::memcmp(before, after, sizeof before) != 0) {
            for (auto& g : graphs) cudaGraphExecDestroy(g.second);
            graphs.clear();
        }
    }

    Slot* next_slot(int32_t m) {
        if (used == slots.size()) {
            Slot sl{};
            for (auto& e : sl.e) CK(cudaEventCreate(&e));
            slots.push_back(sl);
        }
        Slot* sl = &slots[used++];
        sl->m = m;
        sl->small = 0;
        return sl;
    }

    // after a host sync of `stream`: fold the recorded TEDs into stats
    void collect() {
        for (size_t i = 0; i < used; ++i) {
            float a = 0, b = 0;
            if (slots[i].small > 0) {
                CK(cudaEventElapsedTime(&a, slots[i].e[0], slots[i].e[1]));
                stats.small_ms += a;
                stats.small_teds += (uint64_t)slots[i].small;
                continue;
            }
            CK(cudaEventElapsedTime(&a, slots[i].e[0], slots[i].e[1]));
            stats.k1_ms += a;
            if (slots[i].m > 1) {
                CK(cudaEventElapsedTime(&b, slots[i].e[1], slots[i].e[2]));
                stats.k2_ms += b;
                stats.k2_launches += (uint64_t)(slots[i].m - 1);
            }
            stats.teds += 1;
        }
        used = 0;
    }
};

void launch_transpose(Ted& T, const float* X, int64_t N, int32_t d) {
    const int64_t ld = ld_for(N);
    bted::transpose_pad_kernel<<<(unsigned)((ld + 255) / 256), 256, 0, T.stream>>>(X, (int32_t)N, d, T.XT, ld);
    LAUNCHED(1);
}

void launch_gram(Ted& T, int64_t N, int32_t d, int64_t row0, int64_t rows, float gamma, int kernel,
                 float mu, unsigned long long* key_out, unsigned long long* top2 = nullptr) {
    const int64_t ld = ld_for(N);
    const unsigned grid = (unsigned)((rows + kK1Rows - 1) / kK1Rows);
    const size_t smem = sizeof(float) * kK1Rows * d;
    bted::gram_rownorm_kernel<kK1Rows, kK1Threads><<<grid, kK1Threads, smem, T.stream>>>(
        T.XT, ld, d, (int32_t)N, (int32_t)row0, (int32_t)rows, gamma, kernel == BTED_KERNEL_LINEAR ? 1 : 0,
        T.K[0], mu, key_out, T.err, top2);
    LAUNCHED(1);
}

void launch_step(Ted& T, int64_t N, int64_t row0, int64_t rows, int32_t t, float mu, const float* pivot,
                 unsigned long long* keys, unsigned long long* top2 = nullptr) {
    const int64_t ld = ld_for(N);
    const unsigned grid = (unsigned)((rows + kRowsPerK2Cta - 1) / kRowsPerK2Cta);
    bted::deflate_rescore_kernel<kK2Rows, kK2Unroll, kK2Threads><<<grid, kK2Threads, 0, T.stream>>>(
        T.K[(t - 1) & 1], T.K[t & 1], ld, (int32_t)row0, (int32_t)rows, pivot, keys, t, mu, T.sel, T.err, top2);
    LAUNCHED(1);
}

// ---- packed layout (packed.cuh) ----
// (lazily initialised process-wide constants are atomics: the multi-GPU run_batches
// calls them from one host thread per device)
std::atomic<int> g_num_sms{0};
int num_sms() {
    int n = g_num_sms.load(std::memory_order_relaxed);
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 148;
        cudaGetLastError();
        g_num_sms.store(n, std::memory_order_relaxed);
    }
    return n;
}
// K2p configurations (scripts/k2p_variants.cu, profiles/r1/k2p_variants_*.txt):
// default = one CTA per tile with 256-bit loads (k2p_ldg<4>, measured 6.40 /
// 6.75 TB/s at N = 16384 / 32768, above cudaMemcpy D2D); BTED_FLAG_TMA = the
// persistent TMA-ring pipeline (v8 stores, 64-row stages; 5.90 / 6.09 TB/s).
constexpr int kK2pSub = 64;
#define K2P_TMA_KERNEL bted::pk::deflate_packed_v8_kernel<kK2pSub, false>
#define K2P_LDG_KERNEL bted::pk::deflate_packed_ldg_kernel<4>
constexpr size_t kK2pSmem = bted::pk::k2p_smem_bytes(kK2pSub);

void launch_finalize(Ted& T, int64_t N, int nT, const float* Kout, float mu, const unsigned long long* keys,
                     int32_t t, unsigned long long* key_out) {
    const unsigned grid = (unsigned)((int64_t)nT * bted::pk::T / bted::pk::kFinRows);
    bted::pk::finalize_packed_kernel<<<grid, bted::pk::kFinThreads, 0, T.stream>>>(
        T.P, nT, (int32_t)N, Kout, mu, T.sel, keys, t, key_out, T.err, T.refine ? T.top2 : nullptr);
}

// Alg. 1 l.1 + first l.3 on the packed tiles.  (2 kernels: K1p, fin)
void enqueue_head_packed(Ted& T, const float* X, int64_t N, int32_t d, float gamma, int kernel, int32_t m,
                         float mu, unsigned long long* keys) {
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    CK(cudaMemsetAsync(keys, 0, sizeof(unsigned long long) * m, T.stream));
    CK(cudaMemsetAsync(T.sel, 0, (size_t)nT * bted::pk::T, T.stream));
    const int64_t tiles = bted::pk::num_tiles(nT);
    const int lin = kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    // one CTA per tile, then the first scores from the partials
    if (d <= 16)
        bted::pk::gram_packed_kernel<16><<<(unsigned)tiles, bted::pk::kConsumers, 0, T.stream>>>(
            X, (int32_t)N, d, gamma, lin, T.K[0], nT, T.P);
    else
        bted::pk::gram_packed_kernel<32><<<(unsigned)tiles, bted::pk::kConsumers, 0, T.stream>>>(
            X, (int32_t)N, d, gamma, lin, T.K[0], nT, T.P);
    launch_finalize(T, N, nT, T.K[0], mu, keys, 0, keys);
    LAUNCHED(2);
}

// Alg. 1 l.2-6 loop on the packed tiles: per step K2p (deflate + partials) and fin.  (2(m-1) kernels)
void enqueue_loop_packed(Ted& T, int64_t N, int32_t m, float mu, unsigned long long* keys, bool tma) {
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int64_t tiles = bted::pk::num_tiles(nT);
    const unsigned grid = (unsigned)std::min<int64_t>(tiles, (int64_t)num_sms());
    for (int32_t t = 1; t < m; ++t) {
        const float* Kin = T.K[(t - 1) & 1];
        float* Kout = T.K[t & 1];
        if (tma)
            K2P_TMA_KERNEL<<<grid, bted::pk::kConsumers + 32, kK2pSmem, T.stream>>>(
                Kin, Kout, nT, (int32_t)N, T.P, keys, t, mu, T.sel);
        else
            K2P_LDG_KERNEL<<<(unsigned)tiles, bted::pk::kConsumers, 0, T.stream>>>(
                Kin, Kout, nT, (int32_t)N, T.P, keys, t, mu, T.sel);
        launch_finalize(T, N, nT, Kout, mu, keys, t, keys + t);
        LAUNCHED(2);
    }
}

// ---- implicit deflation (implicit.cuh) ----
// persistent tile pass: kTPBlocksPerSM CTAs per SM (never more than the tiles)
unsigned tile_pass_grid(int64_t tiles) {
    return (unsigned)std::min<int64_t>(tiles, (int64_t)bted::im::kTPBlocksPerSM * num_sms());
}
// Tiles each K.l pass pins in L2 (evict-last) for the next pass, which runs in
// the opposite order and starts with them (implicit.cuh tp_produce).  Default
// kL2KeepFrac = 0 of the device L2 (the serpentine order alone measured best);
// BTED_L2_KEEP_MB overrides.
constexpr double kL2KeepFrac = 0.0;
int l2_keep_tiles(int64_t tiles) {
    static std::atomic<int64_t> cached{-1};
    int64_t bytes = cached.load(std::memory_order_relaxed);
    if (bytes < 0) {
        if (const char* e = std::getenv("BTED_L2_KEEP_MB")) {
            bytes = (int64_t)(std::atof(e) * 1048576.0);
        } else {
            int dev = 0, l2 = 0;
            cudaGetDevice(&dev);
            if (cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev) != cudaSuccess) l2 = 0;
            cudaGetLastError();
            bytes = (int64_t)(kL2KeepFrac * l2);
        }
        cached.store(bytes, std::memory_order_relaxed);
    }
    const int64_t tile_bytes = (int64_t)bted::pk::T * bted::pk::T * 4;
    return (int)std::min<int64_t>(tiles, std::max<int64_t>(0, bytes / tile_bytes));
}
// The K.l pass's fp64 partials (nT x NP doubles, rewritten every step and read by kernel C) are stored
// with an L2 evict-last hint when they take at most kP64KeepFrac of L2: they then never reach DRAM,
// whose reads the pass needs (B200, N = 16384, scripts/tp_ablate.cu: 86.9 -> 80.3 us per pass).
// BTED_P64_KEEP = 0 / 1 overrides.
constexpr double kP64KeepFrac = 0.25;
bool keep_partials(int nT) {
    static std::atomic<int64_t> cached{-1};
    int64_t lim = cached.load(std::memory_order_relaxed);
    if (lim < 0) {
        if (const char* e = std::getenv("BTED_P64_KEEP")) {
            lim = std::atoi(e) ? INT64_MAX : 0;
        } else {
            int dev = 0, l2 = 0;
            cudaGetDevice(&dev);
            if (cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev) != cudaSuccess) l2 = 0;
            cudaGetLastError();
            lim = (int64_t)(kP64KeepFrac * l2);
        }
        cached.store(lim, std::memory_order_relaxed);
    }
    return (int64_t)nT * nT * bted::pk::T * 8 <= lim;
}
// head: K1p (the packed Gram, read-only from now on), fp64 norm pass, scores.  (3 kernels)
void ensure_implicit_attrs() {
    static uint64_t done = 0;
    once_per_device(done, [] {
        // two persistent CTAs per SM need the maximum shared-memory carveout
        for (const void* f : {(const void*)bted::im::tile_pass_kernel<true, false>,
                              (const void*)bted::im::tile_pass_kernel<false, false>,
                              (const void*)bted::im::tile_pass_kernel<true, true>,
                              (const void*)bted::im::tile_pass_kernel<false, true>}) {
            CK(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bted::im::tile_pass_smem_bytes));
            CK(cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared));
        }
        CK(cudaFuncSetAttribute(bted::im::ted_loop_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::im::tile_pass_smem_bytes));
        CK(cudaFuncSetAttribute(bted::im::ted_loop_kernel, cudaFuncAttributePreferredSharedMemoryCarveout,
                                (int)cudaSharedmemCarveoutMaxShared));
    });
}

void ensure_gram_tc_attrs() {
    static uint64_t done = 0;
    once_per_device(done, [] {
        CK(cudaFuncSetAttribute(bted::tc::gram_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::tc::kTileSmemBytes));
        CK(cudaFuncSetAttribute(bted::tc::gram_tc_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::tc::kTmaSmemBytes));
        CK(cudaFuncSetAttribute(bted::tc::gram_tc_norm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::tc::kBlockBytes));
        CK(cudaFuncSetAttribute(bted::rc::rc_pass_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::rc::kSmemBytes));
        CK(cudaFuncSetAttribute(bted::rc::rc_pass_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::rc::kSmemBytes));
    });
}
// the recomputing K.l pass: one CTA per SM (never more than the tiles)
unsigned rc_pass_grid(int64_t tiles) { return (unsigned)std::min<int64_t>(tiles, (int64_t)num_sms()); }

// The packed Gram as a 2-D fp32 tensor [tiles * 128 rows][128 columns] for the tensor-core Gram's
// TMA stores (gram_tc.cuh gram_tc_tma_kernel: boxes of 32 columns x 128 rows, 128-byte swizzle).
// cuTensorMapEncodeTiled comes from the driver through the runtime (no libcuda link).
bool k_tensor_map(CUtensorMap* map, float* K, int64_t tiles) {
    static PFN_cuTensorMapEncodeTiled_v12000 encode = [] {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q{};
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            fn = nullptr;
        cudaGetLastError();
        return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    }();
    if (!encode) return false;
    const cuuint64_t dims[2] = {(cuuint64_t)bted::pk::T, (cuuint64_t)tiles * bted::pk::T};
    const cuuint64_t strides[1] = {(cuuint64_t)bted::pk::T * sizeof(float)};
    const cuuint32_t box[2] = {(cuuint32_t)bted::tc::kBoxCols, (cuuint32_t)bted::pk::T};
    const cuuint32_t estr[2] = {1, 1};
    return encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, K, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
// BTED_GRAM_STG=1: the tensor-core Gram with the threads' own stores (A/B only)
bool gram_tma_stores() {
    static const bool off = [] { const char* e = std::getenv("BTED_GRAM_STG"); return e && std::atoi(e); }();
    return !off;
}

void enqueue_head_implicit(Ted& T, const float* X, int64_t N, int32_t d, float gamma, int kernel, int32_t m,
                           float mu, unsigned long long* keys) {
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int64_t NP = (int64_t)nT * bted::pk::T, NPa = (NP + 255) / 256 * 256;
    const int64_t tiles = bted::pk::num_tiles(nT);
    CK(cudaMemsetAsync(keys, 0, sizeof(unsigned long long) * m, T.stream));
    CK(cudaMemsetAsync(T.sel, 0, (size_t)NPa, T.stream));
    CK(cudaMemsetAsync(T.kflag, 0, sizeof(int), T.stream));
    CK(cudaMemsetAsync(T.tctr, 0, sizeof(int) * m, T.stream));
    const int lin = kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    // K1i: the Gram tiles only (the fp64 norm pass below recomputes the first scores)
    auto k1i = [&](auto kern) {
        kern<<<(unsigned)tiles, bted::pk::kConsumers, 0, T.stream>>>(X, (int32_t)N, d, gamma, T.K[0], nT, 0, 1,
                                                                     (const int*)nullptr);
    };
    // d <= 16 (RBF): the tensor-core Gram (gram_tc.cuh: centred expansion, bf16x3 tcgen05.mma,
    // TMEM accumulator); else / BTED_FLAG_NO_TC_GRAM: the CUDA-core direct form -- two columns
    // per lane, four rows at once, 4 CTAs/SM: 243 us at N = 16384 (B200, warm ncu)
    if (d <= 16 && !lin && T.gram_tc) {
        ensure_gram_tc_attrs();
        bted::tc::center_part_kernel<<<bted::tc::kCenterBlocks, bted::tc::kCenterThreads, 0, T.stream>>>(
            X, (int32_t)N, d, T.xctr + bted::tc::kD);
        bted::tc::center_kernel<<<1, 32, 0, T.stream>>>(T.xctr + bted::tc::kD, (int32_t)N, d, T.xctr);
        bted::tc::prep_kernel<<<(unsigned)((NP + bted::tc::kThreads - 1) / bted::tc::kThreads), bted::tc::kThreads, 0,
                                T.stream>>>(X, (int32_t)N, d, nT, T.xctr, T.opA, T.rc ? T.opB : nullptr);
        CK(cudaMemsetAsync(T.xmax, 0, sizeof(int), T.stream));
        bted::tc::gram_tc_norm_kernel<<<(unsigned)nT, bted::tc::kThreads, bted::tc::kBlockBytes, T.stream>>>(
            T.opA, T.xnrm, T.xmax);
        const unsigned g = (unsigned)std::min<int64_t>(tiles, (int64_t)2 * num_sms());
        CUtensorMap kmap;
        if (gram_tma_stores() && k_tensor_map(&kmap, T.K[0], tiles))
            bted::tc::gram_tc_tma_kernel<<<g, bted::tc::kWsThreads, bted::tc::kTmaSmemBytes, T.stream>>>(
                T.opA, T.xnrm, (int32_t)N, gamma, nT, T.xmax, kmap);
        else
            bted::tc::gram_tc_kernel<<<g, bted::tc::kTcThreads, bted::tc::kTileSmemBytes, T.stream>>>(
                T.opA, T.xnrm, (int32_t)N, gamma, T.K[0], nT, T.xmax);
        // the accuracy guard's fallback (exits at once when the tensor-core Gram was written)
        bted::pk::gram_tile2_kernel<16, false, 4><<<(unsigned)std::min<int64_t>(tiles, (int64_t)4 * num_sms()),
                                                     bted::pk::kConsumers, 0, T.stream>>>(
            X, (int32_t)N, d, gamma, T.K[0], nT, 0, 1, T.xmax);
        LAUNCHED(6);
    } else if (d <= 16) {
        if (lin) k1i(bted::pk::gram_tile2_kernel<16, true, 4>); else k1i(bted::pk::gram_tile2_kernel<16, false, 4>);
    } else {
        if (lin) k1i(bted::pk::gram_tile_kernel<32, true>); else k1i(bted::pk::gram_tile_kernel<32, false>);
    }
    T.rc_on = d <= 16 && !lin && T.gram_tc && T.rc;
    T.rc_gamma = gamma;
    if (T.rc_on) {         // the norm pass on recomputed tiles (the stored Gram if the guard failed)
        bted::rc::rc_pass_kernel<true><<<rc_pass_grid(tiles), bted::rc::kThreads, bted::rc::kSmemBytes, T.stream>>>(
            T.opB, T.opA, T.xnrm, T.xmax, gamma, (int32_t)N, T.K[0], nT, nullptr, T.P64, T.kflag);
    } else {
        auto normk = keep_partials(nT) ? bted::im::tile_pass_kernel<true, true> : bted::im::tile_pass_kernel<true, false>;
        normk<<<tile_pass_grid(tiles), bted::im::kTPThreads, bted::im::tile_pass_smem_bytes, T.stream>>>(
            T.K[0], nT, nullptr, T.P64, T.kflag, T.tctr, 0, l2_keep_tiles(tiles), 0, 1);
    }
    bted::im::fin64_kernel<<<(unsigned)(NP / bted::im::kFinRows), bted::im::kThreads, 0, T.stream>>>(
        T.P64, nT, (int32_t)N, T.K[0], mu, T.Lf, NPa, 0, T.hv, T.nv, T.rd, T.sel, keys, 0, keys, T.err,
        T.refine ? T.top2 : nullptr, T.Qc, nullptr, nullptr);
    LAUNCHED(3);
}

bool capturing(cudaStream_t st) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(st, &cs);
    return cs != cudaStreamCaptureStatusNone;
}
// Grid of the persistent loop kernel: every CTA must be resident at once (grid
// barriers), so the grid is the measured occupancy x SMs (0: cannot run).
int loop_kernel_grid() {
    static std::atomic<int> cached{-1};
    int g = cached.load(std::memory_order_relaxed);
    if (g < 0) {
        int nb = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, bted::im::ted_loop_kernel, bted::im::kTPThreads,
                                                          bted::im::tile_pass_smem_bytes) != cudaSuccess)
            nb = 0;
        cudaGetLastError();
        g = std::min(nb, bted::im::kTPBlocksPerSM) * num_sms();
        cached.store(g, std::memory_order_relaxed);
    }
    return g;
}

// loop: per step the new factor column (A), q = K l over the tiles (B), scores (C).
// BTED_FLAG_PERSISTENT_LOOP: all m-1 steps in ONE cooperative persistent kernel (ted_loop_kernel:
// grid barriers between the phases, the TMA producer streams across them).
// Default (or no co-resident grid): 3(m-1) kernels.
uint64_t enqueue_loop_implicit(Ted& T, int64_t N, int32_t m, float mu, unsigned long long* keys) {
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int64_t NP = (int64_t)nT * bted::pk::T, NPa = (NP + 255) / 256 * 256;
    const int64_t tiles = bted::pk::num_tiles(nT);
    const int nA = (int)(NPa / bted::im::kEllRows);
    const int grid = T.split ? 0 : loop_kernel_grid();
    if (grid > 0) {
        CK(cudaMemsetAsync(T.bar, 0, sizeof(int) * bted::im::loop_sync_ints(nA, m), T.stream));
        // BTED_TRACE=<file>: phase timestamps of every CTA and step (debug; eager runs only)
        static const char* trace_path = std::getenv("BTED_TRACE");
        static unsigned long long* trace = nullptr;
        const size_t ntr = (size_t)grid * m * 8;
        if (trace_path && !trace) CK(cudaMalloc(&trace, sizeof(unsigned long long) * ntr * 4));
        bted::im::LoopArgs a{T.K[0], nT, (int32_t)N, T.Lf, NPa, m, mu, T.rd, T.nv, keys, T.ell, T.Qc, T.G,
                             T.hv, T.P64, T.sel, T.err, T.refine ? T.top2 : nullptr, T.kflag,
                             trace_path ? trace : nullptr, T.bar, l2_keep_tiles(tiles)};
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3((unsigned)grid);
        cfg.blockDim = dim3(bted::im::kTPThreads);
        cfg.dynamicSmemBytes = bted::im::tile_pass_smem_bytes;
        cfg.stream = T.stream;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeCooperative;
        attr[0].val.cooperative = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        CK(cudaLaunchKernelEx(&cfg, bted::im::ted_loop_kernel, a));
        LAUNCHED(1);
        if (trace_path && !capturing(T.stream)) {
            std::vector<unsigned long long> h(ntr);
            CK(cudaMemcpyAsync(h.data(), trace, sizeof(unsigned long long) * ntr, cudaMemcpyDeviceToHost, T.stream));
            CK(cudaStreamSynchronize(T.stream));
            if (FILE* f = std::fopen(trace_path, "ab")) {
                const int hdr[3] = {grid, m, 8};
                std::fwrite(hdr, sizeof hdr, 1, f);
                std::fwrite(h.data(), sizeof(unsigned long long), ntr, f);
                std::fclose(f);
            }
        }
        return 1;
    }
    // programmatic dependent launches: each kernel may be scheduled while its
    // predecessor drains (the kernels order themselves with griddepcontrol)
    cudaLaunchAttribute pdl[1];
    pdl[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    pdl[0].val.programmaticStreamSerializationAllowed = 1;
    auto cfg_of = [&](unsigned grid, unsigned block, size_t smem) {
        cudaLaunchConfig_t c{};
        c.gridDim = dim3(grid);
        c.blockDim = dim3(block);
        c.dynamicSmemBytes = smem;
        c.stream = T.stream;
        c.attrs = pdl;
        c.numAttrs = 1;
        return c;
    };
    const cudaLaunchConfig_t cA = cfg_of((unsigned)nA + 1, bted::im::kThreads, 0);      // + the h CTA
    const cudaLaunchConfig_t cB = T.rc_on ? cfg_of(rc_pass_grid(tiles), bted::rc::kThreads, bted::rc::kSmemBytes)
                                          : cfg_of(tile_pass_grid(tiles), bted::im::kTPThreads,
                                                   bted::im::tile_pass_smem_bytes);
    const cudaLaunchConfig_t cC = cfg_of((unsigned)(NP / bted::im::kFinRows), bted::im::kThreads, 0);
    const int keep = l2_keep_tiles(tiles);
    for (int32_t t = 1; t < m; ++t) {
        const int32_t tp = t - 1;
        CK(cudaLaunchKernelEx(&cA, bted::im::ell_kernel, (const float*)T.K[0], nT, (int32_t)N, T.Lf, NPa, tp,
                              (const double*)T.rd, (const double*)T.nv, mu, (const unsigned long long*)keys, t, T.ell,
                              (const double*)T.Qc, T.G, m, T.hv, T.sel, bted::im::XKern{}));
        if (T.rc_on)
            CK(cudaLaunchKernelEx(&cB, bted::rc::rc_pass_kernel<false>, (const uint8_t*)T.opB, (const uint8_t*)T.opA,
                                  (const float*)T.xnrm, (const int*)T.xmax, T.rc_gamma, (int32_t)N,
                                  (const float*)T.K[0], nT, (const double*)T.ell, T.P64, T.kflag));
        else
            CK(cudaLaunchKernelEx(&cB, keep_partials(nT) ? bted::im::tile_pass_kernel<false, true>
                                                         : bted::im::tile_pass_kernel<false, false>,
                                  (const float*)T.K[0], nT,
                                  (const double*)T.ell, T.P64, T.kflag, T.tctr + t, (int)(t & 1),
                                  t + 1 < m ? keep : 0, 0, 1));
        CK(cudaLaunchKernelEx(&cC, bted::im::fin64_kernel, (const double*)T.P64, nT, (int32_t)N,
                              (const float*)T.K[0], mu, (const double*)T.Lf, NPa, tp, (const double*)T.hv, T.nv, T.rd,
                              (const uint8_t*)T.sel, (const unsigned long long*)keys, t, keys + t, T.err,
                              T.refine ? T.top2 : nullptr, T.Qc, (const double*)nullptr, (const double*)nullptr));
        LAUNCHED(3);
    }
    return 3 * (uint64_t)(m - 1);
}

// Alg. 1 l.1 + first l.3: XT, zero keys/sel, K1.  (2 kernels)
void enqueue_head(Ted& T, const float* X, int64_t N, int32_t d, float gamma, int kernel, int32_t m, float mu,
                  unsigned long long* keys) {
    launch_transpose(T, X, N, d);
    CK(cudaMemsetAsync(keys, 0, sizeof(unsigned long long) * m, T.stream));
    CK(cudaMemsetAsync(T.sel, 0, (size_t)N, T.stream));
    launch_gram(T, N, d, 0, N, gamma, kernel, mu, keys, T.refine ? T.top2 : nullptr);
}
// Alg. 1 l.2-6 loop: m-1 fused deflate + rescore steps.  (m-1 kernels)
void enqueue_loop(Ted& T, int64_t N, int32_t m, float mu, unsigned long long* keys) {
    for (int32_t t = 1; t < m; ++t) launch_step(T, N, 0, N, t, mu, nullptr, keys, T.refine ? T.top2 : nullptr);
}

template <class F>
void graph_run(Ted& T, const GraphKey& key, uint64_t nkernels, F&& enqueue) {
    for (auto it = T.graphs.begin(); it != T.graphs.end(); ++it) {
        if (it->first == key) {
            T.graphs.splice(T.graphs.begin(), T.graphs, it);
            CK(cudaGraphLaunch(it->second, T.stream));
            LAUNCHED(nkernels);
            return;
        }
    }
    cudaGraph_t g = nullptr;
    CK(cudaStreamBeginCapture(T.stream, cudaStreamCaptureModeThreadLocal));
    const uint64_t before = g_launches.load();
    try {
        enqueue();
    } catch (...) {
        cudaStreamEndCapture(T.stream, &g);
        if (g) cudaGraphDestroy(g);
        throw;
    }
    g_launches.store(before);   // captured launches run below, counted there
    CK(cudaStreamEndCapture(T.stream, &g));
    cudaGraphExec_t ex = nullptr;
    cudaError_t e = cudaGraphInstantiate(&ex, g, 0);
    cudaGraphDestroy(g);
    CK(e);
    T.graphs.emplace_front(key, ex);
    while (T.graphs.size() > 16) {
        cudaGraphExecDestroy(T.graphs.back().second);
        T.graphs.pop_back();
    }
    CK(cudaGraphLaunch(ex, T.stream));
    LAUNCHED(nkernels);
}

// Run one TED (graph-cached unless no_graph); results stay on the device.
void ensure_packed_attrs() {
    static uint64_t done = 0;
    once_per_device(done, [] {
        CK(cudaFuncSetAttribute(K2P_TMA_KERNEL, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)kK2pSmem));
    });
}

// packed layout unless the caller asks for dense or d is too wide for K1p
bool use_packed(uint32_t flags, int32_t d) { return !(flags & BTED_FLAG_DENSE) && d <= 32; }

// nflag_dst: K4 near-tie count of this TED (packed / implicit engines), nullable.
// forced_keys (host, pinned or pageable; nf entries, flagged kForced): preset
// picks of steps 0..nf-1 (K4 re-run with a corrected prefix; eager launches).
void run_ted(Ted& T, const float* X, int64_t N, int32_t d, float gamma, int kernel, int32_t m, float mu,
             unsigned long long* keys, bool no_graph, bool time_it = true, bool packed = false,
             int* nflag_dst = nullptr, const unsigned long long* forced_keys = nullptr, int nf = 0,
             int* flags_dst = nullptr, uint32_t* cand_dst = nullptr, int* ncand_dst = nullptr) {
    if (forced_keys) no_graph = true;
    const bool implicit = packed && T.implicit && m <= bted::im::kMaxM;
    if (implicit) {
        ensure_implicit_attrs();
        T.reserve_implicit(N, m);
        T.last_nT = (int32_t)((N + bted::pk::T - 1) / bted::pk::T);
    } else if (packed) {
        ensure_packed_attrs();
        T.reserve_packed(N, m);
        T.last_nT = (int32_t)((N + bted::pk::T - 1) / bted::pk::T);
    } else {
        T.reserve(N, N, d, m);
        if (T.refine) {                    // K4 on the dense engine: top-2 keys of every K2 CTA
            const void* top2_before = T.top2;
            T.reserve_refine((int64_t)((N + kRowsPerK2Cta - 1) / kRowsPerK2Cta) * 32, m);
            if (T.top2 != top2_before) { for (auto& g : T.graphs) cudaGraphExecDestroy(g.second); T.graphs.clear(); }
        }
    }
    T.last_packed = packed;
    T.last_rows = N;
    T.last_ld = ld_for(N);
    T.last_buf = implicit ? 0 : (m - 1) & 1;  // implicit: K stays the Gram (buffer 0, never deflated)
    Ted::Slot* sl = (T.timing && time_it) ? T.next_slot(m) : nullptr;
    if (sl) CK(cudaEventRecord(sl->e[0], T.stream));
    auto head = [&] {
        if (implicit) enqueue_head_implicit(T, X, N, d, gamma, kernel, m, mu, keys);
        else if (packed) enqueue_head_packed(T, X, N, d, gamma, kernel, m, mu, keys);
        else enqueue_head(T, X, N, d, gamma, kernel, m, mu, keys);
    };
    auto loop = [&] {
        if (implicit) enqueue_loop_implicit(T, N, m, mu, keys);
        else if (packed) enqueue_loop_packed(T, N, m, mu, keys, T.tma);
        else enqueue_loop(T, N, m, mu, keys);
    };
    const int mode = implicit ? 3 : packed ? (T.tma ? 2 : 1) : 0;
    const uint64_t head_k = implicit ? 3 : 2, loop_k = implicit ? 3 : packed ? 2 : 1;
    const uint64_t loop_n = (implicit && !T.split && loop_kernel_grid() > 0) ? 1 : (uint64_t)(m - 1) * loop_k;
    if (no_graph) {
        head();
    } else {
        GraphKey key{X, N, d, m, kernel, 0, mode, fbits(mu), fbits(gamma), keys};
        graph_run(T, key, head_k, head);
    }
    if (forced_keys && nf > 0)
        CK(cudaMemcpyAsync(keys, forced_keys, sizeof(unsigned long long) * nf, cudaMemcpyHostToDevice, T.stream));
    if (sl) CK(cudaEventRecord(sl->e[1], T.stream));
    if (m > 1) {
        if (no_graph) {
            loop();
        } else {
            GraphKey key{X, N, d, m, kernel, 1, mode, fbits(mu), fbits(gamma), keys};
            graph_run(T, key, loop_n, loop);
        }
    }
    if (sl) CK(cudaEventRecord(sl->e[2], T.stream));
    if (T.refine && nflag_dst) {
        // K4 check; its per-step flags/candidates go to T's buffers or, for a batch
        // TED of Alg. 2, to that batch's own slice (refined later without a re-run)
        bted::rf::neartie_check_kernel<<<m, 256, 0, T.stream>>>(T.top2, T.last_nC, keys, bted::rf::kTau,
                                                               flags_dst ? flags_dst : T.flags,
                                                               cand_dst ? cand_dst : T.cand,
                                                               ncand_dst ? ncand_dst : T.ncand, nflag_dst);
        LAUNCHED(1);
    }
}


}  // namespace

// ------------------------------------------------------------------ context
struct bted_ctx {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bted_kernel kernel = BTED_KERNEL_RBF;
    bted_params params{};
    int64_t N = 0;
    int32_t d = 0;
    float* X = nullptr;       // device N x d
    bool own_X = false;
    bool poisoned = false;
    // shard
    bool is_shard = false;
    int64_t row0 = 0, row1 = 0;
    // tile shard of the implicit engine (bted_ishard_*)
    bool is_ishard = false;
    int32_t srank = 0, snranks = 1, sm_m = 0;
    Ted ted;
    // batches (Alg. 2)
    Ted bted_engine;          // the M x M batch TEDs and the merge TED
    float* Xb = nullptr; size_t xbcap = 0;
    int64_t* winners = nullptr; size_t winnerscap = 0;
    uint32_t* u32a = nullptr; size_t u32acap = 0;
    uint32_t* u32b = nullptr; size_t u32bcap = 0;
    int* count_dev = nullptr; size_t countcap = 0;
    unsigned long long* mkeys = nullptr; size_t mkeyscap = 0;
    void* cub_tmp = nullptr; size_t cub_cap = 0;
    int64_t* out_dev = nullptr; size_t outcap = 0;
    uint32_t* sall = nullptr; size_t sallcap = 0;          // [nb][M] draws (sorted V_b)
    unsigned* shist = nullptr; size_t shistcap = 0;        // radix-select sampler scratch
    int* sint = nullptr; size_t sintcap = 0;
    uint64_t* scand = nullptr; size_t scandcap = 0;
    uint32_t* ssel = nullptr; size_t sselcap = 0;
    int* soff = nullptr; size_t soffcap = 0;
    uint64_t* sks = nullptr; size_t skscap = 0;            // k* (M-th smallest key) per batch
    unsigned* scnt = nullptr; size_t scntcap = 0;          // [nb][G] chunk counts -> offsets
    int* bflag = nullptr; size_t bflagcap = 0;             // K4: near ties per batch TED
    unsigned long long* bkeys = nullptr; size_t bkeyscap = 0; // K4: [nb][m] keys of every batch TED
    int* bsflags = nullptr; size_t bsflagscap = 0;           //     [nb][m] per-step near-tie flags
    int* bncand = nullptr; size_t bncandcap = 0;             //     [nb][m] candidate counts
    uint32_t* bcand = nullptr; size_t bcandcap = 0;          //     [nb][m][kMaxCand] candidates
    // K4 refinement scratch
    uint32_t* rcols = nullptr; size_t rcolscap = 0;
    double* rG = nullptr; size_t rGcap = 0;
    double* rA = nullptr; size_t rAcap = 0;
    double* rW = nullptr; size_t rWcap = 0;
    double* rpart = nullptr; size_t rpartcap = 0;
    double* rdiag = nullptr; size_t rdiagcap = 0;
    double* rout = nullptr; size_t routcap = 0;
    double* rWt = nullptr; size_t rWtcap = 0;             // full re-scoring: W^T (t x N), scores, selected mask
    double* rsc = nullptr; size_t rsccap = 0;
    uint8_t* rmask = nullptr; size_t rmaskcap = 0;
    uint64_t full_refined_steps = 0;
    uint32_t* ridx = nullptr; size_t ridxcap = 0;
    uint64_t refined_steps = 0, corrected_steps = 0;
    // K4 for the cluster-kernel TEDs: per-instance top-2 keys, flags, candidates, counts, forced picks
    unsigned long long* ktop2 = nullptr; size_t ktop2cap = 0;
    int* kflags = nullptr; size_t kflagscap = 0;
    uint32_t* kcand = nullptr; size_t kcandcap = 0;
    int* kncand = nullptr; size_t kncandcap = 0;
    int* knflag = nullptr; size_t knflagcap = 0;
    unsigned long long* kforced = nullptr; size_t kforcedcap = 0;
    int* k4pin = nullptr; size_t k4pincap = 0;            // pinned copy of knflag (read after the next sync)
    struct {                                              // batch K4 decided at the merge's host sync
        bool pending = false, changed = false;
        int ninst = 0; int64_t M = 0; int32_t m = 0; float mu = 0.f;
    } k4b;
    struct {                                              // the same for the large (non-cluster) batch TEDs
        bool pending = false;
        int nb = 0; int64_t M = 0; int32_t m = 0; float mu = 0.f;
    } k4big;
    int* bfpin = nullptr; size_t bfpincap = 0;            // pinned copy of bflag
    float* xall = nullptr; size_t xallcap = 0;             // [nb][M][d] gathered batches
    unsigned long long* kall = nullptr; size_t kallcap = 0; // [nb][m] keys
    // host staging (pinned)
    unsigned long long* hkeys = nullptr; size_t hkeyscap = 0;
    int* herr = nullptr;
    int* xbad = nullptr;      // device: non-finite feature seen by finite_check_kernel
    struct MultiDev* md = nullptr;   // num_devices > 1: the per-device shards / replicas
};

namespace {

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        cudaGetDevice(&prev);
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        cudaGetDevice(&cur);
        if (prev >= 0 && cur != prev) cudaSetDevice(prev);
    }
};

void host_grow(unsigned long long*& p, size_t& cap, size_t n) {
    if (n <= cap) return;
    if (p) cudaFreeHost(p);
    p = nullptr;
    cap = 0;
    CK(cudaMallocHost(&p, sizeof(unsigned long long) * n));
    cap = n;
}

template <class F>
bted_status guarded(bted_ctx* ctx, F&& f) {
    if (!ctx) { set_error("null context"); return BTED_EINVAL; }
    if (ctx->poisoned) { set_error("context poisoned by an earlier CUDA error"); return BTED_ESTATE; }
    try {
        DeviceGuard dg(ctx->device);
        return f();
    } catch (const CudaError& e) {
        ctx->poisoned = true;
        set_error("CUDA error %s (%s) in %s", cudaGetErrorName(e.e), cudaGetErrorString(e.e), e.what);
        cudaGetLastError();
        return e.e == cudaErrorMemoryAllocation ? BTED_ENOMEM : BTED_ECUDA;
    } catch (const NcclError& e) {
        ctx->poisoned = true;
        set_error("%s", e.what.c_str());
        cudaGetLastError();
        return BTED_ENCCL;
    } catch (const std::bad_alloc&) {
        set_error("host allocation failed");
        return BTED_ENOMEM;
    }
}

void launch_finite_check(bted_ctx* ctx) {
    const int64_t n = ctx->N * ctx->d;
    const unsigned g = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 8);
    bted::finite_check_kernel<<<g, 256, 0, ctx->stream>>>(ctx->X, n, ctx->xbad);
    LAUNCHED(1);
}

// a bted_update of non-finite features surfaces at the next host sync
bool take_xbad(bted_ctx* ctx) {
    int v = 0;
    CK(cudaMemcpy(&v, ctx->xbad, sizeof(int), cudaMemcpyDeviceToHost));
    if (v) {
        // the run on the bad features may also have raised the numeric flags: clear all
        CK(cudaMemset(ctx->xbad, 0, sizeof(int)));
        if (ctx->ted.err) CK(cudaMemset(ctx->ted.err, 0, sizeof(int)));
        if (ctx->bted_engine.err) CK(cudaMemset(ctx->bted_engine.err, 0, sizeof(int)));
        set_error("X has non-finite entries (bted_update)");
    }
    return v != 0;
}

// Decode m packed keys on the host; checks the sticky error flag.
bted_status finish_keys(bted_ctx* ctx, Ted& T, const unsigned long long* keys_dev, int32_t m,
                        int64_t* out_idx, float* out_score, const int64_t* map_dev = nullptr) {
    host_grow(ctx->hkeys, ctx->hkeyscap, (size_t)m + 1);
    CK(cudaMemcpyAsync(ctx->hkeys, keys_dev, sizeof(unsigned long long) * m, cudaMemcpyDeviceToHost, T.stream));
    CK(cudaMemcpyAsync(ctx->herr, T.err, sizeof(int), cudaMemcpyDeviceToHost, T.stream));
    if (map_dev) CK(cudaMemcpyAsync(out_idx, map_dev, sizeof(int64_t) * m, cudaMemcpyDeviceToHost, T.stream));
    CK(cudaStreamSynchronize(T.stream));
    T.collect();
    if (ctx->xbad && take_xbad(ctx)) return BTED_EINVAL;
    if (*ctx->herr & bted::im::kErrPeerTimeout) {
        CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream));
        ctx->poisoned = true;
        set_error("multi-GPU exchange: a peer device never published its step (20 s flag wait)");
        return BTED_ENCCL;
    }
    if (*ctx->herr & bted::kSampleOverflow) {
        CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream));
        set_error("batch sampler: candidate bin overflow (internal limit kCandCap)");
        return BTED_ENUMERIC;
    }
    if (*ctx->herr & 4) {
        CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream));
        set_error("persistent TED loop: grid barrier timed out (CTAs not co-resident)");
        return BTED_ECUDA;
    }
    if (*ctx->herr) {
        CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream));
        set_error("non-finite score or non-positive k(v,v)+mu during TED");
        return BTED_ENUMERIC;
    }
    for (int32_t t = 0; t < m; ++t) {
        const unsigned long long k = ctx->hkeys[t] & ~bted::rf::kForced;   // K4-forced picks carry a flag bit
        if (k == 0ull) { set_error("no candidate at step %d (internal)", t); return BTED_ENUMERIC; }
        if (!map_dev) out_idx[t] = (int64_t)(0xFFFFFFFFu - (uint32_t)(k & 0xFFFFFFFFull));
        if (out_score) {
            uint32_t b = (uint32_t)(k >> 32) - 1u;
            std::memcpy(&out_score[t], &b, 4);
        }
    }
    return BTED_OK;
}

bted_status validate_params(const bted_params* p, bted_kernel kernel) {
    if (!p) { set_error("null params"); return BTED_EINVAL; }
    if (kernel != BTED_KERNEL_RBF && kernel != BTED_KERNEL_LINEAR) { set_error("bad kernel"); return BTED_EINVAL; }
    if (kernel == BTED_KERNEL_RBF && !(p->gamma > 0.f && std::isfinite(p->gamma))) {
        set_error("gamma must be > 0 and finite"); return BTED_EINVAL;
    }
    if (p->num_batches < 1) { set_error("num_batches must be >= 1"); return BTED_EINVAL; }
    if (p->num_devices < 0) { set_error("num_devices must be >= 1"); return BTED_EINVAL; }
    if (p->norm_mode != 0 && p->norm_mode != 1) { set_error("norm_mode must be 0 or 1"); return BTED_EINVAL; }
    return BTED_OK;
}

bted_status create_common(const float* X, int64_t N, int32_t d, bted_kernel kernel, const bted_params* params,
                          int64_t row0, int64_t row1, bool shard, bted_ctx** out) {
    if (!out) { set_error("null out"); return BTED_EINVAL; }
    *out = nullptr;
    if (bted_status s = validate_params(params, kernel)) return s;
    if (!X || N < 1 || N >= (int64_t)INT32_MAX || d < 1 || d > 64) {
        set_error("need X != NULL, 1 <= N < 2^31, 1 <= d <= 64"); return BTED_EINVAL;
    }
    if (shard && !(0 <= row0 && row0 < row1 && row1 <= N)) { set_error("need 0 <= row0 < row1 <= N"); return BTED_EINVAL; }
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev < 1) {
        cudaGetLastError();
        set_error("no CUDA device available (%s): libbted has no CPU fallback", cudaGetErrorString(e));
        return BTED_ECUDA;
    }
    bted_ctx* ctx = new (std::nothrow) bted_ctx();
    if (!ctx) { set_error("host allocation failed"); return BTED_ENOMEM; }
    ctx->params = *params;
    ctx->kernel = kernel;
    ctx->N = N;
    ctx->d = d;
    ctx->is_shard = shard;
    ctx->row0 = shard ? row0 : 0;
    ctx->row1 = shard ? row1 : N;
    int dev = params->device;
    if (dev < 0) cudaGetDevice(&dev);
    ctx->device = dev;
    bted_status st = guarded(ctx, [&]() -> bted_status {
        cudaDeviceProp prop;
        CK(cudaGetDeviceProperties(&prop, ctx->device));
        if (prop.major < 10) {
            set_error("device %d is sm_%d%d; libbted is built for sm_100a only", ctx->device, prop.major, prop.minor);
            return BTED_ECUDA;
        }
        if (params->stream) {
            ctx->stream = reinterpret_cast<cudaStream_t>(params->stream);
        } else {
            CK(cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking));
            ctx->own_stream = true;
        }
        ctx->ted.stream = ctx->stream;
        ctx->bted_engine.stream = ctx->stream;
        ctx->ted.timing = ctx->bted_engine.timing = (params->flags & BTED_FLAG_TIMING) != 0;
        ctx->ted.tma = ctx->bted_engine.tma = (params->flags & BTED_FLAG_TMA) != 0;
        ctx->ted.implicit = ctx->bted_engine.implicit = (params->flags & BTED_FLAG_LITERAL) == 0;
        ctx->ted.refine = ctx->bted_engine.refine = (params->flags & BTED_FLAG_NO_REFINE) == 0;
        ctx->ted.split = ctx->bted_engine.split = (params->flags & BTED_FLAG_PERSISTENT_LOOP) == 0;
        ctx->ted.gram_tc = ctx->bted_engine.gram_tc = (params->flags & BTED_FLAG_NO_TC_GRAM) == 0;
        ctx->ted.rc = ctx->bted_engine.rc = (params->flags & BTED_FLAG_RECOMPUTE) != 0;
        CK(cudaMallocHost(&ctx->herr, sizeof(int)));
        if (params->x_on_device) {
            ctx->X = const_cast<float*>(X);
        } else {
            CK(cudaMalloc(&ctx->X, sizeof(float) * N * d));
            ctx->own_X = true;
            CK(cudaMemcpyAsync(ctx->X, X, sizeof(float) * N * d, cudaMemcpyHostToDevice, ctx->stream));
        }
        CK(cudaMalloc(&ctx->xbad, sizeof(int)));
        CK(cudaMemsetAsync(ctx->xbad, 0, sizeof(int), ctx->stream));
        launch_finite_check(ctx);
        CK(cudaMemcpyAsync(ctx->herr, ctx->xbad, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        if (*ctx->herr) { set_error("X has non-finite entries"); return BTED_EINVAL; }
        return BTED_OK;
    });
    if (st != BTED_OK) {
        bted_destroy(ctx);
        return st;
    }
    *out = ctx;
    return BTED_OK;
}

bool mu_ok(float mu) { return mu > 0.f && std::isfinite(mu); }

// cub temp storage: grow to what the largest call needs.
void cub_reserve(bted_ctx* ctx, size_t bytes) {
    if (bytes <= ctx->cub_cap) return;
    if (ctx->cub_tmp) cudaFree(ctx->cub_tmp);
    ctx->cub_tmp = nullptr;
    ctx->cub_cap = 0;
    CK(cudaMalloc(&ctx->cub_tmp, bytes));
    ctx->cub_cap = bytes;
}

int bits_for(uint64_t maxval) {
    int b = 1;
    while (b < 64 && (maxval >> b) != 0) ++b;
    return b;
}

// Alg. 2 l.2 for batches b_begin, b_begin + b_step, ... (nb of them) at once:
// out[k][0..M) = sorted V_{b_begin + k b_step}, by radix select (sample.cuh).
void sample_batches_dev(bted_ctx* ctx, cudaStream_t st, int64_t P, int64_t M, int32_t b_begin, int32_t b_step,
                        int nb, uint64_t seed, uint32_t* out) {
    Nvtx nvtx_("bted sample (Alg. 2 l.2)");
    grow(ctx->shist, ctx->shistcap, (size_t)2 * nb * bted::kSelBins);
    grow(ctx->sint, ctx->sintcap, (size_t)5 * nb + 1);
    grow(ctx->scand, ctx->scandcap, (size_t)nb * bted::kCandCap);
    unsigned* hist0 = ctx->shist;
    unsigned* hist1 = ctx->shist + (size_t)nb * bted::kSelBins;
    int* bstar0 = ctx->sint;
    int* below0 = ctx->sint + nb;
    int* bstar1 = ctx->sint + 2 * nb;
    int* below1 = ctx->sint + 3 * nb;
    unsigned* ncand = reinterpret_cast<unsigned*>(ctx->sint + 4 * nb);
    if (!ctx->bted_engine.err) {
        grow(ctx->bted_engine.err, ctx->bted_engine.errcap, 1);
        CK(cudaMemsetAsync(ctx->bted_engine.err, 0, sizeof(int), st));
    }
    CK(cudaMemsetAsync(ctx->shist, 0, sizeof(unsigned) * 2 * nb * bted::kSelBins, st));
    CK(cudaMemsetAsync(ncand, 0, sizeof(unsigned) * nb, st));
    const unsigned gx = (unsigned)std::max<int64_t>(1, std::min<int64_t>((P + 1023) / 1024, 64));
    // two 12-bit radix levels: the candidate bin holds ~P / 2^24 keys
    bted::sel_hist_kernel<<<dim3(gx, nb), 256, 0, st>>>((uint64_t)P, seed, b_begin, b_step, nullptr, hist0);
    bted::sel_thresh_kernel<<<nb, 1024, 0, st>>>(hist0, M, nullptr, bstar0, below0);
    bted::sel_hist_kernel<<<dim3(gx, nb), 256, 0, st>>>((uint64_t)P, seed, b_begin, b_step, bstar0, hist1);
    bted::sel_thresh_kernel<<<nb, 1024, 0, st>>>(hist1, M, below0, bstar1, below1);
    bted::sel_collect_kernel<<<dim3(gx, nb), 256, 0, st>>>((uint64_t)P, seed, b_begin, b_step, bstar0, bstar1,
                                                            ctx->scand, ncand);
    // k* per batch, then the ordered compaction (V_b ascending, no sort)
    const int G = (int)((P + bted::kCmpChunk - 1) / bted::kCmpChunk);
    grow(ctx->sks, ctx->skscap, (size_t)nb);
    grow(ctx->scnt, ctx->scntcap, (size_t)nb * G);
    bted::sel_finish_kernel<<<nb, 1024, 0, st>>>(M, below1, ctx->scand, ncand, ctx->bted_engine.err, ctx->sks);
    bted::sel_count_kernel<<<dim3(G, nb), bted::kCmpThreads, 0, st>>>((uint64_t)P, seed, b_begin, b_step, ctx->sks,
                                                                     ctx->scnt, ctx->bted_engine.err);
    bted::sel_scan_kernel<<<nb, 1024, 0, st>>>(ctx->scnt, G);
    bted::sel_write_kernel<<<dim3(G, nb), bted::kCmpThreads, 0, st>>>((uint64_t)P, seed, b_begin, b_step, ctx->sks,
                                                                     ctx->scnt, M, out, ctx->bted_engine.err);
    LAUNCHED(9);
}

void gather(bted_ctx* ctx, cudaStream_t st, const uint32_t* idx, int64_t M, float* dst = nullptr) {
    if (!dst) {
        grow(ctx->Xb, ctx->xbcap, (size_t)(M * ctx->d));
        dst = ctx->Xb;
    }
    const int64_t total = M * ctx->d;
    const unsigned g = (unsigned)std::min<int64_t>((total + 255) / 256, 148 * 32);
    bted::gather_rows_kernel<<<g, 256, 0, st>>>(ctx->X, ctx->d, idx, M, dst);
    LAUNCHED(1);
}

// ---- K4: near-tie refinement (refine.cuh) ----
// fp64 closed-form scores of the candidates C after the picks S; returns the
// exact argmax (ties: lowest index) and its score.
void refine_step(bted_ctx* ctx, cudaStream_t st, const float* X, int64_t N, int32_t d,
                 const std::vector<uint32_t>& S, const std::vector<uint32_t>& C, float mu, uint32_t* best,
                 double* best_score) {
    const int t = (int)S.size(), nc = (int)C.size(), ncol = t + nc;
    std::vector<uint32_t> cols(S);
    cols.insert(cols.end(), C.begin(), C.end());
    grow(ctx->rcols, ctx->rcolscap, (size_t)ncol);
    grow(ctx->rG, ctx->rGcap, (size_t)ncol * N);
    grow(ctx->rA, ctx->rAcap, (size_t)std::max(1, t * t));
    grow(ctx->rW, ctx->rWcap, (size_t)bted::rf::kMaxCand * std::max(1, t));
    const int nblk = (int)((N + 255) / 256);
    grow(ctx->rpart, ctx->rpartcap, (size_t)nblk * bted::rf::kMaxCand);
    grow(ctx->rdiag, ctx->rdiagcap, (size_t)bted::rf::kMaxCand);
    grow(ctx->rout, ctx->routcap, (size_t)bted::rf::kMaxCand + 1);
    grow(ctx->ridx, ctx->ridxcap, 1);
    CK(cudaMemcpyAsync(ctx->rcols, cols.data(), sizeof(uint32_t) * ncol, cudaMemcpyHostToDevice, st));
    const int lin = ctx->kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    bted::rf::refine_cols_kernel<<<dim3((unsigned)((N + 255) / 256), (unsigned)ncol), 256, 0, st>>>(
        X, (int32_t)N, d, (double)ctx->params.gamma, lin, ctx->rcols, ctx->rG);
    // A (t x t) in shared memory when it fits; with the candidates' right-hand sides too (mode 2), the
    // triangular solves run on all threads instead of one thread per candidate
    const size_t asmem = sizeof(double) * (size_t)t * (size_t)t;
    const size_t absmem = asmem + sizeof(double) * (size_t)nc * (size_t)t;
    const int amode = absmem <= 48 * 1024 ? 2 : asmem <= 48 * 1024 ? 1 : 0;
    bted::rf::refine_solve_kernel<<<1, 256, amode == 2 ? absmem : amode == 1 ? asmem : 0, st>>>(
        ctx->rG, (int32_t)N, ctx->rcols, t, nc, (double)mu, ctx->rA, ctx->rW, amode);
    bted::rf::refine_resid2_kernel<<<dim3((unsigned)nblk, (unsigned)nc), 256, sizeof(double) * std::max(t, 1), st>>>(
        ctx->rG, (int32_t)N, ctx->rcols, t, ctx->rW, ctx->rpart, ctx->rdiag);
    bted::rf::refine_pick_kernel<<<1, 32, 0, st>>>(ctx->rpart, nblk, ctx->rdiag, ctx->rcols, t, nc, (double)mu,
                                                  ctx->rout, ctx->ridx);
    LAUNCHED(4);
    double sc = 0.0;
    CK(cudaMemcpyAsync(best, ctx->ridx, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&sc, ctx->rout + bted::rf::kMaxCand, sizeof(double), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    *best_score = sc;
}

// fp64 closed-form scores of ALL points after the picks S (refine.cuh, kFlagFull:
// the near-tie candidate list of a step may be incomplete); returns the exact
// argmax over the unselected points (ties: lowest index) and its score.
void refine_full(bted_ctx* ctx, cudaStream_t st, const float* X, int64_t N, int32_t d,
                 const std::vector<uint32_t>& S, float mu, uint32_t* best, double* best_score) {
    const int t = (int)S.size();
    grow(ctx->rcols, ctx->rcolscap, (size_t)std::max(t, 1));
    grow(ctx->rG, ctx->rGcap, (size_t)std::max(t, 1) * N);
    grow(ctx->rA, ctx->rAcap, (size_t)std::max(1, t * t));
    grow(ctx->rWt, ctx->rWtcap, (size_t)std::max(t, 1) * N);
    grow(ctx->rsc, ctx->rsccap, (size_t)N);
    grow(ctx->rmask, ctx->rmaskcap, (size_t)N);
    grow(ctx->rout, ctx->routcap, (size_t)bted::rf::kMaxCand + 1);
    grow(ctx->ridx, ctx->ridxcap, 1);
    std::vector<uint8_t> mask((size_t)N, 0);
    for (uint32_t s : S) mask[s] = 1;
    CK(cudaMemcpyAsync(ctx->rmask, mask.data(), (size_t)N, cudaMemcpyHostToDevice, st));
    const int lin = ctx->kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    if (t > 0) {
        CK(cudaMemcpyAsync(ctx->rcols, S.data(), sizeof(uint32_t) * t, cudaMemcpyHostToDevice, st));
        bted::rf::refine_cols_kernel<<<dim3((unsigned)((N + 255) / 256), (unsigned)t), 256, 0, st>>>(
            X, (int32_t)N, d, (double)ctx->params.gamma, lin, ctx->rcols, ctx->rG);
        bted::rf::refine_chol_kernel<<<1, 256, 0, st>>>(ctx->rG, (int32_t)N, ctx->rcols, t, (double)mu, ctx->rA);
        bted::rf::refine_solve_all_kernel<<<(unsigned)((N + 255) / 256), 256, 0, st>>>(ctx->rG, (int32_t)N, t,
                                                                                      ctx->rA, ctx->rWt);
        LAUNCHED(3);
    }
    const size_t wsmem = sizeof(double) * (size_t)std::max(t, 1) * bted::rf::kAllCand;
    static uint64_t attr = 0;
    once_per_device(attr, [] {
        CK(cudaFuncSetAttribute(bted::rf::refine_all_scores_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)(sizeof(double) * bted::im::kMaxM * bted::rf::kAllCand)));
    });
    bted::rf::refine_all_scores_kernel<<<(unsigned)((N + bted::rf::kAllCand - 1) / bted::rf::kAllCand), 256, wsmem,
                                         st>>>(X, (int32_t)N, d, (double)ctx->params.gamma, lin, ctx->rG, t,
                                               ctx->rWt, ctx->rmask, (double)mu, ctx->rsc);
    bted::rf::refine_all_pick_kernel<<<1, 1024, 0, st>>>(ctx->rsc, (int32_t)N, ctx->rout + bted::rf::kMaxCand,
                                                        ctx->ridx);
    LAUNCHED(2);
    double sc = 0.0;
    CK(cudaMemcpyAsync(best, ctx->ridx, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(&sc, ctx->rout + bted::rf::kMaxCand, sizeof(double), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    *best_score = sc;
}

inline unsigned long long host_pack_key(float score, uint32_t idx) {
    uint32_t b;
    std::memcpy(&b, &score, 4);
    return ((unsigned long long)(b + 1u) << 32) | (unsigned long long)(0xFFFFFFFFu - idx);
}

// Resolve the near ties flagged in the last TED run by T on X (keys on the
// device, T.flags / T.cand filled by its check kernel).  Each flagged step is
// re-scored exactly (fp64); if the exact argmax differs from the GPU's pick,
// the TED is re-run with the corrected prefix forced.  On return `keys` on
// the device holds the final picks (forced ones flagged kForced) and
// scores_out[t] (nullable) the fp32 score of each pick.
// K4 host scan (shared by every engine): the first flagged step after `checked`
// (with >= 2 candidates) is re-scored exactly; returns true with `forced` =
// the flagged keys of steps 0..ts (the corrected pick last) if the exact argmax
// differs from the GPU's pick, false once no flagged step is left.  hk, fl,
// nc, cd: the TED's keys, flags, candidate counts and candidates (host copies).
bool k4_next_correction(bted_ctx* ctx, cudaStream_t st, const float* X, int64_t N, int32_t d, int32_t m, float mu,
                        const std::vector<unsigned long long>& hk, const std::vector<int>& fl,
                        const std::vector<int>& nc, const std::vector<uint32_t>& cd, int& checked,
                        std::vector<unsigned long long>& forced, double* corrected_score = nullptr) {
    const size_t kMC = bted::rf::kMaxCand;
    for (int ts = checked + 1; ts < m; ++ts) {
        const bool full = fl[ts] == bted::rf::kFlagFull;
        if (!fl[ts] || (!full && nc[ts] < 2)) continue;
        std::vector<uint32_t> S(ts), C;
        for (int k = 0; k < ts; ++k) S[k] = 0xFFFFFFFFu - (uint32_t)(hk[k] & 0xFFFFFFFFull);
        uint32_t best = 0;
        double bs = 0.0;
        if (full) {                      // the candidate list may be incomplete: every unselected point
            refine_full(ctx, st, X, N, d, S, mu, &best, &bs);
            ctx->full_refined_steps++;
        } else {
            for (int c = 0; c < nc[ts]; ++c) C.push_back(cd[(size_t)ts * kMC + c]);
            std::sort(C.begin(), C.end());
            refine_step(ctx, st, X, N, d, S, C, mu, &best, &bs);
        }
        ctx->refined_steps++;
        checked = ts;
        const uint32_t pick = 0xFFFFFFFFu - (uint32_t)(hk[ts] & 0xFFFFFFFFull);
        if (best == pick) continue;
        ctx->corrected_steps++;
        forced.assign(ts + 1, 0ull);
        for (int k = 0; k < ts; ++k) forced[k] = hk[k] | bted::rf::kForced;
        forced[ts] = host_pack_key((float)bs, best) | bted::rf::kForced;
        if (corrected_score) *corrected_score = bs;
        return true;
    }
    return false;
}

void refine_ted(bted_ctx* ctx, Ted& T, const float* X, int64_t N, int32_t d, int32_t m, float mu,
                unsigned long long* keys, float* scores_out) {
    Nvtx nvtx_("bted K4 refine");
    cudaStream_t st = T.stream;
    std::vector<unsigned long long> hk(m), forced;
    std::vector<int> fl(m), nc(m);
    std::vector<uint32_t> cd((size_t)m * bted::rf::kMaxCand);
    int checked = -1;
    for (int rounds = 0; rounds <= m; ++rounds) {
        CK(cudaMemcpyAsync(hk.data(), keys, sizeof(unsigned long long) * m, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(fl.data(), T.flags, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(nc.data(), T.ncand, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
        CK(cudaMemcpyAsync(cd.data(), T.cand, sizeof(uint32_t) * cd.size(), cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        double bs = 0.0;
        if (!k4_next_correction(ctx, st, X, N, d, m, mu, hk, fl, nc, cd, checked, forced, &bs)) break;
        if (scores_out) scores_out[checked] = (float)bs;
        // corrected pick: re-run (same engine as the TED) with picks 0..ts forced
        CK(cudaMemsetAsync(T.nflag, 0, sizeof(int), st));
        run_ted(T, X, N, d, ctx->params.gamma, ctx->kernel, m, mu, keys, true, false, T.last_packed, T.nflag,
                forced.data(), (int)forced.size());
        CK(cudaStreamSynchronize(st));      // `forced` (pageable) must outlive the copy
    }
}

// ---- small TEDs: one cluster kernel per launch runs every step (small.cuh) ----
int small_cluster_for(int64_t N) {
    if (N < 1 || N > 4096) return 0;
    for (int C = 1; C <= 16; C *= 2)
        if (bted::sm::smem_bytes((int)N, C) <= bted::sm::kSmemBudget) return C;
    return 0;
}
bool use_small(uint32_t flags, int64_t N) { return !(flags & BTED_FLAG_NO_SMALL) && small_cluster_for(N) > 0; }

template <int C>
void launch_small_c(const float* X, int ninst, int32_t N, int32_t d, float gamma, int kernel, int32_t m, float mu,
                    unsigned long long* keys, int* err, cudaStream_t st, unsigned long long* top2,
                    const unsigned long long* forced, int nforced) {
    static uint64_t attr = 0;
    once_per_device(attr, [] {
        CK(cudaFuncSetAttribute(bted::sm::ted_cluster_kernel<C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                (int)bted::sm::kSmemBudget));
        if (C > 8) CK(cudaFuncSetAttribute(bted::sm::ted_cluster_kernel<C>,
                                           cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
    });
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(ninst * C));
    cfg.blockDim = dim3(bted::sm::kThreads);
    const bool stage_x = bted::sm::smem_core(N, C) + bted::sm::smem_x(N, d) <= bted::sm::kSmemBudget;
    cfg.dynamicSmemBytes = bted::sm::smem_core(N, C) + (stage_x ? bted::sm::smem_x(N, d) : 0);
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = C;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    CK(cudaLaunchKernelEx(&cfg, bted::sm::ted_cluster_kernel<C>, X, N, d, gamma,
                          (int32_t)(kernel == BTED_KERNEL_LINEAR ? 1 : 0), m, mu, keys, err, (int32_t)stage_x,
                          top2, forced, (int32_t)nforced));
    LAUNCHED(1);
}

// ninst independent TEDs on X[inst][N][d] -> keys[inst][m]; err = a Ted's flag
// the cluster size launch_small uses for ninst TEDs of N points (K4 sizes its top-2 buffer by it)
int small_cluster_used(int ninst, int64_t N, int32_t d) {
    int C = small_cluster_for(N);
    for (int c2 = C; c2 > 0 && c2 <= 16; c2 *= 2) {
        if ((int64_t)ninst * c2 > num_sms()) break;
        if (bted::sm::smem_core((int)N, c2) + bted::sm::smem_x((int)N, d) <= bted::sm::kSmemBudget) { C = c2; break; }
    }
    return C;
}

// TEDs of at most 128 points run in one CTA each (small.cuh ted_tiny_kernel<64 / 128>);
// BTED_NO_TINY_TED=1 sends them to the cluster kernel instead (A/B only)
constexpr size_t kTinySmemMax = 200 * 1024;
bool use_tiny_ted(int64_t N, int32_t d) {
    static const bool off = [] { const char* e = std::getenv("BTED_NO_TINY_TED"); return e && std::atoi(e); }();
    // (the staged features must fit: otherwise the cluster kernel, which reads them from global memory)
    return !off && N >= 1 && N <= bted::sm::kTinyMaxN && bted::sm::tiny_smem_bytes((int)N, d) <= kTinySmemMax;
}
// score units per TED instance of launch_small (K4's top-2 layout)
int small_units(int ninst, int64_t N, int32_t d) {
    return use_tiny_ted(N, d) ? bted::sm::tiny_max_for((int)N) : small_cluster_used(ninst, N, d) * bted::sm::kWarps;
}

void launch_small(const float* X, int ninst, int64_t N, int32_t d, float gamma, int kernel, int32_t m, float mu,
                  unsigned long long* keys, int* err, cudaStream_t st, unsigned long long* top2 = nullptr,
                  const unsigned long long* forced = nullptr, int nforced = 0) {
    if (use_tiny_ted(N, d)) {
        const size_t smem = bted::sm::tiny_smem_bytes((int)N, d);
        static uint64_t attr = 0;
        once_per_device(attr, [] {
            CK(cudaFuncSetAttribute(bted::sm::ted_tiny_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)kTinySmemMax));
            CK(cudaFuncSetAttribute(bted::sm::ted_tiny_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                    (int)kTinySmemMax));
        });
        const int kmax = bted::sm::tiny_max_for((int)N);
        auto tk = kmax == 64 ? bted::sm::ted_tiny_kernel<64> : bted::sm::ted_tiny_kernel<128>;
        tk<<<(unsigned)ninst, (unsigned)(4 * kmax), smem, st>>>(
            X, (int32_t)N, d, gamma, (int32_t)(kernel == BTED_KERNEL_LINEAR ? 1 : 0), m, mu, keys, err, top2, forced,
            (int32_t)nforced);
        LAUNCHED(1);
        return;
    }
    // the smallest cluster whose CTAs also hold the staged features, if the
    // ninst clusters still fit on the SMs at once; else the smallest that fits
    const int C = small_cluster_used(ninst, N, d);
    switch (C) {
        case 1: launch_small_c<1>(X, ninst, (int32_t)N, d, gamma, kernel, m, mu, keys, err, st, top2, forced, nforced); break;
        case 2: launch_small_c<2>(X, ninst, (int32_t)N, d, gamma, kernel, m, mu, keys, err, st, top2, forced, nforced); break;
        case 4: launch_small_c<4>(X, ninst, (int32_t)N, d, gamma, kernel, m, mu, keys, err, st, top2, forced, nforced); break;
        case 8: launch_small_c<8>(X, ninst, (int32_t)N, d, gamma, kernel, m, mu, keys, err, st, top2, forced, nforced); break;
        case 16: launch_small_c<16>(X, ninst, (int32_t)N, d, gamma, kernel, m, mu, keys, err, st, top2, forced, nforced); break;
        default: throw CudaError{cudaErrorInvalidValue, "launch_small: N too large"};
    }
}

// ---- K4 for cluster-kernel TEDs (merges, small batches, small bted_select) ----
// Buffers for ninst instances of m steps; returns the top-2 buffer to pass to launch_small.
unsigned long long* small_k4_reserve(bted_ctx* ctx, int ninst, int64_t N, int32_t d, int32_t m) {
    const int nU = small_units(ninst, N, d);
    const int nU1 = small_units(1, N, d);                                  // single-instance re-runs
    grow(ctx->ktop2, ctx->ktop2cap, (size_t)ninst * m * nU * 2 + (size_t)m * nU1 * 2);   // + re-run scratch
    grow(ctx->kflags, ctx->kflagscap, (size_t)ninst * m);
    grow(ctx->kcand, ctx->kcandcap, (size_t)ninst * m * bted::rf::kMaxCand);
    grow(ctx->kncand, ctx->kncandcap, (size_t)ninst * m);
    grow(ctx->knflag, ctx->knflagcap, (size_t)ninst);
    grow(ctx->kforced, ctx->kforcedcap, (size_t)m);
    return ctx->ktop2;
}

// After launch_small(..., top2 = ctx->ktop2): flag near ties of every instance
// (one check launch each, one host sync), then re-score the flagged steps of the
// flagged instances exactly in fp64; a changed pick re-runs that instance with
// the corrected prefix forced.  X: ninst x N x d (device); keys: ninst x m.
// Part 1 (no host sync): the batched near-tie check and an async copy of the
// per-instance flag counts into pinned memory, read by small_k4_refine after
// the caller's next stream synchronisation.
void small_k4_launch(bted_ctx* ctx, cudaStream_t st, int ninst, int64_t N, int32_t d, int32_t m,
                     const unsigned long long* keys) {
    const int nUb = small_units(ninst, N, d);
    if (ctx->k4pincap < (size_t)ninst) {
        if (ctx->k4pin) cudaFreeHost(ctx->k4pin);
        ctx->k4pin = nullptr; ctx->k4pincap = 0;
        CK(cudaHostAlloc(&ctx->k4pin, sizeof(int) * ninst, cudaHostAllocDefault));
        ctx->k4pincap = (size_t)ninst;
    }
    CK(cudaMemsetAsync(ctx->knflag, 0, sizeof(int) * ninst, st));
    bted::rf::neartie_check_kernel<<<dim3(m, ninst), 256, 0, st>>>(ctx->ktop2, nUb, keys, bted::rf::kTau,
                                                                  ctx->kflags, ctx->kcand, ctx->kncand, ctx->knflag);
    LAUNCHED(1);
    CK(cudaMemcpyAsync(ctx->k4pin, ctx->knflag, sizeof(int) * ninst, cudaMemcpyDeviceToHost, st));
}

// Part 2 (after a sync that follows small_k4_launch): re-score the flagged steps of
// the flagged instances in fp64; a changed pick re-runs that instance alone with
// the corrected prefix forced.  Returns true if any pick changed.
bool small_k4_refine(bted_ctx* ctx, cudaStream_t st, const float* X, int ninst, int64_t N, int32_t d, int32_t m,
                     float mu, unsigned long long* keys, int* err) {
    bool any = false;
    for (int k = 0; k < ninst; ++k) any |= ctx->k4pin[k] != 0;
    if (!any) return false;
    const int nUb = small_units(ninst, N, d);
    const int nU1 = small_units(1, N, d);
    const size_t kMC = bted::rf::kMaxCand;
    bool changed = false;
    unsigned long long* rerun_top2 = ctx->ktop2 + (size_t)ninst * m * nUb * 2;
    auto check = [&](int k, const unsigned long long* t2, int nU) {
        bted::rf::neartie_check_kernel<<<m, 256, 0, st>>>(t2, nU, keys + (size_t)k * m,
                                                         bted::rf::kTau, ctx->kflags + (size_t)k * m,
                                                         ctx->kcand + (size_t)k * m * kMC, ctx->kncand + (size_t)k * m,
                                                         ctx->knflag + k);
        LAUNCHED(1);
    };
    std::vector<int> nf(ctx->k4pin, ctx->k4pin + ninst);
    std::vector<unsigned long long> hk(m), forced;
    std::vector<int> fl(m), nc(m);
    std::vector<uint32_t> cd((size_t)m * kMC);
    for (int k = 0; k < ninst; ++k) {
        if (!nf[k]) continue;
        const float* Xk = X + (size_t)k * N * d;
        unsigned long long* kk = keys + (size_t)k * m;
        int checked = -1;
        for (int rounds = 0; rounds <= m; ++rounds) {
            CK(cudaMemcpyAsync(hk.data(), kk, sizeof(unsigned long long) * m, cudaMemcpyDeviceToHost, st));
            CK(cudaMemcpyAsync(fl.data(), ctx->kflags + (size_t)k * m, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
            CK(cudaMemcpyAsync(nc.data(), ctx->kncand + (size_t)k * m, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
            CK(cudaMemcpyAsync(cd.data(), ctx->kcand + (size_t)k * m * kMC, sizeof(uint32_t) * cd.size(),
                               cudaMemcpyDeviceToHost, st));
            CK(cudaStreamSynchronize(st));
            if (!k4_next_correction(ctx, st, Xk, N, d, m, mu, hk, fl, nc, cd, checked, forced)) break;
            changed = true;
            CK(cudaMemcpyAsync(ctx->kforced, forced.data(), sizeof(unsigned long long) * forced.size(),
                               cudaMemcpyHostToDevice, st));
            // the single-instance re-run writes its top-2 to the scratch tail
            launch_small(Xk, 1, N, d, ctx->params.gamma, ctx->kernel, m, mu, kk, err, st, rerun_top2, ctx->kforced,
                         (int)forced.size());
            CK(cudaMemsetAsync(ctx->knflag + k, 0, sizeof(int), st));
            check(k, rerun_top2, nU1);
            CK(cudaStreamSynchronize(st));      // `forced` (pageable) must outlive the copy
        }
    }
    return changed;
}

// Alg. 2 l.1-4 for batches b_begin, b_begin+b_step, ... ; winners on device.
int run_batch_range(bted_ctx* ctx, int64_t M, int32_t m, float mu, int32_t b_begin, int32_t b_step) {
    Nvtx nvtx_("bted batch TEDs (Alg. 2 l.1-4)");
    const int32_t B = ctx->params.num_batches;
    ctx->k4b.pending = false;
    ctx->k4big.pending = false;
    int nb = 0;
    for (int32_t b = b_begin; b < B; b += b_step) ++nb;
    grow(ctx->winners, ctx->winnerscap, (size_t)std::max(nb, 1) * m);
    grow(ctx->mkeys, ctx->mkeyscap, (size_t)m);
    cudaStream_t st = ctx->stream;
    const bool no_graph = (ctx->params.flags & BTED_FLAG_NO_GRAPH) != 0;
    if (nb == 0) return 0;
    // Alg. 2 l.2 for all of this call's batches at once (radix select, sorted V_b)
    grow(ctx->sall, ctx->sallcap, (size_t)nb * M);
    sample_batches_dev(ctx, st, ctx->N, M, b_begin, b_step, nb, ctx->params.seed, ctx->sall);
    if (use_small(ctx->params.flags, M)) {
        // small batches (the paper's M = 500): all batch TEDs in ONE cluster launch
        grow(ctx->xall, ctx->xallcap, (size_t)nb * M * ctx->d);
        grow(ctx->kall, ctx->kallcap, (size_t)nb * m);
        Ted& T = ctx->bted_engine;
        gather(ctx, st, ctx->sall, (int64_t)nb * M, ctx->xall);   // all batches: [nb][M] -> [nb][M][d]
        Ted::Slot* sl = T.timing ? T.next_slot(m) : nullptr;
        if (sl) { sl->small = nb; CK(cudaEventRecord(sl->e[0], st)); }
        unsigned long long* k4t = T.refine ? small_k4_reserve(ctx, nb, M, ctx->d, m) : nullptr;
        launch_small(ctx->xall, nb, M, ctx->d, ctx->params.gamma, ctx->kernel, m, mu, ctx->kall, T.err, st, k4t);
        if (sl) CK(cudaEventRecord(sl->e[1], st));
        if (k4t) {                                       // decided at the caller's next host sync
            small_k4_launch(ctx, st, nb, M, ctx->d, m, ctx->kall);
            ctx->k4b.pending = true;
            ctx->k4b.ninst = nb; ctx->k4b.M = M; ctx->k4b.m = m; ctx->k4b.mu = mu;
        }
        bted::map_winners_batched_kernel<<<dim3((m + 127) / 128, nb), 128, 0, st>>>(ctx->kall, m, ctx->sall, M,
                                                                                    ctx->winners);
        LAUNCHED(1);
        return nb;
    }
    Ted& T = ctx->bted_engine;
    const bool packed = use_packed(ctx->params.flags, ctx->d);
    const bool k4 = T.refine;
    const size_t nC = (size_t)bted::rf::kMaxCand;
    if (k4) {
        grow(ctx->bflag, ctx->bflagcap, (size_t)nb);
        grow(ctx->bkeys, ctx->bkeyscap, (size_t)nb * m);
        grow(ctx->bsflags, ctx->bsflagscap, (size_t)nb * m);
        grow(ctx->bncand, ctx->bncandcap, (size_t)nb * m);
        grow(ctx->bcand, ctx->bcandcap, (size_t)nb * m * nC);
        CK(cudaMemsetAsync(ctx->bflag, 0, sizeof(int) * nb, st));
    }
    for (int k = 0; k < nb; ++k) {
        const uint32_t* idx = ctx->sall + (size_t)k * M;
        gather(ctx, st, idx, M);
        run_ted(T, ctx->Xb, M, ctx->d, ctx->params.gamma, ctx->kernel, m, mu, ctx->mkeys, no_graph, true, packed,
                k4 ? ctx->bflag + k : nullptr, nullptr, 0, k4 ? ctx->bsflags + (size_t)k * m : nullptr,
                k4 ? ctx->bcand + (size_t)k * m * nC : nullptr, k4 ? ctx->bncand + (size_t)k * m : nullptr);
        if (k4)
            CK(cudaMemcpyAsync(ctx->bkeys + (size_t)k * m, ctx->mkeys, sizeof(unsigned long long) * m,
                               cudaMemcpyDeviceToDevice, st));
        bted::map_winners_kernel<<<(m + 127) / 128, 128, 0, st>>>(ctx->mkeys, m, idx, ctx->winners + (size_t)k * m);
        LAUNCHED(1);
    }
    if (k4) {
        // K4 of the batch TEDs, decided at the caller's next host sync (big_k4_resolve):
        // the per-batch near-tie counts go to pinned memory, no sync here
        if (ctx->bfpincap < (size_t)nb) {
            if (ctx->bfpin) cudaFreeHost(ctx->bfpin);
            ctx->bfpin = nullptr; ctx->bfpincap = 0;
            CK(cudaHostAlloc(&ctx->bfpin, sizeof(int) * nb, cudaHostAllocDefault));
            ctx->bfpincap = (size_t)nb;
        }
        CK(cudaMemcpyAsync(ctx->bfpin, ctx->bflag, sizeof(int) * nb, cudaMemcpyDeviceToHost, st));
        ctx->k4big.pending = true;
        ctx->k4big.nb = nb; ctx->k4big.M = M; ctx->k4big.m = m; ctx->k4big.mu = mu;
    }
    return nb;
}

// K4 of the large batch TEDs (after a host sync that follows run_batch_range): the
// near-tie steps of each flagged batch TED are re-scored exactly from its kept
// keys/flags/candidates; a TED is re-run only if a pick changes.  Returns true if
// any batch's winners changed (the union must then be redone).
bool big_k4_resolve(bted_ctx* ctx) {
    if (!ctx->k4big.pending) return false;
    ctx->k4big.pending = false;
    const int nb = ctx->k4big.nb;
    const int64_t M = ctx->k4big.M;
    const int32_t m = ctx->k4big.m;
    const float mu = ctx->k4big.mu;
    Ted& T = ctx->bted_engine;
    cudaStream_t st = ctx->stream;
    const size_t nC = (size_t)bted::rf::kMaxCand;
    const uint64_t corrected0 = ctx->corrected_steps;
    for (int k = 0; k < nb; ++k) {
        if (!ctx->bfpin[k]) continue;
        const uint32_t* idx = ctx->sall + (size_t)k * M;
        gather(ctx, st, idx, M);
        CK(cudaMemcpyAsync(ctx->mkeys, ctx->bkeys + (size_t)k * m, sizeof(unsigned long long) * m,
                           cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(T.flags, ctx->bsflags + (size_t)k * m, sizeof(int) * m, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(T.ncand, ctx->bncand + (size_t)k * m, sizeof(int) * m, cudaMemcpyDeviceToDevice, st));
        CK(cudaMemcpyAsync(T.cand, ctx->bcand + (size_t)k * m * nC, sizeof(uint32_t) * m * nC,
                           cudaMemcpyDeviceToDevice, st));
        refine_ted(ctx, T, ctx->Xb, M, ctx->d, m, mu, ctx->mkeys, nullptr);
        bted::map_winners_kernel<<<(m + 127) / 128, 128, 0, st>>>(ctx->mkeys, m, idx, ctx->winners + (size_t)k * m);
        LAUNCHED(1);
    }
    CK(cudaStreamSynchronize(st));
    return ctx->corrected_steps != corrected0;
}

// After run_batch_range: wait for the batch TEDs, resolve the small-batch K4
// deferred to this sync (ctx->winners updated), check the error words.
bted_status batch_range_finish(bted_ctx* ctx, int nb) {
    *ctx->herr = 0;
    if (nb > 0)
        CK(cudaMemcpyAsync(ctx->herr, ctx->bted_engine.err, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
    CK(cudaStreamSynchronize(ctx->stream));
    ctx->bted_engine.collect();
    big_k4_resolve(ctx);                             // K4 of large batch TEDs (winners updated in place)
    if (ctx->k4b.pending) {                          // K4 of small batch TEDs
        ctx->k4b.pending = false;
        auto& b = ctx->k4b;
        if (small_k4_refine(ctx, ctx->stream, ctx->xall, b.ninst, b.M, ctx->d, b.m, b.mu, ctx->kall,
                            ctx->bted_engine.err)) {
            bted::map_winners_batched_kernel<<<dim3((b.m + 127) / 128, b.ninst), 128, 0, ctx->stream>>>(
                ctx->kall, b.m, ctx->sall, b.M, ctx->winners);
            LAUNCHED(1);
            CK(cudaStreamSynchronize(ctx->stream));
        }
    }
    if (take_xbad(ctx)) return BTED_EINVAL;
    if (nb > 0 && *ctx->herr) {
        CK(cudaMemsetAsync(ctx->bted_engine.err, 0, sizeof(int), ctx->stream));
        set_error((*ctx->herr & bted::kSampleOverflow) ? "batch sampler: candidate bin overflow (internal limit kCandCap)"
                                                     : "non-finite score during a batch TED");
        return BTED_ENUMERIC;
    }
    return BTED_OK;
}

// Alg. 2 l.5-6 on device winners[0..n): returns count, out_idx host [count].
// distinct: the n winners are known to be n distinct valid indices (one batch TED's
// picks), so |X_U| = n without a host round trip
bted_status merge_device(bted_ctx* ctx, const int64_t* winners_dev, int64_t n, int32_t m, float mu,
                         int64_t* out_idx, int32_t* out_count, bool distinct = false) {
    Nvtx nvtx_("bted union + merge (Alg. 2 l.5-6)");
    cudaStream_t st = ctx->stream;
    grow(ctx->u32a, ctx->u32acap, (size_t)n);
    grow(ctx->u32b, ctx->u32bcap, (size_t)n);
    grow(ctx->count_dev, ctx->countcap, 1);
    const unsigned g = (unsigned)std::min<int64_t>((n + 255) / 256, 1024);
    if (!ctx->bted_engine.err) {
        grow(ctx->bted_engine.err, ctx->bted_engine.errcap, 1);
        CK(cudaMemsetAsync(ctx->bted_engine.err, 0, sizeof(int), st));
    }
    if (n <= bted::kUnionMax) {                           // one CTA: sort + unique + drop padding
        bted::union_small_kernel<<<1, bted::kUnionThreads, 0, st>>>(winners_dev, (int)n, ctx->N, ctx->u32a,
                                                                    ctx->count_dev, ctx->bted_engine.err);
        LAUNCHED(1);
    } else {
        bted::i64_to_u32_kernel<<<g, 256, 0, st>>>(winners_dev, n, ctx->N, ctx->u32a, ctx->bted_engine.err);
        LAUNCHED(1);
        size_t need = 0, need2 = 0;
        const int nbits = 32;   // padding (0xFFFFFFFF) must sort last
        CK(cub::DeviceRadixSort::SortKeys(nullptr, need, ctx->u32a, ctx->u32b, (int)n, 0, nbits, st));
        CK(cub::DeviceSelect::Unique(nullptr, need2, ctx->u32b, ctx->u32a, ctx->count_dev, (int)n, st));
        cub_reserve(ctx, std::max(need, need2));
        size_t cap = ctx->cub_cap;
        CK(cub::DeviceRadixSort::SortKeys(ctx->cub_tmp, cap, ctx->u32a, ctx->u32b, (int)n, 0, nbits, st));
        cap = ctx->cub_cap;
        CK(cub::DeviceSelect::Unique(ctx->cub_tmp, cap, ctx->u32b, ctx->u32a, ctx->count_dev, (int)n, st));
        bted::drop_pad_kernel<<<1, 1, 0, st>>>(ctx->u32a, ctx->count_dev);
        LAUNCHED(1);
    }
    int nu = (int)n;
    if (!distinct || ctx->k4b.pending || n > bted::kUnionMax) {
    CK(cudaMemcpyAsync(&nu, ctx->count_dev, sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(ctx->herr, ctx->bted_engine.err, sizeof(int), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));                        // |X_U| sizes the merge TED
    if (*ctx->herr & bted::kBadWinner) {
        CK(cudaMemsetAsync(ctx->bted_engine.err, 0, sizeof(int), st));
        set_error("winner index out of range (>= N)");
        return BTED_EINVAL;
    }
    ctx->bted_engine.collect();
    if (big_k4_resolve(ctx)) {                            // K4 of the large batch TEDs, decided here
        ctx->k4b.changed = true;
        return merge_device(ctx, winners_dev, n, m, mu, out_idx, out_count, distinct);   // the union changed
    }
    if (ctx->k4b.pending) {                               // K4 of the small batch TEDs, decided here
        ctx->k4b.pending = false;
        auto& b = ctx->k4b;
        if (small_k4_refine(ctx, st, ctx->xall, b.ninst, b.M, ctx->d, b.m, b.mu, ctx->kall, ctx->bted_engine.err)) {
            bted::map_winners_batched_kernel<<<dim3((b.m + 127) / 128, b.ninst), 128, 0, st>>>(
                ctx->kall, b.m, ctx->sall, b.M, ctx->winners);
            LAUNCHED(1);
            b.changed = true;
            return merge_device(ctx, winners_dev, n, m, mu, out_idx, out_count, distinct);   // the union changed
        }
    }
    }
    if (nu < 1) { set_error("empty union"); return BTED_ENUMERIC; }
    const int32_t mm = std::min<int32_t>(m, nu);          // reading A12
    gather(ctx, st, ctx->u32a, nu);                       // X[X_U] (A13: fresh Gram)
    grow(ctx->mkeys, ctx->mkeyscap, (size_t)mm);
    grow(ctx->out_dev, ctx->outcap, (size_t)mm);
    if (use_small(ctx->params.flags, nu)) {
        // the merge is small (|X_U| <= B m): one cluster kernel runs all its steps
        Ted& T = ctx->bted_engine;
        if (!T.err) { grow(T.err, T.errcap, 1); CK(cudaMemsetAsync(T.err, 0, sizeof(int), st)); }
        unsigned long long* k4t = T.refine ? small_k4_reserve(ctx, 1, nu, ctx->d, mm) : nullptr;
        launch_small(ctx->Xb, 1, nu, ctx->d, ctx->params.gamma, ctx->kernel, mm, mu, ctx->mkeys, T.err, st, k4t);
        if (k4t) {
            small_k4_launch(ctx, st, 1, nu, ctx->d, mm, ctx->mkeys);
            bted::map_winners_kernel<<<(mm + 127) / 128, 128, 0, st>>>(ctx->mkeys, mm, ctx->u32a, ctx->out_dev);
            LAUNCHED(1);
            bted_status s = finish_keys(ctx, ctx->bted_engine, ctx->mkeys, mm, out_idx, nullptr, ctx->out_dev);
            if (s == BTED_OK && big_k4_resolve(ctx)) {    // (fast path) a batch pick changed: redo l.5-6
                ctx->k4b.changed = true;
                return merge_device(ctx, winners_dev, n, m, mu, out_idx, out_count, distinct);
            }
            if (s == BTED_OK && small_k4_refine(ctx, st, ctx->Xb, 1, nu, ctx->d, mm, mu, ctx->mkeys, T.err)) {
                bted::map_winners_kernel<<<(mm + 127) / 128, 128, 0, st>>>(ctx->mkeys, mm, ctx->u32a,
                                                                         ctx->out_dev);
                LAUNCHED(1);
                s = finish_keys(ctx, ctx->bted_engine, ctx->mkeys, mm, out_idx, nullptr, ctx->out_dev);
            }
            if (s == BTED_OK) *out_count = mm;
            return s;
        }
    } else {
        // size varies with |X_U|: run it eagerly
        run_ted(ctx->bted_engine, ctx->Xb, nu, ctx->d, ctx->params.gamma, ctx->kernel, mm, mu, ctx->mkeys,
                true, /*time_it=*/false, use_packed(ctx->params.flags, ctx->d));
    }
    bted::map_winners_kernel<<<(mm + 127) / 128, 128, 0, st>>>(ctx->mkeys, mm, ctx->u32a, ctx->out_dev);
    LAUNCHED(1);
    bted_status s = finish_keys(ctx, ctx->bted_engine, ctx->mkeys, mm, out_idx, nullptr, ctx->out_dev);
    if (s == BTED_OK && big_k4_resolve(ctx)) {            // (fast path) a batch pick changed: redo l.5-6
        ctx->k4b.changed = true;
        return merge_device(ctx, winners_dev, n, m, mu, out_idx, out_count, distinct);
    }
    if (s == BTED_OK) *out_count = mm;
    return s;
}

}  // namespace

// ------------------------------------------------------------------ row-sharded dense bands (internal)
namespace {
void shard_gram_enqueue(bted_ctx* ctx, float mu, uint64_t* keys_dev) {
    Ted& T = ctx->ted;
    const int64_t rows = ctx->row1 - ctx->row0;
    T.reserve(rows, ctx->N, ctx->d, 2);
    T.last_rows = rows;
    T.last_ld = ld_for(ctx->N);
    T.last_buf = 0;
    launch_transpose(T, ctx->X, ctx->N, ctx->d);
    CK(cudaMemsetAsync(T.sel, 0, (size_t)rows, T.stream));
    // K4: per-CTA top-2 keys of the first kMaxM steps (bted_shard_nearties / bted_shard_refine)
    if (T.refine) T.reserve_refine((rows + kRowsPerK2Cta - 1) / kRowsPerK2Cta * 32, bted::im::kMaxM);
    launch_gram(T, ctx->N, ctx->d, ctx->row0, rows, ctx->params.gamma, ctx->kernel, mu,
                reinterpret_cast<unsigned long long*>(keys_dev), T.refine ? T.top2 : nullptr);
}

void shard_step_enqueue(bted_ctx* ctx, int32_t t, float mu, const float* pivot_dev, uint64_t* keys_dev) {
    Ted& T = ctx->ted;
    const int64_t rows = ctx->row1 - ctx->row0;
    launch_step(T, ctx->N, ctx->row0, rows, t, mu, pivot_dev, reinterpret_cast<unsigned long long*>(keys_dev),
                (T.refine && T.top2 && t < bted::im::kMaxM) ? T.top2 : nullptr);
    T.last_buf = t & 1;
}

void shard_pivot_enqueue(bted_ctx* ctx, int32_t t, const uint64_t* keys_dev, float* col_dev) {
    Ted& T = ctx->ted;
    const int32_t rows = (int32_t)(ctx->row1 - ctx->row0);
    const unsigned g = (unsigned)std::min<int64_t>((rows + 255) / 256, 1024);
    bted::pivot_column_kernel<<<g, 256, 0, T.stream>>>(T.K[t & 1], ld_for(ctx->N), rows,
                                                       reinterpret_cast<const unsigned long long*>(keys_dev), t,
                                                       col_dev);
    LAUNCHED(1);
}

void shard_colnorm_enqueue(bted_ctx* ctx, int32_t t, float mu, const float* pivot_dev,
                           const uint64_t* keys_dev, float* colnorm_dev) {
    Ted& T = ctx->ted;
    const int64_t ld = ld_for(ctx->N);
    const int32_t rows = (int32_t)(ctx->row1 - ctx->row0);
    const int32_t nchunks = (rows + bted::kColChunk - 1) / bted::kColChunk;
    grow(T.P, T.pcap, (size_t)nchunks * (size_t)ld);
    const dim3 grid((unsigned)((ld + 255) / 256), (unsigned)nchunks);
    const auto* keys = reinterpret_cast<const unsigned long long*>(keys_dev);
    if (t == 0)
        bted::deflate_colnorm_kernel<false><<<grid, bted::kColThreads, 0, T.stream>>>(
            T.K[0], nullptr, ld, (int32_t)ctx->row0, rows, nullptr, nullptr, 0, mu, T.sel, T.P);
    else
        bted::deflate_colnorm_kernel<true><<<grid, bted::kColThreads, 0, T.stream>>>(
            T.K[(t - 1) & 1], T.K[t & 1], ld, (int32_t)ctx->row0, rows, pivot_dev, keys, t, mu, T.sel, T.P);
    const unsigned g2 = (unsigned)std::min<int64_t>((ld + 255) / 256, 2048);
    bted::colnorm_reduce_kernel<<<g2, 256, 0, T.stream>>>(T.P, nchunks, ld, colnorm_dev);
    LAUNCHED(2);
    T.last_buf = t & 1;
}

void shard_scores_enqueue(bted_ctx* ctx, int32_t t, float mu, const float* colnorm_dev, uint64_t* keys_dev) {
    Ted& T = ctx->ted;
    const int32_t rows = (int32_t)(ctx->row1 - ctx->row0);
    unsigned g = (unsigned)std::min<int64_t>((rows + 255) / 256, 1184);
    // K4: one CTA per top-2 slot pair of the step (T.last_nC, set by bted_shard_gram),
    // so bted_shard_nearties reads the literal mode's keys like the symmetric mode's
    unsigned long long* top2 = nullptr;
    if (T.refine && T.top2 && t < bted::im::kMaxM && T.last_nC > 0) {
        g = (unsigned)T.last_nC;
        top2 = T.top2 + (int64_t)t * T.last_nC * 2;
    }
    bted::colnorm_scores_kernel<<<g, 256, 0, T.stream>>>(T.K[t & 1], ld_for(ctx->N), (int32_t)ctx->row0, rows,
                                                         colnorm_dev, mu, T.sel,
                                                         reinterpret_cast<unsigned long long*>(keys_dev), t, T.err,
                                                         top2);
    LAUNCHED(1);
}
// K4 for row bands: every band's candidates within tau of the global pick
// (cand_all / ncand_all: host, [nranks][m][kMaxCand] / [nranks][m]; -1 = that
// band's list may be incomplete), merged, then the usual decision on this shard.
bool shard_k4_decide(bted_ctx* ctx, int32_t m, float mu, const unsigned long long* keys_dev, const uint32_t* cand_all,
                     const int32_t* ncand_all, int32_t nranks, std::vector<unsigned long long>& forced) {
    Ted& T = ctx->ted;
    forced.clear();
    if (!T.refine) return false;
    const size_t kMC = bted::rf::kMaxCand;
    std::vector<unsigned long long> hk(m);
    CK(cudaMemcpyAsync(hk.data(), keys_dev, sizeof(unsigned long long) * m, cudaMemcpyDeviceToHost, T.stream));
    CK(cudaStreamSynchronize(T.stream));
    std::vector<int> fl(m, 0), nc(m, 0);
    std::vector<uint32_t> cd((size_t)m * kMC);
    for (int t = 0; t < m; ++t) {
        std::vector<uint32_t> c;
        bool incomplete = false;
        for (int r = 0; r < nranks; ++r) {
            const int n0 = ncand_all[(size_t)r * m + t];
            if (n0 < 0) { incomplete = true; continue; }           // the band's list may miss candidates
            const int n = std::min<int>(n0, (int)kMC);
            for (int q = 0; q < n; ++q) c.push_back(cand_all[((size_t)r * m + t) * kMC + q]);
        }
        std::sort(c.begin(), c.end());
        c.erase(std::unique(c.begin(), c.end()), c.end());
        if (c.size() > kMC) { incomplete = true; c.resize(kMC); }
        fl[t] = incomplete ? bted::rf::kFlagFull : c.size() >= 2 ? bted::rf::kFlagNear : 0;
        nc[t] = (int)c.size();
        std::copy(c.begin(), c.end(), cd.begin() + (size_t)t * kMC);
    }
    int checked = -1;
    return k4_next_correction(ctx, T.stream, ctx->X, ctx->N, ctx->d, m, mu, hk, fl, nc, cd, checked, forced);
}
}  // namespace

// ------------------------------------------------------------------ tile-sharded implicit engine
namespace {
int64_t ishard_local_tiles(const bted_ctx* ctx) {
    const int nT = (int)((ctx->N + bted::pk::T - 1) / bted::pk::T);
    const int64_t all = bted::pk::num_tiles(nT);
    return (all - ctx->srank + ctx->snranks - 1) / ctx->snranks;
}
bted::im::XKern ishard_xk(const bted_ctx* ctx) {
    bted::im::XKern xk;
    xk.X = ctx->X; xk.d = ctx->d; xk.ng = -ctx->params.gamma; xk.linear = ctx->kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    return xk;
}
int64_t ishard_qlen_of(int64_t N) {
    const int64_t NP = (N + bted::pk::T - 1) / bted::pk::T * bted::pk::T;
    return (NP + 255) / 256 * 256;
}

// Alg. 1 l.1 + this shard's part of ||K_:v||^2 into q_dev (on the ctx's device / stream)
void ishard_head_enqueue(bted_ctx* ctx, int32_t m, double* q_dev) {
    Ted& T = ctx->ted;
    const int64_t N = ctx->N, NPa = ishard_qlen_of(N);
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int64_t lt = ishard_local_tiles(ctx);
    ensure_implicit_attrs();
    T.reserve_implicit(N, m, lt);
    ctx->sm_m = m;
    CK(cudaMemsetAsync(T.sel, 0, (size_t)NPa, T.stream));
    CK(cudaMemsetAsync(T.kflag, 0, sizeof(int), T.stream));
    CK(cudaMemsetAsync(T.tctr, 0, sizeof(int) * m, T.stream));
    CK(cudaMemsetAsync(q_dev, 0, sizeof(double) * NPa, T.stream));
    const int lin = ctx->kernel == BTED_KERNEL_LINEAR ? 1 : 0;
    const float g = ctx->params.gamma;
    const int r = ctx->srank, P = ctx->snranks;
    auto k1i = [&](auto kern) {
        kern<<<(unsigned)lt, bted::pk::kConsumers, 0, T.stream>>>(ctx->X, (int32_t)N, ctx->d, g, T.K[0], nT, r, P,
                                                                   (const int*)nullptr);
    };
    if (ctx->d <= 16) {
        if (lin) k1i(bted::pk::gram_tile2_kernel<16, true, 4>); else k1i(bted::pk::gram_tile2_kernel<16, false, 4>);
    } else {
        if (lin) k1i(bted::pk::gram_tile_kernel<32, true>); else k1i(bted::pk::gram_tile_kernel<32, false>);
    }
    bted::im::diag_init_kernel<<<(unsigned)((NPa + 255) / 256), 256, 0, T.stream>>>(ishard_xk(ctx), (int32_t)N,
                                                                                     NPa, T.rd);
    bted::im::tile_pass_kernel<true><<<tile_pass_grid(lt), bted::im::kTPThreads, bted::im::tile_pass_smem_bytes,
                                       T.stream>>>(T.K[0], nT, nullptr, T.P64, T.kflag, T.tctr, 0, 0, r, P);
    bted::im::qpart_kernel<<<(unsigned)std::min<int64_t>((NPa + 255) / 256, 4096), 256, 0, T.stream>>>(
        T.P64, nT, r, P, q_dev);
    LAUNCHED(4);
}

// step t: the new factor column l_t (from keys[t-1]) and this shard's part of K l_t into q_dev
void ishard_step_enqueue(bted_ctx* ctx, int32_t t, float mu, const unsigned long long* keys, double* q_dev) {
    Ted& T = ctx->ted;
    const int64_t N = ctx->N, NPa = ishard_qlen_of(N);
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int nA = (int)(NPa / bted::im::kEllRows);
    const int32_t m = ctx->sm_m;
    bted::im::ell_kernel<<<(unsigned)nA + 1, bted::im::kThreads, 0, T.stream>>>(
        T.K[0], nT, (int32_t)N, T.Lf, NPa, t - 1, T.rd, T.nv, mu, keys, t, T.ell, T.Qc, T.G, m, T.hv, T.sel,
        ishard_xk(ctx));
    bted::im::tile_pass_kernel<false><<<tile_pass_grid(ishard_local_tiles(ctx)), bted::im::kTPThreads,
                                        bted::im::tile_pass_smem_bytes, T.stream>>>(
        T.K[0], nT, T.ell, T.P64, T.kflag, T.tctr + t, (int)(t & 1), 0, ctx->srank, ctx->snranks);
    bted::im::qpart_kernel<<<(unsigned)std::min<int64_t>((NPa + 255) / 256, 4096), 256, 0, T.stream>>>(
        T.P64, nT, ctx->srank, ctx->snranks, q_dev);
    LAUNCHED(3);
}

// scores of step t from the summed q (q_dev) or, with pq, from the devices' partials
void ishard_fin_enqueue(bted_ctx* ctx, int32_t t, float mu, const double* q_dev, unsigned long long* keys,
                        const bted::im::PeerQ* pq = nullptr) {
    Ted& T = ctx->ted;
    const int64_t N = ctx->N, NPa = ishard_qlen_of(N);
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    const int64_t NP = (int64_t)nT * bted::pk::T;
    if (pq)
        bted::im::fin64_peer_kernel<<<(unsigned)(NP / bted::im::kFinRows), bted::im::kThreads, 0, T.stream>>>(
            *pq, nT, (int32_t)N, T.K[0], mu, T.Lf, NPa, t > 0 ? t - 1 : 0, T.hv, T.nv, T.rd, T.sel, keys, t,
            keys + t, T.err, T.refine ? T.top2 : nullptr, T.Qc, t == 0 ? T.rd : nullptr);
    else
        bted::im::fin64_kernel<<<(unsigned)(NP / bted::im::kFinRows), bted::im::kThreads, 0, T.stream>>>(
            T.P64, nT, (int32_t)N, T.K[0], mu, T.Lf, NPa, t > 0 ? t - 1 : 0, T.hv, T.nv, T.rd, T.sel, keys, t,
            keys + t, T.err, T.refine ? T.top2 : nullptr, T.Qc, q_dev, t == 0 ? T.rd : nullptr);
    LAUNCHED(1);
}

// K4 on a tile shard (all shards hold the same keys and reach the same decision):
// true with `forced` = the corrected prefix if a refined pick changes
bool ishard_k4(bted_ctx* ctx, int32_t m, float mu, const unsigned long long* keys,
               std::vector<unsigned long long>& forced) {
    Ted& T = ctx->ted;
    forced.clear();
    if (!T.refine) return false;
    cudaStream_t st = T.stream;
    CK(cudaMemsetAsync(T.nflag, 0, sizeof(int), st));
    bted::rf::neartie_check_kernel<<<m, 256, 0, st>>>(T.top2, T.last_nC, keys, bted::rf::kTau, T.flags, T.cand,
                                                     T.ncand, T.nflag);
    LAUNCHED(1);
    std::vector<unsigned long long> hk(m);
    std::vector<int> fl(m), nc(m);
    std::vector<uint32_t> cd((size_t)m * bted::rf::kMaxCand);
    CK(cudaMemcpyAsync(hk.data(), keys, sizeof(unsigned long long) * m, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(fl.data(), T.flags, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(nc.data(), T.ncand, sizeof(int) * m, cudaMemcpyDeviceToHost, st));
    CK(cudaMemcpyAsync(cd.data(), T.cand, sizeof(uint32_t) * cd.size(), cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
    int checked = -1;
    return k4_next_correction(ctx, st, ctx->X, ctx->N, ctx->d, m, mu, hk, fl, nc, cd, checked, forced);
}
}  // namespace

// ------------------------------------------------------------------ multi-GPU (num_devices > 1)
// One ctx drives G = P devices [device, device + G) from one process (SURVEY
// 8(e)): bted_run_batches sends batch b to device b mod G (replica ctxs, one
// host thread each: the batches are independent, Alg. 2 l.1-4);
// bted_select tile-shards one candidate set (the implicit engine's packed Gram
// tiles k = p mod P on device p; X and the O(N m) fp64 state replicated).  Per
// step the only exchange is the sum of the P partial q = K l vectors: by
// default each device publishes its partial (a release flag in its memory)
// and every device's score kernel (fin64_peer_kernel) sums all P partials
// through peer loads in rank order -- the all-reduce fused into its consumer,
// bitwise the same on every device; BTED_FLAG_NCCL uses ncclAllReduce instead.
// BTED_FLAG_LOOPBACK runs the P shards / G replicas as logical devices on one
// GPU and one stream (the same control flow and kernels; tests).
namespace {

struct NcclApi {
    bool ok = false;
    std::string why;
    ncclResult_t (*CommInitAll)(ncclComm_t*, int, const int*) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
    ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
};
// libnccl.so.2 at run time: the process's already-loaded NCCL (e.g. torch's) if any
NcclApi& nccl_api() {
    static NcclApi a;
    static std::once_flag once;
    std::call_once(once, [] {
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) { a.why = std::string("dlopen(libnccl.so.2): ") + dlerror(); return; }
        auto sym = [&](auto& f, const char* name) { f = reinterpret_cast<std::remove_reference_t<decltype(f)>>(dlsym(h, name)); return f != nullptr; };
        a.ok = sym(a.CommInitAll, "ncclCommInitAll") && sym(a.AllReduce, "ncclAllReduce") &&
               sym(a.GroupStart, "ncclGroupStart") && sym(a.GroupEnd, "ncclGroupEnd") &&
               sym(a.CommGetAsyncError, "ncclCommGetAsyncError") && sym(a.CommAbort, "ncclCommAbort") &&
               sym(a.CommDestroy, "ncclCommDestroy") && sym(a.GetErrorString, "ncclGetErrorString");
        if (!a.ok) a.why = "libnccl.so.2 lacks a required symbol";
    });
    return a;
}
#define NK(expr)                                                                          \
    do {                                                                                  \
        ncclResult_t _r = (expr);                                                         \
        if (_r != ncclSuccess)                                                            \
            throw NcclError{std::string("NCCL ") + nccl_api().GetErrorString(_r) + " in " + #expr}; \
    } while (0)

}  // namespace

struct MultiDev {
    int P = 1;
    bool loopback = false, use_nccl = false;
    std::vector<int> dev;
    std::vector<bted_ctx*> sub;                    // select: tile shards (rank p on dev[p])
    std::vector<bted_ctx*> rep;                    // run_batches: replicas on dev[1..G) (rep[0] unused: the ctx)
    std::vector<double*> qbuf;                     // [P] 2 qlen fp64 (ping-pong by step parity) on dev[p]
    std::vector<double*> qsum;                     // [P] NCCL: the all-reduced q
    std::vector<unsigned long long*> flag;         // [P] publish counters on dev[p]
    std::vector<ncclComm_t> comms;
    int64_t qlen = 0;
    unsigned long long seq = 0;                    // last published counter value
    unsigned long long timeout_ns = 20000000000ull;   // peer flag wait (BTED_PEER_TIMEOUT_MS)
    int drop_publish = -1;                         // debug (BTED_DEBUG_DROP_PUBLISH): never publish on dev p
    int64_t* wall = nullptr; size_t wallcap = 0;   // all batches' winners on dev[0]
    // row bands (BTED_FLAG_DENSE): shard ctxs and their exchange buffers, all on dev[p]
    std::vector<bted_ctx*> band;
    std::vector<unsigned long long*> bkeys;        // [m] keys (band max, then the global max)
    std::vector<float*> col, piv, cn, cns;          // column slice [Bw], pivot [W], partial / summed norms [ld]
    std::vector<unsigned long long*> scratch;
    std::vector<uint32_t*> cand;
    std::vector<int*> ncand;
    int64_t Bw = 0, W = 0, ld = 0;
    int32_t band_m = 0;
};

namespace {

// the shards / replicas and their exchange buffers (re-created lazily, e.g. after bted_update)
void md_drop_replicas(MultiDev* md) {
    for (int p = 0; p < (int)md->band.size(); ++p) {
        DeviceGuard dg(md->dev[p]);
        for (void* q : {(void*)md->bkeys[p], (void*)md->col[p], (void*)md->piv[p], (void*)md->cn[p],
                        (void*)md->cns[p], (void*)md->scratch[p], (void*)md->cand[p], (void*)md->ncand[p]})
            if (q) cudaFree(q);
        bted_destroy(md->band[p]);
    }
    md->band.clear(); md->bkeys.clear(); md->col.clear(); md->piv.clear(); md->cn.clear(); md->cns.clear();
    md->scratch.clear(); md->cand.clear(); md->ncand.clear();
    md->band_m = 0;
    for (auto* c : md->sub) bted_destroy(c);
    for (auto* c : md->rep) if (c) bted_destroy(c);
    md->sub.clear();
    md->rep.clear();
    for (int p = 0; p < (int)md->qbuf.size(); ++p) {
        DeviceGuard dg(md->dev[p]);
        if (md->qbuf[p]) cudaFree(md->qbuf[p]);
        if (p < (int)md->qsum.size() && md->qsum[p]) cudaFree(md->qsum[p]);
        if (md->flag[p]) cudaFree(md->flag[p]);
    }
    md->qbuf.clear();
    md->qsum.clear();
    md->flag.clear();
    md->seq = 0;
    if (!md->comms.empty() && nccl_api().ok)
        for (auto c : md->comms) nccl_api().CommDestroy(c);
    md->comms.clear();
}

void md_release(MultiDev* md) {
    if (!md) return;
    md_drop_replicas(md);
    if (md->wall) { DeviceGuard dg(md->dev[0]); cudaFree(md->wall); }
    delete md;
}

// the ctx's G devices: validated, peer access enabled between every pair
bted_status md_init(bted_ctx* ctx) {
    const int G = std::max(1, ctx->params.num_devices);
    auto* md = new MultiDev();
    md->P = G;
    md->loopback = (ctx->params.flags & BTED_FLAG_LOOPBACK) != 0;
    md->use_nccl = (ctx->params.flags & BTED_FLAG_NCCL) != 0;
    if (const char* e = std::getenv("BTED_PEER_TIMEOUT_MS")) md->timeout_ns = (unsigned long long)(std::atof(e) * 1e6);
    if (const char* e = std::getenv("BTED_DEBUG_DROP_PUBLISH")) md->drop_publish = std::atoi(e);
    ctx->md = md;
    if (G > bted::im::kMaxDev) { set_error("num_devices must be <= %d", bted::im::kMaxDev); return BTED_EINVAL; }
    if (md->loopback && md->use_nccl) { set_error("BTED_FLAG_NCCL needs distinct devices (not LOOPBACK)"); return BTED_EINVAL; }
    int ndev = 0;
    CK(cudaGetDeviceCount(&ndev));
    for (int p = 0; p < G; ++p) md->dev.push_back(md->loopback ? ctx->device : ctx->device + p);
    if (!md->loopback && ctx->device + G > ndev) {
        set_error("num_devices %d from device %d: only %d devices visible", G, ctx->device, ndev);
        return BTED_EINVAL;
    }
    if (!md->loopback) {
        for (int a = 0; a < G; ++a) {
            DeviceGuard dg(md->dev[a]);
            for (int b = 0; b < G; ++b) {
                if (a == b) continue;
                int can = 0;
                CK(cudaDeviceCanAccessPeer(&can, md->dev[a], md->dev[b]));
                if (!can && !md->use_nccl) {
                    set_error("device %d cannot access device %d (no P2P): use BTED_FLAG_NCCL", md->dev[a], md->dev[b]);
                    return BTED_ECUDA;
                }
                if (can) {
                    cudaError_t e = cudaDeviceEnablePeerAccess(md->dev[b], 0);
                    if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) CK(e);
                    cudaGetLastError();
                }
            }
        }
    }
    return BTED_OK;
}

// a ctx on dev[p] with its own copy of X (loopback: adopts the ctx's X and shares its stream)
bted_ctx* md_replica(bted_ctx* ctx, int p) {
    MultiDev& md = *ctx->md;
    bted_params q = ctx->params;
    q.device = md.dev[p];
    q.num_devices = 1;
    q.flags &= ~(uint32_t)(BTED_FLAG_LOOPBACK | BTED_FLAG_NCCL);
    float* X = ctx->X;
    bool own = false;
    if (md.loopback) {
        q.stream = reinterpret_cast<uintptr_t>(ctx->stream);
    } else {
        q.stream = 0;
        DeviceGuard dg(md.dev[p]);
        CK(cudaMalloc(&X, sizeof(float) * ctx->N * ctx->d));
        CK(cudaMemcpyPeer(X, md.dev[p], ctx->X, ctx->device, sizeof(float) * ctx->N * ctx->d));
        own = true;
    }
    q.x_on_device = 1;
    bted_ctx* r = nullptr;
    const bted_status st = create_common(X, ctx->N, ctx->d, ctx->kernel, &q, 0, ctx->N, false, &r);
    if (st != BTED_OK) {
        if (own) { DeviceGuard dg(md.dev[p]); cudaFree(X); }
        throw CudaError{cudaErrorUnknown, "replica context creation"};
    }
    r->own_X = own;
    return r;
}

void md_sync_all(MultiDev& md, const std::vector<bted_ctx*>& cs) {
    for (size_t p = 0; p < cs.size(); ++p) {
        DeviceGuard dg(md.dev[p]);
        CK(cudaStreamSynchronize(cs[p]->stream));
    }
}

// NCCL: wait for every stream with a deadline, polling the communicators' async errors
void md_nccl_wait(MultiDev& md) {
    double limit = 300.0;
    if (const char* e = std::getenv("BTED_NCCL_TIMEOUT_S")) limit = std::atof(e);
    const auto t0 = std::chrono::steady_clock::now();
    for (;;) {
        bool done = true;
        for (int p = 0; p < md.P; ++p) {
            DeviceGuard dg(md.dev[p]);
            const cudaError_t q = cudaStreamQuery(md.sub[p]->stream);
            if (q == cudaErrorNotReady) done = false;
            else if (q != cudaSuccess) CK(q);
            ncclResult_t ar = ncclSuccess;
            NK(nccl_api().CommGetAsyncError(md.comms[p], &ar));
            if (ar != ncclSuccess) {
                for (auto c : md.comms) nccl_api().CommAbort(c);
                md.comms.clear();
                throw NcclError{std::string("NCCL async error: ") + nccl_api().GetErrorString(ar)};
            }
        }
        if (done) return;
        const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (el > limit) {
            for (auto c : md.comms) nccl_api().CommAbort(c);
            md.comms.clear();
            throw NcclError{"NCCL collective did not complete within BTED_NCCL_TIMEOUT_S; communicators aborted"};
        }
        std::this_thread::sleep_for(std::chrono::microseconds(200));
    }
}

// TED(V, mu, m) tile-sharded over the P devices; keys of every shard end identical.
void md_select_loop(bted_ctx* ctx, int32_t m, float mu, const std::vector<unsigned long long>* forced) {
    MultiDev& md = *ctx->md;
    const int P = md.P;
    const int64_t NPa = md.qlen;
    auto pq_of = [&](int slot, unsigned long long expect) {
        bted::im::PeerQ pq{};
        pq.P = P;
        pq.expect = expect;
        pq.timeout_ns = md.timeout_ns;
        for (int p = 0; p < P; ++p) { pq.q[p] = md.qbuf[p] + (size_t)slot * NPa; pq.flag[p] = md.flag[p]; }
        return pq;
    };
    auto exchange = [&](int slot) {                 // after every device enqueued its partial into `slot`
        if (md.use_nccl) {
            NK(nccl_api().GroupStart());
            for (int p = 0; p < P; ++p)
                NK(nccl_api().AllReduce(md.qbuf[p] + (size_t)slot * NPa, md.qsum[p], (size_t)NPa, ncclFloat64, ncclSum,
                                        md.comms[p], md.sub[p]->stream));
            NK(nccl_api().GroupEnd());
            return 0ull;
        }
        const unsigned long long e = ++md.seq;
        for (int p = 0; p < P; ++p) {
            if (p == md.drop_publish) continue;         // debug: a device that stopped (tests the timeout)
            DeviceGuard dg(md.dev[p]);
            bted::im::publish_kernel<<<1, 1, 0, md.sub[p]->stream>>>(md.flag[p], e);
            LAUNCHED(1);
        }
        return e;
    };
    auto fin = [&](int32_t t, int slot, unsigned long long e) {
        const bted::im::PeerQ pq = pq_of(slot, e);
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted_ctx* c = md.sub[p];
            ishard_fin_enqueue(c, t, mu, md.use_nccl ? md.qsum[p] : nullptr, c->ted.keys, md.use_nccl ? nullptr : &pq);
        }
    };
    for (int p = 0; p < P; ++p) {
        DeviceGuard dg(md.dev[p]);
        bted_ctx* c = md.sub[p];
        CK(cudaMemsetAsync(c->ted.keys, 0, sizeof(unsigned long long) * m, c->stream));
        if (forced && !forced->empty())
            CK(cudaMemcpyAsync(c->ted.keys, forced->data(), sizeof(unsigned long long) * forced->size(),
                               cudaMemcpyHostToDevice, c->stream));
        ishard_head_enqueue(c, m, md.qbuf[p]);                     // slot 0
    }
    fin(0, 0, exchange(0));
    for (int32_t t = 1; t < m; ++t) {
        const int slot = t & 1;
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted_ctx* c = md.sub[p];
            ishard_step_enqueue(c, t, mu, c->ted.keys, md.qbuf[p] + (size_t)slot * NPa);
        }
        fin(t, slot, exchange(slot));
    }
    if (md.use_nccl) md_nccl_wait(md);
    else md_sync_all(md, md.sub);
}

bted_status md_select_bands(bted_ctx* ctx, int32_t m, float mu, int64_t* out_idx, float* out_score);

bted_status md_select(bted_ctx* ctx, int32_t m, float mu, int64_t* out_idx, float* out_score) {
    Nvtx nvtx_("bted multi-GPU select");
    MultiDev& md = *ctx->md;
    const int P = md.P;
    if (ctx->d > 32) { set_error("multi-GPU select needs d <= 32"); return BTED_EINVAL; }
    if (m > bted::im::kMaxM) { set_error("multi-GPU select needs m <= %d", bted::im::kMaxM); return BTED_EINVAL; }
    if ((ctx->params.flags & BTED_FLAG_DENSE) || ctx->params.norm_mode == 1)
        return md_select_bands(ctx, m, mu, out_idx, out_score);
    const int nT = (int)((ctx->N + bted::pk::T - 1) / bted::pk::T);
    if (bted::pk::num_tiles(nT) < P) { set_error("fewer Gram tiles than devices"); return BTED_EINVAL; }
    if (md.sub.empty()) {
        md.qlen = ishard_qlen_of(ctx->N);
        for (int p = 0; p < P; ++p) {
            bted_ctx* c = md_replica(ctx, p);
            c->is_ishard = true;
            c->srank = p;
            c->snranks = P;
            md.sub.push_back(c);
            DeviceGuard dg(md.dev[p]);
            double* q = nullptr;
            unsigned long long* f = nullptr;
            CK(cudaMalloc(&q, sizeof(double) * 2 * md.qlen));
            CK(cudaMalloc(&f, sizeof(unsigned long long)));
            CK(cudaMemset(f, 0, sizeof(unsigned long long)));
            md.qbuf.push_back(q);
            md.flag.push_back(f);
            if (md.use_nccl) {
                double* r = nullptr;
                CK(cudaMalloc(&r, sizeof(double) * md.qlen));
                md.qsum.push_back(r);
            }
        }
        if (md.use_nccl) {
            if (!nccl_api().ok) throw NcclError{"BTED_FLAG_NCCL: " + nccl_api().why};
            md.comms.resize(P);
            NK(nccl_api().CommInitAll(md.comms.data(), P, md.dev.data()));
        }
    }
    for (int p = 0; p < P; ++p) {
        DeviceGuard dg(md.dev[p]);
        grow(md.sub[p]->ted.keys, md.sub[p]->ted.keyscap, (size_t)m);
    }
    md_select_loop(ctx, m, mu, nullptr);
    // K4: every shard holds the same keys and features; shard 0 decides, all re-run
    std::vector<float> fixed(m, -1.f);
    bted_ctx* c0 = md.sub[0];
    for (int rounds = 0; rounds <= m; ++rounds) {
        std::vector<unsigned long long> forced;
        DeviceGuard dg(md.dev[0]);
        if (!ishard_k4(c0, m, mu, c0->ted.keys, forced)) break;
        md_select_loop(ctx, m, mu, &forced);
    }
    for (int p = 1; p < P; ++p) {                 // a peer's numeric error / stall surfaces here
        DeviceGuard dg(md.dev[p]);
        CK(cudaMemcpy(ctx->herr, md.sub[p]->ted.err, sizeof(int), cudaMemcpyDeviceToHost));
        if (*ctx->herr & bted::im::kErrPeerTimeout) {
            ctx->poisoned = true;
            set_error("multi-GPU exchange: a peer device never published its step (20 s flag wait)");
            return BTED_ENCCL;
        }
        if (*ctx->herr) { set_error("non-finite score on device %d", md.dev[p]); return BTED_ENUMERIC; }
    }
    DeviceGuard dg(md.dev[0]);
    const bted_status st = finish_keys(c0, c0->ted, c0->ted.keys, m, out_idx, out_score);
    if (st != BTED_OK && c0->poisoned) ctx->poisoned = true;
    return st;
}

// Row bands over the P devices (BTED_FLAG_DENSE): band p = rows [p Bw, (p+1) Bw)
// of the dense K on dev[p].  Per step (Alg. 1 l.3-5): the pivot column slices
// are published and gathered into every device's pivot row (bit-symmetry: column
// s = row s), the band deflates and scores, the band maxima are published and
// max-reduced.  norm_mode 1 (literal) adds the published partial column norms,
// summed in rank order.  Bitwise the same as a dense single-GPU select in the
// symmetric mode (every row's arithmetic depends on N only).
void md_band_setup(bted_ctx* ctx, int32_t m) {
    MultiDev& md = *ctx->md;
    const int P = md.P;
    if (!md.band.empty() && md.band_m >= m) return;
    md_drop_replicas(&md);                       // (re)build: the keys / candidate buffers are sized by m
    const int64_t N = ctx->N;
    md.Bw = (N + P - 1) / P;
    md.ld = ld_for(N);
    md.W = std::max<int64_t>(md.ld, (int64_t)P * md.Bw);
    for (int p = 0; p < P; ++p) {
        bted_params q = ctx->params;
        q.device = md.dev[p];
        q.num_devices = 1;
        q.flags &= ~(uint32_t)(BTED_FLAG_LOOPBACK | BTED_FLAG_NCCL);
        float* X = ctx->X;
        bool own = false;
        DeviceGuard dg(md.dev[p]);
        if (md.loopback) {
            q.stream = reinterpret_cast<uintptr_t>(ctx->stream);
        } else {
            q.stream = 0;
            CK(cudaMalloc(&X, sizeof(float) * N * ctx->d));
            CK(cudaMemcpyPeer(X, md.dev[p], ctx->X, ctx->device, sizeof(float) * N * ctx->d));
            own = true;
        }
        q.x_on_device = 1;
        const int64_t r0 = std::min<int64_t>(N, p * md.Bw), r1 = std::min<int64_t>(N, (p + 1) * md.Bw);
        if (r0 >= r1) throw CudaError{cudaErrorInvalidValue, "row bands: more devices than rows"};
        bted_ctx* c = nullptr;
        if (create_common(X, N, ctx->d, ctx->kernel, &q, r0, r1, true, &c) != BTED_OK) {
            if (own) cudaFree(X);
            throw CudaError{cudaErrorUnknown, "band context creation"};
        }
        c->own_X = own;
        md.band.push_back(c);
        unsigned long long* k = nullptr; float* a = nullptr; float* b = nullptr; float* e = nullptr; float* f = nullptr;
        unsigned long long* sc = nullptr; uint32_t* cd = nullptr; int* nc = nullptr;
        CK(cudaMalloc(&k, sizeof(unsigned long long) * m));
        CK(cudaMalloc(&a, sizeof(float) * md.Bw));
        CK(cudaMemset(a, 0, sizeof(float) * md.Bw));
        CK(cudaMalloc(&b, sizeof(float) * md.W));
        CK(cudaMemset(b, 0, sizeof(float) * md.W));
        CK(cudaMalloc(&e, sizeof(float) * md.W));
        CK(cudaMemset(e, 0, sizeof(float) * md.W));
        CK(cudaMalloc(&f, sizeof(float) * md.W));
        CK(cudaMemset(f, 0, sizeof(float) * md.W));
        CK(cudaMalloc(&sc, sizeof(unsigned long long)));
        CK(cudaMalloc(&cd, sizeof(uint32_t) * m * bted::rf::kMaxCand));
        CK(cudaMalloc(&nc, sizeof(int) * m));
        md.bkeys.push_back(k); md.col.push_back(a); md.piv.push_back(b); md.cn.push_back(e); md.cns.push_back(f);
        md.scratch.push_back(sc); md.cand.push_back(cd); md.ncand.push_back(nc);
        if (md.flag.size() < (size_t)P) {
            unsigned long long* fl = nullptr;
            CK(cudaMalloc(&fl, sizeof(unsigned long long)));
            CK(cudaMemset(fl, 0, sizeof(unsigned long long)));
            md.flag.push_back(fl);
            md.qbuf.push_back(nullptr);
        }
    }
    md.band_m = m;
}

void md_band_loop(bted_ctx* ctx, int32_t m, float mu, bool literal, const std::vector<unsigned long long>* forced) {
    MultiDev& md = *ctx->md;
    const int P = md.P;
    auto peers = [&](auto bufs, unsigned long long e) {
        bted::xg::Peers pk{};
        pk.P = P;
        pk.expect = e;
        pk.timeout_ns = md.timeout_ns;
        for (int p = 0; p < P; ++p) { pk.buf[p] = bufs[p]; pk.flag[p] = md.flag[p]; }
        return pk;
    };
    auto publish = [&]() {
        const unsigned long long e = ++md.seq;
        for (int p = 0; p < P; ++p) {
            if (p == md.drop_publish) continue;
            DeviceGuard dg(md.dev[p]);
            bted::im::publish_kernel<<<1, 1, 0, md.band[p]->stream>>>(md.flag[p], e);
            LAUNCHED(1);
        }
        return e;
    };
    auto keymax = [&](int32_t t, unsigned long long e) {
        const bted::xg::Peers pk = peers(md.bkeys, e);
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted::xg::keymax_kernel<<<1, 32, 0, md.band[p]->stream>>>(pk, t, md.bkeys[p], md.band[p]->ted.err);
            LAUNCHED(1);
        }
    };
    auto sum_scores = [&](int32_t t, unsigned long long e) {
        const bted::xg::Peers pk = peers(md.cn, e);
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted_ctx* c = md.band[p];
            bted::xg::sum_colnorm_kernel<<<(unsigned)std::min<int64_t>((md.ld + 255) / 256, 1024), 256, 0, c->stream>>>(
                pk, md.ld, md.cns[p], c->ted.err);
            LAUNCHED(1);
            shard_scores_enqueue(c, t, mu, md.cns[p], reinterpret_cast<uint64_t*>(md.bkeys[p]));
        }
    };
    for (int p = 0; p < P; ++p) {
        DeviceGuard dg(md.dev[p]);
        bted_ctx* c = md.band[p];
        CK(cudaMemsetAsync(md.bkeys[p], 0, sizeof(unsigned long long) * m, c->stream));
        if (forced && !forced->empty())
            CK(cudaMemcpyAsync(md.bkeys[p], forced->data(), sizeof(unsigned long long) * forced->size(),
                               cudaMemcpyHostToDevice, c->stream));
        if (literal) {
            shard_gram_enqueue(c, mu, reinterpret_cast<uint64_t*>(md.scratch[p]));
            shard_colnorm_enqueue(c, 0, mu, nullptr, nullptr, md.cn[p]);
        } else {
            shard_gram_enqueue(c, mu, reinterpret_cast<uint64_t*>(md.bkeys[p]));
        }
    }
    unsigned long long e = publish();
    if (literal) { sum_scores(0, e); e = publish(); }
    keymax(0, e);
    for (int32_t t = 1; t < m; ++t) {
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            shard_pivot_enqueue(md.band[p], t - 1, reinterpret_cast<uint64_t*>(md.bkeys[p]), md.col[p]);
        }
        e = publish();
        const bted::xg::Peers pc = peers(md.col, e);
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted_ctx* c = md.band[p];
            bted::xg::gather_pivot_kernel<<<(unsigned)std::min<int64_t>((md.W + 255) / 256, 1024), 256, 0, c->stream>>>(
                pc, md.Bw, ctx->N, md.W, md.piv[p], c->ted.err);
            LAUNCHED(1);
            if (literal) shard_colnorm_enqueue(c, t, mu, md.piv[p], reinterpret_cast<uint64_t*>(md.bkeys[p]), md.cn[p]);
            else shard_step_enqueue(c, t, mu, md.piv[p], reinterpret_cast<uint64_t*>(md.bkeys[p]));
        }
        e = publish();
        if (literal) { sum_scores(t, e); e = publish(); }
        keymax(t, e);
    }
    std::vector<bted_ctx*> cs(md.band.begin(), md.band.end());
    md_sync_all(md, cs);
}

bted_status md_select_bands(bted_ctx* ctx, int32_t m, float mu, int64_t* out_idx, float* out_score) {
    MultiDev& md = *ctx->md;
    const int P = md.P;
    const bool literal = ctx->params.norm_mode == 1;
    if (md.use_nccl) { set_error("row bands exchange through peer memory (BTED_FLAG_NCCL: tile-sharded engine only)"); return BTED_EINVAL; }
    if (ctx->N < P) { set_error("row bands: more devices than rows"); return BTED_EINVAL; }
    md_band_setup(ctx, m);
    md_band_loop(ctx, m, mu, literal, nullptr);
    bted_ctx* c0 = md.band[0];
    const size_t kMC = bted::rf::kMaxCand;
    const int mm = std::min<int32_t>(m, bted::im::kMaxM);
    for (int rounds = 0; c0->ted.refine && rounds <= m; ++rounds) {    // K4 over the bands' candidates
        std::vector<uint32_t> ca((size_t)P * m * kMC, 0u);
        std::vector<int32_t> na((size_t)P * m, 0);
        for (int p = 0; p < P; ++p) {
            DeviceGuard dg(md.dev[p]);
            bted_ctx* c = md.band[p];
            CK(cudaMemsetAsync(md.ncand[p], 0, sizeof(int) * m, c->stream));
            if (c->ted.top2) {
                bted::rf::shard_neartie_kernel<<<mm, 256, 0, c->stream>>>(c->ted.top2, c->ted.last_nC, md.bkeys[p],
                                                                        bted::rf::kTau, md.cand[p], md.ncand[p]);
                LAUNCHED(1);
            }
            CK(cudaMemcpyAsync(ca.data() + (size_t)p * m * kMC, md.cand[p], sizeof(uint32_t) * m * kMC,
                               cudaMemcpyDeviceToHost, c->stream));
            CK(cudaMemcpyAsync(na.data() + (size_t)p * m, md.ncand[p], sizeof(int) * m, cudaMemcpyDeviceToHost,
                               c->stream));
            CK(cudaStreamSynchronize(c->stream));
        }
        std::vector<unsigned long long> forced;
        DeviceGuard dg(md.dev[0]);
        if (!shard_k4_decide(c0, m, mu, md.bkeys[0], ca.data(), na.data(), P, forced)) break;
        md_band_loop(ctx, m, mu, literal, &forced);
    }
    for (int p = 1; p < P; ++p) {
        DeviceGuard dg(md.dev[p]);
        CK(cudaMemcpy(ctx->herr, md.band[p]->ted.err, sizeof(int), cudaMemcpyDeviceToHost));
        if (*ctx->herr & bted::im::kErrPeerTimeout) {
            ctx->poisoned = true;
            set_error("multi-GPU exchange: a peer device never published its step (flag wait timed out)");
            return BTED_ENCCL;
        }
        if (*ctx->herr) { set_error("non-finite score on device %d", md.dev[p]); return BTED_ENUMERIC; }
    }
    DeviceGuard dg(md.dev[0]);
    const bted_status st = finish_keys(c0, c0->ted, md.bkeys[0], m, out_idx, out_score);
    if (st != BTED_OK && c0->poisoned) ctx->poisoned = true;
    return st;
}

// Alg. 2 with batch b on device b mod G: one host thread per device runs its
// batches (replica ctx; device 0 = this ctx), then the merge on device 0.
bted_status md_run_batches(bted_ctx* ctx, int64_t M, int32_t m, float mu, int64_t* out_idx, int32_t* out_count,
                           int64_t* out_batch_idx) {
    Nvtx nvtx_("bted multi-GPU run_batches");
    MultiDev& md = *ctx->md;
    const int G = md.P, B = ctx->params.num_batches;
    if (md.rep.empty()) {
        md.rep.assign(G, nullptr);
        for (int p = 1; p < G; ++p) md.rep[p] = md_replica(ctx, p);
    }
    std::vector<bted_status> st(G, BTED_OK);
    std::vector<std::string> msg(G);
    std::vector<int> nbs(G, 0);
    auto work = [&](int p) {
        bted_ctx* c = p == 0 ? ctx : md.rep[p];
        st[p] = guarded(c, [&]() -> bted_status {
            nbs[p] = run_batch_range(c, M, m, mu, p, G);
            return batch_range_finish(c, nbs[p]);
        });
        if (st[p] != BTED_OK) msg[p] = bted_last_error();
    };
    if (md.loopback) {
        for (int p = 0; p < G; ++p) work(p);       // one stream: the replicas run in turn
    } else {
        std::vector<std::thread> th;
        for (int p = 1; p < G; ++p) th.emplace_back(work, p);
        work(0);
        for (auto& t : th) t.join();
    }
    for (int p = 0; p < G; ++p)
        if (st[p] != BTED_OK) { set_error("device %d: %s", md.dev[p], msg[p].c_str()); return st[p]; }
    // l.5 exchange: every batch's winners to device 0, in batch order (b = p + k G)
    grow(md.wall, md.wallcap, (size_t)B * m);
    for (int p = 0; p < G; ++p) {
        bted_ctx* c = p == 0 ? ctx : md.rep[p];
        for (int k = 0; k < nbs[p]; ++k) {
            const int b = p + k * G;
            CK(cudaMemcpyPeerAsync(md.wall + (size_t)b * m, md.dev[0], c->winners + (size_t)k * m, md.dev[p],
                                   sizeof(int64_t) * m, ctx->stream));
        }
    }
    if (out_batch_idx) {
        CK(cudaMemcpyAsync(out_batch_idx, md.wall, sizeof(int64_t) * (size_t)B * m, cudaMemcpyDeviceToHost,
                           ctx->stream));
    }
    return merge_device(ctx, md.wall, (int64_t)B * m, m, mu, out_idx, out_count, B == 1);
}

}  // namespace

// ======================================================================= ABI
extern "C" {

void bted_default_params(bted_params* p) {
    if (!p) return;
    std::memset(p, 0, sizeof *p);
    p->gamma = 1.0f;
    p->device = -1;
    p->num_batches = 1;
    p->num_devices = 1;
    p->norm_mode = 0;
}

bted_status bted_create(const float* X, int64_t N, int32_t d, bted_kernel kernel, const bted_params* params,
                        bted_ctx** out) {
    bted_status st = create_common(X, N, d, kernel, params, 0, N, false, out);
    if (st != BTED_OK || (params->num_devices <= 1 && !(params->flags & BTED_FLAG_NCCL))) return st;
    st = guarded(*out, [&]() { return md_init(*out); });
    if (st != BTED_OK) {
        const std::string why = bted_last_error();
        bted_destroy(*out);
        *out = nullptr;
        set_error("%s", why.c_str());
    }
    return st;
}

bted_status bted_shard_create(const float* X, int64_t N, int32_t d, bted_kernel kernel, int64_t row0,
                              int64_t row1, const bted_params* params, bted_ctx** out) {
    return create_common(X, N, d, kernel, params, row0, row1, true, out);
}

bted_status bted_select(bted_ctx* ctx, int32_t m, float mu, int64_t* out_idx, float* out_score) {
    Nvtx nvtx_("bted_select (Alg. 1)");
    if (!ctx || !out_idx) { set_error("null argument"); return BTED_EINVAL; }
    if (ctx->is_shard || ctx->is_ishard) { set_error("bted_select on a shard context"); return BTED_EINVAL; }
    if (m < 1 || m > ctx->N || !mu_ok(mu)) { set_error("need 1 <= m <= N and mu > 0 finite"); return BTED_EINVAL; }
    // several devices: shard the candidate set -- unless it is small enough for the one-kernel
    // cluster TED (nothing to gain from sharding) or has fewer Gram tiles / rows than devices
    if (ctx->md && !use_small(ctx->params.flags, ctx->N) &&
        bted::pk::num_tiles((int)((ctx->N + bted::pk::T - 1) / bted::pk::T)) >= ctx->md->P && ctx->N >= ctx->md->P)
        return guarded(ctx, [&]() { return md_select(ctx, m, mu, out_idx, out_score); });
    return guarded(ctx, [&]() -> bted_status {
        Ted& T = ctx->ted;
        if (use_small(ctx->params.flags, ctx->N)) {
            grow(T.keys, T.keyscap, (size_t)m);
            if (!T.err) { grow(T.err, T.errcap, 1); CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream)); }
            Ted::Slot* sl = T.timing ? T.next_slot(m) : nullptr;
            if (sl) { sl->small = 1; CK(cudaEventRecord(sl->e[0], T.stream)); }
            unsigned long long* k4t = T.refine ? small_k4_reserve(ctx, 1, ctx->N, ctx->d, m) : nullptr;
            launch_small(ctx->X, 1, ctx->N, ctx->d, ctx->params.gamma, ctx->kernel, m, mu, T.keys, T.err, T.stream,
                         k4t);
            if (sl) CK(cudaEventRecord(sl->e[1], T.stream));
            if (k4t) small_k4_launch(ctx, T.stream, 1, ctx->N, ctx->d, m, T.keys);
            T.last_rows = 0;                       // K lived in shared memory only
            bted_status s = finish_keys(ctx, T, T.keys, m, out_idx, out_score);
            if (s == BTED_OK && k4t && small_k4_refine(ctx, T.stream, ctx->X, 1, ctx->N, ctx->d, m, mu, T.keys, T.err))
                s = finish_keys(ctx, T, T.keys, m, out_idx, out_score);
            return s;
        }
        // engine buffers are sized inside run_ted (the implicit engine needs ~2 N^2
        // bytes, the dense one 8 N^2): only the keys and K4 scratch here
        grow(T.keys, T.keyscap, (size_t)m);
        if (!T.err) { grow(T.err, T.errcap, 1); CK(cudaMemsetAsync(T.err, 0, sizeof(int), T.stream)); }
        const bool packed = use_packed(ctx->params.flags, ctx->d);
        if (T.refine) {
            T.reserve_refine(((ctx->N + bted::pk::T - 1) / bted::pk::T) * bted::pk::T, m);
            CK(cudaMemsetAsync(T.nflag, 0, sizeof(int), T.stream));
        }
        run_ted(T, ctx->X, ctx->N, ctx->d, ctx->params.gamma, ctx->kernel, m, mu, T.keys,
                (ctx->params.flags & BTED_FLAG_NO_GRAPH) != 0, true, packed, T.refine ? T.nflag : nullptr);
        std::vector<float> fixed(m, -1.f);
        if (T.refine) {
            int nf = 0;
            CK(cudaMemcpyAsync(&nf, T.nflag, sizeof(int), cudaMemcpyDeviceToHost, T.stream));
            CK(cudaStreamSynchronize(T.stream));
            if (nf > 0) refine_ted(ctx, T, ctx->X, ctx->N, ctx->d, m, mu, T.keys, fixed.data());
        }
        bted_status st = finish_keys(ctx, T, T.keys, m, out_idx, out_score);
        if (st == BTED_OK && out_score)
            for (int32_t t = 0; t < m; ++t) if (fixed[t] >= 0.f) out_score[t] = fixed[t];
        return st;
    });
}

bted_status bted_batch_teds(bted_ctx* ctx, int64_t M, int32_t m, float mu, int32_t b_begin, int32_t b_step,
                            int64_t* out_winners, int32_t winners_on_device) {
    if (!ctx || !out_winners) { set_error("null argument"); return BTED_EINVAL; }
    if (ctx->is_shard || ctx->is_ishard) { set_error("batch TEDs on a shard context"); return BTED_EINVAL; }
    if (m < 1 || M < m || M > ctx->N || !mu_ok(mu) || b_begin < 0 || b_step < 1) {
        set_error("need 1 <= m <= M <= N, mu > 0, b_begin >= 0, b_step >= 1"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        const int nb = run_batch_range(ctx, M, m, mu, b_begin, b_step);
        if (bted_status s = batch_range_finish(ctx, nb)) return s;
        if (nb > 0) {
            CK(cudaMemcpyAsync(out_winners, ctx->winners, sizeof(int64_t) * (size_t)nb * m,
                               winners_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaStreamSynchronize(ctx->stream));
        }
        return BTED_OK;
    });
}

bted_status bted_merge(bted_ctx* ctx, const int64_t* winners, int64_t n, int32_t winners_on_device, int32_t m,
                       float mu, int64_t* out_idx, int32_t* out_count) {
    if (!ctx || !winners || !out_idx || !out_count) { set_error("null argument"); return BTED_EINVAL; }
    if (ctx->is_shard || ctx->is_ishard) { set_error("merge on a shard context"); return BTED_EINVAL; }
    if (n < 1 || n >= (int64_t)INT32_MAX || m < 1 || !mu_ok(mu)) { set_error("need n >= 1, m >= 1, mu > 0"); return BTED_EINVAL; }
    if (!winners_on_device) {
        for (int64_t i = 0; i < n; ++i)
            if (winners[i] >= ctx->N) { set_error("winner index out of range"); return BTED_EINVAL; }
    }
    return guarded(ctx, [&]() -> bted_status {
        grow(ctx->winners, ctx->winnerscap, (size_t)n);
        if (winners != ctx->winners)
            CK(cudaMemcpyAsync(ctx->winners, winners, sizeof(int64_t) * n,
                               winners_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, ctx->stream));
        return merge_device(ctx, ctx->winners, n, m, mu, out_idx, out_count);
    });
}

bted_status bted_run_batches(bted_ctx* ctx, int64_t M, int32_t m, float mu, int64_t* out_idx, int32_t* out_count,
                             int64_t* out_batch_idx) {
    Nvtx nvtx_("bted_run_batches (Alg. 2)");
    if (!ctx || !out_idx || !out_count) { set_error("null argument"); return BTED_EINVAL; }
    if (ctx->is_shard || ctx->is_ishard) { set_error("run_batches on a shard context"); return BTED_EINVAL; }
    if (m < 1 || M < m || M > ctx->N || !mu_ok(mu)) { set_error("need 1 <= m <= M <= N and mu > 0"); return BTED_EINVAL; }
    if (ctx->md)
        return guarded(ctx, [&]() { return md_run_batches(ctx, M, m, mu, out_idx, out_count, out_batch_idx); });
    return guarded(ctx, [&]() -> bted_status {
        ctx->k4b.changed = false;
        const int nb = run_batch_range(ctx, M, m, mu, 0, 1);
        if (out_batch_idx)
            CK(cudaMemcpyAsync(out_batch_idx, ctx->winners, sizeof(int64_t) * (size_t)nb * m,
                               cudaMemcpyDeviceToHost, ctx->stream));
        bted_status s = merge_device(ctx, ctx->winners, (int64_t)nb * m, m, mu, out_idx, out_count, nb == 1);
        if (s == BTED_OK && out_batch_idx && ctx->k4b.changed) {   // batch K4 changed winners after the copy
            CK(cudaMemcpyAsync(out_batch_idx, ctx->winners, sizeof(int64_t) * (size_t)nb * m,
                               cudaMemcpyDeviceToHost, ctx->stream));
            CK(cudaStreamSynchronize(ctx->stream));
        }
        return s;
    });
}

bted_status bted_sample_batches(int64_t P, int64_t M, int32_t B, uint64_t seed, int64_t* out) {
    if (!out || M < 1 || M > P || P >= (int64_t)INT32_MAX || B < 1) {
        set_error("need 1 <= M <= P < 2^31, B >= 1, out != NULL"); return BTED_EINVAL;
    }
    // a scratch context with no features: only the sampling buffers are used
    bted_params p;
    bted_default_params(&p);
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
        cudaGetLastError();
        set_error("no CUDA device available: libbted has no CPU fallback");
        return BTED_ECUDA;
    }
    bted_ctx* ctx = new (std::nothrow) bted_ctx();
    if (!ctx) return BTED_ENOMEM;
    cudaGetDevice(&ctx->device);
    ctx->params = p;
    bted_status st = guarded(ctx, [&]() -> bted_status {
        CK(cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking));
        ctx->own_stream = true;
        int64_t* dout = nullptr;
        CK(cudaMalloc(&dout, sizeof(int64_t) * (size_t)M * B));
        grow(ctx->sall, ctx->sallcap, (size_t)M * B);
        sample_batches_dev(ctx, ctx->stream, P, M, 0, 1, B, seed, ctx->sall);
        const unsigned g = (unsigned)std::min<int64_t>((M * B + 255) / 256, 4096);
        bted::u32_to_i64_kernel<<<g, 256, 0, ctx->stream>>>(ctx->sall, M * B, dout);
        LAUNCHED(1);
        CK(cudaMemcpyAsync(out, dout, sizeof(int64_t) * (size_t)M * B, cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        cudaFree(dout);
        int e = 0;
        if (ctx->bted_engine.err) CK(cudaMemcpy(&e, ctx->bted_engine.err, sizeof(int), cudaMemcpyDeviceToHost));
        if (e) { set_error("batch sampling candidate overflow"); return BTED_ENUMERIC; }
        return BTED_OK;
    });
    bted_destroy(ctx);
    return st;
}

// ------------------------------------------------------------------ shards
bted_status bted_shard_gram(bted_ctx* ctx, float mu, uint64_t* keys_dev) {
    if (!ctx || !keys_dev || !ctx->is_shard || !mu_ok(mu)) { set_error("bad shard_gram arguments"); return BTED_EINVAL; }
    return guarded(ctx, [&]() -> bted_status {
        shard_gram_enqueue(ctx, mu, keys_dev);
        return BTED_OK;
    });
}

bted_status bted_shard_step(bted_ctx* ctx, int32_t t, float mu, const float* pivot_dev, uint64_t* keys_dev) {
    if (!ctx || !keys_dev || !pivot_dev || !ctx->is_shard || t < 1 || !mu_ok(mu)) {
        set_error("bad shard_step arguments"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        shard_step_enqueue(ctx, t, mu, pivot_dev, keys_dev);
        return BTED_OK;
    });
}

bted_status bted_shard_pivot_column(bted_ctx* ctx, int32_t t, const uint64_t* keys_dev, float* col_dev) {
    if (!ctx || !keys_dev || !col_dev || !ctx->is_shard || t < 0) { set_error("bad pivot_column arguments"); return BTED_EINVAL; }
    return guarded(ctx, [&]() -> bted_status {
        shard_pivot_enqueue(ctx, t, keys_dev, col_dev);
        return BTED_OK;
    });
}

bted_status bted_shard_colnorm(bted_ctx* ctx, int32_t t, float mu, const float* pivot_dev,
                               const uint64_t* keys_dev, float* colnorm_dev) {
    if (!ctx || !colnorm_dev || !ctx->is_shard || t < 0 || (t > 0 && (!pivot_dev || !keys_dev)) || !mu_ok(mu)) {
        set_error("bad shard_colnorm arguments"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        shard_colnorm_enqueue(ctx, t, mu, pivot_dev, keys_dev, colnorm_dev);
        return BTED_OK;
    });
}

bted_status bted_shard_scores(bted_ctx* ctx, int32_t t, float mu, const float* colnorm_dev, uint64_t* keys_dev) {
    if (!ctx || !colnorm_dev || !keys_dev || !ctx->is_shard || t < 0 || !mu_ok(mu)) {
        set_error("bad shard_scores arguments"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        shard_scores_enqueue(ctx, t, mu, colnorm_dev, keys_dev);
        return BTED_OK;
    });
}

// ------------------------------------------------------------------ tile-sharded implicit engine
bted_status bted_ishard_create(const float* X, int64_t N, int32_t d, bted_kernel kernel, int32_t rank, int32_t nranks,
                               const bted_params* params, bted_ctx** out) {
    if (nranks < 1 || rank < 0 || rank >= nranks) { set_error("need 0 <= rank < nranks"); return BTED_EINVAL; }
    if (d > 32) { set_error("the tile-sharded engine needs d <= 32"); return BTED_EINVAL; }
    bted_status st = create_common(X, N, d, kernel, params, 0, 0, false, out);
    if (st != BTED_OK) return st;
    (*out)->is_ishard = true;
    (*out)->srank = rank;
    (*out)->snranks = nranks;
    const int nT = (int)((N + bted::pk::T - 1) / bted::pk::T);
    if (bted::pk::num_tiles(nT) < nranks) {
        bted_destroy(*out); *out = nullptr;
        set_error("fewer Gram tiles than shards"); return BTED_EINVAL;
    }
    return BTED_OK;
}

int64_t bted_ishard_qlen(const bted_ctx* ctx) {
    if (!ctx) return 0;
    return ishard_qlen_of(ctx->N);
}

bted_status bted_ishard_head(bted_ctx* ctx, int32_t m, float mu, double* q_dev) {
    if (!ctx || !q_dev || !ctx->is_ishard || m < 1 || m > ctx->N || m > bted::im::kMaxM || !mu_ok(mu)) {
        set_error("bad ishard_head arguments"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        ishard_head_enqueue(ctx, m, q_dev);
        return BTED_OK;
    });
}

bted_status bted_ishard_step(bted_ctx* ctx, int32_t t, float mu, const uint64_t* keys_dev, double* q_dev) {
    if (!ctx || !q_dev || !keys_dev || !ctx->is_ishard || t < 1 || t >= ctx->sm_m || !mu_ok(mu)) {
        set_error("bad ishard_step arguments (head first; 1 <= t < m)"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        ishard_step_enqueue(ctx, t, mu, reinterpret_cast<const unsigned long long*>(keys_dev), q_dev);
        return BTED_OK;
    });
}

bted_status bted_ishard_fin(bted_ctx* ctx, int32_t t, float mu, const double* q_dev, uint64_t* keys_dev) {
    if (!ctx || !q_dev || !keys_dev || !ctx->is_ishard || t < 0 || t >= ctx->sm_m || !mu_ok(mu)) {
        set_error("bad ishard_fin arguments (head first; 0 <= t < m)"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        ishard_fin_enqueue(ctx, t, mu, q_dev, reinterpret_cast<unsigned long long*>(keys_dev));
        return BTED_OK;
    });
}

bted_status bted_ishard_refine(bted_ctx* ctx, int32_t m, float mu, const uint64_t* keys_dev, uint64_t* forced_host,
                               int32_t* nforced) {
    if (!ctx || !keys_dev || !forced_host || !nforced || !ctx->is_ishard || m < 1 || m != ctx->sm_m || !mu_ok(mu)) {
        set_error("bad ishard_refine arguments"); return BTED_EINVAL;
    }
    *nforced = 0;
    return guarded(ctx, [&]() -> bted_status {
        std::vector<unsigned long long> forced;
        if (ishard_k4(ctx, m, mu, reinterpret_cast<const unsigned long long*>(keys_dev), forced)) {
            for (size_t q = 0; q < forced.size(); ++q) forced_host[q] = forced[q];
            *nforced = (int32_t)forced.size();
        }
        return BTED_OK;
    });
}

bted_status bted_shard_nearties(bted_ctx* ctx, int32_t m, const uint64_t* keys_dev, uint32_t* cand_dev,
                                int32_t* ncand_dev) {
    if (!ctx || !keys_dev || !cand_dev || !ncand_dev || !ctx->is_shard || m < 1) {
        set_error("bad shard_nearties arguments"); return BTED_EINVAL;
    }
    return guarded(ctx, [&]() -> bted_status {
        Ted& T = ctx->ted;
        const int mm = std::min<int32_t>(m, bted::im::kMaxM);
        CK(cudaMemsetAsync(ncand_dev, 0, sizeof(int32_t) * m, T.stream));
        if (!T.refine || !T.top2) return BTED_OK;
        bted::rf::shard_neartie_kernel<<<mm, 256, 0, T.stream>>>(
            T.top2, T.last_nC, reinterpret_cast<const unsigned long long*>(keys_dev), bted::rf::kTau, cand_dev,
            reinterpret_cast<int*>(ncand_dev));
        LAUNCHED(1);
        return BTED_OK;
    });
}

bted_status bted_shard_refine(bted_ctx* ctx, int32_t m, float mu, const uint64_t* keys_dev, const uint32_t* cand_all,
                              const int32_t* ncand_all, int32_t nranks, uint64_t* forced_host, int32_t* nforced) {
    if (!ctx || !keys_dev || !cand_all || !ncand_all || !forced_host || !nforced || !ctx->is_shard || m < 1 ||
        nranks < 1 || !mu_ok(mu)) {
        set_error("bad shard_refine arguments"); return BTED_EINVAL;
    }
    *nforced = 0;
    return guarded(ctx, [&]() -> bted_status {
        std::vector<unsigned long long> forced;
        if (shard_k4_decide(ctx, m, mu, reinterpret_cast<const unsigned long long*>(keys_dev), cand_all, ncand_all,
                            nranks, forced)) {
            std::copy(forced.begin(), forced.end(), forced_host);
            *nforced = (int32_t)forced.size();
        }
        return BTED_OK;
    });
}

int64_t bted_shard_ld(const bted_ctx* ctx) { return ctx ? ld_for(ctx->N) : 0; }

bted_status bted_shard_check(bted_ctx* ctx) {
    return guarded(ctx, [&]() -> bted_status {
        if (!ctx->ted.err) return BTED_OK;
        CK(cudaMemcpyAsync(ctx->herr, ctx->ted.err, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
        CK(cudaStreamSynchronize(ctx->stream));
        if (*ctx->herr) { set_error("non-finite score in a shard step"); return BTED_ENUMERIC; }
        return BTED_OK;
    });
}

bted_status bted_update(bted_ctx* ctx, const float* X, int32_t x_on_device) {
    if (!ctx || !X) { set_error("null argument"); return BTED_EINVAL; }
    return guarded(ctx, [&]() -> bted_status {
        if (!ctx->own_X) {
            CK(cudaMalloc(&ctx->X, sizeof(float) * ctx->N * ctx->d));
            ctx->own_X = true;
        }
        CK(cudaMemcpyAsync(ctx->X, X, sizeof(float) * ctx->N * ctx->d,
                           x_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, ctx->stream));
        // no sync: later work of this ctx is ordered after the copy on its stream;
        // the caller must keep a host X alive until the next call returns.  The
        // finiteness check runs on the device; a bad X fails the next call (EINVAL).
        launch_finite_check(ctx);
        if (ctx->md) {                       // the devices' copies are rebuilt from the new X on next use
            CK(cudaStreamSynchronize(ctx->stream));
            md_drop_replicas(ctx->md);
        }
        return BTED_OK;
    });
}

bted_status bted_host_alloc(size_t bytes, void** out) {
    if (!out || bytes == 0) { set_error("need bytes > 0 and out != NULL"); return BTED_EINVAL; }
    *out = nullptr;
    cudaError_t e = cudaMallocHost(out, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error("cudaMallocHost(%zu): %s", bytes, cudaGetErrorString(e));
        return e == cudaErrorMemoryAllocation ? BTED_ENOMEM : BTED_ECUDA;
    }
    return BTED_OK;
}

void bted_host_free(void* p) {
    if (p) cudaFreeHost(p);
}

bted_status bted_get_stats(bted_ctx* ctx, bted_stats* out) {
    if (!ctx || !out) { set_error("null argument"); return BTED_EINVAL; }
    std::memset(out, 0, sizeof *out);
    std::vector<bted_ctx*> all{ctx};
    if (ctx->md) {                                 // multi-GPU: the replicas' batches + shard 0's K4
        for (auto* c : ctx->md->rep) if (c) all.push_back(c);
        if (!ctx->md->sub.empty()) all.push_back(ctx->md->sub[0]);
    }
    for (bted_ctx* c : all) {
        for (const Stats* a : {&c->ted.stats, &c->bted_engine.stats}) {
            out->teds += a->teds;
            out->k2_launches += a->k2_launches;
            out->k1_ms += a->k1_ms;
            out->k2_ms += a->k2_ms;
            out->small_teds += a->small_teds;
            out->small_ms += a->small_ms;
        }
        out->refined_steps += c->refined_steps;
        out->corrected_steps += c->corrected_steps;
        out->full_refined_steps += c->full_refined_steps;
    }
    return BTED_OK;
}

bted_status bted_reset_stats(bted_ctx* ctx) {
    if (!ctx) { set_error("null argument"); return BTED_EINVAL; }
    std::vector<bted_ctx*> all{ctx};
    if (ctx->md) {
        for (auto* c : ctx->md->rep) if (c) all.push_back(c);
        for (auto* c : ctx->md->sub) all.push_back(c);
    }
    for (bted_ctx* c : all) {
        c->ted.stats = Stats{};
        c->bted_engine.stats = Stats{};
        c->refined_steps = c->corrected_steps = c->full_refined_steps = 0;
    }
    return BTED_OK;
}

// ------------------------------------------------------------------ misc
void bted_destroy(bted_ctx* ctx) {
    if (!ctx) return;
    md_release(ctx->md);
    ctx->md = nullptr;
    {
        DeviceGuard dg(ctx->device);
        if (ctx->stream) cudaStreamSynchronize(ctx->stream);
        ctx->ted.release();
        ctx->bted_engine.release();
        void* bufs[] = {ctx->Xb, ctx->winners, ctx->u32a,
                        ctx->u32b, ctx->count_dev, ctx->mkeys, ctx->cub_tmp, ctx->out_dev, ctx->sall,
                        ctx->xall, ctx->kall, ctx->shist, ctx->sint, ctx->scand, ctx->ssel, ctx->soff,
                        ctx->bflag, ctx->rcols, ctx->rG, ctx->rA, ctx->rW, ctx->rpart, ctx->rdiag, ctx->rout,
                        ctx->ridx, ctx->rWt, ctx->rsc, ctx->rmask, ctx->bkeys, ctx->bsflags, ctx->bncand, ctx->bcand, ctx->sks, ctx->scnt,
                        ctx->ktop2, ctx->kflags, ctx->kcand, ctx->kncand, ctx->knflag, ctx->kforced};
        if (ctx->k4pin) cudaFreeHost(ctx->k4pin);
        if (ctx->bfpin) cudaFreeHost(ctx->bfpin);
        for (void* b : bufs) if (b) cudaFree(b);
        if (ctx->own_X && ctx->X) cudaFree(ctx->X);
        if (ctx->hkeys) cudaFreeHost(ctx->hkeys);
        if (ctx->herr) cudaFreeHost(ctx->herr);
        if (ctx->xbad) cudaFree(ctx->xbad);
        if (ctx->own_stream && ctx->stream) cudaStreamDestroy(ctx->stream);
        cudaGetLastError();
    }
    delete ctx;
}

const char* bted_status_string(bted_status s) {
    switch (s) {
        case BTED_OK: return "BTED_OK";
        case BTED_EINVAL: return "BTED_EINVAL";
        case BTED_ENOMEM: return "BTED_ENOMEM";
        case BTED_ECUDA: return "BTED_ECUDA";
        case BTED_ENCCL: return "BTED_ENCCL";
        case BTED_ENUMERIC: return "BTED_ENUMERIC";
        case BTED_ESTATE: return "BTED_ESTATE";
    }
    return "BTED_UNKNOWN";
}

const char* bted_last_error(void) { return g_last_error.c_str(); }

uint64_t bted_kernel_launches(void) { return g_launches.load(); }

bted_status bted_debug_copy_K(bted_ctx* ctx, int32_t which, float* out, int64_t* ld_out) {
    if (!ctx || !out) { set_error("null argument"); return BTED_EINVAL; }
    return guarded(ctx, [&]() -> bted_status {
        Ted& T = which == 1 ? ctx->bted_engine : ctx->ted;
        if (!T.K[T.last_buf] || T.last_rows == 0) { set_error("no K yet"); return BTED_ESTATE; }
        const int64_t rows = T.last_rows, ld = T.last_ld;
        if (!T.last_packed) {
            CK(cudaMemcpyAsync(out, T.K[T.last_buf], sizeof(float) * rows * ld, cudaMemcpyDeviceToHost, T.stream));
            CK(cudaStreamSynchronize(T.stream));
        } else {
            // unpack the upper-triangular tiles into the dense rows x ld view
            const int nT = T.last_nT, TT = bted::pk::T;
            const size_t n = (size_t)bted::pk::num_tiles(nT) * TT * TT;
            std::vector<float> h(n);
            CK(cudaMemcpyAsync(h.data(), T.K[T.last_buf], sizeof(float) * n, cudaMemcpyDeviceToHost, T.stream));
            CK(cudaStreamSynchronize(T.stream));
            std::memset(out, 0, sizeof(float) * rows * ld);
            for (int64_t i = 0; i < rows; ++i)
                for (int64_t j = 0; j < rows; ++j) {
                    const int I = (int)(i / TT), J = (int)(j / TT), r = (int)(i % TT), c = (int)(j % TT);
                    out[i * ld + j] = I <= J ? h[(size_t)bted::pk::tile_offset(I, J, nT) * TT * TT + r * TT + c]
                                             : h[(size_t)bted::pk::tile_offset(J, I, nT) * TT * TT + c * TT + r];
                }
        }
        if (ld_out) *ld_out = ld;
        return BTED_OK;
    });
}

}  // extern "C"
