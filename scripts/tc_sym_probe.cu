// tc_sym_probe.cu -- does ONE accumulator of bf16 tcgen05.mma give a bit-symmetric
// Gram when each instruction holds both halves of a cross term?
//
// Scheme (x = h + m + l, three bf16 parts; the six kept products):
//   mma 0,1: [h | l] . [l | h]  (features 0-7, 8-15): h_r l_c and l_r h_c in ONE instruction
//   mma 2  : [m] . [m]
//   mma 3,4: [h | m] . [m | h]
//   mma 5  : [h] . [h]
// Under r <-> c every instruction sees the same multiset of 16 products, so D is
// symmetric iff the tensor core's K=16 reduction is a symmetric function of its
// products.  Checks: (a) D_II == D_II^T bitwise, (b) D_IJ == D_JI^T, (c) position
// invariance (permuted rows give permuted results), (d) exact duplicate rows,
// (e) accuracy against fp64.   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/p tc_sym_probe.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <cmath>
#include <vector>
#include <random>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

constexpr int T = 128, D = 16, kChunks = 12;
constexpr uint32_t kSBO = kChunks * 128, kBlockBytes = (T / 8) * kSBO;
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(T >> 3) << 17) | ((uint32_t)(T >> 4) << 24);
// storage chunks: 0 h0-7, 1 l0-7, 2 h8-15, 3 l8-15, 4 m0-7, 5 m8-15, 6 h0-7, 7 m0-7, 8 h8-15, 9 m8-15, 10 h0-7, 11 h8-15
__constant__ int kAStart[6] = {0, 2, 4, 6, 8, 10};
__constant__ int kBStart[6] = {1, 3, 4, 7, 9, 10};
__constant__ int kBLbo[6] = {5, 5, 1, 3, 2, 1};

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %d\n", cudaGetErrorString(e), __LINE__); exit(1); } } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t saddr, uint32_t lbo_bytes) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((kSBO >> 4) & 0x3FFFu) << 32;
    d |= (uint64_t)1 << 46;
    return d;
}
__device__ __forceinline__ void mma(uint32_t t, uint64_t a, uint64_t b, uint32_t acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n"
                 :: "r"(t), "l"(a), "l"(b), "r"(kIdesc), "r"(acc));
}

__global__ void probe(const uint8_t* opI, const uint8_t* opJ, float* out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar;
    __shared__ uint32_t tb;
    const int tid = threadIdx.x, w = tid / 32;
    for (int i = tid; i < (int)kBlockBytes / 16; i += blockDim.x) {
        reinterpret_cast<uint4*>(sm)[i] = reinterpret_cast<const uint4*>(opI)[i];
        reinterpret_cast<uint4*>(sm + kBlockBytes)[i] = reinterpret_cast<const uint4*>(opJ)[i];
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    if (w == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" :: "r"(su32(&tb)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t t = tb;
    if (tid == 0) {
        const uint32_t a = su32(sm), b = su32(sm + kBlockBytes);
        for (int s = 0; s < 6; ++s)
            mma(t, desc(a + 128u * kAStart[s], 128u), desc(b + 128u * kBStart[s], 128u * kBLbo[s]), s > 0);
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(su32(&bar)) : "memory");
    }
    asm volatile("{\n\t.reg .pred P1;\n\tW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t@!P1 bra W;\n\t}" :: "r"(su32(&bar)) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int r = 32 * w + tid % 32;
    for (int c0 = 0; c0 < T; c0 += 8) {
        uint32_t v[8];
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                     : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                     : "r"(t + ((uint32_t)(32 * w) << 16) + (uint32_t)c0));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        for (int q = 0; q < 8; ++q) out[r * T + c0 + q] = __uint_as_float(v[q]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (w == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" :: "r"(t));
}

static uint32_t off(int r, int chunk, int e) { return (uint32_t)(r >> 3) * kSBO + chunk * 128u + (uint32_t)(r & 7) * 16u + e * 2u; }

static void build(const std::vector<float>& X, const std::vector<int>& rows, std::vector<uint8_t>& op) {
    op.assign(kBlockBytes, 0);
    for (int r = 0; r < T; ++r) {
        __nv_bfloat16 h[D], m[D], l[D];
        for (int k = 0; k < D; ++k) {
            const float v = X[rows[r] * D + k];
            h[k] = __float2bfloat16_rn(v);
            const float r1 = v - __bfloat162float(h[k]);
            m[k] = __float2bfloat16_rn(r1);
            l[k] = __float2bfloat16_rn(r1 - __bfloat162float(m[k]));
        }
        const __nv_bfloat16* src[12] = {h, l, h + 8, l + 8, m, m + 8, h, m, h + 8, m + 8, h, h + 8};
        for (int c = 0; c < 12; ++c)
            for (int e = 0; e < 8; ++e) memcpy(op.data() + off(r, c, e), &src[c][e], 2);
    }
}

static std::vector<float> run(const std::vector<uint8_t>& a, const std::vector<uint8_t>& b) {
    uint8_t *da, *db; float* dout;
    CK(cudaMalloc(&da, kBlockBytes)); CK(cudaMalloc(&db, kBlockBytes)); CK(cudaMalloc(&dout, T * T * 4));
    CK(cudaMemcpy(da, a.data(), kBlockBytes, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(db, b.data(), kBlockBytes, cudaMemcpyHostToDevice));
    CK(cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * kBlockBytes));
    probe<<<1, 128, 2 * kBlockBytes>>>(da, db, dout);
    CK(cudaGetLastError()); CK(cudaDeviceSynchronize());
    std::vector<float> o(T * T);
    CK(cudaMemcpy(o.data(), dout, T * T * 4, cudaMemcpyDeviceToHost));
    cudaFree(da); cudaFree(db); cudaFree(dout);
    return o;
}

static int neq(float a, float b) { uint32_t x, y; memcpy(&x, &a, 4); memcpy(&y, &b, 4); return x != y; }

int main() {
    std::mt19937_64 g(7);
    std::normal_distribution<double> nd;
    int fails = 0;
    for (int trial = 0; trial < 6; ++trial) {
        std::vector<float> X(3 * T * D);
        for (auto& v : X) v = (float)(nd(g) * (trial % 3 == 0 ? 1.0 : trial % 3 == 1 ? 0.37 : 3.1));
        if (trial >= 3) for (auto& v : X) v = (float)std::floor(v * 4.0) / 4.0f - 0.3f;   // knob-like grid
        for (int k = 0; k < D; ++k) X[77 * D + k] = X[5 * D + k];                     // exact duplicate rows
        std::vector<int> r0(T), r1(T), r2(T);
        for (int i = 0; i < T; ++i) { r0[i] = i; r1[i] = T + i; r2[i] = 2 * T - 1 - i; }
        std::vector<uint8_t> A0, A1, A2;
        build(X, r0, A0); build(X, r1, A1); build(X, r2, A2);
        auto d00 = run(A0, A0), d01 = run(A0, A1), d10 = run(A1, A0), d02 = run(A0, A2);
        int sym = 0, orient = 0, pos = 0, dup = 0;
        double maxrel = 0;
        for (int r = 0; r < T; ++r)
            for (int c = 0; c < T; ++c) {
                sym += neq(d00[r * T + c], d00[c * T + r]);
                orient += neq(d01[r * T + c], d10[c * T + r]);
                pos += neq(d02[r * T + c], d01[r * T + (T - 1 - c)]);
                if (r == 5) { dup += neq(d00[5 * T + c], d00[77 * T + c]); dup += neq(d01[5 * T + c], d01[77 * T + c]); }
                double ex = 0, nr = 0, nc = 0;
                for (int k = 0; k < D; ++k) {
                    ex += (double)X[r * D + k] * X[(T + c) * D + k];
                    nr += (double)X[r * D + k] * X[r * D + k];
                    nc += (double)X[(T + c) * D + k] * X[(T + c) * D + k];
                }
                maxrel = std::fmax(maxrel, std::fabs(d01[r * T + c] - ex) / std::sqrt(nr * nc));
            }
        printf("trial %d: asym %d  orient %d  pos %d  dup %d  max |err|/(|x||y|) %.3e (= %.2f ulp)\n", trial, sym, orient,
               pos, dup, maxrel, maxrel / std::ldexp(1.0, -24));
        fails += sym + orient + pos + dup;
    }
    printf(fails ? "RESULT: NOT symmetric\n" : "RESULT: symmetric, orientation- and position-invariant\n");
    return 0;
}
