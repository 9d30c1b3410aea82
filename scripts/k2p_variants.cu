// k2p_variants.cu -- design-space microbenchmark for the packed-symmetric
// deflate kernel K2p (TMA ring granularity, L2 cache hints) and the finalize
// kernel.  Not part of the product; results under profiles/.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
//      -I paper_conf_date_sunbg021_b200/csrc scripts/k2p_variants.cu -o scripts/k2pv
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <vector>
#include <cuda_runtime.h>
#include "packed.cuh"

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)
using namespace bted;
using namespace bted::pk;

__global__ void init_packed(float* K, int nT, int N) {
    const int64_t total = num_tiles(nT) * (int64_t)(T * T);
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int64_t k = e / (T * T);
        const int rc = (int)(e % (T * T));
        int I, J;
        tile_ij(k, nT, I, J);
        const int i = I * T + rc / T, j = J * T + rc % T;
        float v = 0.f;
        if (i < N && j < N) { const float d = (float)(i - j); v = expf(-1e-5f * d * d); }
        K[e] = v;
    }
}

template <int kSub, bool kHints, bool kV8 = false>
void launch(const float* A, float* B, int nT, int N, float* P, unsigned long long* keys, uint8_t* sel, int sms) {
    auto kern = kV8 ? deflate_packed_v8_kernel<kSub, kHints> : deflate_packed_kernel<kSub, kHints>;
    static bool set = false;
    if (!set) {
        CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)k2p_smem_bytes(kSub)));
        set = true;
    }
    const int64_t tiles = num_tiles(nT);
    kern<<<(unsigned)std::min<int64_t>(tiles, sms), kConsumers + 32, k2p_smem_bytes(kSub)>>>(
        A, B, nT, N, P, keys, 1, 0.1f, sel);
}

int main(int argc, char** argv) {
    const int N = argc > 1 ? atoi(argv[1]) : 16384;
    const int iters = argc > 2 ? atoi(argv[2]) : 20;
    const int nT = (N + T - 1) / T;
    const size_t n = (size_t)num_tiles(nT) * T * T;
    const size_t NP = (size_t)nT * T;
    float *A, *B, *P, *Pref;
    CK(cudaMalloc(&A, n * 4)); CK(cudaMalloc(&B, n * 4)); CK(cudaMalloc(&P, nT * NP * 4)); CK(cudaMalloc(&Pref, nT * NP * 4));
    unsigned long long* keys; CK(cudaMalloc(&keys, 64 * 8));
    uint8_t* sel; CK(cudaMalloc(&sel, NP)); CK(cudaMemset(sel, 0, NP));
    int* err; CK(cudaMalloc(&err, 4)); CK(cudaMemset(err, 0, 4));
    init_packed<<<148 * 8, 256>>>(A, nT, N);
    CK(cudaDeviceSynchronize());
    int sms = 0; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    const unsigned long long key0 = (((unsigned long long)0x3f800000u + 1) << 32) | (0xFFFFFFFFu - (uint32_t)(N / 3));
    CK(cudaMemcpy(keys, &key0, 8, cudaMemcpyHostToDevice));
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    const double alg = 4.0 * N * (double)N, actual = 2.0 * n * 4;
    // reference outputs from <128,false>
    launch<128, false>(A, B, nT, N, Pref, keys, sel, sms);
    CK(cudaDeviceSynchronize());
    std::vector<float> kref(n), kb(n), pref(nT * NP), pb(nT * NP);
    CK(cudaMemcpy(kref.data(), B, n * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(pref.data(), Pref, nT * NP * 4, cudaMemcpyDeviceToHost));
    auto run = [&](const char* name, std::function<void()> f, bool check) {
        for (int w = 0; w < 3; ++w) f();
        CK(cudaDeviceSynchronize());
        float tot = 0;
        for (int it = 0; it < iters; ++it) {
            CK(cudaEventRecord(e0)); f(); CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
            float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); tot += ms;
        }
        const double ms = tot / iters;
        const char* ok = "-";
        if (check) {
            CK(cudaMemcpy(kb.data(), B, n * 4, cudaMemcpyDeviceToHost));
            CK(cudaMemcpy(pb.data(), P, nT * NP * 4, cudaMemcpyDeviceToHost));
            ok = (!memcmp(kb.data(), kref.data(), n * 4) && !memcmp(pb.data(), pref.data(), nT * NP * 4)) ? "bit-equal" : "DIFF";
        }
        printf("%-36s %8.4f ms  alg %7.1f GB/s  actual %7.1f GB/s  %s\n", name, ms, alg / (ms * 1e-3) / 1e9,
               actual / (ms * 1e-3) / 1e9, ok);
    };
    run("cudaMemcpyDeviceToDevice (same bytes)", [&] { CK(cudaMemcpyAsync(B, A, n * 4, cudaMemcpyDeviceToDevice)); }, false);
    run("k2p<128,nohint>", [&] { launch<128, false>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p<128,hints>", [&] { launch<128, true>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p<64,nohint>", [&] { launch<64, false>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p<64,hints>", [&] { launch<64, true>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p_v8<128,nohint>", [&] { launch<128, false, true>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p_v8<64,nohint>", [&] { launch<64, false, true>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p_v8<64,hints>", [&] { launch<64, true, true>(A, B, nT, N, P, keys, sel, sms); }, true);
    run("k2p_ldg<4>", [&] { deflate_packed_ldg_kernel<4><<<(unsigned)num_tiles(nT), kConsumers>>>(A, B, nT, N, P, keys, 1, 0.1f, sel); }, true);
    run("k2p_ldg<8>", [&] { deflate_packed_ldg_kernel<8><<<(unsigned)num_tiles(nT), kConsumers>>>(A, B, nT, N, P, keys, 1, 0.1f, sel); }, true);
    run("k2p_ldg<2>", [&] { deflate_packed_ldg_kernel<2><<<(unsigned)num_tiles(nT), kConsumers>>>(A, B, nT, N, P, keys, 1, 0.1f, sel); }, true);
    run("finalize", [&] { finalize_packed_kernel<<<nT * T / kFinRows, kFinThreads>>>(P, nT, N, B, 0.1f, sel, keys, 1, keys + 1, err); }, false);
    printf("done N=%d tiles=%lld\n", N, (long long)num_tiles(nT));
    return 0;
}
