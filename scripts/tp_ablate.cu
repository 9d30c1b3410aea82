// Ablation of the implicit tile pass (implicit.cuh tp_consume<false, false, kAbl>)
// at N = 16384: which part of the consumer work keeps q = K l below the
// read-only HBM ceiling (scripts/read_bw.cu).  Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o scripts/tp_ablate scripts/tp_ablate.cu
#include <cstdio>
#include <vector>
#include "../paper_conf_date_sunbg021_b200/csrc/implicit.cuh"
using namespace bted;

template <int kAbl>
__global__ void __launch_bounds__(im::kTPThreads, im::kTPBlocksPerSM)
tp_abl(const float* __restrict__ K, int nT, const double* w, double* P64, int* ctr) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    im::TPSmem& S = *reinterpret_cast<im::TPSmem*>(smem_raw);
    im::tp_init_barriers(S);
    if (threadIdx.x / 32 == im::kTPWarps) {
        if (threadIdx.x % 32 == 0) im::tp_produce<true>(S, K, nT, w, 1, ctr, im::NoWait{});
        return;
    }
    int n = 0, ti = 0, ci = 0;
    im::tp_consume<false, false, kAbl>(S, nT, P64, nullptr, n, ti, ci);
}

__global__ void fill(float* K, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        K[i] = 0.25f + 0.5f * (float)((i * 2654435761u) % 1000) / 1000.f;
}

template <int kAbl>
void run(const char* name, const float* K, int nT, const double* w, double* P64, int grid) {
    int* ctr; cudaMalloc(&ctr, 4);
    auto k = tp_abl<kAbl>;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)im::tile_pass_smem_bytes);
    cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaMemset(ctr, 0, 4);
    k<<<grid, im::kTPThreads, im::tile_pass_smem_bytes>>>(K, nT, w, P64, ctr);
    cudaDeviceSynchronize();
    float best = 1e9, sum = 0; const int R = 20;
    for (int r = 0; r < R; ++r) {
        cudaMemset(ctr, 0, 4);
        cudaEventRecord(e0);
        k<<<grid, im::kTPThreads, im::tile_pass_smem_bytes>>>(K, nT, w, P64, ctr);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1); best = ms < best ? ms : best; sum += ms;
    }
    const double bytes = (double)pk::num_tiles(nT) * pk::T * pk::T * 4;
    printf("%-34s best %7.1f us  avg %7.1f us  %6.0f GB/s (best)  %s\n", name, best * 1e3, sum / R * 1e3,
           bytes / (best * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError()));
}

int main(int argc, char** argv) {
    const int N = argc > 1 ? atoi(argv[1]) : 16384;
    const int nT = (N + 127) / 128;
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t nk = (size_t)pk::num_tiles(nT) * 128 * 128;
    float* K; double *w, *P64;
    cudaMalloc(&K, nk * 4); cudaMalloc(&w, (size_t)nT * 128 * 8); cudaMalloc(&P64, (size_t)nT * nT * 128 * 8);
    fill<<<1184, 256>>>(K, nk);
    std::vector<double> hw((size_t)nT * 128, 0.01);
    cudaMemcpy(w, hw.data(), hw.size() * 8, cudaMemcpyHostToDevice);
    const int grid = im::kTPBlocksPerSM * sms;
    printf("N = %d, tiles %lld, %.1f MB read, grid %d, smem %zu B\n", N, (long long)pk::num_tiles(nT), nk * 4 / 1e6,
           grid, im::tile_pass_smem_bytes);
    run<0>("full (library)", K, nT, w, P64, grid);
    run<1>("no partial stores", K, nT, w, P64, grid);
    run<16>("plain partial stores", K, nT, w, P64, grid);
    run<64>("evict-last partial stores", K, nT, w, P64, grid);
    run<8>("no arithmetic (LDS + arrive)", K, nT, w, P64, grid);
    return 0;
}
