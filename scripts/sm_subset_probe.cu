// How fast does the streaming K.l pass (implicit.cuh tile_pass, the library's
// consumer and producer) run when only S of the SMs stream?  CTAs on SMs with
// %smid >= S exit at once; the rest share the tiles through the pass counter.
// Answers whether a pass split between streaming SMs and SMs that recompute
// their tiles on the tensor cores (rc_pass.cuh) can beat streaming on all SMs.
// Build:
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/sm_subset_probe scripts/sm_subset_probe.cu
#include <cstdio>
#include <vector>
#include "../paper_conf_date_sunbg021_b200/csrc/implicit.cuh"
using namespace bted;

__device__ __forceinline__ unsigned smid() {
    unsigned r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}

__global__ void __launch_bounds__(im::kTPThreads, im::kTPBlocksPerSM)
tp_sub(const float* __restrict__ K, int nT, const double* w, double* P64, int* ctr, unsigned S) {
    extern __shared__ __align__(1024) unsigned char smem_raw[];
    if (smid() >= S) return;
    im::TPSmem& Sm = *reinterpret_cast<im::TPSmem*>(smem_raw);
    im::tp_init_barriers(Sm);
    if (threadIdx.x / 32 == im::kTPWarps) {
        if (threadIdx.x % 32 == 0) im::tp_produce<true>(Sm, K, nT, w, 1, ctr, im::NoWait{});
        return;
    }
    int n = 0, ti = 0, ci = 0;
    im::tp_consume<false, false>(Sm, nT, P64, nullptr, n, ti, ci);
}

__global__ void fill(float* K, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        K[i] = 0.25f + 0.5f * (float)((i * 2654435761u) % 1000) / 1000.f;
}
__global__ void flush(float* b, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        b[i] = (float)i;
}

int main(int argc, char** argv) {
    const int N = argc > 1 ? atoi(argv[1]) : 16384;
    const int nT = (N + 127) / 128;
    int sms = 0; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t nk = (size_t)pk::num_tiles(nT) * 128 * 128;
    float *K, *fb; double *w, *P64; int* ctr;
    const size_t nf = (size_t)64 << 20;                       // 256 MiB: flushes L2 between passes
    cudaMalloc(&K, nk * 4); cudaMalloc(&w, (size_t)nT * 128 * 8); cudaMalloc(&P64, (size_t)nT * nT * 128 * 8);
    cudaMalloc(&ctr, 4); cudaMalloc(&fb, nf * 4);
    fill<<<1184, 256>>>(K, nk);
    std::vector<double> hw((size_t)nT * 128, 0.01);
    cudaMemcpy(w, hw.data(), hw.size() * 8, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(tp_sub, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)im::tile_pass_smem_bytes);
    cudaFuncSetAttribute(tp_sub, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
    const int grid = im::kTPBlocksPerSM * sms;
    const double bytes = (double)nk * 4;
    printf("N = %d, tiles %lld, %.1f MB read, grid %d\n", N, (long long)pk::num_tiles(nT), bytes / 1e6, grid);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int subsets[] = {148, 140, 132, 124, 116, 108, 100, 92, 84, 76, 68};
    for (int S : subsets) {
        if (S > sms) continue;
        float best = 1e9, sum = 0; const int R = 12;
        for (int r = -2; r < R; ++r) {
            flush<<<1184, 256>>>(fb, nf);
            cudaMemset(ctr, 0, 4);
            cudaEventRecord(e0);
            tp_sub<<<grid, im::kTPThreads, im::tile_pass_smem_bytes>>>(K, nT, w, P64, ctr, (unsigned)S);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            if (r >= 0) { best = ms < best ? ms : best; sum += ms; }
        }
        printf("streaming SMs %3d: best %7.1f us  avg %7.1f us  %6.0f GB/s  %.3f tiles/us/SM  %s\n", S, best * 1e3,
               sum / R * 1e3, bytes / (best * 1e-3) / 1e9, pk::num_tiles(nT) / (best * 1e3) / S,
               cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
