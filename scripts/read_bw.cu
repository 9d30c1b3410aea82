// Read-only HBM bandwidth ceiling on B200 (what a read-only pass like the
// implicit tile pass can reach): 256-bit LDG grid-stride reduction and a
// persistent cp.async.bulk ring with no compute.  nvcc -gencode
// arch=compute_100a,code=sm_100a -O3 -o read_bw read_bw.cu && ./read_bw
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void ld8(const float* p, float (&v)[8]) {
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
                 : "l"(p));
}
template <int U>
__global__ void ldg_read(const float* __restrict__ a, size_t n8, float* out) {
    float acc = 0.f;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < n8; i += U * stride) {
        float v[U][8];
#pragma unroll
        for (int u = 0; u < U; ++u) ld8(a + 8 * (i + u * stride), v[u]);
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int q = 0; q < 8; ++q) acc += v[u][q];
    }
    for (; i < n8; i += stride) { float v[8]; ld8(a + 8 * i, v); for (int q = 0; q < 8; ++q) acc += v[q]; }
    if (acc == 12345.f) *out = acc;
}

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int kStages, int kChunk>
__global__ void __launch_bounds__(64) bulk_read(const float* __restrict__ a, size_t nchunks, float* out) {
    extern __shared__ __align__(1024) unsigned char sm[];
    uint64_t* full = reinterpret_cast<uint64_t*>(sm + (size_t)kStages * kChunk);
    uint64_t* empty = full + kStages;
    if (threadIdx.x == 0) {
        for (int q = 0; q < kStages; ++q) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(full + q)));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(su(empty + q)));
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        int n = 0;
        for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++n) {
            const int st = n % kStages;
            const uint32_t ph = ((uint32_t)(n / kStages) & 1u) ^ 1u;
            asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W;\n}"
                         :: "r"(su(empty + st)), "r"(ph) : "memory");
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(su(full + st)), "r"(kChunk) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         :: "r"(su(sm + (size_t)st * kChunk)), "l"(a + c * (kChunk / 4)), "r"(kChunk), "r"(su(full + st)) : "memory");
        }
    } else if (threadIdx.x == 32) {
        int n = 0;
        float acc = 0.f;
        for (size_t c = blockIdx.x; c < nchunks; c += gridDim.x, ++n) {
            const int st = n % kStages;
            const uint32_t ph = (uint32_t)(n / kStages) & 1u;
            asm volatile("{\n.reg .pred P;\nW2: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n@!P bra W2;\n}"
                         :: "r"(su(full + st)), "r"(ph) : "memory");
            acc += reinterpret_cast<const float*>(sm + (size_t)st * kChunk)[0];
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(su(empty + st)) : "memory");
        }
        if (acc == 12345.f) *out = acc;
    }
}

__global__ void fill_rand(float* a, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x)
        a[i] = 0.25f + 0.5f * (float)((i * 2654435761u) % 1000003) / 1000003.f;
}

int main(int argc, char** argv) {
    const bool rnd = argc > 1 && argv[1][0] == 'r';         // "r": non-zero pseudo-random data
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const size_t bytes = (size_t)1 << 30;                     // 1 GiB, >> L2
    float* a; float* out;
    cudaMalloc(&a, bytes); cudaMalloc(&out, 4);
    cudaMemset(a, 0, bytes);
    if (rnd) fill_rand<<<1184, 256>>>(a, bytes / 4);
    printf("data: %s\n", rnd ? "pseudo-random floats in [0.25, 0.75)" : "zeros");
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    auto timeit = [&](const char* name, auto launch) {
        launch(); cudaDeviceSynchronize();
        float best = 1e9;
        for (int r = 0; r < 10; ++r) {
            cudaEventRecord(e0); launch(); cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms;
        }
        printf("%-40s %8.1f us  %7.0f GB/s  (%s)\n", name, best * 1e3, bytes / (best * 1e-3) / 1e9,
               cudaGetErrorString(cudaGetLastError()));
    };
    const size_t n8 = bytes / 32;
    for (int per : {4, 8, 16})
        for (int thr : {256, 512}) {
            char nm[64]; snprintf(nm, 64, "ldg256 U4 %dx%d blocks/SM thr=%d", per, sms, thr);
            timeit(nm, [&] { ldg_read<4><<<per * sms, thr>>>(a, n8, out); });
        }
    {
        constexpr int S = 6, C = 32768;
        auto k = bulk_read<S, C>;
        const int smem = S * C + 2 * S * 8;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        for (int per : {1}) {
            char nm[64]; snprintf(nm, 64, "bulk ring 6x32K, %d CTA/SM", per);
            timeit(nm, [&] { k<<<per * sms, 64, smem>>>(a, bytes / C, out); });
        }
    }
    {
        constexpr int S = 5, C = 16384;
        auto k = bulk_read<S, C>;
        const int smem = S * C + 2 * S * 8;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        for (int per : {1, 2}) {
            char nm[64]; snprintf(nm, 64, "bulk ring 5x16K, %d CTA/SM", per);
            timeit(nm, [&] { k<<<per * sms, 64, smem>>>(a, bytes / C, out); });
        }
    }
    {
        constexpr int S = 12, C = 16384;
        auto k = bulk_read<S, C>;
        const int smem = S * C + 2 * S * 8;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        timeit("bulk ring 12x16K, 1 CTA/SM", [&] { k<<<sms, 64, smem>>>(a, bytes / C, out); });
    }
    // copy for reference (read + write bytes)
    float* b; cudaMalloc(&b, bytes);
    timeit("cudaMemcpy D2D (counting 1x bytes)", [&] { cudaMemcpyAsync(b, a, bytes, cudaMemcpyDeviceToDevice); });
    return 0;
}
