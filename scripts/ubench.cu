// ubench.cu -- per-SM throughput of the per-element operations of the K.l pass on
// B200 (DFMA, fp32->fp64 conversion two ways, MUFU.EX2, FFMA2, SHFL), in results
// per clock per SM: 148 SMs x 4 CTAs x 256 threads, 8 independent chains per
// thread, timed with cudaEvents and converted with the measured SM clock.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o scripts/ubench scripts/ubench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kIters = 4096;

template <int kOp>
__global__ void __launch_bounds__(256) bench(float* out, float seed) {
    double d[8];
    float f[8];
    uint32_t u[8];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
        f[q] = seed + threadIdx.x * 1e-3f + q;
        d[q] = f[q];
        u[q] = __float_as_uint(f[q]);
    }
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (kOp == 0) d[q] = __fma_rn(d[q], 0.999999, 1e-9);                       // DFMA
            if (kOp == 1) { d[q] = __dadd_rn(d[q], (double)f[q]); f[q] = __fadd_rn(f[q], 1e-7f); }   // F2F + DADD
            if (kOp == 2) {                                                              // int conv + DADD
                const uint32_t x = u[q];
                d[q] = __dadd_rn(d[q], __hiloint2double((int)((x >> 3) + 0x38000000u), (int)(x << 29)));
                u[q] = x + 1u;
            }
            if (kOp == 3) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(f[q])); f[q] = y * -0.5f; }
            if (kOp == 4) {                                                              // FFMA2
                unsigned long long a = ((unsigned long long)__float_as_uint(f[q]) << 32) | __float_as_uint(f[q]), r;
                asm volatile("fma.rn.f32x2 %0, %1, %1, %1;" : "=l"(r) : "l"(a));
                f[q] = __uint_as_float((uint32_t)r) * 0.5f;
            }
            if (kOp == 5) d[q] = __dadd_rn(d[q], 1e-9);                                  // DADD alone
            if (kOp == 6) f[q] += __shfl_xor_sync(0xffffffffu, f[q], 1 + q);            // SHFL + FADD
        }
    }
    float s = 0.f;
#pragma unroll
    for (int q = 0; q < 8; ++q) s += (float)d[q] + f[q] + (float)u[q];
    if (s == 1.2345f) out[0] = s;
}

template <int kOp>
void run(const char* name, int per_elem) {
    float* out;
    cudaMalloc(&out, 4);
    int sms = 0, clk = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    const int blocks = sms * 4;
    bench<kOp><<<blocks, 256>>>(out, 1.f);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    bench<kOp><<<blocks, 256>>>(out, 1.f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    const double ops = (double)blocks * 256 * kIters * 8;
    const double per_sm_per_clk = ops / (ms * 1e-3) / sms / (clk * 1e3);
    printf("%-28s %8.3f ms  %7.1f elem/clk/SM (at %d MHz nominal)  [%d instr/elem]\n", name, ms, per_sm_per_clk,
           clk / 1000, per_elem);
    cudaFree(out);
}

int main() {
    run<0>("DFMA", 1);
    run<5>("DADD", 1);
    run<1>("F2F.F64.F32 + DADD + FADD", 3);
    run<2>("LEA.HI+SHL conv + DADD + IADD", 4);
    run<3>("MUFU.EX2 + FMUL", 2);
    run<4>("FFMA2 + FMUL", 2);
    run<6>("SHFL + FADD", 2);
    return 0;
}
