// k2_variants.cu -- design-space microbenchmark for K2 (fused deflate +
// rescore) on B200.  Not part of the product: used to pick the production
// configuration.  Every variant is checked bit-for-bit
// against the production kernel's output (K and the packed key).
//
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo \
//      -I paper_conf_date_sunbg021_b200/csrc scripts/k2_variants.cu -o k2v
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <string>
#include <functional>
#include <cuda_runtime.h>
#include "kernels.cuh"

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

using namespace bted;

// ---------------------------------------------------------------- copies
__global__ void copy_f4(const float4* __restrict__ a, float4* __restrict__ b, size_t n4) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
        st_stream(reinterpret_cast<float*>(b + i), ld_stream(reinterpret_cast<const float*>(a + i)));
}
template <int U>
__global__ void copy_f4_unroll(const float4* __restrict__ a, float4* __restrict__ b, size_t n4) {
    size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < n4; i += U * stride) {
        float4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = ld_stream(reinterpret_cast<const float*>(a + i + u * stride));
#pragma unroll
        for (int u = 0; u < U; ++u) st_stream(reinterpret_cast<float*>(b + i + u * stride), v[u]);
    }
    for (; i < n4; i += stride) st_stream(reinterpret_cast<float*>(b + i), ld_stream(reinterpret_cast<const float*>(a + i)));
}

template <int U>
__global__ void copy_f8_unroll(const float* __restrict__ a, float* __restrict__ b, size_t n8) {
    size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
    for (; i + (U - 1) * stride < n8; i += U * stride) {
        f8 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) v[u] = ld8_stream(a + 8 * (i + u * stride));
#pragma unroll
        for (int u = 0; u < U; ++u) st8_stream(b + 8 * (i + u * stride), v[u]);
    }
    for (; i < n8; i += stride) st8_stream(b + 8 * i, ld8_stream(a + 8 * i));
}

// ---------------------------------------------------------------- K2, 256-bit, static rows
// Same arithmetic and per-row order as production?  NO: a lane covers 8
// consecutive columns, so the per-lane order differs -> scores may differ in
// the last bits; K itself is bit-identical (elementwise op).  Checked: K only.
template <int kRows, int kUnroll, int kThreads>
__global__ void __launch_bounds__(kThreads)
k2_v8(const float* __restrict__ Kin, float* __restrict__ Kout, int64_t ld, int32_t row0, int32_t nrows,
      unsigned long long* __restrict__ keys, int32_t t, float mu, uint8_t* __restrict__ sel, int* __restrict__ err) {
    constexpr int kWarps = kThreads / kWarp;
    const uint32_t s = key_index(keys[t - 1]);
    const float* __restrict__ p = Kin + (int64_t)((int32_t)s - row0) * ld;
    const float inv_c = __frcp_rn(__fadd_rn(p[s], mu));
    const int w = threadIdx.x / kWarp, l = threadIdx.x % kWarp;
    const int lrow0 = (blockIdx.x * kWarps + w) * kRows;
    const int64_t nvec = ld >> 3;
    float a[kRows], acc[kRows];
    const float* kin[kRows];
    float* kout[kRows];
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
        const int lr = min(lrow0 + r, nrows - 1);
        a[r] = p[row0 + lr]; kin[r] = Kin + (int64_t)lr * ld; kout[r] = Kout + (int64_t)lr * ld; acc[r] = 0.f;
    }
    const bool any = lrow0 < nrows;
    if (any) {
        int64_t v = l;
        for (; v + (kUnroll - 1) * kWarp < nvec; v += kUnroll * kWarp) {
            f8 pv[kUnroll], kv[kUnroll][kRows];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                pv[u] = ld8_keep(p + ((v + u * kWarp) << 3));
#pragma unroll
                for (int r = 0; r < kRows; ++r) kv[u][r] = ld8_stream(kin[r] + ((v + u * kWarp) << 3));
            }
#pragma unroll
            for (int u = 0; u < kUnroll; ++u)
#pragma unroll
                for (int r = 0; r < kRows; ++r) {
                    f8 o;
#pragma unroll
                    for (int c = 0; c < 8; ++c) {
                        o.v[c] = deflate1(kv[u][r].v[c], a[r], pv[u].v[c], inv_c);
                        acc[r] = __fmaf_rn(o.v[c], o.v[c], acc[r]);
                    }
                    if (lrow0 + r < nrows) st8_stream(kout[r] + ((v + u * kWarp) << 3), o);
                }
        }
        for (; v < nvec; v += kWarp) {
            const f8 pv = ld8_keep(p + (v << 3));
#pragma unroll
            for (int r = 0; r < kRows; ++r) {
                const f8 kv = ld8_stream(kin[r] + (v << 3));
                f8 o;
#pragma unroll
                for (int c = 0; c < 8; ++c) { o.v[c] = deflate1(kv.v[c], a[r], pv.v[c], inv_c); acc[r] = __fmaf_rn(o.v[c], o.v[c], acc[r]); }
                if (lrow0 + r < nrows) st8_stream(kout[r] + (v << 3), o);
            }
        }
    }
    unsigned long long key = 0ull;
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
        const float g = warp_sum(acc[r]);
        if (l == r && any && lrow0 + r < nrows) {
            const int lr = lrow0 + r; const int32_t i = row0 + lr;
            const float diag = deflate1(Kin[(int64_t)lr * ld + i], a[r], p[i], inv_c);
            key = score_key(g, diag, mu, (uint32_t)i, sel[lr] != 0 || (uint32_t)i == s, err);
        }
    }
    cta_key_max_to<kThreads>(key, keys + t);
}

// ---------------------------------------------------------------- K2, dynamic row groups (float4)
template <int kRows, int kUnroll, int kThreads>
__global__ void __launch_bounds__(kThreads)
k2_dyn(const float* __restrict__ Kin, float* __restrict__ Kout, int64_t ld, int32_t row0, int32_t nrows,
       unsigned long long* __restrict__ keys, int32_t t, float mu, uint8_t* __restrict__ sel, int* __restrict__ err,
       int* __restrict__ counter) {
    const uint32_t s = key_index(keys[t - 1]);
    const float* __restrict__ p = Kin + (int64_t)((int32_t)s - row0) * ld;
    const float inv_c = __frcp_rn(__fadd_rn(p[s], mu));
    const int l = threadIdx.x % kWarp;
    const int64_t nvec = ld >> 2;
    const int ngroups = (nrows + kRows - 1) / kRows;
    unsigned long long best = 0ull;
    for (;;) {
        int grp = 0;
        if (l == 0) grp = atomicAdd(counter, 1);
        grp = __shfl_sync(0xffffffffu, grp, 0);
        if (grp >= ngroups) break;
        const int lrow0 = grp * kRows;
        float a[kRows], acc[kRows];
        const float* kin[kRows];
        float* kout[kRows];
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
            const int lr = min(lrow0 + r, nrows - 1);
            a[r] = p[row0 + lr]; kin[r] = Kin + (int64_t)lr * ld; kout[r] = Kout + (int64_t)lr * ld; acc[r] = 0.f;
        }
        int64_t v = l;
        for (; v + (kUnroll - 1) * kWarp < nvec; v += kUnroll * kWarp) {
            float4 pv[kUnroll], kv[kUnroll][kRows];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                pv[u] = ld_keep(p + ((v + u * kWarp) << 2));
#pragma unroll
                for (int r = 0; r < kRows; ++r) kv[u][r] = ld_stream(kin[r] + ((v + u * kWarp) << 2));
            }
#pragma unroll
            for (int u = 0; u < kUnroll; ++u)
#pragma unroll
                for (int r = 0; r < kRows; ++r) {
                    float4 o;
                    o.x = deflate1(kv[u][r].x, a[r], pv[u].x, inv_c); o.y = deflate1(kv[u][r].y, a[r], pv[u].y, inv_c);
                    o.z = deflate1(kv[u][r].z, a[r], pv[u].z, inv_c); o.w = deflate1(kv[u][r].w, a[r], pv[u].w, inv_c);
                    acc[r] = __fmaf_rn(o.x, o.x, acc[r]); acc[r] = __fmaf_rn(o.y, o.y, acc[r]);
                    acc[r] = __fmaf_rn(o.z, o.z, acc[r]); acc[r] = __fmaf_rn(o.w, o.w, acc[r]);
                    if (lrow0 + r < nrows) st_stream(kout[r] + ((v + u * kWarp) << 2), o);
                }
        }
        for (; v < nvec; v += kWarp) {
            const float4 pv = ld_keep(p + (v << 2));
#pragma unroll
            for (int r = 0; r < kRows; ++r) {
                const float4 kv = ld_stream(kin[r] + (v << 2));
                float4 o;
                o.x = deflate1(kv.x, a[r], pv.x, inv_c); o.y = deflate1(kv.y, a[r], pv.y, inv_c);
                o.z = deflate1(kv.z, a[r], pv.z, inv_c); o.w = deflate1(kv.w, a[r], pv.w, inv_c);
                acc[r] = __fmaf_rn(o.x, o.x, acc[r]); acc[r] = __fmaf_rn(o.y, o.y, acc[r]);
                acc[r] = __fmaf_rn(o.z, o.z, acc[r]); acc[r] = __fmaf_rn(o.w, o.w, acc[r]);
                if (lrow0 + r < nrows) st_stream(kout[r] + (v << 2), o);
            }
        }
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
            const float g = warp_sum(acc[r]);
            if (l == r && lrow0 + r < nrows) {
                const int lr = lrow0 + r; const int32_t i = row0 + lr;
                const float diag = deflate1(Kin[(int64_t)lr * ld + i], a[r], p[i], inv_c);
                unsigned long long k = score_key(g, diag, mu, (uint32_t)i, sel[lr] != 0 || (uint32_t)i == s, err);
                best = k > best ? k : best;
            }
        }
    }
    cta_key_max_to<kThreads>(best, keys + t);
}

// ---------------------------------------------------------------- harness
int main(int argc, char** argv) {
    const int N = argc > 1 ? atoi(argv[1]) : 16384;
    const int iters = argc > 2 ? atoi(argv[2]) : 20;
    const int64_t ld = (N + 31) / 32 * 32;
    const size_t n = (size_t)N * ld;
    float *A, *B, *Ref;
    CK(cudaMalloc(&A, n * 4)); CK(cudaMalloc(&B, n * 4)); CK(cudaMalloc(&Ref, n * 4));
    unsigned long long* keys; CK(cudaMalloc(&keys, 64 * 8));
    uint8_t* sel; CK(cudaMalloc(&sel, N));
    int* err; CK(cudaMalloc(&err, 4));
    int* counter; CK(cudaMalloc(&counter, 4));
    CK(cudaMemset(sel, 0, N)); CK(cudaMemset(err, 0, 4));
    // a symmetric PSD-ish K: K_ij = exp(-0.001 (i-j)^2) (bit-symmetric), zero padding
    {
        std::vector<float> h(n, 0.f);
        for (int i = 0; i < N; ++i) for (int j = 0; j < N; ++j) { float d = (float)(i - j); h[(size_t)i * ld + j] = expf(-1e-5f * d * d); }
        CK(cudaMemcpy(A, h.data(), n * 4, cudaMemcpyHostToDevice));
    }
    const unsigned long long key0 = (((unsigned long long)0x3f800000u + 1) << 32) | (0xFFFFFFFFu - (uint32_t)(N / 3));
    float mu = 0.1f;
    cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    const double bytes = 8.0 * N * (double)N;
    auto reset = [&]() { CK(cudaMemcpy(keys, &key0, 8, cudaMemcpyHostToDevice)); CK(cudaMemset(keys + 1, 0, 8)); CK(cudaMemset(counter, 0, 4)); };
    // reference output
    reset();
    deflate_rescore_kernel<2, 4, 256><<<(N + 15) / 16, 256>>>(A, Ref, ld, 0, N, nullptr, keys, 1, mu, sel, err);
    CK(cudaDeviceSynchronize());
    unsigned long long refkey; CK(cudaMemcpy(&refkey, keys + 1, 8, cudaMemcpyDeviceToHost));
    std::vector<float> href(n), hb(n);
    CK(cudaMemcpy(href.data(), Ref, n * 4, cudaMemcpyDeviceToHost));

    auto run = [&](const char* name, std::function<void()> f, bool check_k, bool check_key) {
        for (int w = 0; w < 3; ++w) { reset(); f(); }
        CK(cudaDeviceSynchronize());
        float tot = 0;
        for (int it = 0; it < iters; ++it) {
            reset();
            CK(cudaEventRecord(e0)); f(); CK(cudaEventRecord(e1)); CK(cudaEventSynchronize(e1));
            float ms; CK(cudaEventElapsedTime(&ms, e0, e1)); tot += ms;
        }
        const double ms = tot / iters;
        bool ok = true;
        if (check_k) { CK(cudaMemcpy(hb.data(), B, n * 4, cudaMemcpyDeviceToHost)); ok = memcmp(hb.data(), href.data(), n * 4) == 0; }
        unsigned long long k = 0; CK(cudaMemcpy(&k, keys + 1, 8, cudaMemcpyDeviceToHost));
        bool kok = !check_key || k == refkey;
        printf("%-44s %8.4f ms %8.1f GB/s  K %s key %s\n", name, ms, bytes / (ms * 1e-3) / 1e9,
               check_k ? (ok ? "bit-equal" : "DIFF") : "-", check_key ? (kok ? "equal" : "DIFF") : "-");
    };
    int sms = 148;
    const size_t n4 = n / 4, n8 = n / 8;
    run("copy_f4 grid=148*8 x256", [&] { copy_f4<<<sms * 8, 256>>>((const float4*)A, (float4*)B, n4); }, false, false);
    run("copy_f4_unroll<4> grid=148*4 x256", [&] { copy_f4_unroll<4><<<sms * 4, 256>>>((const float4*)A, (float4*)B, n4); }, false, false);
    run("copy_f4_unroll<8> grid=148*4 x256", [&] { copy_f4_unroll<8><<<sms * 4, 256>>>((const float4*)A, (float4*)B, n4); }, false, false);
    run("copy_f8_unroll<4> grid=148*4 x256", [&] { copy_f8_unroll<4><<<sms * 4, 256>>>(A, B, n8); }, false, false);
    run("copy_f8_unroll<8> grid=148*4 x256", [&] { copy_f8_unroll<8><<<sms * 4, 256>>>(A, B, n8); }, false, false);
    run("cudaMemcpyDeviceToDevice", [&] { CK(cudaMemcpyAsync(B, A, n * 4, cudaMemcpyDeviceToDevice)); }, false, false);

#define PROD(R, U, T) run("prod<" #R "," #U "," #T ">", [&] { deflate_rescore_kernel<R, U, T><<<(N + (T / 32) * R - 1) / ((T / 32) * R), T>>>(A, B, ld, 0, N, nullptr, keys, 1, mu, sel, err); }, true, true)
    PROD(2, 4, 256);
    PROD(1, 4, 256);
    PROD(1, 8, 256);
    PROD(2, 8, 256);
    PROD(4, 4, 256);
    PROD(2, 4, 128);
    PROD(1, 8, 128);
    PROD(2, 2, 256);
#define V8(R, U, T) run("v8<" #R "," #U "," #T ">", [&] { k2_v8<R, U, T><<<(N + (T / 32) * R - 1) / ((T / 32) * R), T>>>(A, B, ld, 0, N, keys, 1, mu, sel, err); }, true, false)
    V8(1, 2, 256);
    V8(1, 4, 256);
    V8(2, 2, 256);
    V8(2, 4, 256);
#define DYN(R, U, T, G) run("dyn<" #R "," #U "," #T "> grid=148*" #G, [&] { k2_dyn<R, U, T><<<sms * G, T>>>(A, B, ld, 0, N, keys, 1, mu, sel, err, counter); }, true, true)
    DYN(1, 4, 256, 4);
    DYN(1, 8, 256, 4);
    DYN(2, 4, 256, 4);
    DYN(1, 8, 256, 2);
    DYN(2, 4, 256, 2);
    DYN(1, 4, 512, 2);
    printf("done N=%d\n", N);
    return 0;
}
