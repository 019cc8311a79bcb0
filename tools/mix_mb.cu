// mix_mb.cu -- FP32-pipe ceiling of the N-Body inner-loop instruction mix (packed FFMA2 + MUFU.RSQ
// + LDS.128 broadcast), independent of the kernel's dependency structure.
// Per "source step" a thread issues F packed FFMA2 (two lanes each), M MUFU.RSQ and L LDS.128 of a
// broadcast address; the product loop (force_kernel, 4 targets/thread, mass factored) is
// F = 22, M = 4, L = 1. Every op feeds a chain that is consumed at the end, so nothing is dead.
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o mix_mb tools/mix_mb.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {
    unsigned long long r, x = *reinterpret_cast<unsigned long long*>(&a), y = *reinterpret_cast<unsigned long long*>(&b),
                          z = *reinterpret_cast<unsigned long long*>(&c);
    asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(x), "l"(y), "l"(z));
    return *reinterpret_cast<float2*>(&r);
}
__device__ __forceinline__ float rsq(float x) { float r; asm volatile("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x)); return r; }

template <int F, int M, int L, int CH>
__global__ void mix_kernel(float* out, int iters, float seed) {
    __shared__ float4 s[1024];
    for (int i = threadIdx.x; i < 1024; i += blockDim.x) s[i] = make_float4(seed * i, 1.f, 2.f, 3.f);
    __syncthreads();
    float2 acc[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) acc[c] = make_float2(seed + c, seed - c);
    float m[4] = {seed + 1.f, seed + 2.f, seed + 3.f, seed + 4.f};
    float2 k = make_float2(0.999f + threadIdx.x * 1e-9f, 1.001f), b = make_float2(1e-7f, 2e-7f * threadIdx.x);
    unsigned lacc = 0u;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int f = 0; f < F; ++f) acc[f % CH] = ffma2(acc[f % CH], k, b);
#pragma unroll
        for (int u = 0; u < M; ++u) m[u & 3] = rsq(m[u & 3]);
#pragma unroll
        for (int l = 0; l < L; ++l) { float4 v = s[(it + l) & 1023]; lacc ^= __float_as_uint(v.x); }
    }
    float r = __uint_as_float(lacc) + m[0] + m[1] + m[2] + m[3];
#pragma unroll
    for (int c = 0; c < CH; ++c) r += acc[c].x + acc[c].y;
    if (r == 123.456f) out[threadIdx.x] = r;
}

template <int F, int M, int L, int CH>
void run(const char* name, int block, int ctas_per_sm) {
    float* out;
    cudaMalloc(&out, 4096);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int grid = sms * ctas_per_sm, iters = 20000;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    mix_kernel<F, M, L, CH><<<grid, block>>>(out, 100, 1.f);
    cudaEventRecord(a);
    mix_kernel<F, M, L, CH><<<grid, block>>>(out, iters, 1.f);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    int clk_khz;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    const double lane_ops = 2.0 * F * 32.0 * (block / 32) * (double)grid * iters;
    const double per_clk_sm = lane_ops / (ms * 1e-3) / sms / (clk_khz * 1e3);
    printf("{\"what\": \"%s\", \"F\": %d, \"M\": %d, \"L\": %d, \"chains\": %d, \"block\": %d, \"ctas_per_sm\": %d, \"ms\": %.4f, "
           "\"fp32_lane_ops_per_clk_per_sm_at_max_clock\": %.2f, \"fp32_pipe_frac\": %.4f}\n",
           name, F, M, L, CH, block, ctas_per_sm, ms, per_clk_sm, per_clk_sm / 128.0);
    cudaFree(out);
}

int main() {
    run<22, 0, 0, 8>("ffma2 only", 512, 1);
    run<22, 4, 0, 8>("ffma2 + mufu (nbody 1m ratio)", 512, 1);
    run<22, 4, 1, 8>("ffma2 + mufu + lds (nbody 1m mix)", 512, 1);
    run<22, 4, 1, 8>("ffma2 + mufu + lds, 2 ctas", 512, 2);
    run<22, 4, 1, 8>("ffma2 + mufu + lds, 256x4", 256, 4);
    run<11, 2, 1, 6>("small-kernel mix (1 pair/lane)", 896, 1);
    run<22, 4, 0, 12>("ffma2 + mufu, 12 chains", 512, 1);
    run<44, 8, 1, 12>("ffma2 + mufu + lds x2 unroll", 512, 1);
    return 0;
}
