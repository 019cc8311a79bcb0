// Roofline microbenchmarks for the denominators SURVEY.md §7 step 0 asks for:
// FP32 FFMA / packed FFMA2 / FADD2 issue rates, MUFU (XU) rates, and HBM
// read / write / copy bandwidth. Standalone tool (not part of liblime.so).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o microbench microbench.cu
// Output: one JSON object per line.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ unsigned long long f2u(float2 v) { unsigned long long r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(v.x), "f"(v.y)); return r; }
__device__ __forceinline__ float2 u2f(unsigned long long r) { float2 v; asm("mov.b64 {%0,%1}, %2;" : "=f"(v.x), "=f"(v.y) : "l"(r)); return v; }
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) { unsigned long long d; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(f2u(a)), "l"(f2u(b)), "l"(f2u(c))); return u2f(d); }
__device__ __forceinline__ float2 fadd2(float2 a, float2 b) { unsigned long long d; asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(f2u(a)), "l"(f2u(b))); return u2f(d); }
__device__ __forceinline__ float rsq(float x) { float y; asm volatile("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ float ex2(float x) { float y; asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }

__device__ unsigned long long g_cycles[4096];

constexpr int CH = 8;  // independent chains per thread

__global__ void k_ffma(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = threadIdx.x * 1e-3f + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = fmaf(x[c], a, b);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__global__ void k_ffma2(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
    const float2 A = make_float2(a, a), B = make_float2(b, b);
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ffma2(x[c], A, B);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

// FFMA2 whose scalar operands are compile-time constants (ptxas encodes them as immediates)
__global__ void k_ffma2_imm(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ffma2(x[c], make_float2(0.999f, 0.999f), make_float2(1e-3f, 1e-3f));
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
// FFMA2 with one 32-bit register broadcast operand (.F32) and one pair
__global__ void k_ffma2_bcast(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
    float av = a + threadIdx.x * 1e-9f;
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
    const float2 B = make_float2(b + threadIdx.x * 1e-9f, b);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ffma2(x[c], make_float2(av, av), B);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
// FADD2 with an immediate (the 1.5*2^23 rounding trick)
__global__ void k_fadd2_imm(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = fadd2(x[c], make_float2(1e-3f, 1e-3f));
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
__global__ void k_fadd2(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
    const float2 A = make_float2(a, b);
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = fadd2(x[c], A);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__global__ void k_rsq(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 1.0f + threadIdx.x * 1e-3f + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = rsq(x[c]);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__global__ void k_ex2(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 0.5f + threadIdx.x * 1e-6f + c * 1e-3f;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ex2(x[c]) * 0.25f;
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__device__ __forceinline__ float sinf_a(float x) { float y; asm volatile("sin.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ float cosf_a(float x) { float y; asm volatile("cos.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
// sin.approx = FMUL.RZ (radians -> turns, FMA pipe) + MUFU.SIN; the chain keeps x in [-1, 1]
__global__ void k_sin(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 0.3f + threadIdx.x * 1e-6f + c * 1e-3f;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = sinf_a(x[c]);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
// sin and cos of the same argument (the MRI-Q pattern): 2 MUFU per iteration and channel
__global__ void k_sincos(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 0.3f + threadIdx.x * 1e-6f + c * 1e-3f;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = sinf_a(x[c]) + cosf_a(x[c]) * 0.5f;
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
__device__ __forceinline__ float lg2f(float x) { float y; asm volatile("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__device__ __forceinline__ float rcpf(float x) { float y; asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
__global__ void k_lg2(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 3.0f + threadIdx.x * 1e-3f + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = lg2f(x[c]) + 2.5f;
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}
__global__ void k_rcp(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = 1.5f + threadIdx.x * 1e-3f + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = rcpf(x[c]);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

// FFMA2 whose three operands are distinct register pairs (the N-Body accumulate shape) vs the
// uniform-operand FFMA2 above: exposes register-file bank limits of 6-register FFMA2 reads.
__global__ void k_ffma2_3reg(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH], p[CH], q[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
        p[c] = make_float2(a + c * 1e-3f, a - c * 1e-3f);
        q[c] = make_float2(b * c, b + c);
    }
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ffma2(p[c], q[c], x[c]);
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__global__ void k_dfma(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    double x[CH];
    const double A = a, B = b;
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = threadIdx.x * 1e-3 + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = fma(x[c], A, B);
    double s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.0) out[0] = (float)s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

// 8 FFMA2 chains + 4 DFMA chains per iteration: if the FP64 pipe runs beside the FP32 pipe, time
// stays at the FFMA2-only time (lane_ops counted = FP32 lanes only).
__global__ void k_mix(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float2 x[CH];
    double y[4];
    const float2 A = make_float2(a, a), B = make_float2(b, b);
    const double Ad = a, Bd = b;
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = make_float2(threadIdx.x * 1e-3f + c, c);
#pragma unroll
    for (int c = 0; c < 4; ++c) y[c] = threadIdx.x * 1e-3 + c;
    for (int i = 0; i < iters; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c) x[c] = ffma2(x[c], A, B);
#pragma unroll
        for (int c = 0; c < 4; ++c) y[c] = fma(y[c], Ad, Bd);
    }
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c].x + x[c].y;
    for (int c = 0; c < 4; ++c) s += (float)y[c];
    if (s == 12345.f) out[0] = s;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

// F2F.F64.F32 conversion rate
__global__ void k_f2d(float* out, float a, float b, int iters) {
    long long t0 = clock64();
    float x[CH];
    double acc = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = threadIdx.x * 1e-3f + c;
    for (int i = 0; i < iters; ++i)
#pragma unroll
        for (int c = 0; c < CH; ++c) { x[c] = (float)((double)x[c] * 0.999); }
    float s = 0;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += x[c];
    if (s == 12345.f) out[0] = s + (float)acc;
    if (threadIdx.x == 0) g_cycles[blockIdx.x] = clock64() - t0;
}

__global__ void k_read(const float4* __restrict__ in, size_t n4, float* out) {
    float4 acc = make_float4(0, 0, 0, 0);
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x) {
        float4 v;
        asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(in + i));
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    if (acc.x + acc.y + acc.z + acc.w == 12345.f) out[0] = 1;
}

__global__ void k_write(float4* __restrict__ o, size_t n4) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
        __stcs(o + i, make_float4(1, 2, 3, 4));
}

__global__ void k_copy(const float4* __restrict__ in, float4* __restrict__ o, size_t n4) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n4; i += (size_t)gridDim.x * blockDim.x)
        __stcs(o + i, __ldcs(in + i));
}

template <typename F>
static float time_it(F f, int reps) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    f();
    cudaDeviceSynchronize();
    float best = 1e30f;
    for (int r = 0; r < reps; ++r) {
        cudaEventRecord(a);
        f();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms; cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    return best;
}

int main() {
    int dev = 0, sms = 0, l2 = 0, clk = 0;
    CK(cudaGetDevice(&dev));
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    printf("{\"what\": \"device\", \"sms\": %d, \"l2_bytes\": %d, \"clock_khz_attr\": %d}\n", sms, l2, clk);
    float* out; CK(cudaMalloc(&out, 16));
    const int threads = 256, blocks = sms * 4, iters = 1 << 14;
    struct { const char* name; void (*k)(float*, float, float, int); double lane_ops_per_iter; } tests[] = {
        {"ffma", k_ffma, CH}, {"ffma2", k_ffma2, 2.0 * CH}, {"fadd2", k_fadd2, 2.0 * CH},
        {"ffma2_imm", k_ffma2_imm, 2.0 * CH}, {"ffma2_bcast_reg", k_ffma2_bcast, 2.0 * CH},
        {"fadd2_imm", k_fadd2_imm, 2.0 * CH},
        {"mufu_rsq", k_rsq, CH}, {"mufu_ex2(+fmul)", k_ex2, CH},
        {"ffma2_3reg_pairs", k_ffma2_3reg, 2.0 * CH},
        {"mufu_lg2(+fadd)", k_lg2, CH}, {"mufu_rcp", k_rcp, CH},
        {"mufu_sin(+fmul.rz)", k_sin, CH}, {"mufu_sin+cos(+2 fmul.rz, ffma)", k_sincos, 2.0 * CH},
        {"dfma(fp64 lanes)", k_dfma, CH}, {"ffma2+dfma(fp32 lanes only)", k_mix, 2.0 * CH},
        {"f32->f64->f32 roundtrips(+dmul)", k_f2d, CH},
    };
    for (auto& t : tests) {
        float ms = time_it([&] { t.k<<<blocks, threads>>>(out, 0.999f, 1e-3f, iters); }, 5);
        unsigned long long cyc[4096];
        cudaMemcpyFromSymbol(cyc, g_cycles, sizeof(unsigned long long) * blocks);
        unsigned long long cmax = 0;
        for (int i = 0; i < blocks; ++i) if (cyc[i] > cmax) cmax = cyc[i];
        double ops = (double)blocks * threads * iters * t.lane_ops_per_iter;
        double ghz = cmax / (ms * 1e6);
        printf("{\"what\": \"%s\", \"ms\": %.4f, \"lane_ops_per_s\": %.4e, \"sm_ghz_effective\": %.3f, \"lane_ops_per_clk_per_sm\": %.2f}\n",
               t.name, ms, ops / (ms * 1e-3), ghz, ops / ((double)cmax * sms));
    }
    size_t bytes = 1ull << 30, n4 = bytes / 16;
    float4 *a, *b;
    CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes));
    cudaMemset(a, 0, bytes); cudaMemset(b, 0, bytes);
    int gb = sms * 8;
    float ms = time_it([&] { k_read<<<gb, 256>>>(a, n4, out); }, 10);
    printf("{\"what\": \"hbm_read\", \"GBps\": %.1f}\n", bytes / (ms * 1e6));
    ms = time_it([&] { k_write<<<gb, 256>>>(b, n4); }, 10);
    printf("{\"what\": \"hbm_write\", \"GBps\": %.1f}\n", bytes / (ms * 1e6));
    ms = time_it([&] { k_copy<<<gb, 256>>>(a, b, n4); }, 10);
    printf("{\"what\": \"hbm_copy_rw\", \"GBps\": %.1f}\n", 2.0 * bytes / (ms * 1e6));
    return 0;
}
