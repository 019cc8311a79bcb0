// HBM read-stream probe: why do three 64-MiB SoA streams (Black-Scholes inputs) read at only
// ~5.2 TB/s while one 1-GiB stream (reduce_sum) reads at ~6.2 TB/s?  Candidates: fixed
// launch/ramp/tail cost of a ~40-us kernel, DRAM channel aliasing between streams whose bases
// differ by a power of two, the dirty-L2 write-back left by a write flush, grid shape.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/hbm_probe tools/hbm_probe.cu
// Prints one JSON line per variant: best-of-12 microseconds and GB/s of algorithmic bytes.
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ float4 ldnc(const float4* p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}

// NS streams of n4 float4 each; grid-stride over the float4 index; U float4 per stream per
// thread per iteration (U consecutive grid-stride slots).
template <int NS, int U>
__global__ void read_streams(const float4* __restrict__ a, const float4* __restrict__ b,
                             const float4* __restrict__ c, int64_t n4, float* out) {
    const float4* p[3] = {a, b, c};
    float acc = 0.f;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
    for (; i + (U - 1) * stride < n4; i += U * stride) {
        float4 v[NS][U];
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int s = 0; s < NS; ++s) v[s][u] = ldnc(p[s] + i + u * stride);
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
            for (int s = 0; s < NS; ++s) acc += (v[s][u].x + v[s][u].y) + (v[s][u].z + v[s][u].w);
    }
    for (; i < n4; i += stride)
#pragma unroll
        for (int s = 0; s < NS; ++s) { float4 v = ldnc(p[s] + i); acc += (v.x + v.y) + (v.z + v.w); }
    if (acc == 1234.5f) out[0] = acc;
}

// AoSoA: groups of 3 float4 (S4 X4 T4) contiguous; one thread reads its 48-B group.
template <int U>
__global__ void read_aosoa(const float4* __restrict__ g, int64_t ngroups, float* out) {
    float acc = 0.f;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
    for (; i < ngroups; i += stride) {
        float4 v0 = ldnc(g + 3 * i), v1 = ldnc(g + 3 * i + 1), v2 = ldnc(g + 3 * i + 2);
        acc += (v0.x + v1.y) + (v2.z + v0.w) + (v1.x + v2.y) + (v0.z + v1.w) + (v2.x + v0.y) + (v1.z + v2.w);
    }
    if (acc == 1234.5f) out[0] = acc;
}

__global__ void read_flush(const float4* __restrict__ f, int64_t n4, float* out) {
    float acc = 0.f;
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n4;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        float4 v = ldnc(f + i);
        acc += v.x + v.w;
    }
    if (acc == 1234.5f) out[0] = acc;
}
__global__ void empty_kernel() {}

static char* g_flush;
static const size_t FLUSH = 512ull << 20;
static float* g_out;
static cudaEvent_t ea, eb;

template <class F>
static void run(const char* name, double bytes, int flush_mode, F launch) {
    float best = 1e9f;
    for (int r = 0; r < 12; ++r) {
        if (flush_mode == 0) cudaMemsetAsync(g_flush, r, FLUSH);
        else read_flush<<<148 * 8, 256>>>(reinterpret_cast<const float4*>(g_flush), FLUSH / 16, g_out);
        cudaEventRecord(ea);
        launch();
        cudaEventRecord(eb);
        cudaEventSynchronize(eb);
        float ms;
        cudaEventElapsedTime(&ms, ea, eb);
        if (r >= 2 && ms < best) best = ms;
    }
    printf("{\"variant\": \"%s\", \"flush\": \"%s\", \"us\": %.2f, \"GBps\": %.1f}\n", name,
           flush_mode == 0 ? "write" : "read", best * 1e3, bytes / (best * 1e-3) / 1e9);
    fflush(stdout);
}

int main() {
    cudaMalloc(&g_flush, FLUSH);
    cudaMemset(g_flush, 1, FLUSH);
    cudaMalloc(&g_out, 64);
    cudaEventCreate(&ea);
    cudaEventCreate(&eb);
    const int64_t n = 1 << 24;              // options
    const int64_t n4 = n / 4;
    const size_t sb = n * 4;                 // bytes per stream
    // production-like: three separate allocations
    float4 *S, *X, *T;
    cudaMalloc(&S, sb); cudaMalloc(&X, sb); cudaMalloc(&T, sb);
    cudaMemset(S, 0, sb); cudaMemset(X, 0, sb); cudaMemset(T, 0, sb);
    printf("{\"bases\": [\"%p\", \"%p\", \"%p\"]}\n", (void*)S, (void*)X, (void*)T);
    // one big buffer for skewed / single-stream / AoSoA / large-n variants
    const size_t big_bytes = 4 * sb + (64ull << 20);
    char* big;
    cudaMalloc(&big, big_bytes);
    cudaMemset(big, 0, big_bytes);
    const double B = 3.0 * sb;

    run("empty kernel", 0, 0, [&] { empty_kernel<<<1, 32>>>(); });
    for (int fm = 0; fm < 2; ++fm) {
        run("3 streams separate allocs 592x256", B, fm,
            [&] { read_streams<3, 1><<<592, 256>>>(S, X, T, n4, g_out); });
        run("1 stream 3x64MiB contiguous 592x256", B, fm,
            [&] { read_streams<1, 1><<<592, 256>>>(reinterpret_cast<float4*>(big), nullptr, nullptr, 3 * n4, g_out); });
    }
    const int fm = 1;
    for (int grid : {148 * 2, 148 * 4, 148 * 8, 148 * 16})
        for (int thr : {256, 512}) {
            if (grid * thr > 148 * 2048 * 2) continue;
            char nm[128];
            snprintf(nm, sizeof nm, "3 streams separate allocs %dx%d", grid, thr);
            run(nm, B, fm, [&] { read_streams<3, 1><<<grid, thr>>>(S, X, T, n4, g_out); });
            snprintf(nm, sizeof nm, "3 streams separate allocs U2 %dx%d", grid, thr);
            run(nm, B, fm, [&] { read_streams<3, 2><<<grid, thr>>>(S, X, T, n4, g_out); });
        }
    for (size_t skew : {size_t(0), size_t(256), size_t(4096), size_t(65536 + 256), size_t(1 << 20), size_t(3 << 20),
                        size_t(5 << 20) + 4096}) {
        float4* a = reinterpret_cast<float4*>(big);
        float4* b = reinterpret_cast<float4*>(big + sb + skew);
        float4* c = reinterpret_cast<float4*>(big + 2 * (sb + skew));
        char nm[128];
        snprintf(nm, sizeof nm, "3 streams one alloc, skew %zu B 592x256", skew);
        run(nm, B, fm, [&] { read_streams<3, 1><<<592, 256>>>(a, b, c, n4, g_out); });
    }
    run("AoSoA 48-B groups 592x256", B, fm,
        [&] { read_aosoa<1><<<592, 256>>>(reinterpret_cast<float4*>(big), n4, g_out); });
    run("AoSoA 48-B groups 1184x256", B, fm,
        [&] { read_aosoa<1><<<1184, 256>>>(reinterpret_cast<float4*>(big), n4, g_out); });
    // size dependence: one stream of 4x, 1x, 1/4x the bytes
    for (int64_t m : {n4 / 4, n4, 3 * n4, 4 * n4 + (16 << 20) / 16}) {
        char nm[128];
        snprintf(nm, sizeof nm, "1 stream %lld MiB 592x256", (long long)(m * 16 >> 20));
        run(nm, m * 16.0, fm, [&] { read_streams<1, 1><<<592, 256>>>(reinterpret_cast<float4*>(big), nullptr, nullptr, m, g_out); });
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("{\"status\": \"%s\"}\n", cudaGetErrorString(e));
    return 0;
}
