// In-situ all-gather microbenchmark for the persistent config-1 step: 148 CTAs (one per SM), each
// owns 28 of 4096 bodies; per iteration: write own bodies (16 B each), grid barrier, then every CTA
// loads all 64 KB into shared memory. Cycles of the load phase per CTA (median over iterations),
// for write/read flavours and an optional delay between barrier and load.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/allgather_mb tools/allgather_mb.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cstdint>

__device__ __forceinline__ void grid_barrier(unsigned* arrivals, unsigned target) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(arrivals) : "memory");
        unsigned v;
        do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(arrivals) : "memory"); }
        while (static_cast<int>(v - target) < 0);
    }
    __syncthreads();
}

template <int WMODE, int RMODE, int DELAY>
__global__ void __launch_bounds__(896, 1) ag(float4* pos, unsigned* bar, long long* cyc, int iters) {
    extern __shared__ __align__(16) float4 s[];
    const int n = 4096;
    const int b0 = n * blockIdx.x / gridDim.x, b1 = n * (blockIdx.x + 1) / gridDim.x;
    long long tot = 0;
    unsigned target = 0;
    for (int it = 0; it < iters; ++it) {
        const int t = b0 + threadIdx.x;
        if (t < b1) {
            float4 v = make_float4(it, t, 1.f, 2.f);
            if (WMODE == 0) __stcg(pos + t, v);
            else pos[t] = v;
        }
        target += gridDim.x;
        grid_barrier(bar, target);
        if (DELAY) __nanosleep(DELAY);
        const long long t0 = clock64();
        float4 v[5];
#pragma unroll
        for (int k = 0; k < 5; ++k) {
            int i = threadIdx.x + k * 896;
            if (i < n) {
                if (RMODE == 0) v[k] = __ldcg(pos + i);
                else {
                    asm volatile("ld.relaxed.gpu.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v[k].x), "=f"(v[k].y), "=f"(v[k].z), "=f"(v[k].w) : "l"(pos + i));
                }
            }
        }
#pragma unroll
        for (int k = 0; k < 5; ++k) { int i = threadIdx.x + k * 896; if (i < n) s[i + i / 64] = v[k]; }
        __syncthreads();
        if (it >= 2) tot += clock64() - t0;
        target += gridDim.x;
        grid_barrier(bar, target);
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = tot / (iters - 2);
}

template <class F>
void run(const char* name, F kern, float4* pos, unsigned* bar, long long* cyc) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 118784);
    cudaMemset(bar, 0, 8);
    void* args[] = {&pos, &bar, &cyc, nullptr};
    int iters = 20;
    args[3] = &iters;
    cudaLaunchCooperativeKernel((void*)kern, 148, 896, args, 118784, 0);
    cudaDeviceSynchronize();
    std::vector<long long> h(148);
    cudaMemcpy(h.data(), cyc, 148 * 8, cudaMemcpyDeviceToHost);
    std::sort(h.begin(), h.end());
    printf("{\"variant\": \"%s\", \"cyc_min\": %lld, \"cyc_med\": %lld, \"cyc_max\": %lld, \"err\": \"%s\"}\n", name, h[0], h[74], h[147],
           cudaGetErrorString(cudaGetLastError()));
}

int main() {
    float4* pos; unsigned* bar; long long* cyc;
    cudaMalloc(&pos, 65536); cudaMalloc(&bar, 64); cudaMalloc(&cyc, 148 * 8);
    run("stcg_ldcg", ag<0, 0, 0>, pos, bar, cyc);
    run("stwb_ldcg", ag<1, 0, 0>, pos, bar, cyc);
    run("stcg_ldrelaxed", ag<0, 1, 0>, pos, bar, cyc);
    run("stcg_ldcg_delay1us", ag<0, 0, 1000>, pos, bar, cyc);
    run("stcg_ldcg_delay4us", ag<0, 0, 4000>, pos, bar, cyc);
    return 0;
}
