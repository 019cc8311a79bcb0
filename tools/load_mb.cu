// Broadcast-load microbenchmark (config-1 persistent step): every one of 148 CTAs (one per SM)
// brings the same 64 KB (4096 bodies) from L2 into its shared memory. Cycles from start to "all
// landed" per CTA, for: k bulk copies (cp.async.bulk, one mbarrier each) of 64KB/k, or LDG.128 +
// STS by all threads. The source was written by the previous launch (L2-resident).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/load_mb tools/load_mb.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include <cstdint>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/common.cuh"
using namespace lime;

template <int K>
__global__ void __launch_bounds__(896, 1) bulk_kernel(const float4* __restrict__ src, long long* cyc, int reps) {
    extern __shared__ __align__(128) float4 dst[];
    __shared__ __align__(8) uint64_t bar[64];
    if (threadIdx.x < K) mbar_init(&bar[threadIdx.x], 1);
    fence_mbar_init();
    __syncthreads();
    long long acc = 0;
    for (int r = 0; r < reps; ++r) {
        __syncthreads();
        const long long t0 = clock64();
        if (threadIdx.x < K) {
            const uint32_t bytes = 65536 / K;
            mbar_arrive_expect_tx(&bar[threadIdx.x], bytes);
            bulk_g2s(reinterpret_cast<char*>(dst) + threadIdx.x * bytes, reinterpret_cast<const char*>(src) + threadIdx.x * bytes, bytes, &bar[threadIdx.x]);
        }
        if (threadIdx.x < 32) for (int k = 0; k < K; ++k) mbar_wait(&bar[k], r & 1);
        __syncthreads();
        acc += clock64() - t0;
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = acc / reps;
}

__global__ void __launch_bounds__(896, 1) ldg_kernel(const float4* __restrict__ src, long long* cyc, int reps) {
    extern __shared__ __align__(128) float4 dst[];
    long long acc = 0;
    for (int r = 0; r < reps; ++r) {
        __syncthreads();
        const long long t0 = clock64();
        float4 v[5];
#pragma unroll
        for (int k = 0; k < 5; ++k) { int i = threadIdx.x + k * 896; if (i < 4096) v[k] = __ldcg(src + i); }
#pragma unroll
        for (int k = 0; k < 5; ++k) { int i = threadIdx.x + k * 896; if (i < 4096) dst[i] = v[k]; }
        __syncthreads();
        acc += clock64() - t0;
    }
    if (threadIdx.x == 0) cyc[blockIdx.x] = acc / reps;
}

__global__ void touch(float4* p) { int i = blockIdx.x * blockDim.x + threadIdx.x; if (i < 4096) p[i].w += 0.f; }

template <class F>
void run(const char* name, F kern, float4* src, long long* cyc) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 118784);
    for (int it = 0; it < 2; ++it) {
        touch<<<16, 256>>>(src);
        kern<<<148, 896, 118784>>>(src, cyc, 8);
    }
    cudaDeviceSynchronize();
    std::vector<long long> h(148);
    cudaMemcpy(h.data(), cyc, 148 * 8, cudaMemcpyDeviceToHost);
    std::sort(h.begin(), h.end());
    printf("{\"variant\": \"%s\", \"cyc_min\": %lld, \"cyc_med\": %lld, \"cyc_max\": %lld, \"err\": \"%s\"}\n", name, h[0], h[74], h[147],
           cudaGetErrorString(cudaGetLastError()));
}

int main() {
    float4* src; long long* cyc;
    cudaMalloc(&src, 65536); cudaMemset(src, 0, 65536);
    cudaMalloc(&cyc, 148 * 8);
    run("bulk_64x1KB", bulk_kernel<64>, src, cyc);
    run("bulk_32x2KB", bulk_kernel<32>, src, cyc);
    run("bulk_16x4KB", bulk_kernel<16>, src, cyc);
    run("bulk_4x16KB", bulk_kernel<4>, src, cyc);
    run("bulk_1x64KB", bulk_kernel<1>, src, cyc);
    run("ldg_sts", ldg_kernel, src, cyc);
    return 0;
}
