// Black-Scholes fused map+reduce: occupancy / prefetch-depth sweep of the production loop
// (compute-only 34.8 us and loads-only 33.5 us at 592x256 each fit the budget, the combined loop
// does not overlap them: is it latency-bound at 1024 threads/SM?).  Same price4 as production.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/bs_occ tools/bs_occ.cu
#include <cstdio>
#include <vector>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/blackscholes.cu"

namespace lime {
const LaunchOverride& launch_override() { static LaunchOverride o; return o; }
int device_num_sms() { return 148; }
}
using namespace lime;
using namespace lime::bs;

// DEPTH iterations of loads in flight per thread (register ring); fp32 per-thread partials.
template <int BLOCK, int MINB, int DEPTH>
__global__ void __launch_bounds__(BLOCK, MINB) fused(const float* __restrict__ S, const float* __restrict__ X,
                                                    const float* __restrict__ T, int64_t n, Consts c, double* out) {
    float fc = 0.f, fp = 0.f;
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * BLOCK;
    const float4* S4 = reinterpret_cast<const float4*>(S);
    const float4* X4 = reinterpret_cast<const float4*>(X);
    const float4* T4 = reinterpret_cast<const float4*>(T);
    const int64_t i0 = blockIdx.x * static_cast<int64_t>(BLOCK) + threadIdx.x;
    float4 s[DEPTH], x[DEPTH], t[DEPTH];
#pragma unroll
    for (int d = 0; d < DEPTH; ++d) {
        const int64_t j = i0 + d * stride;
        if (j < n4) { s[d] = ld_stream_f4(S4 + j); x[d] = ld_stream_f4(X4 + j); t[d] = ld_stream_f4(T4 + j); }
    }
    for (int64_t i = i0; i < n4; i += DEPTH * stride) {
#pragma unroll
        for (int d = 0; d < DEPTH; ++d) {
            const int64_t j = i + d * stride;
            if (j < n4) {
                const float4 cs = s[d], cx = x[d], ct = t[d];
                const int64_t nx = j + DEPTH * stride;
                if (nx < n4) { s[d] = ld_stream_f4(S4 + nx); x[d] = ld_stream_f4(X4 + nx); t[d] = ld_stream_f4(T4 + nx); }
                float4 cv, pv;
                price4(cs, cx, ct, c, cv, pv);
                fc += (cv.x + cv.y) + (cv.z + cv.w);
                fp += (pv.x + pv.y) + (pv.z + pv.w);
            }
        }
    }
    if (fc + fp == 1234.5f) out[0] = fc;
}


// cp.async ring: each thread prefetches its own next D iterations (3 x 16 B each) into a per-thread
// shared-memory ring -- bytes in flight without holding registers.
__device__ __forceinline__ void cp_async16(void* smem, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(smem))), "l"(g)
                 : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int BLOCK, int MINB, int D>
__global__ void __launch_bounds__(BLOCK, MINB) fused_cp(const float* __restrict__ S, const float* __restrict__ X,
                                                       const float* __restrict__ T, int64_t n, Consts c, double* out) {
    extern __shared__ float4 ring[];                 // [D][3][BLOCK]
    float fc = 0.f, fp = 0.f;
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * BLOCK;
    const float4* P[3] = {reinterpret_cast<const float4*>(S), reinterpret_cast<const float4*>(X),
                          reinterpret_cast<const float4*>(T)};
    const int64_t i0 = blockIdx.x * static_cast<int64_t>(BLOCK) + threadIdx.x;
    auto slot = [&](int d, int k) { return ring + (d * 3 + k) * BLOCK + threadIdx.x; };
#pragma unroll
    for (int d = 0; d < D; ++d) {
        const int64_t j = i0 + d * stride;
        if (j < n4)
#pragma unroll
            for (int k = 0; k < 3; ++k) cp_async16(slot(d, k), P[k] + j);
        cp_commit();
    }
    int d = 0;
    for (int64_t i = i0; i < n4; i += stride) {
        cp_wait<D - 1>();
        const float4 cs = *slot(d, 0), cx = *slot(d, 1), ct = *slot(d, 2);
        const int64_t nx = i + D * stride;
        if (nx < n4)
#pragma unroll
            for (int k = 0; k < 3; ++k) cp_async16(slot(d, k), P[k] + nx);
        cp_commit();
        d = (d + 1 == D) ? 0 : d + 1;
        float4 cv, pv;
        price4(cs, cx, ct, c, cv, pv);
        fc += (cv.x + cv.y) + (cv.z + cv.w);
        fp += (pv.x + pv.y) + (pv.z + pv.w);
    }
    cp_wait<0>();
    if (fc + fp == 1234.5f) out[0] = fc;
}


// map kernel with the cp.async ring (calls and puts stored evict-first)
template <int BLOCK, int MINB, int D>
__global__ void __launch_bounds__(BLOCK, MINB) map_cp(const float* __restrict__ S, const float* __restrict__ X,
                                                     const float* __restrict__ T, int64_t n, Consts c,
                                                     float* __restrict__ call, float* __restrict__ put) {
    extern __shared__ float4 ring[];                 // [D][3][BLOCK]
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * BLOCK;
    const float4* P[3] = {reinterpret_cast<const float4*>(S), reinterpret_cast<const float4*>(X),
                          reinterpret_cast<const float4*>(T)};
    const int64_t i0 = blockIdx.x * static_cast<int64_t>(BLOCK) + threadIdx.x;
    auto slot = [&](int d, int k) { return ring + (d * 3 + k) * BLOCK + threadIdx.x; };
#pragma unroll
    for (int d = 0; d < D; ++d) {
        const int64_t j = i0 + d * stride;
        if (j < n4)
#pragma unroll
            for (int k = 0; k < 3; ++k) cp_async16(slot(d, k), P[k] + j);
        cp_commit();
    }
    int d = 0;
    for (int64_t i = i0; i < n4; i += stride) {
        cp_wait<D - 1>();
        const float4 cs = *slot(d, 0), cx = *slot(d, 1), ct = *slot(d, 2);
        const int64_t nx = i + D * stride;
        if (nx < n4)
#pragma unroll
            for (int k = 0; k < 3; ++k) cp_async16(slot(d, k), P[k] + nx);
        cp_commit();
        d = (d + 1 == D) ? 0 : d + 1;
        float4 cv, pv;
        price4(cs, cx, ct, c, cv, pv);
        st_stream_f4(reinterpret_cast<float4*>(call) + i, cv);
        st_stream_f4(reinterpret_cast<float4*>(put) + i, pv);
    }
    cp_wait<0>();
}

// flush: write 2x L2, then read 2x L2 so the L2 holds clean lines of an unrelated buffer
__global__ void read_flush(const float4* __restrict__ f, int64_t n4, float* out) {
    float acc = 0.f;
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n4;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        float4 v = ld_stream_f4(f + i);
        acc += v.x + v.w;
    }
    if (acc == 1234.5f) out[0] = acc;
}

int main(int argc, char** argv) {
    const bool old_sweep = argc > 1;
    const int64_t n = 1 << 24;
    float *S, *X, *T;
    cudaMalloc(&S, n * 4); cudaMalloc(&X, n * 4); cudaMalloc(&T, n * 4);
    std::vector<float> h(n);
    for (int64_t k = 0; k < n; ++k) h[k] = 5.f + 25.f * ((k * 2654435761u) % 1000) / 1000.f;
    cudaMemcpy(S, h.data(), n * 4, cudaMemcpyHostToDevice);
    for (int64_t k = 0; k < n; ++k) h[k] = 1.f + 99.f * ((k * 40503u) % 1000) / 1000.f;
    cudaMemcpy(X, h.data(), n * 4, cudaMemcpyHostToDevice);
    for (int64_t k = 0; k < n; ++k) h[k] = 0.25f + 9.75f * ((k * 2246822519u) % 1000) / 1000.f;
    cudaMemcpy(T, h.data(), n * 4, cudaMemcpyHostToDevice);
    const size_t FL = 512ull << 20;
    char *flush, *flush2;
    cudaMalloc(&flush, FL); cudaMalloc(&flush2, FL); cudaMemset(flush2, 0, FL);
    double* out; cudaMalloc(&out, 64);
    Consts c = make_consts(0.02f, 0.3f);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](auto kern, int block, int grid, int minb, int depth, int fmode) {
        float best = 1e9;
        for (int r = 0; r < 12; ++r) {
            cudaMemsetAsync(flush, r, FL);
            if (fmode) read_flush<<<1184, 256>>>(reinterpret_cast<const float4*>(flush2), FL / 16, reinterpret_cast<float*>(out));
            cudaEventRecord(a);
            kern<<<grid, block>>>(S, X, T, n, c, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (r >= 2 && ms < best) best = ms;
        }
        cudaFuncAttributes at; cudaFuncGetAttributes(&at, kern);
        int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, block, 0);
        printf("{\"block\": %d, \"minb\": %d, \"depth\": %d, \"grid\": %d, \"regs\": %d, \"local\": %zu, \"ctas_per_sm\": %d, "
               "\"flush\": \"%s\", \"us\": %.2f, \"GBps\": %.1f}\n", block, minb, depth, grid, at.numRegs,
               at.localSizeBytes, occ, fmode ? "write+read" : "write", best * 1e3, 12.0 * n / (best * 1e-3) / 1e9);
        fflush(stdout);
    };
    auto runs = [&](auto kern, int block, int grid, int minb, int depth, size_t smem) {
        float best = 1e9;
        for (int r = 0; r < 12; ++r) {
            cudaMemsetAsync(flush, r, FL);
            read_flush<<<1184, 256>>>(reinterpret_cast<const float4*>(flush2), FL / 16, reinterpret_cast<float*>(out));
            cudaEventRecord(a);
            kern<<<grid, block, smem>>>(S, X, T, n, c, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (r >= 2 && ms < best) best = ms;
        }
        cudaFuncAttributes at; cudaFuncGetAttributes(&at, kern);
        printf("{\"variant\": \"cp.async ring\", \"block\": %d, \"minb\": %d, \"depth\": %d, \"grid\": %d, \"regs\": %d, "
               "\"local\": %zu, \"smem\": %zu, \"us\": %.2f, \"GBps\": %.1f, \"err\": \"%s\"}\n", block, minb, depth, grid,
               at.numRegs, at.localSizeBytes, smem, best * 1e3, 12.0 * n / (best * 1e-3) / 1e9, cudaGetErrorString(cudaGetLastError()));
        fflush(stdout);
    };
#define RUN(B, M, D)                                                                                 \
    do {                                                                                             \
        int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fused<B, M, D>, B, 0);     \
        for (int f = 0; f < 2; ++f) run(fused<B, M, D>, B, occ * 148, M, D, f);                       \
    } while (0)
    if (old_sweep) {
    RUN(256, 4, 1);
    RUN(256, 4, 2);
    RUN(256, 5, 1);
    RUN(256, 6, 1);
    RUN(256, 6, 2);
    RUN(256, 8, 1);
    RUN(128, 12, 1);
    RUN(128, 16, 1);
    RUN(512, 3, 1);
    RUN(512, 4, 1);
    RUN(256, 3, 2);
    RUN(256, 2, 3);
    }
#define RUNCP(B, M, D)                                                                               \
    do {                                                                                             \
        const size_t sm = static_cast<size_t>(D) * 3 * B * 16;                                       \
        cudaFuncSetAttribute(fused_cp<B, M, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm); \
        int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fused_cp<B, M, D>, B, sm);   \
        if (occ > 0) runs(fused_cp<B, M, D>, B, occ * 148, M, D, sm);                                 \
    } while (0)
    RUNCP(256, 4, 2);
    RUNCP(256, 4, 4);
    RUNCP(256, 4, 6);
    RUNCP(256, 5, 3);
    RUNCP(256, 5, 4);
    RUNCP(256, 6, 2);
    RUNCP(256, 6, 3);
    RUNCP(128, 10, 4);
    RUNCP(128, 12, 3);
    float *callp, *putp; cudaMalloc(&callp, n * 4); cudaMalloc(&putp, n * 4);
    auto runm = [&](auto kern, int block, int grid, int minb, int depth, size_t smem) {
        float best = 1e9;
        for (int r = 0; r < 12; ++r) {
            cudaMemsetAsync(flush, r, FL);
            read_flush<<<1184, 256>>>(reinterpret_cast<const float4*>(flush2), FL / 16, reinterpret_cast<float*>(out));
            cudaEventRecord(a);
            kern<<<grid, block, smem>>>(S, X, T, n, c, callp, putp);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (r >= 2 && ms < best) best = ms;
        }
        cudaFuncAttributes at; cudaFuncGetAttributes(&at, kern);
        printf("{\"variant\": \"map cp.async ring\", \"block\": %d, \"minb\": %d, \"depth\": %d, \"grid\": %d, \"regs\": %d, "
               "\"local\": %zu, \"us\": %.2f, \"GBps\": %.1f}\n", block, minb, depth, grid, at.numRegs, at.localSizeBytes,
               best * 1e3, 20.0 * n / (best * 1e-3) / 1e9);
        fflush(stdout);
    };
#define RUNMAP(B, M, D)                                                                              \
    do {                                                                                             \
        const size_t sm = static_cast<size_t>(D) * 3 * B * 16;                                       \
        cudaFuncSetAttribute(map_cp<B, M, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);   \
        int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, map_cp<B, M, D>, B, sm);     \
        if (occ > 0) runm(map_cp<B, M, D>, B, occ * 148, M, D, sm);                                   \
    } while (0)
    RUNMAP(256, 4, 2);
    RUNMAP(256, 4, 4);
    RUNMAP(256, 5, 3);
    RUNMAP(256, 6, 2);
    // production kernel for reference
    {
        void* ws; cudaMalloc(&ws, 1 << 20); cudaMemset(ws, 0, 1 << 20);
        for (int f = 0; f < 2; ++f) {
            float best = 1e9;
            for (int r = 0; r < 12; ++r) {
                cudaMemsetAsync(flush, r, FL);
                if (f) read_flush<<<1184, 256>>>(reinterpret_cast<const float4*>(flush2), FL / 16, reinterpret_cast<float*>(out));
                cudaEventRecord(a);
                map_reduce_kernel<<<592, 256>>>(S, X, T, n, c, out, static_cast<unsigned*>(ws),
                                                reinterpret_cast<double2*>(static_cast<char*>(ws) + 256));
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (r >= 2 && ms < best) best = ms;
            }
            printf("{\"production map_reduce_kernel\": true, \"flush\": \"%s\", \"us\": %.2f}\n", f ? "write+read" : "write", best * 1e3);
        }
        float *call, *put; cudaMalloc(&call, n * 4); cudaMalloc(&put, n * 4);
        for (int f = 0; f < 2; ++f) {
            float best = 1e9;
            for (int r = 0; r < 12; ++r) {
                cudaMemsetAsync(flush, r, FL);
                if (f) read_flush<<<1184, 256>>>(reinterpret_cast<const float4*>(flush2), FL / 16, reinterpret_cast<float*>(out));
                cudaEventRecord(a);
                map_kernel<<<592, 256>>>(S, X, T, n, c, call, put);
                cudaEventRecord(b);
                cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b);
                if (r >= 2 && ms < best) best = ms;
            }
            printf("{\"production map_kernel\": true, \"flush\": \"%s\", \"us\": %.2f}\n", f ? "write+read" : "write", best * 1e3);
        }
    }
    printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
