// Inner-loop microbenchmark for the small-N N-Body design (config 1): how close to the FP32-pipe
// bound does the packed interaction loop run for a given warps/SM (W), target pairs per lane (Q)
// and lane -> split layout, with sources already in shared memory?  One CTA per SM, 148 CTAs;
// cycles between two __syncthreads around `reps` passes over a 128-body split.
//   layout 0: every lane of a warp reads the same split (LDS.128 broadcast)
//   layout 1: lane pairs share a split, 16 splits per warp (padded: conflict-free phases)
//   layout 2: 32 splits per warp (padded)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I include -o tools/nbody_inner_mb tools/nbody_inner_mb.cu
#include <cstdio>
#include <vector>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/nbody.cu"

namespace lime {
const LaunchOverride& launch_override() { static LaunchOverride o; return o; }
int device_num_sms() { return 148; }
int nbody_variant() { return 0; }
bool pdl_enabled() { return false; }
cudaError_t ensure_dynamic_smem(const void*, int) { return cudaSuccess; }
int cached_occupancy(const void*, int, size_t) { return 1; }
void* tensor_map_encoder() { return nullptr; }
}
using namespace lime;
using namespace lime::nbody;

#ifndef MB_L
#define MB_L 128
#endif
constexpr int kL = MB_L, kS = 4096 / MB_L;

template <int W, int Q, int LAYOUT>
__global__ void __launch_bounds__(W * 32, 1) mb(const float4* __restrict__ bodies, int reps, long long* cyc, float4* out) {
    extern __shared__ __align__(16) float4 src[];
    for (int i = threadIdx.x; i < kS * kL; i += blockDim.x) src[(i / kL) * (kL + 1) + i % kL] = bodies[i];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int s;
    if (LAYOUT == 0) s = (warp + blockIdx.x) % kS;
    else if (LAYOUT == 1) s = (warp * 16 + lane / 2) % kS;
    else s = lane % kS;
    Interact<2 * Q, true> it;
#pragma unroll
    for (int r = 0; r < 2 * Q; ++r) it.set(r, bodies[(blockIdx.x * 64 + threadIdx.x * 2 * Q + r) % 4096]);
    it.zero_all();
    __syncthreads();
    const long long t0 = clock64();
    for (int k = 0; k < reps; ++k) split_sum(it, src + s * (kL + 1), kL, kL, 1e-4f);
    __syncthreads();
    const long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
#pragma unroll
    for (int r = 0; r < 2 * Q; ++r) out[(blockIdx.x * blockDim.x + threadIdx.x) * 2 * Q + r] = it.result(r);
}

template <int W, int Q, int LAYOUT>
void run(const float4* bodies, float4* out, long long* cyc, int reps = 16) {
    const int smem = kS * (kL + 1) * 16;
    cudaFuncSetAttribute(mb<W, Q, LAYOUT>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    mb<W, Q, LAYOUT><<<148, W * 32, smem>>>(bodies, reps, cyc, out);
    mb<W, Q, LAYOUT><<<148, W * 32, smem>>>(bodies, reps, cyc, out);
    cudaDeviceSynchronize();
    std::vector<long long> h(148);
    cudaMemcpy(h.data(), cyc, 148 * 8, cudaMemcpyDeviceToHost);
    long long mx = 0;
    double mean = 0;
    for (auto v : h) { mx = v > mx ? v : mx; mean += v / 148.0; }
    const double lane_ops = double(W) * 32 * 2 * Q * kL * reps * 12;
    cudaFuncAttributes fa;
    cudaFuncGetAttributes(&fa, mb<W, Q, LAYOUT>);
    printf("{\"L\": %d, \"reps\": %d, \"W\": %d, \"Q\": %d, \"layout\": %d, \"regs\": %d, \"cycles_mean\": %.0f, \"fp32_pipe_eff\": %.3f, "
           "\"cycles_per_warp_source\": %.2f, \"err\": \"%s\"}\n",
           kL, reps, W, Q, LAYOUT, fa.numRegs, mean, lane_ops / (128.0 * mean), mean / (double(reps) * kL * W / 4.0),
           cudaGetErrorString(cudaGetLastError()));
}

int main() {
    std::vector<float4> h(4096);
    uint32_t st = 1;
    for (auto& b : h) {
        auto u = [&] { st = st * 1664525u + 1013904223u; return (st >> 8) * (1.f / 16777216.f); };
        b.x = 2 * u() - 1; b.y = 2 * u() - 1; b.z = 2 * u() - 1; b.w = 1.f / 4096;
    }
    float4 *bodies, *out;
    long long* cyc;
    cudaMalloc(&bodies, 4096 * 16);
    cudaMalloc(&out, 148 * 1024 * 4 * 16);
    cudaMalloc(&cyc, 148 * 8);
    cudaMemcpy(bodies, h.data(), 4096 * 16, cudaMemcpyHostToDevice);
    for (int reps : {1, 2, 16}) {
        run<28, 1, 1>(bodies, out, cyc, reps);
        run<28, 1, 2>(bodies, out, cyc, reps);
        run<14, 2, 1>(bodies, out, cyc, reps);
        run<28, 2, 1>(bodies, out, cyc, reps);
    }
    return 0;
}
