// kernels.h -- internal launcher interface between abi.cu (validation, C ABI) and the
// kernel translation units. Not installed; the public contract is include/lime.h.
#pragma once
#include <cstddef>
#include <cstdint>
#include <cuda_runtime.h>

namespace lime {

struct LaunchOverride {
    int grid_ctas = 0;
    int block_threads = 0;
    int per_thread = 0;
};
const LaunchOverride& launch_override();
int nbody_variant();   // staging ablation selector (0 = production kernels), see lime_set_nbody_variant
int device_num_sms();
void* tensor_map_encoder();   // PFN_cuTensorMapEncodeTiled (gemm.cu), or null

// ------------------------------------------------------------------ N-Body
namespace nbody {
// Two-level accumulation (part of the result's definition, a function of n_src only): sources are
// cut into chunks of chunk_len(n_src) bodies whose partials are added in order into one of
// splits(n_src) split partials, added in split order. Small problems (n_src <= kSmallMaxSources)
// use 64-body chunks and up to 64 splits (whole warps per SMSP for the latency-bound sizes), larger
// ones 256-body chunks and up to 32 splits (r02: 16 -> 32 -- the 2^20 launch is 8192 -> 16384 CTAs of
// one SM each, so its last wave idles 44 instead of 96 SMs: 377.7 -> 373.4 ms, same-call A/B).
constexpr int kChunk = 256;
#ifndef LIME_MAX_SPLITS              // compile-time A/B override (tools/); the default is the product
#define LIME_MAX_SPLITS 32
#endif
constexpr int kMaxSplits = LIME_MAX_SPLITS;
constexpr int kMaxSplitsF64 = 16;   // the fp64 map's own rule (chunks_per_split_fixed / splits_fixed)
#ifndef LIME_CHUNK_SMALL            // compile-time A/B overrides (tools/); the defaults are the product
#define LIME_CHUNK_SMALL 64
#endif
#ifndef LIME_MAX_SPLITS_SMALL
#define LIME_MAX_SPLITS_SMALL 64
#endif
constexpr int kChunkSmall = LIME_CHUNK_SMALL;
constexpr int kMaxSplitsSmall = LIME_MAX_SPLITS_SMALL;
constexpr int64_t kSmallMaxSources = 8192;
int chunk_len(int64_t n_src);
int64_t chunks_per_split(int64_t n_src);
int splits(int64_t n_src);
int64_t chunks_per_split_fixed(int64_t n_src);   // 256-body chunks, <= kMaxSplitsF64 splits (fp64 map)
int splits_fixed(int64_t n_src);
size_t workspace_bytes(int64_t n_src, int64_t tgt_count);
cudaError_t launch_force(const float4* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count,
                         float eps2, float4* accel, void* ws, cudaStream_t stream);
cudaError_t launch_integrate(float4* pos, float4* vel, const float4* accel, int64_t n, float dt,
                             cudaStream_t stream);
size_t step_workspace_bytes(int64_t n_src, int64_t tgt_count);
cudaError_t launch_step(const float4* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, float eps2,
                        float dt, float4* vel, float4* pos_out, void* ws, cudaStream_t stream);
size_t simulate_workspace_bytes(int64_t n);
cudaError_t launch_simulate(float4* pos, float4* vel, int64_t n, int32_t steps, float eps2, float dt, void* ws,
                            cudaStream_t stream);
}  // namespace nbody

namespace nbody64 {   // F3: double precision
size_t workspace_bytes(int64_t n_src, int64_t tgt_count);
cudaError_t launch_force(const double* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, double eps2,
                         double* accel, void* ws, cudaStream_t stream);
}  // namespace nbody64

// ----------------------------------------------------------- Black-Scholes
namespace bs {
cudaError_t launch_map(const float* S, const float* X, const float* T, int64_t n, float r,
                       float sigma, float* call, float* put, cudaStream_t stream);
cudaError_t launch_map_reduce(const float* S, const float* X, const float* T, int64_t n, float r,
                              float sigma, double* sums, void* ws, cudaStream_t stream);
}  // namespace bs

// -------------------------------------------------------------- Mandelbrot
namespace mandel {
constexpr size_t kWorkspaceBytes = 256;
cudaError_t launch(int32_t width, int32_t row_first, int32_t row_stride, int32_t row_count,
                   float x0, float y0, float dx, float dy, int32_t max_iter, int32_t* counts,
                   void* ws, cudaStream_t stream);
}  // namespace mandel

// ------------------------------------------------------------- Parboil CP / MRI-Q (F2)
namespace parboil {
size_t cp_workspace_bytes(int64_t n_atoms, int64_t points);
size_t mriq_workspace_bytes(int64_t n_k, int64_t n_x);
cudaError_t launch_cp(const float4* atoms, int64_t n_atoms, int32_t nx, int64_t p_begin, int64_t p_count, float z,
                      float h, float* out, void* ws, cudaStream_t stream);
cudaError_t launch_mriq(const float* kspace, int64_t n_k, const float* voxels, int64_t x_begin, int64_t x_count,
                        float* out, void* ws, cudaStream_t stream);
}  // namespace parboil

// ------------------------------------------------------------- JG-Series / JG-Crypt (F4)
namespace jgf {
size_t series_workspace_bytes(bool f64);
cudaError_t launch_series_f32(int64_t n0, int64_t count, float* out, void* ws, cudaStream_t stream);
cudaError_t launch_series_f64(int64_t n0, int64_t count, double* out, void* ws, cudaStream_t stream);
void idea_key_schedule(const uint16_t key[8], uint16_t ek[52], uint16_t dk[52]);
cudaError_t launch_idea(const uint8_t* in, uint8_t* out, int64_t nbytes, const uint16_t* subkeys, cudaStream_t stream);
}  // namespace jgf

// ------------------------------------------------------------------ Matmul
namespace gemm {
cudaError_t launch_bf16(const uint16_t* A, const uint16_t* Bt, float* C, int64_t M, int64_t N,
                        int64_t K, cudaStream_t stream);
}  // namespace gemm

// -------------------------------------------------------------- Reductions
namespace red {
constexpr int kMaxCtas = 148 * 8;
constexpr size_t kWorkspaceBytes = 256 + 16 * kMaxCtas;   // ticket + up to 16-B partial per CTA
enum Op { kSum = 0, kMin = 1, kMax = 2 };
enum Dt { kF32 = 0, kF64 = 1, kI32 = 2, kI64 = 3 };
cudaError_t launch(Op op, Dt dt, const void* x, int64_t n, void* out, void* ws, cudaStream_t stream);
}  // namespace red

}  // namespace lime
