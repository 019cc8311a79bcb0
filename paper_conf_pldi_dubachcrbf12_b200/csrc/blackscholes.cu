// blackscholes.cu -- Black-Scholes streaming map and fused map+reduce (sm_100a).
//
// BASELINE.json config 2 (not in the paper; R5-R6). A3/A7: 128-bit read-only
// streaming loads of the SoA operands (ld.global.nc.L1::no_allocate, PAPER.md L267-275
// vectorisation of read-only arrays) and evict-first 128-bit stores. A8: the fused
// variant never writes call/put; fp64 partials per thread -> warp shuffle -> CTA ->
// last CTA combines CTA partials in index order.
//
// The element function is written for B200's ridge point: 7 MUFU and ~45
// FP32 lane-ops per option. Savings vs the textbook evaluation:
//   * 1/(sigma sqrt T) = rsqrt(T) / sigma  (one MUFU.RSQ gives both sqrt T and its inverse)
//   * ln(S/X) = (lg2 S - lg2 X) ln 2
//   * K phi(d2) = S phi(d1) (exact identity, K = X e^{-rT}) -> one exponential serves both
//     normal-CDF tails (Abramowitz & Stegun 26.2.17, |err| < 7.5e-8).
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace bs {

struct Consts {
    float r_plus_half_s2;   // r + sigma^2/2
    float inv_sigma;        // 1/sigma
    float sigma;
    float neg_r_log2e;      // -r log2(e)
};

constexpr float kLn2 = 0.693147180559945309f;
constexpr float kNegHalfLog2e = -0.721347520444481703f;   // -log2(e)/2
constexpr float kInvSqrt2Pi = 0.398942280401432678f;
constexpr float kAS_p = 0.2316419f;
constexpr float kAS_a1 = 0.319381530f;
constexpr float kAS_a2 = -0.356563782f;
constexpr float kAS_a3 = 1.781477937f;
constexpr float kAS_a4 = -1.821255978f;
constexpr float kAS_a5 = 1.330274429f;

__device__ __forceinline__ float as_poly(float k) {
    return k * fmaf(k, fmaf(k, fmaf(k, fmaf(k, kAS_a5, kAS_a4), kAS_a3), kAS_a2), kAS_a1);
}

__device__ __forceinline__ void price(float S, float X, float T, const Consts& c, float& call, float& put) {
    const float rsT = rsqrt_approx(T);
    const float sqT = T * rsT;
    const float v = c.sigma * sqT;                                   // sigma sqrt T
    const float inv_v = rsT * c.inv_sigma;                           // 1 / (sigma sqrt T)
    const float l = (lg2_approx(S) - lg2_approx(X)) * kLn2;         // ln(S/X)
    const float d1 = fmaf(c.r_plus_half_s2, T, l) * inv_v;
    const float d2 = d1 - v;
    const float K = X * ex2_approx(c.neg_r_log2e * T);              // X e^{-rT}
    const float k1 = rcp_approx(fmaf(kAS_p, fabsf(d1), 1.f));
    const float k2 = rcp_approx(fmaf(kAS_p, fabsf(d2), 1.f));
    const float sphi = S * (kInvSqrt2Pi * ex2_approx(kNegHalfLog2e * d1 * d1));   // S phi(d1) = K phi(d2)
    const float sq1 = sphi * as_poly(k1);                           // S N(-|d1|)
    const float kq2 = sphi * as_poly(k2);                           // K N(-|d2|)
    const float sn1 = d1 >= 0.f ? S - sq1 : sq1;                    // S N(d1)
    const float snm1 = d1 >= 0.f ? sq1 : S - sq1;                   // S N(-d1)
    const float kn2 = d2 >= 0.f ? K - kq2 : kq2;                    // K N(d2)
    const float knm2 = d2 >= 0.f ? kq2 : K - kq2;                   // K N(-d2)
    call = sn1 - kn2;
    put = knm2 - snm1;
}

__global__ void __launch_bounds__(256) map_kernel(const float* __restrict__ S, const float* __restrict__ X,
                                                  const float* __restrict__ T, int64_t n, Consts c,
                                                  float* __restrict__ call, float* __restrict__ put) {
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n4; i += stride) {
        const float4 s = ld_stream_f4(reinterpret_cast<const float4*>(S) + i);
        const float4 x = ld_stream_f4(reinterpret_cast<const float4*>(X) + i);
        const float4 t = ld_stream_f4(reinterpret_cast<const float4*>(T) + i);
        float4 cv, pv;
        price(s.x, x.x, t.x, c, cv.x, pv.x);
        price(s.y, x.y, t.y, c, cv.y, pv.y);
        price(s.z, x.z, t.z, c, cv.z, pv.z);
        price(s.w, x.w, t.w, c, cv.w, pv.w);
        st_stream_f4(reinterpret_cast<float4*>(call) + i, cv);
        st_stream_f4(reinterpret_cast<float4*>(put) + i, pv);
    }
    // ragged tail (n % 4 elements)
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x < (n & 3)) {
        const int64_t e = (n4 << 2) + threadIdx.x;
        float cv, pv;
        price(S[e], X[e], T[e], c, cv, pv);
        call[e] = cv;
        put[e] = pv;
    }
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// ws layout: [0]: u32 ticket counter; [256 B ...]: double2 CTA partials.
__global__ void __launch_bounds__(256) map_reduce_kernel(const float* __restrict__ S, const float* __restrict__ X,
                                                         const float* __restrict__ T, int64_t n, Consts c,
                                                         double* __restrict__ sums, unsigned* ticket,
                                                         double2* __restrict__ partial) {
    __shared__ double2 s_part[8];
    __shared__ int s_last;
    double ac = 0.0, ap = 0.0;
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n4; i += stride) {
        const float4 s = ld_stream_f4(reinterpret_cast<const float4*>(S) + i);
        const float4 x = ld_stream_f4(reinterpret_cast<const float4*>(X) + i);
        const float4 t = ld_stream_f4(reinterpret_cast<const float4*>(T) + i);
        float c0, c1, c2, c3, p0, p1, p2, p3;
        price(s.x, x.x, t.x, c, c0, p0);
        price(s.y, x.y, t.y, c, c1, p1);
        price(s.z, x.z, t.z, c, c2, p2);
        price(s.w, x.w, t.w, c, c3, p3);
        ac += static_cast<double>((c0 + c1) + (c2 + c3));
        ap += static_cast<double>((p0 + p1) + (p2 + p3));
    }
    if (blockIdx.x == gridDim.x - 1 && threadIdx.x < (n & 3)) {
        const int64_t e = (n4 << 2) + threadIdx.x;
        float cv, pv;
        price(S[e], X[e], T[e], c, cv, pv);
        ac += cv;
        ap += pv;
    }
    ac = warp_sum(ac);
    ap = warp_sum(ap);
    const int warp = threadIdx.x >> 5;
    if (lane_id() == 0) s_part[warp] = make_double2(ac, ap);
    __syncthreads();
    if (threadIdx.x == 0) {
        double2 b = s_part[0];
        for (int w = 1; w < (blockDim.x >> 5); ++w) { b.x += s_part[w].x; b.y += s_part[w].y; }
        __stcg(partial + blockIdx.x, b);
        __threadfence();
        s_last = (atomicAdd(ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!s_last) return;
    // Last CTA: combine the CTA partials in index order (warp 0, fixed lane->CTA mapping).
    __threadfence();
    if (warp == 0) {
        double bx = 0.0, by = 0.0;
        for (unsigned k = lane_id(); k < gridDim.x; k += 32) {
            const double2 p = __ldcg(partial + k);
            bx += p.x;
            by += p.y;
        }
        bx = warp_sum(bx);
        by = warp_sum(by);
        if (lane_id() == 0) {
            sums[0] = bx;
            sums[1] = by;
            *ticket = 0u;   // leave the workspace zeroed
        }
    }
}

static Consts make_consts(float r, float sigma) {
    Consts c;
    c.r_plus_half_s2 = r + 0.5f * sigma * sigma;
    c.inv_sigma = 1.0f / sigma;
    c.sigma = sigma;
    c.neg_r_log2e = -r * 1.44269504088896341f;
    return c;
}

static int grid_for(const void* kernel, int64_t n) {
    const int ov = launch_override().grid_ctas;
    if (ov > 0) return ov;
    static int per_sm[2] = {0, 0};
    const int idx = (kernel == reinterpret_cast<const void*>(&map_kernel)) ? 0 : 1;
    if (per_sm[idx] == 0) {
        int b = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, 256, 0);
        per_sm[idx] = b > 0 ? b : 1;
    }
    const int64_t need = ceil_div<int64_t>(mx<int64_t>(n >> 2, 1), 256);
    return static_cast<int>(mn<int64_t>(need, static_cast<int64_t>(per_sm[idx]) * device_num_sms()));
}

cudaError_t launch_map(const float* S, const float* X, const float* T, int64_t n, float r, float sigma,
                       float* call, float* put, cudaStream_t stream) {
    if (n == 0) return cudaSuccess;
    const int grid = grid_for(reinterpret_cast<const void*>(&map_kernel), n);
    map_kernel<<<grid, 256, 0, stream>>>(S, X, T, n, make_consts(r, sigma), call, put);
    return cudaGetLastError();
}

cudaError_t launch_map_reduce(const float* S, const float* X, const float* T, int64_t n, float r,
                              float sigma, double* sums, void* ws, cudaStream_t stream) {
    int grid = grid_for(reinterpret_cast<const void*>(&map_reduce_kernel), n);
    if (grid > red::kMaxCtas) grid = red::kMaxCtas;
    unsigned* ticket = static_cast<unsigned*>(ws);
    double2* partial = reinterpret_cast<double2*>(static_cast<char*>(ws) + 256);
    map_reduce_kernel<<<grid, 256, 0, stream>>>(S, X, T, n, make_consts(r, sigma), sums, ticket, partial);
    return cudaGetLastError();
}

}  // namespace bs
}  // namespace lime
