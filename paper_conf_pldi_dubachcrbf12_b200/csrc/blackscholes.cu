// blackscholes.cu -- Black-Scholes streaming map and fused map+reduce (sm_100a).
//
// BASELINE.json config 2 (not in the paper; R5-R6). A3/A7: 128-bit read-only
// streaming loads of the SoA operands (ld.global.nc.L1::no_allocate, PAPER.md L267-275
// vectorisation of read-only arrays) and evict-first 128-bit stores. A8: the fused
// variant never writes call/put; fp32 partials per thread -> fp64 from the warp up -> CTA ->
// the last CTA (acq_rel ticket) combines the CTA partials in a fixed order with all its threads.
// Both kernels are launched with programmatic
// dependent launch (common.cuh pdl_enter/launch_pdl), so back-to-back launches overlap the
// next grid's launch with this one's drain.
//
// The element function is written for B200's ridge point: 6 MUFU per option,
// two options per packed FFMA2/FMUL2 instruction. Savings vs the textbook evaluation:
//   * 1/(sigma sqrt T) = rsqrt(T) / sigma  (one MUFU.RSQ gives both sqrt T and its inverse)
//   * ln(S/X) = lg2(S rcp X) ln 2 (map; the fused sums use (lg2 S - lg2 X) ln 2)
//   * K phi(d2) = S phi(d1) (exact identity, K = X e^{-rT}) -> one exponential serves both
//     normal-CDF tails (map: a degree-7 Mills-ratio polynomial, |err| < 5e-10; fused sums:
//     Abramowitz & Stegun 26.2.17, |err| < 7.5e-8).
// The map evaluates call and put per option (price2, ~48 FP32 lane-ops); the fused sums use
// price2_wu (~34 lane-ops, no per-option selects), which sums w and u with call = w + u/2 and
// put = w - u/2.
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace bs {

struct Consts {
    float r_plus_half_s2;   // r + sigma^2/2
    float inv_sigma;        // 1/sigma
    float sigma;
    float neg_r_log2e;      // -r log2(e)
    // fused map+reduce element (price2_wu): ln 2 folded into the d1/d2 constants
    float a_l2;             // (r + sigma^2/2) / ln 2
    float b_l2;             // (r - sigma^2/2) / ln 2
    float ln2_over_sigma;   // ln 2 / sigma
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

// Two options per call, packed (FFMA2/FMUL2/FADD2 carry both; MUFU ops are per lane).
// Per option: 6 MUFU (rsqrt T, rcp X + lg2 S/X, ex2 -rT, ex2 -d1^2/2, and ONE rcp shared by the two
// CND k's: k1 = D2/(D1 D2), k2 = D1/(D1 D2)).
struct P2 { float2 call, put; };

// Map element CND (round 2): N(-|x|) = phi(x) M(k), k = 1/(1 + p|x|), p = 0.318, M a degree-7
// polynomial with M(0) = 0 fitted to the Mills ratio N(-x)/phi(x) by a weighted minimax (Lawson) fit
// of phi(x) (M(k) - N(-x)/phi(x)) over x in [0, 40] (tools/fit_mills.py): max |dN| = 5.0e-10, against
// 7.5e-8 for Abramowitz-Stegun 26.2.17 -- whose error times X <= 100 alone used up to 8.9e-6 of the
// 1e-5 element tolerance (r = 0, sigma = 0.3: 1.03e-5 measured; profiles/experiments/bs_accuracy_r02.txt).
constexpr float kM_p = 0.318f;
__device__ __forceinline__ float2 mills7_2(float2 k) {
    float2 p = fma2(k, bcast2(1.1605857361e-01f), bcast2(-6.2049898640e-01f));
    p = fma2(k, p, bcast2(1.0789559974e+00f));
    p = fma2(k, p, bcast2(-4.7603565775e-01f));
    p = fma2(k, p, bcast2(5.7942646417e-01f));
    p = fma2(k, p, bcast2(2.5091390071e-01f));
    p = fma2(k, p, bcast2(3.2449384680e-01f));
    return mul2(k, p);
}
__device__ __forceinline__ float2 abs2(float2 v) { return make_float2(fabsf(v.x), fabsf(v.y)); }

__device__ __forceinline__ P2 price2(float2 S, float2 X, float2 T, const Consts& c) {
    const float2 rsT = make_float2(rsqrt_approx(T.x), rsqrt_approx(T.y));
    const float2 sqT = mul2(T, rsT);
    const float2 v = mul2(bcast2(c.sigma), sqT);                       // sigma sqrt T
    const float2 inv_v = mul2(rsT, bcast2(c.inv_sigma));               // 1 / (sigma sqrt T)
    // ln(S/X) from one lg2 of the fp32 ratio (rcp + lg2: the same two MUFU as lg2 S - lg2 X, one
    // rounding of S/X instead of two rounded logarithms of ~5 subtracted)
    const float2 q = mul2(S, make_float2(rcp_approx(X.x), rcp_approx(X.y)));
    const float2 l = mul2(make_float2(lg2_approx(q.x), lg2_approx(q.y)), bcast2(kLn2));   // ln(S/X)
    const float2 d1 = mul2(fma2(bcast2(c.r_plus_half_s2), T, l), inv_v);
    const float2 d2 = sub2(d1, v);
    const float2 er = mul2(bcast2(c.neg_r_log2e), T);
    const float2 K = mul2(X, make_float2(ex2_approx(er.x), ex2_approx(er.y)));   // X e^{-rT}
    const float2 D1 = fma2(bcast2(kM_p), abs2(d1), bcast2(1.f));
    const float2 D2 = fma2(bcast2(kM_p), abs2(d2), bcast2(1.f));
    const float2 DD = mul2(D1, D2);
    const float2 rr = make_float2(rcp_approx(DD.x), rcp_approx(DD.y));
    const float2 k1 = mul2(D2, rr);                                     // 1 / D1
    const float2 k2 = mul2(D1, rr);                                     // 1 / D2
    const float2 g = mul2(mul2(bcast2(kNegHalfLog2e), d1), d1);
    const float2 sphi = mul2(S, mul2(bcast2(kInvSqrt2Pi), make_float2(ex2_approx(g.x), ex2_approx(g.y))));
    const float2 sq1 = mul2(sphi, mills7_2(k1));                       // S N(-|d1|)
    const float2 kq2 = mul2(sphi, mills7_2(k2));                       // K N(-|d2|) = S phi(d1) poly(k2)
    const float2 s_m = sub2(S, sq1);                                    // S (1 - N(-|d1|))
    const float2 k_m = sub2(K, kq2);
    P2 r;
    const float sn1x = d1.x >= 0.f ? s_m.x : sq1.x, sn1y = d1.y >= 0.f ? s_m.y : sq1.y;       // S N(d1)
    const float snm1x = d1.x >= 0.f ? sq1.x : s_m.x, snm1y = d1.y >= 0.f ? sq1.y : s_m.y;     // S N(-d1)
    const float kn2x = d2.x >= 0.f ? k_m.x : kq2.x, kn2y = d2.y >= 0.f ? k_m.y : kq2.y;       // K N(d2)
    const float knm2x = d2.x >= 0.f ? kq2.x : k_m.x, knm2y = d2.y >= 0.f ? kq2.y : k_m.y;     // K N(-d2)
    r.call = sub2(make_float2(sn1x, sn1y), make_float2(kn2x, kn2y));
    r.put = sub2(make_float2(knm2x, knm2y), make_float2(snm1x, snm1y));
    return r;
}

// ---- fused map+reduce element: the two sums need no per-option call/put selects.
// With A = S N(d1) - S/2 = copysign(S/2 - S N(-|d1|), d1) and B = K N(d2) - K/2 (same form),
//   call = w + u/2, put = w - u/2,  where w = A - B, u = S - K
// (put = call - S + K, put-call parity, holds by construction). The kernel sums w and u only.
// Per option: 6 MUFU as in price2, ~34 FP32 lane-ops (ln 2 and 1/sqrt(2 pi) folded into the
// constants; the AS polynomial carries the sign so S/2 - S N(-|d1|) is one FFMA), 2 LOP3.
constexpr float kASn_a1 = -kAS_a1 * kInvSqrt2Pi;
constexpr float kASn_a2 = -kAS_a2 * kInvSqrt2Pi;
constexpr float kASn_a3 = -kAS_a3 * kInvSqrt2Pi;
constexpr float kASn_a4 = -kAS_a4 * kInvSqrt2Pi;
constexpr float kASn_a5 = -kAS_a5 * kInvSqrt2Pi;
__device__ __forceinline__ float2 as_poly2n(float2 k) {   // -phi-scaled AS polynomial: -poly(k)/sqrt(2 pi)
    float2 p = fma2(k, bcast2(kASn_a5), bcast2(kASn_a4));
    p = fma2(k, p, bcast2(kASn_a3));
    p = fma2(k, p, bcast2(kASn_a2));
    p = fma2(k, p, bcast2(kASn_a1));
    return mul2(k, p);
}
__device__ __forceinline__ void price2_wu(float2 S, float2 X, float2 T, const Consts& c, float2& w, float2& u) {
    const float2 rsT = make_float2(rsqrt_approx(T.x), rsqrt_approx(T.y));
    const float2 q = mul2(rsT, bcast2(c.ln2_over_sigma));                // ln 2 / (sigma sqrt T)
    const float2 lg = sub2(make_float2(lg2_approx(S.x), lg2_approx(S.y)),
                           make_float2(lg2_approx(X.x), lg2_approx(X.y)));  // log2(S/X)
    const float2 d1 = mul2(fma2(bcast2(c.a_l2), T, lg), q);
    const float2 d2 = mul2(fma2(bcast2(c.b_l2), T, lg), q);
    const float2 er = mul2(bcast2(c.neg_r_log2e), T);
    const float2 K = mul2(X, make_float2(ex2_approx(er.x), ex2_approx(er.y)));   // X e^{-rT}
    const float2 D1 = fma2(bcast2(kAS_p), abs2(d1), bcast2(1.f));
    const float2 D2 = fma2(bcast2(kAS_p), abs2(d2), bcast2(1.f));
    const float2 DD = mul2(D1, D2);
    const float2 rr = make_float2(rcp_approx(DD.x), rcp_approx(DD.y));
    const float2 k1 = mul2(D2, rr);                                     // 1 / D1
    const float2 k2 = mul2(D1, rr);                                     // 1 / D2
    const float2 g = mul2(mul2(bcast2(kNegHalfLog2e), d1), d1);
    const float2 se = mul2(S, make_float2(ex2_approx(g.x), ex2_approx(g.y)));   // S phi(d1) sqrt(2 pi)
    const float2 a = fma2(bcast2(0.5f), S, mul2(se, as_poly2n(k1)));   // S/2 - S N(-|d1|)
    const float2 b = fma2(bcast2(0.5f), K, mul2(se, as_poly2n(k2)));   // K/2 - K N(-|d2|)
    w = sub2(make_float2(copysignf(a.x, d1.x), copysignf(a.y, d1.y)),
             make_float2(copysignf(b.x, d2.x), copysignf(b.y, d2.y)));
    u = sub2(S, K);
}

__device__ __forceinline__ void price(float S, float X, float T, const Consts& c, float& call, float& put) {
    const P2 r = price2(bcast2(S), bcast2(X), bcast2(T), c);
    call = r.call.x;
    put = r.put.x;
}

__device__ __forceinline__ void price4(const float4& s, const float4& x, const float4& t, const Consts& c,
                                       float4& cv, float4& pv) {
    const P2 a = price2(make_float2(s.x, s.y), make_float2(x.x, x.y), make_float2(t.x, t.y), c);
    const P2 b = price2(make_float2(s.z, s.w), make_float2(x.z, x.w), make_float2(t.z, t.w), c);
    cv = make_float4(a.call.x, a.call.y, b.call.x, b.call.y);
    pv = make_float4(a.put.x, a.put.y, b.put.x, b.put.y);
}

// Grid-stride sweep over the float4 groups [i, n4), software-pipelined one iteration ahead: the
// next group's 48 B are loaded before this one is priced. (A copy-free two-buffer ring measured
// 1-2 us slower for the fused kernel and 3-5 us for the map: ptxas sinks the ring's look-ahead loads
// below the pricing at the 64-register cap, tools/bs_pdl.cu, profiles/experiments/bs_pdl_loop_r01m.jsonl.)
template <typename F>
__device__ __forceinline__ void sweep_groups(const float4* __restrict__ S4, const float4* __restrict__ X4,
                                             const float4* __restrict__ T4, int64_t i, int64_t n4, int64_t stride,
                                             F&& body) {
    float4 s, x, t;
    if (i < n4) { s = ld_stream_f4(S4 + i); x = ld_stream_f4(X4 + i); t = ld_stream_f4(T4 + i); }
    for (; i < n4; i += stride) {
        const int64_t nx = i + stride;
        float4 s2 = s, x2 = x, t2 = t;
        if (nx < n4) { s2 = ld_stream_f4(S4 + nx); x2 = ld_stream_f4(X4 + nx); t2 = ld_stream_f4(T4 + nx); }
        body(i, s, x, t);
        s = s2; x = x2; t = t2;
    }
}

__global__ void __launch_bounds__(256, 4) map_kernel(const float* __restrict__ S, const float* __restrict__ X,
                                                  const float* __restrict__ T, int64_t n, Consts c,
                                                  float* __restrict__ call, float* __restrict__ put) {
    pdl_enter();
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    sweep_groups(reinterpret_cast<const float4*>(S), reinterpret_cast<const float4*>(X),
                 reinterpret_cast<const float4*>(T), blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x,
                 n4, stride, [&](int64_t i, const float4& s, const float4& x, const float4& t) {
                     float4 cv, pv;
                     price4(s, x, t, c, cv, pv);
                     st_stream_f4(reinterpret_cast<float4*>(call) + i, cv);
                     st_stream_f4(reinterpret_cast<float4*>(put) + i, pv);
                 });
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
__global__ void __launch_bounds__(256, 4) map_reduce_kernel(const float* __restrict__ S, const float* __restrict__ X,
                                                         const float* __restrict__ T, int64_t n, Consts c,
                                                         double* __restrict__ sums, unsigned* ticket,
                                                         double2* __restrict__ partial) {
    __shared__ double2 s_part[8];
    __shared__ int s_last;
    pdl_enter();
    // per-thread partials of w and u in fp32 (a thread prices ~n/(grid*256) options), fp64 from
    // the warp up; sum call = sum w + sum u / 2, sum put = sum w - sum u / 2 (price2_wu)
    float2 aw = make_float2(0.f, 0.f), au = make_float2(0.f, 0.f);
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    sweep_groups(reinterpret_cast<const float4*>(S), reinterpret_cast<const float4*>(X),
                 reinterpret_cast<const float4*>(T), blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x,
                 n4, stride, [&](int64_t, const float4& s, const float4& x, const float4& t) {
                     float2 w0, u0, w1, u1;
                     price2_wu(make_float2(s.x, s.y), make_float2(x.x, x.y), make_float2(t.x, t.y), c, w0, u0);
                     price2_wu(make_float2(s.z, s.w), make_float2(x.z, x.w), make_float2(t.z, t.w), c, w1, u1);
                     aw = add2(aw, add2(w0, w1));
                     au = add2(au, add2(u0, u1));
                 });
    const double w = static_cast<double>(aw.x) + static_cast<double>(aw.y);
    const double hu = 0.5 * (static_cast<double>(au.x) + static_cast<double>(au.y));
    double ac = w + hu, ap = w - hu;
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
        for (int k = 1; k < (blockDim.x >> 5); ++k) { b.x += s_part[k].x; b.y += s_part[k].y; }
        __stcg(partial + blockIdx.x, b);
        // acq_rel ticket: releases this CTA's partial, and the last CTA's thread 0 acquires every
        // other CTA's (the __syncthreads below extends the order to the combining threads)
        unsigned prev;
        asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(prev) : "l"(ticket) : "memory");
        s_last = (prev == gridDim.x - 1);
    }
    __syncthreads();
    if (!s_last) return;
    // Last CTA: combine the CTA partials in a fixed order with every thread: thread t takes partials
    // t, t + 256, ... (at most kMaxCtas / 256 = 5, all loads issued before the adds: one L2 round trip
    // instead of the three of a one-warp loop), then the warp shuffle tree and the warps in order.
    constexpr int kPer = (red::kMaxCtas + 255) / 256;
    double2 pv[kPer];
#pragma unroll
    for (int q = 0; q < kPer; ++q) {
        const unsigned k = threadIdx.x + 256u * q;
        pv[q] = k < gridDim.x ? __ldcg(partial + k) : make_double2(0.0, 0.0);
    }
    double bx = pv[0].x, by = pv[0].y;
#pragma unroll
    for (int q = 1; q < kPer; ++q) { bx += pv[q].x; by += pv[q].y; }
    bx = warp_sum(bx);
    by = warp_sum(by);
    __syncthreads();                               // s_part[] was last read by thread 0 above
    if (lane_id() == 0) s_part[warp] = make_double2(bx, by);
    __syncthreads();
    if (threadIdx.x == 0) {
        double2 b = s_part[0];
        for (int k = 1; k < (blockDim.x >> 5); ++k) { b.x += s_part[k].x; b.y += s_part[k].y; }
        sums[0] = b.x;
        sums[1] = b.y;
        *ticket = 0u;   // leave the workspace zeroed
    }
}

static Consts make_consts(float r, float sigma) {
    Consts c;
    c.r_plus_half_s2 = r + 0.5f * sigma * sigma;
    c.inv_sigma = 1.0f / sigma;
    c.sigma = sigma;
    c.neg_r_log2e = -r * 1.44269504088896341f;
    c.a_l2 = static_cast<float>((static_cast<double>(r) + 0.5 * sigma * static_cast<double>(sigma)) * 1.4426950408889634);
    c.b_l2 = static_cast<float>((static_cast<double>(r) - 0.5 * sigma * static_cast<double>(sigma)) * 1.4426950408889634);
    c.ln2_over_sigma = static_cast<float>(0.6931471805599453 / sigma);
    return c;
}

static int grid_for(const void* kernel, int64_t n) {
    const int ov = launch_override().grid_ctas;
    if (ov > 0) return ov;
    const int per_sm = mx(1, cached_occupancy(kernel, 256, 0));
    const int64_t need = ceil_div<int64_t>(mx<int64_t>(n >> 2, 1), 256);
    return static_cast<int>(mn<int64_t>(need, static_cast<int64_t>(per_sm) * device_num_sms()));
}

cudaError_t launch_map(const float* S, const float* X, const float* T, int64_t n, float r, float sigma,
                       float* call, float* put, cudaStream_t stream) {
    if (n == 0) return cudaSuccess;
    const int grid = grid_for(reinterpret_cast<const void*>(&map_kernel), n);
    return launch_pdl(&map_kernel, dim3(grid), dim3(256), 0, stream, S, X, T, n, make_consts(r, sigma), call, put);
}

cudaError_t launch_map_reduce(const float* S, const float* X, const float* T, int64_t n, float r,
                              float sigma, double* sums, void* ws, cudaStream_t stream) {
    int grid = grid_for(reinterpret_cast<const void*>(&map_reduce_kernel), n);
    if (grid > red::kMaxCtas) grid = red::kMaxCtas;
    unsigned* ticket = static_cast<unsigned*>(ws);
    double2* partial = reinterpret_cast<double2*>(static_cast<char*>(ws) + 256);
    return launch_pdl(&map_reduce_kernel, dim3(grid), dim3(256), 0, stream, S, X, T, n, make_consts(r, sigma), sums,
                      ticket, partial);
}

}  // namespace bs
}  // namespace lime
