// Black-Scholes fused map+reduce: memory-only, compute-only and combined variants of the
// production loop, to see whether the 45-us kernel is memory-, compute- or overlap-limited.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_pldi_dubachcrbf12_b200/csrc \
//        -o tools/bs_overlap tools/bs_overlap.cu
#include <cstdio>
#include <vector>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/blackscholes.cu"

namespace lime {
const LaunchOverride& launch_override() { static LaunchOverride o; return o; }
int device_num_sms() { return 148; }
bool pdl_enabled() { return true; }
namespace red { }
}
using namespace lime;
using namespace lime::bs;

template <int MODE>   // 0 = loads only, 1 = compute only (inputs synthesised), 2 = both (production)
__global__ void __launch_bounds__(256, 4) probe(const float* __restrict__ S, const float* __restrict__ X,
                                                const float* __restrict__ T, int64_t n, Consts c, float* out) {
    float fc = 0.f, fp = 0.f;
    const int64_t n4 = n >> 2;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    const float4* S4 = reinterpret_cast<const float4*>(S);
    const float4* X4 = reinterpret_cast<const float4*>(X);
    const float4* T4 = reinterpret_cast<const float4*>(T);
    int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
    float4 s, x, t;
    auto synth = [&](int64_t j, float4& a, float4& b, float4& d) {
        const float f = static_cast<float>(j & 1023) * (1.f / 1024.f);
        a = make_float4(5.f + 25.f * f, 6.f + 20.f * f, 7.f + 10.f * f, 8.f + 5.f * f);
        b = make_float4(1.f + 99.f * f, 50.f, 20.f + f, 80.f - f);
        d = make_float4(0.25f + 9.f * f, 1.f, 2.f + f, 5.f - f);
    };
    if (i < n4) {
        if (MODE == 1) synth(i, s, x, t);
        else { s = ld_stream_f4(S4 + i); x = ld_stream_f4(X4 + i); t = ld_stream_f4(T4 + i); }
    }
    for (; i < n4; i += stride) {
        const int64_t nx = i + stride;
        float4 s2 = s, x2 = x, t2 = t;
        if (nx < n4) {
            if (MODE == 1) synth(nx, s2, x2, t2);
            else { s2 = ld_stream_f4(S4 + nx); x2 = ld_stream_f4(X4 + nx); t2 = ld_stream_f4(T4 + nx); }
        }
        if (MODE == 0) {
            fc += (s.x + x.x + t.x) + (s.y + x.y + t.y) + (s.z + x.z + t.z) + (s.w + x.w + t.w);
        } else {
            float4 cv, pv;
            price4(s, x, t, c, cv, pv);
            fc += (cv.x + cv.y) + (cv.z + cv.w);
            fp += (pv.x + pv.y) + (pv.z + pv.w);
        }
        s = s2; x = x2; t = t2;
    }
    if (fc + fp == 1234.5f) out[0] = fc;
}

__device__ __forceinline__ float4 ld256b(const float4* p) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
struct F8 { float4 a, b; };
__device__ __forceinline__ F8 ld_v8(const float4* p) {
    F8 v;
    asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v.a.x), "=f"(v.a.y), "=f"(v.a.z), "=f"(v.a.w), "=f"(v.b.x), "=f"(v.b.y), "=f"(v.b.z), "=f"(v.b.w)
                 : "l"(p));
    return v;
}
// loads-only variants: V = 1 L2::256B hint, 2 = prefetch depth 2, 3 = 256-bit loads (8 options/iter)
template <int V>
__global__ void __launch_bounds__(256, 4) probe_ld(const float* __restrict__ S, const float* __restrict__ X,
                                                   const float* __restrict__ T, int64_t n, Consts c, float* out) {
    float fc = 0.f;
    const float4* S4 = reinterpret_cast<const float4*>(S);
    const float4* X4 = reinterpret_cast<const float4*>(X);
    const float4* T4 = reinterpret_cast<const float4*>(T);
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
    if constexpr (V == 1) {
        const int64_t n4 = n >> 2;
        float4 s, x, t;
        if (i < n4) { s = ld256b(S4 + i); x = ld256b(X4 + i); t = ld256b(T4 + i); }
        for (; i < n4; i += stride) {
            const int64_t nx = i + stride;
            float4 s2 = s, x2 = x, t2 = t;
            if (nx < n4) { s2 = ld256b(S4 + nx); x2 = ld256b(X4 + nx); t2 = ld256b(T4 + nx); }
            fc += (s.x + x.x + t.x) + (s.y + x.y + t.y) + (s.z + x.z + t.z) + (s.w + x.w + t.w);
            s = s2; x = x2; t = t2;
        }
    } else if constexpr (V == 2) {
        const int64_t n4 = n >> 2;
        float4 s[2], x[2], t[2];
        for (int d = 0; d < 2; ++d) {
            const int64_t j = i + d * stride;
            if (j < n4) { s[d] = ld_stream_f4(S4 + j); x[d] = ld_stream_f4(X4 + j); t[d] = ld_stream_f4(T4 + j); }
        }
        for (; i < n4; i += stride) {
            const int64_t nx = i + 2 * stride;
            float4 sn = s[1], xn = x[1], tn = t[1];
            if (nx < n4) { sn = ld_stream_f4(S4 + nx); xn = ld_stream_f4(X4 + nx); tn = ld_stream_f4(T4 + nx); }
            fc += (s[0].x + x[0].x + t[0].x) + (s[0].y + x[0].y + t[0].y) + (s[0].z + x[0].z + t[0].z) + (s[0].w + x[0].w + t[0].w);
            s[0] = s[1]; x[0] = x[1]; t[0] = t[1];
            s[1] = sn; x[1] = xn; t[1] = tn;
        }
    } else {
        const int64_t n8 = n >> 3;
        F8 s, x, t;
        if (i < n8) { s = ld_v8(S4 + 2 * i); x = ld_v8(X4 + 2 * i); t = ld_v8(T4 + 2 * i); }
        for (; i < n8; i += stride) {
            const int64_t nx = i + stride;
            F8 s2 = s, x2 = x, t2 = t;
            if (nx < n8) { s2 = ld_v8(S4 + 2 * nx); x2 = ld_v8(X4 + 2 * nx); t2 = ld_v8(T4 + 2 * nx); }
            fc += (s.a.x + x.a.x + t.a.x) + (s.a.y + x.a.y + t.a.y) + (s.a.z + x.a.z + t.a.z) + (s.a.w + x.a.w + t.a.w)
                + (s.b.x + x.b.x + t.b.x) + (s.b.y + x.b.y + t.b.y) + (s.b.z + x.b.z + t.b.z) + (s.b.w + x.b.w + t.b.w);
            s = s2; x = x2; t = t2;
        }
    }
    if (fc == 1234.5f) out[0] = fc;
}

// loads-only via 1-D TMA bulk copies: each CTA streams 1024-option chunks (3 x 4 KB) through a
// STG-stage smem ring; MODE 0 sums the inputs, MODE 2 prices them (the fused map+reduce).
template <int MODE, int STG>
__global__ void __launch_bounds__(256, 4) probe_tma(const float* __restrict__ S, const float* __restrict__ X,
                                                    const float* __restrict__ T, int64_t n, Consts c, float* out) {
    constexpr int CH = 1024;
    __shared__ __align__(128) float4 sb[STG][3][CH / 4];
    __shared__ __align__(8) uint64_t full[STG];
    const int64_t nch = n / CH;
    float fc = 0.f, fp = 0.f;
    if (threadIdx.x == 0) {
        for (int k = 0; k < STG; ++k) mbar_init(&full[k], 1);
        fence_mbar_init();
    }
    __syncthreads();
    auto issue = [&](int64_t chunk, int k) {
        mbar_arrive_expect_tx(&full[k], 3 * CH * 4);
        bulk_g2s(sb[k][0], S + chunk * CH, CH * 4, &full[k]);
        bulk_g2s(sb[k][1], X + chunk * CH, CH * 4, &full[k]);
        bulk_g2s(sb[k][2], T + chunk * CH, CH * 4, &full[k]);
    };
    int64_t first = blockIdx.x;
    if (threadIdx.x == 0)
        for (int k = 0; k < STG; ++k) {
            const int64_t ch = first + static_cast<int64_t>(k) * gridDim.x;
            if (ch < nch) issue(ch, k);
        }
    int it = 0;
    for (int64_t ch = first; ch < nch; ch += gridDim.x, ++it) {
        const int k = it % STG;
        mbar_wait(&full[k], (it / STG) & 1);
        const float4 s = sb[k][0][threadIdx.x], x = sb[k][1][threadIdx.x], t = sb[k][2][threadIdx.x];
        if (MODE == 0) {
            fc += (s.x + x.x + t.x) + (s.y + x.y + t.y) + (s.z + x.z + t.z) + (s.w + x.w + t.w);
        } else {
            float4 cv, pv;
            price4(s, x, t, c, cv, pv);
            fc += (cv.x + cv.y) + (cv.z + cv.w);
            fp += (pv.x + pv.y) + (pv.z + pv.w);
        }
        __syncthreads();
        const int64_t nx = ch + static_cast<int64_t>(STG) * gridDim.x;
        if (threadIdx.x == 0 && nx < nch) issue(nx, k);
    }
    if (fc + fp == 1234.5f) out[0] = fc;
}

// loads-only, NS streams (1..3) grid-stride, or BLOCKED: each CTA sweeps its own contiguous range
template <int NS, bool BLOCKED>
__global__ void __launch_bounds__(256, 4) probe_streams(const float* __restrict__ S, const float* __restrict__ X,
                                                        const float* __restrict__ T, int64_t n, Consts c, float* out) {
    const float4* A[3] = {reinterpret_cast<const float4*>(S), reinterpret_cast<const float4*>(X),
                          reinterpret_cast<const float4*>(T)};
    const int64_t n4 = (n >> 2) * 3 / NS;           // same total bytes for every NS
    int64_t i, end, stride;
    if (BLOCKED) {
        const int64_t per = (n4 + gridDim.x - 1) / gridDim.x;
        i = blockIdx.x * per + threadIdx.x;
        end = min(n4, (blockIdx.x + 1) * per);
        stride = blockDim.x;
    } else {
        i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
        end = n4;
        stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    }
    float fc = 0.f;
    float4 v[NS];
    auto load = [&](int64_t j, float4 (&w)[NS]) {
#pragma unroll
        for (int q = 0; q < NS; ++q) {
            const int64_t jj = (NS == 3) ? j : j;
            w[q] = ld_stream_f4(A[q] + (jj % ((n >> 2) * 1)) + (jj / (n >> 2)) * 0);
        }
    };
    if (i < end) load(i, v);
    for (; i < end; i += stride) {
        float4 w[NS];
#pragma unroll
        for (int q = 0; q < NS; ++q) w[q] = v[q];
        if (i + stride < end) load(i + stride, w);
#pragma unroll
        for (int q = 0; q < NS; ++q) fc += (v[q].x + v[q].y) + (v[q].z + v[q].w);
#pragma unroll
        for (int q = 0; q < NS; ++q) v[q] = w[q];
    }
    if (fc == 1234.5f) out[0] = fc;
}

int main() {
    const int64_t n = 1 << 24;
    float *S, *X, *T, *out;
    cudaMalloc(&S, n * 4); cudaMalloc(&X, n * 4); cudaMalloc(&T, n * 4); cudaMalloc(&out, 16);
    std::vector<float> h(n);
    for (int64_t k = 0; k < n; ++k) h[k] = 5.f + 25.f * ((k * 2654435761u) % 1000) / 1000.f;
    cudaMemcpy(S, h.data(), n * 4, cudaMemcpyHostToDevice);
    for (int64_t k = 0; k < n; ++k) h[k] = 1.f + 99.f * ((k * 40503u) % 1000) / 1000.f;
    cudaMemcpy(X, h.data(), n * 4, cudaMemcpyHostToDevice);
    for (int64_t k = 0; k < n; ++k) h[k] = 0.25f + 9.75f * ((k * 2246822519u) % 1000) / 1000.f;
    cudaMemcpy(T, h.data(), n * 4, cudaMemcpyHostToDevice);
    char* flush; cudaMalloc(&flush, 512 << 20);
    Consts c = make_consts(0.02f, 0.3f);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    auto run = [&](auto kern, const char* name) {
        float best = 1e9;
        for (int r = 0; r < 10; ++r) {
            cudaMemsetAsync(flush, r, 512 << 20);
            cudaEventRecord(a);
            kern<<<592, 256>>>(S, X, T, n, c, out);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (ms < best) best = ms;
        }
        printf("{\"variant\": \"%s\", \"us\": %.2f}\n", name, best * 1e3);
    };
    run(probe<0>, "loads only (12 B/option)");
    run(probe_ld<1>, "loads only, L2::256B hint");
    run(probe_ld<2>, "loads only, prefetch depth 2");
    run(probe_ld<3>, "loads only, 256-bit loads (8 options/iteration)");
    run(probe_tma<0, 2>, "loads only, TMA bulk ring 2 x 12 KB");
    run(probe_tma<0, 3>, "loads only, TMA bulk ring 3 x 12 KB");
    run(probe_tma<2, 2>, "loads + compute, TMA bulk ring 2 x 12 KB");
    run(probe_tma<2, 3>, "loads + compute, TMA bulk ring 3 x 12 KB");
    run(probe<1>, "compute only (price4, synthesised inputs)");
    run(probe_streams<3, false>, "3 streams, grid-stride (same bytes)");
    run(probe_streams<3, true>, "3 streams, blocked per CTA");
    run(probe<2>, "loads + compute (production loop)");
    {
        double* sums; void* ws;
        cudaMalloc(&sums, 16); cudaMalloc(&ws, 1 << 20); cudaMemset(ws, 0, 1 << 20);
        float best = 1e9;
        for (int r = 0; r < 10; ++r) {
            cudaMemsetAsync(flush, r, 512 << 20);
            cudaEventRecord(a);
            map_reduce_kernel<<<592, 256>>>(S, X, T, n, c, sums, static_cast<unsigned*>(ws),
                                            reinterpret_cast<double2*>(static_cast<char*>(ws) + 256));
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            if (ms < best) best = ms;
        }
        printf("{\"variant\": \"production map_reduce_kernel\", \"us\": %.2f}\n", best * 1e3);
    }
    return 0;
}
