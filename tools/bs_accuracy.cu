// bs_accuracy.cu -- element-accuracy A/B of Black-Scholes pricing variants (r02r).
// Reads n and S, X, T (float32) from argv[1], writes call/put per variant to argv[2].
// Variants: bit 0 = ln(S/X) as lg2(S * rcp(X)) instead of lg2 S - lg2 X (same MUFU count);
//           bit 1 = degree-7 Mills-ratio polynomial (max |dN| 5.0e-10) instead of A&S 26.2.17 (7.5e-8).
// build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o tools/bs_accuracy tools/bs_accuracy.cu
#include <cstdio>
#include <cstdlib>
#include <vector>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/common.cuh"
using namespace lime;

__device__ __forceinline__ float poly5(float k) {
    return k * fmaf(k, fmaf(k, fmaf(k, fmaf(k, 1.330274429f, -1.821255978f), 1.781477937f), -0.356563782f), 0.319381530f);
}
__device__ __forceinline__ float poly7(float k) {
    float p = fmaf(k, 1.1605857361e-01f, -6.2049898640e-01f);
    p = fmaf(k, p, 1.0789559974e+00f);
    p = fmaf(k, p, -4.7603565775e-01f);
    p = fmaf(k, p, 5.7942646417e-01f);
    p = fmaf(k, p, 2.5091390071e-01f);
    p = fmaf(k, p, 3.2449384680e-01f);
    return k * p;
}

template <int V>
__global__ void price_kernel(const float* S, const float* X, const float* T, int n, float r, float sigma, float* call, float* put) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    const float s = S[i], x = X[i], t = T[i];
    const float rsT = rsqrt_approx(t);
    const float sqT = t * rsT;
    const float v = sigma * sqT;
    const float inv_v = rsT * (1.0f / sigma);
    float lg;
    if (V & 1) lg = lg2_approx(s * rcp_approx(x));
    else lg = lg2_approx(s) - lg2_approx(x);
    const float l = lg * 0.693147180559945309f;
    const float d1 = fmaf(r + 0.5f * sigma * sigma, t, l) * inv_v;
    const float d2 = d1 - v;
    const float K = x * ex2_approx(-r * 1.44269504088896341f * t);
    const float p = (V & 2) ? 0.318f : 0.2316419f;
    const float D1 = fmaf(p, fabsf(d1), 1.f), D2 = fmaf(p, fabsf(d2), 1.f);
    const float rr = rcp_approx(D1 * D2);
    const float k1 = D2 * rr, k2 = D1 * rr;
    float ph = 0.398942280401432678f * ex2_approx(-0.721347520444481703f * d1 * d1);
    if ((V & 4) && fabsf(d1) < 0.5f) {          // phi(d1) by its Taylor series: x = d1^2/2 <= 1/8, |err| < 1e-10
        const float x = 0.5f * d1 * d1;
        float e = fmaf(x, 1.f / 720.f, -1.f / 120.f);
        e = fmaf(x, e, 1.f / 24.f);
        e = fmaf(x, e, -1.f / 6.f);
        e = fmaf(x, e, 0.5f);
        e = fmaf(x, e, -1.f);
        e = fmaf(x, e, 1.f);
        ph = 0.398942280401432678f * e;
    }
    const float sphi = s * ph;
    const float q1 = (V & 2) ? poly7(k1) : poly5(k1), q2 = (V & 2) ? poly7(k2) : poly5(k2);
    const float sq1 = sphi * q1, kq2 = sphi * q2;             // S N(-|d1|), K N(-|d2|)
    const float s_m = s - sq1, k_m = K - kq2;
    const float sn1 = d1 >= 0.f ? s_m : sq1, snm1 = d1 >= 0.f ? sq1 : s_m;
    const float kn2 = d2 >= 0.f ? k_m : kq2, knm2 = d2 >= 0.f ? kq2 : k_m;
    call[i] = sn1 - kn2;
    put[i] = knm2 - snm1;
}

int main(int argc, char** argv) {
    FILE* f = fopen(argv[1], "rb");
    int n;
    float r, sigma;
    if (fread(&n, 4, 1, f) != 1 || fread(&r, 4, 1, f) != 1 || fread(&sigma, 4, 1, f) != 1) return 1;
    std::vector<float> h(3 * (size_t)n);
    if (fread(h.data(), 4, h.size(), f) != h.size()) return 1;
    fclose(f);
    float *d, *o;
    cudaMalloc(&d, 12 * (size_t)n);
    cudaMalloc(&o, 8 * (size_t)n);
    cudaMemcpy(d, h.data(), 12 * (size_t)n, cudaMemcpyHostToDevice);
    std::vector<float> out(8 * (size_t)n);
    FILE* g = fopen(argv[2], "wb");
    for (int v = 0; v < 8; ++v) {
        const dim3 grid((n + 255) / 256);
        switch (v) {
            case 0: price_kernel<0><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 1: price_kernel<1><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 2: price_kernel<2><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 4: price_kernel<6><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 5: price_kernel<7><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 6: price_kernel<4><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 7: price_kernel<5><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
            case 3: price_kernel<3><<<grid, 256>>>(d, d + n, d + 2 * (size_t)n, n, r, sigma, o, o + n); break;
        }
        cudaMemcpy(out.data(), o, 8 * (size_t)n, cudaMemcpyDeviceToHost);
        fwrite(out.data(), 4, 2 * (size_t)n, g);
    }
    fclose(g);
    return cudaGetLastError() != cudaSuccess;
}
