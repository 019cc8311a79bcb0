// jgf.cu -- the paper's Java Grande benchmarks as maps: JG-Series (Fourier
// coefficients, Table 3) and JG-Crypt (IDEA, L354-355), sm_100a.
//
// JG-Series (reading DESIGN.md R14). Every coefficient n integrates f(x) = (x+1)^x against
// cos/sin(n pi x) on the same 1001 trapezoid nodes, so the map over n has a broadcast operand: the
// node table g_i = w_i f(x_i) (w = 1/2 at the ends, 0 at JGF's skipped node x_{m-1}, 1 elsewhere).
// The phase n pi x_i = 2 pi (n i mod m)/m is reduced EXACTLY in integers, so the trigonometric
// factors come from an m-entry table of e^{2 pi i p/m} (built per call in fp64, rounded to the
// variant's precision) -- no range-reduction error at n = 10^5 and no MUFU.
// B200 form (radix-32 split of the node index, i = 32u + v, g zero-padded to 1024 nodes):
//   sum_i g_i e^{i theta n i} = sum_u U_u * W_u,  U_u = e^{i theta n 32u},  W_u = sum_v g_{32u+v} V_v,
//   V_v = e^{i theta n v}.
// Each thread gathers its coefficient's 32 V_v into REGISTERS (a fully unrolled inner loop indexes
// them statically), so the 1024 inner terms are one packed FFMA2 each (re and im together) with g
// read by LDS.128 broadcasts; only the 32 V and 32 U table reads per coefficient are lane-divergent
// gathers (bank conflicts there cost ~2 % instead of the 2002 conflicting reads per coefficient of
// the direct form). Every factor is an exactly rounded table value; the one extra rounding per U_u W_u
// product is bounded by 2 eps sum_u |W_u| <= 2 eps T[|f|].
//
// JG-Crypt (reading R15): IDEA ECB; each thread enciphers 16-byte units (two blocks) with one
// 128-bit load/store; multiplication modulo 2^16+1 is the branch-free low/high-half form; the 52
// sub-keys are a __grid_constant__ parameter (the paper's constant-memory mapping, L263-266).
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace jgf {

// ------------------------------------------------------------------ JG-Series
constexpr int kSeriesM = 1000;   // JGF: TrapezoidIntegrate(0, 2, 1000, ...)

template <typename T>
__global__ void __launch_bounds__(256) series_tables_kernel(T* g, T* cs, T* sn) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i <= kSeriesM) {
        const double x = (2.0 / kSeriesM) * i;
        const double w = (i == 0 || i == kSeriesM) ? 0.5 : (i == kSeriesM - 1 ? 0.0 : 1.0);
        g[i] = static_cast<T>(w * pow(x + 1.0, x));
    } else if (i < 1024) {
        g[i] = 0;                                    // padding nodes of the radix-32 split
    }
    if (i < kSeriesM) {
        double s, c;
        sincospi(2.0 * i / kSeriesM, &s, &c);   // angle 2 pi i / m
        cs[i] = static_cast<T>(c);
        sn[i] = static_cast<T>(s);
    }
}

constexpr int kSeriesRadix = 32;          // i = 32 u + v; 32 x 32 = 1024 >= m + 1 nodes
constexpr int kSeriesNodes = kSeriesRadix * kSeriesRadix;
constexpr int kSeriesBlock = 128;

// (wr, wi) += g * (vr, vi): one FFMA2 in fp32 (bcast g), two DFMA in fp64
__device__ __forceinline__ float2 cfma(float g, float2 v, float2 w) { return fma2(bcast2(g), v, w); }
__device__ __forceinline__ double2 cfma(double g, double2 v, double2 w) {
    return make_double2(fma(g, v.x, w.x), fma(g, v.y, w.y));
}
template <typename T> struct Vec2;
template <> struct Vec2<float> { using type = float2; };
template <> struct Vec2<double> { using type = double2; };

template <typename T>
__global__ void __launch_bounds__(kSeriesBlock) series_kernel(const T* __restrict__ g, const T* __restrict__ cs,
                                                              const T* __restrict__ sn, int64_t n0, int64_t count,
                                                              T* __restrict__ out) {
    using T2 = typename Vec2<T>::type;
    __shared__ __align__(16) T sg[kSeriesNodes];
    __shared__ T sc[kSeriesM], ss[kSeriesM];
    for (int i = threadIdx.x; i < kSeriesNodes; i += blockDim.x) sg[i] = g[i];      // g[i > m] = 0
    for (int i = threadIdx.x; i < kSeriesM; i += blockDim.x) { sc[i] = cs[i]; ss[i] = sn[i]; }
    __syncthreads();
    const T dx = static_cast<T>(2.0 / kSeriesM);
    for (int64_t k = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; k < count;
         k += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t n = n0 + k;
        const int step = static_cast<int>(n % kSeriesM);
        T2 V[kSeriesRadix];                           // V_v = e^{i theta (n v mod m)}
        int p = 0;
#pragma unroll
        for (int v = 0; v < kSeriesRadix; ++v) {
            V[v].x = sc[p];
            V[v].y = ss[p];
            p += step;
            p -= (p >= kSeriesM) ? kSeriesM : 0;
        }
        const int step_u = p;                         // 32 n mod m
        int q = 0;                                    // 32 n u mod m
        T a = 0, b = 0;
#pragma unroll 1
        for (int u = 0; u < kSeriesRadix; ++u) {
            T2 w0, w1;                                // W_u, even and odd v (two dependency chains)
            w0.x = w0.y = w1.x = w1.y = 0;
            const T* gu = sg + u * kSeriesRadix;
#pragma unroll
            for (int v = 0; v < kSeriesRadix; v += 4) {
                T gv[4];
                if constexpr (sizeof(T) == 4) {
                    const float4 t = *reinterpret_cast<const float4*>(gu + v);
                    gv[0] = t.x; gv[1] = t.y; gv[2] = t.z; gv[3] = t.w;
                } else {
                    const double2 t0 = *reinterpret_cast<const double2*>(gu + v);
                    const double2 t1 = *reinterpret_cast<const double2*>(gu + v + 2);
                    gv[0] = t0.x; gv[1] = t0.y; gv[2] = t1.x; gv[3] = t1.y;
                }
                w0 = cfma(gv[0], V[v + 0], w0);
                w1 = cfma(gv[1], V[v + 1], w1);
                w0 = cfma(gv[2], V[v + 2], w0);
                w1 = cfma(gv[3], V[v + 3], w1);
            }
            const T wr = w0.x + w1.x, wi = w0.y + w1.y;
            const T ur = sc[q], ui = ss[q];
            a = fma(ur, wr, a);
            a = fma(-ui, wi, a);                      // Re(U W)
            b = fma(ur, wi, b);
            b = fma(ui, wr, b);                       // Im(U W)
            q += step_u;
            q -= (q >= kSeriesM) ? kSeriesM : 0;
        }
        if (n == 0) { a = a * static_cast<T>(0.5); b = 0; }   // a_0 = T[f] / 2, b_0 = 0
        out[2 * k + 0] = a * dx;
        out[2 * k + 1] = b * dx;
    }
}

size_t series_workspace_bytes(bool f64) { return (f64 ? 8 : 4) * 3 * 1024 + 256; }

template <typename T>
static cudaError_t launch_series_t(int64_t n0, int64_t count, T* out, void* ws, cudaStream_t stream) {
    T* g = static_cast<T*>(ws);
    T* cs = g + 1024;
    T* sn = cs + 1024;
    series_tables_kernel<T><<<ceil_div(kSeriesNodes, 256), 256, 0, stream>>>(g, cs, sn);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess || count == 0) return e;
    int grid = launch_override().grid_ctas;
    if (grid <= 0) grid = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(count, kSeriesBlock), 16LL * device_num_sms()));
    series_kernel<T><<<grid, kSeriesBlock, 0, stream>>>(g, cs, sn, n0, count, out);
    return cudaGetLastError();
}

cudaError_t launch_series_f32(int64_t n0, int64_t count, float* out, void* ws, cudaStream_t stream) {
    return launch_series_t<float>(n0, count, out, ws, stream);
}
cudaError_t launch_series_f64(int64_t n0, int64_t count, double* out, void* ws, cudaStream_t stream) {
    return launch_series_t<double>(n0, count, out, ws, stream);
}

// ------------------------------------------------------------------ JG-Crypt (IDEA)
struct IdeaKeys {
    uint32_t z[52];
};

__device__ __forceinline__ uint32_t idea_mul(uint32_t a, uint32_t b) {
    // a * b mod (2^16 + 1) on 16-bit operands where 0 stands for 2^16
    const uint32_t p = a * b;
    const uint32_t lo = p & 0xFFFFu, hi = p >> 16;
    const uint32_t r = lo - hi + (lo < hi ? 1u : 0u);
    return (p != 0u ? r : (1u - a - b)) & 0xFFFFu;
}

__device__ __forceinline__ uint2 idea_block(uint2 v, const IdeaKeys& k) {
    // bytes b0..b7 of the block; words are big-endian (R15)
    uint32_t x1 = __byte_perm(v.x, 0, 0x4401), x2 = __byte_perm(v.x, 0, 0x4423);
    uint32_t x3 = __byte_perm(v.y, 0, 0x4401), x4 = __byte_perm(v.y, 0, 0x4423);
#pragma unroll
    for (int r = 0; r < 8; ++r) {
        const uint32_t* z = k.z + 6 * r;
        x1 = idea_mul(x1, z[0]);
        x2 = (x2 + z[1]) & 0xFFFFu;
        x3 = (x3 + z[2]) & 0xFFFFu;
        x4 = idea_mul(x4, z[3]);
        const uint32_t t0 = idea_mul(x1 ^ x3, z[4]);
        const uint32_t t1 = idea_mul((t0 + (x2 ^ x4)) & 0xFFFFu, z[5]);
        const uint32_t t2 = (t0 + t1) & 0xFFFFu;
        x1 ^= t1;
        x4 ^= t2;
        const uint32_t a = x2 ^ t2;
        x2 = x3 ^ t1;
        x3 = a;
    }
    const uint32_t y1 = idea_mul(x1, k.z[48]);
    const uint32_t y2 = (x3 + k.z[49]) & 0xFFFFu;
    const uint32_t y3 = (x2 + k.z[50]) & 0xFFFFu;
    const uint32_t y4 = idea_mul(x4, k.z[51]);
    // back to bytes: word w -> (hi byte, lo byte)
    return make_uint2(__byte_perm(y1, y2, 0x4501), __byte_perm(y3, y4, 0x4501));
}

__global__ void __launch_bounds__(256) idea_kernel(const uint4* __restrict__ in, uint4* __restrict__ out, int64_t units,
                                                   const uint2* __restrict__ tail_in, uint2* __restrict__ tail_out,
                                                   int has_tail, const __grid_constant__ IdeaKeys k) {
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < units;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        uint4 v;
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(in + i));
        const uint2 a = idea_block(make_uint2(v.x, v.y), k);
        const uint2 b = idea_block(make_uint2(v.z, v.w), k);
        out[i] = make_uint4(a.x, a.y, b.x, b.y);
    }
    if (has_tail && blockIdx.x == 0 && threadIdx.x == 0) *tail_out = idea_block(*tail_in, k);
}

cudaError_t launch_idea(const uint8_t* in, uint8_t* out, int64_t nbytes, const uint16_t* subkeys, cudaStream_t stream) {
    if (nbytes == 0) return cudaSuccess;
    IdeaKeys k;
    for (int i = 0; i < 52; ++i) k.z[i] = subkeys[i];
    const int64_t units = nbytes / 16;                 // 16-byte units (two blocks)
    const int has_tail = (nbytes % 16) != 0;           // one trailing 8-byte block
    int grid = launch_override().grid_ctas;
    if (grid <= 0) grid = static_cast<int>(mn<int64_t>(mx<int64_t>(1, ceil_div<int64_t>(units, 256)), 8LL * device_num_sms()));
    idea_kernel<<<grid, 256, 0, stream>>>(reinterpret_cast<const uint4*>(in), reinterpret_cast<uint4*>(out), units,
                                          reinterpret_cast<const uint2*>(in + units * 16),
                                          reinterpret_cast<uint2*>(out + units * 16), has_tail, k);
    return cudaGetLastError();
}

// Host-side key schedule (the cipher's setup, not the hot path): 52 encryption sub-keys by 25-bit
// rotations of the 128-bit key; decryption sub-keys are the multiplicative / additive inverses in
// reverse round order.
static uint16_t mul_inv_host(uint16_t a) {
    if (a <= 1) return a;                               // 0 (= 2^16) and 1 are self-inverse
    int64_t t0 = 1, t1 = 0, r0 = a, r1 = 65537;          // extended Euclid on (a, 65537)
    while (r1 != 0) {
        const int64_t q = r0 / r1;
        int64_t tmp = r0 - q * r1; r0 = r1; r1 = tmp;
        tmp = t0 - q * t1; t0 = t1; t1 = tmp;
    }
    int64_t inv = t0 % 65537;
    if (inv < 0) inv += 65537;
    return static_cast<uint16_t>(inv);
}

void idea_key_schedule(const uint16_t key[8], uint16_t ek[52], uint16_t dk[52]) {
    uint16_t w[8];
    for (int i = 0; i < 8; ++i) w[i] = key[i];
    for (int s = 0; s < 52; ++s) {
        ek[s] = w[s % 8];
        if (s % 8 == 7) {                                // rotate the 128-bit key left by 25 bits
            uint16_t nw[8];
            for (int i = 0; i < 8; ++i)
                nw[i] = static_cast<uint16_t>((w[(i + 1) % 8] << 9) | (w[(i + 2) % 8] >> 7));
            for (int i = 0; i < 8; ++i) w[i] = nw[i];
        }
    }
    // decryption round 1, rounds 2..8 (the two additive keys swapped), output transform
    dk[0] = mul_inv_host(ek[48]);
    dk[1] = static_cast<uint16_t>(-ek[49]);
    dk[2] = static_cast<uint16_t>(-ek[50]);
    dk[3] = mul_inv_host(ek[51]);
    dk[4] = ek[46];
    dk[5] = ek[47];
    for (int k = 2; k <= 8; ++k) {
        const int b = 6 * (9 - k), c = 6 * (8 - k), d = 6 * (k - 1);
        dk[d + 0] = mul_inv_host(ek[b]);
        dk[d + 1] = static_cast<uint16_t>(-ek[b + 2]);
        dk[d + 2] = static_cast<uint16_t>(-ek[b + 1]);
        dk[d + 3] = mul_inv_host(ek[b + 3]);
        dk[d + 4] = ek[c + 4];
        dk[d + 5] = ek[c + 5];
    }
    dk[48] = mul_inv_host(ek[0]);
    dk[49] = static_cast<uint16_t>(-ek[1]);
    dk[50] = static_cast<uint16_t>(-ek[2]);
    dk[51] = mul_inv_host(ek[3]);
}

}  // namespace jgf
}  // namespace lime
