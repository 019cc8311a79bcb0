// jgf.cu -- the paper's Java Grande benchmarks as maps: JG-Series (Fourier
// coefficients, Table 3) and JG-Crypt (IDEA, L354-355), sm_100a.
//
// JG-Series (reading DESIGN.md R14). Every coefficient n integrates f(x) = (x+1)^x against
// cos/sin(n pi x) on the same 1001 trapezoid nodes, so the map over n has a broadcast operand: the
// node table g_i = w_i f(x_i) (w = 1/2 at the ends, 0 at JGF's skipped node x_{m-1}, 1 elsewhere).
// The phase n pi x_i = 2 pi (n i mod m)/m is reduced EXACTLY in integers, so the trigonometric
// factors come from an m-entry table of e^{2 pi i p/m} (device fp64 sincospi, rounded to the
// variant's precision, written once per device by an asynchronous kernel) -- no range-reduction error at n = 10^5 and no MUFU.
// B200 form (radix-R split of the node index, i = R u + v, g zero-padded to 1024 nodes):
//   sum_i g_i e^{i theta n i} = sum_u U_u * W_u,  U_u = e^{i theta (R n u mod m)},
//   W_u = sum_v g_{Ru+v} V_v,  V_v = e^{i theta (n v mod m)}.
// Each thread gathers its coefficient's R values V_v into REGISTERS (a fully unrolled inner loop
// indexes them statically), so each inner term is one packed FFMA2 (re and im together) whose g
// operand comes from the kernel-parameter bank (uniform constant loads); only R + 1024/R table reads
// per coefficient are lane-divergent smem gathers (the direct form did 2002, with 17.7M bank
// conflicts per launch). Every factor is an exactly rounded table value; the one extra rounding per
// U_u W_u product is bounded by 2 eps sum_u |W_u| <= 2 eps T[|f|].
//
// JG-Crypt (reading R15): IDEA ECB; each thread enciphers 16-byte units (two blocks) with one
// 128-bit load/store; multiplication modulo 2^16+1 is the branch-free low/high-half form; the 52
// sub-keys are a __grid_constant__ parameter (the paper's constant-memory mapping, L263-266).
#include "common.cuh"
#include "kernels.h"

#include <cmath>
#include <mutex>

namespace lime {
namespace jgf {

// ------------------------------------------------------------------ JG-Series
constexpr int kSeriesM = 1000;            // JGF: TrapezoidIntegrate(0, 2, 1000, ...)
constexpr int kSeriesNodes = 1024;        // m + 1 = 1001 nodes, zero-padded
constexpr int kSeriesBlock = 128;
constexpr int kSeriesPadded = kSeriesM + kSeriesM / 8 + 1;   // smem table slots (one pad per 8)
__device__ __forceinline__ int series_pos(int p) { return p + (p >> 3); }

// Node weights g_i = w_i (x_i + 1)^{x_i} (w = 1/2 at the ends, 0 at the skipped node x_{m-1}), rounded
// to T, as a kernel parameter: the kernel reads them with compile-time offsets, so they arrive through
// the uniform datapath (LDCU into uniform registers, the FFMA2 broadcast operand) -- A2's constant
// broadcast (L263-266) -- and never touch shared memory.
template <typename T>
struct SeriesNodes {
    T g[kSeriesNodes];
};

// e^{2 pi i p / m}, p < m, rounded to T: a per-device table written once (series_tables_kernel).
__device__ float d_series_cos32[kSeriesM], d_series_sin32[kSeriesM];
__device__ double d_series_cos64[kSeriesM], d_series_sin64[kSeriesM];

template <typename T>
static const SeriesNodes<T>& series_nodes() {
    static const SeriesNodes<T> nodes = [] {
        SeriesNodes<T> s{};
        for (int i = 0; i < kSeriesNodes; ++i) {
            const double x = (2.0 / kSeriesM) * i;
            const double w = (i == 0 || i == kSeriesM) ? 0.5 : (i == kSeriesM - 1 ? 0.0 : 1.0);
            s.g[i] = i <= kSeriesM ? static_cast<T>(w * std::pow(x + 1.0, x)) : T(0);
        }
        return s;
    }();
    return nodes;
}

// e^{2 pi i p/m} for p < m in fp64 (device sincospi: within 1 ulp, exact at the quadrant points),
// and the same values rounded to fp32. One thread per p.
__global__ void series_tables_kernel() {
    const int p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= kSeriesM) return;
    double s, c;
    sincospi(2.0 * p / kSeriesM, &s, &c);
    if (p == 250 || p == 750) c = 0.0;             // exact symmetries keep the quadrant points exact
    if (p == 0 || p == 500) s = 0.0;
    d_series_cos64[p] = c;
    d_series_sin64[p] = s;
    d_series_cos32[p] = static_cast<float>(c);
    d_series_sin32[p] = static_cast<float>(s);
}

// The tables are written once per device by series_tables_kernel, enqueued on the FIRST caller's
// stream (no host synchronisation, lime.h's "never synchronises" contract); an event recorded after
// it orders every later call on any other stream behind it (cudaStreamWaitEvent: a device-side
// dependency, free once the event has completed). Inside a stream capture the event cannot be
// waited on, so a capture that may precede the table's completion carries its own (idempotent:
// same values) table kernel.
static cudaError_t series_tables_ready(cudaStream_t stream) {
    static std::mutex mu;
    static bool done[256] = {};
    static cudaEvent_t ready[256] = {};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev < 0 || dev >= 256) return cudaErrorInvalidDevice;
    cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
    if ((e = cudaStreamIsCapturing(stream, &cap)) != cudaSuccess) return e;
    std::lock_guard<std::mutex> lock(mu);
    if (done[dev]) {
        if (cap == cudaStreamCaptureStatusNone) return cudaStreamWaitEvent(stream, ready[dev], 0);
        if (cudaEventQuery(ready[dev]) == cudaSuccess) return cudaSuccess;
        cudaGetLastError();
        series_tables_kernel<<<ceil_div(kSeriesM, 256), 256, 0, stream>>>();
        return cudaGetLastError();
    }
    series_tables_kernel<<<ceil_div(kSeriesM, 256), 256, 0, stream>>>();
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    if (cap != cudaStreamCaptureStatusNone) return cudaSuccess;   // not marked: the capture holds its own copy
    if ((e = cudaEventCreateWithFlags(&ready[dev], cudaEventDisableTiming)) != cudaSuccess) return e;
    if ((e = cudaEventRecord(ready[dev], stream)) != cudaSuccess) return e;
    done[dev] = true;
    return cudaSuccess;
}

// (wr, wi) += g * (vr, vi): one FFMA2 in fp32 (g broadcast), two DFMA in fp64
__device__ __forceinline__ float2 cfma(float g, float2 v, float2 w) { return fma2(bcast2(g), v, w); }
__device__ __forceinline__ double2 cfma(double g, double2 v, double2 w) {
    return make_double2(fma(g, v.x, w.x), fma(g, v.y, w.y));
}
template <typename T> struct Vec2;
template <> struct Vec2<float> { using type = float2; };
template <> struct Vec2<double> { using type = double2; };
template <typename T> __device__ __forceinline__ const T* series_cos();
template <typename T> __device__ __forceinline__ const T* series_sin();
template <> __device__ __forceinline__ const float* series_cos<float>() { return d_series_cos32; }
template <> __device__ __forceinline__ const float* series_sin<float>() { return d_series_sin32; }
template <> __device__ __forceinline__ const double* series_cos<double>() { return d_series_cos64; }
template <> __device__ __forceinline__ const double* series_sin<double>() { return d_series_sin64; }

// Radix-R split of the node index, i = R u + v: sum_i g_i e^{i theta n i} = sum_u U_u W_u with
// W_u = sum_v g_{Ru+v} V_v, V_v = e^{i theta (n v mod m)}, U_u = e^{i theta (R n u mod m)}. The V_v live
// in registers (fully unrolled loops index them statically), g comes from the parameter bank, so each
// inner term is ONE packed FFMA2 (re and im) and the only lane-divergent accesses are the R + 1024/R
// table gathers per coefficient. R = 16 for both precisions (measured on B200: fp32 R = 16 at 62 regs,
// 8 CTAs/SM: 24.7 us vs R = 32 at 96 regs: 28.9 us; fp64 R = 16 at 108 regs: 46.6 us).
// LIME_SERIES_SPLIT (A/B, tools/time_series.py r02): 1 = one coefficient per thread, whole warps per
// grid-stride iteration (fp32 21.5 us, fp64 31.8 us; the previous per-thread loop: 25.5 / 40.0 us);
// 2 / 4 threads per coefficient: 48 / 130 us fp32 -- lanes with different u ranges turn the node
// weights' constant-bank loads lane-divergent, which serialises them.
#ifndef LIME_SERIES_SPLIT
#define LIME_SERIES_SPLIT 1
#endif
constexpr int kSeriesSplit = LIME_SERIES_SPLIT;
// u-loop unroll (r02 A/B, tools/time_series.py): fp32 1 / 4 / 16 / 64: 21.4 / 20.5 / 19.4 / 27.6 us;
// fp64 1 / 4 / 16: 31.7 / 36.0 / 42.1 us (register pressure at 4 CTAs/SM) -> 16 for fp32, 1 for fp64
#ifndef LIME_SERIES_UNROLL_U
#define LIME_SERIES_UNROLL_U 0
#endif
template <typename T>
constexpr int series_unroll_u() { return LIME_SERIES_UNROLL_U > 0 ? LIME_SERIES_UNROLL_U : (sizeof(T) == 4 ? 16 : 1); }
template <typename T, int R, int SPLIT>
__global__ void __launch_bounds__(kSeriesBlock, sizeof(T) == 4 ? 8 : 4) series_kernel(const __grid_constant__ SeriesNodes<T> G,
                                                              int64_t n0, int64_t count, T* __restrict__ out) {
    using T2 = typename Vec2<T>::type;
    constexpr int NU = kSeriesNodes / R;
    // Table entry p sits at p + p/8: the lanes of a warp gather p = (R n u) mod m for consecutive n,
    // i.e. at a stride of 16u (R = 16), which on the plain layout put most of a warp in one or two
    // banks (ncu r02: 1.57M excess wavefronts per gather instruction, 3.27M conflicts per launch);
    // one pad word per 8 entries spreads the strides -- simulated 8.85 -> 2.07 wavefronts per
    // 32-lane gather, measured 0.52M conflicts. (The launch time did not move: the kernel is
    // latency-bound, one wave of 5.3 warps per SMSP at ~48 % issue; a 2/4/8-way split of each
    // coefficient over threads with the u loop unrolled spilled at 64 registers and ran 2-6x slower.)
    __shared__ T sc[kSeriesPadded], ss[kSeriesPadded];
    const T* gc = series_cos<T>();
    const T* gs = series_sin<T>();
    for (int i = threadIdx.x; i < kSeriesM; i += blockDim.x) { sc[series_pos(i)] = gc[i]; ss[series_pos(i)] = gs[i]; }
    __syncthreads();
    const T dx = static_cast<T>(2.0 / kSeriesM);
    // SPLIT > 1: SPLIT consecutive lanes share coefficient k, each summing NU/SPLIT consecutive u
    // blocks; partial sums added by a shuffle butterfly (whole warps iterate together)
    const int h = static_cast<int>(threadIdx.x) % SPLIT;
    constexpr int NUS = NU / SPLIT;
    static_assert(NU % SPLIT == 0 && 32 % SPLIT == 0, "split must divide the u range and the warp");
    for (int64_t base = blockIdx.x * static_cast<int64_t>(blockDim.x); base < count * SPLIT;
         base += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t k = (base + threadIdx.x) / SPLIT;
        const bool valid = k < count;
        const int64_t n = n0 + (valid ? k : count - 1);
        const int step = static_cast<int>(n % kSeriesM);
        T2 V[R];                                      // V_v = e^{i theta (n v mod m)}
        int p = 0;
#pragma unroll
        for (int v = 0; v < R; ++v) {
            V[v].x = sc[series_pos(p)];
            V[v].y = ss[series_pos(p)];
            p += step;
            p -= (p >= kSeriesM) ? kSeriesM : 0;
        }
        const int step_u = p;                         // R n mod m
        int q = static_cast<int>((static_cast<int64_t>(step_u) * (h * NUS)) % kSeriesM);   // R n u mod m
        T a = 0, b = 0;
        // fp64: g_{Ru+v} for the next u is loaded one iteration ahead (the constant-bank loads at a
        // run-time offset otherwise stall the first DFMA of each chain; 46.4 -> 42.0 us). fp32 is
        // faster without it (24.7 vs 27.6 us: 64-register cap), profiles/experiments/jg_series_variants_r01m.jsonl.
        constexpr bool kAhead = sizeof(T) == 8;
        T gn[R];
#pragma unroll
        for (int v = 0; v < R; ++v) gn[v] = kAhead ? G.g[h * NUS * R + v] : T(0);
        constexpr int kUnrollU = series_unroll_u<T>();
#pragma unroll kUnrollU
        for (int u = h * NUS; u < (h + 1) * NUS; ++u) {
            T g[R];
#pragma unroll
            for (int v = 0; v < R; ++v) g[v] = kAhead ? gn[v] : G.g[u * R + v];
            if constexpr (kAhead) {
                const int un = u + 1 < (h + 1) * NUS ? u + 1 : u;
#pragma unroll
                for (int v = 0; v < R; ++v) gn[v] = G.g[un * R + v];
            }
            const T ur = sc[series_pos(q)], ui = ss[series_pos(q)];
            q += step_u;
            q -= (q >= kSeriesM) ? kSeriesM : 0;
            T2 w0, w1;                                // W_u, even and odd v (two dependency chains)
            w0.x = w0.y = w1.x = w1.y = 0;
#pragma unroll
            for (int v = 0; v < R; ++v) {
                if (v & 1) w1 = cfma(g[v], V[v], w1);
                else       w0 = cfma(g[v], V[v], w0);
            }
            const T wr = w0.x + w1.x, wi = w0.y + w1.y;
            a = fma(ur, wr, a);
            a = fma(-ui, wi, a);                      // Re(U W)
            b = fma(ur, wi, b);
            b = fma(ui, wr, b);                       // Im(U W)
        }
#pragma unroll
        for (int o = 1; o < SPLIT; o <<= 1) {
            a += __shfl_xor_sync(0xffffffffu, a, o);
            b += __shfl_xor_sync(0xffffffffu, b, o);
        }
        if (valid && h == 0) {
            if (n == 0) { a = a * static_cast<T>(0.5); b = 0; }   // a_0 = T[f] / 2, b_0 = 0
            out[2 * k + 0] = a * dx;
            out[2 * k + 1] = b * dx;
        }
    }
}

size_t series_workspace_bytes(bool) { return 256; }   // tables are per-device constants now

template <typename T, int R>
static cudaError_t launch_series_t(int64_t n0, int64_t count, T* out, cudaStream_t stream) {
    if (count == 0) return cudaSuccess;
    cudaError_t e = series_tables_ready(stream);
    if (e != cudaSuccess) return e;
    int grid = launch_override().grid_ctas;
    if (grid <= 0)
        grid = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(count * kSeriesSplit, kSeriesBlock), 16LL * device_num_sms()));
    series_kernel<T, R, kSeriesSplit><<<grid, kSeriesBlock, 0, stream>>>(series_nodes<T>(), n0, count, out);
    return cudaGetLastError();
}

cudaError_t launch_series_f32(int64_t n0, int64_t count, float* out, void*, cudaStream_t stream) {
    return launch_series_t<float, 16>(n0, count, out, stream);
}
cudaError_t launch_series_f64(int64_t n0, int64_t count, double* out, void*, cudaStream_t stream) {
    return launch_series_t<double, 16>(n0, count, out, stream);
}

// ------------------------------------------------------------------ JG-Crypt (IDEA)
struct IdeaKeys {
    uint32_t z[52];
};

__device__ __forceinline__ uint32_t idea_mul(uint32_t a, uint32_t b) {
    // a * b mod (2^16 + 1) on 16-bit operands where 0 stands for 2^16. Only the low 16 bits of a
    // are significant (the callers leave sums unmasked), b is a clean sub-key; the result's low 16
    // bits are the product (bit 16 may be set: p mod 65537 = 65536 stands for 0 mod 2^16). For a, b
    // nonzero p mod 65537 is never 0 (65537 is prime) and the constant-divisor remainder is
    // IMAD.HI + SHF + IMAD; p = 0 exactly when a or b is 2^16, where the product is 1 - a - b.
    a &= 0xFFFFu;
    const uint32_t p = a * b;
    return p != 0u ? p % 65537u : 1u - a - b;
}

__device__ __forceinline__ uint2 idea_block(uint2 v, const IdeaKeys& k) {
    // bytes b0..b7 of the block; words are big-endian (R15). Words are kept modulo 2^16 lazily: only
    // their low 16 bits are significant, idea_mul masks its data operand, the output takes low bytes.
    uint32_t x1 = __byte_perm(v.x, 0, 0x4401), x2 = __byte_perm(v.x, 0, 0x4423);
    uint32_t x3 = __byte_perm(v.y, 0, 0x4401), x4 = __byte_perm(v.y, 0, 0x4423);
#pragma unroll
    for (int r = 0; r < 8; ++r) {
        const uint32_t* z = k.z + 6 * r;
        x1 = idea_mul(x1, z[0]);
        x2 = x2 + z[1];
        x3 = x3 + z[2];
        x4 = idea_mul(x4, z[3]);
        const uint32_t t0 = idea_mul(x1 ^ x3, z[4]);
        const uint32_t t1 = idea_mul(t0 + (x2 ^ x4), z[5]);
        const uint32_t t2 = t0 + t1;
        x1 ^= t1;
        x4 ^= t2;
        const uint32_t a = x2 ^ t2;
        x2 = x3 ^ t1;
        x3 = a;
    }
    const uint32_t y1 = idea_mul(x1, k.z[48]);
    const uint32_t y2 = x3 + k.z[49];
    const uint32_t y3 = x2 + k.z[50];
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
