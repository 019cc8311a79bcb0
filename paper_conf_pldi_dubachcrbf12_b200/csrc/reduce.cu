// reduce.cu -- reductions `!` (sum/min/max x f32/f64/i32/i64) for sm_100a.
//
// PAPER.md L160-163 (a same-typed binary combinator) and L188-189 ("the compiler may infer a
// parallel reduction"); readings DESIGN.md R9. One launch per reduction (A8):
//   per-thread fold over 128-bit vector loads (grid-stride; scalar head/tail for
//   arbitrary natural alignment) -> warp shuffle -> CTA (smem) -> CTA partial ->
//   the last CTA (atomic ticket) combines the partials in CTA-index order -> out.
// Deterministic for a given launch configuration; the workspace ticket self-resets.
#include <cfloat>
#include <climits>
#include <type_traits>
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace red {

// Accumulator policy per (op, element type).
template <Op OP, typename T> struct Policy;

template <typename T> struct SumF {   // float sums accumulate in fp64 (R9)
    using Acc = double;
    __device__ static Acc id() { return 0.0; }
    __device__ static Acc lift(T v) { return static_cast<double>(v); }
    __device__ static Acc comb(Acc a, Acc b) { return a + b; }
};
template <> struct Policy<kSum, float> : SumF<float> {};
template <> struct Policy<kSum, double> : SumF<double> {};
template <typename T, typename U> struct SumI {  // integer sums wrap in the element width
    using Acc = U;
    __device__ static Acc id() { return 0; }
    __device__ static Acc lift(T v) { return static_cast<U>(v); }
    __device__ static Acc comb(Acc a, Acc b) { return a + b; }
};
template <> struct Policy<kSum, int32_t> : SumI<int32_t, uint32_t> {};
template <> struct Policy<kSum, int64_t> : SumI<int64_t, unsigned long long> {};

// Floating min/max: identity NaN (so the result is NaN only if every element is NaN);
// fminf/fmaxf ignore a NaN operand. Empty input is special-cased to +/-inf on the host side.
template <> struct Policy<kMin, float> {
    using Acc = float;
    __device__ static Acc id() { return __int_as_float(0x7fffffff); }
    __device__ static Acc lift(float v) { return v; }
    __device__ static Acc comb(Acc a, Acc b) { return fminf(a, b); }
};
template <> struct Policy<kMax, float> {
    using Acc = float;
    __device__ static Acc id() { return __int_as_float(0x7fffffff); }
    __device__ static Acc lift(float v) { return v; }
    __device__ static Acc comb(Acc a, Acc b) { return fmaxf(a, b); }
};
template <> struct Policy<kMin, double> {
    using Acc = double;
    __device__ static Acc id() { return __longlong_as_double(0x7fffffffffffffffLL); }
    __device__ static Acc lift(double v) { return v; }
    __device__ static Acc comb(Acc a, Acc b) { return fmin(a, b); }
};
template <> struct Policy<kMax, double> {
    using Acc = double;
    __device__ static Acc id() { return __longlong_as_double(0x7fffffffffffffffLL); }
    __device__ static Acc lift(double v) { return v; }
    __device__ static Acc comb(Acc a, Acc b) { return fmax(a, b); }
};
template <typename T, T ID, bool MIN> struct MinMaxI {
    using Acc = T;
    __device__ static Acc id() { return ID; }
    __device__ static Acc lift(T v) { return v; }
    __device__ static Acc comb(Acc a, Acc b) { return MIN ? (b < a ? b : a) : (b > a ? b : a); }
};
template <> struct Policy<kMin, int32_t> : MinMaxI<int32_t, INT_MAX, true> {};
template <> struct Policy<kMax, int32_t> : MinMaxI<int32_t, INT_MIN, false> {};
template <> struct Policy<kMin, int64_t> : MinMaxI<int64_t, LLONG_MAX, true> {};
template <> struct Policy<kMax, int64_t> : MinMaxI<int64_t, LLONG_MIN, false> {};

// L2 (coherent) load of a CTA partial written by another CTA
template <typename A>
__device__ __forceinline__ A ldcg_acc(const A* p) {
    if constexpr (sizeof(A) == 8) {
        const unsigned long long v = __ldcg(reinterpret_cast<const unsigned long long*>(p));
        return *reinterpret_cast<const A*>(&v);
    } else {
        const unsigned v = __ldcg(reinterpret_cast<const unsigned*>(p));
        return *reinterpret_cast<const A*>(&v);
    }
}

template <typename P, typename A>
__device__ __forceinline__ A warp_reduce(A v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = P::comb(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

template <Op OP, typename T>
__global__ void __launch_bounds__(256) reduce_kernel(const T* __restrict__ x, int64_t n, T* out,
                                                     unsigned* ticket, void* partial_raw) {
    using P = Policy<OP, T>;
    using A = typename P::Acc;
    constexpr int V = 16 / sizeof(T);   // elements per 128-bit load
    A* partial = static_cast<A*>(partial_raw);
    pdl_enter();
    __shared__ A s_warp[8];
    __shared__ int s_last;

    A acc = P::id();
    // scalar head up to 16-byte alignment, vector body, scalar tail
    const uintptr_t addr = reinterpret_cast<uintptr_t>(x);
    int64_t head = static_cast<int64_t>(((16 - (addr & 15)) & 15) / sizeof(T));
    if (head > n) head = n;
    const int64_t nv = (n - head) / V;
    const int64_t tail0 = head + nv * V;
    const int64_t gtid = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x;
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    if (gtid < head) acc = P::comb(acc, P::lift(x[gtid]));
    const uint4* xv = reinterpret_cast<const uint4*>(x + head);
    auto fold = [&](const uint4& raw) {
        const T* e = reinterpret_cast<const T*>(&raw);
#pragma unroll
        for (int k = 0; k < V; ++k) acc = P::comb(acc, P::lift(e[k]));
    };
    auto ldv = [&](int64_t i) {
        uint4 raw;
        asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(raw.x), "=r"(raw.y), "=r"(raw.z), "=r"(raw.w) : "l"(xv + i));
        return raw;
    };
    int64_t i = gtid;
    for (; i + 3 * stride < nv; i += 4 * stride) {   // 4 independent 128-bit loads in flight
        const uint4 r0 = ldv(i), r1 = ldv(i + stride), r2 = ldv(i + 2 * stride), r3 = ldv(i + 3 * stride);
        if constexpr (OP == kSum && std::is_same<T, float>::value) {
            // fp32 sums: add the 16 loaded elements in fp32 and widen once -- F2F.F64.F32 runs at
            // ~8 lanes/clk/SM (profiles/microbench), so one conversion per element would cap the
            // kernel below HBM speed.
            const float4 a = reinterpret_cast<const float4&>(r0), b = reinterpret_cast<const float4&>(r1);
            const float4 c = reinterpret_cast<const float4&>(r2), d = reinterpret_cast<const float4&>(r3);
            const float s16 = (((a.x + a.y) + (a.z + a.w)) + ((b.x + b.y) + (b.z + b.w))) +
                              (((c.x + c.y) + (c.z + c.w)) + ((d.x + d.y) + (d.z + d.w)));
            acc = P::comb(acc, P::lift(s16));
        } else {
            fold(r0); fold(r1); fold(r2); fold(r3);
        }
    }
    for (; i < nv; i += stride) fold(ldv(i));
    if (gtid < n - tail0) acc = P::comb(acc, P::lift(x[tail0 + gtid]));

    acc = warp_reduce<P>(acc);
    const int warp = threadIdx.x >> 5;
    if (lane_id() == 0) s_warp[warp] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        A b = s_warp[0];
        for (int w = 1; w < (blockDim.x >> 5); ++w) b = P::comb(b, s_warp[w]);
        partial[blockIdx.x] = b;
        __threadfence();
        s_last = (atomicAdd(ticket, 1u) == gridDim.x - 1);
    }
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    if (warp == 0) {
        // fixed order (deterministic for a given grid): lane l folds partials l, l+32, ... in index
        // order, then the fixed xor-shuffle tree combines the 32 lane values
        A b = P::id();
#pragma unroll 8
        for (unsigned k = lane_id(); k < gridDim.x; k += 32) b = P::comb(b, ldcg_acc(partial + k));   // loads issue ahead
        b = warp_reduce<P>(b);
        if (lane_id() == 0) {
            if constexpr (OP != kSum && std::is_floating_point<T>::value) {
                if (n == 0) b = (OP == kMin) ? static_cast<A>(INFINITY) : static_cast<A>(-INFINITY);  // R9
            }
            *out = static_cast<T>(b);
            *ticket = 0u;
        }
    }
}

template <Op OP, typename T>
static cudaError_t launch_t(const void* x, int64_t n, void* out, void* ws, cudaStream_t stream) {
    const LaunchOverride& ov = launch_override();
    int block = 256;
    int grid = ov.grid_ctas;
    if (grid <= 0) {
        constexpr int V = 16 / sizeof(T);
        const int64_t need = ceil_div<int64_t>(ceil_div<int64_t>(n, V), 256);
        grid = static_cast<int>(mn<int64_t>(mx<int64_t>(need, 1), 4LL * device_num_sms()));
    }
    if (grid > kMaxCtas) grid = kMaxCtas;
    unsigned* ticket = static_cast<unsigned*>(ws);
    void* partial = static_cast<char*>(ws) + 256;
    return launch_pdl(&reduce_kernel<OP, T>, dim3(grid), dim3(block), 0, stream, static_cast<const T*>(x), n,
                      static_cast<T*>(out), ticket, partial);
}

cudaError_t launch(Op op, Dt dt, const void* x, int64_t n, void* out, void* ws, cudaStream_t stream) {
#define LIME_RED_CASE(O, D, T) if (op == O && dt == D) return launch_t<O, T>(x, n, out, ws, stream);
    LIME_RED_CASE(kSum, kF32, float) LIME_RED_CASE(kSum, kF64, double)
    LIME_RED_CASE(kSum, kI32, int32_t) LIME_RED_CASE(kSum, kI64, int64_t)
    LIME_RED_CASE(kMin, kF32, float) LIME_RED_CASE(kMin, kF64, double)
    LIME_RED_CASE(kMin, kI32, int32_t) LIME_RED_CASE(kMin, kI64, int64_t)
    LIME_RED_CASE(kMax, kF32, float) LIME_RED_CASE(kMax, kF64, double)
    LIME_RED_CASE(kMax, kI32, int32_t) LIME_RED_CASE(kMax, kI64, int64_t)
#undef LIME_RED_CASE
    return cudaErrorInvalidValue;
}

}  // namespace red
}  // namespace lime
