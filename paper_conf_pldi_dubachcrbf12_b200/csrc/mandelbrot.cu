// mandelbrot.cu -- bit-exact Mandelbrot escape-count map (sm_100a).
//
// BASELINE.json config 3 (not in the paper; R7). Every multiply/add is one IEEE
// binary32 round-to-nearest operation (no contraction, no subnormal flushing), so the counts
// equal the oracle's exact binary32 emulation bit for bit; tests/test_sass_guards.py checks the
// compiled SASS keeps it that way.
//
// B200 design (DESIGN.md §"Mandelbrot"):
//  * A5/A6c: each lane iterates TWO horizontally adjacent pixels with packed FFMA2
//    (7 packed ops per pixel pair per iteration instead of 16 scalar ones).
//  * Branch-free iteration with sticky "alive" predicates; the warp checks __any_sync once
//    per 32 unrolled iterations, so escaped lanes cost at most 31 extra iterations.
//  * A1: persistent CTAs pull 8x8-pixel warp tiles from a global atomic queue (dynamic
//    load balance: escape times vary by 1000x across the frame); the last warp to finish
//    resets the queue (self-cleaning workspace).
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace mandel {

// A warp tile is (2 * LW) pixels wide and (32 / LW) rows tall (LW lanes per row, 2 pixels per
// lane); the warp votes every UNROLL iterations. Variants are selected by the launch override
// (per_thread = 1..5, see launch()); results never depend on them.

struct Args {
    int32_t width, row_first, row_stride, row_count;
    float x0, y0, dx, dy;
    int32_t max_iter;
    int32_t* counts;
    unsigned* queue;   // [0] next tile, [1] warps finished
    int32_t tiles_x;
    int64_t ntiles;
    unsigned total_warps;
};

// Every binary32 op is written as ONE fused multiply-add whose extra operand makes it exact:
//   a*b = fma(a, b, -0),  a+b = fma(a, 1, b),  a-b = fma(b, -1, a),  (a+a)+c = fma(a, 2, c)
// (the last: a+a = 2a is exact, so R7's two roundings of 2xy + cy collapse into the fma's one;
// 7 packed ops per iteration instead of 8)
// ptxas contracts packed mul.rn/add.rn.f32x2 pairs into FFMA2 even with --fmad=false (observed
// on CUDA 12.9, see tests/test_sass_guards.py), which changes rounding; an FFMA2 cannot be
// contracted further, so this spelling keeps one IEEE rounding per operation of R7.
// n += alive as ONE predicated integer add per pixel: the sticky FSETP.LE.AND's predicate guards
// the add directly (the C++ spellings `n += a`, `if (a) n++` compile to two IADD3 per pixel on
// CUDA 12.9, and this loop is issue-bound: 7 packed FP32 ops = 14 pipe cycles per iteration
// against ~12 issued instructions).
__device__ __forceinline__ void count(int& n, bool alive) {
    asm("{ .reg .pred p; setp.ne.b16 p, %1, 0; @p add.s32 %0, %0, 1; }" : "+r"(n) : "h"(static_cast<short>(alive)));
}

struct State {
    float2 x, y, cx, cy;
    int n0, n1;
    bool a0, a1;
    __device__ __forceinline__ void step() {
        const float2 z = bcast2(-0.0f), one = bcast2(1.0f), mone = bcast2(-1.0f);
        const float2 xx = fma2(x, x, z);
        const float2 yy = fma2(y, y, z);
        const float2 s = fma2(xx, one, yy);          // x^2 + y^2
        a0 = a0 && (s.x <= 4.0f);                    // test before the update (R7); sticky once escaped
        a1 = a1 && (s.y <= 4.0f);
        count(n0, a0);
        count(n1, a1);
        const float2 xy = fma2(x, y, z);
        x = fma2(fma2(yy, mone, xx), one, cx);       // x <- (x^2 - y^2) + cx
        y = fma2(xy, bcast2(2.0f), cy);              // y <- (xy + xy) + cy: xy + xy = 2 xy is exact, so
                                                     // fma(xy, 2, cy) = rn(2 xy + cy) rounds once, as R7
    }
};

template <int LW, int UNROLL>
__global__ void __launch_bounds__(256) mandel_kernel(const __grid_constant__ Args a) {
    constexpr int kTileW = 2 * LW, kTileH = 32 / LW;
    const unsigned lane = lane_id();
    for (;;) {
        int64_t tile = 0;
        if (lane == 0) tile = atomicAdd(a.queue, 1u);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        if (tile >= a.ntiles) break;
        const int32_t tx = static_cast<int32_t>(tile % a.tiles_x);
        const int32_t ty = static_cast<int32_t>(tile / a.tiles_x);
        const int32_t col = tx * kTileW + static_cast<int32_t>(lane % LW) * 2;
        const int32_t k = ty * kTileH + static_cast<int32_t>(lane / LW);
        const bool v0 = (col < a.width) && (k < a.row_count);
        const bool v1 = (col + 1 < a.width) && (k < a.row_count);
        const int32_t py = a.row_first + min(k, a.row_count - 1) * a.row_stride;

        State st;
        st.cx = make_float2(add_rn(a.x0, mul_rn(static_cast<float>(col), a.dx)),
                            add_rn(a.x0, mul_rn(static_cast<float>(col + 1), a.dx)));
        st.cy = bcast2(add_rn(a.y0, mul_rn(static_cast<float>(py), a.dy)));
        st.x = make_float2(0.f, 0.f);
        st.y = make_float2(0.f, 0.f);
        st.n0 = st.n1 = 0;
        st.a0 = st.a1 = true;

        int32_t it = 0;
        while (it + UNROLL <= a.max_iter) {
#pragma unroll
            for (int u = 0; u < UNROLL; ++u) st.step();
            it += UNROLL;
            if (!__any_sync(0xffffffffu, st.a0 || st.a1)) break;
        }
        if (__any_sync(0xffffffffu, st.a0 || st.a1)) {
            for (; it < a.max_iter; ++it) st.step();
        }
        int32_t* row = a.counts + static_cast<int64_t>(k) * a.width;
        if (v0) row[col] = st.n0;
        if (v1) row[col + 1] = st.n1;
    }
    // Self-cleaning queue: the last warp out resets both counters for the next launch.
    if (lane == 0) {
        __threadfence();
        if (atomicAdd(a.queue + 1, 1u) == a.total_warps - 1) {
            a.queue[0] = 0u;
            a.queue[1] = 0u;
        }
    }
}

template <int LW, int UNROLL>
static cudaError_t launch_t(Args& a, cudaStream_t stream) {
    a.tiles_x = ceil_div<int32_t>(a.width, 2 * LW);
    a.ntiles = static_cast<int64_t>(a.tiles_x) * ceil_div<int32_t>(a.row_count, 32 / LW);
    int grid = launch_override().grid_ctas;
    if (grid <= 0) {
        const int per_sm = mx(1, cached_occupancy(reinterpret_cast<const void*>(&mandel_kernel<LW, UNROLL>), 256, 0));
        grid = per_sm * device_num_sms();
        const int64_t need = ceil_div<int64_t>(a.ntiles, 8);
        if (need < grid) grid = static_cast<int>(need);
    }
    a.total_warps = static_cast<unsigned>(grid) * 8u;
    mandel_kernel<LW, UNROLL><<<grid, 256, 0, stream>>>(a);
    return cudaGetLastError();
}

cudaError_t launch(int32_t width, int32_t row_first, int32_t row_stride, int32_t row_count, float x0,
                   float y0, float dx, float dy, int32_t max_iter, int32_t* counts, void* ws,
                   cudaStream_t stream) {
    if (row_count == 0 || width == 0) return cudaSuccess;
    Args a;
    a.width = width;
    a.row_first = row_first;
    a.row_stride = row_stride;
    a.row_count = row_count;
    a.x0 = x0;
    a.y0 = y0;
    a.dx = dx;
    a.dy = dy;
    a.max_iter = max_iter;
    a.counts = counts;
    a.queue = static_cast<unsigned*>(ws);
    // variants (tools/tune_mandel.py): {lanes per row, vote interval}
    const int v = launch_override().per_thread;
    switch (v) {
        case 2: return launch_t<4, 16>(a, stream);
        case 3: return launch_t<4, 8>(a, stream);
        case 4: return launch_t<8, 8>(a, stream);
        case 5: return launch_t<16, 16>(a, stream);
        case 6: return launch_t<8, 32>(a, stream);
        case 7: return launch_t<4, 32>(a, stream);
        case 8: return launch_t<8, 64>(a, stream);
        case 1: return launch_t<8, 16>(a, stream);
        default: return launch_t<4, 32>(a, stream);   // = case 7 (tools/tune_mandel.py: 3.19 vs 3.22 ms for 16x4/16)
    }
}

}  // namespace mandel
}  // namespace lime
