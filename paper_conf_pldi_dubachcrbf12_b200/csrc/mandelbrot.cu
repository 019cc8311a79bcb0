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

#ifndef LIME_MANDEL_LAZY
#define LIME_MANDEL_LAZY 16       // lazy-test block length (0: test every iteration)
#endif

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

// Lazy escape test (round 2). R7 tests x^2 + y^2 <= 4 before every update; the test costs one
// packed op of the 7 and the count/predicate bookkeeping. Escape is permanent: once |z_j|^2 > 4 with
// |c| <= 1.9, |z_{j+1}| >= |z_j|^2 - |c| - (rounding, < 1e-5) > 2.09, and |z| grows from then on
// (overflow gives inf/NaN, which fails the test too). So for such c the update can run B
// iterations without tests, carrying x^2 and y^2 (6 packed ops per iteration, the same IEEE ops as
// R7), and one test at the block end decides: pass -> all B tests of the block passed (count += B);
// fail -> the pixel escaped inside the block: it stops counting, keeps the block-start state, and
// after the warp's loop replays at most B TESTED iterations from that state to find the exact
// escape iteration. Bit-identical to the tested loop; warps with any |c|^2 > 3.6 (the margin covers
// the fp32 evaluation of |c|^2) take the tested loop.
struct Lazy {
    float2 x, y, xx, yy, cx, cy;
    __device__ __forceinline__ void fast() {         // R7's update, no test; xx, yy = squares of (x, y)
        const float2 z = bcast2(-0.0f), one = bcast2(1.0f), mone = bcast2(-1.0f);
        const float2 xy = fma2(x, y, z);
        x = fma2(fma2(yy, mone, xx), one, cx);
        y = fma2(xy, bcast2(2.0f), cy);
        xx = fma2(x, x, z);
        yy = fma2(y, y, z);
    }
};

// The tested loop from `st` until the warp has no live pixel or max_iter: returns via st.
template <int UNROLL>
__device__ __forceinline__ void tested_loop(State& st, int32_t it, int32_t max_iter) {
    while (it + UNROLL <= max_iter) {
#pragma unroll
        for (int u = 0; u < UNROLL; ++u) st.step();
        it += UNROLL;
        if (!__any_sync(0xffffffffu, st.a0 || st.a1)) return;
    }
    if (__any_sync(0xffffffffu, st.a0 || st.a1)) {
        for (; it < max_iter; ++it) st.step();
    }
}

template <int B>
__device__ __forceinline__ void lazy_loop(State& st, int32_t max_iter) {
    Lazy L;
    L.x = st.x; L.y = st.y; L.cx = st.cx; L.cy = st.cy;
    const float2 z = bcast2(-0.0f), one = bcast2(1.0f);
    L.xx = fma2(L.x, L.x, z);
    L.yy = fma2(L.y, L.y, z);
    float2 xs = L.x, ys = L.y;                        // block-start state of a pixel that escaped
    bool e0 = false, e1 = false;                      // escaped inside a lazy block, count pending
    int32_t it = 0;
    while (it + B <= max_iter) {
        if (st.a0) { xs.x = L.x.x; ys.x = L.y.x; }
        if (st.a1) { xs.y = L.x.y; ys.y = L.y.y; }
#pragma unroll
        for (int u = 0; u < B; ++u) L.fast();
        const float2 s = fma2(L.xx, one, L.yy);       // the test of iteration it + B
        if (st.a0) { if (s.x <= 4.0f) st.n0 += B; else { st.a0 = false; e0 = true; } }
        if (st.a1) { if (s.y <= 4.0f) st.n1 += B; else { st.a1 = false; e1 = true; } }
        it += B;
        if (!__any_sync(0xffffffffu, st.a0 || st.a1)) break;
    }
    // pixels still live at it + B > max_iter: finish with tested iterations from where they are
    if (__any_sync(0xffffffffu, st.a0 || st.a1)) {
        st.x = L.x; st.y = L.y;
        for (; it < max_iter; ++it) st.step();
    }
    // escaped pixels: replay their escape block with tests (<= B iterations, stops at the escape)
    if (__any_sync(0xffffffffu, e0 || e1)) {
        State r = st;
        r.x = xs; r.y = ys;
        r.n0 = 0; r.n1 = 0;
        r.a0 = e0; r.a1 = e1;
#pragma unroll 4
        for (int u = 0; u < B; ++u) r.step();
        if (e0) st.n0 += r.n0;
        if (e1) st.n1 += r.n1;
    }
}

template <int LW, int UNROLL, int LAZY>
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

        bool lazy = false;
        if constexpr (LAZY > 0) {                     // every |c| of the warp <= 1.9 (|c|^2 <= 3.6)
            // (uncontracted scalar ops: the SASS guard admits only R7's exact FFMA forms)
            const float c2x = add_rn(mul_rn(st.cx.x, st.cx.x), mul_rn(st.cy.x, st.cy.x));
            const float c2y = add_rn(mul_rn(st.cx.y, st.cx.y), mul_rn(st.cy.y, st.cy.y));
            lazy = __all_sync(0xffffffffu, c2x <= 3.6f && c2y <= 3.6f);
        }
        if (lazy) lazy_loop<(LAZY > 0 ? LAZY : 1)>(st, a.max_iter);
        else tested_loop<UNROLL>(st, 0, a.max_iter);
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

template <int LW, int UNROLL, int LAZY = 0>
static cudaError_t launch_t(Args& a, cudaStream_t stream) {
    a.tiles_x = ceil_div<int32_t>(a.width, 2 * LW);
    a.ntiles = static_cast<int64_t>(a.tiles_x) * ceil_div<int32_t>(a.row_count, 32 / LW);
    int grid = launch_override().grid_ctas;
    if (grid <= 0) {
        const int per_sm = mx(1, cached_occupancy(reinterpret_cast<const void*>(&mandel_kernel<LW, UNROLL, LAZY>), 256, 0));
        grid = per_sm * device_num_sms();
        const int64_t need = ceil_div<int64_t>(a.ntiles, 8);
        if (need < grid) grid = static_cast<int>(need);
    }
    a.total_warps = static_cast<unsigned>(grid) * 8u;
    mandel_kernel<LW, UNROLL, LAZY><<<grid, 256, 0, stream>>>(a);
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
        case 9: return launch_t<4, 32, 16>(a, stream);
        case 10: return launch_t<4, 32, 32>(a, stream);
        case 11: return launch_t<4, 32, 8>(a, stream);
        case 12: return launch_t<8, 32, 16>(a, stream);     // lazy, 16 x 4 tiles
        case 13: return launch_t<2, 32, 16>(a, stream);     // lazy, 4 x 16 tiles
        case 14: return launch_t<4, 32, 12>(a, stream);
        case 15: return launch_t<4, 32, 24>(a, stream);
        case 16: return launch_t<4, 32, 20>(a, stream);
        default: return launch_t<4, 32, LIME_MANDEL_LAZY>(a, stream);   // 8x8 tiles, vote every 32 (tools/tune_mandel.py)
    }
}

}  // namespace mandel
}  // namespace lime
