// nbody.cu -- all-pairs N-Body force map and integrator for sm_100a.
//
// The paper's workload (PAPER.md L106-114 task graph; L108-112 float[[][4]] particles;
// L156-158 the map of computeParticleForces over `particles`; L173-174 "n^2 force
// calculation"). Formula: DESIGN.md R1-R3 (Plummer-softened gravity, G = 1, acceleration).
//
// B200 design (DESIGN.md §"N-Body force map"):
//  * A4 (local-memory tiling, L234-241): the broadcast operand (all sources j) is staged
//    into shared memory as 16-KB tiles by 1-D TMA bulk copies (cp.async.bulk + mbarrier
//    complete_tx), double-buffered; every lane reads the same j (LDS.128 broadcast: no bank
//    conflicts by construction, the B200 form of the paper's conflict padding, L241-255).
//  * A5 (private memory, L228-233): R targets per thread live in registers (register
//    blocking), so each staged source feeds R interactions.
//  * A6a: per interaction 12 FP32 lane-ops + 1 MUFU.RSQ; with R even, pairs of targets use
//    packed FADD2/FFMA2/FMUL2 (6 issue slots per interaction); bit-identical to the scalar
//    variant (each half is one IEEE op in the same order).
//  * A1 (L201-208): results are independent of the launch configuration: a target's sum
//    order is fixed by the chunk grid (128 or 256 bodies) and the split count, both functions of n_src.
//  * A8 (split-j): S = splits(n_src) source ranges are processed by separate CTAs; the last
//    CTA of a target tile to finish (atomic ticket) adds the S partials in s order --
//    one launch, deterministic, self-resetting counters.
#include <cstring>
#include <type_traits>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace nbody {

#ifndef LIME_UNIT_UNROLL           // compile-time A/B overrides (tools/ab_nbody_1m.py); defaults are the product
#define LIME_UNIT_UNROLL 8            // r01t A/B: 8 beats 2, 4, 16 (profiles/experiments/nbody_unroll_ab_r01*.jsonl)
#endif
#ifndef LIME_BODY_UNROLL
#define LIME_BODY_UNROLL 4
#endif
constexpr int kUnitUnroll = LIME_UNIT_UNROLL;
// Small-kernel inner loop unroll (sources), per kernel -- r02 A/B (tools/ab_small_nbody.py, 4096
// bodies, graph / persistent us per step): 4: 10.69 / 10.55, 8: 10.53 / 10.39, 16: 10.73 / 10.29,
// 64 (the whole chunk): 10.39 / 10.41 (profiles/experiments/small_nbody_unroll_r02.json)
#ifndef LIME_SMALL_UNROLL
#define LIME_SMALL_UNROLL 64           // force_small_kernel (one-step map / fused step)
#endif
#ifndef LIME_SIM_UNROLL
#define LIME_SIM_UNROLL 16             // simulate_small_kernel
#endif
constexpr int kBodyUnroll = LIME_BODY_UNROLL;
constexpr int kSmallUnroll = LIME_SMALL_UNROLL;
constexpr int kSimUnroll = LIME_SIM_UNROLL;
constexpr int kTileJ = 1024;   // sources per shared-memory stage (16 KB)
static_assert(kTileJ % kChunk == 0 && kTileJ % kChunkSmall == 0, "stage must hold whole chunks");

int chunk_len(int64_t n_src) { return n_src <= kSmallMaxSources ? kChunkSmall : kChunk; }
static int max_splits(int64_t n_src) { return n_src <= kSmallMaxSources ? kMaxSplitsSmall : kMaxSplits; }
static int64_t cps_rule(int64_t n_src, int chunk, int maxs) {
    const int64_t chunks = ceil_div<int64_t>(n_src, chunk);
    return chunks == 0 ? 1 : ceil_div<int64_t>(chunks, maxs);
}
static int splits_rule(int64_t n_src, int chunk, int maxs) {
    const int64_t chunks = ceil_div<int64_t>(n_src, chunk);
    if (chunks <= 1) return 1;
    return static_cast<int>(ceil_div<int64_t>(chunks, cps_rule(n_src, chunk, maxs)));
}
int64_t chunks_per_split(int64_t n_src) { return cps_rule(n_src, chunk_len(n_src), max_splits(n_src)); }
int splits(int64_t n_src) { return splits_rule(n_src, chunk_len(n_src), max_splits(n_src)); }
int64_t chunks_per_split_fixed(int64_t n_src) { return cps_rule(n_src, kChunk, kMaxSplitsF64); }
int splits_fixed(int64_t n_src) { return splits_rule(n_src, kChunk, kMaxSplitsF64); }

// workspace: [counters: one u32 per 128-target tile, padded to 256 B]
//            [chunk flags: one byte per 256-body source chunk when n_src > kSmallMaxSources, padded to 256 B]
//            [partials: S x count float4]
// The counters are zero-invariant (every launch leaves them zero); the flags are rewritten by
// every launch (prepass_kernel) before the force kernel reads them.
static size_t counters_bytes(int64_t tgt_count) {
    return ((ceil_div<int64_t>(tgt_count, 128) * 4 + 255) / 256) * 256;
}
static bool uses_chunk_flags(int64_t n_src) { return n_src > kSmallMaxSources; }
static size_t flags_bytes(int64_t n_src) {
    return uses_chunk_flags(n_src) ? static_cast<size_t>((ceil_div<int64_t>(n_src, kChunk) + 255) / 256) * 256 : 0;
}
size_t workspace_bytes(int64_t n_src, int64_t tgt_count) {
    const int S = splits(n_src);
    if (S == 1) return 256;
    return counters_bytes(tgt_count) + flags_bytes(n_src) + static_cast<size_t>(S) * static_cast<size_t>(tgt_count) * 16;
}

struct ForceArgs {
    const float4* bodies;
    int64_t n_src;
    int64_t tgt_begin;
    int64_t tgt_count;
    float eps2;
    float4* accel;
    float4* partial;      // [S][tgt_count]
    unsigned* counters;   // [tiles]
    const uint8_t* uniform;   // [ceil(n_src / kChunk)] chunk-uniform-mass flags, or null (n_src <= kSmallMaxSources)
    int splits;
    int chunk;            // chunk_len(n_src)
    int64_t split_len;    // chunks_per_split * chunk
    int tree;             // n_src <= kSmallMaxSources: split partials combined by split_tree_sum
    int tile_major;       // grid (splits, tiles): a tile's S split CTAs are scheduled back to back,
                          // so its partials are combined while still in L2 (else grid (tiles, splits))
};

// Split combine of the small problems (n_src <= kSmallMaxSources): a pairwise tree over
// S2 = next_pow2(S) split partials, zero beyond S -- ((P0 + P1) + (P2 + P3)) + ... -- the order in
// which the small kernels' warp-shuffle butterfly adds them (each level adds a block of 2^k aligned
// splits to its neighbour; IEEE addition is commutative, so both partners get the same bits).
__host__ __device__ __forceinline__ int next_pow2(int s) { int p = 1; while (p < s) p <<= 1; return p; }
__device__ __forceinline__ float4 add3(float4 a, float4 b) { return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, 0.f); }
template <class Load>
__device__ __forceinline__ float4 split_tree_sum(int S, Load load) {
    float4 stack[8];
    int top = 0;
    const int S2 = next_pow2(S);
    for (int i = 0; i < S2; ++i) {
        float4 v = i < S ? load(i) : make_float4(0.f, 0.f, 0.f, 0.f);
        for (int m = i; m & 1; m >>= 1) v = add3(stack[--top], v);    // binary-counter merge
        stack[top++] = v;
    }
    return stack[0];
}

#ifndef LIME_TILE_MAJOR
#define LIME_TILE_MAJOR 1
#endif
#ifndef LIME_DISCARD_PARTIALS
#define LIME_DISCARD_PARTIALS 1
#endif
static bool nbody_tile_major() { return LIME_TILE_MAJOR != 0; }

template <int R, bool kPacked>
struct Interact;

// Scalar: one target per register slot.
template <int R>
struct Interact<R, false> {
    float px[R], py[R], pz[R];
    float ax[R], ay[R], az[R];   // split accumulators (sum of chunk partials)
    float cx[R], cy[R], cz[R];   // chunk partials
    __device__ __forceinline__ void zero_all() {
#pragma unroll
        for (int r = 0; r < R; ++r) ax[r] = ay[r] = az[r] = 0.f;
    }
    __device__ __forceinline__ void set(int r, float4 p) { px[r] = p.x; py[r] = p.y; pz[r] = p.z; }
    __device__ __forceinline__ void chunk_begin() {
#pragma unroll
        for (int r = 0; r < R; ++r) cx[r] = cy[r] = cz[r] = 0.f;
    }
    __device__ __forceinline__ void chunk_end() {
#pragma unroll
        for (int r = 0; r < R; ++r) { ax[r] += cx[r]; ay[r] += cy[r]; az[r] += cz[r]; }
    }
    __device__ __forceinline__ void body(const float4 b, const float eps2) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const float dx = b.x - px[r];
            const float dy = b.y - py[r];
            const float dz = b.z - pz[r];
            const float r2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
            const float inv = rsqrt_approx(r2);
            const float inv2 = inv * inv;
            const float s = (b.w * inv) * inv2;           // m_j (r^2 + eps^2)^{-3/2}
            cx[r] = fmaf(s, dx, cx[r]);
            cy[r] = fmaf(s, dy, cy[r]);
            cz[r] = fmaf(s, dz, cz[r]);
        }
    }
    // Chunk-uniform mass (see prepass_kernel): the chunk partial is sum_j d / R^3 and the
    // common mass multiplies it once at chunk end -- 11 FP32 lane-ops per interaction instead of 12.
    __device__ __forceinline__ void body_unit(const float4 b, const float eps2) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const float dx = b.x - px[r];
            const float dy = b.y - py[r];
            const float dz = b.z - pz[r];
            const float r2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
            const float inv = rsqrt_approx(r2);
            const float s = (inv * inv) * inv;            // (r^2 + eps^2)^{-3/2}
            cx[r] = fmaf(s, dx, cx[r]);
            cy[r] = fmaf(s, dy, cy[r]);
            cz[r] = fmaf(s, dz, cz[r]);
        }
    }
    __device__ __forceinline__ void chunk_end_scaled(const float m) {
#pragma unroll
        for (int r = 0; r < R; ++r) { ax[r] = fmaf(m, cx[r], ax[r]); ay[r] = fmaf(m, cy[r], ay[r]); az[r] = fmaf(m, cz[r], az[r]); }
    }
    __device__ __forceinline__ float4 result(int r) const { return make_float4(ax[r], ay[r], az[r], 0.f); }
};

// Packed: targets (2q, 2q+1) share each FFMA2/FADD2/FMUL2; same per-lane op order as scalar.
template <int R>
struct Interact<R, true> {
    static_assert(R % 2 == 0, "packed variant pairs targets");
    static constexpr int Q = R / 2;
    float2 px[Q], py[Q], pz[Q];
    float2 ax[Q], ay[Q], az[Q];
    float2 cx[Q], cy[Q], cz[Q];
    __device__ __forceinline__ void zero_all() {
#pragma unroll
        for (int q = 0; q < Q; ++q) ax[q] = ay[q] = az[q] = make_float2(0.f, 0.f);
    }
    __device__ __forceinline__ void set(int r, float4 p) {
        if (r & 1) { px[r >> 1].y = p.x; py[r >> 1].y = p.y; pz[r >> 1].y = p.z; }
        else       { px[r >> 1].x = p.x; py[r >> 1].x = p.y; pz[r >> 1].x = p.z; }
    }
    __device__ __forceinline__ void chunk_begin() {
#pragma unroll
        for (int q = 0; q < Q; ++q) cx[q] = cy[q] = cz[q] = make_float2(0.f, 0.f);
    }
    __device__ __forceinline__ void chunk_end() {
#pragma unroll
        for (int q = 0; q < Q; ++q) { ax[q] = add2(ax[q], cx[q]); ay[q] = add2(ay[q], cy[q]); az[q] = add2(az[q], cz[q]); }
    }
    // Stage-interleaved across the Q target pairs (each stage is Q independent packed ops), so a
    // warp always has Q-wide ILP between dependent steps; per-lane op order equals the scalar path.
    __device__ __forceinline__ void body(const float4 b, const float eps2) {
        const float2 e2 = bcast2(eps2);
        float2 dx[Q], dy[Q], dz[Q], r2[Q], inv[Q], t[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) dz[q] = sub2(bcast2(b.z), pz[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dz[q], dz[q], e2);
#pragma unroll
        for (int q = 0; q < Q; ++q) dy[q] = sub2(bcast2(b.y), py[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dy[q], dy[q], r2[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) dx[q] = sub2(bcast2(b.x), px[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dx[q], dx[q], r2[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) inv[q] = make_float2(rsqrt_approx(r2[q].x), rsqrt_approx(r2[q].y));
#pragma unroll
        for (int q = 0; q < Q; ++q) t[q] = mul2(bcast2(b.w), inv[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) inv[q] = mul2(inv[q], inv[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) t[q] = mul2(t[q], inv[q]);            // s = (m_j inv) inv^2
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            cx[q] = fma2(t[q], dx[q], cx[q]);
            cy[q] = fma2(t[q], dy[q], cy[q]);
            cz[q] = fma2(t[q], dz[q], cz[q]);
        }
    }
    // Chunk-uniform mass: 11 packed FP32 ops per target pair and source (see the scalar variant).
    __device__ __forceinline__ void body_unit(const float4 b, const float eps2) {
        const float2 e2 = bcast2(eps2);
        float2 dx[Q], dy[Q], dz[Q], r2[Q], inv[Q], t[Q];
#pragma unroll
        for (int q = 0; q < Q; ++q) dz[q] = sub2(bcast2(b.z), pz[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dz[q], dz[q], e2);
#pragma unroll
        for (int q = 0; q < Q; ++q) dy[q] = sub2(bcast2(b.y), py[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dy[q], dy[q], r2[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) dx[q] = sub2(bcast2(b.x), px[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) r2[q] = fma2(dx[q], dx[q], r2[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) inv[q] = make_float2(rsqrt_approx(r2[q].x), rsqrt_approx(r2[q].y));
#pragma unroll
        for (int q = 0; q < Q; ++q) t[q] = mul2(inv[q], inv[q]);
#pragma unroll
        for (int q = 0; q < Q; ++q) t[q] = mul2(t[q], inv[q]);             // s = (inv inv) inv
#pragma unroll
        for (int q = 0; q < Q; ++q) {
            cx[q] = fma2(t[q], dx[q], cx[q]);
            cy[q] = fma2(t[q], dy[q], cy[q]);
            cz[q] = fma2(t[q], dz[q], cz[q]);
        }
    }
    __device__ __forceinline__ void chunk_end_scaled(const float m) {
        const float2 m2 = bcast2(m);
#pragma unroll
        for (int q = 0; q < Q; ++q) { ax[q] = fma2(m2, cx[q], ax[q]); ay[q] = fma2(m2, cy[q], ay[q]); az[q] = fma2(m2, cz[q], az[q]); }
    }
    __device__ __forceinline__ float4 result(int r) const {
        const int q = r >> 1;
        return (r & 1) ? make_float4(ax[q].y, ay[q].y, az[q].y, 0.f) : make_float4(ax[q].x, ay[q].x, az[q].x, 0.f);
    }
};

// Mass-uniform splits (R11): when every source of a split carries the same mass m
// (bitwise-equal floats, e.g. equal-mass particle sets), m factors out of each chunk sum exactly --
// sum_j m d_j / R_j^3 = m * sum_j d_j / R_j^3 -- so the chunk partials are accumulated without the
// per-interaction mass multiply (11 FP32 lane-ops instead of 12) and scaled once at chunk end.
// Applies to n_src > kSmallMaxSources (the FP32-pipe-bound sizes). A prepass writes one flag per
// 256-body chunk; a split is mass-uniform when all its chunks are. The decision depends only on
// the source data and the split grid (a function of n_src), so target shards and launch
// configurations stay bit-identical.
// The same prepass zeroes this call's split tickets, so stale scratch left in a reused workspace by
// a call with other sizes can never reach a ticket (flags == nullptr: tickets only).
__global__ void __launch_bounds__(256) prepass_kernel(const float4* __restrict__ bodies, int64_t n_src,
                                                      uint8_t* __restrict__ flags, unsigned* __restrict__ counters,
                                                      int64_t ncounters) {
    for (int64_t k = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; k < ncounters;
         k += static_cast<int64_t>(gridDim.x) * blockDim.x)
        counters[k] = 0u;
    if (flags == nullptr) return;
    const int64_t nchunks = ceil_div<int64_t>(n_src, kChunk);
    const int64_t warps = static_cast<int64_t>(gridDim.x) * (blockDim.x >> 5);
    for (int64_t c = blockIdx.x * static_cast<int64_t>(blockDim.x >> 5) + (threadIdx.x >> 5); c < nchunks; c += warps) {
        const int64_t c0 = c * kChunk, c1 = mn<int64_t>(n_src, c0 + kChunk);
        const float m0 = __ldg(&bodies[c0].w);
        bool uni = true;
        for (int64_t j = c0 + lane_id(); j < c1; j += 32) uni &= (__ldg(&bodies[j].w) == m0);
        uni = __all_sync(0xffffffffu, uni);
        if (lane_id() == 0) flags[c] = uni ? 1 : 0;
    }
}

// True when every chunk of the split [j0, j1) is mass-uniform AND all chunks share one mass
// (chunk c's first body against the split's first body). Every thread of the CTA must call it.
template <int BLOCK>
__device__ __forceinline__ bool split_mass_uniform(const float4* bodies, const uint8_t* flags, int64_t j0, int64_t j1) {
    const float m0 = __ldg(&bodies[j0].w);
    bool all = true;
    for (int64_t c = j0 / kChunk + threadIdx.x; c < ceil_div<int64_t>(j1, kChunk); c += BLOCK)
        all &= (flags[c] != 0) && (__ldg(&bodies[c * kChunk].w) == m0);
    return __syncthreads_and(all) != 0;
}

// Output (A7: float4 stores) and split combine (A8), shared by every force-kernel variant: with
// S > 1, each CTA writes its split partials, and the last CTA of a target tile (atomic ticket)
// adds the S partials in split order and resets the ticket.
template <int BLOCK, int R, class IT>
__device__ __forceinline__ void finish_targets(const ForceArgs& a, const IT& it, const bool (&valid)[R], int tile,
                                               int split, int64_t tbase, int* s_last) {
    if (a.splits == 1) {
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * BLOCK;
            if (valid[r]) a.accel[t] = it.result(r);
        }
        return;
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * BLOCK;
        if (valid[r]) __stcg(a.partial + static_cast<int64_t>(split) * a.tgt_count + t, it.result(r));
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) {
        const unsigned prev = atomicAdd(a.counters + tile, 1u);
        *s_last = (prev == static_cast<unsigned>(a.splits - 1));
    }
    __syncthreads();
    if (!*s_last) return;
    __threadfence();
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * BLOCK;
        if (!valid[r]) continue;
        float4 acc;
        if (a.tree) {
            acc = split_tree_sum(a.splits, [&](int s) { return __ldcg(a.partial + static_cast<int64_t>(s) * a.tgt_count + t); });
        } else {
            acc = __ldcg(a.partial + t);
            for (int s = 1; s < a.splits; ++s) {
                const float4 p = __ldcg(a.partial + static_cast<int64_t>(s) * a.tgt_count + t);
                acc.x += p.x; acc.y += p.y; acc.z += p.z;
            }
        }
        acc.w = 0.f;
        a.accel[t] = acc;
    }
#if LIME_DISCARD_PARTIALS
    // The partials are dead once combined: drop their L2 lines without write-back (discard.global.L2),
    // so with the tile-major grid they never reach DRAM. Only lines wholly inside this tile's slice
    // of each split row (other tiles' partials may share a boundary line and are still to be read).
    __syncthreads();                               // every thread has read its partials
    {
        const int64_t t0 = tbase, t1 = mn<int64_t>(a.tgt_count, tbase + static_cast<int64_t>(BLOCK) * R);
        for (int sp = 0; sp < a.splits; ++sp) {
            const uintptr_t lo = reinterpret_cast<uintptr_t>(a.partial + static_cast<int64_t>(sp) * a.tgt_count + t0);
            const uintptr_t hi = reinterpret_cast<uintptr_t>(a.partial + static_cast<int64_t>(sp) * a.tgt_count + t1);
            const uintptr_t l0 = (lo + 127) & ~static_cast<uintptr_t>(127);
            for (uintptr_t l = l0 + static_cast<uintptr_t>(threadIdx.x) * 128; l + 128 <= hi; l += static_cast<uintptr_t>(BLOCK) * 128)
                asm volatile("discard.global.L2 [%0], 128;" :: "l"(l) : "memory");
        }
    }
#endif
    if (threadIdx.x == 0) a.counters[tile] = 0u;    // leave the workspace zeroed
}

template <int BLOCK, int R, bool kPacked, int CHUNK, int MINB = 0, bool UNIT = false>
__global__ void __launch_bounds__(BLOCK, MINB) force_kernel(const __grid_constant__ ForceArgs a) {
    __shared__ __align__(128) float4 sbuf[2][kTileJ];
    __shared__ __align__(8) uint64_t full[2];
    __shared__ int s_last;

    const int tile = a.tile_major ? blockIdx.y : blockIdx.x;
    const int split = a.tile_major ? blockIdx.x : blockIdx.y;
    const int64_t tbase = static_cast<int64_t>(tile) * (BLOCK * R);

    // ---- this split's source range [j0, j1)
    const int64_t j0 = static_cast<int64_t>(split) * a.split_len;
    const int64_t j1 = min(a.n_src, j0 + a.split_len);
    const int ntiles = static_cast<int>(ceil_div<int64_t>(j1 - j0, kTileJ));

    // ---- this thread's targets (A3: one 128-bit read-only load each, coalesced)
    Interact<R, kPacked> it;
    bool valid[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * BLOCK;
        valid[r] = t < a.tgt_count;
        const int64_t i = a.tgt_begin + (valid[r] ? t : a.tgt_count - 1);
        it.set(r, __ldg(a.bodies + i));
    }
    it.zero_all();

    // Mass-uniform splits run the UNIT instantiation, the others the per-body-mass one: the two
    // are launched back to back over the same grid and each CTA leaves if its split is not its
    // kind (the split combine below counts S arrivals per tile across both launches).
    if (a.uniform != nullptr) {
        if (split_mass_uniform<BLOCK>(a.bodies, a.uniform, j0, j1) != UNIT) return;
    } else if (UNIT) {
        return;
    }

    if (threadIdx.x == 0) {
        mbar_init(&full[0], 1);
        mbar_init(&full[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    auto issue = [&](int t) {
        const int64_t base = j0 + static_cast<int64_t>(t) * kTileJ;
        const uint32_t bytes = static_cast<uint32_t>(mn<int64_t>(kTileJ, j1 - base)) * 16u;
        mbar_arrive_expect_tx(&full[t & 1], bytes);
        bulk_g2s(sbuf[t & 1], a.bodies + base, bytes, &full[t & 1]);
    };
    if (threadIdx.x == 0) {
        issue(0);
        if (ntiles > 1) issue(1);
    }

    const float eps2 = a.eps2;
    for (int t = 0; t < ntiles; ++t) {
        mbar_wait(&full[t & 1], (t >> 1) & 1);
        const float4* sb = sbuf[t & 1];
        const int len = static_cast<int>(mn<int64_t>(kTileJ, j1 - (j0 + static_cast<int64_t>(t) * kTileJ)));
        for (int c0 = 0; c0 < len; c0 += CHUNK) {
            const int c1 = min(len, c0 + CHUNK);
            it.chunk_begin();
            if constexpr (UNIT) {
                if (c1 - c0 == CHUNK) {
#pragma unroll kUnitUnroll
                    for (int j = c0; j < c0 + CHUNK; ++j) it.body_unit(sb[j], eps2);
                } else {
                    for (int j = c0; j < c1; ++j) it.body_unit(sb[j], eps2);
                }
                it.chunk_end_scaled(sb[c0].w);
            } else {
                if (c1 - c0 == CHUNK) {
#pragma unroll kBodyUnroll
                    for (int j = c0; j < c0 + CHUNK; ++j) it.body(sb[j], eps2);
                } else {
                    for (int j = c0; j < c1; ++j) it.body(sb[j], eps2);
                }
                it.chunk_end();
            }
        }
        __syncthreads();                            // every lane is done reading this stage
        if (threadIdx.x == 0 && t + 2 < ntiles) issue(t + 2);
    }

    finish_targets<BLOCK, R>(a, it, valid, tile, split, tbase, &s_last);
}

// =====================================================================================
// Small problems (n_src <= kSmallMaxSources, e.g. the paper's 4096 bodies, Table 3): the
// whole problem is one wave, so every SM must carry the same work, spread evenly over its four
// SM sub-partitions (SMSPs), and no SM may wait on a serial phase. One CTA per SM.
//  * Work unit = a GROUP of kGroupTargets = 4 consecutive targets (two packed pairs); a group is
//    2 x S2 lanes (S2 = next_pow2(S)), lane (s, p) summing split s (64-body chunks) for the group's
//    targets 2p, 2p + 1 with split_sum (force_kernel's arithmetic, packed FFMA2/FADD2/FMUL2).
//    Groups are dealt to the CTAs in contiguous ranges of floor or ceil(G / grid) groups (at 4096
//    bodies: 6 or 7 groups = 24 or 28 warps on each of the 148 SMs, 6 or 7 per SMSP). The SMSP
//    balance is what the split count is chosen for: tools/nbody_inner_mb.cu measured that an SM
//    runs as long as its busiest SMSP, so 14 warps (4-4-3-3) take as long as 16.
//  * A4: every CTA stages the source array in shared memory with one 1-D bulk copy per split,
//    each with its own mbarrier, so a lane starts as soon as ITS split has landed. Each split's
//    slice is padded by one float4 (split s at float4 offset s (L + 1)): the splits of an LDS.128
//    phase then sit in different bank quads -- the paper's conflict padding (L241-255).
//  * A8: the S2 split partials of a target are added as a pairwise tree (split_tree_sum's order):
//    a warp-shuffle butterfly over the warp's 16 splits, then the (<= 4) warp block sums in shared
//    memory. force_kernel combines small problems in the same order, so force_kernel,
//    force_small_kernel and simulate_small_kernel agree bit for bit.
// =====================================================================================
#ifndef LIME_GROUP_PAIRS
#define LIME_GROUP_PAIRS 2
#endif
constexpr int kGroupPairs = LIME_GROUP_PAIRS;          // packed target pairs per group (1 or 2)
constexpr int kGroupTargets = 2 * kGroupPairs;
constexpr int kWarpSplits = 32 / kGroupPairs;           // splits one warp of a group covers
#ifndef LIME_SMALL_MAXT
#define LIME_SMALL_MAXT 896
#endif
constexpr int kSmallMaxThreads = LIME_SMALL_MAXT;   // block cap (register budget 65536 / cap)
constexpr size_t kOneCtaPerSmSmem = 116 * 1024;   // > 228 KB / 2 per SM (B200)

// Factored chunks at the small sizes (R11): a 64-body chunk whose masses all equal
// one power of two m = 2^e (-40 <= e <= 20) can be summed as sum_j d_j / R_j^3 and scaled by m once
// -- 11 FP32 lane-ops per interaction instead of 12. Scaling by a power of two is exact, so every
// factored product and partial is exactly m times its per-body counterpart and the chunk partial
// has the per-body form's bits (whenever no intermediate is subnormal or infinite: eps^2 >= 1e-20
// bounds R^-3 by 1e30, and coordinates up to ~1e6 keep m R^-3 |d| normal). The decision therefore
// needs no agreement between kernels, and no scan of the masses before the loop (each such scan
// measured 1.2-2 us per launch): a lane predicts "factored" from three masses of its chunk (first,
// middle, last equal and a power of two in range), checks every mass inside the loop (one LOP3
// per source on the integer pipe: the bits of m_j xor m), and in the rare case a mass differs
// recomputes the chunk in the per-body form. Random masses fail the prediction and go straight
// to the per-body loop; equal power-of-two masses (the workloads' 1/n) take the factored one.
__device__ __forceinline__ bool unit_mass(float m) {
    const uint32_t b = __float_as_uint(m);
    return (b & 0x807fffffu) == 0u && (b >> 23) >= 127u - 40u && (b >> 23) <= 127u + 20u;   // +2^e, -40 <= e <= 20
}
#ifndef LIME_SMALL_FACTOR
#define LIME_SMALL_FACTOR 1
#endif

// One split's contribution for the lane's targets: chunk partials added into the split accumulator
// in chunk order -- the arithmetic of force_kernel (per-body form; factored chunks have its bits).
// kKnown (persistent simulation, whose masses never change): bit c of `known` is set once chunk c
// has been verified factored, so later steps skip the prediction and the check. (In the one-step
// kernel a third loop copy costs registers: 14.4 -> 15.5-16.3 us per 4096-body launch.)
template <int U, bool kKnown, class IT>
__device__ __forceinline__ void split_sum(IT& it, const float4* sb, int len, int chunk, float eps2, bool factor,
                                          uint32_t& known) {
    for (int c0 = 0, c = 0; c0 < len; c0 += chunk, ++c) {
        const int c1 = mn(len, c0 + chunk);
        it.chunk_begin();
        const float m = sb[c0].w;
        if (kKnown && ((known >> c) & 1u)) {
#pragma unroll U
            for (int j = c0; j < c0 + kChunkSmall; ++j) it.body_unit(sb[j], eps2);
            it.chunk_end_scaled(m);
            continue;
        }
        if (LIME_SMALL_FACTOR && factor && c1 - c0 == kChunkSmall && unit_mass(m) && sb[c0 + kChunkSmall / 2].w == m &&
            sb[c1 - 1].w == m) {
            const uint32_t mb = __float_as_uint(m);
            uint32_t diff = 0;
#pragma unroll U
            for (int j = c0; j < c0 + kChunkSmall; ++j) {
                const float4 b = sb[j];
                it.body_unit(b, eps2);
                diff |= __float_as_uint(b.w) ^ mb;
            }
            if (diff == 0) {
                it.chunk_end_scaled(m);
                known |= 1u << c;
                continue;
            }
            it.chunk_begin();                          // a mass differs: the per-body form after all
        }
        if (c1 - c0 == kChunkSmall) {
#pragma unroll U
            for (int j = c0; j < c0 + kChunkSmall; ++j) it.body(sb[j], eps2);
        } else {
            for (int j = c0; j < c1; ++j) it.body(sb[j], eps2);
        }
        it.chunk_end();
    }
}

// TMA staging (n_src % 64 == 0 with 64-body splits, e.g. the paper's 4096 bodies): the sources are
// a 2-D tensor of 8-byte elements, one row per split ([S][2L]); one box of kStageRows rows x (2L + 2)
// columns -- the last two columns are out of bounds and zero-filled -- lands in shared memory with
// a row pitch of (L + 1) float4, i.e. directly in the padded layout. One copy (and mbarrier) per
// 16 splits = one warp block, so a warp starts as soon as its quarter of the sources has landed
// (tools/load_mb.cu: 4 x 16-KB copies into all 148 SMs complete in ~1.1k cycles).
constexpr int kStageRows = 16;
constexpr int kMaxStageCopies = kMaxSplitsSmall / kStageRows;
__device__ __forceinline__ void tma_rows(const CUtensorMap* map, void* dst, uint64_t* bar, int row0) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        :: "r"(smem_addr(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(0), "r"(row0), "r"(smem_addr(bar))
        : "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() { asm volatile("fence.proxy.async.global;" ::: "memory"); }
__host__ __device__ __forceinline__ uint32_t stage_copy_bytes(int L) { return static_cast<uint32_t>(kStageRows * (L + 1) * 16); }
// threads c < copies: arm copy c's barrier and issue it
__device__ __forceinline__ void stage_tma(float4* src, const CUtensorMap* map, int S, int L, uint64_t* tbar) {
    const int c = static_cast<int>(threadIdx.x);
    if (c < ceil_div(S, kStageRows)) {
        mbar_arrive_expect_tx(&tbar[c], stage_copy_bytes(L));
        tma_rows(map, src + static_cast<int64_t>(c) * kStageRows * (L + 1), &tbar[c], c * kStageRows);
    }
}
static bool make_rows_map(CUtensorMap* map, const float4* base, int S, int L) {
    auto fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(tensor_map_encoder());
    if (!fn || 2 * L + 2 > 256) return false;
    const cuuint64_t dims[2] = {static_cast<cuuint64_t>(2 * L), static_cast<cuuint64_t>(S)};
    const cuuint64_t strides[1] = {static_cast<cuuint64_t>(16 * L)};
    const cuuint32_t box[2] = {static_cast<cuuint32_t>(2 * L + 2), static_cast<cuuint32_t>(kStageRows)};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, const_cast<float4*>(base), dims, strides, box, estr,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
static bool small_tma_ok(int64_t n_src, int L) { return L == 64 && n_src % L == 0 && tensor_map_encoder() != nullptr; }

struct SmallPlan {
    int S, S2;           // splits(n_src), next_pow2(S)
    int rows;            // staged source rows (splits; whole 16-row TMA boxes when tma)
    int tma;
    int L;               // split length (bodies)
    int chunk;
    int64_t groups;      // ceil(targets / 4)
    int grid;
    int slots;           // groups a CTA works on at once (its range is done in rounds of `slots`)
    int block;           // slots x 2 S2 lanes, rounded up to whole warps
    size_t smem;
};
// CTA c's groups: [c q + min(c, r), + q + (c < r)) with q = groups / grid, r = groups % grid taken
// on the host (a runtime division per thread costs ~20 SASS instructions).
__device__ __forceinline__ int group_begin(int q, int r, int c) { return c * q + mn(c, r); }
__host__ __device__ __forceinline__ int warp_blocks(int S2) { return S2 > kWarpSplits ? S2 / kWarpSplits : 1; }
__host__ __device__ __forceinline__ size_t small_src_bytes(int S, int L) { return static_cast<size_t>(S) * (L + 1) * 16; }

static SmallPlan small_plan(int64_t n_src, int64_t targets, int max_grid) {
    SmallPlan p;
    p.S = splits(n_src);
    p.S2 = next_pow2(p.S);
    p.chunk = chunk_len(n_src);
    p.L = static_cast<int>(chunks_per_split(n_src) * p.chunk);
    p.groups = ceil_div<int64_t>(targets, kGroupTargets);
    p.tma = small_tma_ok(n_src, p.L) ? 1 : 0;
    p.rows = p.tma ? ceil_div(p.S, kStageRows) * kStageRows : p.S;
    p.grid = static_cast<int>(mx<int64_t>(1, mn<int64_t>(p.groups, max_grid)));
    p.slots = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(p.groups, p.grid), kSmallMaxThreads / (kGroupPairs * p.S2)));
    p.block = ceil_div(p.slots * kGroupPairs * p.S2, 32) * 32;
    p.smem = small_src_bytes(p.rows, p.L) + static_cast<size_t>(p.slots) * warp_blocks(p.S2) * kGroupTargets * 16;
    // One CTA per SM: the dealt ranges assume it, but a CTA this small would let the block
    // scheduler place two on one SM. Asking for more than half an SM's shared memory makes a second
    // resident CTA impossible.
    p.smem = mx<size_t>(p.smem, kOneCtaPerSmSmem);
    return p;
}
// Largest smem any small plan needs (the attribute is set once per device for this bound).
static int small_smem_bound() {
    return static_cast<int>(mx<size_t>(kOneCtaPerSmSmem, small_src_bytes(kMaxSplitsSmall, kSmallMaxSources / kMaxSplitsSmall) +
                                                         (kSmallMaxThreads / 32) * kGroupTargets * 16));   // <= one block sum per warp
}

#ifdef LIME_TRACE
__device__ long long g_lime_trace[kNumSMsB200 * 64 * 8];
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ long long gtimer() { long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
#ifdef LIME_TRACE_GLOBAL
#define LIME_CLOCK() gtimer()        // ns, comparable across SMs (tools/trace_barrier.py)
#else
#define LIME_CLOCK() clock64()
#endif
#define LIME_TRACE_AT(k, slot) \
    do { if (threadIdx.x == 0 && (k) < 64) { g_lime_trace[(blockIdx.x * 64 + (k)) * 8 + (slot)] = LIME_CLOCK(); \
         g_lime_trace[(blockIdx.x * 64 + (k)) * 8 + 7] = smid(); } } while (0)
__device__ long long g_lime_wtrace[kNumSMsB200 * 32 * 2];   // step 20: per warp (data ready, lane sum done)
__device__ int g_lime_step;
#define LIME_WTRACE(slot) \
    do { if (g_lime_step == 20 && (threadIdx.x & 31) == 0) g_lime_wtrace[(blockIdx.x * 32 + (threadIdx.x >> 5)) * 2 + (slot)] = clock64(); } while (0)
#else
#define LIME_TRACE_AT(k, slot) do { } while (0)
#define LIME_WTRACE(slot) do { } while (0)
#endif

// Lane -> work map shared by both small kernels.
struct SmallLane {
    int gslot, s, p;   // group slot in this CTA, split, pair within the group
    __device__ __forceinline__ SmallLane(int S2) {              // kGroupPairs * S2: a power of two
        const int lg = __ffs(kGroupPairs * S2) - 1;
        const int idx = static_cast<int>(threadIdx.x) & ((1 << lg) - 1);
        gslot = static_cast<int>(threadIdx.x) >> lg;
        s = idx / kGroupPairs;
        p = idx % kGroupPairs;
    }
};
// The small path's split length L is 64 or 128 (a power of two: at most 2 x 64 chunks of 64 bodies
// over 64 splits), so the padded slot i + i / L is a shift -- a runtime integer division costs ~20
// instructions, and every warp of the 4096-body kernel did ~10 of them before its loop.
static_assert(kSmallMaxSources / kChunkSmall <= 2 * kMaxSplitsSmall, "split length 64 or 128 (a power of two)");
__device__ __forceinline__ int lg2i(int L) { return __ffs(L) - 1; }
__device__ __forceinline__ int split_of(int i, int L) { return i >> lg2i(L); }
__device__ __forceinline__ int padded(int i, int L) { return i + split_of(i, L); }

#ifndef LIME_STAGE_U
#define LIME_STAGE_U 6
#endif
// All threads: bring bodies [0, n) into their padded slots (LDG.128 + STS.128; tools/load_mb.cu:
// 148 CTAs loading the same 64 KB take ~1.3k cycles this way vs 4.6k for 64 one-split bulk copies,
// whose per-copy cost serialises in the TMA unit). kCoherent: the bodies were written in this
// launch by other CTAs (ld.global.cg, L2), else read-only (ld.global.nc).
template <bool kCoherent>
__device__ __forceinline__ void stage_all(float4* src, const float4* bodies, int64_t n, int L) {
    constexpr int U = LIME_STAGE_U;                    // loads in flight per thread: ceil(4096 / 896) = 5 -> one round trip
    for (int base = static_cast<int>(threadIdx.x); base < n; base += U * static_cast<int>(blockDim.x)) {
        float4 v[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int i = base + u * static_cast<int>(blockDim.x);
            if (i < n) v[u] = kCoherent ? __ldcg(bodies + i) : __ldg(bodies + i);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int i = base + u * static_cast<int>(blockDim.x);
            if (i < n) src[padded(i, L)] = v[u];
        }
    }
}

// The lane's split partial for targets tg + 2p, tg + 2p + 1 (clamped to the last valid target),
// then the butterfly over the warp's splits: lanes 2 (16 w) + p of each group's warp w end up with
// the sum of splits 16 w .. 16 w + 15 (or the whole group when S2 <= 16), stored to wpart.
// Every lane of the CTA's used warps calls it (lanes of split s >= S contribute zero).
template <int U, bool kKnown>
__device__ __forceinline__ void small_lane_sum(const float4* src, const SmallLane& sl, bool active, int64_t tgt_first_src,
                                               int64_t tg, int64_t tcount, int L, int S, int S2, int64_t n, int chunk,
                                               float eps2, float4* wpart, uint64_t* tbar, uint32_t parity,
                                               bool factor, uint32_t& known) {
    Interact<2, true> it;
    it.zero_all();
    LIME_WTRACE(0);
    if (active && sl.s < S) {
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            int64_t t = tg + 2 * sl.p + r;
            t = t < tcount ? t : tcount - 1;
            const int i = static_cast<int>(tgt_first_src + t);
            if (tbar) mbar_wait(&tbar[split_of(i, L) / kStageRows], parity);
            it.set(r, src[padded(i, L)]);
        }
        if (tbar) mbar_wait(&tbar[sl.s / kStageRows], parity);
    }
    // The lanes of a warp can leave the waits at different times; without this the warp runs the
    // split loop once per lane subset (ncu r02, per-lane barriers: 1.44x the interactions issued).
    __syncwarp();
    if (active && sl.s < S) {
        const int64_t j0 = static_cast<int64_t>(sl.s) * L;
        split_sum<U, kKnown>(it, src + static_cast<int64_t>(sl.s) * (L + 1), static_cast<int>(mn<int64_t>(n, j0 + L) - j0), chunk,
                  eps2, factor, known);
    }
    float4 a0 = it.result(0), a1 = it.result(1);
    const int seg = S2 < kWarpSplits ? kGroupPairs * S2 : 32;   // lanes of one group within this warp
#pragma unroll
    for (int o = kGroupPairs; o < 32; o <<= 1) {
        if (o < seg) {                                     // warp-uniform
            a0 = add3(a0, make_float4(__shfl_xor_sync(0xffffffffu, a0.x, o), __shfl_xor_sync(0xffffffffu, a0.y, o),
                                      __shfl_xor_sync(0xffffffffu, a0.z, o), 0.f));
            a1 = add3(a1, make_float4(__shfl_xor_sync(0xffffffffu, a1.x, o), __shfl_xor_sync(0xffffffffu, a1.y, o),
                                      __shfl_xor_sync(0xffffffffu, a1.z, o), 0.f));
        }
    }
    LIME_WTRACE(1);
    if (active && sl.s % kWarpSplits == 0) {
        float4* w = wpart + (static_cast<int64_t>(sl.gslot) * warp_blocks(S2) + sl.s / kWarpSplits) * kGroupTargets;
        w[2 * sl.p] = a0;
        w[2 * sl.p + 1] = a1;
    }
}

// Target (round slot ct) of the CTA: its warp block sums added as the top of the tree.
__device__ __forceinline__ float4 small_target_sum(const float4* wpart, int ct, int S2) {
    const int nb = warp_blocks(S2);
    const float4* w = wpart + static_cast<int64_t>(ct / kGroupTargets) * nb * kGroupTargets + ct % kGroupTargets;
    if (nb == 1) return w[0];
    if (nb == 2) return add3(w[0], w[kGroupTargets]);
    return add3(add3(w[0], w[kGroupTargets]), add3(w[2 * kGroupTargets], w[3 * kGroupTargets]));
}

struct SmallArgs {
    const float4* bodies;
    int64_t n_src, tgt_begin, tgt_count;
    float eps2;
    float4* accel;
    int S, S2, L, chunk;
    int64_t groups;
    int gq, gr;          // groups / grid, groups % grid (group_begin)
    int tma;             // sources staged by TMA row boxes (map), else LDG
    int rows;
    // fused step (lime_map_nbody_step): integrate the targets instead of storing accel
    float4* vel;         // [tgt_count] in/out, or null (force map only)
    float4* pos_out;     // [tgt_count]
    float dt;
};

__global__ void __launch_bounds__(kSmallMaxThreads, 1) force_small_kernel(const __grid_constant__ SmallArgs a,
                                                                         const __grid_constant__ CUtensorMap map) {
    extern __shared__ __align__(128) uint8_t small_smem[];
    float4* src = reinterpret_cast<float4*>(small_smem);                                     // [S][L + 1]
    float4* wpart = reinterpret_cast<float4*>(small_smem + small_src_bytes(a.rows, a.L));   // [slots][blocks][4]
    __shared__ __align__(8) uint64_t tbar[kMaxStageCopies];
    pdl_enter();
    const int64_t gb = group_begin(a.gq, a.gr, static_cast<int>(blockIdx.x));
    const int64_t ge = group_begin(a.gq, a.gr, static_cast<int>(blockIdx.x) + 1);
    if (a.tma) {
        if (threadIdx.x < static_cast<unsigned>(kMaxStageCopies)) mbar_init(&tbar[threadIdx.x], 1);
        fence_mbar_init();
        __syncthreads();
        stage_tma(src, &map, a.S, a.L, tbar);
    } else {
        stage_all<false>(src, a.bodies, a.n_src, a.L);
        __syncthreads();
    }
    const SmallLane sl(a.S2);
    const int slots = static_cast<int>(blockDim.x) >> (__ffs(kGroupPairs * a.S2) - 1);   // a power of two
    const int ct = static_cast<int>(threadIdx.x);
    // rounds of `slots` groups (one round by default); every lane calls small_lane_sum (whole warps
    // take part in its butterfly), lanes beyond the round's groups inactive
    uint32_t known = 0;                                // the lane's verified factored chunks (split_sum)
    for (int64_t r0 = gb; r0 < ge; r0 += slots) {
        const int ng = static_cast<int>(mn<int64_t>(slots, ge - r0));
        small_lane_sum<kSmallUnroll, false>(src, sl, sl.gslot < ng, a.tgt_begin, (r0 + sl.gslot) * kGroupTargets, a.tgt_count, a.L, a.S,
                       a.S2, a.n_src, a.chunk, a.eps2, wpart, a.tma ? tbar : nullptr, 0, a.eps2 >= 1e-20f, known);
        __syncthreads();
        const int64_t t = r0 * kGroupTargets + ct;
        if (ct < ng * kGroupTargets && t < a.tgt_count) {
            const float4 acc = small_target_sum(wpart, ct, a.S2);
            if (a.vel == nullptr) {
                a.accel[t] = acc;
            } else {                                   // integrate_kernel's arithmetic on the old position
                const int i = static_cast<int>(a.tgt_begin + t);
                if (a.tma) mbar_wait(&tbar[split_of(i, a.L) / kStageRows], 0);
                float4 p = src[padded(i, a.L)];
                float4 v = a.vel[t];
                v.x = fmaf(acc.x, a.dt, v.x);
                v.y = fmaf(acc.y, a.dt, v.y);
                v.z = fmaf(acc.z, a.dt, v.z);
                p.x = fmaf(v.x, a.dt, p.x);
                p.y = fmaf(v.y, a.dt, p.y);
                p.z = fmaf(v.z, a.dt, p.z);
                a.vel[t] = v;
                a.pos_out[t] = p;
            }
        }
        __syncthreads();                               // wpart[] is reused by the next round
    }
}

static cudaError_t launch_small(const ForceArgs& f, cudaStream_t stream, float4* vel = nullptr, float4* pos_out = nullptr,
                                float dt = 0.f) {
    const SmallPlan p = small_plan(f.n_src, f.tgt_count, device_num_sms());
    cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&force_small_kernel), small_smem_bound());
    if (e != cudaSuccess) return e;
    SmallArgs a;
    a.bodies = f.bodies;
    a.n_src = f.n_src;
    a.tgt_begin = f.tgt_begin;
    a.tgt_count = f.tgt_count;
    a.eps2 = f.eps2;
    a.accel = f.accel;
    a.S = p.S;
    a.S2 = p.S2;
    a.L = p.L;
    a.chunk = p.chunk;
    a.groups = p.groups;
    a.gq = static_cast<int>(p.groups / p.grid);
    a.gr = static_cast<int>(p.groups % p.grid);
    a.tma = p.tma;
    a.rows = p.rows;
    a.vel = vel;
    a.pos_out = pos_out;
    a.dt = dt;
    CUtensorMap map;
    std::memset(&map, 0, sizeof map);
    if (a.tma && !make_rows_map(&map, f.bodies, p.S, p.L)) return cudaErrorInvalidValue;
    return launch_pdl(&force_small_kernel, dim3(static_cast<unsigned>(p.grid)), dim3(static_cast<unsigned>(p.block)),
                      p.smem, stream, a, map);
}

// =====================================================================================
// Whole simulation in one persistent launch (n <= kSmallMaxSources; the paper's repeated
// task-graph pass, at its own 4096-body size, Table 3). At this size a
// step is a few microseconds of FP32 work, so launch gaps and a separate integrator pass cost as
// much as the forces. One cooperative grid (one CTA per SM, every CTA resident) runs all `steps`
// with force_small_kernel's decomposition: per step each CTA bulk-copies the current positions
// into its padded source slots (one mbarrier per split; the copies read what the other CTAs wrote
// in the previous step, ordered by the grid barrier's release/acquire and a proxy fence), computes
// its groups' split partials and their tree sums; one thread per target applies the integrator
// (integrate_kernel's arithmetic) and stores the new position into the other buffer; then a grid
// barrier. Positions ping-pong between `pos` and a workspace copy. Bit-identical to `steps` x
// (lime_map_nbody + lime_map_nbody_integrate).
// =====================================================================================
struct SimArgs {
    float4* pos;        // [n] in/out
    float4* vel;        // [n] in/out
    float4* pos_alt;    // [n] workspace
    unsigned* bar;      // [2] grid barrier arrivals, exits (zero between launches)
    int64_t n;
    int32_t steps;
    int32_t S, S2, L, chunk;
    int64_t groups;
    int gq, gr;          // groups / grid, groups % grid (group_begin)
    float eps2, dt;
    int tma, rows;
};

__device__ __forceinline__ void grid_barrier(unsigned* arrivals, unsigned target) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(arrivals) : "memory");
        unsigned v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(arrivals) : "memory");
        } while (static_cast<int>(v - target) < 0);     // wrap-safe (counters grow by gridDim.x per step)
    }
    __syncthreads();
}


__global__ void __launch_bounds__(kSmallMaxThreads, 1) simulate_small_kernel(const __grid_constant__ SimArgs a,
                                                                            const __grid_constant__ CUtensorMap map_pos,
                                                                            const __grid_constant__ CUtensorMap map_alt) {
    extern __shared__ __align__(128) uint8_t small_smem[];
    float4* src = reinterpret_cast<float4*>(small_smem);                                     // [S][L + 1]
    float4* wpart = reinterpret_cast<float4*>(small_smem + small_src_bytes(a.rows, a.L));   // [slots][blocks][4]
    __shared__ __align__(8) uint64_t tbar[kMaxStageCopies];
    if (a.tma) {
        if (threadIdx.x < static_cast<unsigned>(kMaxStageCopies)) mbar_init(&tbar[threadIdx.x], 1);
        fence_mbar_init();
        __syncthreads();
    }
    const int64_t gb = group_begin(a.gq, a.gr, static_cast<int>(blockIdx.x));
    const int64_t ge = group_begin(a.gq, a.gr, static_cast<int>(blockIdx.x) + 1);
    const SmallLane sl(a.S2);
    const int slots = static_cast<int>(blockDim.x) >> (__ffs(kGroupPairs * a.S2) - 1);   // a power of two
    const int ct = static_cast<int>(threadIdx.x);      // combine thread: one target of the round's groups
    unsigned barrier_target = 0;
    uint32_t known = 0;                                // verified factored chunks: masses never change

    for (int32_t k = 0; k < a.steps; ++k) {
        const float4* cur = (k & 1) ? a.pos_alt : a.pos;
        float4* nxt = (k & 1) ? a.pos : a.pos_alt;
        LIME_TRACE_AT(k, 0);
#ifdef LIME_TRACE
        if (blockIdx.x == 0 && threadIdx.x == 0) g_lime_step = k;
        __syncthreads();
#endif
        LIME_TRACE_AT(k, 5);
        if (a.tma) {
            // the copies read what every CTA wrote in the previous step (generic-proxy stores,
            // ordered before this point by the grid barrier's release/acquire): proxy fence first
            if (threadIdx.x < static_cast<unsigned>(kMaxStageCopies)) fence_proxy_async_global();
            stage_tma(src, (k & 1) ? &map_alt : &map_pos, a.S, a.L, tbar);
        } else {
            stage_all<true>(src, cur, a.n, a.L);   // what every CTA wrote in the previous step (L2)
            __syncthreads();
        }
        LIME_TRACE_AT(k, 6);
        for (int64_t r0 = gb; r0 < ge; r0 += slots) {
            const int ng = static_cast<int>(mn<int64_t>(slots, ge - r0));
            const int64_t t = r0 * kGroupTargets + ct;
            const bool owner = ct < ng * kGroupTargets && t < a.n;
            float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
            if (owner) v = a.vel[t];                   // issued before the force work: latency hidden
            small_lane_sum<kSimUnroll, true>(src, sl, sl.gslot < ng, 0, (r0 + sl.gslot) * kGroupTargets, a.n, a.L, a.S, a.S2, a.n, a.chunk,
                           a.eps2, wpart, a.tma ? tbar : nullptr, static_cast<uint32_t>(k & 1), a.eps2 >= 1e-20f,
                           known);
            LIME_TRACE_AT(k, 4);
            __syncthreads();
            LIME_TRACE_AT(k, 1);
            if (owner) {
                const float4 acc = small_target_sum(wpart, ct, a.S2);
                if (a.tma) mbar_wait(&tbar[split_of(static_cast<int>(t), a.L) / kStageRows], static_cast<uint32_t>(k & 1));
                float4 pn = src[padded(static_cast<int>(t), a.L)];
                v.x = fmaf(acc.x, a.dt, v.x);
                v.y = fmaf(acc.y, a.dt, v.y);
                v.z = fmaf(acc.z, a.dt, v.z);
                pn.x = fmaf(v.x, a.dt, pn.x);
                pn.y = fmaf(v.y, a.dt, pn.y);
                pn.z = fmaf(v.z, a.dt, pn.z);
                a.vel[t] = v;
                __stcg(nxt + t, pn);
            }
            __syncthreads();                           // wpart[] is reused by the next round
        }
        LIME_TRACE_AT(k, 2);
        const bool last = (k + 1 == a.steps);
        if (!last || (a.steps & 1)) {
            barrier_target += gridDim.x;
            grid_barrier(a.bar, barrier_target);
        }
        LIME_TRACE_AT(k, 3);
    }
    if (a.steps & 1) {                                 // the last step wrote pos_alt; every CTA is past its reads
        for (int64_t t = gb * kGroupTargets + ct; t < mn<int64_t>(a.n, ge * kGroupTargets); t += blockDim.x)
            a.pos[t] = __ldcg(a.pos_alt + t);
    }
    if (threadIdx.x == 0) {                        // the last CTA out leaves the barrier zeroed
        __threadfence();
        if (atomicAdd(a.bar + 1, 1u) == gridDim.x - 1) {
            a.bar[0] = 0u;
            a.bar[1] = 0u;
        }
    }
}

#ifdef LIME_TRACE
extern "C" int lime_debug_trace(void* host, size_t bytes) {
    return static_cast<int>(cudaMemcpyFromSymbol(host, g_lime_trace, mn(bytes, sizeof(g_lime_trace))));
}
extern "C" int lime_debug_wtrace(void* host, size_t bytes) {
    return static_cast<int>(cudaMemcpyFromSymbol(host, g_lime_wtrace, mn(bytes, sizeof(g_lime_wtrace))));
}
#endif

// workspace: [grid barrier, 256 B][force workspace (its tickets first)][pos_alt / accel, n x 16 B] --
// every zero-invariant word sits at an offset that does not depend on n, so a workspace reused
// across sizes stays valid.
static size_t simulate_alt_offset(int64_t n) { return 256 + ((workspace_bytes(n, n) + 255) / 256) * 256; }
size_t simulate_workspace_bytes(int64_t n) { return simulate_alt_offset(n) + static_cast<size_t>(n) * 16; }

cudaError_t launch_simulate(float4* pos, float4* vel, int64_t n, int32_t steps, float eps2, float dt, void* ws,
                            cudaStream_t stream) {
    if (n == 0 || steps == 0) return cudaSuccess;
    char* w = static_cast<char*>(ws);
    float4* alt = reinterpret_cast<float4*>(w + simulate_alt_offset(n));   // pos_alt (persistent) / accel (loop)
    void* fws = w + 256;
    if (n > kSmallMaxSources) {                                  // one force + integrate launch per step
        for (int32_t k = 0; k < steps; ++k) {
            cudaError_t e = launch_force(pos, n, 0, n, eps2, alt, fws, stream);
            if (e == cudaSuccess) e = launch_integrate(pos, vel, alt, n, dt, stream);
            if (e != cudaSuccess) return e;
        }
        return cudaSuccess;
    }
    cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&simulate_small_kernel), small_smem_bound());
    if (e != cudaSuccess) return e;
    int max_grid = device_num_sms();
    const LaunchOverride& ov = launch_override();
    if (ov.grid_ctas > 0) max_grid = mn(max_grid, ov.grid_ctas);
    const SmallPlan p = small_plan(n, n, max_grid);
    const int occ = cached_occupancy(reinterpret_cast<const void*>(&simulate_small_kernel), p.block, p.smem);
    if (occ < 1) return cudaErrorInvalidConfiguration;          // one CTA per SM is all the grid needs
    SimArgs a;
    a.pos = pos;
    a.vel = vel;
    a.pos_alt = alt;
    a.bar = reinterpret_cast<unsigned*>(w);
    a.n = n;
    a.steps = steps;
    a.S = p.S;
    a.S2 = p.S2;
    a.L = p.L;
    a.chunk = p.chunk;
    a.groups = p.groups;
    a.gq = static_cast<int>(p.groups / p.grid);
    a.gr = static_cast<int>(p.groups % p.grid);
    a.eps2 = eps2;
    a.dt = dt;
    a.tma = p.tma;
    a.rows = p.rows;
    CUtensorMap map_pos, map_alt;
    std::memset(&map_pos, 0, sizeof map_pos);
    std::memset(&map_alt, 0, sizeof map_alt);
    if (a.tma && (!make_rows_map(&map_pos, pos, p.S, p.L) || !make_rows_map(&map_alt, alt, p.S, p.L)))
        return cudaErrorInvalidValue;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(static_cast<unsigned>(p.grid));
    cfg.blockDim = dim3(static_cast<unsigned>(p.block));
    cfg.dynamicSmemBytes = p.smem;
    cfg.stream = stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;         // all CTAs co-resident (the grid barrier needs it)
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, simulate_small_kernel, a, map_pos, map_alt);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}
// =====================================================================================
// Staging ablation (the paper's Fig. 8: the same kernel with the
// broadcast array mapped to global, local, texture or constant memory, with or without
// vectorisation; L212-216: every optimisation can be switched off for automated exploration).
// Same arithmetic and summation order as force_kernel, so every variant is bit-identical; only
// where the source bodies come from changes:
//   1 global, scalar     4 x ld.global.f32 per body (L1-cached)
//   2 global, vector     ld.global.v4.f32 per body
//   3 read-only, vector  ld.global.nc.v4.f32 (the image/texture path's B200 equivalent)
//   4 local, scalar      threads copy a 1024-body tile into SoA shared arrays; 4 x LDS.32 per body
//   5 local, vector      threads copy the tile with LDG.128/STS.128; LDS.128 per body
//   6 constant, vector   bodies in __constant__ memory (n_src <= 4096 = 64 KB, Table 2's size)
// (variant 0 = force_kernel: 1-D TMA bulk copies into a double-buffered smem ring). Broadcast
// reads make every smem variant bank-conflict free, so the paper's padding variant has no B200
// counterpart here.
// =====================================================================================
constexpr int kConstBodies = 4096;
__constant__ float4 c_bodies[kConstBodies];

template <int BLOCK, int R, int V>
__global__ void __launch_bounds__(BLOCK) force_ablate_kernel(const __grid_constant__ ForceArgs a) {
    constexpr bool kPacked = (R % 2 == 0);
    __shared__ __align__(128) float4 tile4[(V == 5) ? kTileJ : 1];
    __shared__ float tx[(V == 4) ? kTileJ : 1], ty[(V == 4) ? kTileJ : 1], tz[(V == 4) ? kTileJ : 1],
        tm[(V == 4) ? kTileJ : 1];
    __shared__ int s_last;
    const int tile = a.tile_major ? blockIdx.y : blockIdx.x;
    const int split = a.tile_major ? blockIdx.x : blockIdx.y;
    const int64_t tbase = static_cast<int64_t>(tile) * (BLOCK * R);
    Interact<R, kPacked> it;
    bool valid[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * BLOCK;
        valid[r] = t < a.tgt_count;
        it.set(r, __ldg(a.bodies + a.tgt_begin + (valid[r] ? t : a.tgt_count - 1)));
    }
    it.zero_all();
    const int64_t j0 = static_cast<int64_t>(split) * a.split_len;
    const int64_t j1 = mn<int64_t>(a.n_src, j0 + a.split_len);
    const float eps2 = a.eps2;
    // mass-uniform split: decided exactly as force_kernel decides it (same prepass flags)
    const bool unit = a.uniform != nullptr && split_mass_uniform<BLOCK>(a.bodies, a.uniform, j0, j1);
    const float* bf = reinterpret_cast<const float*>(a.bodies);
    for (int64_t tb = j0; tb < j1; tb += kTileJ) {
        const int len = static_cast<int>(mn<int64_t>(kTileJ, j1 - tb));
        if (V == 4 || V == 5) {
            __syncthreads();
            for (int k = threadIdx.x; k < len; k += BLOCK) {
                const float4 b = a.bodies[tb + k];
                if (V == 5) tile4[k] = b;
                else { tx[k] = b.x; ty[k] = b.y; tz[k] = b.z; tm[k] = b.w; }
            }
            __syncthreads();
        }
        auto src = [&](int j) -> float4 {
            const int64_t g = tb + j;
            if constexpr (V == 1) return make_float4(bf[4 * g], bf[4 * g + 1], bf[4 * g + 2], bf[4 * g + 3]);
            else if constexpr (V == 2) {
                float4 v;
                asm volatile("ld.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(a.bodies + g));
                return v;
            } else if constexpr (V == 3) return __ldg(a.bodies + g);
            else if constexpr (V == 4) return make_float4(tx[j], ty[j], tz[j], tm[j]);
            else if constexpr (V == 5) return tile4[j];
            else return c_bodies[g];
        };
        for (int c0 = 0; c0 < len; c0 += a.chunk) {
            const int c1 = mn(len, c0 + a.chunk);
            it.chunk_begin();
            if (unit) {
                if (c1 - c0 == kChunk) {
#pragma unroll 4
                    for (int j = c0; j < c0 + kChunk; ++j) it.body_unit(src(j), eps2);
                } else {
                    for (int j = c0; j < c1; ++j) it.body_unit(src(j), eps2);
                }
                it.chunk_end_scaled(src(c0).w);
                continue;
            }
            if (c1 - c0 == kChunk) {
#pragma unroll 4
                for (int j = c0; j < c0 + kChunk; ++j) it.body(src(j), eps2);
            } else if (c1 - c0 == kChunkSmall) {
#pragma unroll 4
                for (int j = c0; j < c0 + kChunkSmall; ++j) it.body(src(j), eps2);
            } else {
                for (int j = c0; j < c1; ++j) it.body(src(j), eps2);
            }
            it.chunk_end();
        }
    }
    finish_targets<BLOCK, R>(a, it, valid, tile, split, tbase, &s_last);
}

template <int BLOCK, int R>
static cudaError_t launch_ablate(const ForceArgs& a, int v, cudaStream_t stream) {
    const int64_t tiles = ceil_div<int64_t>(a.tgt_count, static_cast<int64_t>(BLOCK) * R);
    ForceArgs b = a;
    b.tile_major = tiles <= 65535 && nbody_tile_major();
    const dim3 grid = b.tile_major ? dim3(static_cast<unsigned>(b.splits), static_cast<unsigned>(tiles))
                                   : dim3(static_cast<unsigned>(tiles), static_cast<unsigned>(b.splits));
    switch (v) {
        case 1: force_ablate_kernel<BLOCK, R, 1><<<grid, BLOCK, 0, stream>>>(b); break;
        case 2: force_ablate_kernel<BLOCK, R, 2><<<grid, BLOCK, 0, stream>>>(b); break;
        case 3: force_ablate_kernel<BLOCK, R, 3><<<grid, BLOCK, 0, stream>>>(b); break;
        case 4: force_ablate_kernel<BLOCK, R, 4><<<grid, BLOCK, 0, stream>>>(b); break;
        case 5: force_ablate_kernel<BLOCK, R, 5><<<grid, BLOCK, 0, stream>>>(b); break;
        case 6: {
            if (a.n_src > kConstBodies) return cudaErrorInvalidValue;
            cudaError_t e = cudaMemcpyToSymbolAsync(c_bodies, a.bodies, static_cast<size_t>(a.n_src) * 16, 0,
                                                    cudaMemcpyDeviceToDevice, stream);
            if (e != cudaSuccess) return e;
            force_ablate_kernel<BLOCK, R, 6><<<grid, BLOCK, 0, stream>>>(b);
            break;
        }
        default: return cudaErrorInvalidValue;
    }
    return cudaGetLastError();
}

// MINB: 512-thread CTAs get __launch_bounds__(512, 1) (up to 128 registers: R = 4 compiles to 112,
// one CTA = 16 warps per SM); the others leave the register choice to ptxas.
template <int BLOCK, int R>
static cudaError_t launch_one(const ForceArgs& a, cudaStream_t stream) {
    constexpr bool kPacked = (R % 2 == 0);
    constexpr int MINB = BLOCK == 512 ? 1 : 0;
    const int64_t tiles = ceil_div<int64_t>(a.tgt_count, static_cast<int64_t>(BLOCK) * R);
    ForceArgs b = a;
    b.tile_major = tiles <= 65535 && nbody_tile_major();
    const dim3 grid = b.tile_major ? dim3(static_cast<unsigned>(b.splits), static_cast<unsigned>(tiles))
                                   : dim3(static_cast<unsigned>(tiles), static_cast<unsigned>(b.splits));
    if (b.chunk == kChunk) {
        // mass-uniform splits, then the others (each CTA of either launch leaves unless its split is its kind)
        if (b.uniform != nullptr) force_kernel<BLOCK, R, kPacked, kChunk, MINB, true><<<grid, BLOCK, 0, stream>>>(b);
        force_kernel<BLOCK, R, kPacked, kChunk, MINB><<<grid, BLOCK, 0, stream>>>(b);
    } else {
        force_kernel<BLOCK, R, kPacked, kChunkSmall, MINB><<<grid, BLOCK, 0, stream>>>(b);
    }
    return cudaGetLastError();
}

cudaError_t launch_force(const float4* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count,
                         float eps2, float4* accel, void* ws, cudaStream_t stream) {
    if (tgt_count == 0) return cudaSuccess;
    ForceArgs a;
    a.bodies = bodies;
    a.n_src = n_src;
    a.tgt_begin = tgt_begin;
    a.tgt_count = tgt_count;
    a.eps2 = eps2;
    a.accel = accel;
    a.splits = splits(n_src);
    a.chunk = chunk_len(n_src);
    a.split_len = chunks_per_split(n_src) * a.chunk;
    a.tree = n_src <= kSmallMaxSources;
    a.tile_major = 0;
    a.counters = static_cast<unsigned*>(ws);
    a.uniform = nullptr;
    a.partial = reinterpret_cast<float4*>(static_cast<char*>(ws) + counters_bytes(tgt_count) + flags_bytes(n_src));

    const LaunchOverride& ov = launch_override();
    // n_src <= kSmallMaxSources: in-CTA splits (same arithmetic and order, see force_small_kernel);
    // a block_threads / per_thread override selects the general kernel (used by the bit-identity test).
    if (nbody_variant() == 0 && n_src <= kSmallMaxSources && ov.block_threads == 0 && ov.per_thread == 0)
        return launch_small(a, stream);
    if (a.splits > 1) {                               // tickets zeroed (+ mass-uniform chunk flags, R11)
        uint8_t* flags = uses_chunk_flags(n_src) ? reinterpret_cast<uint8_t*>(static_cast<char*>(ws) + counters_bytes(tgt_count))
                                                 : nullptr;
        const int64_t ntiles = ceil_div<int64_t>(tgt_count, 128);
        const int64_t work = flags ? ceil_div<int64_t>(ceil_div<int64_t>(n_src, kChunk), 8) : ceil_div<int64_t>(ntiles, 256);
        const int grid = static_cast<int>(mx<int64_t>(1, mn<int64_t>(work, 4LL * device_num_sms())));
        prepass_kernel<<<grid, 256, 0, stream>>>(bodies, n_src, flags, a.counters, ntiles);
        a.uniform = flags;
    }
    if (nbody_variant() != 0) {                       // F1 staging ablation (general mapping only)
        const int v = nbody_variant();
        if (ov.block_threads == 128 && ov.per_thread == 1) return launch_ablate<128, 1>(a, v, stream);
        if (ov.block_threads == 128) return launch_ablate<128, 2>(a, v, stream);
        return launch_ablate<256, 2>(a, v, stream);
    }
    int block = ov.block_threads, R = ov.per_thread;
    if (block == 0 || R == 0) {
        // Automatic (B200 sweeps: tools/tune_nbody.py, tools/nbody_occ.cu; profiles/tune_nbody_r01.jsonl,
        // profiles/experiments/nbody_unit_sweep_r01*.jsonl): 512 threads x 4 targets (two packed pairs,
        // 112 registers, one CTA per SM) is fastest at 2^17..2^20 targets -- 47.6 vs 49.5 ms for
        // 256 x 2 on the config-5 shard -- and is taken when it still fills >= 6 waves; otherwise
        // 256 x 2, then 128-thread tiles so that there are >= 1.5 work items per SM.
        const int64_t want = 3LL * device_num_sms() / 2;
        const int cand[][2] = {{512, 4}, {256, 2}, {128, 2}, {128, 1}};
        const int64_t need[] = {6LL * device_num_sms(), want, want, 0};
        int pick = 3;
        for (int k = 0; k < 4; ++k) {
            const int64_t items = ceil_div<int64_t>(tgt_count, cand[k][0] * cand[k][1]) * a.splits;
            if (items >= need[k]) { pick = k; break; }
        }
        if (block == 0) block = cand[pick][0];
        if (R == 0) R = cand[pick][1];
    }
    if (block == 512) {
        switch (R) {
            case 2: return launch_one<512, 2>(a, stream);
            case 4: return launch_one<512, 4>(a, stream);
        }
    }
    if (block == 256) {
        switch (R) {
            case 1: return launch_one<256, 1>(a, stream);
            case 2: return launch_one<256, 2>(a, stream);
            case 4: return launch_one<256, 4>(a, stream);
            case 8: return launch_one<256, 8>(a, stream);
        }
    } else if (block == 128) {
        switch (R) {
            case 1: return launch_one<128, 1>(a, stream);
            case 2: return launch_one<128, 2>(a, stream);
            case 4: return launch_one<128, 4>(a, stream);
            case 8: return launch_one<128, 8>(a, stream);
        }
    }
    return cudaErrorInvalidConfiguration;
}

// ------------------------------------------------------------------------ integrator (A9)
__global__ void __launch_bounds__(256) integrate_kernel(float4* __restrict__ pos, float4* __restrict__ vel,
                                                        const float4* __restrict__ accel, int64_t n, float dt) {
    pdl_enter();
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const float4 a = ld_stream_f4(accel + i);
        float4 v = vel[i];
        float4 p = pos[i];
        v.x = fmaf(a.x, dt, v.x);
        v.y = fmaf(a.y, dt, v.y);
        v.z = fmaf(a.z, dt, v.z);
        p.x = fmaf(v.x, dt, p.x);
        p.y = fmaf(v.y, dt, p.y);
        p.z = fmaf(v.z, dt, p.z);
        vel[i] = v;
        pos[i] = p;
    }
}

// Fused step tail for n_src > kSmallMaxSources (lime_map_nbody_step): the integrator on targets
// [tgt_begin, tgt_begin + count), reading the old positions from `bodies` and writing pos_out.
__global__ void __launch_bounds__(256) integrate_out_kernel(const float4* __restrict__ bodies, int64_t tgt_begin,
                                                            float4* __restrict__ vel, const float4* __restrict__ accel,
                                                            float4* __restrict__ pos_out, int64_t n, float dt) {
    pdl_enter();
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const float4 a = ld_stream_f4(accel + i);
        float4 v = vel[i];
        float4 p = __ldg(bodies + tgt_begin + i);
        v.x = fmaf(a.x, dt, v.x);
        v.y = fmaf(a.y, dt, v.y);
        v.z = fmaf(a.z, dt, v.z);
        p.x = fmaf(v.x, dt, p.x);
        p.y = fmaf(v.y, dt, p.y);
        p.z = fmaf(v.z, dt, p.z);
        vel[i] = v;
        pos_out[i] = p;
    }
}

// workspace: [force workspace][accel, tgt_count x 16 B] (the accel part only for n_src > 8192)
static size_t step_accel_offset(int64_t n_src, int64_t tgt_count) {
    return ((workspace_bytes(n_src, tgt_count) + 255) / 256) * 256;
}
size_t step_workspace_bytes(int64_t n_src, int64_t tgt_count) {
    return step_accel_offset(n_src, tgt_count) + (n_src > kSmallMaxSources ? static_cast<size_t>(tgt_count) * 16 : 0);
}

cudaError_t launch_step(const float4* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, float eps2,
                        float dt, float4* vel, float4* pos_out, void* ws, cudaStream_t stream) {
    if (tgt_count == 0) return cudaSuccess;
    const LaunchOverride& ov = launch_override();
    if (nbody_variant() == 0 && n_src <= kSmallMaxSources && ov.block_threads == 0 && ov.per_thread == 0) {
        ForceArgs a;                                   // the small-N kernel with the integrator fused in
        a.bodies = bodies;
        a.n_src = n_src;
        a.tgt_begin = tgt_begin;
        a.tgt_count = tgt_count;
        a.eps2 = eps2;
        a.accel = nullptr;
        return launch_small(a, stream, vel, pos_out, dt);
    }
    float4* accel = reinterpret_cast<float4*>(static_cast<char*>(ws) + step_accel_offset(n_src, tgt_count));
    cudaError_t e = launch_force(bodies, n_src, tgt_begin, tgt_count, eps2, accel, ws, stream);
    if (e != cudaSuccess) return e;
    int grid = ov.grid_ctas;
    if (grid <= 0) grid = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(tgt_count, 256), 8LL * device_num_sms()));
    return launch_pdl(&integrate_out_kernel, dim3(grid), dim3(256), 0, stream, bodies, tgt_begin, vel,
                      static_cast<const float4*>(accel), pos_out, tgt_count, dt);
}

cudaError_t launch_integrate(float4* pos, float4* vel, const float4* accel, int64_t n, float dt,
                             cudaStream_t stream) {
    if (n == 0) return cudaSuccess;
    int grid = launch_override().grid_ctas;
    if (grid <= 0) grid = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(n, 256), 8LL * device_num_sms()));
    return launch_pdl(&integrate_kernel, dim3(grid), dim3(256), 0, stream, pos, vel, accel, n, dt);
}

}  // namespace nbody
}  // namespace lime
