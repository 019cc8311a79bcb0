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
#include <type_traits>

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
#ifndef LIME_SMALL_UNROLL
#define LIME_SMALL_UNROLL 8            // r01t A/B: 4096-body graph / persistent step 12.10 -> 11.85 us (2 is slower)
#endif
constexpr int kBodyUnroll = LIME_BODY_UNROLL;
constexpr int kSmallUnroll = LIME_SMALL_UNROLL;
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
int64_t chunks_per_split_fixed(int64_t n_src) { return cps_rule(n_src, kChunk, kMaxSplits); }
int splits_fixed(int64_t n_src) { return splits_rule(n_src, kChunk, kMaxSplits); }

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
};

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
        float4 acc = __ldcg(a.partial + t);
        for (int s = 1; s < a.splits; ++s) {
            const float4 p = __ldcg(a.partial + static_cast<int64_t>(s) * a.tgt_count + t);
            acc.x += p.x; acc.y += p.y; acc.z += p.z;
        }
        acc.w = 0.f;
        a.accel[t] = acc;
    }
    if (threadIdx.x == 0) a.counters[tile] = 0u;    // leave the workspace zeroed
}

template <int BLOCK, int R, bool kPacked, int CHUNK, int MINB = 0, bool UNIT = false>
__global__ void __launch_bounds__(BLOCK, MINB) force_kernel(const __grid_constant__ ForceArgs a) {
    __shared__ __align__(128) float4 sbuf[2][kTileJ];
    __shared__ __align__(8) uint64_t full[2];
    __shared__ int s_last;

    const int tile = blockIdx.x;
    const int split = blockIdx.y;
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
// splits live inside one CTA instead of across CTAs. A CTA owns 32 targets; each warp owns TWO
// consecutive splits, one per half-warp, and each lane of a half-warp carries a packed PAIR of the
// CTA's targets (lane q of the half: targets 2q, 2q+1), so every FFMA2/FADD2/FMUL2 does two
// interactions -- this launch is issue-bound, and packing halves the FP32 issue slots per
// interaction. Warp w bulk-copies its two splits' sources (<= 2 x 4 KB, contiguous) into its smem
// slice and runs exactly the arithmetic of the general kernel (chunk partials added into the split
// accumulator in chunk order; each half of a packed op rounds exactly like the scalar op); the
// split partials are then added in split order from shared memory. Same summation order as
// force_kernel, hence bit-identical results, with no global partials and no atomic tickets.
// =====================================================================================
// One split's contribution for the lane's targets: chunk partials added into the split accumulator
// in chunk order -- the arithmetic of force_kernel (shared by force_small_kernel and the persistent
// simulation kernel, so all three agree bit for bit).
template <class IT>
__device__ __forceinline__ void split_sum(IT& it, const float4* sb, int len, int chunk, float eps2) {
    for (int c0 = 0; c0 < len; c0 += chunk) {
        const int c1 = mn(len, c0 + chunk);
        it.chunk_begin();
        if (c1 - c0 == kChunkSmall) {
#pragma unroll kSmallUnroll
            for (int j = c0; j < c0 + kChunkSmall; ++j) it.body(sb[j], eps2);
        } else if (c1 - c0 == kChunk) {
#pragma unroll 4
            for (int j = c0; j < c0 + kChunk; ++j) it.body(sb[j], eps2);
        } else {
            for (int j = c0; j < c1; ++j) it.body(sb[j], eps2);
        }
        it.chunk_end();
    }
}

// Lane -> (split, target pair) map of the small kernels: warp w, half h = lane / 16 works on split
// 2w + h for the CTA's targets 2q and 2q + 1 (q = lane % 16).
struct SmallLane {
    int split, q;
    __device__ __forceinline__ SmallLane() {
        const unsigned lane = lane_id();
        split = 2 * static_cast<int>(threadIdx.x >> 5) + static_cast<int>(lane >> 4);
        q = static_cast<int>(lane & 15u);
    }
};

__global__ void __launch_bounds__(16 * kMaxSplitsSmall) force_small_kernel(const __grid_constant__ ForceArgs a) {
    extern __shared__ __align__(128) uint8_t small_smem[];
    float4* src = reinterpret_cast<float4*>(small_smem);                          // [S][split_len]
    float4* part = reinterpret_cast<float4*>(small_smem + a.splits * a.split_len * 16);   // [S][32]
    __shared__ __align__(8) uint64_t bar[kMaxSplitsSmall / 2];

    pdl_enter();
    const int warp = threadIdx.x >> 5;
    const unsigned lane = lane_id();
    const SmallLane sl;
    const int64_t tg = static_cast<int64_t>(blockIdx.x) * 32;
    Interact<2, true> it;
#pragma unroll
    for (int r = 0; r < 2; ++r) {
        const int64_t t = tg + 2 * sl.q + r;
        it.set(r, __ldg(a.bodies + a.tgt_begin + (t < a.tgt_count ? t : a.tgt_count - 1)));
    }
    it.zero_all();

    // this warp's two splits: one contiguous source range
    const int64_t w0 = static_cast<int64_t>(2 * warp) * a.split_len;
    const int64_t w1 = mn<int64_t>(a.n_src, w0 + 2 * a.split_len);
    if (lane == 0) {
        mbar_init(&bar[warp], 1);
        fence_mbar_init();
        mbar_arrive_expect_tx(&bar[warp], static_cast<uint32_t>(w1 - w0) * 16u);
        bulk_g2s(src + w0, a.bodies + w0, static_cast<uint32_t>(w1 - w0) * 16u, &bar[warp]);
    }
    __syncwarp();
    mbar_wait(&bar[warp], 0);
    const int64_t j0 = static_cast<int64_t>(sl.split) * a.split_len;
    const int len = sl.split < a.splits ? static_cast<int>(mn<int64_t>(a.n_src, j0 + a.split_len) - j0) : 0;
    split_sum(it, src + j0, len, a.chunk, a.eps2);
    if (sl.split < a.splits) {
        part[sl.split * 32 + 2 * sl.q] = it.result(0);
        part[sl.split * 32 + 2 * sl.q + 1] = it.result(1);
    }
    __syncthreads();
    const int64_t t = tg + lane;
    if (warp == 0 && t < a.tgt_count) {
        float4 acc = part[lane];
#pragma unroll 8
        for (int s = 1; s < a.splits; ++s) {       // unrolled: the LDS issue ahead of the in-order FADD chain
            const float4 p = part[s * 32 + lane];
            acc.x += p.x; acc.y += p.y; acc.z += p.z;
        }
        acc.w = 0.f;
        a.accel[t] = acc;
    }
}

static cudaError_t launch_small(const ForceArgs& a, cudaStream_t stream) {
    const size_t smem = static_cast<size_t>(a.splits) * a.split_len * 16 + static_cast<size_t>(a.splits) * 32 * 16;
    cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&force_small_kernel),
                                        static_cast<int>(kSmallMaxSources * 16 + kMaxSplitsSmall * 32 * 16));
    if (e != cudaSuccess) return e;
    const int64_t ctas = ceil_div<int64_t>(a.tgt_count, 32);
    return launch_pdl(&force_small_kernel, dim3(static_cast<unsigned>(ctas)), dim3(32 * ceil_div(a.splits, 2)), smem,
                      stream, a);
}

// =====================================================================================
// Whole simulation in one persistent launch (n <= kSmallMaxSources; the paper's repeated
// task-graph pass, at its own 4096-body size, Table 3). At this size a
// step is a few microseconds of FP32 work, so launch gaps and a separate integrator pass cost as
// much as the forces. One cooperative grid (every CTA resident) runs all `steps`: per step each
// warp stages its source split from the current position buffer (L2, ld.global.cg), each CTA
// computes the forces on its 32-target groups exactly as force_small_kernel does, and warp 0
// applies the integrator (integrate_kernel's arithmetic) and writes the new positions into the
// other buffer; then a grid barrier. Positions ping-pong between `pos` and a workspace copy; a
// velocity is only ever touched by its target's thread. Bit-identical to `steps` x
// (lime_map_nbody + lime_map_nbody_integrate).
// (A CTA-pair variant -- clusters of 2, one packed target pair per lane, split partials combined
// through DSMEM -- was measured slower at 4096: 1024 packed warps leave ~2 per SM sub-partition,
// too few to hide the dependent FFMA2/MUFU chains; see profiles/experiments.)
// =====================================================================================
struct SimArgs {
    float4* pos;        // [n] in/out
    float4* vel;        // [n] in/out
    float4* pos_alt;    // [n] workspace
    unsigned* bar;      // [2] grid barrier arrivals, exits (zero between launches)
    int64_t n;
    int32_t steps;
    int32_t splits;
    int32_t chunk;
    int64_t split_len;
    float eps2, dt;
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

__global__ void __launch_bounds__(16 * kMaxSplitsSmall) simulate_small_kernel(const __grid_constant__ SimArgs a) {
    extern __shared__ __align__(128) uint8_t small_smem[];
    float4* src = reinterpret_cast<float4*>(small_smem);                                   // [S][split_len]
    float4* part = reinterpret_cast<float4*>(small_smem + a.splits * a.split_len * 16);   // [S][32]
    const int warp = threadIdx.x >> 5;                // owns splits 2 warp, 2 warp + 1 (force_small_kernel's map)
    const unsigned lane = lane_id();
    const SmallLane sl;
    const int64_t groups = ceil_div<int64_t>(a.n, 32);
    const int64_t w0 = static_cast<int64_t>(2 * warp) * a.split_len;
    const int wlen = static_cast<int>(mn<int64_t>(a.n, w0 + 2 * a.split_len) - w0);
    const int64_t j0 = static_cast<int64_t>(sl.split) * a.split_len;
    const int len = sl.split < a.splits ? static_cast<int>(mn<int64_t>(a.n, j0 + a.split_len) - j0) : 0;
    unsigned barrier_target = 0;

    for (int32_t k = 0; k < a.steps; ++k) {
        const float4* cur = (k & 1) ? a.pos_alt : a.pos;
        float4* nxt = (k & 1) ? a.pos : a.pos_alt;
        for (int j = static_cast<int>(lane); j < wlen; j += 32) src[w0 + j] = __ldcg(cur + w0 + j);
        __syncwarp();
        for (int64_t g = blockIdx.x; g < groups; g += gridDim.x) {
            const int64_t t = g * 32 + lane;
            const bool valid = t < a.n;
            const float4 p = __ldcg(cur + (valid ? t : a.n - 1));
            Interact<2, true> it;
#pragma unroll
            for (int r = 0; r < 2; ++r) {
                const int64_t tr = g * 32 + 2 * sl.q + r;
                it.set(r, __ldcg(cur + (tr < a.n ? tr : a.n - 1)));
            }
            it.zero_all();
            split_sum(it, src + j0, len, a.chunk, a.eps2);
            if (sl.split < a.splits) {
                part[sl.split * 32 + 2 * sl.q] = it.result(0);
                part[sl.split * 32 + 2 * sl.q + 1] = it.result(1);
            }
            __syncthreads();
            if (warp == 0 && valid) {
                float4 acc = part[lane];
#pragma unroll 8
                for (int s = 1; s < a.splits; ++s) {
                    const float4 q = part[s * 32 + lane];
                    acc.x += q.x; acc.y += q.y; acc.z += q.z;
                }
                float4 v = a.vel[t];
                float4 pn = p;
                v.x = fmaf(acc.x, a.dt, v.x);
                v.y = fmaf(acc.y, a.dt, v.y);
                v.z = fmaf(acc.z, a.dt, v.z);
                pn.x = fmaf(v.x, a.dt, pn.x);
                pn.y = fmaf(v.y, a.dt, pn.y);
                pn.z = fmaf(v.z, a.dt, pn.z);
                a.vel[t] = v;
                __stcg(nxt + t, pn);
            }
            __syncthreads();                       // part[] is reused by the next group
        }
        const bool last = (k + 1 == a.steps);
        if (!last || (a.steps & 1)) {
            barrier_target += gridDim.x;
            grid_barrier(a.bar, barrier_target);
        }
    }
    if ((a.steps & 1) && warp == 0) {              // final positions are in pos_alt: copy own targets back
        for (int64_t g = blockIdx.x; g < groups; g += gridDim.x) {
            const int64_t t = g * 32 + lane;
            if (t < a.n) a.pos[t] = __ldcg(a.pos_alt + t);
        }
    }
    if (threadIdx.x == 0) {                        // the last CTA out leaves the barrier zeroed
        __threadfence();
        if (atomicAdd(a.bar + 1, 1u) == gridDim.x - 1) {
            a.bar[0] = 0u;
            a.bar[1] = 0u;
        }
    }
}

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
    SimArgs a;
    a.pos = pos;
    a.vel = vel;
    a.pos_alt = alt;
    a.bar = reinterpret_cast<unsigned*>(w);
    a.n = n;
    a.steps = steps;
    a.splits = splits(n);
    a.chunk = chunk_len(n);
    a.split_len = chunks_per_split(n) * a.chunk;
    a.eps2 = eps2;
    a.dt = dt;
    const int block = 32 * ceil_div(a.splits, 2);
    const size_t smem = static_cast<size_t>(a.splits) * a.split_len * 16 + static_cast<size_t>(a.splits) * 32 * 16;
    cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&simulate_small_kernel),
                                        static_cast<int>(kSmallMaxSources * 16 + kMaxSplitsSmall * 32 * 16));
    if (e != cudaSuccess) return e;
    const int occ = cached_occupancy(reinterpret_cast<const void*>(&simulate_small_kernel), block, smem);
    if (occ < 1) return cudaErrorInvalidConfiguration;
    const int64_t groups = ceil_div<int64_t>(n, 32);
    int grid = static_cast<int>(mn<int64_t>(groups, static_cast<int64_t>(occ) * device_num_sms()));
    const LaunchOverride& ov = launch_override();
    if (ov.grid_ctas > 0) grid = static_cast<int>(mn<int64_t>(grid, ov.grid_ctas));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(static_cast<unsigned>(grid));
    cfg.blockDim = dim3(static_cast<unsigned>(block));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = stream;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeCooperative;         // all CTAs co-resident (the grid barrier needs it)
    at[0].val.cooperative = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    e = cudaLaunchKernelEx(&cfg, simulate_small_kernel, a);
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
    const int tile = blockIdx.x;
    const int split = blockIdx.y;
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
    dim3 grid(static_cast<unsigned>(tiles), static_cast<unsigned>(a.splits));
    switch (v) {
        case 1: force_ablate_kernel<BLOCK, R, 1><<<grid, BLOCK, 0, stream>>>(a); break;
        case 2: force_ablate_kernel<BLOCK, R, 2><<<grid, BLOCK, 0, stream>>>(a); break;
        case 3: force_ablate_kernel<BLOCK, R, 3><<<grid, BLOCK, 0, stream>>>(a); break;
        case 4: force_ablate_kernel<BLOCK, R, 4><<<grid, BLOCK, 0, stream>>>(a); break;
        case 5: force_ablate_kernel<BLOCK, R, 5><<<grid, BLOCK, 0, stream>>>(a); break;
        case 6: {
            if (a.n_src > kConstBodies) return cudaErrorInvalidValue;
            cudaError_t e = cudaMemcpyToSymbolAsync(c_bodies, a.bodies, static_cast<size_t>(a.n_src) * 16, 0,
                                                    cudaMemcpyDeviceToDevice, stream);
            if (e != cudaSuccess) return e;
            force_ablate_kernel<BLOCK, R, 6><<<grid, BLOCK, 0, stream>>>(a);
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
    dim3 grid(static_cast<unsigned>(tiles), static_cast<unsigned>(a.splits));
    if (a.chunk == kChunk) {
        // mass-uniform splits, then the others (each CTA of either launch leaves unless its split is its kind)
        if (a.uniform != nullptr) force_kernel<BLOCK, R, kPacked, kChunk, MINB, true><<<grid, BLOCK, 0, stream>>>(a);
        force_kernel<BLOCK, R, kPacked, kChunk, MINB><<<grid, BLOCK, 0, stream>>>(a);
    } else {
        force_kernel<BLOCK, R, kPacked, kChunkSmall, MINB><<<grid, BLOCK, 0, stream>>>(a);
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

cudaError_t launch_integrate(float4* pos, float4* vel, const float4* accel, int64_t n, float dt,
                             cudaStream_t stream) {
    if (n == 0) return cudaSuccess;
    int grid = launch_override().grid_ctas;
    if (grid <= 0) grid = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(n, 256), 8LL * device_num_sms()));
    return launch_pdl(&integrate_kernel, dim3(grid), dim3(256), 0, stream, pos, vel, accel, n, dt);
}

}  // namespace nbody
}  // namespace lime
