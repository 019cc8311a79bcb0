// parboil.cu -- the paper's other broadcast-operand maps: Parboil-CP
// (Coulombic potential, Table 3) and Parboil-MRI-Q (L353-354), sm_100a.
//
// Both have the N-Body map's shape -- every output element reads the whole broadcast array -- so
// they reuse its B200 design (nbody.cu): the broadcast operand streams through a double-buffered
// shared-memory ring filled by 1-D TMA bulk copies (A4, L234-241) and is read with LDS.128
// broadcasts; each thread keeps U targets in registers as packed pairs (A5, FFMA2/FADD2/FMUL2);
// sources are cut into 256-element chunks (two-level accumulation) and S = splits(n_src) split
// ranges processed by separate CTAs, whose partials the last CTA of a target tile adds in split
// order (A8) -- so results are deterministic and independent of the launch configuration and of
// the target shard.
//
// Element functions (readings DESIGN.md R12, R13):
//   CP     V(p)  += q_j * rsqrt(|p - r_j|^2)                   3 FP32 + 1 MUFU per interaction
//   MRI-Q  t      = kx x + ky y + kz z (turns), f = t - rint(t)
//          (Qr, Qi) += phiMag_k (cos 2 pi f, sin 2 pi f)          ~8 FP32 + 2 MUFU per interaction
// Both are MUFU (XU, 16 lanes/clk/SM) bound.
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace parboil {

constexpr int kChunk = 256;
constexpr int kMaxSplits = 16;
constexpr int kTileJ = 1024;     // sources per smem stage (16 KB)
constexpr int kBlock = 64;       // smallest target-tile block (workspace ticket sizing)
constexpr int kUMin = 2;         // fewest targets per thread of any element type (ticket sizing)

int64_t chunks_per_split(int64_t n_src) {
    const int64_t chunks = ceil_div<int64_t>(n_src, kChunk);
    return chunks == 0 ? 1 : ceil_div<int64_t>(chunks, kMaxSplits);
}
int splits(int64_t n_src) {
    const int64_t chunks = ceil_div<int64_t>(n_src, kChunk);
    if (chunks <= 1) return 1;
    return static_cast<int>(ceil_div<int64_t>(chunks, chunks_per_split(n_src)));
}
static size_t counters_bytes(int64_t targets) {
    return ((ceil_div<int64_t>(targets, kBlock * kUMin) * 4 + 255) / 256) * 256;
}

// ------------------------------------------------------------------ element policies
// CP: targets are lattice points t -> (ix, iy) = (t % nx, t / nx); one fp32 accumulator each.
#ifndef CP_BLOCK
#define CP_BLOCK 128
#endif
#ifndef CP_U
#define CP_U 4
#endif
struct CP {
    using Acc = float;
    static constexpr int kBlock = CP_BLOCK;
    static constexpr int kU = CP_U;  // targets per thread (packed pairs)
    struct Params {
        int32_t nx;
        float z, h;
    };
    struct Tgt {
        float2 x[kU / 2], y2[kU / 2];
    };
    static __device__ __forceinline__ void make_target(const Params& p, const void*, int64_t t, int u, Tgt& tg) {
        const int32_t iy = static_cast<int32_t>(t / p.nx);
        const int32_t ix = static_cast<int32_t>(t - static_cast<int64_t>(iy) * p.nx);
        const float x = static_cast<float>(ix) * p.h;          // fl32(ix h), R12
        const float y = static_cast<float>(iy) * p.h;
        if (u & 1) { tg.x[u >> 1].y = x; tg.y2[u >> 1].y = y; }
        else       { tg.x[u >> 1].x = x; tg.y2[u >> 1].x = y; }
    }
    struct State {
        float2 acc[kU / 2], chunk[kU / 2];
    };
    static __device__ __forceinline__ void zero(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) s.acc[q] = make_float2(0.f, 0.f);
    }
    static __device__ __forceinline__ void chunk_begin(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) s.chunk[q] = make_float2(0.f, 0.f);
    }
    static __device__ __forceinline__ void chunk_end(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) s.acc[q] = add2(s.acc[q], s.chunk[q]);
    }
    static __device__ __forceinline__ void body(const Params& p, const Tgt& tg, float4 a, State& s) {
        const float dz = p.z - a.z;
        const float dz2 = dz * dz;
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) {
            const float2 dx = sub2(tg.x[q], bcast2(a.x));
            const float2 dy = sub2(tg.y2[q], bcast2(a.y));
            const float2 r2 = fma2(dx, dx, fma2(dy, dy, bcast2(dz2)));
            const float2 inv = make_float2(rsqrt_approx(r2.x), rsqrt_approx(r2.y));
            s.chunk[q] = fma2(bcast2(a.w), inv, s.chunk[q]);
        }
    }
    static __device__ __forceinline__ float get(const State& s, int u) {
        return (u & 1) ? s.acc[u >> 1].y : s.acc[u >> 1].x;
    }
};

// MRI-Q: targets are voxels [X][3]; sources are (kx, ky, kz, phiMag) prepared by phimag_kernel.
// MRI-Q tile: 128 threads x 2 targets (one packed pair per thread) -- B200 sweep (tools/tune_parboil.py
// over -DMRIQ_BLOCK / -DMRIQ_U A/B builds, profiles/experiments/tune_parboil_r01.txt): 66.7 us vs 72.7 us
// for 128 x 4; twice the warps of the 4-target tile hide the MUFU.SIN/COS latency better. Results do
// not depend on it (the summation order follows the source chunking only).
#ifndef MRIQ_BLOCK
#define MRIQ_BLOCK 128
#endif
#ifndef MRIQ_U
#define MRIQ_U 2
#endif
struct MRIQ {
    using Acc = float2;
    static constexpr int kBlock = MRIQ_BLOCK;
    static constexpr int kU = MRIQ_U;
    struct Params {
        const float* voxels;
    };
    struct Tgt {
        float2 x[kU / 2], y[kU / 2], z[kU / 2];
    };
    static __device__ __forceinline__ void make_target(const Params& p, const void*, int64_t t, int u, Tgt& tg) {
        const float x = p.voxels[3 * t + 0], y = p.voxels[3 * t + 1], z = p.voxels[3 * t + 2];
        if (u & 1) { tg.x[u >> 1].y = x; tg.y[u >> 1].y = y; tg.z[u >> 1].y = z; }
        else       { tg.x[u >> 1].x = x; tg.y[u >> 1].x = y; tg.z[u >> 1].x = z; }
    }
    struct State {
        float2 qr[kU / 2], qi[kU / 2], cr[kU / 2], ci[kU / 2];
    };
    static __device__ __forceinline__ void zero(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) s.qr[q] = s.qi[q] = make_float2(0.f, 0.f);
    }
    static __device__ __forceinline__ void chunk_begin(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) s.cr[q] = s.ci[q] = make_float2(0.f, 0.f);
    }
    static __device__ __forceinline__ void chunk_end(State& s) {
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) { s.qr[q] = add2(s.qr[q], s.cr[q]); s.qi[q] = add2(s.qi[q], s.ci[q]); }
    }
    static __device__ __forceinline__ void body(const Params&, const Tgt& tg, float4 k, State& s) {
        constexpr float kTwoPi = 6.28318530717958647692f;
#pragma unroll
        for (int q = 0; q < kU / 2; ++q) {
            const float2 t = fma2(bcast2(k.x), tg.x[q], fma2(bcast2(k.y), tg.y[q], mul2(bcast2(k.z), tg.z[q])));
            // f = t - rint(t) in [-1/2, 1/2] turn: (t + 1.5*2^23) - 1.5*2^23 rounds t to an integer
            // for |t| < 2^22 with two FADD2 (no XU instruction).
            const float2 rn = sub2(add2(t, bcast2(12582912.0f)), bcast2(12582912.0f));
            const float2 f = sub2(t, rn);
            const float2 a = mul2(f, bcast2(kTwoPi));
            float2 sn, cs;
            __sincosf(a.x, &sn.x, &cs.x);
            __sincosf(a.y, &sn.y, &cs.y);
            s.cr[q] = fma2(bcast2(k.w), cs, s.cr[q]);
            s.ci[q] = fma2(bcast2(k.w), sn, s.ci[q]);
        }
    }
    static __device__ __forceinline__ float2 get(const State& s, int u) {
        return (u & 1) ? make_float2(s.qr[u >> 1].y, s.qi[u >> 1].y) : make_float2(s.qr[u >> 1].x, s.qi[u >> 1].x);
    }
};

template <class E>
struct Args {
    const float4* src;          // [n_src] broadcast operand
    int64_t n_src;
    int64_t tgt_begin, tgt_count;
    typename E::Params p;
    typename E::Acc* out;       // [tgt_count]
    typename E::Acc* partial;   // [S][tgt_count]
    unsigned* counters;
    int splits;
    int64_t split_len;
};

__device__ __forceinline__ float acc_add(float a, float b) { return a + b; }
__device__ __forceinline__ float2 acc_add(float2 a, float2 b) { return make_float2(a.x + b.x, a.y + b.y); }

template <class E, int BLOCK>
__global__ void __launch_bounds__(BLOCK) bmap_kernel(const __grid_constant__ Args<E> a) {
    __shared__ __align__(128) float4 sbuf[2][kTileJ];
    __shared__ __align__(8) uint64_t full[2];
    __shared__ int s_last;
    using Acc = typename E::Acc;

    const int tile = blockIdx.x;
    const int split = blockIdx.y;
    const int64_t tbase = static_cast<int64_t>(tile) * (BLOCK * E::kU);
    typename E::Tgt tg;
    bool valid[E::kU];
#pragma unroll
    for (int u = 0; u < E::kU; ++u) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(u) * BLOCK;
        valid[u] = t < a.tgt_count;
        E::make_target(a.p, nullptr, a.tgt_begin + (valid[u] ? t : a.tgt_count - 1), u, tg);
    }
    typename E::State st;
    E::zero(st);

    const int64_t j0 = static_cast<int64_t>(split) * a.split_len;
    const int64_t j1 = mn<int64_t>(a.n_src, j0 + a.split_len);
    const int ntiles = static_cast<int>(ceil_div<int64_t>(j1 - j0, kTileJ));
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
        bulk_g2s(sbuf[t & 1], a.src + base, bytes, &full[t & 1]);
    };
    if (threadIdx.x == 0) {
        issue(0);
        if (ntiles > 1) issue(1);
    }
    for (int t = 0; t < ntiles; ++t) {
        mbar_wait(&full[t & 1], (t >> 1) & 1);
        const float4* sb = sbuf[t & 1];
        const int len = static_cast<int>(mn<int64_t>(kTileJ, j1 - (j0 + static_cast<int64_t>(t) * kTileJ)));
        for (int c0 = 0; c0 < len; c0 += kChunk) {
            const int c1 = mn(len, c0 + kChunk);
            E::chunk_begin(st);
            if (c1 - c0 == kChunk) {
#pragma unroll 4
                for (int j = c0; j < c0 + kChunk; ++j) E::body(a.p, tg, sb[j], st);
            } else {
                for (int j = c0; j < c1; ++j) E::body(a.p, tg, sb[j], st);
            }
            E::chunk_end(st);
        }
        __syncthreads();
        if (threadIdx.x == 0 && t + 2 < ntiles) issue(t + 2);
    }

    if (a.splits == 1) {
#pragma unroll
        for (int u = 0; u < E::kU; ++u) {
            const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(u) * BLOCK;
            if (valid[u]) a.out[t] = E::get(st, u);
        }
        return;
    }
#pragma unroll
    for (int u = 0; u < E::kU; ++u) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(u) * BLOCK;
        if (valid[u]) a.partial[static_cast<int64_t>(split) * a.tgt_count + t] = E::get(st, u);
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = (atomicAdd(a.counters + tile, 1u) == static_cast<unsigned>(a.splits - 1));
    __syncthreads();
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int u = 0; u < E::kU; ++u) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(u) * BLOCK;
        if (!valid[u]) continue;
        const volatile Acc* vp = a.partial;
        Acc acc = const_cast<const Acc&>(vp[t]);
        for (int s = 1; s < a.splits; ++s) acc = acc_add(acc, const_cast<const Acc&>(vp[static_cast<int64_t>(s) * a.tgt_count + t]));
        a.out[t] = acc;
        // leave the workspace zero-filled: stale partials could otherwise sit where a later call
        // with other sizes keeps its tickets
        for (int s = 0; s < a.splits; ++s) a.partial[static_cast<int64_t>(s) * a.tgt_count + t] = Acc{};
    }
    if (threadIdx.x == 0) a.counters[tile] = 0u;
}

// MRI-Q preprocessing (Parboil's ComputePhiMag): (kx, ky, kz, phiR, phiI) -> (kx, ky, kz, phiR^2 + phiI^2)
__global__ void __launch_bounds__(256) phimag_kernel(const float* __restrict__ k, int64_t n, float4* __restrict__ out) {
    for (int64_t i = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; i < n;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const float pr = k[5 * i + 3], pi = k[5 * i + 4];
        out[i] = make_float4(k[5 * i + 0], k[5 * i + 1], k[5 * i + 2], fmaf(pr, pr, pi * pi));
    }
}

template <class E>
static cudaError_t launch_bmap(Args<E>& a, void* ws, cudaStream_t stream) {
    a.splits = splits(a.n_src);
    a.split_len = chunks_per_split(a.n_src) * kChunk;
    a.counters = static_cast<unsigned*>(ws);
    a.partial = reinterpret_cast<typename E::Acc*>(static_cast<char*>(ws) + counters_bytes(a.tgt_count));
    // target-tile width: E::kBlock threads x kU targets by default (tools/tune_parboil.py sweep);
    // a block_threads override of 64 / 128 / 256 selects another (results never depend on it)
    int block = launch_override().block_threads;
    if (block != 64 && block != 128 && block != 256) block = E::kBlock;
    const int64_t tiles = ceil_div<int64_t>(a.tgt_count, static_cast<int64_t>(block) * E::kU);
    dim3 grid(static_cast<unsigned>(tiles), static_cast<unsigned>(a.splits));
    if (block == 64) bmap_kernel<E, 64><<<grid, 64, 0, stream>>>(a);
    else if (block == 128) bmap_kernel<E, 128><<<grid, 128, 0, stream>>>(a);
    else bmap_kernel<E, 256><<<grid, 256, 0, stream>>>(a);
    return cudaGetLastError();
}

size_t cp_workspace_bytes(int64_t n_atoms, int64_t points) {
    return counters_bytes(points) + (splits(n_atoms) > 1 ? static_cast<size_t>(splits(n_atoms)) * points * 4 : 0) + 256;
}

// MRI-Q workspace: [counters][split partials][phiMag table]. The counters sit at offset 0 whatever the
// sizes, so a workspace reused with other sizes still has zeroed counters where the next call looks.
static size_t mriq_table_offset(int64_t n_k, int64_t n_x) {
    const size_t b = counters_bytes(n_x) + (splits(n_k) > 1 ? static_cast<size_t>(splits(n_k)) * n_x * 8 : 0);
    return ((b + 255) / 256) * 256;
}
size_t mriq_workspace_bytes(int64_t n_k, int64_t n_x) {
    return mriq_table_offset(n_k, n_x) + static_cast<size_t>(n_k) * 16 + 256;
}

cudaError_t launch_cp(const float4* atoms, int64_t n_atoms, int32_t nx, int64_t p_begin, int64_t p_count, float z,
                      float h, float* out, void* ws, cudaStream_t stream) {
    if (p_count == 0) return cudaSuccess;
    Args<CP> a;
    a.src = atoms;
    a.n_src = n_atoms;
    a.tgt_begin = p_begin;
    a.tgt_count = p_count;
    a.p.nx = nx;
    a.p.z = z;
    a.p.h = h;
    a.out = out;
    return launch_bmap(a, ws, stream);
}

cudaError_t launch_mriq(const float* kspace, int64_t n_k, const float* voxels, int64_t x_begin, int64_t x_count,
                        float* out, void* ws, cudaStream_t stream) {
    if (x_count == 0) return cudaSuccess;
    float4* k4 = reinterpret_cast<float4*>(static_cast<char*>(ws) + mriq_table_offset(n_k, x_count));
    const int g = static_cast<int>(mn<int64_t>(ceil_div<int64_t>(n_k, 256), 4LL * device_num_sms()));
    phimag_kernel<<<mx(g, 1), 256, 0, stream>>>(kspace, n_k, k4);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return e;
    Args<MRIQ> a;
    a.src = k4;
    a.n_src = n_k;
    a.tgt_begin = x_begin;
    a.tgt_count = x_count;
    a.p.voxels = voxels;
    a.out = reinterpret_cast<float2*>(out);
    return launch_bmap(a, ws, stream);
}

}  // namespace parboil
}  // namespace lime
