// nbody64.cu -- double-precision N-Body force map (Table 3
// "N-Body ... Float / Double", L319-323 single- and double-precision variants, L372-373 "double
// precision ... approximately 2-3x slower than single-precision" on the GTX 580).
//
// Same map, same readings (R1-R3), same summation structure as nbody.cu's fp32 kernel (S split
// partials added in split order by the last CTA of a target tile), on fp64 bodies. On B200 the
// FP64 pipe is a separate ~64 lanes/clk/SM unit (profiles/microbench: 58.9 DFMA lanes/clk/SM);
// per interaction: 3 DADD + 3 DFMA (r^2) + one MUFU.RSQ64H (~2^-20) refined to full precision by
// the 2nd-order correction (1+e)^(-3/2) ~ 1 - 3/2 e + 15/8 e^2, e = r^2 y0^2 - 1 (|e| ~ 2^-19,
// residual ~ e^3 < 2^-55), 3 DMUL + 3 DFMA (accumulate) -- 16 FP64 ops: FP64-pipe bound.
#include "common.cuh"
#include "kernels.h"

namespace lime {
namespace nbody64 {

constexpr int kTileJ = 512;     // bodies per smem stage (16 KB)
constexpr int kBlock = 128;
constexpr int kR = 2;           // targets per thread

struct Args {
    const double4* bodies;
    int64_t n_src, tgt_begin, tgt_count;
    double eps2;
    double4* accel;
    double4* partial;
    unsigned* counters;
    int splits;
    int64_t split_len;
};

static size_t counters_bytes(int64_t tgt_count) {
    return ((ceil_div<int64_t>(tgt_count, kBlock * kR) * 4 + 255) / 256) * 256;
}
size_t workspace_bytes(int64_t n_src, int64_t tgt_count) {
    const int S = nbody::splits_fixed(n_src);
    return counters_bytes(tgt_count) + (S > 1 ? static_cast<size_t>(S) * tgt_count * 32 : 0) + 256;
}

__device__ __forceinline__ double rsqrt_approx_f64(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    return y;
}

__device__ __forceinline__ double4 ld_body(const double4* p) {
    const double2* q = reinterpret_cast<const double2*>(p);
    const double2 a = __ldg(q), b = __ldg(q + 1);
    return make_double4(a.x, a.y, b.x, b.y);
}

__global__ void __launch_bounds__(kBlock) force64_kernel(const __grid_constant__ Args a) {
    __shared__ __align__(128) double4 sbuf[2][kTileJ];
    __shared__ __align__(8) uint64_t full[2];
    __shared__ int s_last;
    const int tile = blockIdx.x, split = blockIdx.y;
    const int64_t tbase = static_cast<int64_t>(tile) * (kBlock * kR);
    double px[kR], py[kR], pz[kR], ax[kR], ay[kR], az[kR];
    bool valid[kR];
#pragma unroll
    for (int r = 0; r < kR; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * kBlock;
        valid[r] = t < a.tgt_count;
        const double4 p = ld_body(a.bodies + a.tgt_begin + (valid[r] ? t : a.tgt_count - 1));
        px[r] = p.x; py[r] = p.y; pz[r] = p.z;
        ax[r] = ay[r] = az[r] = 0.0;
    }
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
        const uint32_t bytes = static_cast<uint32_t>(mn<int64_t>(kTileJ, j1 - base)) * 32u;
        mbar_arrive_expect_tx(&full[t & 1], bytes);
        bulk_g2s(sbuf[t & 1], a.bodies + base, bytes, &full[t & 1]);
    };
    if (threadIdx.x == 0) {
        issue(0);
        if (ntiles > 1) issue(1);
    }
    const double eps2 = a.eps2;
    for (int t = 0; t < ntiles; ++t) {
        mbar_wait(&full[t & 1], (t >> 1) & 1);
        const double4* sb = sbuf[t & 1];
        const int len = static_cast<int>(mn<int64_t>(kTileJ, j1 - (j0 + static_cast<int64_t>(t) * kTileJ)));
#pragma unroll 2
        for (int j = 0; j < len; ++j) {
            const double4 b = sb[j];
#pragma unroll
            for (int r = 0; r < kR; ++r) {
                const double dx = b.x - px[r], dy = b.y - py[r], dz = b.z - pz[r];
                const double r2 = fma(dx, dx, fma(dy, dy, fma(dz, dz, eps2)));
                const double y0 = rsqrt_approx_f64(r2);
                const double y2 = y0 * y0;
                const double e = fma(r2, y2, -1.0);
                const double c = fma(e, fma(1.875, e, -1.5), 1.0);      // (1 + e)^(-3/2), 2nd order
                const double s = ((b.w * y0) * y2) * c;                 // m_j (r^2 + eps^2)^(-3/2)
                ax[r] = fma(s, dx, ax[r]);
                ay[r] = fma(s, dy, ay[r]);
                az[r] = fma(s, dz, az[r]);
            }
        }
        __syncthreads();
        if (threadIdx.x == 0 && t + 2 < ntiles) issue(t + 2);
    }
    auto store = [&](double4* p, int r) {
        double2* q = reinterpret_cast<double2*>(p);
        q[0] = make_double2(ax[r], ay[r]);
        q[1] = make_double2(az[r], 0.0);
    };
    if (a.splits == 1) {
#pragma unroll
        for (int r = 0; r < kR; ++r) {
            const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * kBlock;
            if (valid[r]) store(a.accel + t, r);
        }
        return;
    }
#pragma unroll
    for (int r = 0; r < kR; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * kBlock;
        if (valid[r]) store(a.partial + static_cast<int64_t>(split) * a.tgt_count + t, r);
    }
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = (atomicAdd(a.counters + tile, 1u) == static_cast<unsigned>(a.splits - 1));
    __syncthreads();
    if (!s_last) return;
    __threadfence();
#pragma unroll
    for (int r = 0; r < kR; ++r) {
        const int64_t t = tbase + threadIdx.x + static_cast<int64_t>(r) * kBlock;
        if (!valid[r]) continue;
        double sx = 0.0, sy = 0.0, sz = 0.0;
        for (int s = 0; s < a.splits; ++s) {
            const double2* q = reinterpret_cast<const double2*>(a.partial + static_cast<int64_t>(s) * a.tgt_count + t);
            const double2 u = __ldcg(q), v = __ldcg(q + 1);
            sx = (s == 0) ? u.x : sx + u.x;
            sy = (s == 0) ? u.y : sy + u.y;
            sz = (s == 0) ? v.x : sz + v.x;
        }
        ax[r] = sx; ay[r] = sy; az[r] = sz;
        store(a.accel + t, r);
        // leave the workspace zero-filled (stale partials could sit where a later call keeps tickets)
        for (int s = 0; s < a.splits; ++s) {
            double2* q = reinterpret_cast<double2*>(a.partial + static_cast<int64_t>(s) * a.tgt_count + t);
            __stcg(q, make_double2(0.0, 0.0));
            __stcg(q + 1, make_double2(0.0, 0.0));
        }
    }
    if (threadIdx.x == 0) a.counters[tile] = 0u;
}

cudaError_t launch_force(const double* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, double eps2,
                         double* accel, void* ws, cudaStream_t stream) {
    if (tgt_count == 0) return cudaSuccess;
    Args a;
    a.bodies = reinterpret_cast<const double4*>(bodies);
    a.n_src = n_src;
    a.tgt_begin = tgt_begin;
    a.tgt_count = tgt_count;
    a.eps2 = eps2;
    a.accel = reinterpret_cast<double4*>(accel);
    a.splits = nbody::splits_fixed(n_src);
    a.split_len = nbody::chunks_per_split_fixed(n_src) * nbody::kChunk;
    a.counters = static_cast<unsigned*>(ws);
    a.partial = reinterpret_cast<double4*>(static_cast<char*>(ws) + counters_bytes(tgt_count));
    const int64_t tiles = ceil_div<int64_t>(tgt_count, static_cast<int64_t>(kBlock) * kR);
    force64_kernel<<<dim3(static_cast<unsigned>(tiles), static_cast<unsigned>(a.splits)), kBlock, 0, stream>>>(a);
    return cudaGetLastError();
}

}  // namespace nbody64
}  // namespace lime
