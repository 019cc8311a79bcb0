// gemm.cu -- dense matrix multiply as a map of dot products on the 5th-gen tensor cores (sm_100a).
//
// BASELINE.json config 4 (not in the paper; R8): C[i][j] = sum_k A[i][k] Bt[j][k],
// A [M][K], Bt [N][K] bf16 (K-major: each output element is the dot product of two contiguous
// K-vectors), C [M][N] fp32. The only dense contraction of the path, so the only kernel on the
// tensor cores (north_star).
//
// Design (DESIGN.md §"Matmul"): persistent, warp-specialised, one CTA per SM:
//   warp 0      TMA producer: 2-D tensor-map loads (128B swizzle -- the B200 form of the paper's
//               bank-conflict padding, L241-255) of A/B K-slices into a STAGES-deep smem ring
//               (A4: local-memory tiling of the broadcast operand, L234-241)
//   warp 1      TMEM allocator + single-thread tcgen05.mma issuer (kind::f16, BF16 x BF16 -> FP32,
//               accumulator in TMEM), tcgen05.commit releases smem stages / publishes accumulators
//   warps 2..5  epilogue: tcgen05.ld TMEM -> registers -> fp32 C (A7), double-buffered TMEM
//               accumulators (2 x 256 columns) so the epilogue of tile t overlaps the MMAs of t+1.
#include <cstring>

#include <cuda.h>
#include <cudaTypedefs.h>

#include "common.cuh"
#include "kernels.h"

#ifndef LIME_GEMM_SNAKE
#define LIME_GEMM_SNAKE 1
#endif

namespace lime {
namespace gemm {

constexpr int BM = 128;            // UMMA_M (cta_group::1)
constexpr int BN = 256;            // UMMA_N
constexpr int BK = 64;             // one 128-byte swizzle atom of bf16
constexpr int UMMA_K = 16;
constexpr int STAGES = 4;
constexpr int kThreads = 192;      // 6 warps
constexpr uint32_t kStageA = BM * BK * 2;       // 16 KB
constexpr uint32_t kStageB = BN * BK * 2;       // 32 KB
constexpr uint32_t kStageBytes = kStageA + kStageB;
constexpr uint32_t kTmemCols = 512;             // 2 accumulators x 256 fp32 columns
constexpr int kGroupM = 16;                     // raster: 16 M-blocks share B tiles in L2
constexpr size_t kSmemBytes = 1024 /*align slack*/ + STAGES * kStageBytes + 256 /*barriers*/;

// ------------------------------------------------------------------ PTX wrappers (sm_100a)
__device__ __forceinline__ void tma_load_2d(const CUtensorMap* map, void* dst, uint64_t* bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        :: "r"(smem_addr(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_addr(bar))
        : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" :: "l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                 :: "r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}"
        :: "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc) : "memory");
}
// 32 lanes x 32 consecutive fp32 columns: thread i gets TMEM lane (quadrant*32 + i), columns c..c+31
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float (&v)[32]) {
    uint32_t r[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

// UMMA shared-memory descriptor: K-major operand, 128-byte swizzle, 8-row core-matrix groups
// 1024 B apart (SBO), LBO unused (1), descriptor version 1 (sm_100).
__device__ __forceinline__ uint64_t smem_desc_sw128(uint32_t saddr) {
    return static_cast<uint64_t>((saddr >> 4) & 0x3FFF) | (static_cast<uint64_t>(1) << 16) |
           (static_cast<uint64_t>(1024 >> 4) << 32) | (static_cast<uint64_t>(1) << 46) |
           (static_cast<uint64_t>(2) << 61);
}
// Instruction descriptor: kind::f16, A = B = BF16, D = F32, both K-major, M = BM, N = BN.
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | (static_cast<uint32_t>(BN >> 3) << 17) |
                            (static_cast<uint32_t>(BM >> 4) << 24);

struct Params {
    float* C;
    int M, N, K;
    int num_m, num_n, num_k;
    int num_tiles;
};

__device__ __forceinline__ void tile_coords(int t, const Params& p, int& mb, int& nb) {
    const int per_group = kGroupM * p.num_n;
    const int g = t / per_group;
    const int first_m = g * kGroupM;
    const int gm = min(p.num_m - first_m, kGroupM);
    const int r = t - g * per_group;
    mb = first_m + r % gm;
    nb = r / gm;
#if LIME_GEMM_SNAKE
    // serpentine sweep: odd groups walk the N tiles backwards, so the Bt tiles the previous group
    // touched last -- still in L2 -- are the first ones this group reads
    if (g & 1) nb = p.num_n - 1 - nb;
#endif
}

__global__ void __launch_bounds__(kThreads, 1)
gemm_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
            const __grid_constant__ Params p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * kStageBytes);
    uint64_t* empty = full + STAGES;
    uint64_t* tfull = empty + STAGES;
    uint64_t* tempty = tfull + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;

    if (warp == 0 && lane == 0) {
        prefetch_tmap(&tmap_a);
        prefetch_tmap(&tmap_b);
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], 4);     // one arrive per epilogue warp
        }
        fence_mbar_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_addr(tmem_slot)), "r"(kTmemCols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        // ----------------------------------------------------------- TMA producer
        if (lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            for (int t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
                int mb, nb;
                tile_coords(t, p, mb, nb);
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    uint8_t* sa = smem + s * kStageBytes;
                    mbar_arrive_expect_tx(&full[s], kStageBytes);
                    tma_load_2d(&tmap_a, sa, &full[s], kb * BK, mb * BM);
                    tma_load_2d(&tmap_b, sa + kStageA, &full[s], kb * BK, nb * BN);
                    if (++s == STAGES) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        // ----------------------------------------------------------- MMA issuer
        if (lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            int local = 0;
            for (int t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++local) {
                const int acc = local & 1;
                mbar_wait(&tempty[acc], ((local >> 1) & 1) ^ 1);
                tc_fence_after();
                const uint32_t dtm = tmem_base + static_cast<uint32_t>(acc * BN);
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&full[s], ph);
                    tc_fence_after();
                    const uint32_t sa = smem_addr(smem + s * kStageBytes);
                    const uint32_t sb = sa + kStageA;
#pragma unroll
                    for (int k = 0; k < BK / UMMA_K; ++k) {
                        tc_mma(dtm, smem_desc_sw128(sa + k * UMMA_K * 2), smem_desc_sw128(sb + k * UMMA_K * 2), kIdesc,
                               (kb | k) != 0);
                    }
                    tc_commit(&empty[s]);            // frees this smem stage when the MMAs retire
                    if (++s == STAGES) { s = 0; ph ^= 1; }
                }
                tc_commit(&tfull[acc]);              // accumulator complete
            }
        }
        __syncwarp();
    } else {
        // ----------------------------------------------------------- epilogue (warps 2..5)
        const int quad = warp & 3;                   // TMEM lane quadrant this warp may access
        const int row_in_tile = quad * 32 + lane;
        int local = 0;
        for (int t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++local) {
            const int acc = local & 1;
            int mb, nb;
            tile_coords(t, p, mb, nb);
            mbar_wait(&tfull[acc], (local >> 1) & 1);
            tc_fence_after();
            const int row = mb * BM + row_in_tile;
            const uint32_t tbase = tmem_base + (static_cast<uint32_t>(quad * 32) << 16) + static_cast<uint32_t>(acc * BN);
            float* crow = p.C + static_cast<int64_t>(row) * p.N;
            const bool vec_ok = (p.N & 3) == 0;
#pragma unroll 1
            for (int c = 0; c < BN; c += 32) {
                float v[32];
                tmem_ld32(tbase + c, v);
                const int col0 = nb * BN + c;
                if (row < p.M) {
                    if (vec_ok && col0 + 32 <= p.N) {
#pragma unroll
                        for (int q = 0; q < 8; ++q)
                            st_stream_f4(reinterpret_cast<float4*>(crow + col0) + q,
                                         make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]));
                    } else {
#pragma unroll
                        for (int q = 0; q < 32; ++q)
                            if (col0 + q < p.N) crow[col0 + q] = v[q];
                    }
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&tempty[acc]);
        }
    }

    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem_base), "r"(kTmemCols) : "memory");
    }
}

// =====================================================================================
// 2-CTA variant (cta_group::2): a CTA pair on one TPC computes a 256 x 256 tile. Each CTA stages
// its 128-row half of A and its 128-row half of Bt (per K-slice: 16 + 16 KB), so each SM's smem
// and L2 traffic per flop is 2/3 of the 1-CTA 128 x 256 tile's; the leader CTA's single thread
// issues tcgen05.mma.cta_group::2 (M = 256, N = 256, K = 16) reading both CTAs' smem, and each
// CTA's TMEM receives its own 128 accumulator rows.
// =====================================================================================
namespace two {
constexpr int BM = 128;                 // rows of A per CTA (pair tile: 256)
constexpr int BN = 256;                 // pair tile N (each CTA stages 128 rows of Bt)
constexpr int STAGES = 6;
constexpr uint32_t kStageA = BM * BK * 2;            // 16 KB
constexpr uint32_t kStageB = (BN / 2) * BK * 2;      // 16 KB
constexpr uint32_t kStageBytes = kStageA + kStageB;
// epilogue staging for TMA stores: per epilogue warp two 32 x 32 fp32 boxes (4 KB each, 128B-swizzled)
constexpr uint32_t kEpiBox = 32 * 32 * 4;
constexpr uint32_t kEpiBytes = 4 * 2 * kEpiBox;
constexpr size_t kSmemBytes = 1024 + STAGES * kStageBytes + kEpiBytes + 256;
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | (static_cast<uint32_t>(BN >> 3) << 17) |
                            (static_cast<uint32_t>(256 >> 4) << 24);
}  // namespace two

__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" :: "r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx_cluster(uint32_t cluster_addr, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cluster.shared::cluster.b64 _, [%0], %1;"
                 :: "r"(cluster_addr), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_load_2d_pair(const CUtensorMap* map, void* dst, uint32_t leader_bar, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
        :: "r"(smem_addr(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(leader_bar)
        : "memory");
}
__device__ __forceinline__ void tc_mma_pair(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}"
        :: "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void tc_commit_pair(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                 :: "r"(smem_addr(bar)), "h"(static_cast<uint16_t>(3)) : "memory");
}

// TMA tensor store of one smem box (bulk-group completion; no mbarrier)
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, const void* src, int c0, int c1) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                 :: "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_addr(src)) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void st_shared_f4(uint32_t addr, float a, float b, float c, float d) {
    asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" :: "r"(addr), "f"(a), "f"(b), "f"(c), "f"(d) : "memory");
}

struct Params2 {
    float* C;
    int tma_store;             // 1: C is written through tmap_c (N % 4 == 0, 16-B aligned C)
    int M, N, K;
    int group;                 // raster group: pair-tile rows that sweep the N tiles together
    int num_m, num_n, num_k;   // num_m counts 256-row pair tiles
    int num_tiles;
};

__device__ __forceinline__ void tile_coords2(int t, const Params2& p, int& mb, int& nb) {
    const int G = p.group;     // raster group of pair-tile rows sharing Bt tiles in L2
    const int per_group = G * p.num_n;
    const int g = t / per_group;
    const int first_m = g * G;
    const int gm = min(p.num_m - first_m, G);
    const int r = t - g * per_group;
    mb = first_m + r % gm;
    nb = r / gm;
#if LIME_GEMM_SNAKE
    // serpentine sweep: odd groups walk the N tiles backwards, so the Bt tiles the previous group
    // touched last -- still in L2 -- are the first ones this group reads
    if (g & 1) nb = p.num_n - 1 - nb;
#endif
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(kThreads, 1)
gemm2_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
             const __grid_constant__ CUtensorMap tmap_c, const __grid_constant__ Params2 p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* epi = smem + two::STAGES * two::kStageBytes;                 // 1024-B aligned staging
    uint64_t* full = reinterpret_cast<uint64_t*>(epi + two::kEpiBytes);
    uint64_t* empty = full + two::STAGES;
    uint64_t* tfull = empty + two::STAGES;
    uint64_t* tempty = tfull + 2;
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();
    const bool leader = (rank == 0);
    const int cluster = blockIdx.x >> 1;
    const int nclusters = gridDim.x >> 1;

    if (warp == 0 && lane == 0) {
        prefetch_tmap(&tmap_a);
        prefetch_tmap(&tmap_b);
        if (p.tma_store) prefetch_tmap(&tmap_c);
        for (int s = 0; s < two::STAGES; ++s) {
            mbar_init(&full[s], 1);      // leader's producer arms it with both CTAs' tx bytes
            mbar_init(&empty[s], 1);     // released by the leader's MMA commit (multicast to both CTAs)
        }
        for (int a = 0; a < 2; ++a) {
            mbar_init(&tfull[a], 1);
            mbar_init(&tempty[a], 8);    // 4 epilogue warps x 2 CTAs (leader's copy is the one used)
        }
        fence_mbar_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_addr(tmem_slot)), "r"(kTmemCols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    cluster_sync();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            for (int t = cluster; t < p.num_tiles; t += nclusters) {
                int mb, nb;
                tile_coords2(t, p, mb, nb);
                const int arow = mb * 256 + static_cast<int>(rank) * two::BM;
                const int brow = nb * two::BN + static_cast<int>(rank) * (two::BN / 2);
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    uint8_t* sa = smem + s * two::kStageBytes;
                    const uint32_t lbar = mapa_shared(smem_addr(&full[s]), 0);
                    // only the leader arms its barrier, for both CTAs' bytes; the peer's TMA
                    // complete_tx lands on the same barrier (no remote arrive on the hot loop)
                    if (leader) mbar_arrive_expect_tx(&full[s], 2 * two::kStageBytes);
                    tma_load_2d_pair(&tmap_a, sa, lbar, kb * BK, arow);
                    tma_load_2d_pair(&tmap_b, sa + two::kStageA, lbar, kb * BK, brow);
                    if (++s == two::STAGES) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        if (leader && lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            int local = 0;
            for (int t = cluster; t < p.num_tiles; t += nclusters, ++local) {
                const int acc = local & 1;
                mbar_wait(&tempty[acc], ((local >> 1) & 1) ^ 1);
                tc_fence_after();
                const uint32_t dtm = tmem_base + static_cast<uint32_t>(acc * two::BN);
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&full[s], ph);
                    tc_fence_after();
                    const uint32_t sa = smem_addr(smem + s * two::kStageBytes);
                    const uint32_t sb = sa + two::kStageA;
#pragma unroll
                    for (int k = 0; k < BK / UMMA_K; ++k)
                        tc_mma_pair(dtm, smem_desc_sw128(sa + k * UMMA_K * 2), smem_desc_sw128(sb + k * UMMA_K * 2),
                                    two::kIdesc, (kb | k) != 0);
                    tc_commit_pair(&empty[s]);
                    if (++s == two::STAGES) { s = 0; ph ^= 1; }
                }
                tc_commit_pair(&tfull[acc]);
            }
        }
        __syncwarp();
    } else {
        const int quad = warp & 3;
        const int row_in_tile = quad * 32 + lane;
        const uint32_t tempty_leader0 = mapa_shared(smem_addr(&tempty[0]), 0);
        int local = 0;
        for (int t = cluster; t < p.num_tiles; t += nclusters, ++local) {
            const int acc = local & 1;
            int mb, nb;
            tile_coords2(t, p, mb, nb);
            mbar_wait(&tfull[acc], (local >> 1) & 1);
            tc_fence_after();
            const int row = mb * 256 + static_cast<int>(rank) * two::BM + row_in_tile;
            const uint32_t tbase = tmem_base + (static_cast<uint32_t>(quad * 32) << 16) + static_cast<uint32_t>(acc * two::BN);
            float* crow = p.C + static_cast<int64_t>(row) * p.N;
            const bool vec_ok = (p.N & 3) == 0;
            if (p.tma_store) {
                // TMEM -> registers -> this warp's 128B-swizzled 32 x 32 smem box -> one TMA store of
                // full 128-byte lines (the direct path writes each row's 16-byte pieces from 32 lanes:
                // 8x the L2 write requests); two boxes in turn, a box is rewritten only after the
                // store issued from it two chunks earlier has read it. The store clips at M and N.
                const uint32_t box0 = smem_addr(epi + (quad * 2) * two::kEpiBox);
                const int row0 = mb * 256 + static_cast<int>(rank) * two::BM + quad * 32;
#pragma unroll 1
                for (int c = 0; c < two::BN; c += 32) {
                    float v[32];
                    tmem_ld32(tbase + c, v);
                    const uint32_t box = box0 + static_cast<uint32_t>(((c >> 5) & 1) * two::kEpiBox);
                    if (lane == 0) bulk_wait_read<1>();
                    __syncwarp();
#pragma unroll
                    for (int q = 0; q < 8; ++q)
                        st_shared_f4(box + static_cast<uint32_t>(lane * 128 + ((q ^ (lane & 7)) << 4)), v[4 * q],
                                     v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]);
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_2d(&tmap_c, epi + (box - smem_addr(epi)), nb * two::BN + c, row0);
                        bulk_commit();
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive_cluster(tempty_leader0 + static_cast<uint32_t>(acc * 8));
                continue;
            }
#pragma unroll 1
            for (int c = 0; c < two::BN; c += 32) {
                float v[32];
                tmem_ld32(tbase + c, v);
                const int col0 = nb * two::BN + c;
                if (row < p.M) {
                    if (vec_ok && col0 + 32 <= p.N) {
#pragma unroll
                        for (int q = 0; q < 8; ++q)
                            st_stream_f4(reinterpret_cast<float4*>(crow + col0) + q,
                                         make_float4(v[4 * q], v[4 * q + 1], v[4 * q + 2], v[4 * q + 3]));
                    } else {
#pragma unroll
                        for (int q = 0; q < 32; ++q)
                            if (col0 + q < p.N) crow[col0 + q] = v[q];
                    }
                }
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive_cluster(tempty_leader0 + static_cast<uint32_t>(acc * 8));
        }
        if (p.tma_store && lane == 0) bulk_wait_all();   // staging smem must outlive the stores
    }

    tc_fence_before();
    cluster_sync();
    if (warp == 1) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" :: "r"(tmem_base), "r"(kTmemCols) : "memory");
    }
}

// =====================================================================================
// Wide pair tile (round 2): a CTA pair computes 256 x 512 of C as two N = 256 halves H0 | H1 that
// fill each SM's 512 TMEM columns. Per 64-element K slice each CTA stages 128 rows of A and 2 x 128
// rows of Bt (48 KB), so a call moves 3/4 of the 256 x 256 tile's L2->SM bytes (8192^3: 6.4 vs
// 8.6 GB -- what cuBLAS moves; the kernel is power-capped, so fewer bytes buy clock).
// With no spare TMEM for a second accumulator, the tile boundary is overlapped instead:
//  * 8 epilogue warps (two per TMEM lane quadrant, 128 columns each) pull a half into registers
//    (4 x tcgen05.ld.32x32b.x32, one wait) and release it at once; the global stores (TMA, one
//    32 x 32 smem box per warp) follow from registers while the next tile's MMAs run;
//  * the MMA thread starts tile t+1 on H0 as soon as H0 is released and defers the H1 MMAs of
//    the first STAGES - 1 K slices (their smem stages stay held) until H1 is released too.
// =====================================================================================
namespace wide {
constexpr int BM = 128;                   // rows of A per CTA (pair tile: 256)
constexpr int BN = 512;                   // pair tile N: two N = 256 MMAs per K step
constexpr int STAGES = 4;
constexpr int kThreads = 320;             // producer, MMA, 8 epilogue warps
constexpr uint32_t kStageA = BM * BK * 2;             // 16 KB
constexpr uint32_t kStageBh = 128 * BK * 2;           // 16 KB per half (this CTA's 128 rows of an N = 256 chunk)
constexpr uint32_t kStageBytes = kStageA + 2 * kStageBh;
constexpr uint32_t kEpiBox = 32 * 32 * 4;             // one 32 x 32 fp32 box per epilogue warp
constexpr uint32_t kEpiBytes = 8 * kEpiBox;
constexpr size_t kSmemBytes = 1024 + STAGES * kStageBytes + kEpiBytes + 256;
constexpr int kDefer = STAGES - 1;
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | (static_cast<uint32_t>(256 >> 3) << 17) |
                            (static_cast<uint32_t>(256 >> 4) << 24);
}  // namespace wide

// 4 x 32 consecutive fp32 columns of this warp's TMEM lane quadrant, one wait
__device__ __forceinline__ void tmem_ld128(uint32_t taddr, uint32_t (&r)[128]) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        asm volatile(
            "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
            "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
            "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
            : "=r"(r[32 * q + 0]), "=r"(r[32 * q + 1]), "=r"(r[32 * q + 2]), "=r"(r[32 * q + 3]), "=r"(r[32 * q + 4]),
              "=r"(r[32 * q + 5]), "=r"(r[32 * q + 6]), "=r"(r[32 * q + 7]), "=r"(r[32 * q + 8]), "=r"(r[32 * q + 9]),
              "=r"(r[32 * q + 10]), "=r"(r[32 * q + 11]), "=r"(r[32 * q + 12]), "=r"(r[32 * q + 13]),
              "=r"(r[32 * q + 14]), "=r"(r[32 * q + 15]), "=r"(r[32 * q + 16]), "=r"(r[32 * q + 17]),
              "=r"(r[32 * q + 18]), "=r"(r[32 * q + 19]), "=r"(r[32 * q + 20]), "=r"(r[32 * q + 21]),
              "=r"(r[32 * q + 22]), "=r"(r[32 * q + 23]), "=r"(r[32 * q + 24]), "=r"(r[32 * q + 25]),
              "=r"(r[32 * q + 26]), "=r"(r[32 * q + 27]), "=r"(r[32 * q + 28]), "=r"(r[32 * q + 29]),
              "=r"(r[32 * q + 30]), "=r"(r[32 * q + 31])
            : "r"(taddr + static_cast<uint32_t>(32 * q)));
    }
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(wide::kThreads, 1)
gemm_wide_kernel(const __grid_constant__ CUtensorMap tmap_a, const __grid_constant__ CUtensorMap tmap_b,
                 const __grid_constant__ CUtensorMap tmap_c, const __grid_constant__ Params2 p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
    uint8_t* epi = smem + wide::STAGES * wide::kStageBytes;
    uint64_t* full = reinterpret_cast<uint64_t*>(epi + wide::kEpiBytes);
    uint64_t* empty = full + wide::STAGES;
    uint64_t* tfull = empty + wide::STAGES;
    uint64_t* tempty = tfull + 1;                      // [2]: H0, H1 released
    uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

    const int warp = threadIdx.x >> 5;
    const int lane = threadIdx.x & 31;
    const uint32_t rank = cluster_ctarank();
    const bool leader = (rank == 0);
    const int cluster = blockIdx.x >> 1;
    const int nclusters = gridDim.x >> 1;

    if (warp == 0 && lane == 0) {
        prefetch_tmap(&tmap_a);
        prefetch_tmap(&tmap_b);
        prefetch_tmap(&tmap_c);
        for (int s = 0; s < wide::STAGES; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], 1);
        }
        mbar_init(&tfull[0], 1);
        mbar_init(&tempty[0], 16);       // 8 epilogue warps x 2 CTAs (the leader's copy is the one used)
        mbar_init(&tempty[1], 16);
        fence_mbar_init();
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;"
                     :: "r"(smem_addr(tmem_slot)), "r"(kTmemCols) : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    }
    tc_fence_before();
    cluster_sync();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_slot;

    if (warp == 0) {
        if (lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            for (int t = cluster; t < p.num_tiles; t += nclusters) {
                int mb, nb;
                tile_coords2(t, p, mb, nb);
                const int arow = mb * 256 + static_cast<int>(rank) * wide::BM;
                const int brow = nb * wide::BN + static_cast<int>(rank) * 128;
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&empty[s], ph ^ 1);
                    uint8_t* sa = smem + s * wide::kStageBytes;
                    const uint32_t lbar = mapa_shared(smem_addr(&full[s]), 0);
                    if (leader) mbar_arrive_expect_tx(&full[s], 2 * wide::kStageBytes);
                    tma_load_2d_pair(&tmap_a, sa, lbar, kb * BK, arow);
                    tma_load_2d_pair(&tmap_b, sa + wide::kStageA, lbar, kb * BK, brow);
                    tma_load_2d_pair(&tmap_b, sa + wide::kStageA + wide::kStageBh, lbar, kb * BK, brow + 256);
                    if (++s == wide::STAGES) { s = 0; ph ^= 1; }
                }
            }
        }
    } else if (warp == 1) {
        if (leader && lane == 0) {
            int s = 0;
            uint32_t ph = 0;
            int local = 0;
            auto mma_half = [&](int st, int kb, int h) {
                const uint32_t sa = smem_addr(smem + st * wide::kStageBytes);
                const uint32_t sb = sa + wide::kStageA + static_cast<uint32_t>(h) * wide::kStageBh;
#pragma unroll
                for (int k = 0; k < BK / UMMA_K; ++k)
                    tc_mma_pair(tmem_base + static_cast<uint32_t>(h * 256), smem_desc_sw128(sa + k * UMMA_K * 2),
                                smem_desc_sw128(sb + k * UMMA_K * 2), wide::kIdesc, (kb | k) != 0);
            };
            for (int t = cluster; t < p.num_tiles; t += nclusters, ++local) {
                const uint32_t par = static_cast<uint32_t>(local & 1) ^ 1u;
                mbar_wait(&tempty[0], par);                // H0 drained (previous tile)
                tc_fence_after();
                int dst[wide::kDefer], dkb[wide::kDefer], nd = 0;
                bool h1_free = false;
                for (int kb = 0; kb < p.num_k; ++kb) {
                    mbar_wait(&full[s], ph);
                    tc_fence_after();
                    mma_half(s, kb, 0);
                    if (!h1_free && nd < wide::kDefer) {   // H1 still draining: hold this stage
                        dst[nd] = s;
                        dkb[nd] = kb;
                        ++nd;
                    } else {
                        if (!h1_free) {
                            mbar_wait(&tempty[1], par);
                            tc_fence_after();
                            h1_free = true;
                            for (int d = 0; d < nd; ++d) {
                                mma_half(dst[d], dkb[d], 1);
                                tc_commit_pair(&empty[dst[d]]);
                            }
                            nd = 0;
                        }
                        mma_half(s, kb, 1);
                        tc_commit_pair(&empty[s]);
                    }
                    if (++s == wide::STAGES) { s = 0; ph ^= 1; }
                }
                if (!h1_free) {                            // num_k <= kDefer
                    mbar_wait(&tempty[1], par);
                    tc_fence_after();
                    for (int d = 0; d < nd; ++d) {
                        mma_half(dst[d], dkb[d], 1);
                        tc_commit_pair(&empty[dst[d]]);
                    }
                }
                tc_commit_pair(&tfull[0]);
            }
        }
        __syncwarp();
    } else {
        // ----------------------------------------------------------- epilogue (warps 2..9)
        const int quad = warp & 3;
        const int colpart = (warp - 2) >> 2;               // 128-column part of each half
        const uint32_t tempty_leader = mapa_shared(smem_addr(&tempty[0]), 0);
        const uint32_t box = smem_addr(epi + (warp - 2) * wide::kEpiBox);
        int local = 0;
        for (int t = cluster; t < p.num_tiles; t += nclusters, ++local) {
            int mb, nb;
            tile_coords2(t, p, mb, nb);
            mbar_wait(&tfull[0], static_cast<uint32_t>(local & 1));
            tc_fence_after();
            const int row0 = mb * 256 + static_cast<int>(rank) * wide::BM + quad * 32;
#pragma unroll 1
            for (int h = 0; h < 2; ++h) {
                uint32_t r[128];
                tmem_ld128(tmem_base + (static_cast<uint32_t>(quad * 32) << 16) +
                               static_cast<uint32_t>(h * 256 + colpart * 128), r);
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive_cluster(tempty_leader + static_cast<uint32_t>(h * 8));
#pragma unroll
                for (int b = 0; b < 4; ++b) {
                    if (lane == 0) bulk_wait_read<0>();    // the previous store has read the box
                    __syncwarp();
#pragma unroll
                    for (int q = 0; q < 8; ++q)
                        st_shared_f4(box + static_cast<uint32_t>(lane * 128 + ((q ^ (lane & 7)) << 4)),
                                     __uint_as_float(r[32 * b + 4 * q]), __uint_as_float(r[32 * b + 4 * q + 1]),
                                     __uint_as_float(r[32 * b + 4 * q + 2]), __uint_as_float(r[32 * b + 4 * q + 3]));
                    fence_proxy_async_smem();
                    __syncwarp();
                    if (lane == 0) {
                        tma_store_2d(&tmap_c, epi + (box - smem_addr(epi)), nb * wide::BN + h * 256 + colpart * 128 + b * 32,
                                     row0);
                        bulk_commit();
                    }
                }
            }
        }
        if (lane == 0) bulk_wait_all();
    }

    tc_fence_before();
    cluster_sync();
    if (warp == 1) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" :: "r"(tmem_base), "r"(kTmemCols) : "memory");
    }
}

// ------------------------------------------------------------------ host side
}  // namespace gemm

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda); resolved once,
// thread-safe (function-local static). Shared with nbody.cu's TMA staging.
void* tensor_map_encoder() {
    static void* const fn = [] {
        void* ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            ptr = nullptr;
        return ptr;
    }();
    return fn;
}

namespace gemm {
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(tensor_map_encoder());
}

static bool make_map(CUtensorMap* map, const void* base, uint64_t rows, uint64_t K, uint32_t box_rows) {
    auto fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {K, rows};
    const cuuint64_t strides[1] = {K * 2};
    const cuuint32_t box[2] = {static_cast<cuuint32_t>(BK), box_rows};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
              CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// C [M][N] fp32 for the epilogue's TMA stores: 32 x 32 boxes (128-byte rows), 128B swizzle
static bool make_map_c(CUtensorMap* map, void* base, uint64_t rows, uint64_t cols) {
    auto fn = encode_fn();
    if (!fn) return false;
    const cuuint64_t dims[2] = {cols, rows};
    const cuuint64_t strides[1] = {cols * 4};
    const cuuint32_t box[2] = {32, 32};
    const cuuint32_t estr[2] = {1, 1};
    return fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t launch_bf16(const uint16_t* A, const uint16_t* Bt, float* C, int64_t M, int64_t N, int64_t K,
                        cudaStream_t stream) {
    const LaunchOverride& ov = launch_override();
    // per_thread override: 1 = 1-CTA kernel, 2 = 256 x 256 pair tile, 3 = the same with direct
    // stores, 4 = 256 x 512 pair tile; default: wide tile when it fits, else 256 x 256.
    const bool c_tma_ok = (N & 3) == 0 && (reinterpret_cast<uintptr_t>(C) & 15) == 0;
    const bool wide_tile = ov.per_thread == 4 || (ov.per_thread == 0 && M >= 256 && N >= 512 && c_tma_ok);
    const bool pair = ov.per_thread == 2 || ov.per_thread == 3 || (ov.per_thread == 0 && M >= 256);
    CUtensorMap ma, mb;
    if (wide_tile) {
        CUtensorMap mc;
        if (!c_tma_ok || !make_map(&ma, A, M, K, wide::BM) || !make_map(&mb, Bt, N, K, 128) || !make_map_c(&mc, C, M, N))
            return cudaErrorInvalidValue;
        Params2 p;
        p.C = C;
        p.tma_store = 1;
        p.M = static_cast<int>(M);
        p.N = static_cast<int>(N);
        p.K = static_cast<int>(K);
        p.num_m = static_cast<int>(ceil_div<int64_t>(M, 256));
        p.num_n = static_cast<int>(ceil_div<int64_t>(N, wide::BN));
        p.num_k = static_cast<int>(ceil_div<int64_t>(K, BK));
        p.num_tiles = p.num_m * p.num_n;
        p.group = ov.block_threads > 0 ? ov.block_threads : 8;   // override: raster group (sweep)
        cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&gemm_wide_kernel), static_cast<int>(wide::kSmemBytes));
        if (e != cudaSuccess) return e;
        int clusters = ov.grid_ctas > 0 ? mx(1, ov.grid_ctas / 2) : device_num_sms() / 2;
        clusters = mn(clusters, p.num_tiles);
        gemm_wide_kernel<<<2 * clusters, wide::kThreads, wide::kSmemBytes, stream>>>(ma, mb, mc, p);
        return cudaGetLastError();
    }
    if (pair) {
        if (!make_map(&ma, A, M, K, two::BM) || !make_map(&mb, Bt, N, K, two::BN / 2)) return cudaErrorInvalidValue;
        Params2 p;
        p.C = C;
        p.M = static_cast<int>(M);
        p.N = static_cast<int>(N);
        p.K = static_cast<int>(K);
        p.num_m = static_cast<int>(ceil_div<int64_t>(M, 256));
        p.num_n = static_cast<int>(ceil_div<int64_t>(N, two::BN));
        p.num_k = static_cast<int>(ceil_div<int64_t>(K, BK));
        p.num_tiles = p.num_m * p.num_n;
        p.group = ov.block_threads > 0 ? ov.block_threads : 8;   // override: raster group (sweep)
        CUtensorMap mc;
        std::memset(&mc, 0, sizeof mc);
        p.tma_store = ((N & 3) == 0 && (reinterpret_cast<uintptr_t>(C) & 15) == 0 && ov.per_thread != 3 &&
                       make_map_c(&mc, C, M, N)) ? 1 : 0;
        cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&gemm2_kernel), static_cast<int>(two::kSmemBytes));
        if (e != cudaSuccess) return e;
        int clusters = ov.grid_ctas > 0 ? mx(1, ov.grid_ctas / 2) : device_num_sms() / 2;
        clusters = mn(clusters, p.num_tiles);
        gemm2_kernel<<<2 * clusters, kThreads, two::kSmemBytes, stream>>>(ma, mb, mc, p);
        return cudaGetLastError();
    }
    if (!make_map(&ma, A, M, K, BM) || !make_map(&mb, Bt, N, K, BN)) return cudaErrorInvalidValue;
    Params p;
    p.C = C;
    p.M = static_cast<int>(M);
    p.N = static_cast<int>(N);
    p.K = static_cast<int>(K);
    p.num_m = static_cast<int>(ceil_div<int64_t>(M, BM));
    p.num_n = static_cast<int>(ceil_div<int64_t>(N, BN));
    p.num_k = static_cast<int>(ceil_div<int64_t>(K, BK));
    p.num_tiles = p.num_m * p.num_n;
    cudaError_t e = ensure_dynamic_smem(reinterpret_cast<const void*>(&gemm_kernel), static_cast<int>(kSmemBytes));
    if (e != cudaSuccess) return e;
    int grid = ov.grid_ctas;
    if (grid <= 0) grid = device_num_sms();
    grid = mn(grid, p.num_tiles);
    gemm_kernel<<<grid, kThreads, kSmemBytes, stream>>>(ma, mb, p);
    return cudaGetLastError();
}

}  // namespace gemm
}  // namespace lime
