// N-Body force map: occupancy sweep of the production kernel (force_kernel's MINB launch bound).
// ncu at 2^20: FP32 pipe 84 % busy at 32 warps/SM (58 registers); do more resident warps hide the
// MUFU/FFMA2 dependency chains better?  Same arithmetic => outputs must be bit-identical.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I include -o tools/nbody_occ tools/nbody_occ.cu
#include <cstdio>
#include <cstring>
#include <vector>
#include "../paper_conf_pldi_dubachcrbf12_b200/csrc/nbody.cu"

namespace lime {
const LaunchOverride& launch_override() { static LaunchOverride o; return o; }
int device_num_sms() { return 148; }
int nbody_variant() { return 0; }
}
using namespace lime;
using namespace lime::nbody;

static uint64_t sm64(uint64_t& s) {
    uint64_t z = (s += 0x9E3779B97F4A7C15ull);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

int main(int argc, char** argv) {
    const int64_t n = 1 << 20;
    const int64_t count = argc > 1 ? atoll(argv[1]) : (1 << 17);
    std::vector<float4> h(n);
    uint64_t st = 5;
    for (auto& b : h) {
        b.x = 2.f * ((sm64(st) >> 40) * (1.f / 16777216.f)) - 1.f;
        b.y = 2.f * ((sm64(st) >> 40) * (1.f / 16777216.f)) - 1.f;
        b.z = 2.f * ((sm64(st) >> 40) * (1.f / 16777216.f)) - 1.f;
        b.w = 1.f / n;
    }
    const bool mixed = argc > 2 && argv[2][0] == 'm';   // unequal masses: every chunk takes the 12-op path
    if (mixed) for (auto& b : h) b.w = (0.5f + ((sm64(st) >> 40) * (1.f / 16777216.f))) / n;
    float4 *bodies, *acc, *ref;
    cudaMalloc(&bodies, n * 16); cudaMalloc(&acc, count * 16); cudaMalloc(&ref, count * 16);
    cudaMemcpy(bodies, h.data(), n * 16, cudaMemcpyHostToDevice);
    void* ws; const size_t wsb = workspace_bytes(n, count);
    cudaMalloc(&ws, wsb); cudaMemset(ws, 0, wsb);
    ForceArgs a;
    a.bodies = bodies; a.n_src = n; a.tgt_begin = 0; a.tgt_count = count; a.eps2 = 1e-4f;
    a.splits = splits(n); a.chunk = chunk_len(n); a.split_len = chunks_per_split(n) * a.chunk;
    a.counters = static_cast<unsigned*>(ws);
    a.partial = reinterpret_cast<float4*>(static_cast<char*>(ws) + counters_bytes(count) + flags_bytes(n));
    uint8_t* flags = reinterpret_cast<uint8_t*>(static_cast<char*>(ws) + counters_bytes(count));
    prepass_kernel<<<512, 256>>>(bodies, n, flags, a.counters, ceil_div<int64_t>(count, 128));
    a.uniform = flags;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float4> hr(count), hg(count);
    bool have_ref = false;
    auto run = [&](auto kern, int block, int R, int minb) {
        const int64_t tiles = ceil_div<int64_t>(count, static_cast<int64_t>(block) * R);
        dim3 grid(static_cast<unsigned>(tiles), static_cast<unsigned>(a.splits));
        a.accel = have_ref ? acc : ref;
        kern<<<grid, block>>>(a);
        cudaDeviceSynchronize();
        float best = 1e30f, tot = 0.f;
        const int reps = 6;
        for (int r = 0; r < reps; ++r) {
            cudaEventRecord(e0);
            kern<<<grid, block>>>(a);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            best = ms < best ? ms : best;
            tot += ms;
        }
        bool same = true;
        if (have_ref) {
            cudaMemcpy(hg.data(), acc, count * 16, cudaMemcpyDeviceToHost);
            same = std::memcmp(hg.data(), hr.data(), count * 16) == 0;
        } else {
            cudaMemcpy(hr.data(), ref, count * 16, cudaMemcpyDeviceToHost);
            have_ref = true;
        }
        cudaFuncAttributes at; cudaFuncGetAttributes(&at, kern);
        int occ = 0; cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, block, 0);
        const double inter = double(count) * n;
        printf("{\"masses\": \"%s\", \"block\": %d, \"R\": %d, \"minb\": %d, \"regs\": %d, \"local\": %zu, \"ctas_per_sm\": %d, "
               "\"best_ms\": %.3f, \"mean_ms\": %.3f, \"Gint_s\": %.1f, \"frac_fp32\": %.4f, \"bit_identical\": %s}\n",
               mixed ? "mixed" : "equal", block, R, minb, at.numRegs, at.localSizeBytes, occ, best, tot / reps, inter / (best * 1e-3) / 1e9,
               20.0 * inter / (best * 1e-3) / 74.44992e12, same ? "true" : "false");
        fflush(stdout);
    };
    // production path (prepass + both force instantiations) through launch_force
    {
        auto lf = [&](const ForceArgs& aa) { launch_force(bodies, n, 0, count, 1e-4f, aa.accel, ws, 0); };
        a.accel = ref;
        lf(a);
        cudaDeviceSynchronize();
        float best = 1e30f;
        for (int r = 0; r < 6; ++r) {
            cudaEventRecord(e0); lf(a); cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1); best = ms < best ? ms : best;
        }
        cudaMemcpy(hr.data(), ref, count * 16, cudaMemcpyDeviceToHost);
        have_ref = true;
        const double inter = double(count) * n;
        printf("{\"masses\": \"%s\", \"path\": \"launch_force (production)\", \"best_ms\": %.3f, \"Gint_s\": %.1f, \"frac_fp32\": %.4f}\n",
               mixed ? "mixed" : "equal", best, inter / (best * 1e-3) / 1e9, 20.0 * inter / (best * 1e-3) / 74.44992e12);
        fflush(stdout);
    }
    run(force_kernel<256, 2, true, kChunk, 0, false>, 256, 2, 0);    // per-body-mass instantiation alone
    if (argc > 3 && argv[3][0] == 'w') {              // wide tiles (mass-uniform, equal masses)
        run(force_kernel<512, 4, true, kChunk, 1, true>, 512, 4, 1);
        run(force_kernel<384, 4, true, kChunk, 1, true>, 384, 4, 1);
        run(force_kernel<384, 6, true, kChunk, 1, true>, 384, 6, 1);
        run(force_kernel<256, 6, true, kChunk, 1, true>, 256, 6, 1);
        run(force_kernel<256, 6, true, kChunk, 2, true>, 256, 6, 2);
        run(force_kernel<320, 4, true, kChunk, 1, true>, 320, 4, 1);
        run(force_kernel<448, 4, true, kChunk, 1, true>, 448, 4, 1);
        run(force_kernel<512, 4, true, kChunk, 1, false>, 512, 4, 1);   // per-body-mass form
    } else if (argc > 3 && argv[3][0] == 'u') {       // mass-uniform instantiations (equal masses)
        run(force_kernel<256, 2, true, kChunk, 0, true>, 256, 2, 0);
        run(force_kernel<256, 4, true, kChunk, 3, true>, 256, 4, 3);
        run(force_kernel<256, 4, true, kChunk, 2, true>, 256, 4, 2);
        run(force_kernel<128, 4, true, kChunk, 5, true>, 128, 4, 5);
        run(force_kernel<128, 4, true, kChunk, 4, true>, 128, 4, 4);
        run(force_kernel<128, 8, true, kChunk, 3, true>, 128, 8, 3);
        run(force_kernel<256, 8, true, kChunk, 1, true>, 256, 8, 1);
        run(force_kernel<512, 2, true, kChunk, 2, true>, 512, 2, 2);
        run(force_kernel<512, 2, true, kChunk, 1, true>, 512, 2, 1);
        run(force_kernel<512, 4, true, kChunk, 1, true>, 512, 4, 1);
        run(force_kernel<64, 4, true, kChunk, 6, true>, 64, 4, 6);
        run(force_kernel<64, 4, true, kChunk, 8, true>, 64, 4, 8);
        run(force_kernel<256, 4, true, kChunk, 3, false>, 256, 4, 3);    // (per-body mass form, for the record)
    } else if (argc > 3) {
        run(force_kernel<256, 2, true, kChunk, 1>, 256, 2, 1);
        run(force_kernel<256, 2, true, kChunk, 4>, 256, 2, 4);
        run(force_kernel<256, 2, true, kChunk, 5>, 256, 2, 5);
        run(force_kernel<256, 4, true, kChunk, 4>, 256, 4, 4);
        run(force_kernel<128, 4, true, kChunk, 8>, 128, 4, 8);
    }
    a.uniform = nullptr;   // per-body masses everywhere: the pre-R11 production kernel
    run(force_kernel<256, 2, true, kChunk, 0, false>, 256, 2, 0);
    printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
