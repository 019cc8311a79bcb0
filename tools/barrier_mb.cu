// Grid-barrier latency microbenchmark (persistent config-1 kernel): 148 CTAs x 896 threads, one per
// SM (cooperative launch), `iters` back-to-back barriers with no work; ns per barrier (globaltimer).
//   variant 0: __syncthreads; t0: __threadfence; red.release.gpu add; ld.acquire poll (product)
//   variant 1: same, atomicAdd (returns) instead of red
//   variant 2: per-CTA flag words (no atomic): t0 stores flag[cta] = epoch (st.release), warp 0's
//              lanes poll the 148 flags (ld.acquire), __all_sync
//   variant 3: as 2 but relaxed polling + one fence.acq_rel after
//   variant 4: no __threadfence (red.release only); 5: + relaxed polling and one acquire fence;
//   6: fence.acq_rel instead of __threadfence; 7: as 5 with ld.volatile polling
//   8/9/10: two-level counter, 16/8/32 groups
//   11/12: counter + broadcast go-flags (each CTA polls its own line; acquire / relaxed+fence)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/barrier_mb tools/barrier_mb.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>

template <int V>
__device__ __forceinline__ void gbar(unsigned* cnt, unsigned* flags, unsigned target, unsigned epoch) {
    __syncthreads();
    if (V == 11 || V == 12) {   // counter + broadcast: the last arriver writes every CTA's own go-flag line
        if (threadIdx.x < 32) {
            unsigned last = 0;
            if (threadIdx.x == 0) {
                __threadfence();
                unsigned old;
                asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(cnt), "r"(1u) : "memory");
                last = (old + 1 == target) ? 1u : 0u;
            }
            last = __shfl_sync(0xffffffffu, last, 0);
            if (last) {
                for (unsigned c = threadIdx.x; c < gridDim.x; c += 32)
                    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flags + c * 32), "r"(epoch) : "memory");
            }
            if (threadIdx.x == 0) {
                unsigned v;
                do {
                    if (V == 11) asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + blockIdx.x * 32) : "memory");
                    else asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + blockIdx.x * 32) : "memory");
                } while (static_cast<int>(v - epoch) < 0);
                if (V == 12) asm volatile("fence.acq_rel.gpu;" ::: "memory");
            }
        }
        __syncthreads();
        return;
    }
    if (V >= 8) {   // two levels: G sub-counters (own 128-B lines), the last of each group bumps the top
        constexpr int G = V == 8 ? 16 : (V == 9 ? 8 : 32);
        if (threadIdx.x == 0) {
            const unsigned g = blockIdx.x % G;
            const unsigned members = (gridDim.x - g + G - 1) / G;
            unsigned* sub = flags + g * 32;
            __threadfence();
            unsigned old;
            asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(sub), "r"(1u) : "memory");
            if (old + 1 == members * epoch) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(cnt) : "memory");
            unsigned v;
            do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(cnt) : "memory"); }
            while (static_cast<int>(v - static_cast<unsigned>(G) * epoch) < 0);
        }
        __syncthreads();
        return;
    }
    if (V <= 1 || V >= 4) {
        if (threadIdx.x == 0) {
            if (V <= 1) __threadfence();
            if (V == 6) asm volatile("fence.acq_rel.gpu;" ::: "memory");
            if (V == 0 || V >= 4) asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(cnt) : "memory");
            else atomicAdd(cnt, 1u);
            unsigned v;
            if (V == 5) {
                do { asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(cnt) : "memory"); }
                while (static_cast<int>(v - target) < 0);
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
            } else if (V == 7) {
                do { asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(v) : "l"(cnt) : "memory"); }
                while (static_cast<int>(v - target) < 0);
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
            } else {
                do { asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(cnt) : "memory"); }
                while (static_cast<int>(v - target) < 0);
            }
        }
    } else {
        if (threadIdx.x == 0) {
            __threadfence();
            asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flags + blockIdx.x * 32), "r"(epoch) : "memory");
        }
        if (threadIdx.x < 32) {
            bool ok;
            do {
                ok = true;
                for (unsigned c = threadIdx.x; c < gridDim.x; c += 32) {
                    unsigned v;
                    if (V == 2) asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + c * 32) : "memory");
                    else asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flags + c * 32) : "memory");
                    ok &= static_cast<int>(v - epoch) >= 0;
                }
                ok = __all_sync(0xffffffffu, ok);
            } while (!ok);
            if (V == 3) asm volatile("fence.acq_rel.gpu;" ::: "memory");
        }
    }
    __syncthreads();
}

template <int V>
__global__ void __launch_bounds__(896, 1) bk(unsigned* cnt, unsigned* flags, long long* out, int iters) {
    unsigned target = 0;
    long long t0 = 0;
    for (int i = 0; i < iters; ++i) {
        if (i == 4) { asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0)); }
        target += gridDim.x;
        gbar<V>(cnt, flags, target, static_cast<unsigned>(i + 1));
    }
    long long t1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
    if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}

template <int V>
void run(unsigned* cnt, unsigned* flags, long long* out) {
    cudaFuncSetAttribute(bk<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, 118784);
    int iters = 1004;
    for (int rep = 0; rep < 2; ++rep) {
        cudaMemset(cnt, 0, 64);
        cudaMemset(flags, 0, 148 * 128);
        void* args[] = {&cnt, &flags, &out, &iters};
        cudaLaunchCooperativeKernel((void*)bk<V>, 148, 896, args, 118784, 0);
        cudaDeviceSynchronize();
    }
    std::vector<long long> h(148);
    cudaMemcpy(h.data(), out, 148 * 8, cudaMemcpyDeviceToHost);
    std::sort(h.begin(), h.end());
    printf("{\"variant\": %d, \"ns_per_barrier\": %.1f, \"err\": \"%s\"}\n", V, h[74] / 1000.0, cudaGetErrorString(cudaGetLastError()));
}

int main() {
    unsigned *cnt, *flags; long long* out;
    cudaMalloc(&cnt, 64); cudaMalloc(&flags, 148 * 128); cudaMalloc(&out, 148 * 8);
    run<0>(cnt, flags, out); run<1>(cnt, flags, out); run<4>(cnt, flags, out); run<5>(cnt, flags, out);
    run<6>(cnt, flags, out); run<7>(cnt, flags, out); run<0>(cnt, flags, out);
    run<8>(cnt, flags, out); run<9>(cnt, flags, out); run<10>(cnt, flags, out);
    run<11>(cnt, flags, out); run<12>(cnt, flags, out); run<0>(cnt, flags, out); run<11>(cnt, flags, out);
    return 0;
}
