// abi.cu -- the extern "C" boundary of liblime.so (contract: include/lime.h).
//
// Host-side only: argument validation (in the documented order), device check, workspace
// check, then the launcher in the kernel translation unit. Validation never touches the
// GPU, so the error paths are testable on a machine without one.
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <atomic>
#include <map>
#include <mutex>
#include <tuple>

#include "../../include/lime.h"
#include "common.cuh"
#include "kernels.h"

namespace lime {

static thread_local char g_last_error[512] = "";
static thread_local LaunchOverride g_override;
static thread_local int g_nbody_variant = 0;

const LaunchOverride& launch_override() { return g_override; }
int nbody_variant() { return g_nbody_variant; }
bool pdl_enabled() {
    static const bool on = std::getenv("LIME_NO_PDL") == nullptr;
    return on;
}

cudaError_t ensure_dynamic_smem(const void* kernel, int bytes) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    static std::mutex mu;
    static std::map<std::pair<const void*, int>, int> set;     // (kernel, device) -> bytes allowed
    std::lock_guard<std::mutex> lock(mu);
    auto it = set.find({kernel, dev});
    if (it != set.end() && it->second >= bytes) return cudaSuccess;
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess) set[{kernel, dev}] = bytes;
    return e;
}

int cached_occupancy(const void* kernel, int block, size_t smem) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return 0; }
    static std::mutex mu;
    static std::map<std::tuple<const void*, int, size_t, int>, int> occ;
    std::lock_guard<std::mutex> lock(mu);
    const auto key = std::make_tuple(kernel, block, smem, dev);
    auto it = occ.find(key);
    if (it != occ.end()) return it->second;
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, block, smem) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    occ[key] = b;
    return b;
}

int device_num_sms() {
    static std::atomic<int> cached[64];   // zero-initialised (static storage)
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return kNumSMsB200;
    if (cached[dev] == 0) {
        int sms = 0;
        if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || sms <= 0) {
            cudaGetLastError();
            return kNumSMsB200;
        }
        cached[dev] = sms;
    }
    return cached[dev];
}

static lime_status fail(lime_status s, const char* fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_last_error, sizeof g_last_error, fmt, ap);
    va_end(ap);
    return s;
}

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
static bool overlap(const void* a, size_t abytes, const void* b, size_t bbytes) {
    if (abytes == 0 || bbytes == 0) return false;
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(a), b0 = reinterpret_cast<uintptr_t>(b);
    return a0 < b0 + bbytes && b0 < a0 + abytes;
}

static lime_status check_device() {
    static std::atomic<int> ok_cache[64];   // 0 unknown, 1 ok, 2 bad
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(LIME_ERR_UNSUPPORTED, "no CUDA device: %s", cudaGetErrorString(e));
    }
    if (dev >= 0 && dev < 64 && ok_cache[dev] == 1) return LIME_OK;
    int major = 0, minor = 0;
    cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
    if (major != 10 || minor != 0) {
        if (dev >= 0 && dev < 64) ok_cache[dev] = 2;
        return fail(LIME_ERR_UNSUPPORTED, "device %d is sm_%d%d; liblime is built for sm_100a (B200) only",
                    dev, major, minor);
    }
    if (dev >= 0 && dev < 64) ok_cache[dev] = 1;
    return LIME_OK;
}

static lime_status launched(cudaError_t e, const char* what) {
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(LIME_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
    }
    return LIME_OK;
}

}  // namespace lime

using namespace lime;

#define LIME_TRY(expr)                              \
    do {                                            \
        const lime_status s__ = (expr);             \
        if (s__ != LIME_OK) return s__;             \
    } while (0)

extern "C" {

int lime_abi_version(void) { return LIME_ABI_VERSION; }

const char* lime_status_str(int s) {
    switch (s) {
        case LIME_OK: return "LIME_OK";
        case LIME_ERR_INVALID_ARG: return "LIME_ERR_INVALID_ARG";
        case LIME_ERR_MISALIGNED: return "LIME_ERR_MISALIGNED";
        case LIME_ERR_ALIASING: return "LIME_ERR_ALIASING";
        case LIME_ERR_UNSUPPORTED: return "LIME_ERR_UNSUPPORTED";
        case LIME_ERR_CUDA: return "LIME_ERR_CUDA";
        case LIME_ERR_WORKSPACE: return "LIME_ERR_WORKSPACE";
        default: return "LIME_ERR_UNKNOWN";
    }
}

const char* lime_last_error(void) { return g_last_error; }

lime_status lime_device_check(void) { return check_device(); }

int lime_num_sms(void) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) {
        cudaGetLastError();
        return 0;
    }
    return device_num_sms();
}

void lime_set_launch_override(int grid_ctas, int block_threads, int per_thread) {
    g_override.grid_ctas = grid_ctas > 0 ? grid_ctas : 0;
    g_override.block_threads = block_threads > 0 ? block_threads : 0;
    g_override.per_thread = per_thread > 0 ? per_thread : 0;
}

int lime_set_nbody_variant(int variant) {
    if (variant < 0 || variant > 6) return LIME_ERR_INVALID_ARG;
    g_nbody_variant = variant;
    return LIME_OK;
}

// ============================================================================== N-Body
size_t lime_map_nbody_workspace_bytes(int64_t n_src, int64_t tgt_count) {
    if (n_src < 0 || tgt_count < 0) return 0;
    return nbody::workspace_bytes(n_src, tgt_count);
}

int lime_nbody_splits(int64_t n_src) { return n_src < 0 ? 0 : nbody::splits(n_src); }

lime_status lime_map_nbody(const float* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count,
                           float eps2, float* accel, void* ws, size_t ws_bytes, void* stream) {
    if (n_src < 0 || tgt_begin < 0 || tgt_count < 0 || tgt_begin > n_src || tgt_count > n_src - tgt_begin)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody: shard [%lld, %lld+%lld) outside [0, %lld)",
                    (long long)tgt_begin, (long long)tgt_begin, (long long)tgt_count, (long long)n_src);
    if (!(std::isfinite(eps2) && eps2 >= 1.17549435e-38f))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody: eps2 must be finite and >= FLT_MIN (got %g)", (double)eps2);
    if (tgt_count == 0) return LIME_OK;
    if (!bodies || !accel || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody: null pointer");
    if (!aligned16(bodies) || !aligned16(accel) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_nbody: bodies, accel and ws must be 16-byte aligned");
    if (overlap(accel, tgt_count * 16, bodies, n_src * 16))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody: accel overlaps bodies");
    if (overlap(ws, ws_bytes, bodies, n_src * 16) || overlap(ws, ws_bytes, accel, tgt_count * 16))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody: workspace overlaps an operand");
    LIME_TRY(check_device());
    const size_t need = nbody::workspace_bytes(n_src, tgt_count);
    if (ws_bytes < need)
        return fail(LIME_ERR_WORKSPACE, "lime_map_nbody: workspace %zu B < %zu B", ws_bytes, need);
    return launched(nbody::launch_force(reinterpret_cast<const float4*>(bodies), n_src, tgt_begin, tgt_count, eps2,
                                        reinterpret_cast<float4*>(accel), ws, static_cast<cudaStream_t>(stream)),
                    "lime_map_nbody");
}

size_t lime_map_nbody_f64_workspace_bytes(int64_t n_src, int64_t tgt_count) {
    if (n_src < 0 || tgt_count < 0) return 0;
    return nbody64::workspace_bytes(n_src, tgt_count);
}

lime_status lime_map_nbody_f64(const double* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, double eps2,
                               double* accel, void* ws, size_t ws_bytes, void* stream) {
    if (n_src < 0 || tgt_begin < 0 || tgt_count < 0 || tgt_begin > n_src || tgt_count > n_src - tgt_begin)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_f64: shard outside [0, n_src)");
    if (!(std::isfinite(eps2) && eps2 >= 2.2250738585072014e-308))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_f64: eps2 must be finite and >= DBL_MIN");
    if (tgt_count == 0) return LIME_OK;
    if (!bodies || !accel || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_f64: null pointer");
    if (!aligned16(bodies) || !aligned16(accel) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_nbody_f64: bodies, accel and ws must be 16-byte aligned");
    if (overlap(accel, tgt_count * 32, bodies, n_src * 32) || overlap(ws, ws_bytes, bodies, n_src * 32) ||
        overlap(ws, ws_bytes, accel, tgt_count * 32))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody_f64: output/workspace overlap");
    LIME_TRY(check_device());
    if (ws_bytes < nbody64::workspace_bytes(n_src, tgt_count))
        return fail(LIME_ERR_WORKSPACE, "lime_map_nbody_f64: workspace too small");
    return launched(nbody64::launch_force(bodies, n_src, tgt_begin, tgt_count, eps2, accel, ws,
                                          static_cast<cudaStream_t>(stream)),
                    "lime_map_nbody_f64");
}

lime_status lime_map_nbody_integrate(float* pos, float* vel, const float* accel, int64_t n, float dt, void* stream) {
    if (n < 0) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_integrate: n < 0");
    if (!std::isfinite(dt)) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_integrate: dt not finite");
    if (n == 0) return LIME_OK;
    if (!pos || !vel || !accel) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_integrate: null pointer");
    if (!aligned16(pos) || !aligned16(vel) || !aligned16(accel))
        return fail(LIME_ERR_MISALIGNED, "lime_map_nbody_integrate: operands must be 16-byte aligned");
    const size_t b = static_cast<size_t>(n) * 16;
    if (overlap(pos, b, vel, b) || overlap(accel, b, pos, b) || overlap(accel, b, vel, b))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody_integrate: pos, vel and accel must be disjoint");
    LIME_TRY(check_device());
    return launched(nbody::launch_integrate(reinterpret_cast<float4*>(pos), reinterpret_cast<float4*>(vel),
                                            reinterpret_cast<const float4*>(accel), n, dt,
                                            static_cast<cudaStream_t>(stream)),
                    "lime_map_nbody_integrate");
}

size_t lime_map_nbody_step_workspace_bytes(int64_t n_src, int64_t tgt_count) {
    if (n_src < 0 || tgt_count < 0) return 0;
    return nbody::step_workspace_bytes(n_src, tgt_count);
}

lime_status lime_map_nbody_step(const float* bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count, float eps2,
                                float dt, float* vel, float* pos_out, void* ws, size_t ws_bytes, void* stream) {
    if (n_src < 0 || tgt_begin < 0 || tgt_count < 0 || tgt_begin > n_src || tgt_count > n_src - tgt_begin)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_step: shard [%lld, %lld+%lld) outside [0, %lld)",
                    (long long)tgt_begin, (long long)tgt_begin, (long long)tgt_count, (long long)n_src);
    if (!(std::isfinite(eps2) && eps2 >= 1.17549435e-38f) || !std::isfinite(dt))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_step: eps2 must be finite and >= FLT_MIN, dt finite");
    if (tgt_count == 0) return LIME_OK;
    if (!bodies || !vel || !pos_out || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_nbody_step: null pointer");
    if (!aligned16(bodies) || !aligned16(vel) || !aligned16(pos_out) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_nbody_step: bodies, vel, pos_out and ws must be 16-byte aligned");
    const size_t tb = static_cast<size_t>(tgt_count) * 16, nb = static_cast<size_t>(n_src) * 16;
    if (overlap(pos_out, tb, bodies, nb) || overlap(vel, tb, bodies, nb) || overlap(vel, tb, pos_out, tb))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody_step: bodies, vel and pos_out must be disjoint");
    if (overlap(ws, ws_bytes, bodies, nb) || overlap(ws, ws_bytes, vel, tb) || overlap(ws, ws_bytes, pos_out, tb))
        return fail(LIME_ERR_ALIASING, "lime_map_nbody_step: workspace overlaps an operand");
    LIME_TRY(check_device());
    const size_t need = nbody::step_workspace_bytes(n_src, tgt_count);
    if (ws_bytes < need) return fail(LIME_ERR_WORKSPACE, "lime_map_nbody_step: workspace %zu B < %zu B", ws_bytes, need);
    return launched(nbody::launch_step(reinterpret_cast<const float4*>(bodies), n_src, tgt_begin, tgt_count, eps2, dt,
                                       reinterpret_cast<float4*>(vel), reinterpret_cast<float4*>(pos_out), ws,
                                       static_cast<cudaStream_t>(stream)),
                    "lime_map_nbody_step");
}

static lime_status sim_validate(const char* fn, int64_t n, int32_t steps, float eps2, float dt) {
    if (n < 0 || steps < 0) return fail(LIME_ERR_INVALID_ARG, "%s: n or steps < 0", fn);
    if (!(std::isfinite(eps2) && eps2 >= 1.17549435e-38f) || !std::isfinite(dt))
        return fail(LIME_ERR_INVALID_ARG, "%s: bad eps2 or dt", fn);
    return LIME_OK;
}

size_t lime_nbody_simulate_workspace_bytes(int64_t n) {
    if (n < 0) return 0;
    return nbody::simulate_workspace_bytes(n);
}

lime_status lime_nbody_simulate(float* pos, float* vel, int64_t n, int32_t steps, float eps2, float dt, void* ws,
                                size_t ws_bytes, void* stream) {
    LIME_TRY(sim_validate("lime_nbody_simulate", n, steps, eps2, dt));
    if (n == 0) return LIME_OK;
    if (!pos || !vel || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_nbody_simulate: null pointer");
    if (!aligned16(pos) || !aligned16(vel) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_nbody_simulate: pos, vel, ws must be 16-byte aligned");
    const size_t b = static_cast<size_t>(n) * 16;
    if (overlap(pos, b, vel, b) || overlap(ws, ws_bytes, pos, b) || overlap(ws, ws_bytes, vel, b))
        return fail(LIME_ERR_ALIASING, "lime_nbody_simulate: pos, vel and ws must be disjoint");
    LIME_TRY(check_device());
    if (ws_bytes < lime_nbody_simulate_workspace_bytes(n))
        return fail(LIME_ERR_WORKSPACE, "lime_nbody_simulate: workspace too small");
    return launched(nbody::launch_simulate(reinterpret_cast<float4*>(pos), reinterpret_cast<float4*>(vel), n, steps,
                                           eps2, dt, ws, static_cast<cudaStream_t>(stream)),
                    "lime_nbody_simulate");
}

// ws layout: [simulate workspace (zero-invariant words at fixed offsets)][pos n*16][vel n*16]
static size_t sim_host_state_offset(int64_t n) { return ((nbody::simulate_workspace_bytes(n) + 255) / 256) * 256; }
size_t lime_nbody_simulate_host_workspace_bytes(int64_t n) {
    if (n < 0) return 0;
    return sim_host_state_offset(n) + static_cast<size_t>(n) * 32;
}

lime_status lime_nbody_simulate_host(float* h_pos, float* h_vel, int64_t n, int32_t steps, float eps2, float dt,
                                     void* ws, size_t ws_bytes, void* stream) {
    LIME_TRY(sim_validate("lime_nbody_simulate_host", n, steps, eps2, dt));
    if (n == 0) return LIME_OK;
    if (!h_pos || !h_vel || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_nbody_simulate_host: null pointer");
    if (!aligned16(ws)) return fail(LIME_ERR_MISALIGNED, "lime_nbody_simulate_host: ws must be 16-byte aligned");
    const size_t b = static_cast<size_t>(n) * 16;
    if (overlap(h_pos, b, h_vel, b)) return fail(LIME_ERR_ALIASING, "lime_nbody_simulate_host: h_pos overlaps h_vel");
    LIME_TRY(check_device());
    if (ws_bytes < lime_nbody_simulate_host_workspace_bytes(n))
        return fail(LIME_ERR_WORKSPACE, "lime_nbody_simulate_host: workspace too small");
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    char* w = static_cast<char*>(ws);
    void* d_ws = w;
    float4* d_pos = reinterpret_cast<float4*>(w + sim_host_state_offset(n));
    float4* d_vel = reinterpret_cast<float4*>(w + sim_host_state_offset(n) + b);
    cudaError_t e = cudaMemcpyAsync(d_pos, h_pos, b, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(d_vel, h_vel, b, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = nbody::launch_simulate(d_pos, d_vel, n, steps, eps2, dt, d_ws, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(h_pos, d_pos, b, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(h_vel, d_vel, b, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    return launched(e, "lime_nbody_simulate_host");
}

// ======================================================================= Black-Scholes
static lime_status bs_validate(const char* fn, const float* S, const float* X, const float* T, int64_t n,
                               float r, float sigma) {
    if (n < 0) return fail(LIME_ERR_INVALID_ARG, "%s: n < 0", fn);
    if (!std::isfinite(r) || !(sigma > 0.f) || !std::isfinite(sigma))
        return fail(LIME_ERR_INVALID_ARG, "%s: r must be finite and sigma finite and > 0", fn);
    if (n > 0 && (!S || !X || !T)) return fail(LIME_ERR_INVALID_ARG, "%s: null input", fn);
    if (n > 0 && (!aligned16(S) || !aligned16(X) || !aligned16(T)))
        return fail(LIME_ERR_MISALIGNED, "%s: S, X, T must be 16-byte aligned", fn);
    return LIME_OK;
}

lime_status lime_map_blackscholes(const float* S, const float* X, const float* T, int64_t n, float r, float sigma,
                                  float* call, float* put, void* stream) {
    LIME_TRY(bs_validate("lime_map_blackscholes", S, X, T, n, r, sigma));
    if (n == 0) return LIME_OK;
    if (!call || !put) return fail(LIME_ERR_INVALID_ARG, "lime_map_blackscholes: null output");
    if (!aligned16(call) || !aligned16(put))
        return fail(LIME_ERR_MISALIGNED, "lime_map_blackscholes: call, put must be 16-byte aligned");
    const size_t b = static_cast<size_t>(n) * 4;
    for (const void* in : {static_cast<const void*>(S), static_cast<const void*>(X), static_cast<const void*>(T)})
        if (overlap(call, b, in, b) || overlap(put, b, in, b))
            return fail(LIME_ERR_ALIASING, "lime_map_blackscholes: an output overlaps an input");
    if (overlap(call, b, put, b)) return fail(LIME_ERR_ALIASING, "lime_map_blackscholes: call overlaps put");
    LIME_TRY(check_device());
    return launched(bs::launch_map(S, X, T, n, r, sigma, call, put, static_cast<cudaStream_t>(stream)),
                    "lime_map_blackscholes");
}

lime_status lime_map_reduce_blackscholes_sum(const float* S, const float* X, const float* T, int64_t n, float r,
                                             float sigma, double* sums, void* ws, size_t ws_bytes, void* stream) {
    LIME_TRY(bs_validate("lime_map_reduce_blackscholes_sum", S, X, T, n, r, sigma));
    if (!sums || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_reduce_blackscholes_sum: null sums or ws");
    if (!aligned16(ws)) return fail(LIME_ERR_MISALIGNED, "lime_map_reduce_blackscholes_sum: ws must be 16-byte aligned");
    const size_t b = static_cast<size_t>(n) * 4;
    for (const void* in : {static_cast<const void*>(S), static_cast<const void*>(X), static_cast<const void*>(T)})
        if (overlap(sums, 16, in, b) || overlap(ws, ws_bytes, in, b))
            return fail(LIME_ERR_ALIASING, "lime_map_reduce_blackscholes_sum: sums/ws overlap an input");
    if (overlap(sums, 16, ws, ws_bytes)) return fail(LIME_ERR_ALIASING, "lime_map_reduce_blackscholes_sum: sums overlaps ws");
    LIME_TRY(check_device());
    if (ws_bytes < red::kWorkspaceBytes)
        return fail(LIME_ERR_WORKSPACE, "lime_map_reduce_blackscholes_sum: workspace %zu B < %zu B", ws_bytes,
                    red::kWorkspaceBytes);
    return launched(bs::launch_map_reduce(S, X, T, n, r, sigma, sums, ws, static_cast<cudaStream_t>(stream)),
                    "lime_map_reduce_blackscholes_sum");
}

// ========================================================================== Mandelbrot
size_t lime_mandelbrot_workspace_bytes(void) { return mandel::kWorkspaceBytes; }

lime_status lime_map_mandelbrot(int32_t width, int32_t height, int32_t row_first, int32_t row_stride,
                                int32_t row_count, float x0, float y0, float dx, float dy, int32_t max_iter,
                                int32_t* counts, void* ws, size_t ws_bytes, void* stream) {
    if (width <= 0 || height <= 0 || row_stride < 1 || row_count < 0 || row_first < 0 || row_first >= height ||
        max_iter < 0)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_mandelbrot: bad geometry or max_iter");
    if (row_count > 0 && static_cast<int64_t>(row_first) + static_cast<int64_t>(row_count - 1) * row_stride >= height)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_mandelbrot: addressed rows exceed height");
    if (!std::isfinite(x0) || !std::isfinite(y0) || !std::isfinite(dx) || !std::isfinite(dy))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_mandelbrot: non-finite region");
    if (row_count == 0) return LIME_OK;
    if (!counts || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_mandelbrot: null pointer");
    if ((reinterpret_cast<uintptr_t>(counts) & 3u) != 0 || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_mandelbrot: counts must be 4-B and ws 16-B aligned");
    if (overlap(counts, static_cast<size_t>(row_count) * width * 4, ws, ws_bytes))
        return fail(LIME_ERR_ALIASING, "lime_map_mandelbrot: counts overlaps ws");
    LIME_TRY(check_device());
    if (ws_bytes < mandel::kWorkspaceBytes) return fail(LIME_ERR_WORKSPACE, "lime_map_mandelbrot: workspace too small");
    return launched(mandel::launch(width, row_first, row_stride, row_count, x0, y0, dx, dy, max_iter, counts, ws,
                                   static_cast<cudaStream_t>(stream)),
                    "lime_map_mandelbrot");
}

// ======================================================================= Parboil CP / MRI-Q
size_t lime_map_coulomb_workspace_bytes(int64_t n_atoms, int64_t p_count) {
    if (n_atoms < 0 || p_count < 0) return 0;
    return parboil::cp_workspace_bytes(n_atoms, p_count);
}

lime_status lime_map_coulomb(const float* atoms, int64_t n_atoms, int32_t nx, int32_t ny, int64_t p_begin,
                             int64_t p_count, float z, float h, float* V, void* ws, size_t ws_bytes, void* stream) {
    const int64_t np = static_cast<int64_t>(nx) * ny;
    if (n_atoms < 0 || nx < 1 || ny < 1 || p_begin < 0 || p_count < 0 || p_begin > np || p_count > np - p_begin)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_coulomb: bad sizes or shard");
    if (!std::isfinite(z) || !std::isfinite(h) || !(h > 0.f))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_coulomb: z must be finite and h finite and > 0");
    if (p_count == 0) return LIME_OK;
    if ((n_atoms > 0 && !atoms) || !V || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_coulomb: null pointer");
    if ((n_atoms > 0 && !aligned16(atoms)) || (reinterpret_cast<uintptr_t>(V) & 3u) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_coulomb: atoms/ws 16-B, V 4-B aligned");
    if (overlap(V, p_count * 4, atoms, n_atoms * 16) || overlap(ws, ws_bytes, atoms, n_atoms * 16) ||
        overlap(ws, ws_bytes, V, p_count * 4))
        return fail(LIME_ERR_ALIASING, "lime_map_coulomb: output/workspace overlap");
    LIME_TRY(check_device());
    if (ws_bytes < parboil::cp_workspace_bytes(n_atoms, p_count))
        return fail(LIME_ERR_WORKSPACE, "lime_map_coulomb: workspace too small");
    return launched(parboil::launch_cp(reinterpret_cast<const float4*>(atoms), n_atoms, nx, p_begin, p_count, z, h, V,
                                       ws, static_cast<cudaStream_t>(stream)),
                    "lime_map_coulomb");
}

size_t lime_map_mriq_workspace_bytes(int64_t n_k, int64_t x_count) {
    if (n_k < 0 || x_count < 0) return 0;
    return parboil::mriq_workspace_bytes(n_k, x_count);
}

lime_status lime_map_mriq(const float* kspace, int64_t n_k, const float* voxels, int64_t n_x, int64_t x_begin,
                          int64_t x_count, float* Q, void* ws, size_t ws_bytes, void* stream) {
    if (n_k < 0 || n_x < 0 || x_begin < 0 || x_count < 0 || x_begin > n_x || x_count > n_x - x_begin)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_mriq: bad sizes or shard");
    if (x_count == 0) return LIME_OK;
    if ((n_k > 0 && !kspace) || !voxels || !Q || !ws) return fail(LIME_ERR_INVALID_ARG, "lime_map_mriq: null pointer");
    if ((reinterpret_cast<uintptr_t>(kspace) & 3u) || (reinterpret_cast<uintptr_t>(voxels) & 3u) ||
        (reinterpret_cast<uintptr_t>(Q) & 7u) || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "lime_map_mriq: kspace/voxels 4-B, Q 8-B, ws 16-B aligned");
    const size_t qb = static_cast<size_t>(x_count) * 8;
    if (overlap(Q, qb, kspace, n_k * 20) || overlap(Q, qb, voxels, n_x * 12) || overlap(ws, ws_bytes, kspace, n_k * 20) ||
        overlap(ws, ws_bytes, voxels, n_x * 12) || overlap(ws, ws_bytes, Q, qb))
        return fail(LIME_ERR_ALIASING, "lime_map_mriq: output/workspace overlap");
    LIME_TRY(check_device());
    if (ws_bytes < parboil::mriq_workspace_bytes(n_k, x_count))
        return fail(LIME_ERR_WORKSPACE, "lime_map_mriq: workspace too small");
    return launched(parboil::launch_mriq(kspace, n_k, voxels, x_begin, x_count, Q, ws, static_cast<cudaStream_t>(stream)),
                    "lime_map_mriq");
}

// ========================================================================= JG-Series / JG-Crypt
size_t lime_map_series_workspace_bytes(void) { return jgf::series_workspace_bytes(true); }

static lime_status series_entry(const char* fn, int64_t n0, int64_t count, void* out, size_t esz, void* ws,
                                size_t ws_bytes, void* stream) {
    if (n0 < 0 || count < 0 || n0 > (1LL << 40) || count > (1LL << 40))
        return fail(LIME_ERR_INVALID_ARG, "%s: n0, count must be in [0, 2^40]", fn);
    if (count == 0) return LIME_OK;
    if (!out || !ws) return fail(LIME_ERR_INVALID_ARG, "%s: null pointer", fn);
    if ((reinterpret_cast<uintptr_t>(out) % esz) != 0 || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "%s: out needs natural alignment, ws 16-B", fn);
    if (overlap(out, static_cast<size_t>(count) * 2 * esz, ws, ws_bytes))
        return fail(LIME_ERR_ALIASING, "%s: out overlaps ws", fn);
    LIME_TRY(check_device());
    if (ws_bytes < jgf::series_workspace_bytes(esz == 8)) return fail(LIME_ERR_WORKSPACE, "%s: workspace too small", fn);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    return launched(esz == 8 ? jgf::launch_series_f64(n0, count, static_cast<double*>(out), ws, s)
                             : jgf::launch_series_f32(n0, count, static_cast<float*>(out), ws, s),
                    fn);
}

lime_status lime_map_series_f32(int64_t n0, int64_t count, float* out, void* ws, size_t ws_bytes, void* stream) {
    return series_entry("lime_map_series_f32", n0, count, out, 4, ws, ws_bytes, stream);
}

lime_status lime_map_series_f64(int64_t n0, int64_t count, double* out, void* ws, size_t ws_bytes, void* stream) {
    return series_entry("lime_map_series_f64", n0, count, out, 8, ws, ws_bytes, stream);
}

void lime_idea_key_schedule(const uint16_t* key, uint16_t* ek, uint16_t* dk) {
    if (!key || !ek || !dk) return;
    jgf::idea_key_schedule(key, ek, dk);
}

lime_status lime_map_idea(const uint8_t* in, uint8_t* out, int64_t nbytes, const uint16_t* subkeys, void* stream) {
    if (nbytes < 0 || (nbytes % 8) != 0) return fail(LIME_ERR_INVALID_ARG, "lime_map_idea: nbytes must be a multiple of 8");
    if (nbytes == 0) return LIME_OK;
    if (!in || !out || !subkeys) return fail(LIME_ERR_INVALID_ARG, "lime_map_idea: null pointer");
    if (!aligned16(in) || !aligned16(out)) return fail(LIME_ERR_MISALIGNED, "lime_map_idea: in/out must be 16-byte aligned");
    if (overlap(in, nbytes, out, nbytes)) return fail(LIME_ERR_ALIASING, "lime_map_idea: out overlaps in");
    LIME_TRY(check_device());
    return launched(jgf::launch_idea(in, out, nbytes, subkeys, static_cast<cudaStream_t>(stream)), "lime_map_idea");
}

// ============================================================================== Matmul
lime_status lime_map_matmul_bf16(const uint16_t* A, const uint16_t* Bt, float* C, int64_t M, int64_t N, int64_t K,
                                 void* stream) {
    if (M < 1 || N < 1 || K < 8 || (K % 8) != 0)
        return fail(LIME_ERR_INVALID_ARG, "lime_map_matmul_bf16: need M, N >= 1 and K >= 8, K %% 8 == 0");
    // the kernels index rows, TMA coordinates and tiles in int32: every padded dimension and the
    // tile count must stay below 2^31
    constexpr int64_t kDimMax = (1LL << 31) - 512;
    if (M > kDimMax || N > kDimMax || K > kDimMax ||
        ((M + 255) / 256) * ((N + 255) / 256) > static_cast<int64_t>(INT32_MAX))
        return fail(LIME_ERR_INVALID_ARG, "lime_map_matmul_bf16: dimension or tile count exceeds the int32 range");
    if (!A || !Bt || !C) return fail(LIME_ERR_INVALID_ARG, "lime_map_matmul_bf16: null pointer");
    if (!aligned16(A) || !aligned16(Bt) || !aligned16(C))
        return fail(LIME_ERR_MISALIGNED, "lime_map_matmul_bf16: A, Bt, C must be 16-byte aligned");
    const size_t cb = static_cast<size_t>(M) * N * 4;
    if (overlap(C, cb, A, static_cast<size_t>(M) * K * 2) || overlap(C, cb, Bt, static_cast<size_t>(N) * K * 2))
        return fail(LIME_ERR_ALIASING, "lime_map_matmul_bf16: C overlaps an input");
    LIME_TRY(check_device());
    cudaError_t e = gemm::launch_bf16(A, Bt, C, M, N, K, static_cast<cudaStream_t>(stream));
    if (e == cudaErrorNotSupported) return fail(LIME_ERR_UNSUPPORTED, "lime_map_matmul_bf16: not supported");
    return launched(e, "lime_map_matmul_bf16");
}

// ========================================================================== Reductions
size_t lime_reduce_workspace_bytes(void) { return red::kWorkspaceBytes; }

static lime_status reduce_entry(const char* fn, red::Op op, red::Dt dt, size_t esz, const void* x, int64_t n,
                                void* out, size_t osz, void* ws, size_t ws_bytes, void* stream) {
    if (n < 0) return fail(LIME_ERR_INVALID_ARG, "%s: n < 0", fn);
    if ((n > 0 && !x) || !out || !ws) return fail(LIME_ERR_INVALID_ARG, "%s: null pointer", fn);
    if ((reinterpret_cast<uintptr_t>(x) % esz) != 0 || (reinterpret_cast<uintptr_t>(out) % osz) != 0 || !aligned16(ws))
        return fail(LIME_ERR_MISALIGNED, "%s: x/out need natural alignment, ws 16-B", fn);
    const size_t xb = static_cast<size_t>(n) * esz;
    if (overlap(out, osz, x, xb) || overlap(ws, ws_bytes, x, xb) || overlap(ws, ws_bytes, out, osz))
        return fail(LIME_ERR_ALIASING, "%s: out/ws overlap", fn);
    LIME_TRY(check_device());
    if (ws_bytes < red::kWorkspaceBytes) return fail(LIME_ERR_WORKSPACE, "%s: workspace too small", fn);
    return launched(red::launch(op, dt, x, n, out, ws, static_cast<cudaStream_t>(stream)), fn);
}

#define LIME_REDUCE_ENTRY(OPN, OPE, DTN, DTE, T)                                                            \
    lime_status lime_reduce_##OPN##_##DTN(const T* x, int64_t n, T* out, void* ws, size_t ws_bytes,         \
                                          void* stream) {                                                   \
        return reduce_entry("lime_reduce_" #OPN "_" #DTN, OPE, DTE, sizeof(T), x, n, out, sizeof(T), ws,    \
                            ws_bytes, stream);                                                              \
    }
LIME_REDUCE_ENTRY(sum, red::kSum, f32, red::kF32, float)
LIME_REDUCE_ENTRY(sum, red::kSum, f64, red::kF64, double)
LIME_REDUCE_ENTRY(sum, red::kSum, i32, red::kI32, int32_t)
LIME_REDUCE_ENTRY(sum, red::kSum, i64, red::kI64, int64_t)
LIME_REDUCE_ENTRY(min, red::kMin, f32, red::kF32, float)
LIME_REDUCE_ENTRY(min, red::kMin, f64, red::kF64, double)
LIME_REDUCE_ENTRY(min, red::kMin, i32, red::kI32, int32_t)
LIME_REDUCE_ENTRY(min, red::kMin, i64, red::kI64, int64_t)
LIME_REDUCE_ENTRY(max, red::kMax, f32, red::kF32, float)
LIME_REDUCE_ENTRY(max, red::kMax, f64, red::kF64, double)
LIME_REDUCE_ENTRY(max, red::kMax, i32, red::kI32, int32_t)
LIME_REDUCE_ENTRY(max, red::kMax, i64, red::kI64, int64_t)
#undef LIME_REDUCE_ENTRY

}  // extern "C"
