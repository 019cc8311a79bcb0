/*
 * lime.h -- C ABI of liblime.so, the B200-native (sm_100a) map `@` / reduce `!`
 * hot path of Lime (Dubach, Cheng, Rabbah, Bacon, Fink, PLDI 2012).
 *
 * Citations Lnnn are lines of the decoded `fulltext` of PAPER.md.
 *
 * ---------------------------------------------------------------------------
 * Conventions (apply to every entry point unless its comment says otherwise)
 * ---------------------------------------------------------------------------
 * Semantics. A map `@` applies a pure element function to each element of an
 *   immutable value array and returns a NEW array (L149-157 §3.2; purity from
 *   "static and local" + value-typed arguments, L184-189). A reduce `!`
 *   combines elements with a binary combinator of one type (L160-163). Every
 *   map here computes out[t] = f(in[begin + t], broadcast operands) for
 *   t in [0, count); the result does not depend on how many threads run it
 *   (L205-208).
 * Pointers. Unless the name ends in `_host`, every array pointer is a DEVICE
 *   pointer (e.g. a torch CUDA tensor's data_ptr()) owned by the caller. The
 *   library keeps no pointer after returning and allocates/frees nothing.
 * Layout. Dense row-major arrays of primitives (L297-301). float4 operands and
 *   `*_workspace` buffers must be 16-byte aligned.
 * Value semantics. Inputs are never written (L136-143); an output range that
 *   overlaps an input range is rejected with LIME_ERR_ALIASING. The integrator
 *   is the documented exception (in/out state; it is the paper's stateful sink
 *   task, L112-113, not a filter).
 * Streams. `stream` is a cudaStream_t passed as void* (NULL = legacy default
 *   stream). All work is enqueued asynchronously on it; the library never
 *   synchronises, except `_host` entry points, which synchronise `stream`
 *   before returning (their outputs are host memory). The streaming kernels
 *   (Black-Scholes, reductions, the small N-Body map, the integrator) are
 *   launched with programmatic dependent launch: their first instruction waits
 *   until every earlier grid on the stream has completed and its writes are
 *   visible, so stream order is unchanged; only the launch itself overlaps the
 *   previous grid's drain. Setting LIME_NO_PDL in the environment disables it.
 * Workspaces. Entry points taking (ws, ws_bytes) need a device scratch buffer
 *   of at least the size returned by the matching *_workspace_bytes() query,
 *   ZERO-FILLED before its first use; every call leaves every word a later
 *   call relies on zero again (self-resetting counters; split partials are
 *   re-zeroed by the CTA that consumes them, and lime_map_nbody zeroes its own
 *   tickets in a prepass), so one buffer can be reused by consecutive calls of
 *   ANY sizes on the same stream. Two calls that run concurrently need two
 *   workspaces.
 * Errors. Every entry point returns lime_status; no C++ exception crosses the
 *   ABI. Validation order: arguments (LIME_ERR_INVALID_ARG) -> alignment
 *   (LIME_ERR_MISALIGNED) -> aliasing (LIME_ERR_ALIASING) -> device check
 *   (LIME_ERR_UNSUPPORTED: current device is not compute capability 10.0)
 *   -> workspace size (LIME_ERR_WORKSPACE) -> launch (LIME_ERR_CUDA from
 *   cudaGetLastError). Nothing is enqueued when a non-OK status is returned.
 *   Faults inside asynchronous work surface at the next synchronisation, as
 *   in CUDA. lime_last_error() gives a thread-local message for the last
 *   non-OK status. Count 0 is a valid no-op for maps.
 */
#ifndef LIME_H
#define LIME_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    LIME_OK = 0,
    LIME_ERR_INVALID_ARG = 1,
    LIME_ERR_MISALIGNED = 2,
    LIME_ERR_ALIASING = 3,
    LIME_ERR_UNSUPPORTED = 4,
    LIME_ERR_CUDA = 5,
    LIME_ERR_WORKSPACE = 6
} lime_status;

#define LIME_ABI_VERSION 1

/* ABI version (LIME_ABI_VERSION). */
int lime_abi_version(void);
/* Static string naming a status code. */
const char *lime_status_str(int status);
/* Thread-local detail for the last non-OK status returned on this thread ("" if none). */
const char *lime_last_error(void);
/* LIME_OK iff the current CUDA device is an sm_100 part (B200); else LIME_ERR_UNSUPPORTED. */
lime_status lime_device_check(void);
/* Number of SMs of the current device (0 if no device). */
int lime_num_sms(void);
/* Test/tuning hook (paper L204-205 "number of threads ... requested by the user", L380-385
 * offline tuning): override the launch configuration of the next calls on this thread.
 * grid_ctas = 0 / block_threads = 0 / per_thread = 0 restore the automatic choice. Each
 * kernel documents which knobs it honours; results of maps never depend on them. */
void lime_set_launch_override(int grid_ctas, int block_threads, int per_thread);

/* ===========================================================================
 * N-Body all-pairs force map (the paper's workload: L106-114 task graph,
 * L108-112 float[[][4]] particles -> per-particle force, L156-158 "each
 * application of the map function computes the force interactions between a
 * particle p and all other particles", L173-174 "n^2 force calculation").
 * Formula (paper omits it, L157-158; R1-R3):
 *   accel[t] = sum_{j=0}^{n_src-1} m_j (p_j - p_i) (|p_j - p_i|^2 + eps2)^{-3/2},
 *   i = tgt_begin + t, G = 1, self term included (exactly 0).
 *   bodies  [n_src][4] float (x, y, z, m), 16-B aligned  -- the mapped array AND
 *           the broadcast operand staged through shared memory (L234-255).
 *   accel   [tgt_count][4] float (ax, ay, az, 0), 16-B aligned, must not
 *           overlap bodies.
 *   eps2    Plummer softening, finite and > 0 (eps2 <= 0 makes the self term 0/0).
 *   0 <= tgt_begin, 0 <= tgt_count, tgt_begin + tgt_count <= n_src.
 * Summation order (deterministic, independent of launch config and of the
 * target shard): sources are cut into chunks (64 bodies when n_src <= 8192,
 * else 256); each chunk is summed in j order into a chunk partial; chunk
 * partials are added in order into one of S = nbody_splits(n_src) split
 * partials (S <= 64 when n_src <= 8192, else <= 32); split partials are added
 * as a pairwise tree over next_pow2(S) leaves when n_src <= 8192, else in s
 * order (R11).
 * Mass-uniform splits (n_src > 8192; R11): when every body of a
 * split has the same mass m (bitwise-equal floats), each chunk partial is
 * sum_j (p_j - p_i) / R^3 and is added as m * partial (exact algebra, one fewer
 * FP32 multiply per interaction); for a power-of-two m this rounds exactly like
 * the per-body form. A prepass kernel computes the per-chunk flags (and zeroes
 * the split tickets) on `stream` before the force kernels.
 * Range: the self term needs (eps2)^{-3/2} * max(m_j, 1) finite in fp32.
 * Launch override: grid ignored; block_threads in {128, 256} with per_thread in {1, 2, 4, 8},
 * or block_threads 512 with per_thread in {2, 4}.
 * =========================================================================== */
size_t lime_map_nbody_workspace_bytes(int64_t n_src, int64_t tgt_count);
/* Staging ablation (the paper's Fig. 8 memory-mapping variants, L391-398,
 * and "any of the optimizations [can] be enabled and disabled", L212-216): selects, for the
 * following lime_map_nbody calls on this thread, where the broadcast source array is read from:
 * 0 = production kernels (TMA-staged shared memory), 1 = global scalar loads, 2 = global 128-bit
 * loads, 3 = read-only (non-coherent) 128-bit loads, 4 = shared memory copied by threads, scalar
 * reads, 5 = shared memory copied by threads, 128-bit reads, 6 = __constant__ memory (n_src <=
 * 4096; includes a 64-KB device-to-device copy per call). Results are bit-identical for every
 * variant. Returns LIME_ERR_INVALID_ARG for an unknown variant. */
int lime_set_nbody_variant(int variant);
int lime_nbody_splits(int64_t n_src);
lime_status lime_map_nbody(const float *bodies, int64_t n_src, int64_t tgt_begin,
                           int64_t tgt_count, float eps2, float *accel,
                           void *ws, size_t ws_bytes, void *stream);

/* Double-precision N-Body force map (Table 3 "N-Body
 * ... Float / Double", L319-323, L372-373): the same map on bodies
 * [n_src][4] double (x, y, z, m) -> accel [tgt_count][4] double (ax, ay, az, 0),
 * eps2 finite and >= DBL_MIN; pointers 16-B aligned; same shard rules and the
 * same split summation order as lime_map_nbody. The inverse square root is the
 * MUFU approximation refined to full double precision.
 * ws: lime_map_nbody_f64_workspace_bytes(n_src, tgt_count) bytes, zeroed once. */
size_t lime_map_nbody_f64_workspace_bytes(int64_t n_src, int64_t tgt_count);
lime_status lime_map_nbody_f64(const double *bodies, int64_t n_src, int64_t tgt_begin,
                               int64_t tgt_count, double eps2, double *accel,
                               void *ws, size_t ws_bytes, void *stream);

/* N-Body integrator (the `forceAccumulator` sink, L112-114; R4):
 * semi-implicit Euler on n bodies, in place:
 *   vel.xyz += accel.xyz * dt ;  pos.xyz += vel.xyz * dt ;  pos.w (mass), vel.w kept.
 * pos, vel, accel: [n][4] float, 16-B aligned; accel must not overlap pos/vel;
 * pos and vel must not overlap each other. dt finite.
 * Launch override: grid_ctas honoured. */
lime_status lime_map_nbody_integrate(float *pos, float *vel, const float *accel, int64_t n,
                                     float dt, void *stream);

/* One N-Body step of a target shard with the integrator fused into the force map
 * (the task graph's `computeForces => forceAccumulator` edge, PAPER.md L106-114;
 * A9): for t in [0, tgt_count), with a_t the acceleration lime_map_nbody computes
 * for target tgt_begin + t against all n_src bodies and p_t = bodies[tgt_begin + t],
 *   vel[t].xyz += a_t.xyz * dt ;  pos_out[t] = p_t with .xyz += vel[t].xyz * dt
 * (pos_out.w = p_t.w, vel.w kept) -- bit-identical to lime_map_nbody followed by
 * lime_map_nbody_integrate on the shard, without materialising the accelerations
 * (n_src <= 8192: one launch; larger: force map into ws, then the integrator).
 * bodies [n_src][4], vel and pos_out [tgt_count][4] float, device, 16-B aligned,
 * pairwise disjoint (pos_out is written out of place: the map reads every body).
 * ws: lime_map_nbody_step_workspace_bytes(n_src, tgt_count) bytes, zeroed once.
 * Errors as lime_map_nbody, plus LIME_ERR_ALIASING for overlapping vel/pos_out. */
size_t lime_map_nbody_step_workspace_bytes(int64_t n_src, int64_t tgt_count);
lime_status lime_map_nbody_step(const float *bodies, int64_t n_src, int64_t tgt_begin,
                                int64_t tgt_count, float eps2, float dt, float *vel,
                                float *pos_out, void *ws, size_t ws_bytes, void *stream);

/* `steps` complete N-Body simulation steps on DEVICE buffers (the paper's task
 * graph run repeatedly, `particles => computeForces => forceAccumulator`,
 * PAPER.md L106-114; its 4096-body size, Table 3): per step the force map
 * over all n targets against all n sources, then the integrator, with results
 * bit-identical to `steps` x (lime_map_nbody(pos, n, 0, n, ...) +
 * lime_map_nbody_integrate). pos, vel: [n][4] float, device, 16-B aligned,
 * disjoint, updated in place. n <= 8192: one persistent cooperative launch (all
 * CTAs resident, a grid barrier between steps, positions ping-ponged through
 * ws); larger n: one force + one integrator launch per step. Do not run two
 * calls sharing one ws concurrently (the grid barrier lives in ws).
 * ws: lime_nbody_simulate_workspace_bytes(n) bytes, device, zero-filled once. */
size_t lime_nbody_simulate_workspace_bytes(int64_t n);
lime_status lime_nbody_simulate(float *pos, float *vel, int64_t n, int32_t steps, float eps2,
                                float dt, void *ws, size_t ws_bytes, void *stream);

/* One complete N-Body simulation step through HOST buffers (end-to-end entry,
 * PAPER.md Fig. 6 / §4.3 L275-286 host<->device transport): copies h_pos and
 * h_vel ([n][4] float, host memory, pinned for best speed) to the device
 * scratch `ws`, runs lime_nbody_simulate(steps) on them, copies the new state back into h_pos / h_vel and
 * synchronises `stream`. ws: lime_nbody_simulate_host_workspace_bytes(n) bytes,
 * device, zero-filled before first use. */
size_t lime_nbody_simulate_host_workspace_bytes(int64_t n);
lime_status lime_nbody_simulate_host(float *h_pos, float *h_vel, int64_t n, int32_t steps,
                                     float eps2, float dt, void *ws, size_t ws_bytes,
                                     void *stream);

/* ===========================================================================
 * Black-Scholes European options (BASELINE.json config 2; not in the paper --
 * a transcendental streaming map of the kind it evaluates, SURVEY.md §0.2;
 * DESIGN.md R5). Per option i:
 *   d1 = (ln(S/X) + (r + sigma^2/2) T) / (sigma sqrt T), d2 = d1 - sigma sqrt T
 *   call[i] = S N(d1) - X e^{-rT} N(d2),  put[i] = X e^{-rT} N(-d2) - S N(-d1)
 * S, X, T: [n] float (SoA), 16-B aligned; call, put: [n] float, 16-B aligned,
 * no overlap with inputs or each other. S, X, T > 0, sigma > 0 (not checked
 * per element: a non-positive element yields NaN/inf in its own outputs only).
 * N(-|d|) = phi(d) M(1/(1 + 0.318|d|)) with M a degree-7 polynomial fitted to
 * the Mills ratio (|err| < 5e-10; tools/fit_mills.py); ln(S/X) = ln2 lg2(S/X).
 * Accuracy: |price - exact| <= 1e-5 max(|exact|, 1), measured over S in [5, 30],
 * X in [1, 100], T in [0.25, 10], r in [0, 0.1], sigma in [0.01, 2].
 * Launch override: grid_ctas honoured.
 * =========================================================================== */
lime_status lime_map_blackscholes(const float *S, const float *X, const float *T, int64_t n,
                                  float r, float sigma, float *call, float *put, void *stream);

/* Fused map+reduce (`!` over `@` without materialising the map, L160-163,
 * L188-189; R6): sums[0] = sum_i call[i], sums[1] = sum_i put[i]
 * (device double[2]), accumulated in fp64 from the warp level up (per-thread
 * partials fp32), CTA partials combined in a fixed order by the last CTA
 * (deterministic for a given launch configuration). The element is the same
 * closed form rearranged for summation: with A = S N(d1) - S/2 and
 * B = K N(d2) - K/2 (K = X e^{-rT}), call = (A - B) + (S - K)/2 and
 * put = (A - B) - (S - K)/2, so only the sums of A - B and S - K are formed
 * (put-call parity holds by construction). Tolerance vs the
 * oracle: 1e-5 relative on each sum. ws: lime_reduce_workspace_bytes() bytes.
 * Launch override: grid_ctas honoured. */
lime_status lime_map_reduce_blackscholes_sum(const float *S, const float *X, const float *T,
                                             int64_t n, float r, float sigma, double *sums,
                                             void *ws, size_t ws_bytes, void *stream);

/* ===========================================================================
 * Mandelbrot escape counts (BASELINE.json config 3; not in the paper; an
 * integer-output compute-bound map; R7). Bit-exact binary32:
 *   cx = x0 + px*dx, cy = y0 + py*dy, z0 = 0; count n while n < max_iter and
 *   x^2 + y^2 <= 4: x <- (x^2 - y^2) + cx, y <- (xy + xy) + cy.
 * Output counts [row_count][width] int32; output row k is image row
 * py = row_first + k*row_stride (row_stride = P, row_first = rank gives the
 * cyclic multi-GPU shard). width, height > 0; 0 <= row_first < height;
 * row_stride >= 1; every addressed py < height; max_iter >= 0.
 * ws: lime_mandelbrot_workspace_bytes() bytes (tile-queue counters).
 * Launch override: grid_ctas honoured; per_thread 1..8 selects the warp tile
 * shape / vote interval (tools/tune_mandel.py; results bit-identical).
 * =========================================================================== */
size_t lime_mandelbrot_workspace_bytes(void);
lime_status lime_map_mandelbrot(int32_t width, int32_t height, int32_t row_first,
                                int32_t row_stride, int32_t row_count, float x0, float y0,
                                float dx, float dy, int32_t max_iter, int32_t *counts,
                                void *ws, size_t ws_bytes, void *stream);

/* ===========================================================================
 * Dense matrix multiply as a map of dot products (BASELINE.json config 4; not
 * in the paper; R8): C[i][j] = sum_k A[i][k] * Bt[j][k].
 * A [M][K] bf16 bits (uint16), Bt [N][K] bf16 bits (K-major both), C [M][N]
 * float (fp32 accumulate, tcgen05 tensor cores). M, N >= 1; K >= 8 and
 * K % 8 == 0 (16-byte TMA row stride); M, N, K <= 2^31 - 512 and
 * ceil(M/256) * ceil(N/256) <= 2^31 - 1 (int32 rows, TMA coordinates and tile
 * indices; else LIME_ERR_INVALID_ARG); A, Bt, C 16-B aligned; C must not
 * overlap A or Bt. Accumulation order is fixed by K (per-K-slice MMAs in
 * order), so C does not depend on the launch configuration. For M >= 256 a
 * CTA pair (cta_group::2) computes 256 x 256 tiles; C is written by TMA tensor
 * stores when N % 4 == 0, else by direct stores (same bits).
 * Launch override: grid_ctas (persistent CTAs); block_threads = tile raster
 * group; per_thread 1 = one-CTA kernel, 2 = pair kernel, 3 = pair kernel with
 * the direct-store epilogue.
 * =========================================================================== */
lime_status lime_map_matmul_bf16(const uint16_t *A, const uint16_t *Bt, float *C, int64_t M,
                                 int64_t N, int64_t K, void *stream);

/* ===========================================================================
 * Parboil-CP: Coulombic potential on one lattice slice (Table 3;
 * SURVEY.md §8(f) F2; definition DESIGN.md R12): a map over lattice points with
 * the atom array as broadcast operand,
 *   V[t] = sum_j q_j / |p_t - r_j|,  t = p_begin + k (k in [0, p_count)),
 *   p_t = (fl32(ix h), fl32(iy h), z), ix = t % nx, iy = t / nx.
 * atoms [n_atoms][4] float (x, y, z, q), 16-B aligned; V [p_count] float, must
 * not overlap atoms. nx, ny >= 1; 0 <= p_begin <= p_begin + p_count <= nx*ny;
 * h > 0 and z finite. A lattice point exactly on an atom gives inf (no
 * softening, as in Parboil). Sum order: 256-atom chunks, split partials,
 * split order (deterministic, launch- and shard-independent).
 * ws: lime_map_coulomb_workspace_bytes(n_atoms, p_count) bytes, zeroed once.
 * =========================================================================== */
size_t lime_map_coulomb_workspace_bytes(int64_t n_atoms, int64_t p_count);
lime_status lime_map_coulomb(const float *atoms, int64_t n_atoms, int32_t nx, int32_t ny, int64_t p_begin,
                             int64_t p_count, float z, float h, float *V, void *ws, size_t ws_bytes,
                             void *stream);

/* ===========================================================================
 * Parboil-MRI-Q (Table 3; definition
 * DESIGN.md R13): a map over voxels with the k-space samples as broadcast
 * operand, Q[i] = (Qr, Qi) = sum_k |phi_k|^2 (cos, sin)(2 pi k.x_i),
 * i = x_begin + m (m in [0, x_count)).
 * kspace [n_k][5] float (kx, ky, kz, phiR, phiI); voxels [n_x][3] float; Q
 * [x_count][2] float, 8-B aligned, must not overlap the inputs. The phase is
 * reduced to [-1/2, 1/2] turn before the (MUFU) sine/cosine, so |k.x| must
 * stay below 2^22 turns. ws: lime_map_mriq_workspace_bytes(n_k, x_count) bytes
 * (holds the (kx, ky, kz, |phi|^2) table and the split partials), zeroed once.
 * =========================================================================== */
size_t lime_map_mriq_workspace_bytes(int64_t n_k, int64_t x_count);
lime_status lime_map_mriq(const float *kspace, int64_t n_k, const float *voxels, int64_t n_x, int64_t x_begin,
                          int64_t x_count, float *Q, void *ws, size_t ws_bytes, void *stream);

/* ===========================================================================
 * JG-Series (Table 3; definition DESIGN.md
 * R14 = the Java Grande "Series" kernel incl. its trapezoid loop): coefficient
 * pairs of f(x) = (x+1)^x on [0, 2], out[k] = (a_n, b_n) for n = n0 + k,
 * k in [0, count): a_0 = T[f]/2, b_0 = 0, a_n = T[f cos(n pi x)],
 * b_n = T[f sin(n pi x)], 1000-step trapezoid. out [count][2] float (f32) or
 * double (f64), naturally aligned. Phases are reduced exactly in integers
 * ((n i) mod 1000) before table lookup, so any n up to 2^40 is accurate.
 * ws: lime_map_series_workspace_bytes() bytes (node and cos/sin tables).
 * =========================================================================== */
size_t lime_map_series_workspace_bytes(void);
lime_status lime_map_series_f32(int64_t n0, int64_t count, float *out, void *ws, size_t ws_bytes,
                                void *stream);
lime_status lime_map_series_f64(int64_t n0, int64_t count, double *out, void *ws, size_t ws_bytes,
                                void *stream);

/* ===========================================================================
 * JG-Crypt (Table 3; definition DESIGN.md
 * R15): IDEA in ECB mode, a map over 8-byte blocks (four big-endian 16-bit
 * words). lime_idea_key_schedule (HOST pointers, no device work) expands a
 * 128-bit key key[8] into the 52 encryption sub-keys ek and decryption
 * sub-keys dk. lime_map_idea enciphers nbytes (a multiple of 8) from `in` to
 * `out` (device, 16-B aligned, no overlap) with the 52 sub-keys `subkeys`
 * (HOST pointer; copied into the launch parameters): pass ek to encrypt, dk
 * to decrypt. Bit-exact.
 * =========================================================================== */
void lime_idea_key_schedule(const uint16_t *key, uint16_t *ek, uint16_t *dk);
lime_status lime_map_idea(const uint8_t *in, uint8_t *out, int64_t nbytes, const uint16_t *subkeys,
                          void *stream);

/* ===========================================================================
 * Reductions `!` over an array x[n] (L160-163; L188-189 "the compiler may
 * infer a parallel reduction"; R9). Tree: per-thread fold ->
 * warp shuffle -> CTA -> last CTA combines the CTA partials in index order.
 * `out` is a DEVICE pointer to one element of the result type:
 *   sum_f32 -> float (accumulated in fp64 above the thread level)
 *   sum_f64 -> double, sum_i32 -> int32 (wraps), sum_i64 -> int64 (wraps)
 *   min/max -> the element type; NaN ignored (fmin/fmax); NaN only if all NaN.
 * Empty input writes the identity (0, +inf/-inf, INT_MAX/INT_MIN).
 * x needs only natural alignment of its element type. ws:
 * lime_reduce_workspace_bytes() bytes. Launch override: grid_ctas, block_threads.
 * =========================================================================== */
size_t lime_reduce_workspace_bytes(void);
lime_status lime_reduce_sum_f32(const float *x, int64_t n, float *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_sum_f64(const double *x, int64_t n, double *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_sum_i32(const int32_t *x, int64_t n, int32_t *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_sum_i64(const int64_t *x, int64_t n, int64_t *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_min_f32(const float *x, int64_t n, float *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_min_f64(const double *x, int64_t n, double *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_min_i32(const int32_t *x, int64_t n, int32_t *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_min_i64(const int64_t *x, int64_t n, int64_t *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_max_f32(const float *x, int64_t n, float *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_max_f64(const double *x, int64_t n, double *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_max_i32(const int32_t *x, int64_t n, int32_t *out, void *ws, size_t ws_bytes, void *stream);
lime_status lime_reduce_max_i64(const int64_t *x, int64_t n, int64_t *out, void *ws, size_t ws_bytes, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* LIME_H */
