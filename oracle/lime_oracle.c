/*
 * lime_oracle.c -- plain, slow, obviously-correct CPU oracle for the Lime
 * map (@) / reduce (!) hot path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (paper_conf_pldi_dubachcrbf12_b200/) never imports, links or calls it, and it
 * shares no code, header, table or constant generator with the CUDA path.
 *
 * Build: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fPIC -shared
 *        (x86-64 SSE arithmetic: no x87 excess precision, no contraction).
 * Single-threaded; every loop runs in the order the definition states.
 *
 * Citations: Lnnn = line nnn of the decoded `fulltext` of /root/reference/PAPER.md
 * (SURVEY.md §0 shows how to reproduce the numbering).
 *
 * Semantics (§3.2): map `@` applies a function to each
 * element of an aggregate and returns a NEW aggregate; reduce `!` combines the
 * elements with a binary combinator of one type (L160-163). Each map below
 * computes out[t] = f(in[begin + t], broadcast operands) for t = 0..count-1.
 *
 * Pins: every function is pinned in tests/test_oracle_pins.py against facts
 * fixed outside this file (textbook values, closed forms, invariants, brute
 * force). Parity-unpinned items are listed in DESIGN.md §"Parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>
#include <string.h>
#include <xmmintrin.h>

#define ORACLE_ABI_VERSION 1
int oracle_abi_version(void) { return ORACLE_ABI_VERSION; }

/* Guard against FTZ/DAZ inherited from a fast-math library loaded into the
 * same process (SURVEY.md §8(c) C-mandelbrot): default MXCSR = round to
 * nearest, all exceptions masked, FTZ=0, DAZ=0. */
static void oracle_fp_env(void) { _mm_setcsr(0x1F80); }

/* ------------------------------------------------------------------------
 * N-Body (§3 task graph; L108-112 float[[][4]] particles
 * x,y,z,mass -> per-particle force; L156-158 "each application of the map
 * function computes the force interactions between a particle p and all other
 * particles"; the formula itself is omitted by the paper (L157-158)).
 *
 * Reading (R1-R3): Plummer-softened Newtonian gravity, G = 1,
 * acceleration (force / m_i) is returned:
 *   a_i = sum_{j=0}^{N-1} m_j (p_j - p_i) / (|p_j - p_i|^2 + eps2)^{3/2}
 * evaluated in double from the fp32 inputs, in sequential j order, self term
 * included (it is exactly 0 since p_i - p_i = 0).
 * Output: accel[t*3 + c], double. If mag != NULL, mag[t] receives
 *   A_i = sum_j m_j |p_j - p_i| / (|p_j - p_i|^2 + eps2)^{3/2}
 * (sum of contribution magnitudes, used by the tolerance guard).
 * ---------------------------------------------------------------------- */
void oracle_nbody_accel(const float *bodies, int64_t n_src, int64_t tgt_begin,
                        int64_t tgt_count, float eps2, double *accel, double *mag)
{
    oracle_fp_env();
    const double e2 = (double)eps2;
    for (int64_t t = 0; t < tgt_count; ++t) {
        const int64_t i = tgt_begin + t;
        const double xi = bodies[4 * i + 0];
        const double yi = bodies[4 * i + 1];
        const double zi = bodies[4 * i + 2];
        double ax = 0.0, ay = 0.0, az = 0.0, am = 0.0;
        for (int64_t j = 0; j < n_src; ++j) {
            const double dx = (double)bodies[4 * j + 0] - xi;
            const double dy = (double)bodies[4 * j + 1] - yi;
            const double dz = (double)bodies[4 * j + 2] - zi;
            const double mj = (double)bodies[4 * j + 3];
            const double d2 = dx * dx + dy * dy + dz * dz;
            const double r2 = d2 + e2;
            const double s = mj / (r2 * sqrt(r2));     /* m_j (r^2+eps^2)^{-3/2} */
            ax += s * dx;
            ay += s * dy;
            az += s * dz;
            am += s * sqrt(d2);
        }
        accel[3 * t + 0] = ax;
        accel[3 * t + 1] = ay;
        accel[3 * t + 2] = az;
        if (mag) mag[t] = am;
    }
}

/* N-Body integrator = the `forceAccumulator` sink task, which "computes a new
 * position for each particle"; one task-graph pass is one
 * simulation step (L113-114). Reading (R4): semi-implicit Euler,
 *   v' = v + a dt ;  p' = p + v' dt ;  w (mass) unchanged,
 * in double from fp32 state. pos/vel are [n][4]; accel is [n][4] fp32 (the
 * device output layout: float4 with w = 0). Results written to pos_out/vel_out
 * ([n][4] double). */
void oracle_nbody_integrate(const float *pos, const float *vel, const float *accel,
                            int64_t n, float dt, double *pos_out, double *vel_out)
{
    oracle_fp_env();
    const double h = (double)dt;
    for (int64_t i = 0; i < n; ++i) {
        for (int c = 0; c < 3; ++c) {
            const double v = (double)vel[4 * i + c] + (double)accel[4 * i + c] * h;
            vel_out[4 * i + c] = v;
            pos_out[4 * i + c] = (double)pos[4 * i + c] + v * h;
        }
        vel_out[4 * i + 3] = (double)vel[4 * i + 3];
        pos_out[4 * i + 3] = (double)pos[4 * i + 3];
    }
}

/* ------------------------------------------------------------------------
 * Black-Scholes European call/put (not in the paper; BASELINE.json config 2,
 * a "transcendental streaming map of the kind it evaluates").
 * Textbook closed form (Black & Scholes 1973; Hull, "Options, Futures and
 * Other Derivatives", §"Black-Scholes-Merton pricing formulas"):
 *   d1 = (ln(S/X) + (r + sigma^2/2) T) / (sigma sqrt(T)),  d2 = d1 - sigma sqrt(T)
 *   C  = S N(d1) - X e^{-rT} N(d2)
 *   P  = X e^{-rT} N(-d2) - S N(-d1)
 *   N(x) = erfc(-x / sqrt(2)) / 2   (standard normal CDF)
 * evaluated in double from fp32 inputs. */
static double oracle_cnd(double x) { return 0.5 * erfc(-x / sqrt(2.0)); }
double oracle_normal_cdf(double x) { oracle_fp_env(); return oracle_cnd(x); }

void oracle_blackscholes(const float *S, const float *X, const float *T, int64_t n,
                         float r, float sigma, double *call, double *put)
{
    oracle_fp_env();
    const double rr = (double)r, sg = (double)sigma;
    for (int64_t i = 0; i < n; ++i) {
        const double s = S[i], x = X[i], t = T[i];
        const double sqt = sqrt(t);
        const double d1 = (log(s / x) + (rr + 0.5 * sg * sg) * t) / (sg * sqt);
        const double d2 = d1 - sg * sqt;
        const double kx = x * exp(-rr * t);
        call[i] = s * oracle_cnd(d1) - kx * oracle_cnd(d2);
        put[i] = kx * oracle_cnd(-d2) - s * oracle_cnd(-d1);
    }
}

/* Fused map+reduce reference: the reduction `!` with `+`
 * as the combinator over the map's output, "total premium" read as the two
 * sums (Sum C_i, Sum P_i) (R6). Neumaier-compensated left fold in
 * double, so the reference sum is accurate to ~1 ulp of double. */
void oracle_blackscholes_sums(const float *S, const float *X, const float *T, int64_t n,
                              float r, float sigma, double *sums /* [2] */)
{
    oracle_fp_env();
    const double rr = (double)r, sg = (double)sigma;
    double sc = 0.0, cc = 0.0, sp = 0.0, cp = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        const double s = S[i], x = X[i], t = T[i];
        const double sqt = sqrt(t);
        const double d1 = (log(s / x) + (rr + 0.5 * sg * sg) * t) / (sg * sqt);
        const double d2 = d1 - sg * sqt;
        const double kx = x * exp(-rr * t);
        const double c = s * oracle_cnd(d1) - kx * oracle_cnd(d2);
        const double p = kx * oracle_cnd(-d2) - s * oracle_cnd(-d1);
        double tt = sc + c;
        cc += (fabs(sc) >= fabs(c)) ? (sc - tt) + c : (c - tt) + sc;
        sc = tt;
        tt = sp + p;
        cp += (fabs(sp) >= fabs(p)) ? (sp - tt) + p : (p - tt) + sp;
        sp = tt;
    }
    sums[0] = sc + cc;
    sums[1] = sp + cp;
}

/* ------------------------------------------------------------------------
 * Mandelbrot escape counts (not in the paper; BASELINE.json config 3, an
 * integer-output compute-bound map). Reading (R7): EXACT fp32
 * emulation -- every * and + is one IEEE binary32 round-to-nearest operation,
 * no contraction, no FTZ, in exactly this order:
 *   cx = x0 + (float)px * dx ;  cy = y0 + (float)py * dy ;  x = y = 0 ; n = 0
 *   while n < max_iter:
 *     xx = x*x ; yy = y*y
 *     if xx + yy > 4: break
 *     xy = x*y ; x = (xx - yy) + cx ; y = (xy + xy) + cy ; n = n + 1
 * Output int32 n (non-escaping points count max_iter). */
int32_t oracle_mandelbrot_point(float cx, float cy, int32_t max_iter)
{
    oracle_fp_env();
    float x = 0.0f, y = 0.0f;   /* binary32 SSE arithmetic, -ffp-contract=off */
    int32_t n = 0;
    while (n < max_iter) {
        const float xx = x * x;
        const float yy = y * y;
        if (xx + yy > 4.0f) break;
        const float xy = x * y;
        x = (xx - yy) + cx;
        y = (xy + xy) + cy;
        ++n;
    }
    return n;
}

/* Rows py = row_first + k*row_stride, k = 0..row_count-1 (row_stride = P gives
 * the cyclic multi-GPU shard); counts is [row_count][width]. */
void oracle_mandelbrot(int32_t width, int32_t height, int32_t row_first, int32_t row_stride,
                       int32_t row_count, float x0, float y0, float dx, float dy,
                       int32_t max_iter, int32_t *counts)
{
    (void)height;
    oracle_fp_env();
    for (int32_t k = 0; k < row_count; ++k) {
        const int32_t py = row_first + k * row_stride;
        const float fy = (float)py * dy;
        const float cy = y0 + fy;
        for (int32_t px = 0; px < width; ++px) {
            const float fx = (float)px * dx;
            const float cx = x0 + fx;
            counts[(int64_t)k * width + px] = oracle_mandelbrot_point(cx, cy, max_iter);
        }
    }
}

/* ------------------------------------------------------------------------
 * Dense matrix multiply as a map of dot products (not in the paper;
 * BASELINE.json config 4). Reading (R8): A [M][K] and Bt [N][K] are
 * K-major bf16 bit patterns; C[i][j] = sum_k A[i][k] * Bt[j][k], in double,
 * sequential k. bf16 -> value: bits << 16 reinterpreted as binary32 (exact). */
static double bf16_value(uint16_t b)
{
    uint32_t u = (uint32_t)b << 16;
    float f;
    memcpy(&f, &u, sizeof f);
    return (double)f;
}

void oracle_matmul_bf16(const uint16_t *A, const uint16_t *Bt, int64_t M, int64_t N, int64_t K,
                        double *C)
{
    oracle_fp_env();
    for (int64_t i = 0; i < M; ++i)
        for (int64_t j = 0; j < N; ++j) {
            double acc = 0.0;
            for (int64_t k = 0; k < K; ++k)
                acc += bf16_value(A[i * K + k]) * bf16_value(Bt[j * K + k]);
            C[i * N + j] = acc;
        }
}

/* Sampled entries: C[rows[s]][cols[s]] for s = 0..n_samples-1, plus the
 * magnitude bound absC[s] = sum_k |A_ik| |Bt_jk| (used by the tolerance). */
void oracle_matmul_bf16_entries(const uint16_t *A, const uint16_t *Bt, int64_t K,
                                const int64_t *rows, const int64_t *cols, int64_t n_samples,
                                double *C, double *absC)
{
    oracle_fp_env();
    for (int64_t s = 0; s < n_samples; ++s) {
        const int64_t i = rows[s], j = cols[s];
        double acc = 0.0, mag = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            const double p = bf16_value(A[i * K + k]) * bf16_value(Bt[j * K + k]);
            acc += p;
            mag += fabs(p);
        }
        C[s] = acc;
        if (absC) absC[s] = mag;
    }
}

/* ------------------------------------------------------------------------
 * Reductions `!` ("an operator or method followed by ! ...
 * apply to two arguments of the same type and produce a result of that type";
 * L188-189 "the compiler may infer a parallel reduction").
 * Readings (R9): sums are left folds; floating sums are compensated
 * (Neumaier) in double and returned in double; integer sums wrap in two's
 * complement of the element width; min/max ignore NaN (fmin semantics) and
 * return NaN only when every element is NaN. Empty input -> identity
 * (0, +inf / -inf, INT_MAX / INT_MIN). */
double oracle_reduce_sum_f32(const float *x, int64_t n)
{
    oracle_fp_env();
    double s = 0.0, c = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        const double v = x[i], t = s + v;
        c += (fabs(s) >= fabs(v)) ? (s - t) + v : (v - t) + s;
        s = t;
    }
    return s + c;
}

double oracle_reduce_sum_f64(const double *x, int64_t n)
{
    oracle_fp_env();
    double s = 0.0, c = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        const double v = x[i], t = s + v;
        c += (fabs(s) >= fabs(v)) ? (s - t) + v : (v - t) + s;
        s = t;
    }
    return s + c;
}

int32_t oracle_reduce_sum_i32(const int32_t *x, int64_t n)
{
    uint32_t s = 0;
    for (int64_t i = 0; i < n; ++i) s += (uint32_t)x[i];
    int32_t r;
    memcpy(&r, &s, sizeof r);
    return r;
}

int64_t oracle_reduce_sum_i64(const int64_t *x, int64_t n)
{
    uint64_t s = 0;
    for (int64_t i = 0; i < n; ++i) s += (uint64_t)x[i];
    int64_t r;
    memcpy(&r, &s, sizeof r);
    return r;
}

float oracle_reduce_min_f32(const float *x, int64_t n)
{
    float m = INFINITY;
    int any = 0, all_nan = 1;
    for (int64_t i = 0; i < n; ++i) {
        any = 1;
        if (isnan(x[i])) continue;
        all_nan = 0;
        if (x[i] < m) m = x[i];
    }
    return (any && all_nan) ? NAN : m;
}

float oracle_reduce_max_f32(const float *x, int64_t n)
{
    float m = -INFINITY;
    int any = 0, all_nan = 1;
    for (int64_t i = 0; i < n; ++i) {
        any = 1;
        if (isnan(x[i])) continue;
        all_nan = 0;
        if (x[i] > m) m = x[i];
    }
    return (any && all_nan) ? NAN : m;
}

double oracle_reduce_min_f64(const double *x, int64_t n)
{
    double m = INFINITY;
    int any = 0, all_nan = 1;
    for (int64_t i = 0; i < n; ++i) {
        any = 1;
        if (isnan(x[i])) continue;
        all_nan = 0;
        if (x[i] < m) m = x[i];
    }
    return (any && all_nan) ? NAN : m;
}

double oracle_reduce_max_f64(const double *x, int64_t n)
{
    double m = -INFINITY;
    int any = 0, all_nan = 1;
    for (int64_t i = 0; i < n; ++i) {
        any = 1;
        if (isnan(x[i])) continue;
        all_nan = 0;
        if (x[i] > m) m = x[i];
    }
    return (any && all_nan) ? NAN : m;
}

int32_t oracle_reduce_min_i32(const int32_t *x, int64_t n)
{
    int32_t m = INT32_MAX;
    for (int64_t i = 0; i < n; ++i) if (x[i] < m) m = x[i];
    return m;
}

int32_t oracle_reduce_max_i32(const int32_t *x, int64_t n)
{
    int32_t m = INT32_MIN;
    for (int64_t i = 0; i < n; ++i) if (x[i] > m) m = x[i];
    return m;
}

int64_t oracle_reduce_min_i64(const int64_t *x, int64_t n)
{
    int64_t m = INT64_MAX;
    for (int64_t i = 0; i < n; ++i) if (x[i] < m) m = x[i];
    return m;
}

int64_t oracle_reduce_max_i64(const int64_t *x, int64_t n)
{
    int64_t m = INT64_MIN;
    for (int64_t i = 0; i < n; ++i) if (x[i] > m) m = x[i];
    return m;
}

/* ------------------------------------------------------------------------
 * Parboil-CP: Coulombic potential on one lattice slice (Table 3,
 * "Parboil-CP Coulombic Potential 62KB -> 1MB Float"). The
 * paper describes only the benchmark name and sizes; reading DESIGN.md R12:
 * direct Coulomb summation
 *   V[iy][ix] = sum_j q_j / sqrt((x - x_j)^2 + (y - y_j)^2 + (z - z_j)^2),
 *   x = fl32(ix * h), y = fl32(iy * h)  (grid coordinates are the fp32 products),
 * evaluated in double from the fp32 inputs, sequential j, for lattice rows
 * iy0 .. iy0+ny-1 (out/mag are [ny][nx]). atoms is [n][4] (x, y, z, q). If
 * mag != NULL it receives sum_j |q_j| / r_j. */
void oracle_coulomb_potential(const float *atoms, int64_t n_atoms, int32_t nx, int32_t iy0, int32_t ny,
                              float z, float h, double *out, double *mag)
{
    oracle_fp_env();
    for (int32_t r = 0; r < ny; ++r) {
        const int32_t iy = iy0 + r;
        const float yf = (float)iy * h;
        for (int32_t ix = 0; ix < nx; ++ix) {
            const float xf = (float)ix * h;
            double v = 0.0, m = 0.0;
            for (int64_t j = 0; j < n_atoms; ++j) {
                const double dx = (double)xf - (double)atoms[4 * j + 0];
                const double dy = (double)yf - (double)atoms[4 * j + 1];
                const double dz = (double)z - (double)atoms[4 * j + 2];
                const double r = sqrt(dx * dx + dy * dy + dz * dz);
                v += (double)atoms[4 * j + 3] / r;
                m += fabs((double)atoms[4 * j + 3]) / r;
            }
            out[(int64_t)r * nx + ix] = v;
            if (mag) mag[(int64_t)r * nx + ix] = m;
        }
    }
}

/* ------------------------------------------------------------------------
 * Parboil-MRI-Q: the Q matrix of non-Cartesian MRI reconstruction (PAPER.md
 * Table 3, "Parboil-MRIQ Magnetic Resonance Imaging 432KB -> 256KB
 * Float"). Reading DESIGN.md R13 (Parboil's definition):
 *   phiMag_k = phiR_k^2 + phiI_k^2
 *   Qr(x) = sum_k phiMag_k cos(2 pi (kx_k x + ky_k y + kz_k z))
 *   Qi(x) = sum_k phiMag_k sin(2 pi (kx_k x + ky_k y + kz_k z))
 * in double from the fp32 inputs, sequential k. kspace is [K][5] floats
 * (kx, ky, kz, phiR, phiI); voxels is [X][3] (x, y, z); out is [X][2]
 * (Qr, Qi). If mag != NULL it receives sum_k phiMag_k. */
void oracle_mriq(const float *kspace, int64_t n_k, const float *voxels, int64_t n_x, double *out,
                 double *mag)
{
    oracle_fp_env();
    const double two_pi = 6.283185307179586476925286766559;
    for (int64_t i = 0; i < n_x; ++i) {
        const double x = voxels[3 * i + 0], y = voxels[3 * i + 1], zz = voxels[3 * i + 2];
        double qr = 0.0, qi = 0.0, m = 0.0;
        for (int64_t k = 0; k < n_k; ++k) {
            const double pr = kspace[5 * k + 3], pi = kspace[5 * k + 4];
            const double phimag = pr * pr + pi * pi;
            const double arg = two_pi * ((double)kspace[5 * k + 0] * x + (double)kspace[5 * k + 1] * y +
                                         (double)kspace[5 * k + 2] * zz);
            qr += phimag * cos(arg);
            qi += phimag * sin(arg);
            m += phimag;
        }
        out[2 * i + 0] = qr;
        out[2 * i + 1] = qi;
        if (mag) mag[i] = m;
    }
}

/* ------------------------------------------------------------------------
 * N-Body, double precision (Table 3: "N-Body ... 64KB / 128KB
 * 48KB / 128KB Float / Double"; L319-323 single- and double-precision variants;
 * SURVEY.md §8(f) F3). Same definition as oracle_nbody_accel (R1-R3) on fp64
 * bodies [n][4] (x, y, z, m); accel [count][3] double; mag optional. */
void oracle_nbody_accel_f64(const double *bodies, int64_t n_src, int64_t tgt_begin, int64_t tgt_count,
                            double eps2, double *accel, double *mag)
{
    oracle_fp_env();
    for (int64_t t = 0; t < tgt_count; ++t) {
        const int64_t i = tgt_begin + t;
        const double xi = bodies[4 * i + 0], yi = bodies[4 * i + 1], zi = bodies[4 * i + 2];
        double ax = 0.0, ay = 0.0, az = 0.0, am = 0.0;
        for (int64_t j = 0; j < n_src; ++j) {
            const double dx = bodies[4 * j + 0] - xi;
            const double dy = bodies[4 * j + 1] - yi;
            const double dz = bodies[4 * j + 2] - zi;
            const double d2 = dx * dx + dy * dy + dz * dz;
            const double r2 = d2 + eps2;
            const double s = bodies[4 * j + 3] / (r2 * sqrt(r2));
            ax += s * dx;
            ay += s * dy;
            az += s * dz;
            am += s * sqrt(d2);
        }
        accel[3 * t + 0] = ax;
        accel[3 * t + 1] = ay;
        accel[3 * t + 2] = az;
        if (mag) mag[t] = am;
    }
}

/* ------------------------------------------------------------------------
 * JG-Series: Fourier coefficient analysis (Table 3 "JG-Series
 * Fourier coefficient analysis 780KB / 1560KB Float / Double"; SURVEY.md §8(f)
 * F4). The paper ports the Java Grande Forum "Series" kernel; reading
 * DESIGN.md R14 follows that kernel step by step: the first N coefficient
 * pairs of f(x) = (x+1)^x on [0, 2] with omega = pi,
 *   a_0 = T(0, 0) / 2, b_0 = 0 ;  a_n = T(n pi, cos), b_n = T(n pi, sin) (n >= 1)
 * where T is JGF's TrapezoidIntegrate(0, 2, m, omega_n, select):
 *   dx = 2/m; r = g(0)/2; for i = 1 .. m-2: r += g(x_i); r = (r + g(2)/2) dx
 * -- JGF's loop `--nsteps; while (--nsteps > 0)` visits the interior nodes
 * x_1 .. x_{m-2} only (node x_{m-1} is skipped), and that is kept. Nodes are
 * x_i = i dx (one rounding; JGF accumulates x += dx, a < 1e-12 difference).
 * g(x) = f(x) [select 0], f(x) cos(omega x) [1], f(x) sin(omega x) [2].
 * In double. out[k][2] = (a_n, b_n) for n = n0 + k; mag[k] = T over |f|. */
static double series_g(double x, double omegan, int select)
{
    const double f = pow(x + 1.0, x);
    if (select == 0) return f;
    return select == 1 ? f * cos(omegan * x) : f * sin(omegan * x);
}

static double series_trapezoid(double x0, double x1, int32_t nsteps, double omegan, int select)
{
    const double dx = (x1 - x0) / nsteps;
    double r = series_g(x0, omegan, select) / 2.0;
    if (nsteps != 1)
        for (int32_t i = 1; i < nsteps - 1; ++i) r += series_g(x0 + i * dx, omegan, select);
    return (r + series_g(x1, omegan, select) / 2.0) * dx;
}

void oracle_series(int64_t n0, int64_t count, int32_t m, double *out, double *mag)
{
    oracle_fp_env();
    const double omega = 3.1415926535897932;
    for (int64_t k = 0; k < count; ++k) {
        const int64_t n = n0 + k;
        if (n == 0) {
            out[2 * k + 0] = series_trapezoid(0.0, 2.0, m, 0.0, 0) / 2.0;
            out[2 * k + 1] = 0.0;
        } else {
            out[2 * k + 0] = series_trapezoid(0.0, 2.0, m, omega * (double)n, 1);
            out[2 * k + 1] = series_trapezoid(0.0, 2.0, m, omega * (double)n, 2);
        }
        if (mag) mag[k] = series_trapezoid(0.0, 2.0, m, 0.0, 0);    /* f > 0: T[|f|] = T[f] */
    }
}

/* ------------------------------------------------------------------------
 * JG-Crypt: IDEA block cipher over a byte array (Table 3
 * "JG-Crypt IDEA encryption 3MB 3MB Byte"). Reading
 * DESIGN.md R15: IDEA (Lai & Massey 1991) in ECB mode, 8-byte blocks of four
 * big-endian 16-bit words, 8 rounds + output transform, 52 sub-keys from the
 * 128-bit key (25-bit rotations); decryption uses the inverted sub-keys. The
 * byte array length must be a multiple of 8. */
static uint16_t idea_mul(uint16_t a, uint16_t b)
{
    /* multiplication modulo 2^16 + 1, with 0 standing for 2^16 */
    const uint32_t aa = a ? a : 65536u, bb = b ? b : 65536u;
    const uint64_t p = ((uint64_t)aa * bb) % 65537u;
    return (uint16_t)(p == 65536u ? 0 : p);
}

static uint16_t idea_mul_inv(uint16_t a)
{
    /* a^(65537-2) mod 65537 (Fermat), with 0 <-> 2^16 */
    const uint64_t mod = 65537u;
    uint64_t base = a ? a : 65536u, r = 1, e = mod - 2;
    while (e) {
        if (e & 1) r = (r * base) % mod;
        base = (base * base) % mod;
        e >>= 1;
    }
    return (uint16_t)(r == 65536u ? 0 : r);
}

void oracle_idea_keys(const uint16_t key[8], uint16_t ek[52], uint16_t dk[52])
{
    /* encryption sub-keys: the 128-bit key, then repeatedly rotated left by 25 bits */
    uint8_t k[16];
    for (int i = 0; i < 8; ++i) { k[2 * i] = (uint8_t)(key[i] >> 8); k[2 * i + 1] = (uint8_t)key[i]; }
    for (int s = 0; s < 52; ++s) {
        const int rot = 25 * (s / 8);               /* bits rotated so far */
        const int w = s % 8;
        uint16_t v = 0;
        for (int b = 0; b < 16; ++b) {
            const int bit = (16 * w + b + rot) % 128;   /* MSB-first bit index in k */
            v = (uint16_t)((v << 1) | ((k[bit / 8] >> (7 - bit % 8)) & 1));
        }
        ek[s] = v;
    }
    /* decryption sub-keys */
    dk[0] = idea_mul_inv(ek[48]);
    dk[1] = (uint16_t)(0u - ek[49]);
    dk[2] = (uint16_t)(0u - ek[50]);
    dk[3] = idea_mul_inv(ek[51]);
    for (int r = 1; r < 8; ++r) {
        const int e = 48 - 6 * r, d = 6 * r;
        dk[d - 2] = ek[e + 4];
        dk[d - 1] = ek[e + 5];
        dk[d + 0] = idea_mul_inv(ek[e + 0]);
        dk[d + 1] = (uint16_t)(0u - ek[e + 2]);     /* middle rounds swap the two additive keys */
        dk[d + 2] = (uint16_t)(0u - ek[e + 1]);
        dk[d + 3] = idea_mul_inv(ek[e + 3]);
    }
    dk[46] = ek[4];
    dk[47] = ek[5];
    dk[48] = idea_mul_inv(ek[0]);
    dk[49] = (uint16_t)(0u - ek[1]);
    dk[50] = (uint16_t)(0u - ek[2]);
    dk[51] = idea_mul_inv(ek[3]);
}

static void idea_block(const uint8_t in[8], uint8_t out[8], const uint16_t z[52])
{
    uint16_t x1 = (uint16_t)(in[0] << 8 | in[1]), x2 = (uint16_t)(in[2] << 8 | in[3]);
    uint16_t x3 = (uint16_t)(in[4] << 8 | in[5]), x4 = (uint16_t)(in[6] << 8 | in[7]);
    for (int r = 0; r < 8; ++r) {
        const uint16_t *k = z + 6 * r;
        x1 = idea_mul(x1, k[0]);
        x2 = (uint16_t)(x2 + k[1]);
        x3 = (uint16_t)(x3 + k[2]);
        x4 = idea_mul(x4, k[3]);
        const uint16_t t0 = idea_mul((uint16_t)(x1 ^ x3), k[4]);
        const uint16_t t1 = idea_mul((uint16_t)(t0 + (x2 ^ x4)), k[5]);
        const uint16_t t2 = (uint16_t)(t0 + t1);
        x1 ^= t1;
        x4 ^= t2;
        const uint16_t a = (uint16_t)(x2 ^ t2);
        x2 = (uint16_t)(x3 ^ t1);
        x3 = a;
    }
    const uint16_t y1 = idea_mul(x1, z[48]);
    const uint16_t y2 = (uint16_t)(x3 + z[49]);      /* undo the last round's swap */
    const uint16_t y3 = (uint16_t)(x2 + z[50]);
    const uint16_t y4 = idea_mul(x4, z[51]);
    out[0] = (uint8_t)(y1 >> 8); out[1] = (uint8_t)y1; out[2] = (uint8_t)(y2 >> 8); out[3] = (uint8_t)y2;
    out[4] = (uint8_t)(y3 >> 8); out[5] = (uint8_t)y3; out[6] = (uint8_t)(y4 >> 8); out[7] = (uint8_t)y4;
}

/* ECB over nbytes (multiple of 8) with sub-keys z (ek to encrypt, dk to decrypt) */
void oracle_idea(const uint8_t *in, uint8_t *out, int64_t nbytes, const uint16_t z[52])
{
    for (int64_t i = 0; i + 8 <= nbytes; i += 8) idea_block(in + i, out + i, z);
}
