"""GPU parity away from the benchmark's input recipe: the same maps on other softening
lengths, other body distributions (two offset clusters, a cube far from the origin, random masses),
other Black-Scholes market parameters and other Mandelbrot regions, against the oracle with the
north_star tolerances (N-Body 1e-4, Black-Scholes 1e-5, Mandelbrot bit-exact). Sizes cover both N-Body
paths (n <= 8192: small kernels; n > 8192: split-j force_kernel) with ragged tails."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import BS_TOL, NBODY_RTOL, nbody_rel_err

pytestmark = pytest.mark.gpu


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _u(seed, stream, n):
    return inputs.uniform24(seed, stream, n).astype(np.float64)


def _gauss(seed, stream, n):
    # Box-Muller on two seeded uniform streams (input generation only)
    u1 = np.maximum(_u(seed, stream, n), 2.0 ** -24)
    u2 = _u(seed, stream + 1, n)
    return np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)


def two_clusters(n, seed):
    """Two Gaussian clusters (sigma 0.05 and 0.1) at distance 1.5, mass ratio 3:1, masses U[0.5, 1.5)/n."""
    b = np.empty((n, 4), dtype=np.float32)
    half = n // 3
    for c in range(3):
        g = _gauss(seed, 2 * c, n)
        centre = np.where(np.arange(n) < half, 1.5 if c == 0 else 0.0, 0.0)
        b[:, c] = centre + np.where(np.arange(n) < half, 0.05, 0.1) * g
    b[:, 3] = (0.5 + _u(seed, 7, n)) / n
    return b


def far_cube(n, seed):
    """The recipe's unit cube moved to (1000, -2000, 500): fp32 coordinates keep ~6e-5 absolute resolution."""
    b = inputs.nbody_bodies(n, seed=seed)
    b[:, 0] += np.float32(1000.0)
    b[:, 1] += np.float32(-2000.0)
    b[:, 2] += np.float32(500.0)
    return b


@pytest.mark.parametrize("n", [1000, 4096, 12289])
@pytest.mark.parametrize("eps2", [1e-20, 1e-8, 1e-2, 1.0])
def test_nbody_softening_lengths(lime, n, eps2):
    b = inputs.nbody_bodies(n, seed=200 + n)
    e = np.float32(eps2)
    acc = lime.map_nbody(_dev(b), float(e)).cpu().numpy()
    if n <= 4096:
        ref, mag = oracle.nbody_accel(b, e, with_mag=True)
        err = nbody_rel_err(acc, ref, mag)
    else:
        rows = np.concatenate([np.arange(0, 40), np.arange(n // 2, n // 2 + 40), np.arange(n - 40, n)])
        ref, mag = oracle.nbody_accel_rows(b, e, rows, threads=8)
        err = nbody_rel_err(acc[rows], ref, mag)
    assert err.max() <= NBODY_RTOL, (n, eps2, err.max())


@pytest.mark.parametrize("dist", ["two_clusters", "far_cube"])
@pytest.mark.parametrize("n", [777, 4096, 8193, 20000])
def test_nbody_distributions(lime, dist, n):
    b = {"two_clusters": two_clusters, "far_cube": far_cube}[dist](n, 300 + n)
    e = np.float32(1e-4)
    acc = lime.map_nbody(_dev(b), float(e)).cpu().numpy()
    rows = np.unique(np.concatenate([np.arange(0, 64), np.arange(n // 3 - 32, n // 3 + 32), np.arange(n - 64, n)]))
    ref, mag = oracle.nbody_accel_rows(b, e, rows, threads=8)
    err = nbody_rel_err(acc[rows], ref, mag)
    assert err.max() <= NBODY_RTOL, (dist, n, err.max())
    # shards are slices of the full map on these inputs too
    part = lime.map_nbody(_dev(b), float(e), n // 3, n - n // 3).cpu().numpy()
    assert np.array_equal(part, acc[n // 3:])


# r = 0, sigma = 0.3 measured 1.03e-5 with the Abramowitz-Stegun CND; low sigma sqrt(T) near
# the forward at-the-money point is the worst conditioned case of the fp32 form (sigma = 0.05: 9.7e-6)
@pytest.mark.parametrize("r,sigma", [(0.0, 0.30), (0.10, 0.05), (0.05, 1.0), (0.02, 0.01), (0.0, 0.10), (0.05, 0.20), (0.1, 2.0)])
def test_blackscholes_market_parameters(lime, r, sigma):
    n = (1 << 18) + 5
    S, X, T = inputs.blackscholes_options(n, seed=400)
    r32, s32 = np.float32(r), np.float32(sigma)
    call, put = lime.map_blackscholes(_dev(S), _dev(X), _dev(T), float(r32), float(s32))
    c_ref, p_ref = oracle.blackscholes(S, X, T, r32, s32)
    for got, ref in ((call, c_ref), (put, p_ref)):
        err = np.abs(got.cpu().numpy().astype(np.float64) - ref) / np.maximum(np.abs(ref), 1.0)
        assert err.max() <= BS_TOL, (r, sigma, err.max())
    sums = lime.map_reduce_blackscholes_sum(_dev(S), _dev(X), _dev(T), float(r32), float(s32)).cpu().numpy()
    sc, sp = oracle.blackscholes_sums(S, X, T, r32, s32)
    assert abs(sums[0] - sc) <= BS_TOL * max(abs(sc), n) and abs(sums[1] - sp) <= BS_TOL * max(abs(sp), n)


@pytest.mark.parametrize("x0,y0,span,max_iter", [
    (-0.7453, 0.1127, 6.5e-3, 3000),      # seahorse valley (spirals, long escapes)
    (-1.7686, -0.0017, 3.4e-3, 2048),     # the period-3 mini-brot on the real axis
    (0.2501, -0.0005, 1.0e-3, 4096),      # just outside the cusp at 1/4 (slow escapes)
    (-2.0, -2.0, 4.0, 100),               # whole plane incl. |c| > 2 (escape before the first update)
])
def test_mandelbrot_regions_bit_exact(lime, x0, y0, span, max_iter):
    W, H = 96, 72
    x0, y0 = float(np.float32(x0)), float(np.float32(y0))
    dx, dy = float(np.float32(span / W)), float(np.float32(span / H))
    got = lime.map_mandelbrot(W, H, x0, y0, dx, dy, max_iter).cpu().numpy()
    ref = oracle.mandelbrot(W, H, 0, 1, H, x0, y0, dx, dy, max_iter)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("dist", ["uniform", "two_clusters", "far_cube"])
@pytest.mark.parametrize("eps2", [1e-12, 1e-4, 1.0])
def test_nbody_f64_variants(lime, dist, eps2):
    n = 3001
    b = {"uniform": lambda n, s: inputs.nbody_bodies(n, seed=s), "two_clusters": two_clusters,
         "far_cube": far_cube}[dist](n, 500).astype(np.float64)
    acc = lime.map_nbody_f64(_dev(b), eps2).cpu().numpy()
    ref, mag = oracle.nbody_accel_f64(b, eps2, with_mag=True)
    assert nbody_rel_err(acc, ref, mag).max() <= 1e-12, (dist, eps2)


def test_matmul_wide_dynamic_range(lime):
    # bf16 operands with exponents spread over 2^-20 .. 2^20 (products over 2^-40 .. 2^40): the fp32
    # tensor-core accumulation against sum_k |A_ik Bt_jk| (north_star 1e-3), ragged M/N/K
    M, N, K = 300, 520, 264
    A, Bt = inputs.matmul_operands(M, N, K, seed=600)
    def spread(bits, seed):
        e = (np.floor(_u(seed, 0, bits.size) * 41) - 20).reshape(bits.shape)
        f = inputs.bf16_bits_to_f32(bits).astype(np.float64) * np.exp2(e)
        return inputs._f32_to_bf16_bits(f.astype(np.float32))
    A, Bt = spread(A, 601), spread(Bt, 602)
    C = lime.map_matmul_bf16(_dev(A.view(np.int16)).view(torch.bfloat16), _dev(Bt.view(np.int16)).view(torch.bfloat16))
    ref = oracle.matmul_bf16(A, Bt)
    mag = np.abs(inputs.bf16_bits_to_f32(A)).astype(np.float64) @ np.abs(inputs.bf16_bits_to_f32(Bt)).astype(np.float64).T
    assert (np.abs(C.cpu().numpy() - ref) / np.maximum(mag, 1e-300)).max() <= 1e-3
