"""GPU parity: Black-Scholes map and fused map+reduce vs the oracle (through the C ABI)."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import BS_TOL

pytestmark = pytest.mark.gpu
R, SIG = np.float32(inputs.BS_R), np.float32(inputs.BS_SIGMA)


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _check(S, X, T, call, put, r=R, sig=SIG):
    c_ref, p_ref = oracle.blackscholes(S, X, T, r, sig)
    ec = np.abs(call.astype(np.float64) - c_ref) / np.maximum(np.abs(c_ref), 1.0)
    ep = np.abs(put.astype(np.float64) - p_ref) / np.maximum(np.abs(p_ref), 1.0)
    return max(ec.max(initial=0), ep.max(initial=0))


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 7, 1000, (1 << 20) + 3])
def test_map_matches_oracle(lime, n):
    S, X, T = inputs.blackscholes_options(n, seed=20 + n % 97)
    c, p = lime.map_blackscholes(_dev(S), _dev(X), _dev(T), float(R), float(SIG))
    assert _check(S, X, T, c.cpu().numpy(), p.cpu().numpy()) <= BS_TOL


def test_map_full_config_and_parity(lime):
    n = 1 << 24
    S, X, T = inputs.blackscholes_options(n, seed=2)
    Sd, Xd, Td = _dev(S), _dev(X), _dev(T)
    c, p = lime.map_blackscholes(Sd, Xd, Td, float(R), float(SIG))
    c, p = c.cpu().numpy(), p.cpu().numpy()
    assert _check(S, X, T, c, p) <= BS_TOL
    kx = X.astype(np.float64) * np.exp(-float(R) * T.astype(np.float64))
    parity = np.abs((c.astype(np.float64) - p) - (S - kx)) / np.maximum(S, X)
    assert parity.max() <= 1e-5
    assert torch.equal(Sd.cpu(), torch.from_numpy(S))               # input untouched


def test_tails_and_extremes(lime):
    # deep in/out of the money, very short/long maturities: |d| well beyond 5
    S = np.array([5, 30, 5, 30, 100, 1, 50, 50], dtype=np.float32)
    X = np.array([100, 1, 90, 2, 1, 100, 50, 50], dtype=np.float32)
    T = np.array([0.25, 0.25, 10, 10, 0.01, 0.01, 0.0001, 50], dtype=np.float32)
    c, p = lime.map_blackscholes(_dev(S), _dev(X), _dev(T), float(R), float(SIG))
    assert _check(S, X, T, c.cpu().numpy(), p.cpu().numpy()) <= BS_TOL


@pytest.mark.parametrize("n", [0, 1, 5, 4099, 1 << 24])
def test_fused_sums(lime, n):
    S, X, T = inputs.blackscholes_options(n, seed=2)
    sums = lime.map_reduce_blackscholes_sum(_dev(S), _dev(X), _dev(T), float(R), float(SIG)).cpu().numpy()
    sc, sp = oracle.blackscholes_sums(S, X, T, R, SIG)
    assert abs(sums[0] - sc) <= BS_TOL * max(abs(sc), 1.0)
    assert abs(sums[1] - sp) <= BS_TOL * max(abs(sp), 1.0)
    again = lime.map_reduce_blackscholes_sum(_dev(S), _dev(X), _dev(T), float(R), float(SIG)).cpu().numpy()
    assert np.array_equal(sums, again)                               # deterministic, ws self-resets


@pytest.mark.parametrize("k", range(8))
def test_fused_single_option_tails(lime, k):
    # the fused kernel's element (sums of w = A - B and u = S - K; call = w + u/2, put = w - u/2)
    # on one tail option at a time, padded to a multiple of 4 with copies so the vector path runs
    S = np.array([5, 30, 5, 30, 100, 1, 50, 50], dtype=np.float32)
    X = np.array([100, 1, 90, 2, 1, 100, 50, 50], dtype=np.float32)
    T = np.array([0.25, 0.25, 10, 10, 0.01, 0.01, 0.0001, 50], dtype=np.float32)
    s, x, t = (np.repeat(a[k:k + 1], 8) for a in (S, X, T))
    sums = lime.map_reduce_blackscholes_sum(_dev(s), _dev(x), _dev(t), float(R), float(SIG)).cpu().numpy()
    sc, sp = oracle.blackscholes_sums(s, x, t, R, SIG)
    assert abs(sums[0] - sc) <= BS_TOL * max(abs(sc), 8.0)       # per option: 1e-5 * max(|price|, 1)
    assert abs(sums[1] - sp) <= BS_TOL * max(abs(sp), 8.0)


@pytest.mark.parametrize("grid", [1, 7, 148, 255, 256, 257, 1184])
def test_fused_sums_launch_configs(lime, grid):
    # the last CTA combines every CTA partial (up to kMaxCtas = 1184: five per thread)
    n = (1 << 20) + 3
    S, X, T = inputs.blackscholes_options(n, seed=9)
    sc, sp = oracle.blackscholes_sums(S, X, T, R, SIG)
    with lime.launch_override(grid_ctas=grid):
        sums = lime.map_reduce_blackscholes_sum(_dev(S), _dev(X), _dev(T), float(R), float(SIG)).cpu().numpy()
        again = lime.map_reduce_blackscholes_sum(_dev(S), _dev(X), _dev(T), float(R), float(SIG)).cpu().numpy()
    assert abs(sums[0] - sc) <= BS_TOL * abs(sc) and abs(sums[1] - sp) <= BS_TOL * abs(sp), grid
    assert np.array_equal(sums, again)
