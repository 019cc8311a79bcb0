"""GPU parity at index spaces beyond 2^31 elements ("int64 index"; §8(c): edge cases
include the maximum sizes). Inputs are a seeded pattern of P elements repeated to n > 2^31 (P prime to
every tile and vector width), so the expected values follow from the oracle on the pattern:
elements are checked one by one in windows at the start, around index 2^31 and at the end; reductions
and sums by the period decomposition q * f(pattern) + f(pattern[:rem]) with the oracle's f. Peak device
memory ~45 GB (Black-Scholes: three inputs + two outputs of 2^31 + 3 floats)."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import BS_TOL, MATMUL_RTOL

pytestmark = pytest.mark.gpu
BIG = (1 << 31)
R, SIG = np.float32(inputs.BS_R), np.float32(inputs.BS_SIGMA)


def _windows(n):
    return [(0, 64), (BIG - 64, min(BIG + 64, n)), (n - 64, n)]


def _take(t: torch.Tensor, wins) -> np.ndarray:
    return np.concatenate([t[a:b].cpu().numpy() for a, b in wins])


def _tile(pattern: np.ndarray, n: int) -> torch.Tensor:
    p = torch.from_numpy(np.ascontiguousarray(pattern)).cuda()
    return p.repeat(n // len(pattern) + 1)[:n].contiguous()


def _free():
    torch.cuda.synchronize()
    torch.cuda.empty_cache()


def _wrap32(v: int) -> int:
    v &= 0xFFFFFFFF
    return v - (1 << 32) if v >= (1 << 31) else v


def test_reduce_i32_beyond_2_31(lime):
    n, P = BIG + 37, 1009
    pat = inputs.reduce_array(P, "i32", seed=41)
    x = _tile(pat, n)
    # plant extremes past index 2^31: only an int64 index reaches them
    x[BIG + 5] = torch.iinfo(torch.int32).min
    x[n - 1] = torch.iinfo(torch.int32).max
    q, rem = divmod(n, P)
    s = q * oracle.reduce("sum", pat, "i32") + oracle.reduce("sum", pat[:rem], "i32")
    s += -(2 ** 31) - int(pat[(BIG + 5) % P]) + (2 ** 31 - 1) - int(pat[(n - 1) % P])
    assert lime.reduce_sum(x).item() == _wrap32(s)
    assert lime.reduce_min(x).item() == -(2 ** 31)
    assert lime.reduce_max(x).item() == 2 ** 31 - 1
    del x
    _free()


def test_reduce_f32_sum_beyond_2_31(lime):
    n, P = BIG + 37, 1009
    pat = inputs.reduce_array(P, "f32", seed=42)
    x = _tile(pat, n)
    q, rem = divmod(n, P)
    ref = q * oracle.reduce("sum", pat, "f32") + oracle.reduce("sum", pat[:rem], "f32")
    tol = 1e-5 * (q + 1) * float(np.abs(pat.astype(np.float64)).sum())
    assert abs(lime.reduce_sum(x).item() - ref) <= tol
    del x
    _free()


def test_blackscholes_beyond_2_31(lime):
    n, P = BIG + 3, (1 << 20) + 7
    Sp, Xp, Tp = inputs.blackscholes_options(P, seed=43)
    S, X, T = _tile(Sp, n), _tile(Xp, n), _tile(Tp, n)
    # fused map+reduce first (no outputs allocated), by the period decomposition
    sums = lime.map_reduce_blackscholes_sum(S, X, T, float(R), float(SIG)).cpu().numpy()
    q, rem = divmod(n, P)
    fc, fp = oracle.blackscholes_sums(Sp, Xp, Tp, R, SIG)
    rc, rp = oracle.blackscholes_sums(Sp[:rem], Xp[:rem], Tp[:rem], R, SIG)
    sc, sp = q * fc + rc, q * fp + rp
    assert abs(sums[0] - sc) <= BS_TOL * abs(sc), (sums[0], sc)
    assert abs(sums[1] - sp) <= BS_TOL * abs(sp), (sums[1], sp)
    # the map, element by element in the windows
    call, put = lime.map_blackscholes(S, X, T, float(R), float(SIG))
    wins = _windows(n)
    k = np.concatenate([np.arange(a, b) for a, b in wins]) % P
    c_ref, p_ref = oracle.blackscholes(Sp[k], Xp[k], Tp[k], R, SIG)
    c, p = _take(call, wins).astype(np.float64), _take(put, wins).astype(np.float64)
    assert (np.abs(c - c_ref) / np.maximum(np.abs(c_ref), 1.0)).max() <= BS_TOL
    assert (np.abs(p - p_ref) / np.maximum(np.abs(p_ref), 1.0)).max() <= BS_TOL
    del S, X, T, call, put
    _free()


def test_mandelbrot_frame_beyond_2_31_pixels(lime):
    W, H, it = 65536, 32769, 24                  # W * H = 2^31 + 2^16 pixels; row 32768 starts at 2^31
    dx, dy = 3.0 / W, 3.0 / 32768
    out = lime.map_mandelbrot(W, H, -2.0, -1.5, dx, dy, it)
    for r in (0, 16384, 32767, 32768):
        ref = oracle.mandelbrot(W, H, r, 1, 1, -2.0, -1.5, dx, dy, it)
        assert np.array_equal(out[r:r + 1].cpu().numpy(), ref), r
    del out
    _free()


def test_matmul_output_beyond_2_31_entries(lime):
    # ragged M (not a multiple of the 256-row pair tile), ragged K (72 = 64 + 8), N % 4 == 0 (wide
    # pair tile, TMA-store epilogue): C has 65600 x 32776 = 2^31 + 51,200 entries
    M, N, K = 65600, 32776, 72
    A, Bt = inputs.matmul_operands(M, N, K, seed=44)
    Ad = torch.from_numpy(np.ascontiguousarray(A).view(np.int16)).cuda().view(torch.bfloat16)
    Bd = torch.from_numpy(np.ascontiguousarray(Bt).view(np.int16)).cuda().view(torch.bfloat16)
    C = lime.map_matmul_bf16(Ad, Bd)
    rng = np.random.default_rng(44)
    cross = BIG // N                                       # the row in which the linear index passes 2^31
    rows = np.concatenate([[0, 1, 255, 256], np.arange(cross - 2, cross + 3), np.arange(M - 70, M)])
    cols = np.concatenate([np.arange(0, 8), rng.choice(N, 24, replace=False), np.arange(N - 8, N)])
    rr, cc = np.repeat(rows, len(cols)), np.tile(cols, len(rows))
    ref, mag = oracle.matmul_bf16_entries(A, Bt, rr, cc, threads=8)
    got = np.concatenate([C[int(r)].cpu().numpy()[cols] for r in rows]).astype(np.float64)
    assert (np.abs(got - ref) / np.maximum(mag, 1e-30)).max() <= MATMUL_RTOL
    del Ad, Bd, C
    _free()
