"""GPU parity: tcgen05 bf16 matmul (map of dot products) vs the oracle."""
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import MATMUL_RTOL

pytestmark = pytest.mark.gpu


def _bf(a_bits):
    return torch.from_numpy(np.ascontiguousarray(a_bits).view(np.int16)).cuda().view(torch.bfloat16)


def _check(C, A, Bt, rows=None, cols=None):
    if rows is None:
        ref = oracle.matmul_bf16(A, Bt)
        mag = np.abs(inputs.bf16_bits_to_f32(A)).astype(np.float64) @ np.abs(inputs.bf16_bits_to_f32(Bt)).astype(np.float64).T
        err = np.abs(C.astype(np.float64) - ref) / np.maximum(mag, 1e-30)
        fro = np.linalg.norm(C - ref) / max(np.linalg.norm(ref), 1e-30)
        return err.max(), fro
    ref, mag = oracle.matmul_bf16_entries(A, Bt, rows, cols, threads=os.cpu_count() or 8)
    err = np.abs(C[rows, cols].astype(np.float64) - ref) / np.maximum(mag, 1e-30)
    return err.max(), 0.0


@pytest.mark.parametrize("M,N,K", [(128, 256, 64), (1, 1, 8), (33, 47, 72), (300, 520, 200), (256, 512, 1024),
                                   (1000, 1000, 1000), (8192 // 8, 64, 128), (129, 257, 4104),
                                   (300, 517, 64), (513, 1030, 136)])
def test_matmul_small_matches_oracle(lime, M, N, K):
    A, Bt = inputs.matmul_operands(M, N, K, seed=M + N + K)
    C = lime.map_matmul_bf16(_bf(A), _bf(Bt)).cpu().numpy()
    e, fro = _check(C, A, Bt)
    assert e <= MATMUL_RTOL and fro <= MATMUL_RTOL, (M, N, K, e, fro)


def test_matmul_identity_exact(lime):
    K = 256
    A = inputs.bf16_uniform(300, K, 5, 0)
    I = inputs._f32_to_bf16_bits(np.eye(K, dtype=np.float32))
    C = lime.map_matmul_bf16(_bf(A), _bf(I)).cpu().numpy()
    assert np.array_equal(C, inputs.bf16_bits_to_f32(A))


def test_matmul_config4_sampled(lime):
    M = N = K = 8192
    A, Bt = inputs.matmul_operands(M, N, K, seed=4)
    C = lime.map_matmul_bf16(_bf(A), _bf(Bt)).cpu().numpy()
    rng = np.random.default_rng(1)
    r = rng.integers(0, M, 65536)
    c = rng.integers(0, N, 65536)
    e, _ = _check(C, A, Bt, r, c)
    assert e <= MATMUL_RTOL, e
    # SURVEY.md §8(c) C-matmul pin 5: 64 full rows and 64 full columns (every tile row/column of
    # the 256x256 pair tiles is hit), in one threaded oracle call each
    rows = rng.choice(M, 64, replace=False)
    e, _ = _check(C, A, Bt, np.repeat(rows, N), np.tile(np.arange(N), 64))
    assert e <= MATMUL_RTOL, ("rows", e)
    cols = rng.choice(N, 64, replace=False)
    e, _ = _check(C, A, Bt, np.tile(np.arange(M), 64), np.repeat(cols, M))
    assert e <= MATMUL_RTOL, ("cols", e)


def test_matmul_launch_independent(lime):
    A, Bt = inputs.matmul_operands(1024, 1024, 512, seed=9)
    C0 = lime.map_matmul_bf16(_bf(A), _bf(Bt))
    for g in (1, 7, 64):
        with lime.launch_override(grid_ctas=g):
            assert torch.equal(lime.map_matmul_bf16(_bf(A), _bf(Bt)), C0)


@pytest.mark.parametrize("M,N,K", [(300, 520, 200), (1024, 1024, 512), (513, 1028, 136)])
def test_matmul_epilogue_forms_identical(lime, M, N, K):
    # the 2-CTA kernel's TMA-store epilogue (default for N % 4 == 0) and its direct st.global form
    # (launch override per_thread=3; the path N % 4 != 0 takes) write the same bits, ragged M/N included
    A, Bt = inputs.matmul_operands(M, N, K, seed=M + 3 * N + K)
    C_tma = lime.map_matmul_bf16(_bf(A), _bf(Bt))
    with lime.launch_override(per_thread=3):
        C_st = lime.map_matmul_bf16(_bf(A), _bf(Bt))
    assert torch.equal(C_tma, C_st)
    e, fro = _check(C_tma.cpu().numpy(), A, Bt)
    assert e <= MATMUL_RTOL and fro <= MATMUL_RTOL


@pytest.mark.parametrize("M,N,K", [(256, 512, 64), (300, 520, 136), (513, 1028, 200), (1024, 1536, 512),
                                   (257, 4100, 8)])
def test_matmul_tile_kernels_identical(lime, M, N, K):
    # 1-CTA 128x256, pair 256x256 (TMA-store and direct epilogues) and the wide 256x512 pair tile
    # (default for M >= 256, N >= 512) add every dot product in the same K order -> the same bits;
    # K <= 192 exercises the wide tile's deferred-H1 path with fewer K slices than held stages,
    # grid_ctas=2 (one pair doing every tile) its accumulator-release parity across many tiles
    A, Bt = inputs.matmul_operands(M, N, K, seed=M + 5 * N + K)
    C_def = lime.map_matmul_bf16(_bf(A), _bf(Bt))
    for pt in (1, 2, 3, 4):
        with lime.launch_override(per_thread=pt):
            assert torch.equal(lime.map_matmul_bf16(_bf(A), _bf(Bt)), C_def), pt
    with lime.launch_override(per_thread=4, grid_ctas=2):
        assert torch.equal(lime.map_matmul_bf16(_bf(A), _bf(Bt)), C_def)
    for g in (1, 3, 16):
        with lime.launch_override(per_thread=4, block_threads=g):
            assert torch.equal(lime.map_matmul_bf16(_bf(A), _bf(Bt)), C_def), g
    e, fro = _check(C_def.cpu().numpy(), A, Bt)
    assert e <= MATMUL_RTOL and fro <= MATMUL_RTOL
