"""C-ABI checks that need no GPU: liblime.so loads, exports every symbol include/lime.h declares,
and rejects bad arguments in the documented order before touching the device."""
import ctypes as C
import os
import re
import subprocess

import pytest

import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import build as lime_build
from testutil import ROOT

HEADER = os.path.join(ROOT, "include", "lime.h")


@pytest.fixture(scope="module")
def L():
    lime_build.build()
    return lime.load()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(lime_[a-z0-9_]+)\s*\(", src)))


def test_header_declares_expected_surface():
    names = declared_functions()
    for must in ("lime_map_nbody", "lime_map_nbody_integrate", "lime_map_blackscholes",
                 "lime_map_reduce_blackscholes_sum", "lime_map_mandelbrot", "lime_map_matmul_bf16",
                 "lime_reduce_sum_f32", "lime_reduce_max_i64", "lime_nbody_simulate_host",
                 "lime_nbody_simulate"):
        assert must in names


def test_every_declared_symbol_is_exported_and_bound(L):
    lib = os.path.join(os.path.dirname(lime.__file__), "liblime.so")
    nm = subprocess.run(["nm", "-D", "--defined-only", lib], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r" T (lime_[a-z0-9_]+)$", nm, flags=re.M))
    for name in declared_functions():
        assert name in exported, name
        assert name in lime.SIGNATURES, name
        assert getattr(L, name) is not None
    assert set(lime.SIGNATURES) == set(declared_functions())


def test_version_and_status_strings(L):
    assert L.lime_abi_version() == 1
    assert L.lime_status_str(0) == b"LIME_OK"
    assert L.lime_status_str(3) == b"LIME_ERR_ALIASING"
    assert L.lime_status_str(99) == b"LIME_ERR_UNKNOWN"


# Fake, never-dereferenced device addresses: validation is pure host arithmetic.
A0 = 0x7F0000000000
A1 = 0x7F0010000000
WS = 0x7F0020000000


def test_nbody_validation_order(L):
    f = L.lime_map_nbody
    assert f(A0, -1, 0, 0, 1e-4, A1, WS, 1 << 20, None) == 1          # n < 0
    assert f(A0, 10, 5, 6, 1e-4, A1, WS, 1 << 20, None) == 1          # shard outside [0, n)
    assert f(A0, 10, 0, 10, 0.0, A1, WS, 1 << 20, None) == 1          # eps2 <= 0
    assert f(A0, 10, 0, 10, float("nan"), A1, WS, 1 << 20, None) == 1
    assert f(A0, 10, 0, 0, 1e-4, A1, WS, 1 << 20, None) == 0          # empty map: no-op
    assert f(None, 10, 0, 10, 1e-4, A1, WS, 1 << 20, None) == 1       # null
    assert f(A0 + 4, 10, 0, 10, 1e-4, A1, WS, 1 << 20, None) == 2     # misaligned
    assert f(A0, 10, 0, 10, 1e-4, A0 + 32, WS, 1 << 20, None) == 3    # accel overlaps bodies
    assert b"overlaps" in L.lime_last_error()


def test_nbody_step_validation(L):
    # lime_map_nbody_step (round 2): arguments -> alignment -> aliasing -> device, like lime_map_nbody
    f = L.lime_map_nbody_step
    wsb = L.lime_map_nbody_step_workspace_bytes(10, 10)
    assert wsb >= L.lime_map_nbody_workspace_bytes(10, 10)
    assert L.lime_map_nbody_step_workspace_bytes(1 << 20, 1 << 17) >= (1 << 17) * 16   # accel for the general path
    assert f(A0, 10, 5, 6, 1e-4, 1e-3, A1, A1 + 512, WS, wsb, None) == 1          # shard outside [0, n)
    assert f(A0, 10, 0, 10, 1e-4, float("nan"), A1, A1 + 512, WS, wsb, None) == 1  # dt not finite
    assert f(A0, 10, 0, 0, 1e-4, 1e-3, A1, A1 + 512, WS, wsb, None) == 0          # empty shard: no-op
    assert f(A0, 10, 0, 10, 1e-4, 1e-3, None, A1 + 512, WS, wsb, None) == 1       # null vel
    assert f(A0, 10, 0, 10, 1e-4, 1e-3, A1 + 8, A1 + 512, WS, wsb, None) == 2     # misaligned vel
    assert f(A0, 10, 0, 10, 1e-4, 1e-3, A1, A0 + 16, WS, wsb, None) == 3          # pos_out overlaps bodies
    assert f(A0, 10, 0, 10, 1e-4, 1e-3, A1, A1 + 64, WS, wsb, None) == 3          # vel overlaps pos_out


def test_integrate_and_bs_validation(L):
    assert L.lime_map_nbody_integrate(A0, A0 + 64, A1, 8, 1e-3, None) == 3      # pos/vel overlap
    assert L.lime_map_nbody_integrate(A0, A1, WS, 8, float("inf"), None) == 1   # dt not finite
    g = L.lime_map_blackscholes
    assert g(A0, A0 + 4096, A0 + 8192, 16, 0.02, 0.0, A1, A1 + 4096, None) == 1   # sigma <= 0
    assert g(A0, A0 + 4096, A0 + 8192, 16, 0.02, 0.3, A1, A1 + 4096 + 8, None) == 2
    assert g(A0, A0 + 4096, A0 + 8192, 16, 0.02, 0.3, A0 + 4096, A1, None) == 3   # call == X
    assert g(A0, A0 + 4096, A0 + 8192, 0, 0.02, 0.3, A1, A1, None) == 0          # n = 0


def test_simulate_validation(L):
    f = L.lime_nbody_simulate
    wsb = L.lime_nbody_simulate_workspace_bytes(64)
    assert wsb >= 64 * 16 + 256
    assert f(A0, A1, 64, -1, 1e-4, 1e-3, WS, wsb, None) == 1                    # steps < 0
    assert f(A0, A1, 64, 2, 0.0, 1e-3, WS, wsb, None) == 1                      # eps2 <= 0
    assert f(A0, A1, 64, 2, 1e-4, float("nan"), WS, wsb, None) == 1             # dt not finite
    assert f(A0, A1, 0, 2, 1e-4, 1e-3, None, 0, None) == 0                      # n = 0: no-op
    assert f(A0, None, 64, 2, 1e-4, 1e-3, WS, wsb, None) == 1                   # null vel
    assert f(A0 + 8, A1, 64, 2, 1e-4, 1e-3, WS, wsb, None) == 2                 # misaligned
    assert f(A0, A0 + 512, 64, 2, 1e-4, 1e-3, WS, wsb, None) == 3               # pos/vel overlap
    assert f(A0, A1, 64, 2, 1e-4, 1e-3, A1 + 16, wsb, None) == 3                # ws overlaps vel
    h = L.lime_nbody_simulate_host
    assert L.lime_nbody_simulate_host_workspace_bytes(64) >= wsb + 64 * 32
    assert h(A0, A0 + 64, 8, 1, 1e-4, 1e-3, WS, 1 << 20, None) == 3             # h_pos/h_vel overlap


def test_mandelbrot_matmul_reduce_validation(L):
    m = L.lime_map_mandelbrot
    assert m(0, 8, 0, 1, 8, -2, -1.5, 0.1, 0.1, 10, A1, WS, 256, None) == 1       # width 0
    assert m(8, 8, 0, 2, 5, -2, -1.5, 0.1, 0.1, 10, A1, WS, 256, None) == 1       # rows beyond height
    assert m(8, 8, 0, 1, 8, -2, -1.5, 0.1, 0.1, -1, A1, WS, 256, None) == 1       # max_iter < 0
    mm = L.lime_map_matmul_bf16
    assert mm(A0, A1, WS, 16, 16, 12, None) == 1                                    # K % 8 != 0
    assert mm(A0 + 2, A1, WS, 16, 16, 16, None) == 2
    assert mm(A0, A1, A0 + 16, 16, 16, 16, None) == 3                               # C overlaps A
    assert mm(A0, A1, WS, 1 << 31, 16, 16, None) == 1                               # M = 2^31 (int32 rows)
    assert mm(A0, A1, WS, 16, (1 << 31) - 256, 16, None) == 1                       # padded N overflows
    assert mm(A0, A1, WS, 1 << 30, 1 << 30, 16, None) == 1                          # 2^40 tiles
    r = L.lime_reduce_sum_f32
    assert r(A0, -1, A1, WS, 1 << 16, None) == 1
    assert r(A0 + 2, 10, A1, WS, 1 << 16, None) == 2                                # f32 at 2-B offset
    assert r(A0, 10, A0 + 8, WS, 1 << 16, None) == 3                                # out inside x


def test_no_device_reports_unsupported(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    # valid arguments reach the device check, which fails cleanly without a GPU
    assert L.lime_device_check() == 4
    assert L.lime_map_nbody(A0, 10, 0, 10, 1e-4, A1, WS, 1 << 20, None) == 4


def test_workspace_queries_and_split_rule(L):
    # splits depend on n_src only (deterministic order across shards/launches)
    # n_src <= 8192: 64-body chunks, <= 64 splits; larger: 256-body chunks, <= 32 splits
    assert L.lime_nbody_splits(1) == 1 and L.lime_nbody_splits(64) == 1
    assert L.lime_nbody_splits(65) == 2 and L.lime_nbody_splits(129) == 3
    assert L.lime_nbody_splits(4096) == 64
    assert L.lime_nbody_splits(4097) == 33          # 65 chunks, 2 per split
    assert L.lime_nbody_splits(8192) == 64          # 128 chunks, 2 per split
    assert L.lime_nbody_splits(8193) == 17          # 33 chunks of 256, 2 per split
    assert L.lime_nbody_splits(1 << 20) == 32
    assert L.lime_map_nbody_workspace_bytes(1 << 20, 1 << 17) >= 32 * (1 << 17) * 16
    assert L.lime_reduce_workspace_bytes() >= 256
    assert L.lime_mandelbrot_workspace_bytes() >= 8
