"""CPU oracle for the Lime map/reduce hot path -- TEST INFRASTRUCTURE ONLY.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` and
`--impl reference` legs may import this package. The product package
(`paper_conf_pldi_dubachcrbf12_b200`) never imports it; the two share no code.

The arithmetic lives in `lime_oracle.c` (plain single-threaded C, fp64, built
with -ffp-contract=off). This module only compiles it and marshals numpy
arrays through ctypes; each wrapper names the C function (and so the PAPER.md
passage cited there) that it calls.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "lime_oracle.c")
_LIB = os.path.join(_HERE, "_build", "liblime_oracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-msse2"]

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liblime_oracle.so (gcc, no CUDA). Returns the library path."""
    os.makedirs(os.path.dirname(_LIB), exist_ok=True)
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            _lib = C.CDLL(build())
            _declare(_lib)
    return _lib


_p = C.c_void_p
_i64 = C.c_int64
_i32 = C.c_int32
_f = C.c_float
_d = C.c_double


def _declare(L):
    sig = {
        "oracle_abi_version": (C.c_int, []),
        "oracle_nbody_accel": (None, [_p, _i64, _i64, _i64, _f, _p, _p]),
        "oracle_nbody_integrate": (None, [_p, _p, _p, _i64, _f, _p, _p]),
        "oracle_nbody_accel_f64": (None, [_p, _i64, _i64, _i64, _d, _p, _p]),
        "oracle_normal_cdf": (_d, [_d]),
        "oracle_blackscholes": (None, [_p, _p, _p, _i64, _f, _f, _p, _p]),
        "oracle_blackscholes_sums": (None, [_p, _p, _p, _i64, _f, _f, _p]),
        "oracle_mandelbrot_point": (_i32, [_f, _f, _i32]),
        "oracle_mandelbrot": (None, [_i32, _i32, _i32, _i32, _i32, _f, _f, _f, _f, _i32, _p]),
        "oracle_matmul_bf16": (None, [_p, _p, _i64, _i64, _i64, _p]),
        "oracle_matmul_bf16_entries": (None, [_p, _p, _i64, _p, _p, _i64, _p, _p]),
        "oracle_coulomb_potential": (None, [_p, _i64, _i32, _i32, _i32, _f, _f, _p, _p]),
        "oracle_mriq": (None, [_p, _i64, _p, _i64, _p, _p]),
        "oracle_series": (None, [_i64, _i64, _i32, _p, _p]),
        "oracle_idea_keys": (None, [_p, _p, _p]),
        "oracle_idea": (None, [_p, _p, _i64, _p]),
        "oracle_reduce_sum_f32": (_d, [_p, _i64]),
        "oracle_reduce_sum_f64": (_d, [_p, _i64]),
        "oracle_reduce_sum_i32": (_i32, [_p, _i64]),
        "oracle_reduce_sum_i64": (_i64, [_p, _i64]),
        "oracle_reduce_min_f32": (_f, [_p, _i64]),
        "oracle_reduce_max_f32": (_f, [_p, _i64]),
        "oracle_reduce_min_f64": (_d, [_p, _i64]),
        "oracle_reduce_max_f64": (_d, [_p, _i64]),
        "oracle_reduce_min_i32": (_i32, [_p, _i64]),
        "oracle_reduce_max_i32": (_i32, [_p, _i64]),
        "oracle_reduce_min_i64": (_i64, [_p, _i64]),
        "oracle_reduce_max_i64": (_i64, [_p, _i64]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args


def _ptr(a: np.ndarray | None):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


# ------------------------------------------------------------------ N-Body
def nbody_accel(bodies, eps2: float, tgt_begin: int = 0, tgt_count: int | None = None,
                with_mag: bool = False):
    """oracle_nbody_accel: a_i (double [count][3]); optionally A_i ([count])."""
    b = _c(bodies, np.float32).reshape(-1, 4)
    n = b.shape[0]
    if tgt_count is None:
        tgt_count = n - tgt_begin
    acc = np.zeros((tgt_count, 3), dtype=np.float64)
    mag = np.zeros(tgt_count, dtype=np.float64) if with_mag else None
    lib().oracle_nbody_accel(_ptr(b), n, tgt_begin, tgt_count, float(eps2), _ptr(acc), _ptr(mag))
    return (acc, mag) if with_mag else acc


def nbody_accel_f64(bodies, eps2: float, tgt_begin: int = 0, tgt_count: int | None = None,
                    with_mag: bool = False):
    """oracle_nbody_accel_f64: double bodies [n][4] -> a_i double [count][3] (optionally A_i)."""
    b = _c(bodies, np.float64).reshape(-1, 4)
    n = b.shape[0]
    if tgt_count is None:
        tgt_count = n - tgt_begin
    acc = np.zeros((tgt_count, 3), dtype=np.float64)
    mag = np.zeros(tgt_count, dtype=np.float64) if with_mag else None
    lib().oracle_nbody_accel_f64(_ptr(b), n, tgt_begin, tgt_count, float(eps2), _ptr(acc), _ptr(mag))
    return (acc, mag) if with_mag else acc


def nbody_accel_rows(bodies, eps2: float, rows, threads: int = 1, with_mag: bool = True):
    """Accelerations of an arbitrary list of targets (each one oracle call), optionally
    spread over `threads` host threads (the C code itself stays single-threaded)."""
    b = _c(bodies, np.float32).reshape(-1, 4)
    n = b.shape[0]
    rows = np.asarray(rows, dtype=np.int64)
    acc = np.zeros((len(rows), 3), dtype=np.float64)
    mag = np.zeros(len(rows), dtype=np.float64)
    L = lib()

    def work(lo, hi):
        for k in range(lo, hi):
            L.oracle_nbody_accel(_ptr(b), n, int(rows[k]), 1, float(eps2),
                                 acc[k:k + 1].ctypes.data, mag[k:k + 1].ctypes.data)

    _parallel(work, len(rows), threads)
    return (acc, mag) if with_mag else acc


def nbody_integrate(pos, vel, accel, dt: float):
    """oracle_nbody_integrate: (pos', vel') as double [n][4]."""
    p, v, a = (_c(x, np.float32).reshape(-1, 4) for x in (pos, vel, accel))
    n = p.shape[0]
    po = np.zeros((n, 4), dtype=np.float64)
    vo = np.zeros((n, 4), dtype=np.float64)
    lib().oracle_nbody_integrate(_ptr(p), _ptr(v), _ptr(a), n, float(dt), _ptr(po), _ptr(vo))
    return po, vo


# ----------------------------------------------------------- Black-Scholes
def normal_cdf(x: float) -> float:
    """oracle_normal_cdf: N(x) = erfc(-x/sqrt 2)/2."""
    return float(lib().oracle_normal_cdf(float(x)))


def blackscholes(S, X, T, r: float, sigma: float):
    """oracle_blackscholes: (call, put) double arrays."""
    S, X, T = (_c(a, np.float32) for a in (S, X, T))
    n = S.shape[0]
    call = np.zeros(n, dtype=np.float64)
    put = np.zeros(n, dtype=np.float64)
    lib().oracle_blackscholes(_ptr(S), _ptr(X), _ptr(T), n, float(r), float(sigma), _ptr(call), _ptr(put))
    return call, put


def blackscholes_sums(S, X, T, r: float, sigma: float):
    """oracle_blackscholes_sums: (sum call, sum put), compensated double."""
    S, X, T = (_c(a, np.float32) for a in (S, X, T))
    out = np.zeros(2, dtype=np.float64)
    lib().oracle_blackscholes_sums(_ptr(S), _ptr(X), _ptr(T), S.shape[0], float(r), float(sigma), _ptr(out))
    return float(out[0]), float(out[1])


# -------------------------------------------------------------- Mandelbrot
def mandelbrot_point(cx: float, cy: float, max_iter: int) -> int:
    return int(lib().oracle_mandelbrot_point(float(cx), float(cy), int(max_iter)))


def mandelbrot(width, height, row_first, row_stride, row_count, x0, y0, dx, dy, max_iter,
               threads: int = 1):
    """oracle_mandelbrot: int32 [row_count][width]; `threads` splits rows over host
    threads (each call is the single-threaded C loop on a disjoint row range)."""
    out = np.zeros((row_count, width), dtype=np.int32)
    L = lib()
    threads = max(1, min(threads, row_count if row_count > 0 else 1))
    if threads == 1:
        if row_count > 0:
            L.oracle_mandelbrot(width, height, row_first, row_stride, row_count, float(x0), float(y0),
                                float(dx), float(dy), max_iter, out.ctypes.data)
        return out

    # Thread k takes rows k, k + threads, ... (the escape time varies strongly from row to row, so
    # interleaving balances the threads); each part is the same single-threaded C loop over a
    # row set with stride row_stride * threads, written into its own dense array.
    def work(k):
        cnt = len(range(k, row_count, threads))
        if cnt:
            part = np.zeros((cnt, width), dtype=np.int32)
            L.oracle_mandelbrot(width, height, row_first + k * row_stride, row_stride * threads, cnt,
                                float(x0), float(y0), float(dx), float(dy), max_iter, part.ctypes.data)
            out[k::threads] = part

    ts = [threading.Thread(target=work, args=(k,)) for k in range(threads)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    return out


# ----------------------------------------------------------------- Matmul
def matmul_bf16(A_bits, Bt_bits):
    """oracle_matmul_bf16: C double [M][N]."""
    A = _c(A_bits, np.uint16)
    Bt = _c(Bt_bits, np.uint16)
    M, K = A.shape
    N = Bt.shape[0]
    Cm = np.zeros((M, N), dtype=np.float64)
    lib().oracle_matmul_bf16(_ptr(A), _ptr(Bt), M, N, K, _ptr(Cm))
    return Cm


def matmul_bf16_entries(A_bits, Bt_bits, rows, cols, threads: int = 1):
    """oracle_matmul_bf16_entries: (C[rows,cols], sum_k |A_ik Bt_jk|) sampled."""
    A = _c(A_bits, np.uint16)
    Bt = _c(Bt_bits, np.uint16)
    K = A.shape[1]
    rows = _c(rows, np.int64)
    cols = _c(cols, np.int64)
    n = rows.shape[0]
    Cv = np.zeros(n, dtype=np.float64)
    Av = np.zeros(n, dtype=np.float64)
    L = lib()

    def work(lo, hi):
        if hi > lo:
            L.oracle_matmul_bf16_entries(_ptr(A), _ptr(Bt), K, rows[lo:hi].ctypes.data,
                                         cols[lo:hi].ctypes.data, hi - lo,
                                         Cv[lo:hi].ctypes.data, Av[lo:hi].ctypes.data)

    _parallel(work, n, threads, chunked=True)
    return Cv, Av


# ------------------------------------------------------------ Parboil CP / MRI-Q
def coulomb_potential(atoms, nx: int, ny: int, z: float, h: float, iy0: int = 0, threads: int = 1):
    """oracle_coulomb_potential: V double [ny][nx] for lattice rows iy0..iy0+ny-1, and
    sum_j |q_j| / r_j; `threads` splits the rows (each part is the single-threaded C loop)."""
    a = _c(atoms, np.float32).reshape(-1, 4)
    V = np.zeros((ny, nx), dtype=np.float64)
    M = np.zeros((ny, nx), dtype=np.float64)
    L = lib()

    def work(lo, hi):
        if hi > lo:
            L.oracle_coulomb_potential(a.ctypes.data, a.shape[0], nx, iy0 + lo, hi - lo, float(z), float(h),
                                       V[lo:hi].ctypes.data, M[lo:hi].ctypes.data)

    _parallel(work, ny, threads)
    return V, M


def mriq(kspace, voxels, threads: int = 1):
    """oracle_mriq: (Qr, Qi) double [X][2] and sum_k phiMag_k [X]."""
    ks = _c(kspace, np.float32).reshape(-1, 5)
    vx = _c(voxels, np.float32).reshape(-1, 3)
    out = np.zeros((vx.shape[0], 2), dtype=np.float64)
    mag = np.zeros(vx.shape[0], dtype=np.float64)
    L = lib()

    def work(lo, hi):
        if hi > lo:
            L.oracle_mriq(ks.ctypes.data, ks.shape[0], vx[lo:hi].ctypes.data, hi - lo,
                          out[lo:hi].ctypes.data, mag[lo:hi].ctypes.data)

    _parallel(work, vx.shape[0], threads)
    return out, mag


# ----------------------------------------------------------- JG-Series / JG-Crypt (F4)
def series(n0: int, count: int, m: int = 1000, threads: int = 1):
    """oracle_series: (a_n, b_n) double [count][2] and the bound T[|f|] [count]."""
    out = np.zeros((count, 2), dtype=np.float64)
    mag = np.zeros(count, dtype=np.float64)
    L = lib()

    def work(lo, hi):
        if hi > lo:
            L.oracle_series(n0 + lo, hi - lo, m, out[lo:hi].ctypes.data, mag[lo:hi].ctypes.data)

    _parallel(work, count, threads)
    return out, mag


def idea_keys(key):
    """oracle_idea_keys: (encryption, decryption) sub-keys, uint16 [52] each."""
    k = _c(key, np.uint16)
    ek = np.zeros(52, dtype=np.uint16)
    dk = np.zeros(52, dtype=np.uint16)
    lib().oracle_idea_keys(_ptr(k), _ptr(ek), _ptr(dk))
    return ek, dk


def idea(data, subkeys):
    """oracle_idea: IDEA-ECB of a byte array (len % 8 == 0) with the given 52 sub-keys."""
    d = _c(data, np.uint8)
    z = _c(subkeys, np.uint16)
    out = np.zeros_like(d)
    lib().oracle_idea(_ptr(d), _ptr(out), d.shape[0], _ptr(z))
    return out


# ------------------------------------------------------------- Reductions
_RED_DT = {"f32": np.float32, "f64": np.float64, "i32": np.int32, "i64": np.int64}


def reduce(op: str, x, dtype: str):
    """oracle_reduce_<op>_<dtype>."""
    a = _c(x, _RED_DT[dtype])
    return getattr(lib(), f"oracle_reduce_{op}_{dtype}")(_ptr(a), a.shape[0])


# ---------------------------------------------------------------- helpers
def _parallel(work, n: int, threads: int, chunked: bool = False):
    threads = max(1, min(threads, n if n > 0 else 1))
    if threads == 1:
        work(0, n)
        return
    bounds = np.linspace(0, n, threads + 1).astype(int)
    ts = [threading.Thread(target=work, args=(int(bounds[k]), int(bounds[k + 1]))) for k in range(threads)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
