"""paper_conf_pldi_dubachcrbf12_b200 -- B200-native map `@` / reduce `!` hot path of Lime
(Dubach et al., PLDI 2012).

Thin Python binding over the C ABI of liblime.so (contract: include/lime.h). This module only
marshals arguments: torch CUDA tensors -> device pointers, the current CUDA stream, zeroed
workspaces. Every step of the path runs in the CUDA kernels; there is no CPU fallback -- if the
library is missing, load() raises.

Public API (names follow the ABI):
    map_nbody, map_nbody_integrate, map_nbody_step, nbody_simulate, nbody_simulate_host,
    map_blackscholes, map_reduce_blackscholes_sum,
    map_mandelbrot, map_matmul_bf16,
    reduce_sum / reduce_min / reduce_max (f32, f64, i32, i64),
    launch_override (context manager; PAPER.md L204-205 user-chosen thread counts).
"""
from __future__ import annotations

import contextlib
import ctypes as C
import os
import threading

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liblime.so")

STATUS = {0: "LIME_OK", 1: "LIME_ERR_INVALID_ARG", 2: "LIME_ERR_MISALIGNED", 3: "LIME_ERR_ALIASING",
          4: "LIME_ERR_UNSUPPORTED", 5: "LIME_ERR_CUDA", 6: "LIME_ERR_WORKSPACE"}


class LimeError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status


_lib = None
_lock = threading.Lock()
_p, _i64, _i32, _f, _sz, _int = C.c_void_p, C.c_int64, C.c_int32, C.c_float, C.c_size_t, C.c_int

# Signatures of every symbol include/lime.h declares (tests check the two agree).
SIGNATURES = {
    "lime_abi_version": (_int, []),
    "lime_status_str": (C.c_char_p, [_int]),
    "lime_last_error": (C.c_char_p, []),
    "lime_device_check": (_int, []),
    "lime_num_sms": (_int, []),
    "lime_set_launch_override": (None, [_int, _int, _int]),
    "lime_map_nbody_workspace_bytes": (_sz, [_i64, _i64]),
    "lime_set_nbody_variant": (_int, [_int]),
    "lime_nbody_splits": (_int, [_i64]),
    "lime_map_nbody": (_int, [_p, _i64, _i64, _i64, _f, _p, _p, _sz, _p]),
    "lime_map_nbody_integrate": (_int, [_p, _p, _p, _i64, _f, _p]),
    "lime_map_nbody_step_workspace_bytes": (_sz, [_i64, _i64]),
    "lime_map_nbody_step": (_int, [_p, _i64, _i64, _i64, _f, _f, _p, _p, _p, _sz, _p]),
    "lime_map_nbody_f64_workspace_bytes": (_sz, [_i64, _i64]),
    "lime_map_nbody_f64": (_int, [_p, _i64, _i64, _i64, C.c_double, _p, _p, _sz, _p]),
    "lime_nbody_simulate_workspace_bytes": (_sz, [_i64]),
    "lime_nbody_simulate": (_int, [_p, _p, _i64, _i32, _f, _f, _p, _sz, _p]),
    "lime_nbody_simulate_host_workspace_bytes": (_sz, [_i64]),
    "lime_nbody_simulate_host": (_int, [_p, _p, _i64, _i32, _f, _f, _p, _sz, _p]),
    "lime_map_blackscholes": (_int, [_p, _p, _p, _i64, _f, _f, _p, _p, _p]),
    "lime_map_reduce_blackscholes_sum": (_int, [_p, _p, _p, _i64, _f, _f, _p, _p, _sz, _p]),
    "lime_mandelbrot_workspace_bytes": (_sz, []),
    "lime_map_mandelbrot": (_int, [_i32, _i32, _i32, _i32, _i32, _f, _f, _f, _f, _i32, _p, _p, _sz, _p]),
    "lime_map_matmul_bf16": (_int, [_p, _p, _p, _i64, _i64, _i64, _p]),
    "lime_reduce_workspace_bytes": (_sz, []),
    "lime_map_coulomb_workspace_bytes": (_sz, [_i64, _i64]),
    "lime_map_coulomb": (_int, [_p, _i64, _i32, _i32, _i64, _i64, _f, _f, _p, _p, _sz, _p]),
    "lime_map_series_workspace_bytes": (_sz, []),
    "lime_map_series_f32": (_int, [_i64, _i64, _p, _p, _sz, _p]),
    "lime_map_series_f64": (_int, [_i64, _i64, _p, _p, _sz, _p]),
    "lime_idea_key_schedule": (None, [_p, _p, _p]),
    "lime_map_idea": (_int, [_p, _p, _i64, _p, _p]),
    "lime_map_mriq_workspace_bytes": (_sz, [_i64, _i64]),
    "lime_map_mriq": (_int, [_p, _i64, _p, _i64, _i64, _i64, _p, _p, _sz, _p]),
}
for _op in ("sum", "min", "max"):
    for _dt in ("f32", "f64", "i32", "i64"):
        SIGNATURES[f"lime_reduce_{_op}_{_dt}"] = (_int, [_p, _i64, _p, _p, _sz, _p])


def load(path: str | None = None):
    """Load liblime.so (raises if it is missing -- never falls back)."""
    global _lib
    with _lock:
        if _lib is None:
            p = path or os.environ.get("LIME_LIBRARY") or LIB_PATH   # LIME_LIBRARY: A/B builds (tools/)
            if not os.path.exists(p):
                raise RuntimeError(f"liblime.so not built ({p}); run `python -m paper_conf_pldi_dubachcrbf12_b200.build`")
            lib = C.CDLL(p)
            for name, (res, args) in SIGNATURES.items():
                fn = getattr(lib, name)
                fn.restype = res
                fn.argtypes = args
            _lib = lib
    return _lib


def _check(status: int, what: str):
    if status != 0:
        raise LimeError(status, f"{what}: {load().lime_last_error().decode()}")


def _stream(device) -> int:
    return torch.cuda.current_stream(device).cuda_stream


def _dev_tensor(t: torch.Tensor, dtype, name: str, ndim_last: int | None = None, numel: int | None = None,
                device=None):
    """Validate one operand or output: a contiguous CUDA tensor of `dtype`, optionally of shape
    [n][ndim_last], with exactly `numel` elements, on `device`. The C ABI cannot see tensor extents,
    so every size the kernels rely on is checked here (a mistake would otherwise be an out-of-bounds
    device access, not an error)."""
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if ndim_last is not None and (t.dim() != 2 or t.shape[1] != ndim_last):
        raise ValueError(f"{name} must have shape [n][{ndim_last}]")
    if numel is not None and t.numel() != numel:
        raise ValueError(f"{name} must have {numel} elements, got {t.numel()}")
    if device is not None and t.device != torch.device(device):
        raise ValueError(f"{name} is on {t.device}, expected {device} (all operands on one device)")
    return t


def _device(device) -> torch.device:
    dev = torch.device(device)
    if dev.type != "cuda":
        raise TypeError(f"device must be a CUDA device, got {dev}")
    return torch.device("cuda", dev.index if dev.index is not None else torch.cuda.current_device())


# Zero-filled, self-resetting workspaces, one per (device, stream, kind).
_ws_cache: dict = {}


def workspace(device, kind: str, nbytes: int) -> torch.Tensor:
    dev = torch.device(device)
    key = (dev.index, _stream(dev), kind)
    buf = _ws_cache.get(key)
    if buf is None or buf.numel() < nbytes:
        buf = torch.zeros(max(int(nbytes), 256), dtype=torch.uint8, device=dev)
        _ws_cache[key] = buf
    return buf


@contextlib.contextmanager
def launch_override(grid_ctas: int = 0, block_threads: int = 0, per_thread: int = 0):
    """Override the launch configuration on this thread (results never depend on it)."""
    L = load()
    L.lime_set_launch_override(grid_ctas, block_threads, per_thread)
    try:
        yield
    finally:
        L.lime_set_launch_override(0, 0, 0)


NBODY_VARIANTS = {0: "tma_smem (production)", 1: "global_scalar", 2: "global_vec", 3: "readonly_vec",
                  4: "local_scalar", 5: "local_vec", 6: "constant_vec"}


@contextlib.contextmanager
def nbody_variant(variant: int):
    """Select the N-Body staging variant (F1 ablation, Fig. 8) on this thread."""
    L = load()
    _check(L.lime_set_nbody_variant(variant), "lime_set_nbody_variant")
    try:
        yield
    finally:
        L.lime_set_nbody_variant(0)


def num_sms() -> int:
    return int(load().lime_num_sms())


# ------------------------------------------------------------------------ N-Body
def nbody_splits(n_src: int) -> int:
    return int(load().lime_nbody_splits(n_src))


def _target_range(n: int, tgt_begin: int, tgt_count: int | None) -> int:
    """Element count of the output range (the C ABI itself rejects a range outside [0, n))."""
    if tgt_count is None:
        tgt_count = n - tgt_begin
    return max(int(tgt_count), 0)


def map_nbody(bodies: torch.Tensor, eps2: float, tgt_begin: int = 0, tgt_count: int | None = None,
              out: torch.Tensor | None = None) -> torch.Tensor:
    """accel[t] for targets [tgt_begin, tgt_begin+tgt_count) of bodies [n][4] (x,y,z,m)."""
    L = load()
    _dev_tensor(bodies, torch.float32, "bodies", 4)
    n = bodies.shape[0]
    tgt_count = _target_range(n, tgt_begin, tgt_count)
    dev = bodies.device
    if out is None:
        out = torch.empty((tgt_count, 4), dtype=torch.float32, device=dev)
    _dev_tensor(out, torch.float32, "out", 4, numel=4 * tgt_count, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "nbody", L.lime_map_nbody_workspace_bytes(n, tgt_count))
        _check(L.lime_map_nbody(bodies.data_ptr(), n, tgt_begin, tgt_count, eps2, out.data_ptr(),
                                ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_nbody")
    return out


def map_nbody_f64(bodies: torch.Tensor, eps2: float, tgt_begin: int = 0, tgt_count: int | None = None,
                  out: torch.Tensor | None = None) -> torch.Tensor:
    """Double-precision N-Body map (F3): bodies [n][4] float64 -> accel [count][4] float64."""
    L = load()
    _dev_tensor(bodies, torch.float64, "bodies", 4)
    n = bodies.shape[0]
    tgt_count = _target_range(n, tgt_begin, tgt_count)
    dev = bodies.device
    if out is None:
        out = torch.empty((tgt_count, 4), dtype=torch.float64, device=dev)
    _dev_tensor(out, torch.float64, "out", 4, numel=4 * tgt_count, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "nbody64", L.lime_map_nbody_f64_workspace_bytes(n, tgt_count))
        _check(L.lime_map_nbody_f64(bodies.data_ptr(), n, tgt_begin, tgt_count, eps2, out.data_ptr(),
                                    ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_nbody_f64")
    return out


def map_nbody_integrate(pos: torch.Tensor, vel: torch.Tensor, accel: torch.Tensor, dt: float) -> None:
    """In-place semi-implicit Euler step of pos/vel ([n][4] each)."""
    L = load()
    _dev_tensor(pos, torch.float32, "pos", 4)
    n, dev = pos.shape[0], pos.device
    _dev_tensor(vel, torch.float32, "vel", 4, numel=4 * n, device=dev)
    _dev_tensor(accel, torch.float32, "accel", 4, numel=4 * n, device=dev)
    with torch.cuda.device(dev):
        _check(L.lime_map_nbody_integrate(pos.data_ptr(), vel.data_ptr(), accel.data_ptr(), n, dt, _stream(dev)),
               "lime_map_nbody_integrate")


def map_nbody_step(bodies: torch.Tensor, eps2: float, dt: float, vel: torch.Tensor, tgt_begin: int = 0,
                   tgt_count: int | None = None, out: torch.Tensor | None = None) -> torch.Tensor:
    """Fused force map + integrator for targets [tgt_begin, tgt_begin+tgt_count): updates vel
    ([count][4]) in place and returns the new positions ([count][4], out of place)."""
    L = load()
    _dev_tensor(bodies, torch.float32, "bodies", 4)
    n = bodies.shape[0]
    tgt_count = _target_range(n, tgt_begin, tgt_count)
    dev = bodies.device
    _dev_tensor(vel, torch.float32, "vel", 4, numel=4 * tgt_count, device=dev)
    if out is None:
        out = torch.empty((tgt_count, 4), dtype=torch.float32, device=dev)
    _dev_tensor(out, torch.float32, "out", 4, numel=4 * tgt_count, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "nbody_step", L.lime_map_nbody_step_workspace_bytes(n, tgt_count))
        _check(L.lime_map_nbody_step(bodies.data_ptr(), n, tgt_begin, tgt_count, eps2, dt, vel.data_ptr(),
                                     out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_nbody_step")
    return out


def nbody_simulate(pos: torch.Tensor, vel: torch.Tensor, steps: int, eps2: float, dt: float) -> None:
    """`steps` force+integrate steps on device state pos/vel ([n][4] float32, updated in place); one
    persistent launch for n <= 8192."""
    L = load()
    _dev_tensor(pos, torch.float32, "pos", 4)
    n, dev = pos.shape[0], pos.device
    _dev_tensor(vel, torch.float32, "vel", 4, numel=4 * n, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "nbody_sim", L.lime_nbody_simulate_workspace_bytes(n))
        _check(L.lime_nbody_simulate(pos.data_ptr(), vel.data_ptr(), n, steps, eps2, dt, ws.data_ptr(), ws.numel(),
                                     _stream(dev)), "lime_nbody_simulate")


def nbody_simulate_host(h_pos: torch.Tensor, h_vel: torch.Tensor, steps: int, eps2: float, dt: float,
                        device="cuda") -> None:
    """End-to-end: host (pinned) state in, `steps` force+integrate steps on the GPU, host state out."""
    L = load()
    for t, nm in ((h_pos, "h_pos"), (h_vel, "h_vel")):
        if t.is_cuda or t.dtype != torch.float32 or not t.is_contiguous() or t.dim() != 2 or t.shape[1] != 4:
            raise ValueError(f"{nm} must be a contiguous host float32 [n][4] tensor")
    if h_vel.shape[0] != h_pos.shape[0]:
        raise ValueError("h_pos and h_vel must have the same length")
    n = h_pos.shape[0]
    dev = _device(device)
    with torch.cuda.device(dev):
        ws = workspace(dev, "nbody_host", L.lime_nbody_simulate_host_workspace_bytes(n))
        _check(L.lime_nbody_simulate_host(h_pos.data_ptr(), h_vel.data_ptr(), n, steps, eps2, dt, ws.data_ptr(),
                                          ws.numel(), _stream(dev)), "lime_nbody_simulate_host")


# ------------------------------------------------------------------ Black-Scholes
def _options(S, X, T):
    _dev_tensor(S, torch.float32, "S")
    n, dev = S.numel(), S.device
    _dev_tensor(X, torch.float32, "X", numel=n, device=dev)
    _dev_tensor(T, torch.float32, "T", numel=n, device=dev)
    return n, dev


def map_blackscholes(S, X, T, r: float, sigma: float, call=None, put=None):
    L = load()
    n, dev = _options(S, X, T)
    call = torch.empty(n, dtype=torch.float32, device=dev) if call is None else call
    put = torch.empty(n, dtype=torch.float32, device=dev) if put is None else put
    _dev_tensor(call, torch.float32, "call", numel=n, device=dev)
    _dev_tensor(put, torch.float32, "put", numel=n, device=dev)
    with torch.cuda.device(dev):
        _check(L.lime_map_blackscholes(S.data_ptr(), X.data_ptr(), T.data_ptr(), n, r, sigma, call.data_ptr(),
                                       put.data_ptr(), _stream(dev)), "lime_map_blackscholes")
    return call, put


def map_reduce_blackscholes_sum(S, X, T, r: float, sigma: float, out=None) -> torch.Tensor:
    """Device float64[2] = (sum call, sum put), fused (the map is never materialised)."""
    L = load()
    n, dev = _options(S, X, T)
    out = torch.empty(2, dtype=torch.float64, device=dev) if out is None else out
    _dev_tensor(out, torch.float64, "out", numel=2, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "reduce", L.lime_reduce_workspace_bytes())
        _check(L.lime_map_reduce_blackscholes_sum(S.data_ptr(), X.data_ptr(), T.data_ptr(), n, r, sigma,
                                                  out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)),
               "lime_map_reduce_blackscholes_sum")
    return out


# ----------------------------------------------------------------- Mandelbrot
def map_mandelbrot(width: int, height: int, x0: float, y0: float, dx: float, dy: float, max_iter: int,
                   row_first: int = 0, row_stride: int = 1, row_count: int | None = None,
                   device="cuda", out=None) -> torch.Tensor:
    L = load()
    if row_count is None:
        row_count = len(range(row_first, height, row_stride))
    dev = out.device if out is not None else _device(device)
    out = torch.empty((row_count, width), dtype=torch.int32, device=dev) if out is None else out
    _dev_tensor(out, torch.int32, "out", numel=max(row_count, 0) * max(width, 0), device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "mandel", L.lime_mandelbrot_workspace_bytes())
        _check(L.lime_map_mandelbrot(width, height, row_first, row_stride, row_count, x0, y0, dx, dy, max_iter,
                                     out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_mandelbrot")
    return out


# --------------------------------------------------------------------- Matmul
def map_matmul_bf16(A: torch.Tensor, Bt: torch.Tensor, out=None) -> torch.Tensor:
    """C[M][N] fp32 = A[M][K] . Bt[N][K]^T (bf16 in, tcgen05 tensor cores)."""
    L = load()
    _dev_tensor(A, torch.bfloat16, "A")
    if A.dim() != 2:
        raise ValueError("A must be [M][K]")
    M, K = A.shape
    dev = A.device
    _dev_tensor(Bt, torch.bfloat16, "Bt", device=dev)
    if Bt.dim() != 2 or Bt.shape[1] != K:
        raise ValueError("Bt must be [N][K] with A's K")
    N = Bt.shape[0]
    out = torch.empty((M, N), dtype=torch.float32, device=dev) if out is None else out
    _dev_tensor(out, torch.float32, "out", numel=M * N, device=dev)
    with torch.cuda.device(dev):
        _check(L.lime_map_matmul_bf16(A.data_ptr(), Bt.data_ptr(), out.data_ptr(), M, N, K, _stream(dev)),
               "lime_map_matmul_bf16")
    return out


# --------------------------------------------------------- Parboil CP / MRI-Q (F2)
def map_coulomb(atoms: torch.Tensor, nx: int, ny: int, z: float, h: float, p_begin: int = 0,
                p_count: int | None = None, out=None) -> torch.Tensor:
    """Coulombic potential V[p] over lattice points [p_begin, p_begin+p_count) of an nx x ny slice."""
    L = load()
    _dev_tensor(atoms, torch.float32, "atoms", 4)
    dev = atoms.device
    p_count = _target_range(nx * ny, p_begin, p_count)
    out = torch.empty(p_count, dtype=torch.float32, device=dev) if out is None else out
    _dev_tensor(out, torch.float32, "out", numel=p_count, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "coulomb", L.lime_map_coulomb_workspace_bytes(atoms.shape[0], p_count))
        _check(L.lime_map_coulomb(atoms.data_ptr(), atoms.shape[0], nx, ny, p_begin, p_count, z, h, out.data_ptr(),
                                  ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_coulomb")
    return out


def map_mriq(kspace: torch.Tensor, voxels: torch.Tensor, x_begin: int = 0, x_count: int | None = None,
             out=None) -> torch.Tensor:
    """MRI-Q: (Qr, Qi) [x_count][2] for voxels [x_begin, x_begin+x_count)."""
    L = load()
    _dev_tensor(voxels, torch.float32, "voxels", 3)
    dev = voxels.device
    _dev_tensor(kspace, torch.float32, "kspace", 5, device=dev)
    n_x = voxels.shape[0]
    x_count = _target_range(n_x, x_begin, x_count)
    out = torch.empty((x_count, 2), dtype=torch.float32, device=dev) if out is None else out
    _dev_tensor(out, torch.float32, "out", numel=2 * x_count, device=dev)
    with torch.cuda.device(dev):
        ws = workspace(dev, "mriq", L.lime_map_mriq_workspace_bytes(kspace.shape[0], x_count))
        _check(L.lime_map_mriq(kspace.data_ptr(), kspace.shape[0], voxels.data_ptr(), n_x, x_begin, x_count,
                               out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_mriq")
    return out


# ------------------------------------------------------- JG-Series / JG-Crypt (F4)
def map_series(n0: int, count: int, dtype=torch.float32, device="cuda", out=None) -> torch.Tensor:
    """JG-Series coefficient pairs (a_n, b_n) for n in [n0, n0+count) -> [count][2]."""
    L = load()
    if dtype not in (torch.float32, torch.float64):
        raise TypeError("dtype must be float32 or float64")
    dev = out.device if out is not None else _device(device)
    out = torch.empty((count, 2), dtype=dtype, device=dev) if out is None else out
    _dev_tensor(out, dtype, "out", numel=2 * max(count, 0), device=dev)
    fn = L.lime_map_series_f64 if dtype == torch.float64 else L.lime_map_series_f32
    with torch.cuda.device(dev):
        ws = workspace(dev, "series", L.lime_map_series_workspace_bytes())
        _check(fn(n0, count, out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)), "lime_map_series")
    return out


def idea_key_schedule(key):
    """IDEA sub-keys (ek, dk), each 52 uint16 words, from a 128-bit key given as 8 uint16 words."""
    import numpy as np
    k = np.ascontiguousarray(key, dtype=np.uint16)
    if k.shape != (8,):
        raise ValueError("key must be 8 16-bit words")
    ek = np.zeros(52, dtype=np.uint16)
    dk = np.zeros(52, dtype=np.uint16)
    load().lime_idea_key_schedule(k.ctypes.data, ek.ctypes.data, dk.ctypes.data)
    return ek, dk


def map_idea(data: torch.Tensor, subkeys, out=None) -> torch.Tensor:
    """IDEA-ECB of a uint8 CUDA tensor (length % 8 == 0) with 52 sub-keys (ek encrypts, dk decrypts)."""
    import numpy as np
    L = load()
    _dev_tensor(data, torch.uint8, "data")
    dev = data.device
    z = np.ascontiguousarray(subkeys, dtype=np.uint16)
    if z.shape != (52,):
        raise ValueError("subkeys must be 52 16-bit words")
    out = torch.empty_like(data) if out is None else out
    _dev_tensor(out, torch.uint8, "out", numel=data.numel(), device=dev)
    with torch.cuda.device(dev):
        _check(L.lime_map_idea(data.data_ptr(), out.data_ptr(), data.numel(), z.ctypes.data, _stream(dev)),
               "lime_map_idea")
    return out


# ----------------------------------------------------------------- Reductions
_RED_DT = {torch.float32: "f32", torch.float64: "f64", torch.int32: "i32", torch.int64: "i64"}


def _reduce(op: str, x: torch.Tensor, out=None) -> torch.Tensor:
    L = load()
    if x.dtype not in _RED_DT:
        raise TypeError(f"unsupported dtype {x.dtype}")
    _dev_tensor(x, x.dtype, "x")
    dev = x.device
    out = torch.empty((), dtype=x.dtype, device=dev) if out is None else out
    _dev_tensor(out, x.dtype, "out", numel=1, device=dev)
    fn = getattr(L, f"lime_reduce_{op}_{_RED_DT[x.dtype]}")
    with torch.cuda.device(dev):
        ws = workspace(dev, "reduce", L.lime_reduce_workspace_bytes())
        _check(fn(x.data_ptr(), x.numel(), out.data_ptr(), ws.data_ptr(), ws.numel(), _stream(dev)),
               f"lime_reduce_{op}")
    return out


def reduce_sum(x, out=None):
    return _reduce("sum", x, out)


def reduce_min(x, out=None):
    return _reduce("min", x, out)


def reduce_max(x, out=None):
    return _reduce("max", x, out)
