"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic: it only draws the immutable
value arrays the map/reduce operators consume (§3.1 "value
arrays must be initialized at construction time"). Both sides of every parity
test take their inputs from here; nothing here depends on `oracle/` or on the
CUDA library.

Generator: SplitMix64 used as a counter-based generator. Element i of stream s
under seed q is mix(q' + (i+1)*GOLDEN) with q' = mix(q*GOLDEN + s + 1); the top
24 bits give u = k * 2^-24 in [0, 1), exactly representable in fp32.

Recipes (DESIGN.md §"Input recipe"):
  * N-Body: positions U[-1,1)^3 (x=2u-1 exact in fp32), mass m_i = 1/N,
    v0 = 0 (PAPER.md L108-110 gives float[[][4]] = x,y,z,mass but not the
    distribution; reading (v) in DESIGN.md).
  * Black-Scholes: S U[5,30], X U[1,100], T U[0.25,10] (fp32).
  * Matmul: A, Bt U[-1,1) rounded to bf16 (RNE), stored as uint16 bit patterns.
  * Reductions: see reduce_array().
"""
from __future__ import annotations

import numpy as np

GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _mix(z: np.ndarray) -> np.ndarray:
    z = z.copy()
    z ^= z >> np.uint64(30)
    z *= _M1
    z ^= z >> np.uint64(27)
    z *= _M2
    z ^= z >> np.uint64(31)
    return z


def _stream_key(seed: int, stream: int) -> np.uint64:
    with np.errstate(over="ignore"):
        k = np.array([np.uint64(seed) * GOLDEN + np.uint64(stream + 1)], dtype=np.uint64)
    return _mix(k)[0]


def splitmix64(seed: int, stream: int, n: int, offset: int = 0) -> np.ndarray:
    """n raw 64-bit draws of stream `stream` under `seed`, elements [offset, offset+n)."""
    key = _stream_key(seed, stream)
    idx = np.arange(offset + 1, offset + n + 1, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = key + idx * GOLDEN
    return _mix(z)


def uniform24(seed: int, stream: int, n: int, offset: int = 0) -> np.ndarray:
    """u in [0,1) with 24-bit granularity, as float32 (exact)."""
    bits = splitmix64(seed, stream, n, offset) >> np.uint64(40)
    return (bits.astype(np.float64) * (1.0 / 16777216.0)).astype(np.float32)


def _chunked(fn, n: int, chunk: int = 1 << 24):
    parts = [fn(o, min(chunk, n - o)) for o in range(0, n, chunk)]
    return np.concatenate(parts) if parts else fn(0, 0)


# ----------------------------------------------------------------- N-Body
def nbody_bodies(n: int, seed: int = 1) -> np.ndarray:
    """[n][4] float32 AoS (x, y, z, m): positions U[-1,1)^3, m = 1/n."""
    out = np.empty((n, 4), dtype=np.float32)
    for c in range(3):
        out[:, c] = 2.0 * uniform24(seed, c, n).astype(np.float64) - 1.0
    out[:, 3] = np.float32(1.0 / max(n, 1))
    return out


def nbody_velocities(n: int) -> np.ndarray:
    """[n][4] float32, v0 = 0 (w unused, kept 0)."""
    return np.zeros((n, 4), dtype=np.float32)


# ----------------------------------------------------------- Black-Scholes
BS_R = 0.02
BS_SIGMA = 0.30


def blackscholes_options(n: int, seed: int = 2):
    """S U[5,30], X U[1,100], T U[0.25,10] as three float32 arrays (SoA)."""
    def draw(stream, lo, hi):
        return _chunked(lambda o, m: (lo + (hi - lo) * uniform24(seed, stream, m, o).astype(np.float64)).astype(np.float32), n)
    return draw(0, 5.0, 30.0), draw(1, 1.0, 100.0), draw(2, 0.25, 10.0)


# ----------------------------------------------------------------- Matmul
def _f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    b = x.astype(np.float32).view(np.uint32).astype(np.uint64)
    rounded = (b + np.uint64(0x7FFF) + ((b >> np.uint64(16)) & np.uint64(1))) >> np.uint64(16)
    return rounded.astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (b.astype(np.uint32) << np.uint32(16)).view(np.float32)


def bf16_uniform(rows: int, cols: int, seed: int, stream: int) -> np.ndarray:
    """[rows][cols] uint16 bf16 bit patterns of U[-1,1) rounded to nearest-even."""
    n = rows * cols
    flat = _chunked(lambda o, m: _f32_to_bf16_bits(2.0 * uniform24(seed, stream, m, o) - np.float32(1.0)), n)
    return flat.reshape(rows, cols)


def matmul_operands(M: int, N: int, K: int, seed: int = 4):
    """A [M][K] and Bt [N][K] (K-major: 'map of dot products'), bf16 bits."""
    return bf16_uniform(M, K, seed, 0), bf16_uniform(N, K, seed, 1)


# ------------------------------------------------------------- Reductions
def reduce_array(n: int, dtype: str, seed: int = 6) -> np.ndarray:
    """Synthetic reduction operand.

    f32/f64: U[-1,1) scaled by 1000; i32: uniform in [-2^20, 2^20);
    i64: uniform in [-2^40, 2^40).
    """
    u = _chunked(lambda o, m: uniform24(seed, 0, m, o), n).astype(np.float64)
    if dtype == "f32":
        return ((2.0 * u - 1.0) * 1000.0).astype(np.float32)
    if dtype == "f64":
        lo = _chunked(lambda o, m: uniform24(seed, 1, m, o), n).astype(np.float64)
        return (2.0 * u - 1.0 + lo * 2.0 ** -24) * 1000.0
    raw = _chunked(lambda o, m: splitmix64(seed, 2, m, o), n)
    if dtype == "i32":
        return ((raw >> np.uint64(43)).astype(np.int64) - (1 << 20)).astype(np.int32)
    if dtype == "i64":
        return (raw >> np.uint64(23)).astype(np.int64) - (1 << 40)
    raise ValueError(dtype)


# ------------------------------------------------- Parboil CP / MRI-Q
CP_NX = CP_NY = 512        # Table 3: 1 MB float output = 512 x 512 (L353)
CP_ATOMS = 3968            # Table 3: 62 KB float4 input ~ 3968 atoms (L353)
CP_H = 0.1                 # lattice spacing (Parboil CP's default grid spacing)
CP_Z = 25.6                # slice through the middle of the 51.2-wide box


def cp_atoms(n: int = CP_ATOMS, seed: int = 7, box: float = CP_NX * CP_H) -> np.ndarray:
    """[n][4] float32 (x, y, z, q): positions U[0, box)^3, charges U[-1, 1)."""
    out = np.empty((n, 4), dtype=np.float32)
    for c in range(3):
        out[:, c] = (box * uniform24(seed, c, n).astype(np.float64)).astype(np.float32)
    out[:, 3] = (2.0 * uniform24(seed, 3, n).astype(np.float64) - 1.0).astype(np.float32)
    return out


MRIQ_VOXELS = 32768        # Table 3: 256 KB float output = 32768 x (Qr, Qi) (L353-354)
MRIQ_K = 3072              # Table 3: 432 KB input = 32768 x 3 floats + 3072 x (kx, ky, kz, phiR) ...


def mriq_kspace(n: int = MRIQ_K, seed: int = 8) -> np.ndarray:
    """[n][5] float32 (kx, ky, kz, phiR, phiI): k U[-32, 32)^3, phi U[-1, 1)^2."""
    out = np.empty((n, 5), dtype=np.float32)
    for c in range(3):
        out[:, c] = (64.0 * uniform24(seed, c, n).astype(np.float64) - 32.0).astype(np.float32)
    for c in (3, 4):
        out[:, c] = (2.0 * uniform24(seed, c, n).astype(np.float64) - 1.0).astype(np.float32)
    return out


def mriq_voxels(n: int = MRIQ_VOXELS, seed: int = 9) -> np.ndarray:
    """[n][3] float32 (x, y, z): U[-0.5, 0.5)^3."""
    out = np.empty((n, 3), dtype=np.float32)
    for c in range(3):
        out[:, c] = (uniform24(seed, c, n).astype(np.float64) - 0.5).astype(np.float32)
    return out


# ------------------------------------------------------- JG-Series / JG-Crypt
SERIES_N = 100_000          # Table 3: 780 KB of fp32 (a_n, b_n) pairs (L355; JGF size B)
CRYPT_BYTES = 3 << 20       # Table 3: 3 MB byte array (L354-355)


def crypt_data(nbytes: int = CRYPT_BYTES, seed: int = 10) -> np.ndarray:
    """nbytes uniform random bytes (uint8)."""
    return _chunked(lambda o, m: (splitmix64(seed, 0, m, o) & np.uint64(0xFF)).astype(np.uint8), nbytes)


def crypt_key(seed: int = 11) -> np.ndarray:
    """A seeded 128-bit IDEA key as eight 16-bit words."""
    return (splitmix64(seed, 0, 8) & np.uint64(0xFFFF)).astype(np.uint16)
