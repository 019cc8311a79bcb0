"""Shared test helpers (paths, tolerances). No method arithmetic lives here."""
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- tolerances
NBODY_RTOL = 1e-4      # north_star: fp32 N-body forces after reordered summation
BS_TOL = 1e-5          # north_star: Black-Scholes prices, |d| <= 1e-5 * max(|ref|, 1)
MATMUL_RTOL = 1e-3     # north_star: fp32-accumulate matmul, relative to sum_k |A_ik B_jk|


def nbody_rel_err(a_gpu, a_ref, mag):
    """Per-target ||a_gpu - a_ref|| / max(||a_ref||, 1e-3 * A_i) (SURVEY.md §8(c) C-nbody)."""
    import numpy as np
    a_gpu = np.asarray(a_gpu, dtype=np.float64)[:, :3]
    num = np.linalg.norm(a_gpu - a_ref, axis=1)
    den = np.maximum(np.linalg.norm(a_ref, axis=1), 1e-3 * np.asarray(mag))
    den = np.where(den == 0, 1.0, den)
    return num / den
