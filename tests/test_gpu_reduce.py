"""GPU parity: reductions `!` vs the oracle (sum/min/max x f32/f64/i32/i64)."""
import math

import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs

pytestmark = pytest.mark.gpu
TORCH = {"f32": torch.float32, "f64": torch.float64, "i32": torch.int32, "i64": torch.int64}


@pytest.mark.parametrize("dt", ["f32", "f64", "i32", "i64"])
@pytest.mark.parametrize("n", [0, 1, 3, 17, 1000, (1 << 20) + 5])
@pytest.mark.parametrize("offset", [0, 1])
def test_reduce_matches_oracle(lime, dt, n, offset):
    x = inputs.reduce_array(n + offset, dt, seed=n)[offset:]
    xd = torch.from_numpy(inputs.reduce_array(n + offset, dt, seed=n)).cuda()[offset:]
    for op in ("sum", "min", "max"):
        got = getattr(lime, f"reduce_{op}")(xd).item()
        ref = oracle.reduce(op, x, dt)
        if op == "sum" and dt in ("f32", "f64"):
            tol = 1e-5 * float(np.abs(x.astype(np.float64)).sum()) if dt == "f32" else 1e-12 * float(np.abs(x).sum())
            assert abs(got - ref) <= tol + (1e-6 if dt == "f32" else 0.0), (op, dt, n, got, ref)
        else:
            assert got == ref or (math.isinf(ref) and got == ref), (op, dt, n, got, ref)


def test_reduce_exact_and_special(lime):
    ones = torch.ones(1 << 24, dtype=torch.float32, device="cuda")
    assert lime.reduce_sum(ones).item() == float(1 << 24)
    wrap = torch.tensor([2**31 - 1, 1], dtype=torch.int32, device="cuda")
    assert lime.reduce_sum(wrap).item() == -(2**31)
    z = torch.tensor([float("nan"), 3.0, -1.0, float("nan")], dtype=torch.float32, device="cuda")
    assert lime.reduce_min(z).item() == -1.0 and lime.reduce_max(z).item() == 3.0
    assert math.isnan(lime.reduce_sum(z).item())
    assert math.isnan(lime.reduce_min(torch.tensor([float("nan")], device="cuda")).item())
    e = torch.zeros(0, dtype=torch.float32, device="cuda")
    assert lime.reduce_min(e).item() == math.inf and lime.reduce_max(e).item() == -math.inf


def test_reduce_launch_configs_agree(lime):
    x = torch.from_numpy(inputs.reduce_array(1 << 20, "i64", seed=3)).cuda()
    ref = lime.reduce_sum(x).item()
    for g in (1, 7, 148, 1184):
        with lime.launch_override(grid_ctas=g):
            assert lime.reduce_sum(x).item() == ref
