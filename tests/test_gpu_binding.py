"""The Python binding validates every operand and output before handing raw pointers to the C ABI
(the ABI cannot see tensor extents), and the library is safe to drive from several host
threads and streams at once."""
import threading

import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs

pytestmark = pytest.mark.gpu


def test_size_dtype_device_checks(lime):
    n = 1000
    S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=1))
    with pytest.raises(ValueError):
        lime.map_blackscholes(S, X[:-1], T, 0.02, 0.3)                       # X shorter than S
    with pytest.raises(ValueError):
        lime.map_blackscholes(S, X, T, 0.02, 0.3, call=torch.empty(n - 4, device="cuda"))
    with pytest.raises(TypeError):
        lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, out=torch.empty(2, device="cuda"))   # f32 out
    with pytest.raises(TypeError):
        lime.map_blackscholes(S, X.cpu(), T, 0.02, 0.3)                      # host operand
    b = torch.from_numpy(inputs.nbody_bodies(256, seed=2)).cuda()
    with pytest.raises(ValueError):
        lime.map_nbody(b, 1e-4, 0, 256, out=torch.empty((128, 4), device="cuda"))
    with pytest.raises(ValueError):
        lime.map_nbody_integrate(b.clone(), torch.zeros((255, 4), device="cuda"), torch.zeros_like(b), 1e-3)
    with pytest.raises(TypeError):
        lime.reduce_sum(torch.ones(100, dtype=torch.float64, device="cuda"), out=torch.empty((), device="cuda"))
    with pytest.raises(ValueError):
        lime.map_mandelbrot(64, 64, -2.0, -1.5, 3 / 64, 3 / 64, 50, out=torch.empty((63, 64), dtype=torch.int32,
                                                                                       device="cuda"))
    A = torch.zeros((64, 32), dtype=torch.bfloat16, device="cuda")
    with pytest.raises(ValueError):
        lime.map_matmul_bf16(A, torch.zeros((64, 40), dtype=torch.bfloat16, device="cuda"))
    with pytest.raises(ValueError):
        lime.map_matmul_bf16(A, A, out=torch.empty((64, 63), device="cuda"))
    with pytest.raises(ValueError):
        lime.map_series(0, 10, out=torch.empty((9, 2), device="cuda"))


def test_two_threads_two_streams(lime):
    # two host threads, each on its own stream, each running a different kernel family repeatedly
    # (the smem-attribute / occupancy caches are per device and locked; workspaces are per stream)
    b = torch.from_numpy(inputs.nbody_bodies(4096, seed=3)).cuda()
    A, Bt = inputs.matmul_operands(512, 512, 256, seed=3)
    Ad = torch.from_numpy(A.view(np.int16)).cuda().view(torch.bfloat16)
    Bd = torch.from_numpy(Bt.view(np.int16)).cuda().view(torch.bfloat16)
    ref_acc = lime.map_nbody(b, 1e-4).clone()
    ref_mm = lime.map_matmul_bf16(Ad, Bd).clone()
    ref_series = lime.map_series(0, 5000).clone()
    torch.cuda.synchronize()
    errors = []

    def run(kind):
        try:
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                for _ in range(20):
                    if kind == 0:
                        out = lime.map_nbody(b, 1e-4)
                        ok = torch.equal(out, ref_acc)
                    elif kind == 1:
                        out = lime.map_matmul_bf16(Ad, Bd)
                        ok = torch.equal(out, ref_mm)
                    else:
                        out = lime.map_series(0, 5000)
                        ok = torch.equal(out, ref_series)
                    s.synchronize()
                    if not ok:
                        errors.append(kind)
        except Exception as e:  # noqa: BLE001
            errors.append(repr(e))

    ts = [threading.Thread(target=run, args=(k,)) for k in (0, 1, 2)]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not errors, errors


def test_series_tables_first_use_on_side_stream(lime):
    # the JG-Series tables are written asynchronously on the first caller's stream; calls on other
    # streams are ordered behind them by an event (no host synchronisation), so a first call on a
    # side stream followed by a call on the default stream agree with the oracle
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        a = lime.map_series(0, 64)
    b = lime.map_series(0, 64)
    torch.cuda.synchronize()
    assert torch.equal(a, b)
    ref, mag = oracle.series(0, 64)
    assert (np.abs(b.cpu().numpy() - ref) / mag[:, None]).max() <= 1e-6
