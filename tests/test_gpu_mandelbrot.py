"""GPU parity: Mandelbrot escape counts, bit-exact vs the oracle's binary32 emulation."""
import os

import numpy as np
import pytest
import torch

import oracle
from testutil import golden

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("W,H,max_iter", [(256, 256, 256), (1000, 37, 100), (17, 9, 1), (64, 64, 0), (333, 200, 1024)])
def test_small_frames_bit_exact(lime, W, H, max_iter):
    dx, dy = 3.0 / W, 3.0 / H
    gpu = lime.map_mandelbrot(W, H, -2.0, -1.5, dx, dy, max_iter).cpu().numpy()
    ref = oracle.mandelbrot(W, H, 0, 1, H, -2.0, -1.5, dx, dy, max_iter)
    assert np.array_equal(gpu, ref)


def test_hand_checked_points(lime):
    g = golden("mandelbrot_points.json")
    for cx, cy, n in g["points"]:
        out = lime.map_mandelbrot(1, 1, float(np.float32(cx)), float(np.float32(cy)), 0.0, 0.0, g["max_iter"])
        assert int(out.item()) == n, (cx, cy)


def test_cyclic_shards(lime):
    W = H = 512
    d = 3.0 / 512
    full = lime.map_mandelbrot(W, H, -2.0, -1.5, d, d, 300).cpu()
    for P in (2, 3, 8):
        for r in range(P):
            sh = lime.map_mandelbrot(W, H, -2.0, -1.5, d, d, 300, row_first=r, row_stride=P).cpu()
            assert torch.equal(sh, full[r::P])


def test_full_frame_config3(lime):
    # SURVEY.md §8(c) C-mandelbrot pin 4: the whole 8192^2 frame of config 3, element by element,
    # against the oracle (threaded over host cores by interleaved rows; every row is still the plain
    # single-threaded C loop), plus the frame checksum and determinism.
    f = golden("mandelbrot_points.json")["frame"]
    W, H = f["width"], f["height"]
    gpu = lime.map_mandelbrot(W, H, f["x0"], f["y0"], f["dx"], f["dy"], f["max_iter"]).cpu().numpy()
    ref = oracle.mandelbrot(W, H, 0, 1, H, f["x0"], f["y0"], f["dx"], f["dy"], f["max_iter"],
                            threads=os.cpu_count() or 1)
    bad = np.argwhere(gpu != ref)
    assert bad.size == 0, (len(bad), bad[:8].tolist())
    assert int(gpu.sum(dtype=np.int64)) == f["checksum"]
    again = lime.map_mandelbrot(W, H, f["x0"], f["y0"], f["dx"], f["dy"], f["max_iter"]).cpu().numpy()
    assert np.array_equal(gpu, again)


@pytest.mark.parametrize("x0,y0,w,h,span,max_iter", [
    (-1.95, -0.05, 200, 100, 0.1, 3000),      # |c| straddles 1.9: lazy and tested warps side by side
    (0.2, -0.05, 256, 128, 0.1, 5000),        # near the cusp c = 1/4: long, slowly escaping orbits
    (-0.75, 0.05, 256, 64, 0.02, 4000),       # the neck between the cardioid and the period-2 bulb
    (-2.0, -1.5, 97, 61, 3.0, 1000),          # whole region, ragged tiles, max_iter not a block multiple
])
def test_lazy_escape_test_bit_exact(lime, x0, y0, w, h, span, max_iter):
    # round 2: warps whose |c| <= 1.9 skip the per-iteration test and replay the escape block
    # (DESIGN.md §5.4); the default kernel must equal the always-tested loop (launch override
    # per_thread=7) and the oracle bit for bit
    dx, dy = span / w, span / w
    gpu = lime.map_mandelbrot(w, h, x0, y0, dx, dy, max_iter).cpu().numpy()
    with lime.launch_override(per_thread=7):
        tested = lime.map_mandelbrot(w, h, x0, y0, dx, dy, max_iter).cpu().numpy()
    ref = oracle.mandelbrot(w, h, 0, 1, h, float(np.float32(x0)), float(np.float32(y0)), float(np.float32(dx)),
                            float(np.float32(dy)), max_iter, threads=os.cpu_count() or 1)
    assert np.array_equal(gpu, tested)
    assert np.array_equal(gpu, ref)
