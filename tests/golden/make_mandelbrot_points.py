#!/usr/bin/env python
"""Reproduce the Mandelbrot goldens of tests/golden/mandelbrot_points.json from independent code.

Provenance note: the near-boundary escape counts (33, 315, 30, 97) and the
8192^2 frame checksum 11,856,987,162 were first measured by the survey's throw-away probe
(SURVEY.md Appendix A). This script recomputes them with code that shares nothing with either
side of the parity test: not oracle/lime_oracle.c, not the CUDA kernels -- numpy binary32 scalars
and arrays, one IEEE op per numpy operation (numpy never contracts a*b+c into an FMA), following
DESIGN.md reading R7 literally:

    cx = x0 + px*dx, cy = y0 + py*dy                      (binary32)
    z0 = 0; count = 0
    while count < max_iter and not (x*x + y*y > 4):        (test BEFORE the update)
        x, y = (x*x - y*y) + cx, (x*y + x*y) + cy
        count += 1

The points are also checked against their closed-form/hand-derived values (c = 1 -> 3 updates;
Boll/Klebanoff: n ~ pi/eps near c = -3/4 + i eps and n ~ pi/sqrt(c - 1/4) past the cusp).

    python tests/golden/make_mandelbrot_points.py            # points only (a second)
    python tests/golden/make_mandelbrot_points.py --frame    # + the 8192^2 checksum (minutes, all cores)
"""
from __future__ import annotations

import json
import math
import multiprocessing as mp
import os
import sys

import numpy as np

f32 = np.float32
HERE = os.path.dirname(os.path.abspath(__file__))


def escape_count(cx: float, cy: float, max_iter: int) -> int:
    """R7 for one point, numpy float32 scalars (each op rounds once to binary32)."""
    cx, cy = f32(cx), f32(cy)
    x = y = f32(0.0)
    four = f32(4.0)
    n = 0
    while n < max_iter:
        xx, yy = x * x, y * y
        if xx + yy > four:
            break
        xy = x * y
        x, y = (xx - yy) + cx, (xy + xy) + cy
        n += 1
    return n


def frame_rows(args) -> int:
    """Sum of the escape counts of image rows [r0, r1) (vectorised over a row, binary32)."""
    r0, r1, width, x0, y0, dx, dy, max_iter = args
    px = np.arange(width, dtype=np.float32)
    cxs = f32(x0) + px * f32(dx)
    total = 0
    with np.errstate(over="ignore", invalid="ignore"):
        for r in range(r0, r1):
            cy0 = f32(y0) + f32(r) * f32(dy)
            cx = cxs.copy()
            cy = np.full(width, cy0, dtype=np.float32)
            x = np.zeros(width, dtype=np.float32)
            y = np.zeros(width, dtype=np.float32)
            cnt = np.zeros(width, dtype=np.int64)
            live = np.arange(width)
            for _ in range(max_iter):
                xx, yy = x * x, y * y
                keep = ~(xx + yy > f32(4.0))
                if not keep.all():
                    x, y, xx, yy, cx, cy, live = (a[keep] for a in (x, y, xx, yy, cx, cy, live))
                    if live.size == 0:
                        break
                xy = x * y
                x, y = (xx - yy) + cx, (xy + xy) + cy
                cnt[live] += 1
            total += int(cnt.sum())
    return total


def main():
    with open(os.path.join(HERE, "mandelbrot_points.json")) as f:
        g = json.load(f)
    ok = True
    for cx, cy, n in g["points"]:
        got = escape_count(cx, cy, g["max_iter"])
        print(f"c = ({cx}, {cy}): {got} (golden {n})")
        ok &= got == n
    # hand/closed-form cross-checks of the near-boundary counts (order of magnitude only)
    for eps, n in ((0.1, 33), (0.01, 315)):
        assert abs(n - math.pi / eps) / (math.pi / eps) < 0.1
    for c, n in ((0.26, 30), (0.251, 97)):
        assert abs(n - math.pi / math.sqrt(c - 0.25)) / (math.pi / math.sqrt(c - 0.25)) < 0.1
    if "--frame" in sys.argv:
        fr = g["frame"]
        H = fr["height"]
        step = 16
        jobs = [(r, min(H, r + step), fr["width"], fr["x0"], fr["y0"], fr["dx"], fr["dy"], fr["max_iter"])
                for r in range(0, H, step)]
        with mp.Pool(os.cpu_count()) as pool:
            total = sum(pool.imap_unordered(frame_rows, jobs))
        print(f"frame checksum {total} (golden {fr['checksum']})")
        ok &= total == fr["checksum"]
    print("OK" if ok else "MISMATCH")
    return 0 if ok else 1


if __name__ == "__main__":
    sys.exit(main())
