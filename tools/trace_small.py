"""Phase trace of the persistent 4096-body simulation (config 1): needs a library built with
-DLIME_TRACE (tools/build_variant.py). Thread 0 of every CTA records clock64 at four points of each
of the first 64 steps: step start, all split partials done, combine+integrate done, after the grid
barrier. Prints per-phase cycle statistics over steps 8..63 and all CTAs."""
import ctypes as C
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402

L = lime.load()
n = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
p = torch.from_numpy(inputs.nbody_bodies(n, seed=1)).cuda()
v = torch.zeros_like(p)
for _ in range(3):
    lime.nbody_simulate(p, v, 64, 1e-4, 1e-3)
torch.cuda.synchronize()
buf = np.zeros(148 * 64 * 8, dtype=np.int64)
L.lime_debug_trace.argtypes = [C.c_void_p, C.c_size_t]
assert L.lime_debug_trace(buf.ctypes.data, buf.nbytes) == 0
t = buf.reshape(148, 64, 8)[:, 8:, :].astype(np.float64)
nxt = np.roll(buf.reshape(148, 64, 8)[:, :, 0], -1, axis=1)[:, 8:63].astype(np.float64)
per_cta = np.median(t[:, :, 1] - t[:, :, 0], axis=1)
w0 = np.median(t[:, :, 4] - t[:, :, 0], axis=1)
sm = buf.reshape(148, 64, 8)[:, 10, 7]
print("smids unique:", len(set(sm.tolist())), "per-CTA compute median:", per_cta.astype(int).tolist())
print("warp0 lane-sum done:", w0.astype(int).tolist())
wb = np.zeros(148 * 32 * 2, dtype=np.int64)
L.lime_debug_wtrace.argtypes = [C.c_void_p, C.c_size_t]
assert L.lime_debug_wtrace(wb.ctypes.data, wb.nbytes) == 0
wb = wb.reshape(148, 32, 2).astype(np.float64)
st20 = buf.reshape(148, 64, 8)[:, 20, 0].astype(np.float64)
for c in (0, 1, 50):
    used = wb[c, :, 1] > 0
    print("cta", c, "ready", (wb[c, used, 0] - st20[c]).astype(int).tolist())
    print("cta", c, "done ", (wb[c, used, 1] - st20[c]).astype(int).tolist())
res = {"n": n, "pre_stage_cyc": np.percentile(t[:, :, 5] - t[:, :, 0], [0, 50, 100]).tolist(),
       "stage_cyc": np.percentile(t[:, :, 6] - t[:, :, 5], [0, 50, 100]).tolist(),
       "compute_cyc": np.percentile(t[:, :, 1] - t[:, :, 0], [0, 50, 100]).tolist(),
       "combine_cyc": np.percentile(t[:, :, 2] - t[:, :, 1], [0, 50, 100]).tolist(),
       "barrier_cyc": np.percentile(t[:, :, 3] - t[:, :, 2], [0, 50, 100]).tolist(),
       "step_cyc": np.percentile(nxt - t[:, :55, 0], [0, 50, 100]).tolist()}
print(json.dumps(res))
