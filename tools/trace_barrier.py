"""Cross-CTA timeline of the persistent 4096-body step on a -DLIME_TRACE -DLIME_TRACE_GLOBAL build
(globaltimer ns, comparable across SMs): per step, when each CTA arrives at the grid barrier
(slot 2) and when it leaves (slot 3); prints the spread of arrivals, the release latency after
the last arrival, and which CTAs arrive last."""
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
p = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
v = torch.zeros_like(p)
for _ in range(3):
    lime.nbody_simulate(p, v, 64, 1e-4, 1e-3)
torch.cuda.synchronize()
buf = np.zeros(148 * 64 * 8, dtype=np.int64)
L.lime_debug_trace.argtypes = [C.c_void_p, C.c_size_t]
assert L.lime_debug_trace(buf.ctypes.data, buf.nbytes) == 0
t = buf.reshape(148, 64, 8)[:, 8:62, :].astype(np.float64)
arr = t[:, :, 2]                       # barrier arrival
rel = t[:, :, 3]                       # barrier exit
start = t[:, :, 0]
spread = arr.max(0) - arr.min(0)
lat = rel.min(0) - arr.max(0)
exit_spread = rel.max(0) - rel.min(0)
last = np.argmax(arr, axis=0)
step_ns = np.diff(start.min(0))
late = np.bincount(last, minlength=148)
print(json.dumps({"arrival_spread_ns": np.percentile(spread, [0, 50, 100]).tolist(),
                  "release_after_last_arrival_ns": np.percentile(lat, [0, 50, 100]).tolist(),
                  "exit_spread_ns": np.percentile(exit_spread, [0, 50, 100]).tolist(),
                  "step_ns": np.percentile(step_ns, [0, 50, 100]).tolist(),
                  "last_arriver_counts": {int(c): int(n) for c, n in enumerate(late) if n},
                  "arrival_rank_mean_of_top5": [int(c) for c in np.argsort(-(arr - arr.min(0)).mean(1))[:5]],
                  "sm_of_cta": buf.reshape(148, 64, 8)[:, 10, 7].tolist()[:20]}))
