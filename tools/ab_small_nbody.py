"""A/B of the 4096-body N-Body paths (config 1) for the library LIME_LIBRARY points at: one force
launch (L2 flushed), 100 force+integrate steps as a CUDA graph, 100 steps in one persistent launch,
each timed as bench.py does; plus the max relative error of the forces against the fp64 oracle."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist, inputs  # noqa: E402
import oracle  # noqa: E402  (test infrastructure: accuracy check only)

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
res = {"lib": os.environ.get("LIME_LIBRARY", "default"), "splits_4096": lime.nbody_splits(4096)}
for n in (4096, 8192, 2048):
    b_np = inputs.nbody_bodies(n, seed=1)
    b = torch.from_numpy(b_np).cuda()
    acc = torch.empty_like(b)
    med, _ = bench.time_launches(lambda: lime.map_nbody(b, 1e-4, 0, n, out=acc), 50, 5, flush)
    res[f"force_{n}_us"] = med * 1e3
    ref = np.asarray(oracle.nbody_accel(b_np, 1e-4))[:, :3]
    got = acc.cpu().numpy().astype(np.float64)[:, :3]
    res[f"force_{n}_max_rel_err"] = float(np.max(np.abs(got - ref)) / np.max(np.abs(ref)))
sim = ldist.NBodySim(torch.from_numpy(inputs.nbody_bodies(4096, seed=1)), 1e-4, 1e-3, "cuda")
g = sim.capture(100)
med, _ = bench.time_launches(g.replay, 10, 2, flush)
res["graph_step_us"] = med * 1e3 / 100
p = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
v = torch.zeros_like(p)
med, _ = bench.time_launches(lambda: lime.nbody_simulate(p, v, 100, 1e-4, 1e-3), 10, 2, flush)
res["simulate_step_us"] = med * 1e3 / 100
print(json.dumps(res))
