"""A/B of the fused Black-Scholes kernels at 2^24 options: warp-specialised TMA ring (default) vs the
register-prefetch kernel (launch override per_thread=1); cold (L2 flushed, single launch) and steady
(back-to-back over two input sets), as bench.py times them; sums checked against the oracle."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
import bench  # noqa: E402
import oracle  # noqa: E402  (accuracy check only)

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
n = 1 << 24
host = [inputs.blackscholes_options(n, seed=sd) for sd in (2, 12)]
sets = [tuple(torch.from_numpy(a).cuda() for a in h) for h in host]
ref = oracle.blackscholes_sums(*host[0], inputs.BS_R, inputs.BS_SIGMA)
sums = [torch.empty(2, dtype=torch.float64, device="cuda") for _ in sets]
for rnd in range(2):
    for pt, name in ((0, "ws_tma_ring"), (1, "register_prefetch")):
        with lime.launch_override(per_thread=pt):
            cold, _ = bench.time_launches(lambda: lime.map_reduce_blackscholes_sum(*sets[0], inputs.BS_R, inputs.BS_SIGMA, sums[0]),
                                          30, 5, flush)
            fns = [lambda k=k: lime.map_reduce_blackscholes_sum(*sets[k], inputs.BS_R, inputs.BS_SIGMA, sums[k]) for k in range(2)]
            steady = bench.time_back_to_back(fns, 20, 5, flush)
            got = lime.map_reduce_blackscholes_sum(*sets[0], inputs.BS_R, inputs.BS_SIGMA).cpu().numpy()
        rel = [abs(got[i] - ref[i]) / abs(ref[i]) for i in range(2)]
        print(json.dumps({"lib": os.environ.get("LIME_LIBRARY", "default"), "kernel": name, "cold_us": cold * 1e3,
                          "steady_us": steady * 1e3, "cold_frac": 12.0 * n / (cold * 1e-3) / 1e9 / 6549.1,
                          "steady_frac": 12.0 * n / (steady * 1e-3) / 1e9 / 6549.1, "rel_err": rel}), flush=True)
