"""Time the Black-Scholes map and fused map+reduce (L2 flushed before every launch). Variants tried
and dropped are recorded in profiles/experiments/blackscholes_*.json*."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
from bench import time_launches  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
n = 1 << 24
S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
c = torch.empty(n, device="cuda"); p = torch.empty(n, device="cuda"); sm = torch.empty(2, dtype=torch.float64, device="cuda")
ref_c = lime.map_blackscholes(S, X, T, 0.02, 0.3)[0].clone()
for v, nm in ((0, "reg_prefetch"),):
    with lime.launch_override(per_thread=v):
        m = time_launches(lambda: lime.map_blackscholes(S, X, T, 0.02, 0.3, c, p), 30, 5, flush)[0]
        f = time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm), 30, 5, flush)[0]
        same = bool(torch.equal(c, ref_c))
    print(json.dumps({"variant": nm, "map_us": m * 1e3, "fused_us": f * 1e3, "map_GBs": 20 * n / m / 1e6,
                      "fused_GBs": 12 * n / f / 1e6, "map_identical": same, "sums": sm.tolist()}), flush=True)
