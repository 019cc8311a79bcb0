"""Time the Black-Scholes map and fused map+reduce (L2 flushed before every launch). Variants tried
and dropped are recorded in profiles/experiments/blackscholes_*.json*."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
from bench import time_back_to_back, time_launches  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
n = 1 << 24
S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
c = torch.empty(n, device="cuda"); p = torch.empty(n, device="cuda"); sm = torch.empty(2, dtype=torch.float64, device="cuda")
S2, X2, T2 = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=12))
sm2 = torch.empty(2, dtype=torch.float64, device="cuda")
ref_c = lime.map_blackscholes(S, X, T, 0.02, 0.3)[0].clone()
from oracle import blackscholes_sums as _osums  # noqa: E402  (tools may call the oracle)
ref_s = _osums(S.cpu().numpy(), X.cpu().numpy(), T.cpu().numpy(), 0.02, 0.3)
variants = [(int(a.split("=")[0]), a.split("=")[1]) for a in sys.argv[1:]] or [(0, "production")]
for v, nm in variants:
    with lime.launch_override(per_thread=v):
        m = time_launches(lambda: lime.map_blackscholes(S, X, T, 0.02, 0.3, c, p), 30, 5, flush)[0]
        f = time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm), 30, 5, flush)[0]
        same = bool(torch.equal(c, ref_c))
        fs = time_back_to_back([lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm),
                                lambda: lime.map_reduce_blackscholes_sum(S2, X2, T2, 0.02, 0.3, sm2)], 20, 5, flush)
    print(json.dumps({"variant": nm, "map_us": m * 1e3, "fused_us": f * 1e3, "fused_steady_us": fs * 1e3, "map_GBs": 20 * n / m / 1e6,
                      "fused_GBs": 12 * n / f / 1e6, "map_identical": same, "sums": sm.tolist(),
                      "sums_rel_err": [abs(a - b) / abs(b) for a, b in zip(sm.tolist(), ref_s)]}), flush=True)
