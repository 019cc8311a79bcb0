import os, sys, json, torch
sys.path.insert(0, '/root/repo')
import bench
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
n = 1 << 24
S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
S2, X2, T2 = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=12))
sm = torch.empty(2, dtype=torch.float64, device="cuda"); sm2 = torch.empty(2, dtype=torch.float64, device="cuda")
for g in (0, 148, 296, 444, 592, 740, 888, 1184):
    with lime.launch_override(grid_ctas=g):
        cold = bench.time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm), 30, 5, flush)[0] * 1e3
        st = bench.time_back_to_back([lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm),
                                      lambda: lime.map_reduce_blackscholes_sum(S2, X2, T2, 0.02, 0.3, sm2)], 20, 5, flush) * 1e3
    print(json.dumps({"grid": g, "cold_us": round(cold, 2), "steady_us": round(st, 2)}))
