import sys, os, json, torch
sys.path.insert(0, os.getcwd())
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from bench import time_launches
lime.load()
out = {}
for lg in (20, 22, 24):
    n = 1 << lg
    S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
    sm = torch.empty(2, dtype=torch.float64, device="cuda")
    c = torch.empty(n, device="cuda"); p = torch.empty(n, device="cuda")
    out[f"fused_2^{lg}_hot_ns_per_opt"] = 1e6 * time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm), 30, 5, None)[0] / n
    out[f"map_2^{lg}_hot_ns_per_opt"] = 1e6 * time_launches(lambda: lime.map_blackscholes(S, X, T, 0.02, 0.3, c, p), 30, 5, None)[0] / n
print(json.dumps(out))
