import json, sys, torch
sys.path.insert(0, '.')
import paper_conf_pldi_dubachcrbf12_b200 as lime
import bench
lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
x = torch.empty(1 << 20, device="cuda")
for cnt in (1, 128, 1000, 10000, 50000, 100000, 200000):
    for dt in (torch.float32,):
        so = torch.empty((cnt, 2), dtype=dt, device="cuda")
        med, _ = bench.time_launches(lambda: lime.map_series(0, cnt, dtype=dt, out=so), 20, 3, flush)
        print(json.dumps({"count": cnt, "us": med * 1e3}), flush=True)
# reference: an empty-ish launch through the same path (reduce of 1 element)
med, _ = bench.time_launches(lambda: lime.reduce_sum(x[:1]), 20, 3, flush)
print(json.dumps({"reduce_1_elem_us": med * 1e3}))
