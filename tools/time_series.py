import sys, torch
sys.path.insert(0, '.')
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
import bench
lime.load()
props = torch.cuda.get_device_properties(0)
flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
for dt in (torch.float32, torch.float64):
    so = torch.empty((inputs.SERIES_N, 2), dtype=dt, device="cuda")
    med, _ = bench.time_launches(lambda: lime.map_series(0, inputs.SERIES_N, dtype=dt, out=so), 20, 3, flush)
    print(dt, "series us", med * 1e3)
