"""Time the config-3 Mandelbrot map (8192^2, 1024 iterations) as bench.py does; one JSON line."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
W = 8192
cnt = torch.empty((W, W), dtype=torch.int32, device="cuda")
med, _ = bench.time_launches(lambda: lime.map_mandelbrot(W, W, -2.0, -1.5, 3.0 / W, 3.0 / W, 1024, out=cnt), 10, 2, flush,
                             writes_output=True)
s = int(cnt.sum(dtype=torch.int64).item())
print(json.dumps({"ms": med, "sum": s, "sum_ok": s == 11856987162,
                  "frac_fp32": 7 * 11856987162 / (med * 1e-3) / (148 * 128 * 1.965e9)}))
