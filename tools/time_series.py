"""Time JG-Series (fp32 and fp64) as bench.py does; one JSON line per dtype. (The variants measured
with it are recorded in profiles/experiments/jg_series_variants_r01m.jsonl.)"""
import json
import sys

import torch

sys.path.insert(0, '.')
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
import bench  # noqa: E402

lime.load()
props = torch.cuda.get_device_properties(0)
flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
for pt, name in ((0, "production"),):
    for dt in (torch.float32, torch.float64):
        so = torch.empty((inputs.SERIES_N, 2), dtype=dt, device="cuda")
        with lime.launch_override(per_thread=pt):
            med, _ = bench.time_launches(lambda: lime.map_series(0, inputs.SERIES_N, dtype=dt, out=so), 20, 3, flush)
        print(json.dumps({"variant": name, "dtype": str(dt), "us": med * 1e3, "checksum": float(so.double().abs().sum())}),
              flush=True)
