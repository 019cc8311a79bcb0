"""A/B of the config-5 force launch (2^17-target P=8 shard and the full 2^20) for the library
LIME_LIBRARY points at, timed as bench.py does (L2 flushed before every launch)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
n = 1 << 20
b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
acc = torch.empty_like(b)
res = {"lib": os.environ.get("LIME_LIBRARY", "default")}
med, _ = bench.time_launches(lambda: lime.map_nbody(b, 1e-4, 0, 1 << 17, out=acc[: 1 << 17]), 5, 1, flush)
res["shard_p8_ms"] = med
shard = acc[: 1 << 17].clone()
med, _ = bench.time_launches(lambda: lime.map_nbody(b, 1e-4, 0, n, out=acc), 2, 1, flush)
res["full_ms"] = med
res["shard_bit_identical_to_full"] = bool(torch.equal(shard, acc[: 1 << 17]))
res["checksum"] = float(acc[:, :3].double().abs().sum().item())
bm_np = inputs.nbody_bodies(n, seed=5)
bm_np[:, 3] = ((0.5 + inputs.uniform24(5, 99, n)) / n).astype(np.float32)   # bench.py's mixed-mass shard
bm = torch.from_numpy(bm_np).cuda()
med, _ = bench.time_launches(lambda: lime.map_nbody(bm, 1e-4, 0, 1 << 17, out=acc[: 1 << 17]), 5, 1, flush)
res["shard_p8_mixed_ms"] = med
res["checksum_mixed"] = float(acc[:, :3].double().abs().sum().item())
print(json.dumps(res))
