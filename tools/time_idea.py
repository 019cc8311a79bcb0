"""Time JG-Crypt (IDEA-ECB over the Table 3 3 MiB) as bench.py does; one JSON line."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
data = torch.from_numpy(inputs.crypt_data()).cuda()
ek, _ = lime.idea_key_schedule(inputs.crypt_key())
enc = torch.empty_like(data)
med, _ = bench.time_launches(lambda: lime.map_idea(data, ek, out=enc), 30, 3, flush)
print(json.dumps({"idea_us": med * 1e3}))
