"""Launch-floor probe: event-timed (bench.time_launches) duration of trivial launches, to read the
short-kernel numbers against. Run once with and once without LIME_NO_PDL=1."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
x = torch.ones(1 << 20, device="cuda")
out = torch.empty(1, device="cuda")
res = {"pdl": os.environ.get("LIME_NO_PDL") is None}
res["torch_add_1_elem_us"] = bench.time_launches(lambda: x[:1].add_(0.0), 30, 3, flush)[0] * 1e3
res["lime_reduce_1_elem_us"] = bench.time_launches(lambda: lime.reduce_sum(x[:1], out=out), 30, 3, flush)[0] * 1e3
res["lime_reduce_1M_us"] = bench.time_launches(lambda: lime.reduce_sum(x, out=out), 30, 3, flush)[0] * 1e3
print(json.dumps(res))
