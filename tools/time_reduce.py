"""Event-timed reductions (L2 flushed before each launch): 2^28 f32 sum (the bench config) and smaller sizes."""
import json, os, sys
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
res = {}
for lg in (16, 20, 24, 28):
    x = torch.from_numpy(inputs.reduce_array(1 << lg, "f32", seed=3)).cuda()
    out = torch.empty((), device="cuda")
    res[f"sum_f32_2^{lg}_us"] = bench.time_launches(lambda: lime.reduce_sum(x, out=out), 20, 3, flush)[0] * 1e3
print(json.dumps(res))
