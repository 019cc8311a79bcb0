"""Sweep the Mandelbrot launch variants (launch override per_thread) on the config-3 frame: time
(L2 flushed) and bit-exactness against the tested loop (per_thread=7)."""
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
with lime.launch_override(per_thread=7):
    ref = lime.map_mandelbrot(W, W, -2.0, -1.5, 3.0 / W, 3.0 / W, 1024).clone()
cnt = torch.empty((W, W), dtype=torch.int32, device="cuda")
for pt in [int(x) for x in sys.argv[1:]]:
    with lime.launch_override(per_thread=pt):
        ms, _ = bench.time_launches(lambda: lime.map_mandelbrot(W, W, -2.0, -1.5, 3.0 / W, 3.0 / W, 1024, out=cnt), 10, 2,
                                    flush, writes_output=True)
    print(json.dumps({"per_thread": pt, "ms": ms, "bit_exact": bool(torch.equal(cnt, ref))}), flush=True)
