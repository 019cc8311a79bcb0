"""Sweep Mandelbrot warp-tile shapes / vote intervals (bit-identical results; time only). The
production default is variant 7 (8x8 px, vote/32)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from bench import time_launches  # noqa: E402

NAMES = {1: "16x4 px, vote/16", 2: "8x8 px, vote/16", 3: "8x8 px, vote/8", 4: "16x4 px, vote/8",
         5: "32x2 px, vote/16", 6: "16x4 px, vote/32", 7: "8x8 px, vote/32", 8: "16x4 px, vote/64"}


def main():
    lime.load()
    flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
    W = 8192
    out = torch.empty((W, W), dtype=torch.int32, device="cuda")
    ref = None
    for v in range(1, 9):
        with lime.launch_override(per_thread=v):
            ms = time_launches(lambda: lime.map_mandelbrot(W, W, -2.0, -1.5, 3 / W, 3 / W, 1024, out=out), 10, 2, flush, writes_output=True)[0]
        if ref is None:
            ref = out.clone()
        print(json.dumps({"variant": NAMES[v], "ms": ms, "bit_identical": bool(torch.equal(out, ref))}), flush=True)


if __name__ == "__main__":
    main()
