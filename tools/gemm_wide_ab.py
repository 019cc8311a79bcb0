"""A/B of the 256x512 pair tile (default) against the 256x256 pair tile (per_thread=2) at 8192^3,
the wide tile's raster group sweep, and cuBLAS; timed as bench.py does (L2 flushed dirty)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
from bench import time_launches  # noqa: E402

lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
M = 8192
A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
C = torch.empty((M, M), device="cuda")
with lime.launch_override(per_thread=2):
    ref = lime.map_matmul_bf16(A, B).clone()
groups = [int(g) for g in sys.argv[1:]] or [8]


def t_pair():
    with lime.launch_override(per_thread=2):
        return time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush, writes_output=True)[0]


def t_wide(g):
    with lime.launch_override(block_threads=g):
        ms = time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush, writes_output=True)[0]
    assert torch.equal(C, ref)
    return ms


res = {"pair_256x256": [], "cublas_fp32_out": [], "cublas_bf16_out": []}
for g in groups:
    res[f"wide_256x512_g{g}"] = []
for rnd in range(3):                    # interleaved rounds: clock/thermal drift hits every arm alike
    res["pair_256x256"].append(t_pair())
    for g in groups:
        res[f"wide_256x512_g{g}"].append(t_wide(g))
    res["cublas_fp32_out"].append(time_launches(lambda: torch.mm(A, B.t(), out_dtype=torch.float32), 20, 3, flush,
                                                writes_output=True)[0])
    res["cublas_bf16_out"].append(time_launches(lambda: torch.mm(A, B.t()), 20, 3, flush, writes_output=True)[0])
for k, v in res.items():
    print(json.dumps({"arm": k, "ms": v, "ms_min": min(v), "TF_best": 2 * M**3 / min(v) / 1e9}), flush=True)
