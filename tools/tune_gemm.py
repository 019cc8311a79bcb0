"""Sweep the 2-CTA GEMM's tile raster group (launch override block_threads) at 8192^3."""
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
ref = lime.map_matmul_bf16(A, B).clone()
for g in (1, 2, 4, 8, 16, 32):
    with lime.launch_override(block_threads=g):
        ms = time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush, writes_output=True)[0]
    print(json.dumps({"group": g, "ms": ms, "TF": 2 * M**3 / ms / 1e9, "identical": bool(torch.equal(C, ref))}), flush=True)
cub = time_launches(lambda: torch.mm(A, B.t(), out_dtype=torch.float32), 20, 3, flush, writes_output=True)[0]
print(json.dumps({"cublas_fp32_out_ms": cub, "TF": 2 * M**3 / cub / 1e9}))
