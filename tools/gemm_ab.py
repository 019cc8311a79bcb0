import sys, os, numpy as np, torch, json
sys.path.insert(0, os.getcwd())
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
sys.path.insert(0, "tools")
from bench import time_launches
lime.load()
def bf(a): return torch.from_numpy(np.ascontiguousarray(a).view(np.int16)).cuda().view(torch.bfloat16)
res = {}
for (M, N, K) in [(512, 256, 64), (1000, 1000, 1000), (1536, 768, 4096), (33, 47, 72), (600, 300, 520), (2048, 2048, 2048)]:
    A, Bt = inputs.matmul_operands(M, N, K, seed=M + N + K)
    with lime.launch_override(per_thread=2):
        C2 = lime.map_matmul_bf16(bf(A), bf(Bt))
    with lime.launch_override(per_thread=3):
        C3 = lime.map_matmul_bf16(bf(A), bf(Bt))
    torch.cuda.synchronize()
    res[f"{M}x{N}x{K}"] = bool(torch.equal(C2, C3)), float((C2 - C3).abs().max())
print(json.dumps(res))
M = 8192
A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
C = torch.empty((M, M), device="cuda")
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
out = {}
for pt in (2, 3):
    for g in ((4, 8) if pt == 2 else (1, 2, 4)):
        with lime.launch_override(per_thread=pt, block_threads=g):
            out[f"pt{pt}_g{g}"] = time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush)[0]
out["cublas_fp32"] = time_launches(lambda: torch.mm(A, B.t(), out_dtype=torch.float32, out=C), 20, 3, flush)[0]
with lime.launch_override(per_thread=3):
    C3 = lime.map_matmul_bf16(A, B).clone()
with lime.launch_override(per_thread=2):
    C2 = lime.map_matmul_bf16(A, B)
out["equal_8192"] = bool(torch.equal(C2, C3))
print(json.dumps(out))
