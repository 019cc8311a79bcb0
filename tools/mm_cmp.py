import sys, torch, numpy as np
sys.path.insert(0, '.')
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
lime.load()
M = 8192
A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
C = torch.empty((M, M), device="cuda")
for _ in range(3):
    lime.map_matmul_bf16(A, B, C)
    torch.mm(A, B.t(), out_dtype=torch.float32)
torch.cuda.synchronize()
