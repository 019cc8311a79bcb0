# A/B of GEMM builds (LIME_LIBRARY): 8192^3 time beside cuBLAS fp32-out, interleaved rounds; then ncu DRAM bytes
for r in 1 2 3; do for L in "$@"; do
LIME_LIBRARY=gpurun_ab/$L/liblime.so timeout 200 python - <<'PY'
import os, sys, json, numpy as np, torch
sys.path.insert(0, '.')
import paper_conf_pldi_dubachcrbf12_b200 as lime
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from bench import time_launches
lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
M = 8192
A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
C = torch.empty((M, M), device="cuda")
ms = time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush, writes_output=True)[0]
cub = time_launches(lambda: torch.mm(A, B.t(), out_dtype=torch.float32), 20, 3, flush, writes_output=True)[0]
print(json.dumps({"lib": os.environ["LIME_LIBRARY"], "ms": round(ms, 4), "cublas_fp32_ms": round(cub, 4), "ratio": round(cub / ms, 4), "csum": float(C[::97, ::89].double().sum())}))
PY
done; done
for L in "$@"; do echo $L; LIME_LIBRARY=gpurun_ab/$L/liblime.so timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__cycles_elapsed.avg.per_second --clock-control none -k regex:gemm -c 1 python tools/prof_kernels.py matmul 2 2>&1 | grep -E "dram__bytes|gpu__time|per_second"; done
