"""Quick GEMM check/timing for both cta_group variants (dev tool; the parity tests live in tests/)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402


def bf(bits):
    return torch.from_numpy(np.ascontiguousarray(bits).view(np.int16)).cuda().view(torch.bfloat16)


def main():
    lime.load()
    for M, N, K in [(256, 256, 64), (300, 520, 200), (512, 1024, 4096), (1000, 1000, 1000), (129, 257, 4104)]:
        A, Bt = inputs.matmul_operands(M, N, K, seed=M + N)
        Ad, Bd = bf(A), bf(Bt)
        ref = (Ad.double() @ Bd.double().t())
        mag = (Ad.double().abs() @ Bd.double().abs().t())
        for path in (1, 2):
            with lime.launch_override(per_thread=path):
                C = lime.map_matmul_bf16(Ad, Bd)
            torch.cuda.synchronize()
            err = ((C.double() - ref).abs() / mag.clamp_min(1e-30)).max().item()
            print(f"M{M} N{N} K{K} path{path} maxrel {err:.3e}", flush=True)
    M = N = K = 8192
    A, Bt = inputs.matmul_operands(M, N, K, seed=4)
    Ad, Bd = bf(A), bf(Bt)
    for path in (1, 2):
        with lime.launch_override(per_thread=path):
            C = lime.map_matmul_bf16(Ad, Bd)
            torch.cuda.synchronize()
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
            ts = []
            for _ in range(10):
                ev[0].record(); lime.map_matmul_bf16(Ad, Bd, out=C); ev[1].record(); torch.cuda.synchronize()
                ts.append(ev[0].elapsed_time(ev[1]))
        print(f"8192^3 path{path}: {min(ts):.4f} ms  {2*M*N*K/min(ts)/1e9:.1f} TF", flush=True)
    r = torch.randint(0, M, (4096,), device="cuda")
    c = torch.randint(0, N, (4096,), device="cuda")
    ref = (Ad[r].double() * Bd[c].double()).sum(1)
    print("8192 sampled maxabs", (C[r, c].double() - ref).abs().max().item())


if __name__ == "__main__":
    main()
