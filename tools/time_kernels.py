"""Time individual hot-path kernels at their BASELINE.json sizes (L2 flushed before each launch)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
from bench import time_launches  # noqa: E402


def main(which):
    lime.load()
    flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
    out = {}
    if "bs" in which:
        n = 1 << 24
        S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
        c = torch.empty(n, device="cuda"); p = torch.empty(n, device="cuda"); sm = torch.empty(2, dtype=torch.float64, device="cuda")
        out["bs_map_ms"] = time_launches(lambda: lime.map_blackscholes(S, X, T, 0.02, 0.3, c, p), 30, 5, flush)[0]
        out["bs_fused_ms"] = time_launches(lambda: lime.map_reduce_blackscholes_sum(S, X, T, 0.02, 0.3, sm), 30, 5, flush)[0]
        out["bs_map_GBs"] = 20 * n / out["bs_map_ms"] / 1e6
        out["bs_fused_GBs"] = 12 * n / out["bs_fused_ms"] / 1e6
    if "mandel" in which:
        W = 8192
        cnt = torch.empty((W, W), dtype=torch.int32, device="cuda")
        out["mandel_ms"] = time_launches(lambda: lime.map_mandelbrot(W, W, -2.0, -1.5, 3 / W, 3 / W, 1024, out=cnt), 10, 2, flush)[0]
        out["mandel_checksum"] = int(cnt.sum(dtype=torch.int64).item())
    if "matmul" in which:
        M = 8192
        A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
        B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
        C = torch.empty((M, M), device="cuda")
        out["matmul_ms"] = time_launches(lambda: lime.map_matmul_bf16(A, B, C), 20, 3, flush)[0]
        out["matmul_TF"] = 2 * M**3 / out["matmul_ms"] / 1e9
        out["cublas_bf16out_ms"] = time_launches(lambda: torch.matmul(A, B.t()), 20, 3, flush)[0]
        try:
            Cf = torch.empty((M, M), device="cuda")
            out["cublas_fp32out_ms"] = time_launches(lambda: torch.mm(A, B.t(), out_dtype=torch.float32, out=Cf), 20, 3, flush)[0]
        except Exception as e:  # noqa: BLE001
            out["cublas_fp32out_ms"] = f"unavailable: {e}"[:120]
    if "nbody" in which:
        n = 4096
        b = torch.from_numpy(inputs.nbody_bodies(n, seed=1)).cuda()
        acc = torch.empty_like(b)
        out["nbody4096_us"] = 1e3 * time_launches(lambda: lime.map_nbody(b, 1e-4, out=acc), 50, 5, flush)[0]
    if "nbody1m" in which:
        n = 1 << 20
        b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
        acc = torch.empty_like(b)
        ms = time_launches(lambda: lime.map_nbody(b, 1e-4, out=acc), 3, 1, flush)[0]
        out["nbody1m_ms"] = ms
        out["nbody1m_frac"] = 20.0 * n * n / (ms * 1e-3) / 74.45e12
    if "nbody64" in which:
        for n, cnt in ((4096, 4096), (1 << 20, 1 << 17)):
            b = torch.from_numpy(inputs.nbody_bodies(n, seed=1).astype(np.float64)).cuda()
            acc = torch.empty((cnt, 4), dtype=torch.float64, device="cuda")
            ms = time_launches(lambda: lime.map_nbody_f64(b, 1e-4, 0, cnt, out=acc), 5 if n > 4096 else 30, 2, flush)[0]
            out[f"nbody64_{n}x{cnt}_ms"] = ms
            out[f"nbody64_{n}x{cnt}_Gint_s"] = n * cnt / ms / 1e6
    if "parboil" in which:
        atoms = torch.from_numpy(inputs.cp_atoms()).cuda()
        V = torch.empty(inputs.CP_NX * inputs.CP_NY, device="cuda")
        out["cp_us"] = 1e3 * time_launches(lambda: lime.map_coulomb(atoms, inputs.CP_NX, inputs.CP_NY, inputs.CP_Z, inputs.CP_H, out=V), 30, 3, flush)[0]
        k = torch.from_numpy(inputs.mriq_kspace()).cuda()
        vx = torch.from_numpy(inputs.mriq_voxels()).cuda()
        Q = torch.empty((vx.shape[0], 2), device="cuda")
        out["mriq_us"] = 1e3 * time_launches(lambda: lime.map_mriq(k, vx, out=Q), 30, 3, flush)[0]
    if "series" in which:
        for dt, nm in ((torch.float32, "f32"), (torch.float64, "f64")):
            so = torch.empty((inputs.SERIES_N, 2), dtype=dt, device="cuda")
            out[f"series_{nm}_us"] = 1e3 * time_launches(lambda: lime.map_series(0, inputs.SERIES_N, dtype=dt, out=so), 20, 3, flush)[0]
    if "sim" in which:
        p = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
        v = torch.zeros_like(p)
        out["sim4096_us_per_step"] = 10 * time_launches(lambda: lime.nbody_simulate(p, v, 100, 1e-4, 1e-3), 10, 2, flush)[0]
    if "reduce" in which:
        x = torch.ones(1 << 28, dtype=torch.float32, device="cuda")
        r = torch.empty((), dtype=torch.float32, device="cuda")
        out["reduce_ms"] = time_launches(lambda: lime.reduce_sum(x, r), 20, 3, flush)[0]
        out["reduce_GBs"] = 4 * (1 << 28) / out["reduce_ms"] / 1e6
    print(json.dumps(out))


if __name__ == "__main__":
    main(sys.argv[1:] or ["bs", "mandel", "matmul", "nbody", "reduce"])
