"""Launch one hot-path kernel a few times at its BASELINE.json size, for ncu captures.

    ncu --set full --clock-control none --import-source on -k regex:<kernel> -s 1 -c 1 \
        -o gpurun_out/prof_<which> python tools/prof_kernels.py <which>

which: nbody1m | nbody1m_p8 | nbody4096 | sim4096 | nbody64 | bs_map | bs_fused | mandel | matmul | reduce | cp | mriq
       | series | idea
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402


def main(which: str, reps: int = 3):
    lime.load()
    if which.startswith("nbody") and which != "nbody64":
        n = 4096 if which == "nbody4096" else 1 << 20
        b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
        cnt = n // 8 if which.endswith("_p8") else n
        out = torch.empty((cnt, 4), dtype=torch.float32, device="cuda")
        for _ in range(reps):
            lime.map_nbody(b, 1e-4, 0, cnt, out=out)
    elif which.startswith("bs"):
        n = 1 << 24
        S, X, T = (torch.from_numpy(a).cuda() for a in inputs.blackscholes_options(n, seed=2))
        for _ in range(reps):
            if which == "bs_map":
                lime.map_blackscholes(S, X, T, inputs.BS_R, inputs.BS_SIGMA)
            else:
                lime.map_reduce_blackscholes_sum(S, X, T, inputs.BS_R, inputs.BS_SIGMA)
    elif which == "mandel":
        W = 8192
        for _ in range(reps):
            lime.map_mandelbrot(W, W, -2.0, -1.5, 3.0 / W, 3.0 / W, 1024)
    elif which == "matmul":
        M = 8192
        A = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 0).view(np.int16)).cuda().view(torch.bfloat16)
        B = torch.from_numpy(inputs.bf16_uniform(M, M, 4, 1).view(np.int16)).cuda().view(torch.bfloat16)
        for _ in range(reps):
            lime.map_matmul_bf16(A, B)
    elif which == "cp":
        atoms = torch.from_numpy(inputs.cp_atoms()).cuda()
        for _ in range(reps):
            lime.map_coulomb(atoms, inputs.CP_NX, inputs.CP_NY, inputs.CP_Z, inputs.CP_H)
    elif which == "mriq":
        k = torch.from_numpy(inputs.mriq_kspace()).cuda()
        vx = torch.from_numpy(inputs.mriq_voxels()).cuda()
        for _ in range(reps):
            lime.map_mriq(k, vx)
    elif which == "sim4096":
        p = torch.from_numpy(inputs.nbody_bodies(4096, seed=1)).cuda()
        v = torch.zeros_like(p)
        for _ in range(reps):
            lime.nbody_simulate(p, v, 100, 1e-4, 1e-3)
    elif which == "nbody64":
        b = torch.from_numpy(inputs.nbody_bodies(1 << 20, seed=5).astype(np.float64)).cuda()
        for _ in range(reps):
            lime.map_nbody_f64(b, 1e-4, 0, 1 << 17)     # bench.py's nbody_f64 shape
    elif which == "series":
        for _ in range(reps):
            lime.map_series(0, inputs.SERIES_N)
    elif which == "idea":
        data = torch.from_numpy(inputs.crypt_data()).cuda()
        ek, _ = lime.idea_key_schedule(inputs.crypt_key())
        for _ in range(reps):
            lime.map_idea(data, ek)
    elif which == "reduce":
        x = torch.ones(1 << 28, dtype=torch.float32, device="cuda")
        for _ in range(reps):
            lime.reduce_sum(x)
    else:
        raise SystemExit(f"unknown {which}")
    torch.cuda.synchronize()


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 3)
