"""Small invocations of every hot-path kernel for compute-sanitizer (memcheck / racecheck / synccheck).

    compute-sanitizer --tool memcheck python tools/sanitize_small.py
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402


def main():
    lime.load()
    dev = "cuda"
    b = torch.from_numpy(inputs.nbody_bodies(1000, seed=1)).to(dev)
    lime.map_nbody(b, 1e-4)                                   # small path (in-CTA splits)
    with lime.launch_override(block_threads=128, per_thread=2):
        lime.map_nbody(b, 1e-4, 100, 517)                     # general kernel, ragged shard
    big = torch.from_numpy(inputs.nbody_bodies(9000, seed=2)).to(dev)
    lime.map_nbody(big, 1e-4, 0, 700)                         # general kernel, S = 12 splits
    v = torch.zeros_like(b)
    p = b.clone()
    lime.nbody_simulate(p, v, 3, 1e-4, 1e-3)                  # persistent cooperative kernel
    lime.map_nbody_integrate(p, v, lime.map_nbody(p, 1e-4), 1e-3)
    lime.map_nbody_f64(b.double(), 1e-4)
    # round 2: TMA row-box staging (n % 64 == 0), the fused step (small and general n), the
    # 8192-body LDG staging and the persistent kernel on the TMA path
    t = torch.from_numpy(inputs.nbody_bodies(1024, seed=4)).to(dev)
    lime.map_nbody(t, 1e-4, 100, 333)
    vt = torch.zeros((333, 4), dtype=torch.float32, device=dev)
    lime.map_nbody_step(t, 1e-4, 1e-3, vt, 100, 333)
    lime.map_nbody_step(big, 1e-4, 1e-3, torch.zeros((700, 4), dtype=torch.float32, device=dev), 0, 700)
    e8 = torch.from_numpy(inputs.nbody_bodies(8192, seed=5)).to(dev)
    lime.map_nbody(e8, 1e-4, 0, 257)
    pt, vv = t.clone(), torch.zeros_like(t)
    lime.nbody_simulate(pt, vv, 3, 1e-4, 1e-3)
    # round 2: factored power-of-two chunks -- predicted and verified (chunk 1 one mass off: the
    # per-body redo), cached across steps in the persistent kernel
    mx = t.clone()
    mx[64 + 7, 3] *= 2.0
    lime.map_nbody(mx, 1e-4)
    lime.nbody_simulate(mx.clone(), torch.zeros_like(mx), 3, 1e-4, 1e-3)
    S, X, T = (torch.from_numpy(a).to(dev) for a in inputs.blackscholes_options(4099, seed=3))
    lime.map_blackscholes(S, X, T, inputs.BS_R, inputs.BS_SIGMA)
    lime.map_reduce_blackscholes_sum(S, X, T, inputs.BS_R, inputs.BS_SIGMA)
    lime.map_mandelbrot(67, 33, -2.0, -1.5, 3 / 67, 3 / 33, 64)
    A = torch.from_numpy(inputs.bf16_uniform(300, 136, 4, 0).view(np.int16)).to(dev).view(torch.bfloat16)
    B = torch.from_numpy(inputs.bf16_uniform(260, 136, 4, 1).view(np.int16)).to(dev).view(torch.bfloat16)
    lime.map_matmul_bf16(A, B)
    B2 = torch.from_numpy(inputs.bf16_uniform(1030, 136, 4, 2).view(np.int16)).to(dev).view(torch.bfloat16)
    lime.map_matmul_bf16(A, B2)                               # 256 x 512 pair tile, ragged M and N
    x = torch.randn(100003, device=dev)
    lime.reduce_sum(x), lime.reduce_min(x), lime.reduce_max(x)
    atoms = torch.from_numpy(inputs.cp_atoms(300)).to(dev)
    lime.map_coulomb(atoms, 37, 11, inputs.CP_Z, inputs.CP_H)
    k = torch.from_numpy(inputs.mriq_kspace(500)).to(dev)
    vx = torch.from_numpy(inputs.mriq_voxels(777)).to(dev)
    lime.map_mriq(k, vx)
    lime.map_series(0, 1000)
    lime.map_series(5, 333, dtype=torch.float64)
    data = torch.from_numpy(inputs.crypt_data(4104)).to(dev)
    ek, _ = lime.idea_key_schedule(inputs.crypt_key())
    lime.map_idea(data, ek)
    torch.cuda.synchronize()
    print("sanitize_small ok")


if __name__ == "__main__":
    main()
