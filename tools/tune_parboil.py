"""Sweep the Parboil-CP / MRI-Q target-tile block (64 / 128 / 256 threads x 4 targets) on B200;
results must be bit-identical across blocks (the summation order depends on the source chunking
only). Prints one JSON line per (map, block)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402


def main():
    lime.load()
    props = torch.cuda.get_device_properties(0)
    flush = torch.empty(2 * props.L2_cache_size, dtype=torch.uint8, device="cuda")
    atoms = torch.from_numpy(inputs.cp_atoms()).cuda()
    k = torch.from_numpy(inputs.mriq_kspace()).cuda()
    vx = torch.from_numpy(inputs.mriq_voxels()).cuda()
    cases = {
        "cp": (lambda: lime.map_coulomb(atoms, inputs.CP_NX, inputs.CP_NY, inputs.CP_Z, inputs.CP_H),
               float(atoms.shape[0]) * inputs.CP_NX * inputs.CP_NY),
        "mriq": (lambda: lime.map_mriq(k, vx), float(k.shape[0]) * vx.shape[0]),
    }
    for name, (fn, inter) in cases.items():
        ref = None
        for block in (64, 128, 256):
            with lime.launch_override(block_threads=block):
                out = fn()
                med, _ = bench.time_launches(fn, 20, 3, flush)
            same = True if ref is None else bool(torch.equal(out, ref))
            ref = out if ref is None else ref
            print(json.dumps({"map": name, "block": block, "us": med * 1e3, "inter_per_s": inter / (med * 1e-3),
                              "bit_identical": same}), flush=True)


if __name__ == "__main__":
    main()
