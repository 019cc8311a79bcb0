"""One N-Body staging-variant launch for ncu (F1, Fig. 8): warm-up outside the profiled
range, then exactly one lime_map_nbody call between cudaProfilerStart/Stop.

    ncu --set full --profile-from-start off -k regex:force -o OUT python tools/prof_ablation.py CASE VARIANT
CASE: config1_n4096 | config5_p8; VARIANT: small (production small-N path) or 0..6 (NBODY_VARIANTS)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402

CASES = {"config1_n4096": (4096, 4096, (128, 2)), "config5_p8": (1 << 20, 1 << 17, (256, 2))}


def main(case, variant):
    lime.load()
    n, cnt, ov = CASES[case]
    b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
    out = torch.empty((cnt, 4), dtype=torch.float32, device="cuda")
    if variant == "small":
        call = lambda: lime.map_nbody(b, 1e-4, 0, cnt, out=out)
        call()
        torch.cuda.synchronize()
        torch.cuda.profiler.start()
        call()
        torch.cuda.synchronize()
        torch.cuda.profiler.stop()
        return
    with lime.nbody_variant(int(variant)), lime.launch_override(block_threads=ov[0], per_thread=ov[1]):
        lime.map_nbody(b, 1e-4, 0, cnt, out=out)
        torch.cuda.synchronize()
        torch.cuda.profiler.start()
        lime.map_nbody(b, 1e-4, 0, cnt, out=out)
        torch.cuda.synchronize()
        torch.cuda.profiler.stop()


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
