"""Sweep the N-Body force kernel's launch variants (exhaustive offline tuning of
thread count / mapping). Results are bit-identical across variants; only time changes."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402


def timeit(fn, reps):
    fn()
    torch.cuda.synchronize()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 * reps)]
    for i in range(reps):
        ev[2 * i].record()
        fn()
        ev[2 * i + 1].record()
    torch.cuda.synchronize()
    return min(ev[2 * i].elapsed_time(ev[2 * i + 1]) for i in range(reps))


def main():
    lime.load()
    cases = [("n4096", 4096, 4096, 20), ("p8", 1 << 20, 1 << 17, 3), ("p1", 1 << 20, 1 << 20, 2)]
    variants = [(0, 0)] + [(b, r) for b in (128, 256) for r in (1, 2, 4, 8)]
    for name, n, cnt, reps in cases:
        b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
        out = torch.empty((cnt, 4), dtype=torch.float32, device="cuda")
        ref = None
        for blk, r in variants:
            with lime.launch_override(block_threads=blk, per_thread=r):
                ms = timeit(lambda: lime.map_nbody(b, 1e-4, 0, cnt, out=out), reps)
                res = out.clone()
            if ref is None:
                ref = res
            same = bool(torch.equal(res, ref))
            print(json.dumps({"case": name, "block": blk, "R": r, "ms": ms,
                              "Gint_s": n * cnt / (ms * 1e-3) / 1e9, "bit_identical": same}), flush=True)


if __name__ == "__main__":
    main()
