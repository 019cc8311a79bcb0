"""F1: the paper's Fig. 8 memory-mapping ablation rebuilt on B200 for the N-Body force map.
Times every staging variant (bit-identical results) at the paper's 4096 bodies (config 1) and at
the config-5 per-GPU shape of P = 8 (2^17 targets x 2^20 sources). L2 flushed before each launch."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_dubachcrbf12_b200 as lime  # noqa: E402
from paper_conf_pldi_dubachcrbf12_b200 import inputs  # noqa: E402
from bench import time_launches  # noqa: E402


def main():
    lime.load()
    flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
    for name, n, cnt, reps, ov in [("config1_n4096", 4096, 4096, 30, (128, 2)), ("config5_p8", 1 << 20, 1 << 17, 3, (256, 2))]:
        b = torch.from_numpy(inputs.nbody_bodies(n, seed=5)).cuda()
        out = torch.empty((cnt, 4), dtype=torch.float32, device="cuda")
        ref = lime.map_nbody(b, 1e-4, 0, cnt).clone()
        rows = []
        if n <= 8192:
            ms = time_launches(lambda: lime.map_nbody(b, 1e-4, 0, cnt, out=out), reps, 3, flush)[0]
            rows.append(("small_path (production, in-CTA splits)", ms, True))
        for v in range(0, 7):
            if v == 6 and n > 4096:
                continue
            with lime.nbody_variant(v), lime.launch_override(block_threads=ov[0], per_thread=ov[1]):
                ms = time_launches(lambda: lime.map_nbody(b, 1e-4, 0, cnt, out=out), reps, 2, flush)[0]
                same = bool(torch.equal(out, ref))
            rows.append((lime.NBODY_VARIANTS[v], ms, same))
        best = min(r[1] for r in rows)
        for nm, ms, same in rows:
            print(json.dumps({"case": name, "variant": nm, "ms": ms, "Ginteractions_s": n * cnt / ms / 1e6,
                              "rel_to_best": best / ms, "bit_identical": same}), flush=True)


if __name__ == "__main__":
    main()
