"""bench.py's N > 1 path on the one GPU: two ranks under torchrun over gloo (LIME_DIST_BACKEND=gloo;
NCCL needs a GPU per rank), small headline size. Checks the contract line and that every sharded
config is reported with a max-over-ranks time."""
import json
import os
import subprocess
import sys

import pytest

from testutil import ROOT, golden

pytestmark = pytest.mark.gpu


@pytest.mark.timeout(900)
def test_bench_two_ranks_gloo():
    env = dict(os.environ, LIME_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29517", "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "3", "--bodies", "16384", "--no-extras"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=850)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["config"]["targets_per_gpu"] == 8192
    sc = d["sharded_configs"]
    for k in ("blackscholes_map_reduce_strong", "blackscholes_map_reduce_weak", "mandelbrot_cyclic_rows",
              "matmul_row_blocks"):
        assert sc[k]["value"] > 0, k
    # both ranks' rows together are the full frame: its checksum (survey probe, tests/golden)
    assert sc["mandelbrot_cyclic_rows"]["checksum"] == golden("mandelbrot_points.json")["frame"]["checksum"]
    assert sc["mandelbrot_cyclic_rows"]["rows_per_gpu"] == 4096
    assert sc["matmul_row_blocks"]["rows_per_gpu"] == 4096
