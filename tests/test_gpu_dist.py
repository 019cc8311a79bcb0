"""Multi-rank N-Body simulation with the real CUDA kernels: two ranks share the one GPU over gloo
(NCCL needs a GPU per rank) and must reproduce the single-rank trajectory bit for bit, because a
target's force sum order depends only on N (R11)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, steps, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist
        from paper_conf_pldi_dubachcrbf12_b200 import inputs
        torch.cuda.set_device(0)
        bodies = torch.from_numpy(inputs.nbody_bodies(n, seed=51))
        sim = ldist.NBodySim(bodies, 1e-4, 1e-3, "cuda:0")
        for _ in range(steps):
            sim.step()
        mom = sim.momentum().cpu()
        pos = [torch.empty_like(sim.pos) for _ in range(world)]
        dist.all_gather(pos, sim.pos)
        if rank == 0:
            q.put((torch.cat(pos).cpu().numpy(), mom.numpy()))
    finally:
        dist.destroy_process_group()


def _run(world, n, steps):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, n, steps, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = q.get(timeout=300)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


@pytest.mark.timeout(600)
def test_two_ranks_reproduce_one_rank_with_cuda_kernels():
    n, steps = 8192, 3
    p2, m2 = _run(2, n, steps)
    p1, m1 = _run(1, n, steps)
    assert np.array_equal(p2, p1)
    assert np.abs(m1).max() < 1e-6 and np.allclose(m2, m1, atol=1e-12)
