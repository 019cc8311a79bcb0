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


# ------------------------------------------------------------------------------------------------
# Every sharded config on the real CUDA kernels, reassembled and compared with the ORACLE (not with
# one rank): two ranks over gloo on the one GPU (the NCCL path differs only in the backend).
MAND = (1000, 777, 512)               # width, height (ragged over 2 ranks: 389 + 388), max_iter
MMS = (1000, 520, 264)                # M (ragged: 500 + 500 ... and 1000 % 3), N, K
BS_N = (1 << 20) + 37                 # options, ragged tail
NB_N = 4098                           # N-Body one step vs the oracle (divisible by 2 and 3)


def _worker_oracle(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_pldi_dubachcrbf12_b200 as lime
        from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist
        from paper_conf_pldi_dubachcrbf12_b200 import inputs
        torch.cuda.set_device(0)
        dev = "cuda:0"
        # config 2: strong (shard of one global array) and weak (each rank's own 2^20 options)
        S, X, T = (torch.from_numpy(a).to(dev) for a in inputs.blackscholes_options(BS_N, seed=21))
        strong = ldist.blackscholes_shard_total(S, X, T, inputs.BS_R, inputs.BS_SIGMA).cpu()
        Sw, Xw, Tw = (torch.from_numpy(a).to(dev) for a in inputs.blackscholes_options(1 << 20, seed=100 + rank))
        weak = ldist.blackscholes_total(Sw, Xw, Tw, inputs.BS_R, inputs.BS_SIGMA).cpu()
        # config 3: cyclic rows, gathered
        W, H, it = MAND
        loc = ldist.mandelbrot_cyclic(W, H, -2.0, -1.5, 3.0 / W, 3.0 / H, it, device=dev)
        frame = ldist.gather_cyclic_rows(loc.cpu(), H)
        # config 4: row blocks, gathered
        A, Bt = (torch.from_numpy(a.view(np.int16)).to(dev).view(torch.bfloat16)
                 for a in inputs.matmul_operands(*MMS, seed=22))
        C = ldist.gather_row_blocks(ldist.matmul_row_block(A, Bt).cpu(), MMS[0])
        # config 5 (shape of config 1): one sharded step
        bodies = torch.from_numpy(inputs.nbody_bodies(NB_N, seed=23))
        sim = ldist.NBodySim(bodies, 1e-4, 1e-3, dev)
        sim.gather()
        sim.force_fn(sim.pos_full, sim.begin, sim.count, sim.eps2, sim.accel)
        acc = [torch.empty_like(sim.accel) for _ in range(world)]
        dist.all_gather(acc, sim.accel)
        sim.integrate_fn(sim.pos, sim.vel, sim.accel, sim.dt)
        pos = [torch.empty_like(sim.pos) for _ in range(world)]
        dist.all_gather(pos, sim.pos)
        if rank == 0:
            q.put((strong.numpy(), weak.numpy(), frame.numpy(), C.numpy(), torch.cat(acc).cpu().numpy(),
                   torch.cat(pos).cpu().numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(900)
@pytest.mark.parametrize("world", [2, 3])
def test_sharded_configs_match_oracle(world):
    import oracle
    from paper_conf_pldi_dubachcrbf12_b200 import inputs
    from testutil import BS_TOL, MATMUL_RTOL, NBODY_RTOL, nbody_rel_err

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker_oracle, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    strong, weak, frame, C, acc, pos = q.get(timeout=600)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    threads = os.cpu_count() or 1
    # Black-Scholes: |d| <= 1e-5 |ref| (the sum of 1e-5-accurate prices)
    ref = np.array(oracle.blackscholes_sums(*inputs.blackscholes_options(BS_N, seed=21), inputs.BS_R, inputs.BS_SIGMA))
    assert np.all(np.abs(strong - ref) <= BS_TOL * np.abs(ref)), (strong, ref)
    refw = sum(np.array(oracle.blackscholes_sums(*inputs.blackscholes_options(1 << 20, seed=100 + r), inputs.BS_R,
                                                 inputs.BS_SIGMA)) for r in range(world))
    assert np.all(np.abs(weak - refw) <= BS_TOL * np.abs(refw)), (weak, refw)
    # Mandelbrot: bit-exact over the whole reassembled frame
    W, H, it = MAND
    assert np.array_equal(frame, oracle.mandelbrot(W, H, 0, 1, H, -2.0, -1.5, 3.0 / W, 3.0 / H, it, threads=threads))
    # matmul: per-entry relative to sum_k |A_ik B_jk|
    A, Bt = inputs.matmul_operands(*MMS, seed=22)
    Cref = oracle.matmul_bf16(A, Bt)
    mag = np.abs(inputs.bf16_bits_to_f32(A)).astype(np.float64) @ np.abs(inputs.bf16_bits_to_f32(Bt)).astype(np.float64).T
    assert (np.abs(C - Cref) / np.maximum(mag, 1e-30)).max() <= MATMUL_RTOL
    # N-Body: the gathered forces of every shard vs the oracle, then the integrated positions
    b = inputs.nbody_bodies(NB_N, seed=23)
    aref, amag = oracle.nbody_accel(b, np.float32(1e-4), with_mag=True)
    assert nbody_rel_err(acc, aref, amag).max() <= NBODY_RTOL
    pref, _ = oracle.nbody_integrate(b, np.zeros_like(b), acc, np.float32(1e-3))
    assert np.abs(pos - pref).max() <= 1e-6
