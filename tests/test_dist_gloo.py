"""Multi-rank partition/exchange logic on CPU: world_size 2 over gloo (no GPU).

The map/integrator callables are test stand-ins built on the oracle (test infrastructure);
what is under test is paper_conf_pldi_dubachcrbf12_b200.dist: shard ranges, the all-gather of
positions each step, the all-reduce of Black-Scholes partials, the cyclic Mandelbrot rows.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist
from paper_conf_pldi_dubachcrbf12_b200 import inputs

EPS2, DT = 1e-4, 1e-3


def _force(pos_full, begin, count, eps2, out):
    a = oracle.nbody_accel(pos_full.numpy(), np.float32(eps2), begin, count)
    out[:, :3] = torch.from_numpy(a.astype(np.float32))
    out[:, 3] = 0


def _integrate(pos, vel, accel, dt):
    p, v = oracle.nbody_integrate(pos.numpy(), vel.numpy(), accel.numpy(), np.float32(dt))
    pos.copy_(torch.from_numpy(p.astype(np.float32)))
    vel.copy_(torch.from_numpy(v.astype(np.float32)))


def _bs_fused(S, X, T, r, sigma):
    return torch.tensor(oracle.blackscholes_sums(S.numpy(), X.numpy(), T.numpy(), r, sigma), dtype=torch.float64)


def _mandel_fn(width, height, x0, y0, dx, dy, max_iter, row_first, row_stride, row_count, device, out):
    return torch.from_numpy(oracle.mandelbrot(width, height, row_first, row_stride, row_count, x0, y0, dx, dy,
                                              max_iter))


def _mm_fn(A, Bt, out):
    return torch.from_numpy(oracle.matmul_bf16(A.numpy().view(np.uint16), Bt.numpy().view(np.uint16)))


MW, MH, MITER = 40, 37, 200          # ragged: 37 rows over 2 ranks (19 + 18)
MM = (45, 24, 16)                    # ragged: 45 rows of C over 2 ranks (23 + 22)


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
        bodies = torch.from_numpy(inputs.nbody_bodies(n, seed=31))
        sim = ldist.NBodySim(bodies, EPS2, DT, "cpu", force_fn=_force, integrate_fn=_integrate)
        for _ in range(steps):
            sim.step()
        mom = sim.momentum()
        pos = [torch.empty_like(sim.pos) for _ in range(world)]
        dist.all_gather(pos, sim.pos)
        S, X, T = (torch.from_numpy(a) for a in inputs.blackscholes_options(1000, seed=4))
        b, c = ldist.shard_range(1000, rank, world)
        tot = ldist.blackscholes_total(S[b:b + c], X[b:b + c], T[b:b + c], inputs.BS_R, inputs.BS_SIGMA,
                                       fused_fn=_bs_fused)
        tot_s = ldist.blackscholes_shard_total(S, X, T, inputs.BS_R, inputs.BS_SIGMA, fused_fn=_bs_fused)
        loc = ldist.mandelbrot_cyclic(MW, MH, -2.0, -1.5, 3.0 / MW, 3.0 / MH, MITER, device="cpu", map_fn=_mandel_fn)
        frame = ldist.gather_cyclic_rows(loc, MH)
        A, Bt = (torch.from_numpy(a.view(np.int16)) for a in inputs.matmul_operands(*MM, seed=3))
        C = ldist.gather_row_blocks(ldist.matmul_row_block(A, Bt, mm_fn=_mm_fn), MM[0])
        if rank == 0:
            q.put((torch.cat(pos).numpy(), mom.numpy(), tot.numpy(), tot_s.numpy(), frame.numpy(), C.numpy()))
    finally:
        dist.destroy_process_group()


def _run(world, n, steps):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, n, steps, q)) for r in range(world)]
    for p in ps:
        p.start()
    out = q.get(timeout=240)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    return out


def test_shard_helpers():
    for n in (0, 1, 7, 1 << 20):
        for w in (1, 2, 3, 8):
            parts = [ldist.shard_range(n, r, w) for r in range(w)]
            assert sum(c for _, c in parts) == n
            assert all(parts[k][0] + parts[k][1] == parts[k + 1][0] for k in range(w - 1))
    for n in (0, 3, 1000, (1 << 20) + 37):
        for w in (1, 2, 3, 8):
            parts = [ldist.shard_range_aligned(n, r, w, 4) for r in range(w)]
            assert sum(c for _, c in parts) == n and all(b % 4 == 0 for b, _ in parts)
            assert all(parts[k][0] + parts[k][1] == parts[k + 1][0] for k in range(w - 1))
    rows = []
    for k in range(3):
        first, stride, count = ldist.cyclic_rows(10, k, 3)
        rows += [first + i * stride for i in range(count)]
    assert sorted(rows) == list(range(10))


@pytest.mark.timeout(300)
def test_two_rank_nbody_and_bs_match_single_rank():
    n, steps = 64, 3
    pos2, mom2, tot2, tots2, frame2, C2 = _run(2, n, steps)
    pos1, mom1, tot1, tots1, frame1, C1 = _run(1, n, steps)
    assert np.array_equal(pos2, pos1)                  # sharded all-gather sim == single rank
    assert np.allclose(mom2, mom1, atol=1e-12)
    assert abs(mom1).max() < 1e-6                       # momentum conserved (Sum m v ~ 0)
    np.testing.assert_allclose(tot2, tot1, rtol=1e-13)  # all-reduce of partials
    ref = oracle.blackscholes_sums(*inputs.blackscholes_options(1000, seed=4), inputs.BS_R, inputs.BS_SIGMA)
    np.testing.assert_allclose(tot1, ref, rtol=1e-15)
    np.testing.assert_allclose(tots2, ref, rtol=1e-13)   # strong-scaled shards + all-reduce
    # cyclic Mandelbrot rows and matmul row blocks, reassembled, equal the unsharded oracle exactly
    full = oracle.mandelbrot(MW, MH, 0, 1, MH, -2.0, -1.5, 3.0 / MW, 3.0 / MH, MITER)
    assert np.array_equal(frame2, full) and np.array_equal(frame1, full)
    Cref = oracle.matmul_bf16(*inputs.matmul_operands(*MM, seed=3))
    assert np.array_equal(C2, Cref) and np.array_equal(C1, Cref)
