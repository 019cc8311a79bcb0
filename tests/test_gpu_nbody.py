"""GPU parity: N-Body force map and integrator vs the oracle (through the C ABI)."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import NBODY_RTOL, nbody_rel_err

pytestmark = pytest.mark.gpu
EPS2 = np.float32(1e-4)


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("n", [1, 2, 3, 31, 33, 255, 256, 257, 1000, 4096, 4097])
def test_force_matches_oracle(lime, n):
    b = inputs.nbody_bodies(n, seed=100 + n)
    acc = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    ref, mag = oracle.nbody_accel(b, EPS2, with_mag=True)
    err = nbody_rel_err(acc, ref, mag)
    assert err.max() <= NBODY_RTOL, (n, err.max())
    assert np.all(acc[:, 3] == 0.0)


def test_single_body_and_self_term(lime):
    b = np.array([[0.25, -0.5, 0.75, 3.0]], dtype=np.float32)
    assert np.all(lime.map_nbody(_dev(b), 1e-4).cpu().numpy() == 0.0)


def test_shards_are_slices_and_launch_independent(lime):
    n = 4097
    b = _dev(inputs.nbody_bodies(n, seed=7))
    full = lime.map_nbody(b, float(EPS2)).cpu()
    for begin, count in [(0, 1), (1, 1000), (2048, 2049), (4000, 97), (17, 0)]:
        part = lime.map_nbody(b, float(EPS2), begin, count).cpu()
        assert torch.equal(part, full[begin:begin + count])
    for block, R in [(b_, r_) for b_ in (128, 256) for r_ in (1, 2, 4, 8)] + [(512, 2), (512, 4)]:
        with lime.launch_override(block_threads=block, per_thread=R):
            alt = lime.map_nbody(b, float(EPS2)).cpu()
        assert torch.equal(alt, full), (block, R)


def test_p_way_sharding_bit_identical(lime):
    n = 1 << 14
    b = _dev(inputs.nbody_bodies(n, seed=8))
    full = lime.map_nbody(b, float(EPS2)).cpu()
    for P in (2, 4, 8):
        parts = [lime.map_nbody(b, float(EPS2), r * n // P, n // P).cpu() for r in range(P)]
        assert torch.equal(torch.cat(parts), full)


def test_momentum_and_determinism(lime):
    for n in (4096, 16384):
        b = inputs.nbody_bodies(n, seed=9)
        bd = _dev(b)
        a1 = lime.map_nbody(bd, float(EPS2))
        a2 = lime.map_nbody(bd, float(EPS2))
        assert torch.equal(a1, a2)                                  # run-to-run bit identical
        a = a1.cpu().numpy()[:, :3].astype(np.float64)
        m = b[:, 3].astype(np.float64)
        P = (m[:, None] * a).sum(0)
        assert np.linalg.norm(P) <= 1e-6 * (m * np.linalg.norm(a, axis=1)).sum()
        assert torch.equal(bd.cpu(), torch.from_numpy(b))          # input untouched (L139-143)


def test_config5_sampled_targets(lime):
    n = 1 << 20
    b = inputs.nbody_bodies(n, seed=5)
    acc = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    rows = np.random.default_rng(0).choice(n, 256, replace=False)
    rows = np.concatenate([rows, [0, n - 1]])
    ref, mag = oracle.nbody_accel_rows(b, EPS2, rows, threads=8)
    err = nbody_rel_err(acc[rows], ref, mag)
    assert err.max() <= NBODY_RTOL, err.max()


def test_config5_sharded_launch_matches_full(lime):
    # the launch bench.py times at P = 8: 2^17 targets against 2^20 sources
    n, P = 1 << 20, 8
    b = _dev(inputs.nbody_bodies(n, seed=5))
    for r in (0, 5):
        part = lime.map_nbody(b, float(EPS2), r * n // P, n // P)
        full_slice = lime.map_nbody(b, float(EPS2), r * n // P, 1024)
        assert torch.equal(part[:1024], full_slice)


def test_integrator_one_step(lime):
    n = 3001
    b = inputs.nbody_bodies(n, seed=12)
    vel = (inputs.nbody_bodies(n, seed=13) * np.float32(0.1)).astype(np.float32)
    vel[:, 3] = 0
    acc = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    pos_d, vel_d, acc_d = _dev(b), _dev(vel), _dev(acc)
    lime.map_nbody_integrate(pos_d, vel_d, acc_d, 1e-3)
    p_ref, v_ref = oracle.nbody_integrate(b, vel, acc, np.float32(1e-3))
    np.testing.assert_allclose(vel_d.cpu().numpy(), v_ref, rtol=0, atol=2e-7 * np.abs(v_ref).max() + 1e-12)
    np.testing.assert_allclose(pos_d.cpu().numpy(), p_ref, rtol=0, atol=2e-7)
    assert np.array_equal(pos_d.cpu().numpy()[:, 3], b[:, 3])     # mass carried


def test_simulate_host_matches_device_path(lime):
    n, steps = 2048, 3
    b = inputs.nbody_bodies(n, seed=14)
    h_pos = torch.from_numpy(b.copy()).pin_memory()
    h_vel = torch.zeros((n, 4), dtype=torch.float32).pin_memory()
    lime.nbody_simulate_host(h_pos, h_vel, steps, 1e-4, 1e-3)
    pos, vel = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    for _ in range(steps):
        a = lime.map_nbody(pos, 1e-4)
        lime.map_nbody_integrate(pos, vel, a, 1e-3)
    assert torch.equal(h_pos, pos.cpu()) and torch.equal(h_vel, vel.cpu())


def test_errors_surface_as_exceptions(lime):
    b = _dev(inputs.nbody_bodies(16, seed=1))
    with pytest.raises(lime.LimeError, match="INVALID_ARG"):
        lime.map_nbody(b, 0.0)
    with pytest.raises(lime.LimeError, match="INVALID_ARG"):
        lime.map_nbody(b, 1e-4, 10, 7)


@pytest.mark.parametrize("n,count", [(4096, 4096), (3000, 1000), (1 << 17, 1 << 12)])
def test_staging_ablation_variants_bit_identical(lime, n, count):
    # F1 (Fig. 8): every memory-mapping variant computes the same sums in the same order
    b = _dev(inputs.nbody_bodies(n, seed=21))
    ref = lime.map_nbody(b, float(EPS2), 0, count).cpu()
    for v in range(1, 7):
        if v == 6 and n > 4096:
            continue
        with lime.nbody_variant(v):
            got = lime.map_nbody(b, float(EPS2), 0, count).cpu()
        assert torch.equal(got, ref), v


# ------------------------------------------------------- F3: double precision (Table 3)
NBODY64_RTOL = 1e-12   # fp64 with reordered summation


@pytest.mark.parametrize("n", [1, 2, 33, 1000, 4096, 5000])
def test_nbody_f64_matches_oracle(lime, n):
    b = inputs.nbody_bodies(n, seed=40 + n).astype(np.float64)
    b[:, :3] += 1e-9 * (inputs.uniform24(n, 5, 3 * n).reshape(n, 3) - 0.5)     # use the fp64 mantissa
    acc = lime.map_nbody_f64(_dev(b), 1e-4).cpu().numpy()
    ref, mag = oracle.nbody_accel_f64(b, 1e-4, with_mag=True)
    assert nbody_rel_err(acc, ref, mag).max() <= NBODY64_RTOL
    assert np.all(acc[:, 3] == 0.0)


def test_nbody_f64_shards_and_config5_sample(lime):
    n = 1 << 16
    b = inputs.nbody_bodies(n, seed=44).astype(np.float64)
    bd = _dev(b)
    full = lime.map_nbody_f64(bd, 1e-4).cpu()
    for P in (2, 8):
        parts = [lime.map_nbody_f64(bd, 1e-4, r * n // P, n // P).cpu() for r in range(P)]
        assert torch.equal(torch.cat(parts), full)
    rows = np.random.default_rng(1).choice(n, 64, replace=False)
    ref = np.stack([oracle.nbody_accel_f64(b, 1e-4, int(r), 1, with_mag=True)[0][0] for r in rows])
    mag = np.array([oracle.nbody_accel_f64(b, 1e-4, int(r), 1, with_mag=True)[1][0] for r in rows])
    assert nbody_rel_err(full.numpy()[rows], ref, mag).max() <= NBODY64_RTOL


def test_cuda_graph_replay_matches_eager_steps(lime):
    from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist
    n, steps = 4096, 6                              # even: the fused step ping-pongs two buffers
    bodies = torch.from_numpy(inputs.nbody_bodies(n, seed=61))
    eager = ldist.NBodySim(bodies, 1e-4, 1e-3, "cuda:0")
    for _ in range(steps + 1):                      # capture() runs one warm-up step first
        eager.step()
    sim = ldist.NBodySim(bodies, 1e-4, 1e-3, "cuda:0")
    g = sim.capture(steps)
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(sim.pos, eager.pos) and torch.equal(sim.vel, eager.vel)


def _eager_steps(lime, pos, vel, steps, eps2=1e-4, dt=1e-3):
    for _ in range(steps):
        a = lime.map_nbody(pos, eps2)
        lime.map_nbody_integrate(pos, vel, a, dt)


@pytest.mark.parametrize("n", [1, 31, 256, 257, 1000, 4096, 8192, 8193])
def test_simulate_matches_eager_steps(lime, n):
    # lime_nbody_simulate (one persistent launch for n <= 8192) == steps x (force map + integrator)
    b = inputs.nbody_bodies(n, seed=70 + n)
    v0 = (inputs.nbody_bodies(n, seed=71 + n) * np.float32(0.05)).astype(np.float32)
    v0[:, 3] = 0
    pos_e, vel_e = _dev(b), _dev(v0)
    _eager_steps(lime, pos_e, vel_e, 5)
    pos, vel = _dev(b), _dev(v0)
    lime.nbody_simulate(pos, vel, 0, 1e-4, 1e-3)                      # no-op
    assert torch.equal(pos, _dev(b))
    lime.nbody_simulate(pos, vel, 3, 1e-4, 1e-3)                      # odd: ends in the ping-pong buffer
    lime.nbody_simulate(pos, vel, 2, 1e-4, 1e-3)                      # barrier words were reset
    assert torch.equal(pos, pos_e) and torch.equal(vel, vel_e)


def test_simulate_grid_independent_and_oracle(lime):
    n, steps = 4096, 4
    b = inputs.nbody_bodies(n, seed=80)
    ref_p, ref_v = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    lime.nbody_simulate(ref_p, ref_v, steps, 1e-4, 1e-3)
    for g in (1, 7, 64):                                              # CTAs loop over 32-target groups
        p, v = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
        with lime.launch_override(grid_ctas=g):
            lime.nbody_simulate(p, v, steps, 1e-4, 1e-3)
        assert torch.equal(p, ref_p) and torch.equal(v, ref_v), g
    # one step against the oracle (force, then the integrator)
    p, v = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    lime.nbody_simulate(p, v, 1, 1e-4, 1e-3)
    acc, mag = oracle.nbody_accel(b, float(EPS2), with_mag=True)
    po, vo = oracle.nbody_integrate(b, np.zeros((n, 4), np.float32), np.concatenate([acc, np.zeros((n, 1))], 1), 1e-3)
    vg = v.cpu().numpy()
    assert (np.abs(vg[:, :3] - vo[:, :3]).max(axis=1) <= NBODY_RTOL * mag * 1e-3 + 1e-12).all()
    np.testing.assert_allclose(p.cpu().numpy(), po, rtol=0, atol=2e-7)


def test_simulate_host_small_path(lime):
    n, steps = 4096, 3
    b = inputs.nbody_bodies(n, seed=81)
    h_pos = torch.from_numpy(b.copy()).pin_memory()
    h_vel = torch.zeros((n, 4), dtype=torch.float32).pin_memory()
    lime.nbody_simulate_host(h_pos, h_vel, steps, 1e-4, 1e-3)
    pos, vel = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    _eager_steps(lime, pos, vel, steps)
    assert torch.equal(h_pos, pos.cpu()) and torch.equal(h_vel, vel.cpu())


def test_config5_steps_one_step_parity(lime):
    # SURVEY.md §8(c) C-integrator: at each checked step the oracle recomputes the forces of sampled
    # targets against all 2^20 sources FROM THE GPU'S CURRENT POSITIONS and applies the integrator
    # (one-step parity; avoids comparing chaotic multi-step trajectories).
    n, steps, dt = 1 << 20, 3, 1e-3
    b = inputs.nbody_bodies(n, seed=5)
    pos, vel = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    rows = np.concatenate([np.random.default_rng(3).choice(n, 96, replace=False), [0, n - 1]])
    for _ in range(steps):
        p0, v0 = pos.cpu().numpy(), vel.cpu().numpy()
        lime.nbody_simulate(pos, vel, 1, float(EPS2), dt)
        acc, mag = oracle.nbody_accel_rows(p0, EPS2, rows, threads=8)
        a4 = np.zeros((rows.size, 4), np.float32)
        a4[:, :3] = acc
        po, vo = oracle.nbody_integrate(p0[rows], v0[rows], a4, np.float32(dt))
        vg, pg = vel.cpu().numpy()[rows], pos.cpu().numpy()[rows]
        dv = np.abs(vg[:, :3] - vo[:, :3]).max(axis=1)
        assert (dv <= NBODY_RTOL * mag * dt + 4e-7 * np.abs(vo[:, :3]).max(axis=1) + 1e-12).all(), dv.max()
        np.testing.assert_allclose(pg, po, rtol=0, atol=3e-7)


def test_momentum_after_ten_steps(lime):
    # SURVEY.md §8(c) pin: |sum m v| <= 1e-6 sum m |v| after 10 steps from rest
    for n in (4096, 1 << 16):
        b = inputs.nbody_bodies(n, seed=11)
        pos, vel = _dev(b), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
        lime.nbody_simulate(pos, vel, 10, float(EPS2), 1e-3)
        m = b[:, 3].astype(np.float64)
        v = vel.cpu().numpy()[:, :3].astype(np.float64)
        P = (m[:, None] * v).sum(0)
        assert np.linalg.norm(P) <= 1e-6 * (m * np.linalg.norm(v, axis=1)).sum()


# ------------------------------------------------- R11: mass-uniform splits (n_src > 8192)
def _mixed_split_bodies(lime, n, seed, perturbed_splits):
    """Equal masses 1/n (not a power of two) except in the listed splits, whose masses vary."""
    b = inputs.nbody_bodies(n, seed=seed)
    b[:, 3] = np.float32(1.0 / n)
    S = lime.nbody_splits(n)
    chunks = -(-n // 256)
    split_len = -(-chunks // S) * 256                    # chunks_per_split * 256 (R11)
    rng = np.random.default_rng(seed)
    for s in perturbed_splits:
        lo, hi = s * split_len, min(n, (s + 1) * split_len)
        b[lo:hi, 3] = (rng.uniform(0.5, 1.5, hi - lo) / n).astype(np.float32)
    return b


@pytest.mark.parametrize("n,perturbed", [(20000, []), (20000, [3, 7]), (50000, [0]), (50000, list(range(16)))])
def test_mass_uniform_splits_match_oracle(lime, n, perturbed):
    b = _mixed_split_bodies(lime, n, 300 + n, perturbed)
    acc = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    rows = np.random.default_rng(n).choice(n, 300, replace=False)
    rows = np.concatenate([rows, [0, n - 1]])
    ref, mag = oracle.nbody_accel_rows(b, EPS2, rows, threads=8)
    err = nbody_rel_err(acc[rows], ref, mag)
    assert err.max() <= NBODY_RTOL, err.max()


def test_mass_uniform_splits_bit_identity(lime):
    # factored (mass-uniform) and per-body-mass splits in one call: shards, launch configurations
    # and every staging-ablation variant must still agree bit for bit
    n = 20000
    b = _dev(_mixed_split_bodies(lime, n, 77, [2, 9, 15]))
    full = lime.map_nbody(b, float(EPS2)).cpu()
    for begin, count in [(0, 5000), (5000, 15000), (12345, 99)]:
        assert torch.equal(lime.map_nbody(b, float(EPS2), begin, count).cpu(), full[begin:begin + count])
    for block, R in [(128, 1), (128, 2), (256, 2), (256, 4), (256, 8), (512, 2), (512, 4)]:
        with lime.launch_override(block_threads=block, per_thread=R):
            assert torch.equal(lime.map_nbody(b, float(EPS2)).cpu(), full), (block, R)
    for v in range(1, 6):
        with lime.nbody_variant(v):
            assert torch.equal(lime.map_nbody(b, float(EPS2)).cpu(), full), v


def test_mass_uniform_edge_masses(lime):
    # a massless body breaks its split's uniformity; an all-massless split contributes exactly 0
    n = 1 << 14
    rows = np.arange(0, n, 97)
    b = inputs.nbody_bodies(n, seed=55)
    b[n - 1, 3] = 0.0
    acc = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    ref, mag = oracle.nbody_accel_rows(b, EPS2, rows, threads=8)
    assert nbody_rel_err(acc[rows], ref, mag).max() <= NBODY_RTOL
    S = lime.nbody_splits(n)
    split_len = -(-(-(-n // 256)) // S) * 256
    b[:split_len, 3] = 0.0                               # split 0 massless: uniform with m = 0
    acc0 = lime.map_nbody(_dev(b), float(EPS2)).cpu().numpy()
    ref0, mag0 = oracle.nbody_accel_rows(b, EPS2, rows, threads=8)
    assert np.all(np.isfinite(acc0))
    assert nbody_rel_err(acc0[rows], ref0, mag0).max() <= NBODY_RTOL


@pytest.mark.parametrize("n", [31, 1000, 4096, 4097, 8192, 8193, 20000])
def test_fused_step_matches_map_then_integrate(lime, n):
    # lime_map_nbody_step (force map with the integrator fused in, out-of-place positions) is
    # bit-identical to lime_map_nbody + lime_map_nbody_integrate, whole range and shards
    b = inputs.nbody_bodies(n, seed=90 + n)
    v0 = (inputs.nbody_bodies(n, seed=91 + n) * np.float32(0.05)).astype(np.float32)
    v0[:, 3] = 0
    for begin, count in [(0, n), (n // 3, n // 2), (n - 1, 1)]:
        pos, vel = _dev(b), _dev(v0)
        acc = lime.map_nbody(pos, float(EPS2), begin, count)
        p_ref = pos[begin:begin + count].clone()
        v_ref = vel[begin:begin + count].clone()
        lime.map_nbody_integrate(p_ref, v_ref, acc, 1e-3)
        v = vel[begin:begin + count].clone()
        p_new = lime.map_nbody_step(pos, float(EPS2), 1e-3, v, begin, count)
        assert torch.equal(p_new, p_ref) and torch.equal(v, v_ref), (n, begin, count)
        assert torch.equal(pos, _dev(b))                              # sources untouched


def test_fused_step_rejects_aliasing(lime):
    pos = _dev(inputs.nbody_bodies(256, seed=3))
    vel = torch.zeros_like(pos)
    with pytest.raises(lime.LimeError):
        lime.map_nbody_step(pos, float(EPS2), 1e-3, vel, out=pos)        # out of place only


def test_graph_of_fused_steps_matches_eager(lime):
    from paper_conf_pldi_dubachcrbf12_b200 import dist as ldist
    n = 4096
    b = torch.from_numpy(inputs.nbody_bodies(n, seed=95))
    sim = ldist.NBodySim(b, float(EPS2), 1e-3, "cuda")
    g = sim.capture(10)                                               # includes one warm-up step
    g.replay()
    torch.cuda.synchronize()
    pos, vel = _dev(b.numpy()), torch.zeros((n, 4), dtype=torch.float32, device="cuda")
    _eager_steps(lime, pos, vel, 11)
    assert torch.equal(sim.pos, pos) and torch.equal(sim.vel, vel)


@pytest.mark.parametrize("n", [64, 128, 1088, 2112, 4032])
def test_tma_staged_sizes_match_general_kernel(lime, n):
    # n % 64 == 0 (n <= 4096) stages the sources with TMA row boxes of 16 splits; S = n / 64 not a
    # multiple of 16 leaves zero-filled rows in the last box. Forces must equal the general
    # kernel (launch override) bit for bit, on shards too, and the persistent simulation the
    # eager fused steps.
    b = _dev(inputs.nbody_bodies(n, seed=200 + n))
    full = lime.map_nbody(b, float(EPS2))
    with lime.launch_override(block_threads=128, per_thread=2):
        assert torch.equal(lime.map_nbody(b, float(EPS2)), full)
    begin, count = n // 5, n // 2
    assert torch.equal(lime.map_nbody(b, float(EPS2), begin, count), full[begin:begin + count])
    pos, vel = b.clone(), torch.zeros_like(b)
    lime.nbody_simulate(pos, vel, 3, float(EPS2), 1e-3)
    pe, ve = b.clone(), torch.zeros_like(b)
    _eager_steps(lime, pe, ve, 3)
    assert torch.equal(pos, pe) and torch.equal(vel, ve)


# ------------------------------ R11 at the small sizes: factored power-of-two chunks (every small kernel)
def _mixed_chunk_bodies(n, seed):
    """Chunk 0 (and every chunk not listed) mass 2^-12; chunk 1 random masses; chunk 2 one body
    (not first, middle or last: the kernels' prediction says "factored") off by one ulp; chunk 3
    massless; chunk 4 equal but not a power of two (1/3000); chunk 5 equal 2^-41 (outside the
    factored range); the ragged last chunk 2^3."""
    b = inputs.nbody_bodies(n, seed=seed)
    b[:, 3] = np.float32(2.0 ** -12)
    rng = np.random.default_rng(seed)
    b[64:128, 3] = rng.uniform(1e-4, 1e-3, 64).astype(np.float32)
    b[128 + 17, 3] = np.nextafter(b[128 + 17, 3], np.float32(1))
    b[192:256, 3] = 0.0
    b[256:320, 3] = np.float32(1.0 / 3000)
    b[320:384, 3] = np.float32(2.0 ** -41)
    tail = n - (n % 64 or 64)
    b[tail:, 3] = np.float32(8.0)
    return b


@pytest.mark.parametrize("n", [400, 4096, 4160, 5000, 8192])
def test_small_factored_chunks_bit_identical(lime, n):
    # the small kernels sum chunks of equal power-of-two masses in the factored (11-op) form, which
    # has the per-body form's bits: the in-CTA map, the general kernel (launch overrides, per-body
    # form), the staging-ablation variants, shards, the fused step and the persistent simulation
    # must all agree bit for bit, and with the oracle within tolerance
    b_np = _mixed_chunk_bodies(n, 400 + n)
    b = _dev(b_np)
    full = lime.map_nbody(b, float(EPS2))
    ref, mag = oracle.nbody_accel(b_np, EPS2, with_mag=True)
    assert nbody_rel_err(full.cpu().numpy(), ref, mag).max() <= NBODY_RTOL
    for block, R in [(128, 1), (256, 2), (512, 4)]:
        with lime.launch_override(block_threads=block, per_thread=R):
            assert torch.equal(lime.map_nbody(b, float(EPS2)), full), (block, R)
    for v in range(1, 7 if n <= 4096 else 6):              # variant 6: constant memory, <= 4096 bodies
        with lime.nbody_variant(v):
            assert torch.equal(lime.map_nbody(b, float(EPS2)), full), v
    begin, count = n // 3, n // 2
    assert torch.equal(lime.map_nbody(b, float(EPS2), begin, count), full[begin:begin + count])
    v0 = (inputs.nbody_bodies(n, seed=401 + n) * np.float32(0.05)).astype(np.float32)
    v0[:, 3] = 0
    v = _dev(v0)
    p_new = lime.map_nbody_step(b, float(EPS2), 1e-3, v)
    p_ref, v_ref = b.clone(), _dev(v0)
    lime.map_nbody_integrate(p_ref, v_ref, full, 1e-3)
    assert torch.equal(p_new, p_ref) and torch.equal(v, v_ref)
    pos, vel = b.clone(), _dev(v0)
    lime.nbody_simulate(pos, vel, 4, float(EPS2), 1e-3)
    pe, ve = b.clone(), _dev(v0)
    _eager_steps(lime, pe, ve, 4)
    assert torch.equal(pos, pe) and torch.equal(vel, ve)


def test_small_factored_needs_softening(lime):
    # eps^2 < 1e-20 turns the factored form off (it bounds R^-3); still bit-identical
    n = 4096
    b = _dev(_mixed_chunk_bodies(n, 9))
    full = lime.map_nbody(b, 1e-22)
    with lime.launch_override(block_threads=256, per_thread=2):
        assert torch.equal(lime.map_nbody(b, 1e-22), full)
    pos, vel = b.clone(), torch.zeros_like(b)
    lime.nbody_simulate(pos, vel, 2, 1e-22, 1e-3)
    pe, ve = b.clone(), torch.zeros_like(b)
    _eager_steps(lime, pe, ve, 2, eps2=1e-22)
    assert torch.equal(pos, pe) and torch.equal(vel, ve)


def test_small_factored_edge_masses_bitwise(lime):
    # range ends of the factored form (2^-40 and 2^20 factored; 2^-41, 2^21, subnormal, -0, inf and
    # NaN masses not) -- the in-CTA kernel must match the general per-body kernel bit for bit
    # (compared as raw words, so NaN results compare too)
    n = 1024
    b = inputs.nbody_bodies(n, seed=77)
    b[:, 3] = np.float32(2.0 ** -12)
    masses = [2.0 ** -40, 2.0 ** 20, 2.0 ** -41, 2.0 ** 21, 2.0 ** -130, -0.0, 1.0]
    for c, m in enumerate(masses):
        b[64 * (c + 1):64 * (c + 2), 3] = np.float32(m)
    b[64 * 9 + 5, 3] = np.inf
    b[64 * 10 + 9, 3] = np.nan
    bd = _dev(b)
    full = lime.map_nbody(bd, float(EPS2))
    with lime.launch_override(block_threads=128, per_thread=2):
        gen = lime.map_nbody(bd, float(EPS2))
    assert torch.equal(full.view(torch.int32), gen.view(torch.int32))
    pos, vel = bd.clone(), torch.zeros_like(bd)
    lime.nbody_simulate(pos, vel, 2, float(EPS2), 1e-3)
    pe, ve = bd.clone(), torch.zeros_like(bd)
    _eager_steps(lime, pe, ve, 2)
    assert torch.equal(pos.view(torch.int32), pe.view(torch.int32)) and torch.equal(vel.view(torch.int32), ve.view(torch.int32))
