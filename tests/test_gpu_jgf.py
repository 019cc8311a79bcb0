"""GPU parity for F4: JG-Series (fp32 and fp64) and JG-Crypt IDEA vs the oracle."""
import os

import numpy as np
import pytest
import torch

import oracle
from paper_conf_pldi_dubachcrbf12_b200 import inputs
from testutil import golden

pytestmark = pytest.mark.gpu
THREADS = os.cpu_count() or 1
SERIES_TOL = {torch.float32: 1e-6, torch.float64: 1e-10}   # |d| <= tol * T[|f|]


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
def test_series_first_coefficients_and_jgf_values(lime, dtype):
    out = lime.map_series(0, 4, dtype=dtype).cpu().numpy()
    ref = np.array(golden("jgf_series_ref.json")["ref"])
    bound = oracle.series(0, 1)[1][0]                                # T[|f|]
    assert np.abs(out - ref).max() <= max(SERIES_TOL[dtype] * bound, 1e-11)


def _congruent(n):
    """DESIGN.md R14b: with nodes x_i = 2i/m (m = 1000), cos/sin(pi (n + m) x_i) = cos/sin(pi n x_i
    + 2 pi i), so a_n and b_n are periodic in n with period m for n >= 1; n maps to the index in
    [1, m] with the same residue, where the oracle's fp64 phase n*pi*x is accurate to ~1e-12 rad."""
    n = np.asarray(n, dtype=np.int64)
    return (n - 1) % 1000 + 1


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("n0,count", [(0, 1), (0, 1000), (99_000, 1000), (123_456_789, 257)])
def test_series_matches_oracle(lime, dtype, n0, count):
    out = lime.map_series(n0, count, dtype=dtype).cpu().numpy()
    if dtype == torch.float64 and n0 > 1_000_000:
        # the oracle's double cos(n pi x) carries an argument error ~ n pi x 2^-53 (~1e-7 rad at
        # n ~ 1e8), above the fp64 tolerance; compare with the congruent coefficients instead
        # (R14b periodicity, pinned on the oracle by test_oracle_pins.test_series_periodic_in_n)
        idx = _congruent(np.arange(n0, n0 + count))
        ref = np.empty((count, 2))
        mag = np.empty(count)
        for k, n in enumerate(idx):
            r, m = oracle.series(int(n), 1)
            ref[k], mag[k] = r[0], m[0]
    else:
        ref, mag = oracle.series(n0, count, threads=THREADS)
    assert (np.abs(out - ref) / mag[:, None]).max() <= SERIES_TOL[dtype]


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
def test_series_large_n_periodic(lime, dtype):
    # the GPU reduces the phase exactly in integers, so the periodicity holds bit for bit at any n
    # (up to the int64 range of n * i): a_{n + k m} = a_n
    base = lime.map_series(1, 1000, dtype=dtype)
    for n0 in (1001, 1_000_001, 123_456_001, ((1 << 40) // 1000) * 1000 + 1):   # all = 1 (mod m)
        assert torch.equal(lime.map_series(n0, 1000, dtype=dtype), base), n0


def test_series_table3_size_sampled_and_shards(lime):
    full = lime.map_series(0, inputs.SERIES_N)
    idx = np.random.default_rng(2).choice(inputs.SERIES_N, 512, replace=False)
    for k in idx[:64]:
        ref, mag = oracle.series(int(k), 1)
        assert (np.abs(full[int(k)].cpu().numpy() - ref[0]) / mag[0]).max() <= SERIES_TOL[torch.float32]
    half = inputs.SERIES_N // 2
    assert torch.equal(torch.cat([lime.map_series(0, half), lime.map_series(half, half)]), full)


def test_idea_key_schedule_and_vector(lime):
    g = golden("idea_test_vector.json")
    ek, dk = lime.idea_key_schedule(g["key"])
    oek, odk = oracle.idea_keys(g["key"])
    assert np.array_equal(ek, oek) and np.array_equal(dk, odk)
    pt = torch.tensor(g["plaintext_bytes"] * 2, dtype=torch.uint8, device="cuda")   # 16 bytes
    ct = lime.map_idea(pt, ek).cpu().numpy()
    assert ct[:8].tolist() == g["ciphertext_bytes"] and ct[8:].tolist() == g["ciphertext_bytes"]


@pytest.mark.parametrize("nbytes", [8, 16, 24, 4096 + 8, inputs.CRYPT_BYTES])
def test_idea_matches_oracle_and_round_trips(lime, nbytes):
    data = inputs.crypt_data(nbytes, seed=nbytes)
    key = inputs.crypt_key()
    ek, dk = lime.idea_key_schedule(key)
    d = torch.from_numpy(data).cuda()
    enc = lime.map_idea(d, ek)
    assert np.array_equal(enc.cpu().numpy(), oracle.idea(data, oracle.idea_keys(key)[0]))
    assert torch.equal(lime.map_idea(enc, dk), d)            # JGF validates decrypt(encrypt(x)) == x
    assert torch.equal(d.cpu(), torch.from_numpy(data))
