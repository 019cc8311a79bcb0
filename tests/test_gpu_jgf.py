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


@pytest.mark.parametrize("dtype", [torch.float32, torch.float64])
@pytest.mark.parametrize("n0,count", [(0, 1), (0, 1000), (99_000, 1000), (123_456_789, 257)])
def test_series_matches_oracle(lime, dtype, n0, count):
    if dtype == torch.float64 and n0 > 1_000_000:
        # the oracle's double cos(n pi x) carries an argument error ~ n pi x 2^-53 (~1e-7 rad at
        # n ~ 1e8) that exceeds the fp64 tolerance; the GPU reduces the phase exactly
        pytest.skip("oracle argument precision limits the fp64 comparison to n <= 1e6")
    out = lime.map_series(n0, count, dtype=dtype).cpu().numpy()
    ref, mag = oracle.series(n0, count, threads=THREADS)
    assert (np.abs(out - ref) / mag[:, None]).max() <= SERIES_TOL[dtype]


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
