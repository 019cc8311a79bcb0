"""GPU: a workspace reused across calls of different sizes (the binding caches one per kind) must
give the same results as a fresh one -- no stale partials or flags may reach a later call's split
tickets (include/lime.h "Workspaces")."""
import numpy as np
import pytest
import torch

import paper_conf_pldi_dubachcrbf12_b200 as lime_pkg
from paper_conf_pldi_dubachcrbf12_b200 import inputs

pytestmark = pytest.mark.gpu


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _fresh(fn):
    lime_pkg._ws_cache.clear()
    out = fn().cpu()
    lime_pkg._ws_cache.clear()
    return out


# (n_src, tgt_begin, tgt_count): small target tiles first, then larger counter regions over
# regions earlier calls filled with partials / flags
NBODY_SEQ = [(1 << 15, 0, 1000), (20000, 0, 20000), (50000, 0, 50000), (9000, 0, 9000),
             (1 << 15, 100, 30000), (50000, 7, 1234)]


def test_nbody_workspace_reuse_across_sizes(lime):
    bodies = {n: _dev(inputs.nbody_bodies(n, seed=n)) for n in {s[0] for s in NBODY_SEQ}}
    fresh = [_fresh(lambda: lime.map_nbody(bodies[n], 1e-4, b, c)) for n, b, c in NBODY_SEQ]
    for _ in range(2):
        for (n, b, c), ref in zip(NBODY_SEQ, fresh):
            assert torch.equal(lime.map_nbody(bodies[n], 1e-4, b, c).cpu(), ref), (n, b, c)


def test_nbody_f64_workspace_reuse_across_sizes(lime):
    seq = [(20000, 0, 500), (5000, 0, 5000), (20000, 0, 20000), (5000, 10, 100)]
    bodies = {n: _dev(inputs.nbody_bodies(n, seed=n).astype(np.float64)) for n in {s[0] for s in seq}}
    fresh = [_fresh(lambda: lime.map_nbody_f64(bodies[n], 1e-4, b, c)) for n, b, c in seq]
    for _ in range(2):
        for (n, b, c), ref in zip(seq, fresh):
            assert torch.equal(lime.map_nbody_f64(bodies[n], 1e-4, b, c).cpu(), ref), (n, b, c)


def test_coulomb_workspace_reuse_across_sizes(lime):
    seq = [(3968, 64, 64), (1000, 256, 256), (3968, 512, 512), (500, 100, 37)]
    atoms = {na: _dev(inputs.cp_atoms(na, seed=na)) for na in {s[0] for s in seq}}
    fresh = [_fresh(lambda: lime.map_coulomb(atoms[na], nx, ny, 25.6, 0.1)) for na, nx, ny in seq]
    for _ in range(2):
        for (na, nx, ny), ref in zip(seq, fresh):
            assert torch.equal(lime.map_coulomb(atoms[na], nx, ny, 25.6, 0.1).cpu(), ref), (na, nx, ny)


def test_mriq_workspace_reuse_across_sizes(lime):
    seq = [(3072, 1000), (512, 32768), (3072, 32768), (100, 77)]
    ks = {nk: _dev(inputs.mriq_kspace(nk, seed=nk)) for nk in {s[0] for s in seq}}
    vs = {nx: _dev(inputs.mriq_voxels(nx, seed=nx)) for nx in {s[1] for s in seq}}
    fresh = [_fresh(lambda: lime.map_mriq(ks[nk], vs[nx])) for nk, nx in seq]
    for _ in range(2):
        for (nk, nx), ref in zip(seq, fresh):
            assert torch.equal(lime.map_mriq(ks[nk], vs[nx]).cpu(), ref), (nk, nx)
