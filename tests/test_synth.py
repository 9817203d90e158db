"""Synthetic input generator: determinism and the recipe of DESIGN.md §4 (CPU)."""
import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import synth


def test_deterministic():
    a, b = synth.make_problem("tiny"), synth.make_problem("tiny")
    for x, y in [(a.rec.xyz, b.rec.xyz), (a.rec.q, b.rec.q), (a.lig.type, b.lig.type), (a.spots, b.spots)]:
        np.testing.assert_array_equal(x, y)


@pytest.mark.parametrize("name", ["tiny", "small", "medium"])
def test_sizes_density_charge(name):
    p = synth.make_problem(name)
    cfg = p.cfg
    assert p.rec.xyz.shape == (cfg.n_rec, 3) and p.rec.xyz.dtype == np.float32
    assert p.lig.xyz.shape == (cfg.n_lig, 3) and p.spots.shape == (cfg.n_spots, 3)
    assert abs(float(p.rec.q.astype(np.float64).sum())) < 1e-3          # neutral
    r = np.linalg.norm(p.rec.xyz - p.rec.xyz.mean(0), axis=1).max()
    rho = cfg.n_rec / (4 / 3 * np.pi * r ** 3)
    assert 0.09 < rho < 0.125
    # minimum separation of the jittered lattice >= 0.4 a
    if cfg.n_rec <= 3000:
        d = np.linalg.norm(p.rec.xyz[:, None] - p.rec.xyz[None], axis=-1)
        d[np.diag_indices_from(d)] = 9
        assert d.min() > 0.8
    comp = np.bincount(p.rec.type, minlength=7) / cfg.n_rec
    if cfg.n_rec >= 3000:
        assert abs(comp[synth.T_H] - 0.395) < 0.03 and abs(comp[synth.T_C] - 0.31) < 0.03
    # spots on the surface shell
    c = p.rec.xyz.mean(0)
    ds = np.linalg.norm(p.spots - c, axis=1)
    assert ds.min() >= r - 3.0 - 1e-3
    assert len(np.unique(p.spots, axis=0)) == cfg.n_spots


def test_sweep_library():
    p = synth.make_problem("sweep")
    assert len(p.ligands) == 256
    sizes = [len(m.q) for m in p.ligands]
    assert min(sizes) >= 15 and max(sizes) <= 80


def test_poses_in_region():
    spot, q, t = synth.make_poses(1000, 7, 3.0, seed=1)
    assert spot.min() >= 0 and spot.max() < 7
    assert np.all(np.abs(t) <= 3.0)
    np.testing.assert_allclose(np.linalg.norm(q, axis=1), 1, atol=1e-6)
