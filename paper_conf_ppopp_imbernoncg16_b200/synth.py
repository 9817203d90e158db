"""Seeded synthetic inputs shaped like the paper's workloads.

This module holds NO arithmetic of the method (no scoring, no pose transform,
no Philox, no metaheuristic step).  It only draws receptor / ligand / spot /
pose arrays with numpy so that both the CUDA path and the fp64 oracle are fed
identical canonical fp32/int32 inputs.

Recipe:
  * receptor: N atoms in a ball at protein density rho = 0.116 atoms/A^3,
    jittered cubic lattice a = rho^(-1/3) (jitter +-0.3a), keep the N points
    nearest the centre (the paper's receptors 2BSM 3264 / 2BXG 8609 atoms,
    PAPER.md Table 5);
  * atom types by protein composition (H 39.5 %, HD 11 %, C 31 %, O 9.5 %,
    N 8.5 %, S 0.5 %), charges ~ N(mu_type, sigma_type), net charge removed;
  * ligand: the same generator with n atoms, centred (2BSM 45 / 2BXG 32
    ligand atoms, Table 5);
  * spots: receptor atoms in the outer 3 A shell, stride-selected to the
    configured count ("spots are identified by finding out a specific type of
    atoms in the protein", §3.1 P:84 -- here: surface atoms);
  * microbenchmark poses: uniform random unit quaternions and uniform
    translations in the spot box.
"""
from __future__ import annotations

from dataclasses import dataclass, field
import numpy as np

# type ids of the built-in table (include/vs.h)
T_C, T_N, T_O, T_S, T_H, T_HD, T_X = range(7)
TYPE_NAMES = ["C", "N", "O", "S", "H", "HD", "X"]

_COMPOSITION = [(T_H, 0.395), (T_HD, 0.11), (T_C, 0.31), (T_O, 0.095), (T_N, 0.085), (T_S, 0.005)]
_CHARGE = {T_C: (0.05, 0.25), T_N: (-0.45, 0.15), T_O: (-0.55, 0.10), T_S: (-0.15, 0.10),
           T_H: (0.08, 0.05), T_HD: (0.35, 0.05)}
DENSITY = 0.116  # atoms / A^3


@dataclass
class Config:
    name: str
    n_rec: int
    n_lig: int
    n_spots: int
    population: int
    generations: int
    index: int
    n_ligands: int = 1              # screening sweep: library size
    lig_min: int = 0                # screening sweep: ligand size range
    lig_max: int = 0

    @property
    def data_seed(self) -> int:
        return 1000 + self.index


# BASELINE.json "configs" (index = position in that list)
CONFIGS = {
    "tiny": Config("tiny", 300, 12, 4, 32, 10, 0),
    "small": Config("small", 3000, 30, 64, 128, 50, 1),
    "medium": Config("medium", 10000, 45, 500, 256, 100, 2),
    "large": Config("large", 30000, 60, 2000, 512, 100, 3),
    "sweep": Config("sweep", 10000, 0, 500, 64, 50, 4, n_ligands=256, lig_min=15, lig_max=80),
}


def _ball_points(n: int, rng: np.random.Generator) -> np.ndarray:
    """n jittered-lattice points nearest the origin (float64)."""
    a = DENSITY ** (-1.0 / 3.0)
    radius = (3.0 * n / (4.0 * np.pi * DENSITY)) ** (1.0 / 3.0)
    m = int(np.ceil(radius / a)) + 2
    g = np.arange(-m, m + 1, dtype=np.float64) * a
    pts = np.stack(np.meshgrid(g, g, g, indexing="ij"), -1).reshape(-1, 3)
    pts = pts + rng.uniform(-0.3 * a, 0.3 * a, size=pts.shape)
    d = np.linalg.norm(pts, axis=1)
    order = np.argsort(d, kind="stable")[:n]
    return pts[order]


def _types_and_charges(n: int, rng: np.random.Generator) -> tuple[np.ndarray, np.ndarray]:
    ids = np.array([t for t, _ in _COMPOSITION], dtype=np.int32)
    p = np.array([w for _, w in _COMPOSITION], dtype=np.float64)
    p = p / p.sum()
    types = rng.choice(ids, size=n, p=p).astype(np.int32)
    q = np.empty(n, dtype=np.float64)
    for t, (mu, sd) in _CHARGE.items():
        sel = types == t
        q[sel] = rng.normal(mu, sd, size=int(sel.sum()))
    q -= q.mean()
    return types, q


@dataclass
class Molecule:
    xyz: np.ndarray      # [n,3] float32, A
    q: np.ndarray        # [n] float32, e
    type: np.ndarray     # [n] int32


def make_molecule(n: int, rng: np.random.Generator, centre=(0.0, 0.0, 0.0)) -> Molecule:
    pts = _ball_points(n, rng)
    pts = pts - pts.mean(axis=0) + np.asarray(centre, dtype=np.float64)
    types, q = _types_and_charges(n, rng)
    return Molecule(pts.astype(np.float32), q.astype(np.float32), types)


def surface_spots(rec: Molecule, n_spots: int, shell: float = 3.0) -> np.ndarray:
    """Spot centres = receptor atoms of the outer `shell` A, stride-selected."""
    xyz = rec.xyz.astype(np.float64)
    c = xyz.mean(axis=0)
    d = np.linalg.norm(xyz - c, axis=1)
    cand = np.nonzero(d >= d.max() - shell)[0]
    # deterministic angular order so a stride spreads spots over the surface
    v = xyz[cand] - c
    key = np.arctan2(v[:, 1], v[:, 0]) + 10.0 * np.round(np.arccos(np.clip(v[:, 2] / np.maximum(d[cand], 1e-9), -1, 1)), 1)
    cand = cand[np.argsort(key, kind="stable")]
    if n_spots <= len(cand):
        pick = cand[(np.arange(n_spots) * len(cand)) // n_spots]
    else:  # more spots than surface atoms: wrap around (still distinct ids)
        pick = cand[np.arange(n_spots) % len(cand)]
    return rec.xyz[pick].astype(np.float32)


@dataclass
class Problem:
    cfg: Config
    rec: Molecule
    lig: Molecule
    spots: np.ndarray                       # [n_spots,3] float32
    ligands: list = field(default_factory=list)   # sweep only: list[Molecule]


def make_problem(name: str, n_spots: int | None = None) -> Problem:
    cfg = CONFIGS[name]
    rng = np.random.default_rng(cfg.data_seed)
    rec = make_molecule(cfg.n_rec, rng)
    spots = surface_spots(rec, n_spots if n_spots is not None else cfg.n_spots)
    if cfg.n_ligands > 1:
        sizes = rng.integers(cfg.lig_min, cfg.lig_max + 1, size=cfg.n_ligands)
        ligs = [make_molecule(int(s), rng) for s in sizes]
        return Problem(cfg, rec, ligs[0], spots, ligs)
    lig = make_molecule(cfg.n_lig, rng)
    return Problem(cfg, rec, lig, spots)


def make_custom(n_rec: int, n_lig: int, n_spots: int, seed: int) -> Problem:
    cfg = Config(f"custom{n_rec}x{n_lig}", n_rec, n_lig, n_spots, 32, 2, -1)
    rng = np.random.default_rng(seed)
    rec = make_molecule(n_rec, rng)
    lig = make_molecule(n_lig, rng)
    return Problem(cfg, rec, lig, surface_spots(rec, n_spots))


def make_poses(n: int, n_spots: int, half_width: float, seed: int, spread: float = 1.0):
    """Random poses: spot ids, unit quaternions (w,x,y,z) and translations.

    `spread` scales the translation range relative to the spot box
    (spread <= 1 keeps every pose inside the region).
    """
    rng = np.random.default_rng(seed)
    spot = rng.integers(0, n_spots, size=n).astype(np.int32)
    q = rng.normal(size=(n, 4))
    q /= np.linalg.norm(q, axis=1, keepdims=True)
    t = rng.uniform(-half_width * spread, half_width * spread, size=(n, 3))
    return spot, q.astype(np.float32), t.astype(np.float32)
