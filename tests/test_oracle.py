"""Pins of the fp64 oracle against things other than itself (CPU only).

Each test names what it pins.  "P:N" = PAPER.md line; "Rn" = DESIGN.md §3
reading.  The paper prints no worked example and no scoring formula, so the
pins are closed forms of the chosen pair terms, invariances of the
definition, an independent textbook-form brute force (sigma/epsilon LJ with
scipy's rotation), Random123 known-answer vectors and metaheuristic
invariants.
"""
import json
import math
import os

import numpy as np
import pytest
from scipy.spatial.transform import Rotation

from paper_conf_ppopp_imbernoncg16_b200 import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")
TYPE_ID = {n: i for i, n in enumerate(synth.TYPE_NAMES)}
SIGMA = {"C": 3.400, "N": 3.250, "O": 2.960, "S": 3.564, "H": 2.650, "HD": 1.069, "X": 0.0}
EPS = {"C": 0.1094, "N": 0.170, "O": 0.210, "S": 0.250, "H": 0.0157, "HD": 0.0157, "X": 0.0}
ROLE = {"C": 0, "N": 2, "O": 2, "S": 0, "H": 0, "HD": 1, "X": 0}
F32 = lambda x: float(np.float32(x))  # the ABI carries fp32 parameters
ID_Q = np.array([1, 0, 0, 0], np.float32)
ZERO_T = np.zeros(3, np.float32)


def mk(oracle_mod, lig, rec, spots=((0.0, 0.0, 0.0),), **sp):
    """lig/rec: lists of (type name, charge, xyz)."""
    sp.setdefault("cutoff", 0.0)
    return oracle_mod.Oracle(
        np.array([a[2] for a in rec], np.float32), np.array([a[1] for a in rec], np.float32),
        np.array([TYPE_ID[a[0]] for a in rec], np.int32),
        np.array([a[2] for a in lig], np.float32), np.array([a[1] for a in lig], np.float32),
        np.array([TYPE_ID[a[0]] for a in lig], np.int32),
        np.array(spots, np.float32), oracle_mod.score_params(**sp))


def textbook_pair(ti, qi, tj, qj, r, rc=math.inf, k=F32(332.0636), hb_eps=5.0, r0=F32(1.9)):
    """Independent formulation: 4 eps_ij [(s_ij/r)^12 - (s_ij/r)^6] with geometric
    combining, DDD Coulomb k qi qj / (4 r^2) (R3), 12-10 HB (R5), shifted cutoff (R6)."""
    r = max(r, 0.1)  # r^2 >= 0.01 (R7)
    if r >= rc:
        return 0.0
    e_ij = math.sqrt(F32(EPS[ti]) * F32(EPS[tj]))
    s_ij = math.sqrt(F32(SIGMA[ti]) * F32(SIGMA[tj]))
    lj = 4.0 * e_ij * ((s_ij / r) ** 12 - (s_ij / r) ** 6) if s_ij > 0 else 0.0
    es = k * F32(qi) * F32(qj) / (4.0 * r * r)
    if rc < math.inf:
        es *= (1.0 - (r / rc) ** 2) ** 2
    hb = 0.0
    if {ROLE[ti], ROLE[tj]} == {1, 2}:
        # well of depth hb_eps at r0: eps [5 (r0/r)^12 - 6 (r0/r)^10]
        hb = hb_eps * (5.0 * (r0 / r) ** 12 - 6.0 * (r0 / r) ** 10)
    return lj + es + hb


def textbook_score(prob_lig, prob_rec, spot, q, t, rc=math.inf):
    lig_xyz = prob_lig.xyz.astype(np.float64)
    cen = np.float32(lig_xyz.mean(axis=0))
    local = (prob_lig.xyz - cen).astype(np.float64)          # fp32 subtraction then widen (R11)
    R = Rotation.from_quat([q[1], q[2], q[3], q[0]]).as_matrix()  # scalar-last convention
    x = spot.astype(np.float64) + t.astype(np.float64) + local @ R.T
    tot = 0.0
    for i in range(len(x)):
        d = np.linalg.norm(prob_rec.xyz.astype(np.float64) - x[i], axis=1)
        for j in range(len(d)):
            tot += textbook_pair(synth.TYPE_NAMES[prob_lig.type[i]], prob_lig.q[i],
                                 synth.TYPE_NAMES[prob_rec.type[j]], prob_rec.q[j], d[j], rc)
    return tot


# ---------------------------------------------------------------- pair terms
@pytest.mark.parametrize("a,b", [("C", "C"), ("C", "O"), ("N", "O"), ("S", "H"), ("HD", "C"), ("HD", "HD"), ("O", "O")])
def test_lj_minimum_is_minus_eps(oracle_mod, a, b):
    """12-6 LJ: minimum -sqrt(eps_a eps_b) at r = 2^(1/6) sqrt(s_a s_b) (R4 closed form)."""
    rmin = 2 ** (1 / 6) * math.sqrt(F32(SIGMA[a]) * F32(SIGMA[b]))
    want = -math.sqrt(F32(EPS[a]) * F32(EPS[b]))
    vals = []
    for r in (rmin * 0.999, rmin, rmin * 1.001):
        # ligand atom at the spot centre, receptor atom at distance r on x
        o = mk(oracle_mod, [(a, 0.0, (0, 0, 0))], [(b, 0.0, (r, 0, 0))])
        vals.append(o.score_one(0, ID_Q, ZERO_T))
    # receptor x is rounded to fp32: compare at the rounded distance
    r32 = F32(rmin)
    e_at = 4 * -want * ((math.sqrt(F32(SIGMA[a]) * F32(SIGMA[b])) / r32) ** 12 -
                        (math.sqrt(F32(SIGMA[a]) * F32(SIGMA[b])) / r32) ** 6)
    assert vals[1] == pytest.approx(want, rel=1e-6)
    assert vals[1] == pytest.approx(e_at, rel=1e-12)
    assert vals[0] > vals[1] and vals[2] > vals[1]


def test_hb_minimum_is_minus_hb_eps(oracle_mod):
    """12-10 HB: C/r^12 - D/r^10 with C = 5 eps r0^12, D = 6 eps r0^10 has minimum -eps at r0 (R5)."""
    r0 = F32(1.9)
    for lig, rec in [("HD", "O"), ("O", "HD"), ("HD", "N"), ("N", "HD")]:
        o = mk(oracle_mod, [(lig, 0.0, (0, 0, 0))], [(rec, 0.0, (r0, 0, 0))])
        ref_lj = mk(oracle_mod, [(lig, 0.0, (0, 0, 0))], [(rec, 0.0, (r0, 0, 0))], hb_eps=0.0)
        e_hb = o.score_one(0, ID_Q, ZERO_T) - ref_lj.score_one(0, ID_Q, ZERO_T)
        assert e_hb == pytest.approx(-5.0, rel=1e-12)
    # no HB between donor-donor, acceptor-acceptor, or non-polar atoms
    for lig, rec in [("HD", "HD"), ("O", "N"), ("C", "O"), ("H", "O")]:
        a = mk(oracle_mod, [(lig, 0.0, (0, 0, 0))], [(rec, 0.0, (2.5, 0, 0))]).score_one(0, ID_Q, ZERO_T)
        b = mk(oracle_mod, [(lig, 0.0, (0, 0, 0))], [(rec, 0.0, (2.5, 0, 0))], hb_eps=0.0).score_one(0, ID_Q, ZERO_T)
        assert a == b


def test_ddd_coulomb_closed_form(oracle_mod):
    """eps(r) = 4r: E r^2 = k qi qj / 4 for every r (R3); dummy type X has no LJ/HB."""
    k = F32(332.0636)
    for r in (0.5, 1.0, 3.0, 7.25, 40.0):
        o = mk(oracle_mod, [("X", 0.5, (0, 0, 0))], [("X", -0.25, (r, 0, 0))])
        assert o.score_one(0, ID_Q, ZERO_T) * r * r == pytest.approx(k * 0.5 * -0.25 / 4, rel=1e-12)


def test_constant_dielectric_closed_form(oracle_mod):
    k = F32(332.0636)
    o = mk(oracle_mod, [("X", 0.5, (0, 0, 0))], [("X", -0.25, (2.0, 0, 0))], dielectric=1, eps_r=4.0)
    assert o.score_one(0, ID_Q, ZERO_T) == pytest.approx(k * 0.5 * -0.25 / (4.0 * 2.0), rel=1e-12)


def test_cutoff_shift_and_truncation(oracle_mod):
    """Shift S = (1 - r^2/rc^2)^2: S(rc/sqrt2) = 1/4; zero at and beyond rc; LJ/HB hard-truncated (R6)."""
    rc = 12.0
    r = F32(rc / math.sqrt(2))
    cut = mk(oracle_mod, [("X", 0.5, (0, 0, 0))], [("X", -0.5, (r, 0, 0))], cutoff=rc)
    allp = mk(oracle_mod, [("X", 0.5, (0, 0, 0))], [("X", -0.5, (r, 0, 0))], cutoff=0.0)
    s = (1 - r * r / 144.0) ** 2
    assert s == pytest.approx(0.25, rel=1e-6)
    assert cut.score_one(0, ID_Q, ZERO_T) / allp.score_one(0, ID_Q, ZERO_T) == pytest.approx(s, rel=1e-12)
    for rr in (12.0, 12.5, 30.0):
        o = mk(oracle_mod, [("S", 0.5, (0, 0, 0))], [("S", -0.5, (rr, 0, 0))], cutoff=rc)
        assert o.score_one(0, ID_Q, ZERO_T) == 0.0
    # LJ just inside the cutoff is unshifted
    o1 = mk(oracle_mod, [("S", 0.0, (0, 0, 0))], [("S", 0.0, (11.5, 0, 0))], cutoff=rc)
    o2 = mk(oracle_mod, [("S", 0.0, (0, 0, 0))], [("S", 0.0, (11.5, 0, 0))], cutoff=0.0)
    assert o1.score_one(0, ID_Q, ZERO_T) == o2.score_one(0, ID_Q, ZERO_T) != 0.0


def test_r2_clamp(oracle_mod):
    """r^2 <- max(r^2, 0.01): coincident atoms give the r = 0.1 value, finite (R7)."""
    a = mk(oracle_mod, [("C", 0.3, (0, 0, 0))], [("O", -0.3, (0, 0, 0))]).score_one(0, ID_Q, ZERO_T)
    b = mk(oracle_mod, [("C", 0.3, (0, 0, 0))], [("O", -0.3, (0.1, 0, 0))]).score_one(0, ID_Q, ZERO_T)
    assert math.isfinite(a) and a == pytest.approx(b, rel=1e-6)
    c = mk(oracle_mod, [("C", 0.3, (0, 0, 0))], [("O", -0.3, (0.05, 0, 0))]).score_one(0, ID_Q, ZERO_T)
    assert c == a


def test_golden_worked_examples(oracle_mod):
    """E1-E4 hand-computed examples (tests/golden/pair_examples.json)."""
    gold = json.load(open(os.path.join(GOLD, "pair_examples.json")))
    for name, ex in gold.items():
        if name.startswith("_"):
            continue
        o = mk(oracle_mod, [tuple(a) for a in ex["lig"]], [tuple(a) for a in ex["rec"]])
        assert o.score_one(0, ID_Q, ZERO_T) == pytest.approx(ex["energy"], rel=1e-6), name


def test_pair_role_swap_symmetry(oracle_mod):
    """Swapping which molecule is 'ligand' and which is 'receptor' leaves e(i,j) unchanged."""
    for a, b in [("HD", "O"), ("C", "N"), ("S", "HD")]:
        e1 = mk(oracle_mod, [(a, 0.2, (0, 0, 0))], [(b, -0.4, (2.7, 0, 0))]).score_one(0, ID_Q, ZERO_T)
        e2 = mk(oracle_mod, [(b, -0.4, (0, 0, 0))], [(a, 0.2, (2.7, 0, 0))]).score_one(0, ID_Q, ZERO_T)
        assert e1 == e2


# ---------------------------------------------------------------- transform
def test_quaternion_90_about_z(oracle_mod):
    """q = (cos45, 0, 0, sin45) maps local (1,0,0) to (0,1,0) (R11)."""
    lig = [("X", 0.0, (-1, 0, 0)), ("X", 0.5, (1, 0, 0))]
    rec = [("X", 0.5, (0, 3, 0))]
    o = mk(oracle_mod, lig, rec)
    q = np.array([math.cos(math.pi / 4), 0, 0, math.sin(math.pi / 4)], np.float32)
    e = o.score_one(0, q, ZERO_T)
    # charged ligand atom now at (0,1,0): distance 2 to the receptor atom
    assert e == pytest.approx(F32(332.0636) * 0.25 / (4 * 4.0), rel=1e-6)
    # identity pose: x = c + t + l
    t = np.array([0.0, 2.0, 0.0], np.float32)
    e_id = o.score_one(0, ID_Q, t)    # charged atom at (1,2,0): r^2 = 1 + 1
    assert e_id == pytest.approx(F32(332.0636) * 0.25 / (4 * 2.0), rel=1e-12)


def test_quaternion_sign_and_scale(oracle_mod):
    """R(q) = R(-q) = R(lambda q): homogeneous form (R11)."""
    prob = synth.make_custom(60, 7, 2, seed=5)
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params(cutoff=0.0))
    q = np.array([0.3, -0.5, 0.7, 0.2], np.float32)
    t = np.array([0.5, -1.0, 2.0], np.float32)
    e = o.score_one(1, q, t)
    assert o.score_one(1, -q, t) == pytest.approx(e, rel=1e-12)
    assert o.score_one(1, np.float32(4.0) * q, t) == pytest.approx(e, rel=1e-12)
    assert o.score_one(1, np.float32(0.5) * q, t) == pytest.approx(e, rel=1e-12)


def test_joint_rigid_motion_invariance(oracle_mod):
    """Rotate+translate receptor, spot and pose jointly -> same score (fp64).

    Exact variant: 180-degree rotations and dyadic translations keep every fp32
    input exact, so the fp64 score must agree to ~1e-12.  General variant:
    arbitrary rotation (inputs re-rounded to fp32) within 1e-5."""
    prob = synth.make_custom(80, 9, 3, seed=11)
    # quantise coordinates to a 1/1024 grid so dyadic translations are exact
    for m in (prob.rec, prob.lig):
        m.xyz[:] = np.round(m.xyz * 1024) / 1024
    prob.spots[:] = np.round(prob.spots * 1024) / 1024
    sp = oracle_mod.score_params(cutoff=0.0)
    base = oracle_mod.Oracle.from_problem(prob, sp)
    rng = np.random.default_rng(3)
    q = rng.normal(size=4).astype(np.float32)
    t = rng.uniform(-2, 2, 3).astype(np.float32)
    e0 = base.score_one(2, q, t)

    def moved(Rm, Qq, d):
        rec = synth.Molecule((prob.rec.xyz.astype(np.float64) @ Rm.T + d).astype(np.float32), prob.rec.q, prob.rec.type)
        spots = (prob.spots.astype(np.float64) @ Rm.T + d).astype(np.float32)
        o = oracle_mod.Oracle(rec.xyz, rec.q, rec.type, prob.lig.xyz, prob.lig.q, prob.lig.type, spots, sp)
        w1, x1, y1, z1 = Qq
        w2, x2, y2, z2 = q.astype(np.float64)
        q2 = np.array([w1 * w2 - x1 * x2 - y1 * y2 - z1 * z2, w1 * x2 + x1 * w2 + y1 * z2 - z1 * y2,
                       w1 * y2 - x1 * z2 + y1 * w2 + z1 * x2, w1 * z2 + x1 * y2 - y1 * x2 + z1 * w2], np.float32)
        t2 = (Rm @ t.astype(np.float64)).astype(np.float32)
        return o.score_one(2, q2, t2)

    # exact: 180 deg about x, then about y; dyadic shift
    for Qq in ([0, 1, 0, 0], [0, 0, 1, 0], [0, 0, 0, 1]):
        Rm = Rotation.from_quat([Qq[1], Qq[2], Qq[3], Qq[0]]).as_matrix().round()
        assert moved(Rm, np.array(Qq, float), np.array([16.0, -8.0, 4.0])) == pytest.approx(e0, rel=1e-11)
    # general rotation
    Qq = rng.normal(size=4)
    Qq /= np.linalg.norm(Qq)
    Rm = Rotation.from_quat([Qq[1], Qq[2], Qq[3], Qq[0]]).as_matrix()
    assert moved(Rm, Qq, np.array([3.3, -1.7, 0.4])) == pytest.approx(e0, rel=1e-5)


def test_receptor_permutation_invariance(oracle_mod):
    prob = synth.make_custom(150, 10, 2, seed=2)
    sp = oracle_mod.score_params(cutoff=0.0)
    o1 = oracle_mod.Oracle.from_problem(prob, sp)
    perm = np.random.default_rng(0).permutation(150)
    o2 = oracle_mod.Oracle(prob.rec.xyz[perm], prob.rec.q[perm], prob.rec.type[perm], prob.lig.xyz, prob.lig.q,
                           prob.lig.type, prob.spots, sp)
    spot, q, t = synth.make_poses(20, 2, 3.0, seed=1)
    a, b = o1.score(spot, q, t), o2.score(spot, q, t)
    np.testing.assert_allclose(a, b, rtol=1e-11, atol=1e-12)


@pytest.mark.parametrize("rc", [math.inf, 12.0, 6.0])
def test_brute_force_matches_textbook_form(oracle_mod, rc):
    """Independent brute force (textbook sigma/eps LJ, scipy rotation) on tiny inputs."""
    prob = synth.make_custom(120, 8, 3, seed=7)
    sp = oracle_mod.score_params(cutoff=0.0 if rc == math.inf else rc)
    o = oracle_mod.Oracle.from_problem(prob, sp)
    spot, q, t = synth.make_poses(6, 3, 3.0, seed=9)
    got = o.score(spot, q, t)
    for p in range(6):
        want = textbook_score(prob.lig, prob.rec, prob.spots[spot[p]], q[p], t[p], rc)
        assert got[p] == pytest.approx(want, rel=1e-9, abs=1e-9)


def test_ligand_centred_on_fp32_centroid(oracle_mod):
    prob = synth.make_custom(30, 11, 1, seed=4)
    o = oracle_mod.Oracle.from_problem(prob)
    cen = np.float32(prob.lig.xyz.astype(np.float64).mean(axis=0))
    np.testing.assert_array_equal(o.ligand_local(), prob.lig.xyz - cen)


# ---------------------------------------------------------------- RNG
@pytest.mark.parametrize("ctr,key,want", [
    ([0, 0, 0, 0], [0, 0], [0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8]),
    ([0xffffffff] * 4, [0xffffffff] * 2, [0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd]),
    ([0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344], [0xa4093822, 0x299f31d0],
     [0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1]),
])
def test_philox_known_answers(oracle_mod, ctr, key, want):
    """Random123 Philox4x32-10 known-answer vectors (R23)."""
    assert list(oracle_mod.philox(ctr, key)) == want


def test_u01_v11_exact(oracle_mod):
    assert oracle_mod.u01(0) == 0.0
    assert oracle_mod.u01(0xFFFFFFFF) == 1.0 - 2.0 ** -24
    assert oracle_mod.u01(0x80000000) == 0.5
    assert oracle_mod.v11(0) == -1.0
    assert oracle_mod.v11(0x80000000) == 0.0
    assert oracle_mod.v11(0xFFFFFFFF) == 1.0 - 2.0 ** -23
    for w in (1 << 8, 12345678, 0xDEADBEEF):
        assert oracle_mod.u01(w) == (w >> 8) / 2.0 ** 24


def test_init_pose_unit_and_in_region(oracle_mod):
    prob = synth.make_custom(30, 5, 3, seed=1)
    o = oracle_mod.Oracle.from_problem(prob)
    qs = []
    for s in range(3):
        for i in range(200):
            p = o.init_pose(42, s, i)
            n = float(np.linalg.norm(p[:4].astype(np.float64)))
            assert abs(n - 1.0) <= 4 * 2.0 ** -23
            assert np.all(np.abs(p[4:]) <= 3.0)
            qs.append(p[:4])
    qs = np.array(qs, np.float64)
    # uniform on S^3: E[q_k^2] = 1/4, E[q_k] = 0
    assert np.allclose((qs ** 2).mean(0), 0.25, atol=0.03)
    assert np.allclose(qs.mean(0), 0.0, atol=0.06)
    assert not np.array_equal(o.init_pose(42, 0, 0), o.init_pose(43, 0, 0))


# ---------------------------------------------------------------- metaheuristic
def test_improve_count(oracle_mod):
    """m = clamp(round-half-up(f P), 1, P) with fp32 f (R17)."""
    assert oracle_mod.improve_count(oracle_mod.mh_preset(3, population=5)) == 1
    assert oracle_mod.improve_count(oracle_mod.mh_preset(3, population=64)) == 13
    assert oracle_mod.improve_count(oracle_mod.mh_preset(3, population=256)) == 51
    assert oracle_mod.improve_count(oracle_mod.mh_preset(2, population=64)) == 64
    assert oracle_mod.improve_count(oracle_mod.mh_preset(3, population=3, improve_frac=0.5)) == 2
    assert oracle_mod.improve_count(oracle_mod.mh_preset(3, population=3, improve_frac=0.01)) == 1


def test_select_and_include_tie_rules(oracle_mod):
    """(score, index) order; Include keeps S before Scom on ties (R19, R25)."""
    J = oracle_mod.select_improve([3.0, 1.0, 1.0, 0.5, 2.0], 3)
    assert list(J) == [3, 1, 2]
    o = oracle_mod.include([1.0, 2.0, 2.0], [2.0, 0.5, 1.0])
    assert list(o) == [4, 0, 5]
    o = oracle_mod.include([1.0, 2.0, 3.0], [2.0, 2.0, 9.0])
    assert list(o) == [0, 1, 3]


def _tiny(oracle_mod, rc=12.0):
    prob = synth.make_problem("tiny")
    return prob, oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params(cutoff=rc))


def test_run_g0_f0_is_min_over_initial_population(oracle_mod):
    """G = 0, f = 0: vs_run reduces exactly to brute force over the initial poses."""
    prob, o = _tiny(oracle_mod)
    mp = oracle_mod.mh_preset(1, population=32, generations=0)
    pose, best = o.run(mp, 42)
    for s in range(prob.cfg.n_spots):
        init = np.array([o.init_pose(42, s, i) for i in range(32)])
        sc = o.score(np.full(32, s, np.int32), init[:, :4], init[:, 4:])
        k = int(np.argmin(sc))
        assert best[s] == sc[k]
        np.testing.assert_array_equal(pose[s], init[k])


def test_run_elitism_monotone_in_generations(oracle_mod):
    """Best score never increases with more generations (counter-based RNG: run G is a prefix of G+1)."""
    prob, o = _tiny(oracle_mod)
    prev = None
    for G in range(0, 6):
        _, best = o.run(oracle_mod.mh_preset(3, population=16, generations=G), 7)
        if prev is not None:
            assert np.all(best <= prev)
        prev = best


def test_local_search_never_worsens(oracle_mod):
    prob, o = _tiny(oracle_mod)
    _, b0 = o.run(oracle_mod.mh_preset(1, population=32, generations=0), 5)
    _, b1 = o.run(oracle_mod.mh_preset(4, population=32), 5)   # G = 0, f = 1, L = 8
    assert np.all(b1 <= b0)
    assert np.any(b1 < b0)


def test_combine_identical_parents(oracle_mod):
    """Blend of two identical parents (no mutation) returns the parent up to normalisation rounding."""
    prob, o = _tiny(oracle_mod)
    mp = oracle_mod.mh_preset(1, population=8, p_mut=0.0)
    p = o.init_pose(1, 0, 0)
    S = np.tile(p, (8, 1))
    for j in range(8):
        c = o.combine_child(mp, 3, 0, 1, j, S)
        np.testing.assert_array_equal(c[4:], p[4:])
        np.testing.assert_allclose(c[:4], p[:4], atol=3e-7)


def test_ls_proposal_stays_in_region(oracle_mod):
    prob, o = _tiny(oracle_mod)
    mp = oracle_mod.mh_preset(2, ls_trans=5.0)
    p = np.array([1, 0, 0, 0, 2.9, -2.9, 0.0], np.float32)
    for j in range(50):
        c = o.ls_proposal(mp, 1, 0, 1, 0, j, p)
        assert np.all(np.abs(c[4:]) <= 3.0)
        assert abs(np.linalg.norm(c[:4].astype(np.float64)) - 1) < 1e-6


def test_optimizer_finds_lj_minimum(oracle_mod):
    """1-atom C ligand vs 1-atom C receptor (q = 0): global optimum -eps at r_min (loose)."""
    o = mk(oracle_mod, [("C", 0.0, (0, 0, 0))], [("C", 0.0, (0, 0, 0))], spots=[(3.5, 0.5, 0.0)], cutoff=12.0)
    mp = oracle_mod.mh_preset(2, population=24, generations=15)
    pose, best = o.run(mp, 1)
    assert -F32(0.1094) <= best[0] < -0.104
    r = np.linalg.norm(np.array([3.5, 0.5, 0.0]) + pose[0, 4:])
    assert abs(r - 2 ** (1 / 6) * 3.4) < 0.15


# ---------------------------------------------------------------- ABI errors
def test_abi_errors(oracle_mod):
    prob, o = _tiny(oracle_mod)
    with pytest.raises(oracle_mod.OracleError) as e:
        o.score([0], [[0, 0, 0, 0]], [[0, 0, 0]])
    assert e.value.status == oracle_mod.ERR_ZERO_QUATERNION
    with pytest.raises(oracle_mod.OracleError) as e:
        o.score([0], [[1, 0, 0, 0]], [[3.5, 0, 0]])
    assert e.value.status == oracle_mod.ERR_POSE_OUT_OF_REGION
    with pytest.raises(oracle_mod.OracleError) as e:
        o.score([9], [[1, 0, 0, 0]], [[0, 0, 0]])
    assert e.value.status == oracle_mod.ERR_INVALID_ARGUMENT
    with pytest.raises(oracle_mod.OracleError):
        o.run(oracle_mod.mh_preset(1, population=1, generations=3), 1)
    with pytest.raises(oracle_mod.OracleError):
        oracle_mod.Oracle(prob.rec.xyz, prob.rec.q, prob.rec.type + 9, prob.lig.xyz, prob.lig.q, prob.lig.type,
                          prob.spots)
    # all-pairs mode accepts any translation
    _, oa = _tiny(oracle_mod, rc=0.0)
    assert np.isfinite(oa.score([0], [[1, 0, 0, 0]], [[30.0, 0, 0]]))[0]


def test_parallel_neighbourhood_ls(oracle_mod):
    """N4: best-of-K proposals per Improve step; K = 1 is plain hill climbing (same streams); never worse."""
    prob, o = _tiny(oracle_mod)
    mp1 = oracle_mod.mh_preset(4, population=32)
    assert mp1.ls_neighbours == 1
    p0 = o.init_pose(5, 0, 0)
    np.testing.assert_array_equal(o.ls_proposal(mp1, 5, 0, 0, 3, 7, p0), o.ls_proposal(mp1, 5, 0, 0, 3, 7, p0, k=0))
    mp4 = oracle_mod.mh_preset(4, population=32, ls_neighbours=4)
    # proposal k of step l uses counter 2 (l K + k): step 1, k 0 of K = 4 is step 4 of K = 1
    np.testing.assert_array_equal(o.ls_proposal(mp4, 5, 0, 0, 1, 7, p0, k=0), o.ls_proposal(mp1, 5, 0, 0, 4, 7, p0))
    _, b0 = o.run(oracle_mod.mh_preset(1, population=32, generations=0), 5)
    _, b1 = o.run(mp1, 5)
    _, b4 = o.run(mp4, 5)
    assert np.all(b1 <= b0) and np.all(b4 <= b0)
    assert np.mean(b4) <= np.mean(b1) + 1e-9
    with pytest.raises(oracle_mod.OracleError):
        o.run(oracle_mod.mh_preset(4, ls_neighbours=0), 5)
