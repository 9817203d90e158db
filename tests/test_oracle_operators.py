"""Pins of the oracle's population operators (Algorithm 1, §3.1) against what
probability and rotation algebra fix -- not against re-typed formulas (CPU only).

  * Select (R13): a binary tournament on ranks of a sorted population picks rank r with
    probability (2 (P - r) - 1) / P^2 (the minimum of two independent uniform ranks); the two parents'
    tournaments are independent; p1 != p2.
  * Combine (R14): the child's translation lies on the segment [t1, t2] at the crossover
    parameter alpha (alpha measured from parent 1); its rotation lies on the short great-circle arc
    between q1 and the hemisphere-aligned q2, at the blend weights (1 - alpha, alpha).
  * Mutation gate (R15): the mutated fraction of children is Binomial(n, p_mut).
  * Initialize (R12): translations uniform on [-T, T]^3 (Kolmogorov-Smirnov), independent axes.
  * perturb (R16): the proposal's rotation is R(dq) R(q) -- dq applied in the spot frame
    after q -- checked with scipy's rotation composition; dq is a small rotation bounded by the step.

The random draws (alpha, the perturbation's words) come from the oracle's Philox and u01 / v11
exports, which tests/test_oracle.py pins to the Random123 known-answer vectors and exact values.
"""
import math

import numpy as np
import pytest
from scipy import stats
from scipy.spatial.transform import Rotation

from paper_conf_ppopp_imbernoncg16_b200 import synth

TAG_CROSS, TAG_MUT, TAG_LS = 4, 5, 6


def words(oracle_mod, seed, i, s, g, tag, k):
    """The Philox words of stream (i, s, g, tag, k) (R23) from the pinned Philox export."""
    return oracle_mod.philox([i, s, g, (tag << 24) | k], [seed & 0xFFFFFFFF, seed >> 32])


@pytest.fixture(scope="module")
def tiny(oracle_mod):
    prob = synth.make_problem("tiny")
    return prob, oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())


def distinct_population(P, seed=0, negate_half=False):
    """A sorted population of P distinct poses (7 floats each) in the T = 3 box."""
    rng = np.random.default_rng(seed)
    q = rng.normal(size=(P, 4))
    q /= np.linalg.norm(q, axis=1, keepdims=True)
    if negate_half:
        q[1::2] *= -1.0
    t = rng.uniform(-3.0, 3.0, size=(P, 3))
    return np.concatenate([q, t], 1).astype(np.float32)


# ------------------------------------------------------------------ Select
@pytest.mark.parametrize("P", [16, 13])
def test_select_rank_distribution(oracle_mod, P):
    mp = oracle_mod.mh_preset(3, population=P)
    n = 24000
    p1 = np.empty(n, np.int64)
    p2 = np.empty(n, np.int64)
    for k in range(n):
        j, g, s = k % P, 1 + (k // P) % 50, k // (50 * P)
        p1[k], p2[k] = oracle_mod.select_parents(mp, 12345, s, g, j)
    assert np.all((p1 >= 0) & (p1 < P) & (p2 >= 0) & (p2 < P))
    assert np.all(p1 != p2)
    r = np.arange(P)
    want = (2 * (P - r) - 1) / P ** 2                    # P(min(U1, U2) = r)
    assert abs(want.sum() - 1.0) < 1e-12
    obs = np.bincount(p1, minlength=P)
    chi = stats.chisquare(obs, n * want)
    assert chi.pvalue > 1e-3, (obs, n * want)
    # the same test rejects the plausible slips: max instead of min, a single uniform draw
    for bad in ((2 * r + 1) / P ** 2, np.full(P, 1.0 / P)):
        assert stats.chisquare(obs, n * bad).pvalue < 1e-12
    # parent 2: an independent tournament, except that a collision moves it to the next rank
    q2 = p2.copy()
    coll = ((p1 + 1) % P == p2)
    # independence of the two tournaments where no collision can have occurred (p2 != p1 + 1)
    keep = ~coll
    tab = np.zeros((P, P))
    np.add.at(tab, (p1[keep], q2[keep]), 1.0)
    expect = np.outer(want, want)
    expect[r, r] = 0.0                                   # p1 == p2 never survives
    expect[r, (r + 1) % P] = 0.0                         # excluded cells (collisions and their targets)
    expect *= keep.sum() / expect.sum()
    m = expect > 5
    chi2 = (((tab - expect) ** 2)[m] / expect[m]).sum()
    dof = m.sum() - 1
    assert stats.chi2.sf(chi2, dof) > 1e-4


def test_select_streams_differ_by_child_generation_spot(oracle_mod):
    mp = oracle_mod.mh_preset(3, population=64)
    a = [oracle_mod.select_parents(mp, 1, 0, 1, j) for j in range(64)]
    b = [oracle_mod.select_parents(mp, 1, 0, 2, j) for j in range(64)]
    c = [oracle_mod.select_parents(mp, 1, 1, 1, j) for j in range(64)]
    d = [oracle_mod.select_parents(mp, 2, 0, 1, j) for j in range(64)]
    assert len({tuple(a), tuple(b), tuple(c), tuple(d)}) == 4


# ------------------------------------------------------------------ Combine
def _alpha(oracle_mod, seed, j, s, g):
    return float(oracle_mod.u01(int(words(oracle_mod, seed, j, s, g, TAG_CROSS, 0)[0])))


@pytest.mark.parametrize("negate_half", [False, True])
def test_combine_child_on_parent_segment_and_arc(oracle_mod, tiny, negate_half):
    prob, o = tiny
    P = 16
    mp = oracle_mod.mh_preset(3, population=P, p_mut=0.0)
    S = distinct_population(P, seed=3, negate_half=negate_half)
    seed, s = 99, 1
    n_flip = 0
    for g in (1, 2, 3):
        for j in range(P):
            p1, p2 = oracle_mod.select_parents(mp, seed, s, g, j)
            c = o.combine_child(mp, seed, s, g, j, S).astype(np.float64)
            a = _alpha(oracle_mod, seed, j, s, g)
            t1, t2 = S[p1, 4:].astype(np.float64), S[p2, 4:].astype(np.float64)
            # translation: t1 + alpha (t2 - t1), measured from parent 1 (fp32 rounding of two ops)
            np.testing.assert_allclose(c[4:], t1 + a * (t2 - t1), rtol=0, atol=4e-7 * 3.0)
            # rotation: unit, in span{q1, q2'} with q2' the hemisphere-aligned parent 2, weights (1 - alpha, alpha)
            q1, q2 = S[p1, :4].astype(np.float64), S[p2, :4].astype(np.float64)
            if q1 @ q2 < 0:
                q2 = -q2
                n_flip += 1
            qc = c[:4]
            assert abs(np.linalg.norm(qc) - 1.0) < 1e-6
            B = np.stack([q1, q2], 1)
            coef, *_ = np.linalg.lstsq(B, qc, rcond=None)
            assert np.linalg.norm(B @ coef - qc) < 2e-6                   # on the great circle
            assert coef[0] >= -1e-6 and coef[1] >= -1e-6                  # on the short arc
            assert abs(coef[1] / coef.sum() - a) < 2e-5 * (1.0 + 1.0 / max(1e-3, abs(q1 @ q2))) or \
                abs(q1 @ q2) > 0.99999                                    # weights (1 - alpha, alpha)
    if negate_half:
        assert n_flip > 0                                                 # the hemisphere flip was exercised


def test_combine_alpha_zero_limit(oracle_mod, tiny):
    """Children whose alpha is tiny sit (to fp32 rounding) on parent 1, not parent 2."""
    prob, o = tiny
    P = 8
    mp = oracle_mod.mh_preset(3, population=P, p_mut=0.0)
    S = distinct_population(P, seed=5)
    seen = 0
    for g in range(1, 400):
        for j in range(P):
            a = _alpha(oracle_mod, 7, j, 0, g)
            if a < 0.02:
                p1, p2 = oracle_mod.select_parents(mp, 7, 0, g, j)
                c = o.combine_child(mp, 7, 0, g, j, S)
                d1 = np.abs(c[4:] - S[p1, 4:]).max()
                d2 = np.abs(c[4:] - S[p2, 4:]).max()
                assert d1 <= 0.02 * 6.0 + 1e-6 and d1 < d2
                seen += 1
    assert seen >= 10


# ------------------------------------------------------------------ mutation gate
@pytest.mark.parametrize("p_mut", [0.1, 0.3])
def test_mutation_fraction_is_binomial(oracle_mod, tiny, p_mut):
    prob, o = tiny
    P = 32
    S = distinct_population(P, seed=11)
    mp0 = oracle_mod.mh_preset(3, population=P, p_mut=0.0)
    mp1 = oracle_mod.mh_preset(3, population=P, p_mut=p_mut)
    n = mutated = 0
    for g in range(1, 121):
        for j in range(P):
            c0 = o.combine_child(mp0, 5, 2, g, j, S)
            c1 = o.combine_child(mp1, 5, 2, g, j, S)
            n += 1
            if not np.array_equal(c0, c1):
                mutated += 1
                # a mutation moves t by at most mut_trans per axis (then the clamp) and keeps q unit
                assert np.all(np.abs(c1[4:] - c0[4:]) <= mp1.mut_trans + 1e-6)
                assert abs(np.linalg.norm(c1[:4].astype(np.float64)) - 1.0) < 1e-6
    sd = math.sqrt(n * p_mut * (1 - p_mut))
    assert abs(mutated - n * p_mut) < 4.5 * sd, (mutated, n * p_mut, sd)
    # p_mut = 1: every child is mutated
    mpa = oracle_mod.mh_preset(3, population=P, p_mut=1.0)
    assert all(not np.array_equal(o.combine_child(mpa, 5, 2, 1, j, S), o.combine_child(mp0, 5, 2, 1, j, S))
               for j in range(P))


# ------------------------------------------------------------------ Initialize
def test_init_translation_uniform_in_box(oracle_mod):
    prob = synth.make_custom(30, 5, 3, seed=1)
    o = oracle_mod.Oracle.from_problem(prob)
    t = np.array([o.init_pose(2024, s, i)[4:] for s in range(3) for i in range(1500)], np.float64)
    T = 3.0
    for k in range(3):
        ks = stats.kstest(t[:, k], stats.uniform(loc=-T, scale=2 * T).cdf)
        assert ks.pvalue > 1e-3, (k, ks)
        assert t[:, k].min() >= -T and t[:, k].max() <= T
    # independent axes
    cc = np.corrcoef(t.T)
    assert np.all(np.abs(cc[np.triu_indices(3, 1)]) < 0.05)
    # the rotation and the translation are not drawn from the same words
    q = np.array([o.init_pose(2024, 0, i)[:4] for i in range(1500)], np.float64)
    assert np.all(np.abs([np.corrcoef(q[:, a], t[:1500, b])[0, 1] for a in range(4) for b in range(3)]) < 0.1)


# ------------------------------------------------------------------ perturb (LS proposal)
@pytest.mark.parametrize("K,k", [(1, 0), (3, 2)])
def test_perturb_rotation_composes_in_spot_frame(oracle_mod, tiny, K, k):
    prob, o = tiny
    mp = oracle_mod.mh_preset(2, ls_neighbours=K, ls_rot=0.3)
    seed, s, g = 31, 2, 4
    rng = np.random.default_rng(8)
    n_left = n_right_fail = 0
    for trial in range(60):
        j, l = int(rng.integers(0, 64)), int(rng.integers(0, 8))
        q = rng.normal(size=4)
        q /= np.linalg.norm(q)
        pose = np.concatenate([q, rng.uniform(-2.0, 2.0, 3)]).astype(np.float32)
        out = o.ls_proposal(mp, seed, s, g, l, j, pose, k=k)
        kk = 2 * (l * K + k)                                   # LS counter of proposal k of step l (R31)
        b = words(oracle_mod, seed, j, s, g, TAG_LS, kk + 1)
        dr = float(np.float32(mp.ls_rot))
        dq = np.array([1.0] + [dr * float(oracle_mod.v11(int(b[c]))) for c in range(3)])
        rot = lambda wxyz: Rotation.from_quat([wxyz[1], wxyz[2], wxyz[3], wxyz[0]])   # scipy: scalar last
        R_out = rot(out[:4].astype(np.float64)).as_matrix()
        left = (rot(dq) * rot(pose[:4].astype(np.float64))).as_matrix()      # R(dq) R(q)
        right = (rot(pose[:4].astype(np.float64)) * rot(dq)).as_matrix()     # R(q) R(dq)
        assert np.abs(R_out - left).max() < 5e-6
        n_left += 1
        if np.abs(R_out - right).max() > 1e-3:
            n_right_fail += 1
        # dq is a small rotation: angle <= 2 atan(dr sqrt 3)
        ang = np.linalg.norm((rot(out[:4].astype(np.float64)) * rot(pose[:4].astype(np.float64)).inv()).as_rotvec())
        assert ang <= 2 * math.atan(dr * math.sqrt(3)) + 1e-5
        # translation: moved by at most ls_trans per axis, clamped to the box
        assert np.all(np.abs(out[4:] - pose[4:]) <= mp.ls_trans + 1e-6) and np.all(np.abs(out[4:]) <= 3.0)
    assert n_left == 60 and n_right_fail > 50          # the test tells the two composition orders apart


def test_perturb_translation_uses_first_word_block(oracle_mod, tiny):
    """The translation step of proposal (l, k) moves each axis by ls_trans * v11 of the words of counter 2(lK + k)
    -- uniform on [-ls_trans, ls_trans) -- so over many children the per-axis step is uniform (KS)."""
    prob, o = tiny
    mp = oracle_mod.mh_preset(2, ls_trans=0.5)
    pose = np.array([1, 0, 0, 0, 0, 0, 0], np.float32)
    d = np.array([o.ls_proposal(mp, 3, 0, 1, 0, j, pose)[4:] for j in range(3000)], np.float64)
    for c in range(3):
        assert stats.kstest(d[:, c], stats.uniform(loc=-0.5, scale=1.0).cdf).pvalue > 1e-3
