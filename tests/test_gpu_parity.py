"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Bars (BASELINE.json north_star):
  * scores: |gpu - oracle| <= max(1e-4 |oracle|, 1e-3 kcal/mol) per pose;
  * pose generation from a Philox stream: bit-exact;
  * vs_run best score within 1e-3 relative of the oracle on identical streams.
Decisions taken on scores (Improve's accept, sorts) are checked exactly against
the GPU's own fp32 scores, and against the oracle's fp64 scores except at near
ties (|gap| below the per-pose tolerance), where both outcomes are correct.
"""
import math

import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import synth, vs

pytestmark = pytest.mark.gpu


def tol(ref):
    return np.maximum(1e-4 * np.abs(ref), 1e-3)


def assert_scores(gpu, ref, what=""):
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    err = np.abs(gpu - ref)
    bad = err > tol(ref)
    assert not bad.any(), f"{what}: {bad.sum()} / {len(ref)} poses out of tolerance; worst err/tol " \
                          f"{(err / tol(ref)).max():.3g} at {int(np.argmax(err / tol(ref)))}"
    return float((err / tol(ref)).max())


@pytest.fixture(scope="module")
def gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    vs.load()
    return torch


def both(oracle_mod, prob, cutoff=12.0, ligand=None, **kw):
    sp_o = oracle_mod.score_params(cutoff=cutoff, **kw)
    sp_g = vs.score_params(cutoff=cutoff, **kw)
    return (vs.Context.from_problem(prob, sp_g, ligand=ligand),
            oracle_mod.Oracle.from_problem(prob, sp_o, ligand=ligand))


# ------------------------------------------------------------------ RNG
def test_device_philox_known_answers(gpu, oracle_mod):
    kat = [([0, 0, 0, 0], [0, 0], [0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8]),
           ([0xffffffff] * 4, [0xffffffff] * 2, [0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd]),
           ([0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344], [0xa4093822, 0x299f31d0],
            [0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1])]
    for ctr, key, want in kat:
        assert list(vs.debug_philox([ctr], key)[0]) == want
    rng = np.random.default_rng(0)
    ctr = rng.integers(0, 2 ** 32, size=(4096, 4), dtype=np.uint64).astype(np.uint32)
    key = [0x12345678, 0x9abcdef0]
    got = vs.debug_philox(ctr, key)
    for i in range(0, 4096, 97):
        assert list(got[i]) == list(oracle_mod.philox(ctr[i], key))


# ------------------------------------------------------------------ scoring parity
@pytest.mark.parametrize("cutoff", [12.0, 0.0])
@pytest.mark.parametrize("name", ["tiny", "small"])
def test_score_parity_all_poses(gpu, oracle_mod, name, cutoff):
    prob = synth.make_problem(name)
    g, o = both(oracle_mod, prob, cutoff)
    n = 300 if name == "tiny" else 96
    spot, q, t = synth.make_poses(n, prob.cfg.n_spots, 3.0, seed=17)
    # mix in near-contact poses: scaled-down translations towards the spot atom
    t[: n // 3] *= 0.2
    assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t), f"{name} rc={cutoff}")


@pytest.mark.parametrize("name", ["medium", "large"])
def test_score_parity_sampled_full_size(gpu, oracle_mod, name):
    """Full-size problem, large batch through the GPU; the oracle checks a sample."""
    prob = synth.make_problem(name)
    g, o = both(oracle_mod, prob, 12.0)
    n = 20000
    spot, q, t = synth.make_poses(n, prob.cfg.n_spots, 3.0, seed=5)
    got = g.score_poses(spot, q, t)
    idx = np.random.default_rng(1).choice(n, 12, replace=False)
    assert_scores(got[idx], o.score(spot[idx], q[idx], t[idx]), name)
    assert np.all(np.isfinite(got))


@pytest.mark.parametrize("name,dielectric", [("medium", 0), ("large", 0), ("medium", 1), ("large", 1)])
def test_all_pairs_full_size_sampled(gpu, oracle_mod, name, dielectric):
    """Paper mode (no cutoff, every receptor atom) at full size: the fp32 sums over 10k / 30k atoms stay within
    the 1e-4 tolerance, for the distance-dependent and the constant dielectric (N3)."""
    prob = synth.make_problem(name)
    kw = dict(dielectric=1, eps_r=4.0) if dielectric else {}
    g, o = both(oracle_mod, prob, 0.0, **kw)
    n = 4096
    spot, q, t = synth.make_poses(n, prob.cfg.n_spots, 3.0, seed=31)
    got = g.score_poses(spot, q, t)
    idx = np.random.default_rng(2).choice(n, 8, replace=False)
    worst = assert_scores(got[idx], o.score(spot[idx], q[idx], t[idx]), f"{name} all-pairs diel={dielectric}")
    print(f"worst err/tol {worst:.3f}")


@pytest.mark.parametrize("n_lig", [1, 7, 9, 64, 65, 100, 256])
def test_ragged_ligand_sizes(gpu, oracle_mod, n_lig):
    """Ligands that are not a multiple of the 8-atom register block, and > 64 atoms (chunked CTAs)."""
    prob = synth.make_custom(1500, n_lig, 5, seed=n_lig)
    for cutoff in (12.0, 0.0):
        g, o = both(oracle_mod, prob, cutoff)
        spot, q, t = synth.make_poses(70, 5, 3.0, seed=3)
        assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t), f"n_lig={n_lig} rc={cutoff}")


@pytest.mark.parametrize("mix", ["no_hbond", "all_hbond", "hbond_heavy"])
def test_ligand_class_mixes(gpu, oracle_mod, mix):
    """Ligands whose H-bond-capable share selects every slot layout: none (H = 0), only H-bond atoms
    (H = CELL_KP, no class-0 slots) and more H-bond than other atoms (class-0 items overflowing or not);
    ragged pose counts per spot give partially filled chunks; scoring and a short M3 / N4 run."""
    prob = synth.make_custom(2500, 23, 6, seed=17)
    rng = np.random.default_rng(5)
    pick = {"no_hbond": [synth.T_C, synth.T_H, synth.T_S], "all_hbond": [synth.T_N, synth.T_O, synth.T_HD],
            "hbond_heavy": [synth.T_N, synth.T_O, synth.T_HD, synth.T_HD, synth.T_C]}[mix]
    prob.lig.type[:] = rng.choice(pick, size=len(prob.lig.type)).astype(np.int32)
    for cutoff in (12.0, 0.0):
        g, o = both(oracle_mod, prob, cutoff)
        spot, q, t = synth.make_poses(301, 6, 3.0, seed=9)
        spot[:37] = 2                                       # one crowded spot, others ragged
        assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t), f"{mix} rc={cutoff}")
    g, o = both(oracle_mod, prob, 12.0)
    for K in (1, 3):
        _, sg = g.run(vs.mh_preset(3, population=24, generations=2, ls_neighbours=K), 8)
        _, so = o.run(oracle_mod.mh_preset(3, population=24, generations=2, ls_neighbours=K), 8)
        assert np.all(np.abs(sg - so) <= 1e-3 * np.maximum(np.abs(so), 1.0)), (mix, K, sg, so)


def test_long_lists_streamed_whole(gpu, oracle_mod):
    """Cutoff lists longer than the cell sort's limit (16384 atoms: here rc = 70 A on a 25k-atom receptor)
    are streamed whole instead of cell-culled; scores still match the brute-force cutoff definition."""
    prob = synth.make_custom(25000, 30, 3, seed=23)
    g, o = both(oracle_mod, prob, 70.0)
    assert g.list_lengths().max() > 16384
    spot, q, t = synth.make_poses(200, 3, 3.0, seed=4)
    got = g.score_poses(spot, q, t)
    idx = np.arange(0, 200, 25)
    assert_scores(got[idx], o.score(spot[idx], q[idx], t[idx]))


def test_list_tiles_ragged_and_empty(gpu, oracle_mod):
    """Spot far outside the receptor (empty cutoff list) and list lengths across tile boundaries."""
    prob = synth.make_custom(700, 13, 4, seed=2)
    prob.spots[3] = prob.spots[3] + np.float32(80.0)   # nothing within reach
    g, o = both(oracle_mod, prob, 12.0)
    lens = g.list_lengths()
    assert lens[3] == 0 and lens[:3].min() > 128
    spot, q, t = synth.make_poses(64, 4, 3.0, seed=8)
    got = g.score_poses(spot, q, t)
    assert np.all(got[spot == 3] == 0.0)
    assert_scores(got, o.score(spot, q, t))


def test_binned_lists_equal_all_pairs_cutoff(gpu, oracle_mod):
    """Binning is exact: per-spot lists give the brute-force cutoff score for in-region poses,
    including poses on the region boundary."""
    prob = synth.make_problem("small")
    g, o = both(oracle_mod, prob, 12.0)
    spot, q, t = synth.make_poses(64, prob.cfg.n_spots, 3.0, seed=4)
    t[:16] = np.sign(t[:16]) * np.float32(3.0)   # corners of the region box
    assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t))


def test_quaternion_conventions_on_gpu(gpu, oracle_mod):
    prob = synth.make_problem("tiny")
    g, o = both(oracle_mod, prob, 0.0)
    spot, q, t = synth.make_poses(40, 4, 3.0, seed=6)
    a = g.score_poses(spot, q, t)
    b = g.score_poses(spot, -q, t)
    c = g.score_poses(spot, 4.0 * q, t)
    assert_scores(a, o.score(spot, q, t))
    assert_scores(b, o.score(spot, q, t))
    assert_scores(c, o.score(spot, q, t))


@pytest.mark.parametrize("kw", [dict(dielectric=1, eps_r=4.0), dict(hb_eps=0.0), dict(r2_min=0.25)])
def test_score_param_variants(gpu, oracle_mod, kw):
    prob = synth.make_problem("tiny")
    for cutoff in (12.0, 0.0):
        g, o = both(oracle_mod, prob, cutoff, **kw)
        spot, q, t = synth.make_poses(128, 4, 3.0, seed=12)
        assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t), str(kw))


def test_custom_type_table(gpu, oracle_mod):
    import ctypes as C
    prob = synth.make_problem("tiny")
    sig = np.array([3.1, 2.8, 2.2, 3.0, 2.0, 1.2, 0.5], np.float32)
    eps = np.array([0.2, 0.1, 0.3, 0.05, 0.02, 0.01, 0.0], np.float32)
    role = np.array([0, 1, 2, 2, 0, 1, 0], np.int32)
    kw = dict(n_types=7, type_sigma=sig.ctypes.data_as(C.POINTER(C.c_float)),
              type_eps=eps.ctypes.data_as(C.POINTER(C.c_float)), type_hb_role=role.ctypes.data_as(C.POINTER(C.c_int)))
    g, o = both(oracle_mod, prob, 12.0, **kw)
    spot, q, t = synth.make_poses(100, 4, 3.0, seed=2)
    assert_scores(g.score_poses(spot, q, t), o.score(spot, q, t))


def test_score_errors_and_empty(gpu, oracle_mod):
    prob = synth.make_problem("tiny")
    g, _ = both(oracle_mod, prob, 12.0)
    assert len(g.score_poses(np.zeros(0, np.int32), np.zeros((0, 4)), np.zeros((0, 3)))) == 0
    cases = [([0], [[0, 0, 0, 0]], [[0, 0, 0]], vs.ERR_ZERO_QUATERNION),
             ([0], [[1, 0, 0, 0]], [[0, 3.01, 0]], vs.ERR_POSE_OUT_OF_REGION),
             ([4], [[1, 0, 0, 0]], [[0, 0, 0]], vs.ERR_INVALID_ARGUMENT),
             ([0], [[1, 0, np.nan, 0]], [[0, 0, 0]], vs.ERR_INVALID_ARGUMENT)]
    for s, q, t, code in cases:
        with pytest.raises(vs.VSError) as e:
            g.score_poses(np.array(s, np.int32), np.array(q, np.float32), np.array(t, np.float32))
        assert e.value.status == code
    # the ctx stays usable after argument errors
    assert np.isfinite(g.score_poses(np.array([1], np.int32), np.array([[1, 0, 0, 0]], np.float32),
                                     np.zeros((1, 3), np.float32)))[0]


def test_device_entry_point(gpu, oracle_mod):
    torch = gpu
    prob = synth.make_problem("small")
    g, o = both(oracle_mod, prob, 12.0)
    spot, q, t = synth.make_poses(5000, prob.cfg.n_spots, 3.0, seed=21)
    q[7] = 0.0            # invalid -> NaN
    t[8, 0] = 9.0         # out of region -> NaN
    spot[9] = 999         # bad spot -> NaN
    spot_d = torch.from_numpy(np.where(spot < prob.cfg.n_spots, spot, 0)).cuda()
    spot_d[9] = 999
    qd, td = torch.from_numpy(q).cuda(), torch.from_numpy(t).cuda()
    out = torch.zeros(5000, device="cuda")
    g.score_poses_device(spot_d, qd, td, out)
    torch.cuda.synchronize()
    res = out.cpu().numpy()
    assert np.isnan(res[[7, 8, 9]]).all()
    ok = np.setdiff1d(np.arange(5000), [7, 8, 9])
    host = g.score_poses(spot[ok], q[ok], t[ok])
    np.testing.assert_array_equal(res[ok], host)            # same kernel, same bits
    idx = ok[::250]
    assert_scores(res[idx], o.score(spot[idx], q[idx], t[idx]))


def test_stats_count_pairs(gpu, oracle_mod):
    """`pairs` = workload pairs, n_lig x list length of the pose's spot per scored pose (the whole receptor in
    all-pairs mode); `pairs_evaluated` = item slots x receptor atoms streamed per chunk: every list atom in
    all-pairs mode (plus the padding slots of a chunk), in cutoff mode only the atoms of the cell rows within rc
    of a chunk's bounding box that are also within rc of the bounding box of the item's slot pair."""
    prob = synth.make_problem("tiny")
    spot, q, t = synth.make_poses(100, 4, 3.0, seed=2)
    g, _ = both(oracle_mod, prob, 0.0)
    g.reset_stats()
    g.set_timing(True)
    g.score_poses(spot, q, t)
    st = g.stats()
    full = 100 * prob.cfg.n_rec * prob.cfg.n_lig
    assert st["poses_scored"] == 100 and st["pairs"] == full
    assert full <= st["pairs_evaluated"] <= 1.5 * full
    assert st["score_launches"] == 1 and st["timed_launches"] == 1 and st["score_ms"] > 0
    gm = vs.Context.from_problem(synth.make_problem("medium"), vs.score_params(cutoff=12.0))
    pm = synth.make_problem("medium")
    spot, q, t = synth.make_poses(4000, pm.cfg.n_spots, 3.0, seed=2)
    gm.reset_stats()
    gm.score_poses(spot, q, t)
    st = gm.stats()
    full = int(sum(int(gm.list_lengths()[s]) for s in spot)) * pm.cfg.n_lig
    assert st["poses_scored"] == 4000 and st["pairs"] == full
    assert 0.25 * full < st["pairs_evaluated"] < full     # culling skips 30-60 %
    sc = gm.score_poses(spot[:1], q[:1], t[:1])
    assert gm.stats()["pairs"] == full + int(gm.list_lengths()[spot[0]]) * pm.cfg.n_lig and np.isfinite(sc).all()


# ------------------------------------------------------------------ metaheuristic
def _run_pair(oracle_mod, name="tiny", cutoff=12.0):
    prob = synth.make_problem(name)
    return prob, both(oracle_mod, prob, cutoff)


def test_run_free_running_matches_oracle(gpu, oracle_mod):
    prob, (g, o) = _run_pair(oracle_mod)
    for m in (1, 2, 3):
        mp_g = vs.mh_preset(m, population=prob.cfg.population, generations=prob.cfg.generations)
        mp_o = oracle_mod.mh_preset(m, population=prob.cfg.population, generations=prob.cfg.generations)
        pg, sg = g.run(mp_g, 42)
        po, so = o.run(mp_o, 42)
        rel = np.abs(sg - so) / np.maximum(np.abs(so), 1e-3)
        assert np.all(rel <= 1e-3), (m, sg, so)


def test_run_m4_neighbourhood(gpu, oracle_mod):
    prob, (g, o) = _run_pair(oracle_mod)
    pg, sg = g.run(vs.mh_preset(4, population=128), 3)
    po, so = o.run(oracle_mod.mh_preset(4, population=128), 3)
    assert np.all(np.abs(sg - so) <= 1e-3 * np.maximum(np.abs(so), 1.0))


def test_run_g0_f0_reduces_to_min_of_scored_initial_poses(gpu, oracle_mod):
    """G = 0, f = 0: vs_run is the argmin over the scored initial poses, bit for bit (a pose's score does not depend
    on the launch that scores it: the list splits are canonical, vs_cells.cu header)."""
    prob, (g, o) = _run_pair(oracle_mod)
    P = 32
    pose, best = g.run(vs.mh_preset(1, population=P, generations=0), 9)
    init = np.array([[o.init_pose(9, s, i) for i in range(P)] for s in range(4)])
    for s in range(4):
        sc = g.score_poses(np.full(P, s, np.int32), init[s, :, :4], init[s, :, 4:])
        k = int(np.argmin(sc))
        assert best[s] == sc[k]
        np.testing.assert_array_equal(pose[s], init[s, k])


def test_run_deterministic_and_chunk_independent(gpu, oracle_mod):
    prob, (g, _) = _run_pair(oracle_mod, "small")
    mp = vs.mh_preset(3, population=64, generations=4)
    p1, s1 = g.run(mp, 5)
    p2, s2 = g.run(mp, 5)
    np.testing.assert_array_equal(p1, p2)
    np.testing.assert_array_equal(s1, s2)
    ids = np.arange(prob.cfg.n_spots, dtype=np.int32)[::-1].copy()
    parts = [g.run(mp, 5, ids[a:a + 23]) for a in range(0, len(ids), 23)]
    pc = np.concatenate([p for p, _ in parts])
    sc = np.concatenate([s for _, s in parts])
    np.testing.assert_array_equal(pc, p1[ids])
    np.testing.assert_array_equal(sc, s1[ids])


def test_context_churn_bitwise(gpu, oracle_mod):
    """Contexts created and destroyed back to back, alternating configurations: the device memory cache hands each
    destroyed context's blocks (with their stale contents) to the next one.  Every run and every scoring call must
    equal the first one of the same configuration bit for bit, and the first tiny run must match the oracle."""
    probs = [synth.make_problem("tiny"), synth.make_problem("small")]
    ref = {}
    for i in range(6):
        k = i % 2
        prob = probs[k]
        g = vs.Context.from_problem(prob, vs.score_params())
        mp = vs.mh_preset(3, population=32, generations=3)
        p, s = g.run(mp, 11)
        spot, q, t = synth.make_poses(300, prob.cfg.n_spots, 3.0, seed=4)
        sc = g.score_poses(spot, q, t)
        g.close()
        if k not in ref:
            ref[k] = (p, s, sc)
            if k == 0:
                o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
                assert_scores(sc, o.score(spot, q, t), "churn tiny")
        else:
            for a, b in zip((p, s, sc), ref[k]):
                np.testing.assert_array_equal(a, b)
        if i == 3:
            vs.release_cached_memory(0)  # later contexts allocate from the driver again: same results


def test_run_errors(gpu, oracle_mod):
    prob, (g, _) = _run_pair(oracle_mod)
    with pytest.raises(vs.VSError):
        g.run(vs.mh_preset(1, population=1, generations=2), 1)
    with pytest.raises(vs.VSError):
        g.run(vs.mh_preset(1), 1, np.array([7], np.int32))
    with pytest.raises(vs.VSError):
        g.run(vs.mh_preset(1, population=4096), 1)


@pytest.mark.parametrize("preset,P,G,K,cutoff", [(3, 32, 4, 1, 12.0), (2, 16, 2, 1, 12.0), (4, 64, 0, 1, 12.0),
                                                (3, 32, 2, 2, 12.0), (4, 64, 0, 3, 12.0),
                                                (3, 32, 3, 1, 0.0), (4, 64, 0, 2, 0.0)])
def test_lockstep_trace(gpu, oracle_mod, preset, P, G, K, cutoff):
    """Every stage of Algorithm 1 on the GPU re-derived by the oracle from the GPU's own state:
    pose generation byte-exact, decisions exact on GPU scores, scores within tolerance.
    K > 1: parallel-neighbourhood Improve (best of K proposals per step, N4); cutoff 0: all-pairs (paper) mode."""
    prob, (g, o) = _run_pair(oracle_mod, cutoff=cutoff)
    seed = 77
    mp_g = vs.mh_preset(preset, population=P, generations=G, ls_neighbours=K)
    mp_o = oracle_mod.mh_preset(preset, population=P, generations=G, ls_neighbours=K)
    m = oracle_mod.improve_count(mp_o)
    events = []
    g.run_trace(mp_g, seed, None, lambda *e: events.append(e))
    spots = range(prob.cfg.n_spots)
    prev = None       # population before the current stage
    sorted_S = None
    J = None
    n_near_ties = 0
    for stage, gen, l, pop, idx in events:
        if stage == vs.TRACE_INIT:
            for s in spots:
                for i in range(P):
                    np.testing.assert_array_equal(pop[s, i, :7], o.init_pose(seed, s, i))
            prev = pop
        elif stage == vs.TRACE_COMBINED:
            for s in spots:
                for j in range(P):
                    want = o.combine_child(mp_o, seed, s, gen, j, sorted_S[s, :, :7])
                    np.testing.assert_array_equal(pop[s, j, :7], want)
            prev = pop
        elif stage == vs.TRACE_SCORED:
            for s in spots:
                np.testing.assert_array_equal(pop[s, :, :7], prev[s, :, :7])
                assert_scores(pop[s, :, 7], o.score(np.full(P, s, np.int32), pop[s, :, :4], pop[s, :, 4:7]))
            prev = pop
        elif stage == vs.TRACE_SELECT:
            # the selected set is exact, listed in (score, index) order
            for s in spots:
                want = oracle_mod.select_improve(prev[s, :, 7].astype(np.float64), m)
                np.testing.assert_array_equal(np.sort(idx[s]), np.sort(want))
                sc = prev[s, idx[s], 7]
                assert np.all((np.diff(sc) > 0) | ((np.diff(sc) == 0) & (np.diff(idx[s]) > 0)))
            J = idx
        elif stage == vs.TRACE_LS:
            for s in spots:
                js = set(J[s].tolist())
                for j in range(P):
                    if j not in js:
                        np.testing.assert_array_equal(pop[s, j], prev[s, j])
                        continue
                    props = [o.ls_proposal(mp_o, seed, s, gen, l, j, prev[s, j, :7], k=k) for k in range(K)]
                    e_props = [o.score_one(s, p[:4], p[4:]) for p in props]
                    e_old = o.score_one(s, prev[s, j, :4], prev[s, j, 4:7])
                    kbest = int(np.argmin(e_props))
                    accepted = not np.array_equal(pop[s, j], prev[s, j])
                    if accepted:
                        hit = [k for k in range(K) if np.array_equal(pop[s, j, :7], props[k])]
                        assert hit, (s, j)
                        assert pop[s, j, 7] < prev[s, j, 7]
                        assert_scores([pop[s, j, 7]], [e_props[hit[0]]])
                        if hit[0] != kbest:   # another proposal is best in fp64: only at a near tie
                            assert abs(e_props[hit[0]] - e_props[kbest]) <= 2 * tol(e_props[kbest])
                            n_near_ties += 1
                    if accepted != (e_props[kbest] < e_old):
                        assert abs(e_props[kbest] - e_old) <= 2 * tol(e_old), (s, j, e_props[kbest], e_old)
                        n_near_ties += 1
            prev = pop
        elif stage == vs.TRACE_SORTED:
            for s in spots:
                order = np.argsort(prev[s, :, 7], kind="stable")
                np.testing.assert_array_equal(pop[s], prev[s, order])
            sorted_S = pop
            prev = pop
        elif stage == vs.TRACE_INCLUDED:
            for s in spots:
                origin = oracle_mod.include(sorted_S[s, :, 7].astype(np.float64), prev[s, :, 7].astype(np.float64))
                both_pop = np.concatenate([sorted_S[s], prev[s]])
                np.testing.assert_array_equal(pop[s], both_pop[origin])
            sorted_S = pop
            prev = pop
    assert n_near_ties <= 2


def test_run_parallel_neighbourhood_free_running(gpu, oracle_mod):
    """N4: M4 with K = 4 proposals per Improve step, GPU vs oracle on identical streams."""
    prob, (g, o) = _run_pair(oracle_mod)
    _, sg = g.run(vs.mh_preset(4, population=96, ls_neighbours=4), 21)
    _, so = o.run(oracle_mod.mh_preset(4, population=96, ls_neighbours=4), 21)
    assert np.all(np.abs(sg - so) <= 1e-3 * np.maximum(np.abs(so), 1.0))


def test_graph_replay_matches_direct_launches(gpu, oracle_mod):
    """vs_run captures a CUDA graph on the second identical call and replays it: results are bit-identical to
    direct launches for any seed and any spot ids of the same count (the seed and ids live in device memory)."""
    prob, (g, _) = _run_pair(oracle_mod, "small")
    mp = vs.mh_preset(3, population=64, generations=3)
    ids_a = np.arange(0, 40, dtype=np.int32)
    ids_b = np.arange(20, 60, dtype=np.int32)[::-1].copy()
    r1 = g.run(mp, 1, ids_a)          # direct
    r2 = g.run(mp, 2, ids_a)          # captured
    r3 = g.run(mp, 3, ids_b)          # replayed
    r4 = g.run(mp, 1, ids_a)          # replayed
    fresh = vs.Context.from_problem(prob, vs.score_params(cutoff=12.0))
    f3 = fresh.run(mp, 3, ids_b)
    for x, y in [(r1, r4), (r3, f3)]:
        np.testing.assert_array_equal(x[0], y[0])
        np.testing.assert_array_equal(x[1], y[1])
    assert not np.array_equal(r1[1], r2[1])
    st = g.stats()
    assert st["kernel_launches"] > 0 and st["poses_scored"] > 0


def test_run_extreme_sizes(gpu, oracle_mod):
    """Largest population (2048: 4096-key include sort), a 256-atom ligand (43 groups), a single spot, and
    duplicated spot ids (same global id -> identical results)."""
    prob = synth.make_custom(900, 256, 3, seed=9)
    g, o = both(oracle_mod, prob, 12.0)
    mp_g = vs.mh_preset(3, population=2048, generations=1, ls_steps=1)
    mp_o = oracle_mod.mh_preset(3, population=2048, generations=1, ls_steps=1)
    pg, sg = g.run(mp_g, 4, np.array([2], np.int32))
    po, so = o.run(mp_o, 4, np.array([2], np.int32))
    assert abs(sg[0] - so[0]) <= 1e-3 * max(abs(so[0]), 1.0)
    pd, sd = g.run(vs.mh_preset(2, population=16, generations=2), 5, np.array([1, 1, 0, 1], np.int32))
    np.testing.assert_array_equal(sd[0], sd[1])
    np.testing.assert_array_equal(sd[0], sd[3])
    np.testing.assert_array_equal(pd[0], pd[3])
