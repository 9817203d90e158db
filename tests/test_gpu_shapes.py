"""Launch shapes never change a result; the instrumentation counts what it claims.

The pair kernel cuts a scoring launch into warps by a launch shape (KP item pairs per lane: 64 KP items per chunk;
one warp per chunk and canonical list split) chosen per launch for speed (vs_api.cu choose_shape).  An item's
energy is the fixed fp64 tree (e_0 + e_1) + (e_2 + e_3) of its S split energies whatever the shape (vs_cells.cu
header), so scores, vs_run results and the scores of vs_score_poses vs vs_run are bitwise identical across shapes.
VS_SHAPE=kp (read at vs_create) forces a shape for these tests.
"""
import os

import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import synth, vs

pytestmark = pytest.mark.gpu
SHAPES = {1: ["2", "1"], 2: ["2", "1"], 4: ["2", "1"]}


@pytest.fixture(scope="module")
def torch():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def ctx_with_shape(prob, shape, S=1, **sp):
    old = os.environ.get("VS_SHAPE")
    if shape:
        os.environ["VS_SHAPE"] = shape
    try:
        return vs.Context.from_problem(prob, vs.score_params(list_splits=S, **sp))
    finally:
        if old is None:
            os.environ.pop("VS_SHAPE", None)
        else:
            os.environ["VS_SHAPE"] = old


@pytest.mark.parametrize("S", [1, 2, 4])
@pytest.mark.parametrize("cutoff", [12.0, 0.0])
@pytest.mark.parametrize("name", ["small", "custom_hb"])
def test_scores_bitwise_across_shapes(torch, oracle_mod, name, cutoff, S):
    if name == "custom_hb":          # every H-bond slot layout: H-bond-heavy ligand (H = 2 at KP 2)
        prob = synth.make_custom(2500, 23, 6, seed=17)
        rng = np.random.default_rng(5)
        prob.lig.type[:] = rng.choice([synth.T_N, synth.T_O, synth.T_HD, synth.T_HD, synth.T_C],
                                      size=len(prob.lig.type)).astype(np.int32)
    else:
        prob = synth.make_problem(name)
    spot, q, t = synth.make_poses(3000, prob.cfg.n_spots, 3.0, seed=13)
    t[:1000] *= 0.3
    ref = None
    for sh in SHAPES[S]:
        got = ctx_with_shape(prob, sh, S, cutoff=cutoff).score_poses(spot, q, t)
        if ref is None:
            ref = got
            o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params(cutoff=cutoff))
            idx = np.arange(0, len(spot), 150)
            r = o.score(spot[idx], q[idx], t[idx])
            assert np.all(np.abs(got[idx] - r) <= np.maximum(1e-4 * np.abs(r), 1e-3))
        np.testing.assert_array_equal(got, ref, err_msg=f"shape {sh}")


@pytest.mark.parametrize("S", [1, 4])
def test_run_bitwise_across_shapes_and_entry_points(torch, S):
    prob = synth.make_problem("small")
    mp = vs.mh_preset(3, population=64, generations=3)
    ref = None
    for sh in [None] + SHAPES[S]:
        g = ctx_with_shape(prob, sh, S)
        p, s = g.run(mp, 17)
        if ref is None:
            ref = (p, s)
            # the best score of a run is the score vs_score_poses gives its pose (a pose's score is a function of
            # the pose alone)
            again = g.score_poses(np.arange(prob.cfg.n_spots, dtype=np.int32), p[:, :4], p[:, 4:])
            np.testing.assert_array_equal(again, s)
        else:
            np.testing.assert_array_equal(p, ref[0], err_msg=f"shape {sh}")
            np.testing.assert_array_equal(s, ref[1], err_msg=f"shape {sh}")


@pytest.mark.parametrize("name", ["small", "medium"])
def test_item_class_layout_bitwise(torch, name):
    """The merged item layout (every ligand atom in the H-bond slots, one curve order: the default for ligands with at
    most a third of H-bond atoms) and the class-separated layout give bitwise identical scores and runs."""
    prob = synth.make_problem(name)
    spot, q, t = synth.make_poses(2000, prob.cfg.n_spots, 3.0, seed=4)
    mp = vs.mh_preset(3, population=32, generations=2)
    ids = np.arange(min(prob.cfg.n_spots, 16), dtype=np.int32)
    res = []
    for m in ("0", "1"):
        old = os.environ.get("VS_CELL_MERGE")
        os.environ["VS_CELL_MERGE"] = m
        try:
            g = vs.Context.from_problem(prob, vs.score_params())
        finally:
            if old is None:
                os.environ.pop("VS_CELL_MERGE", None)
            else:
                os.environ["VS_CELL_MERGE"] = old
        res.append((g.score_poses(spot, q, t), g.run(mp, 9, ids)))
    np.testing.assert_array_equal(res[0][0], res[1][0])
    np.testing.assert_array_equal(res[0][1][0], res[1][1][0])
    np.testing.assert_array_equal(res[0][1][1], res[1][1][1])


def test_list_splits_change_only_rounding(torch, oracle_mod):
    """S = 1, 2, 4 canonical splits: a summation order; every variant within the tolerance of the oracle and within
    fp32 rounding of each other."""
    prob = synth.make_problem("small")
    spot, q, t = synth.make_poses(2000, prob.cfg.n_spots, 3.0, seed=21)
    got = {S: vs.Context.from_problem(prob, vs.score_params(list_splits=S)).score_poses(spot, q, t) for S in (1, 2, 4)}
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    idx = np.arange(0, 2000, 40)
    r = o.score(spot[idx], q[idx], t[idx])
    for S, v in got.items():
        assert np.all(np.abs(v[idx] - r) <= np.maximum(1e-4 * np.abs(r), 1e-3)), S
        assert np.all(np.abs(v - got[1]) <= 1e-5 * np.maximum(np.abs(got[1]), 1.0)), S
    assert not np.array_equal(got[4], got[1])           # a different (valid) rounding
    with pytest.raises(vs.VSError):
        vs.Context.from_problem(prob, vs.score_params(list_splits=3))


def test_census_counts_pairs_within_cutoff(torch, oracle_mod):
    """VS_TIMING_CENSUS: pairs_within equals the oracle's count of pairs with r^2 < rc^2 (the decision is taken in
    fp32 on the GPU and fp64 in the oracle: pairs within rounding of rc may differ), scores bitwise unchanged."""
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    spot, q, t = synth.make_poses(400, prob.cfg.n_spots, 3.0, seed=2)
    plain = g.score_poses(spot, q, t)
    g.reset_stats()
    g.set_timing(vs.TIMING_CENSUS)
    cen = g.score_poses(spot, q, t)
    st = g.stats()
    np.testing.assert_array_equal(cen, plain)
    o.score(spot, q, t)
    want = o.pairs_within()
    assert abs(st["pairs_within"] - want) <= 2 + 1e-6 * want, (st["pairs_within"], want)
    g.set_timing(0)
    g.reset_stats()
    g.score_poses(spot, q, t)
    ev = g.stats()["pairs_evaluated"]                  # census launches count within-rc pairs instead
    assert st["pairs_within"] < ev < st["pairs"]
    # a census run gives the same result as a plain one
    mp = vs.mh_preset(3, population=32, generations=2)
    g.set_timing(0)
    p0, s0 = g.run(mp, 3)
    g.set_timing(vs.TIMING_CENSUS)
    p1, s1 = g.run(mp, 3)
    np.testing.assert_array_equal(s0, s1)


def test_kernel_intervals_inside_graph_replays(torch):
    """VS_TIMING_KERNEL records every pair-kernel launch interval, also in replayed CUDA graphs."""
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    mp = vs.mh_preset(3, population=64, generations=2)
    g.set_timing(vs.TIMING_KERNEL)
    st = torch.cuda.Stream()
    bp = torch.empty((prob.cfg.n_spots, 7), device="cuda")
    bs = torch.empty(prob.cfg.n_spots, device="cuda")
    for _ in range(2):                     # direct, then captured
        g.run_async(mp, 1, None, bp, bs, st)
    st.synchronize()
    g.reset_stats()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(3):                     # replays
        g.run_async(mp, 1, None, bp, bs, st)
    e1.record(st)
    st.synchronize()
    s = g.stats()
    wall = e0.elapsed_time(e1)
    assert s["pair_timed_launches"] == s["score_launches"] > 0
    assert 0 < s["pair_busy_ms"] <= wall * 1.01 + 0.05
    assert s["pair_launch_ms"] >= s["pair_busy_ms"] * 0.999
    # warp-time: positive, at most 24 resident one-warp CTAs per SM on average over the busy time
    assert 0 < s["pair_warp_ms"] <= 24 * 148 * s["pair_busy_ms"] * 1.01
    # the raw intervals (vs_pair_intervals): as many as timed launches, their sum and union are the stats'
    iv = g.pair_intervals().astype(np.int64)
    assert len(iv) == s["pair_timed_launches"] and np.all(iv[:, 1] >= iv[:, 0])
    assert abs((iv[:, 1] - iv[:, 0]).sum() * 1e-6 - s["pair_launch_ms"]) < 1e-3
    import bench
    assert abs(bench.union_ms(iv) - s["pair_busy_ms"]) < 1e-3


def test_graph_cache_keeps_several_shapes(torch):
    """Runs of a few chunk sizes (a multi-GPU queue's chunks) each replay their own CUDA graph (LRU of 4): results
    equal direct launches bit for bit whatever the interleaving."""
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    mp = vs.mh_preset(3, population=32, generations=2)
    chunks = [np.arange(0, 10, dtype=np.int32), np.arange(10, 30, dtype=np.int32), np.arange(30, 64, dtype=np.int32),
              np.arange(5, 12, dtype=np.int32), np.arange(40, 45, dtype=np.int32)]
    ref = [g.run(mp, 3, ids) for ids in chunks]                  # direct launches (first sight of each shape)
    st = torch.cuda.Stream()
    for rep in range(3):                                          # second sight captures, then replays; 5 shapes > 4
        for ids, (rp, rs) in zip(chunks, ref):
            bp = torch.empty((len(ids), 7), device="cuda")
            bs = torch.empty(len(ids), device="cuda")
            g.run_async(mp, 3, ids, bp, bs, st)
            st.synchronize()
            np.testing.assert_array_equal(bs.cpu().numpy(), rs)
            np.testing.assert_array_equal(bp.cpu().numpy(), rp)


def test_long_lists_and_splits(torch, oracle_mod):
    """Lists streamed whole (> 16384 atoms: cut by position into the S canonical splits) give the same scores for
    every S within fp32 rounding and the oracle's within tolerance; the census counts them."""
    prob = synth.make_custom(25000, 30, 3, seed=23)
    spot, q, t = synth.make_poses(120, 3, 3.0, seed=4)
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params(cutoff=70.0))
    ref = o.score(spot, q, t)
    for S in (1, 2, 4):
        g = vs.Context.from_problem(prob, vs.score_params(cutoff=70.0, list_splits=S))
        assert g.list_lengths().max() > 16384
        got = g.score_poses(spot, q, t)
        assert np.all(np.abs(got - ref) <= np.maximum(1e-4 * np.abs(ref), 1e-3)), S
        g.set_timing(vs.TIMING_CENSUS)
        g.reset_stats()
        np.testing.assert_array_equal(g.score_poses(spot, q, t), got)
        assert g.stats()["pairs_within"] > 0


def test_census_all_pairs_counts_every_pair(torch):
    prob = synth.make_problem("tiny")
    g = vs.Context.from_problem(prob, vs.score_params(cutoff=0.0))
    g.set_timing(vs.TIMING_CENSUS)
    g.reset_stats()
    spot, q, t = synth.make_poses(50, prob.cfg.n_spots, 3.0, seed=1)
    g.score_poses(spot, q, t)
    st = g.stats()
    assert st["pairs_within"] == st["pairs"] == 50 * prob.cfg.n_rec * prob.cfg.n_lig


def test_no_hbond_ligand_kp1(torch, oracle_mod):
    """A ligand without H-bond atoms (H = 0: no H-bond slot pairs at KP 1 or 2) through both shapes and a run."""
    prob = synth.make_custom(2500, 23, 6, seed=17)
    prob.lig.type[:] = synth.T_C
    spot, q, t = synth.make_poses(500, 6, 3.0, seed=2)
    res = [ctx_with_shape(prob, sh, 1).score_poses(spot, q, t) for sh in ("2", "1")]
    np.testing.assert_array_equal(res[0], res[1])
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    r = o.score(spot[:60], q[:60], t[:60])
    assert np.all(np.abs(res[0][:60] - r) <= np.maximum(1e-4 * np.abs(r), 1e-3))


@pytest.mark.parametrize("preset,K", [(3, 1), (1, 1), (4, 3)])
def test_run_stats_count_scored_poses_and_pairs(torch, preset, K):
    """vs_run's `poses_scored` and `pairs` (workload pairs: n_lig x list length of the pose's spot per scored pose):
    every spot scores (G + 1) x (P + L m K) poses -- the initial / offspring rounds and Improve's proposals, m =
    round(f P) (S§8(c) R17)."""
    prob = synth.make_problem("small")
    g = vs.Context.from_problem(prob, vs.score_params())
    mp = vs.mh_preset(preset, population=32, generations=3 if preset != 4 else 0, ls_neighbours=K)
    ids = np.array([3, 0, 17, 5, 3], dtype=np.int32)[:4]
    g.reset_stats()
    g.run(mp, 5, ids)
    g.run(mp, 6)
    st = g.stats()
    m = max(1, min(mp.population, int(np.floor(float(np.float32(mp.improve_frac)) * mp.population + 0.5)))) \
        if mp.improve_frac > 0 else 0
    per = (mp.generations + 1) * (mp.population + (mp.ls_steps * m * K if mp.improve_frac > 0 else 0))
    L = g.list_lengths()
    n_all = prob.cfg.n_spots
    assert st["poses_scored"] == per * (len(ids) + n_all)
    assert st["pairs"] == per * prob.cfg.n_lig * (int(sum(int(L[s]) for s in ids)) + int(sum(int(x) for x in L)))


@pytest.mark.parametrize("S", [1, 4])
def test_list_grid_changes_only_rounding(torch, oracle_mod, S):
    """The per-spot list grid (cells per axis, a context property: 18 for 1-2 splits, 20 for 4; VS_CELL_GRID forces
    it) decides which list atoms a chunk streams and their order inside a cell row, never which pairs contribute:
    scores agree with the oracle at every grid, the within-rc census count is identical, and grids differ only by
    fp32 summation order."""
    prob = synth.make_problem("small")
    spot, q, t = synth.make_poses(3000, prob.cfg.n_spots, 3.0, seed=23)
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    idx = np.arange(0, 3000, 10)
    ref = o.score(spot[idx], q[idx], t[idx])
    got, within = {}, {}
    for G in (8, 12, 16, 20, 24):
        old = os.environ.get("VS_CELL_GRID")
        os.environ["VS_CELL_GRID"] = str(G)
        try:
            g = vs.Context.from_problem(prob, vs.score_params(list_splits=S))
        finally:
            if old is None:
                os.environ.pop("VS_CELL_GRID", None)
            else:
                os.environ["VS_CELL_GRID"] = old
        g.reset_stats()
        g.set_timing(vs.TIMING_CENSUS)
        got[G] = g.score_poses(spot, q, t)
        within[G] = g.stats()["pairs_within"]
        assert np.all(np.abs(got[G][idx] - ref) <= np.maximum(1e-4 * np.abs(ref), 1e-3)), G
    assert len(set(within.values())) == 1, within
    for G in got:
        np.testing.assert_allclose(got[G], got[16], rtol=2e-6, atol=1e-4)
