"""Screening sweep (N1): unit schedule on CPU; GPU sweep vs the oracle per ligand."""
import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import screen, synth


def test_unit_schedule_covers_each_pair_once():
    sizes = [15, 80, 33, 80, 20]
    for ranks in (1, 2, 8):
        u = screen.unit_schedule(sizes, 37, ranks, min_chunk=4)
        seen = [(li, s) for li, a, b in u for s in range(a, b)]
        assert sorted(seen) == [(li, s) for li in range(5) for s in range(37)]
        first = [li for li, a, b in u]
        assert first[0] in (1, 3)                     # largest ligands first (LPT)
        if ranks == 1:
            assert len(u) == 5


def test_ligand_seeds_distinct():
    s = {screen.ligand_seed(42, i) for i in range(1000)}
    assert len(s) == 1000 and all(0 <= x < 2 ** 64 for x in s)


@pytest.mark.gpu
def test_screen_matches_oracle(oracle_mod):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ppopp_imbernoncg16_b200 import vs
    rng = np.random.default_rng(3)
    rec = synth.make_molecule(600, rng)
    spots = synth.surface_spots(rec, 6)
    ligs = [synth.make_molecule(n, rng) for n in (9, 23, 70)]
    mp_g = vs.mh_preset(3, population=16, generations=3)
    mp_o = oracle_mod.mh_preset(3, population=16, generations=3)
    sc = screen.Screen(rec, spots, ligs, vs.score_params(), mp_g, seed=11)
    pose = torch.zeros((3, 6, 7), device="cuda")
    score = torch.zeros((3, 6), device="cuda")
    for li, a, b in screen.unit_schedule([len(l.q) for l in ligs], 6, 2, min_chunk=2):
        sc.run_unit(li, a, b, pose[li, a:b], score[li, a:b])
    torch.cuda.synchronize()
    got = score.cpu().numpy()
    for li, L in enumerate(ligs):
        o = oracle_mod.Oracle(rec.xyz, rec.q, rec.type, L.xyz, L.q, L.type, spots, oracle_mod.score_params())
        _, want = o.run(mp_o, screen.ligand_seed(11, li))
        np.testing.assert_allclose(got[li], want, rtol=1e-3, atol=1e-3)
    sc.close()
