"""Lockstep check of a GPU vs_run against the oracle (test infrastructure; SURVEY.md §8(c) "Near ties").

The GPU dumps its population after every stage of Algorithm 1 (vs_run_trace); the oracle re-derives each stage
from the GPU's own state: pose generation byte-exact (Philox + fp32 single ops, R23/R24), Select / Include / sort
decisions exact on the GPU's fp32 scores, scores within the per-pose tolerance of the fp64 definition, and every
Improve accept decision equal to the fp64 one except at a near tie (|gap| <= 2 x tolerance, R26), where both
outcomes are correct.  Sort-like decisions (Select's best m, the generation-0 sort, Include's best P) are exact
on the GPU's scores; where the rounded fp64 scores would order two elements differently, their fp64 gap must be a
near tie too.  Returns the near ties per spot row: a free-running oracle run can leave the GPU's trajectory only at
one of them.
"""
import numpy as np

from paper_conf_ppopp_imbernoncg16_b200 import vs


def tol(ref):
    return np.maximum(1e-4 * np.abs(ref), 1e-3)


def check_scores(gpu, ref, what=""):
    gpu = np.asarray(gpu, np.float64)
    ref = np.asarray(ref, np.float64)
    err = np.abs(gpu - ref)
    bad = err > tol(ref)
    assert not bad.any(), f"{what}: {bad.sum()} / {len(ref)} out of tolerance; worst err/tol {(err / tol(ref)).max():.3g}"


def lockstep(oracle_mod, g, o, mp_g, mp_o, seed, ids=None, n_spots=None):
    P = mp_o.population
    K = mp_o.ls_neighbours
    m = oracle_mod.improve_count(mp_o)
    spots = np.arange(n_spots, dtype=np.int32) if ids is None else np.asarray(ids, np.int32)
    R = len(spots)
    events = []
    g.run_trace(mp_g, seed, None if ids is None else spots, lambda *e: events.append(e))
    near = np.zeros(R, np.int64)
    prev = sorted_S = J = None
    ref = ref_S = None          # fp64 oracle scores of prev / sorted_S

    def order_ties(r, gpu_keep, ref_sc, n_keep):
        """The GPU kept gpu_keep (indices into ref_sc) as the best n_keep; the fp64 scores may only disagree at a
        near tie around the boundary."""
        want = np.argsort(np.float32(ref_sc), kind="stable")[:n_keep]
        diff = np.setxor1d(want, gpu_keep)
        if len(diff):
            bound = np.sort(ref_sc)[n_keep - 1] if n_keep <= len(ref_sc) else np.inf
            for x in diff:
                assert abs(ref_sc[x] - bound) <= 2 * tol(bound), (r, x, ref_sc[x], bound)
            near[r] += 1

    def rank_ties(r, ref_sorted):
        """Ranks feed Select's tournaments: where the fp64 scores (rounded to fp32) of two neighbours in the GPU's
        order are inverted, the gap must be a near tie."""
        f = np.float32(ref_sorted)
        inv = np.nonzero(f[1:] < f[:-1])[0]
        for i in inv:
            assert abs(ref_sorted[i + 1] - ref_sorted[i]) <= 2 * tol(ref_sorted[i]), (r, i, ref_sorted[i:i + 2])
        near[r] += len(inv)

    for stage, gen, l, pop, idx in events:
        if stage == vs.TRACE_INIT:
            for r, s in enumerate(spots):
                for i in range(P):
                    np.testing.assert_array_equal(pop[r, i, :7], o.init_pose(seed, int(s), i))
            prev = pop
        elif stage == vs.TRACE_COMBINED:
            for r, s in enumerate(spots):
                for j in range(P):
                    want = o.combine_child(mp_o, seed, int(s), gen, j, sorted_S[r, :, :7])
                    np.testing.assert_array_equal(pop[r, j, :7], want)
            prev = pop
        elif stage == vs.TRACE_SCORED:
            np.testing.assert_array_equal(pop[:, :, :7], prev[:, :, :7])
            sp = np.repeat(spots, P)
            flat = pop.reshape(R * P, 8)
            ref = o.score(sp, flat[:, :4], flat[:, 4:7])
            check_scores(flat[:, 7], ref, f"scored g={gen}")
            ref = ref.reshape(R, P)
            prev = pop
        elif stage == vs.TRACE_SELECT:
            for r in range(R):
                want = oracle_mod.select_improve(prev[r, :, 7].astype(np.float64), m)
                np.testing.assert_array_equal(np.sort(idx[r]), np.sort(want))
                sc = prev[r, idx[r], 7]
                assert np.all((np.diff(sc) > 0) | ((np.diff(sc) == 0) & (np.diff(idx[r]) > 0)))
                order_ties(r, idx[r], ref[r], m)
            J = idx
        elif stage == vs.TRACE_LS:
            props, owner = [], []
            for r, s in enumerate(spots):
                for j in J[r]:
                    for k in range(K):
                        props.append(o.ls_proposal(mp_o, seed, int(s), gen, l, int(j), prev[r, j, :7], k=k))
                        owner.append((r, int(j), k))
            props = np.array(props, np.float32)
            sp = np.array([spots[r] for r, _, _ in owner], np.int32)
            e_props = o.score(sp, props[:, :4], props[:, 4:])
            olds = np.array([prev[r, j, :7] for r, j, _ in owner[::K]], np.float32)
            e_old = o.score(sp[::K], olds[:, :4], olds[:, 4:])
            for n, (r, j, _) in enumerate(owner[::K]):
                ep = e_props[n * K:(n + 1) * K]
                kbest = int(np.argmin(ep))
                accepted = not np.array_equal(pop[r, j], prev[r, j])
                if accepted:
                    hit = [k for k in range(K) if np.array_equal(pop[r, j, :7], props[n * K + k])]
                    assert hit, (r, j)
                    assert pop[r, j, 7] < prev[r, j, 7]
                    check_scores([pop[r, j, 7]], [ep[hit[0]]])
                    ref[r, j] = ep[hit[0]]
                    if hit[0] != kbest:   # another proposal is best in fp64: only at a near tie
                        assert abs(ep[hit[0]] - ep[kbest]) <= 2 * tol(ep[kbest])
                        near[r] += 1
                if accepted != (ep[kbest] < e_old[n]):
                    assert abs(ep[kbest] - e_old[n]) <= 2 * tol(e_old[n]), (r, j, ep[kbest], e_old[n])
                    near[r] += 1
            for r in range(R):                      # elements outside J unchanged
                keep = np.setdiff1d(np.arange(P), J[r])
                np.testing.assert_array_equal(pop[r, keep], prev[r, keep])
            prev = pop
        elif stage == vs.TRACE_SORTED:
            for r in range(R):
                order = np.argsort(prev[r, :, 7], kind="stable")
                np.testing.assert_array_equal(pop[r], prev[r, order])
                ref[r] = ref[r, order]
                rank_ties(r, ref[r])
            sorted_S = pop
            ref_S = ref.copy()
            prev = pop
        elif stage == vs.TRACE_INCLUDED:
            new_ref = np.empty_like(ref)
            for r in range(R):
                origin = oracle_mod.include(sorted_S[r, :, 7].astype(np.float64), prev[r, :, 7].astype(np.float64))
                both_pop = np.concatenate([sorted_S[r], prev[r]])
                np.testing.assert_array_equal(pop[r], both_pop[origin])
                both_ref = np.concatenate([ref_S[r], ref[r]])
                order_ties(r, origin, both_ref, P)
                new_ref[r] = both_ref[origin]
                rank_ties(r, new_ref[r])
            ref = new_ref
            sorted_S = pop
            ref_S = ref.copy()
            prev = pop
    return near
