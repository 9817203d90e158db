"""Multi-process logic of the multi-GPU driver on CPU (gloo, world_size 2).

The dynamic chunk queue + one gather must give every spot exactly once and
the same per-spot result as a single process (the RNG is keyed by the global
spot id).  The oracle stands in for the GPU runner here (test only).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ppopp_imbernoncg16_b200 import dist as vdist


def test_chunk_schedule_covers_once():
    for n, r in [(500, 8), (7, 4), (1, 3), (2000, 2), (64, 1), (0, 2)]:
        sch = vdist.chunk_schedule(n, r, min_chunk=4)
        covered = [i for a, b in sch for i in range(a, b)]
        assert covered == list(range(n))
        if r > 1 and len(sch) > 2:
            sizes = [b - a for a, b in sch]
            assert sizes[0] >= sizes[-1]            # guided: large first
            assert sizes[-1] <= max(4, n // (2 * r))  # short tail


def test_best_per_spot():
    rec = np.array([[1, -2.0, 1, 0, 0, 0, 0, 0, 0], [1, -3.0, 0, 1, 0, 0, 0, 0, 0], [0, 5.0, 1, 0, 0, 0, 1, 1, 1]],
                   np.float32)
    pose, score = vdist.best_per_spot(rec, 3)
    assert score[1] == -3.0 and pose[1, 1] == 1 and score[0] == 5.0 and np.isnan(score[2])


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, mode, out_path):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem("tiny")
    o = oracle.Oracle.from_problem(prob, oracle.score_params())
    mp_ = oracle.mh_preset(3, population=16, generations=2)
    n = prob.cfg.n_spots
    if mode == "strong":
        store = dist.distributed_c10d._get_default_store()
        parts = []

        def work(a, b):
            ids = np.arange(a, b, dtype=np.int32)
            pose, sc = o.run(mp_, 42, ids)
            parts.append(vdist.pack(ids, pose, sc.astype(np.float32)))

        vdist.claim_chunks(store, "q0", vdist.chunk_schedule(n, world, 1), work)
        rec = np.concatenate(parts) if parts else np.zeros((0, vdist.REC), np.float32)
    else:  # weak: independent executions with seed + rank, best-of on rank 0
        pose, sc = o.run(mp_, 42 + rank)
        rec = vdist.pack(np.arange(n, dtype=np.int32), pose, sc.astype(np.float32))
    allrec = vdist.gather_records(torch.from_numpy(rec), torch.device("cpu"))
    if rank == 0:
        np.save(out_path, allrec.numpy())
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["strong", "weak"])
def test_queue_and_gather_gloo(tmp_path, mode, oracle_mod):
    out = str(tmp_path / "rec.npy")
    mp.spawn(_worker, args=(2, _free_port(), mode, out), nprocs=2, join=True)
    rec = np.load(out)
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem("tiny")
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    mp_ = oracle_mod.mh_preset(3, population=16, generations=2)
    n = prob.cfg.n_spots
    if mode == "strong":
        assert sorted(rec[:, 0].astype(int).tolist()) == list(range(n))   # every spot exactly once
        pose, sc = o.run(mp_, 42)
        got_pose, got_sc = vdist.best_per_spot(rec, n)
        np.testing.assert_array_equal(got_sc, sc.astype(np.float32))
        np.testing.assert_array_equal(got_pose, pose)
    else:
        assert len(rec) == 2 * n
        runs = [o.run(mp_, 42 + r)[1].astype(np.float32) for r in range(2)]
        _, got_sc = vdist.best_per_spot(rec, n)
        np.testing.assert_array_equal(got_sc, np.minimum(runs[0], runs[1]))


def test_percent_and_shares():
    """Eq. (1): Percent = t / t_slowest; shares proportional to 1/Percent (R27)."""
    p = vdist.percent_from_times([2.0, 1.0, 4.0])
    assert p == [0.5, 0.25, 1.0]
    sh = vdist.shares_from_percent(p, 700)
    sizes = [b - a for a, b in sh]
    assert sum(sizes) == 700 and sh[0][0] == 0 and sh[-1][1] == 700
    assert sizes == [200, 400, 100]
    assert vdist.shares_from_percent([1.0, 1.0], 5) in ([(0, 3), (3, 5)], [(0, 2), (2, 5)])


def _warm_worker(rank, world, port, out_path):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # rank 1 is "two times faster" (Percent = 0.5)
    rng = vdist.warmup_split(lambda: 2.0 if rank == 0 else 1.0, 90, torch.device("cpu"))
    out = [None] * world
    dist.all_gather_object(out, rng)
    if rank == 0:
        np.save(out_path, np.array(out))
    dist.destroy_process_group()


def test_warmup_split_gloo(tmp_path):
    out = str(tmp_path / "split.npy")
    mp.spawn(_warm_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    split = np.load(out)
    assert split.tolist() == [[0, 30], [30, 90]]
