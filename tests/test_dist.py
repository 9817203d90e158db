"""Multi-process logic of the multi-GPU driver on CPU (gloo, world_size 2).

The dynamic chunk queue (ChunkQueue + run_dynamic with chunks in flight) + ONE fixed-size gather must give every
spot exactly once and the same per-spot result as a single process (the RNG is keyed by the global spot id);
the warm-up split (Eq. 1) must size the shares by 1 / Percent.  The oracle stands in for the GPU runner
here (test only).
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
    for n, k in [(500, 8), (500, 16), (7, 4), (3, 8), (0, 2)]:
        ch = vdist.equal_chunks(n, k)
        assert [i for a, b in ch for i in range(a, b)] == list(range(n))
        if n >= k:
            assert max(b - a for a, b in ch) - min(b - a for a, b in ch) <= 1


def test_run_dynamic_slots_and_order():
    """Up to `slots` chunks in flight; a slot is waited for before it is reused; every chunk once."""
    q = vdist.ChunkQueue(None, "k", 5)
    log = []
    sched = [(0, 2), (2, 4), (4, 6), (6, 8), (8, 10)]
    done = vdist.run_dynamic(q, sched, 2, lambda s, a, b: log.append(("L", s, a)), lambda s: log.append(("W", s)))
    assert done == [0, 1, 2, 3, 4]
    assert log == [("L", 0, 0), ("L", 1, 2), ("W", 0), ("L", 0, 4), ("W", 1), ("L", 1, 6), ("W", 0), ("L", 0, 8),
                   ("W", 1), ("W", 0)]
    assert vdist.ChunkQueue(None, "k", 0).claim() is None


def test_assemble_and_best_of():
    t0 = vdist.empty_records(4, "cpu").numpy().copy()
    t1 = t0.copy()
    t0[0] = [0, -1, 1, 0, 0, 0, 0, 0, 0]
    t0[2] = [2, -3, 1, 0, 0, 0, 1, 1, 1]
    t1[1] = [1, -2, 0, 1, 0, 0, 0, 0, 0]
    t1[3] = [3, 5, 0, 0, 1, 0, 0, 0, 0]
    pose, score, owner = vdist.assemble([t0, t1], 4)
    assert score.tolist() == [-1, -2, -3, 5] and owner.tolist() == [0, 1, 0, 1] and pose[1, 1] == 1
    with pytest.raises(RuntimeError):
        vdist.assemble([t0, t0], 4)                  # spots run twice
    with pytest.raises(RuntimeError):
        vdist.assemble([t0], 4)                      # spots never run
    full0 = np.array([[i, -i, 1, 0, 0, 0, 0, 0, 0] for i in range(3)], np.float32)
    full1 = full0.copy()
    full1[1, 1] = -7
    _, sc = vdist.best_of([full0, full1])
    assert sc.tolist() == [0, -7, -2]


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
    rec = vdist.empty_records(n, "cpu")
    if mode == "queue":
        store = dist.distributed_c10d._get_default_store()
        sched = vdist.equal_chunks(n, 3)      # 3 chunks, 2 ranks, 2 slots each: dynamic claims

        def launch(slot, a, b):
            ids = np.arange(a, b, dtype=np.int32)
            pose, sc = o.run(mp_, 42, ids)
            vdist.fill_records(rec, a, b, torch.from_numpy(pose), torch.from_numpy(sc.astype(np.float32)))

        vdist.run_dynamic(vdist.ChunkQueue(store, "q0", len(sched)), sched, 2, launch, lambda s: None)
    else:  # replicas: independent executions with seed + rank, best-of on rank 0
        pose, sc = o.run(mp_, 42 + rank)
        vdist.fill_records(rec, 0, n, torch.from_numpy(pose), torch.from_numpy(sc.astype(np.float32)))
    tables = vdist.gather_fixed(rec, torch.device("cpu"))
    if rank == 0:
        np.save(out_path, np.stack([t.numpy() for t in tables]))
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["queue", "replicas"])
def test_queue_and_gather_gloo(tmp_path, mode, oracle_mod):
    out = str(tmp_path / "rec.npy")
    mp.spawn(_worker, args=(2, _free_port(), mode, out), nprocs=2, join=True)
    tables = np.load(out)
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem("tiny")
    o = oracle_mod.Oracle.from_problem(prob, oracle_mod.score_params())
    mp_ = oracle_mod.mh_preset(3, population=16, generations=2)
    n = prob.cfg.n_spots
    assert tables.shape == (2, n, vdist.REC)
    if mode == "queue":
        pose, sc = o.run(mp_, 42)
        got_pose, got_sc, owner = vdist.assemble(list(tables), n)   # every spot exactly once
        np.testing.assert_array_equal(got_sc, sc.astype(np.float32))
        np.testing.assert_array_equal(got_pose, pose)
        assert set(owner.tolist()) <= {0, 1}
    else:
        runs = [o.run(mp_, 42 + r)[1].astype(np.float32) for r in range(2)]
        _, got_sc = vdist.best_of(list(tables))
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
    rng, times = vdist.warmup_split(lambda: 2.0 if rank == 0 else 1.0, 90, torch.device("cpu"))
    out = [None] * world
    dist.all_gather_object(out, (rng, times))
    if rank == 0:
        np.save(out_path, np.array([list(r) + t for r, t in out]))
    dist.destroy_process_group()


def test_warmup_split_gloo(tmp_path):
    out = str(tmp_path / "split.npy")
    mp.spawn(_warm_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    split = np.load(out)
    assert split.tolist() == [[0, 30, 2.0, 1.0], [30, 90, 2.0, 1.0]]
