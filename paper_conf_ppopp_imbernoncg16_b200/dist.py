"""Multi-GPU plumbing: one process per GPU, spots dealt by a dynamic queue, one gather.

Spots are independent (§3.1) and independent executions need no
communication; "the final solution is chosen from all independent executions"
(§3.3).  The paper's abstract asks for a "dynamic assignment of jobs to
heterogeneous resources" (P:9); its heterogeneous scheduler is a warm-up
measured static split (Eq. 1).  Here:

  * queue (default): the spots are cut into chunks; ranks claim chunk indices
    with an atomic fetch-add on the torch.distributed store (``ChunkQueue``)
    and keep up to ``slots`` chunks in flight (``run_dynamic``): a rank that
    finishes early claims more, so faster GPUs take more spots;
  * warmup: Eq. (1) -- every rank times a few metaheuristic generations, the
    times are gathered, Percent = t / t_slowest, and each rank takes a
    contiguous share of the spots proportional to 1 / Percent (``warmup_split``);
  * replicas: every rank runs the whole workload as an independent execution
    with its own seed; rank 0 keeps the best per spot.

The RNG is keyed by the global spot id, so a spot's result does not depend on
which rank or chunk ran it.  The only data-path collective is ONE fixed-size
gather of per-spot records [n_spots, REC] (NaN where the rank did not run the
spot): ``gather_fixed``, then ``assemble`` on rank 0.
"""
from __future__ import annotations

import math
from typing import Callable, Sequence

import numpy as np
import torch
import torch.distributed as dist

REC = 9  # spot id, score, w, x, y, z, tx, ty, tz


# ---------------------------------------------------------------- schedules
def equal_chunks(n_items: int, n_chunks: int) -> list[tuple[int, int]]:
    """n_chunks contiguous ranges of near-equal size covering 0..n_items once (empty ranges dropped)."""
    out = []
    for i in range(max(1, n_chunks)):
        a, b = n_items * i // max(1, n_chunks), n_items * (i + 1) // max(1, n_chunks)
        if b > a:
            out.append((a, b))
    return out


def chunk_schedule(n_items: int, n_ranks: int, min_chunk: int = 1) -> list[tuple[int, int]]:
    """Guided self-scheduling: chunk = max(min_chunk, ceil(remaining / (2 n_ranks)))."""
    out, start = [], 0
    if n_ranks <= 1:
        return [(0, n_items)] if n_items > 0 else []
    while start < n_items:
        rem = n_items - start
        c = max(min_chunk, math.ceil(rem / (2 * n_ranks)))
        c = min(c, rem)
        out.append((start, start + c))
        start += c
    return out


class ChunkQueue:
    """Chunk indices handed out once each: an atomic fetch-add on the c10d store shared by the ranks
    (``store``), or a local counter for a single process (``store=None``)."""

    def __init__(self, store, key: str, n: int):
        self.store, self.key, self.n, self.local = store, key, n, 0

    def claim(self) -> int | None:
        if self.store is None:
            i = self.local
            self.local += 1
        else:
            i = int(self.store.add(self.key, 1)) - 1
        return i if i < self.n else None


def claim_chunks(store, key: str, schedule: Sequence[tuple[int, int]],
                 work: Callable[[int, int], None]) -> list[int]:
    """Claim chunk indices from the shared counter until the schedule is exhausted (one at a time)."""
    q = ChunkQueue(store, key, len(schedule))
    done = []
    while (i := q.claim()) is not None:
        work(*schedule[i])
        done.append(i)
    return done


def run_dynamic(queue: ChunkQueue, schedule: Sequence[tuple[int, int]], slots: int,
                launch: Callable[[int, int, int], None], wait: Callable[[int], None]) -> list[int]:
    """Keep up to ``slots`` chunks in flight: whenever a slot is free, claim the next chunk and
    ``launch(slot, a, b)`` it (asynchronous); ``wait(slot)`` blocks until that slot's chunk is done.
    Returns the chunk indices this process ran, in claim order."""
    done, busy = [], [False] * max(1, slots)
    s = 0
    while True:
        if busy[s]:
            wait(s)
            busy[s] = False
        i = queue.claim()
        if i is None:
            break
        launch(s, *schedule[i])
        busy[s] = True
        done.append(i)
        s = (s + 1) % len(busy)
    for k in range(len(busy)):
        if busy[k]:
            wait(k)
    return done


# ---------------------------------------------------------------- records
def pack(spot_ids: np.ndarray, pose: np.ndarray, score: np.ndarray) -> np.ndarray:
    rec = np.zeros((len(spot_ids), REC), np.float32)
    rec[:, 0] = spot_ids
    rec[:, 1] = score
    rec[:, 2:] = pose
    return rec


def empty_records(n_spots: int, device) -> torch.Tensor:
    """[n_spots, REC] float32, NaN-filled: row s is filled by the rank that ran spot s."""
    return torch.full((n_spots, REC), float("nan"), dtype=torch.float32, device=device)


def fill_records(rec: torch.Tensor, a: int, b: int, pose: torch.Tensor, score: torch.Tensor) -> None:
    """Rows a..b of the fixed-size record table from a chunk's device outputs (pose [b-a, 7], score [b-a])."""
    rec[a:b, 0] = torch.arange(a, b, dtype=torch.float32, device=rec.device)
    rec[a:b, 1] = score
    rec[a:b, 2:] = pose


def gather_fixed(rec: torch.Tensor, device) -> list[torch.Tensor] | None:
    """ONE gather of every rank's fixed-size [n, REC] record table to rank 0 (NCCL over NVLink, or gloo).
    Returns the per-rank tables on rank 0, None elsewhere; a single process returns [rec]."""
    if not dist.is_initialized() or dist.get_world_size() == 1:
        return [rec]
    t = rec.to(device)
    bufs = [torch.empty_like(t) for _ in range(dist.get_world_size())] if dist.get_rank() == 0 else None
    dist.gather(t, bufs, dst=0)
    return bufs


def assemble(tables: Sequence[np.ndarray], n_spots: int) -> tuple[np.ndarray, np.ndarray, np.ndarray]:
    """Merge the per-rank record tables: (pose [n, 7], score [n], owner rank [n]).  Every spot must have been run
    by exactly one rank (raises otherwise)."""
    owner = np.full(n_spots, -1, np.int64)
    pose = np.full((n_spots, 7), np.nan, np.float32)
    score = np.full(n_spots, np.nan, np.float32)
    for r, t in enumerate(tables):
        t = np.asarray(t)
        have = ~np.isnan(t[:, 0])
        if np.any(have & (owner >= 0)):
            raise RuntimeError(f"spots run twice (rank {r}): {np.nonzero(have & (owner >= 0))[0][:8]}")
        if np.any(t[have, 0] != np.nonzero(have)[0]):
            raise RuntimeError("record table rows out of place")
        owner[have] = r
        score[have] = t[have, 1]
        pose[have] = t[have, 2:]
    if np.any(owner < 0):
        raise RuntimeError(f"spots never run: {np.nonzero(owner < 0)[0][:8]}")
    return pose, score, owner


def best_of(tables: Sequence[np.ndarray]) -> tuple[np.ndarray, np.ndarray]:
    """Replicas: the best (lowest score; ties -> lowest rank) of every rank's full table, per spot."""
    t = np.stack([np.asarray(x) for x in tables])            # [ranks, n, REC]
    k = np.argmin(np.where(np.isnan(t[:, :, 1]), np.inf, t[:, :, 1]), axis=0)
    rows = t[k, np.arange(t.shape[1])]
    return rows[:, 2:], rows[:, 1]


def best_per_spot(records: np.ndarray, n_spots: int) -> tuple[np.ndarray, np.ndarray]:
    """Best (lowest score; ties -> first record) per spot id of a list of records; NaN where a spot is missing."""
    score = np.full(n_spots, np.nan, np.float32)
    pose = np.full((n_spots, 7), np.nan, np.float32)
    for r in records:
        if np.isnan(r[0]):
            continue
        s = int(r[0])
        if np.isnan(score[s]) or r[1] < score[s]:
            score[s] = r[1]
            pose[s] = r[2:]
    return pose, score


# ---------------------------------------------------------------- heterogeneity-aware static split (N2)
def percent_from_times(times: Sequence[float]) -> list[float]:
    """Eq. (1): Percent = Ex.time(actual GPU) / Ex.time(slowest GPU)."""
    slowest = max(times)
    return [t / slowest for t in times]


def shares_from_percent(percent: Sequence[float], n_items: int) -> list[tuple[int, int]]:
    """Each rank's contiguous item range, sized proportional to its speed 1/Percent ("each
    OpenMP thread then calculates the number of conformations it is in charge of"; reading R27:
    share proportional to 1/Percent).  Largest-remainder rounding; ranges cover 0..n_items once."""
    speed = [1.0 / max(p, 1e-12) for p in percent]
    tot = sum(speed)
    raw = [n_items * s / tot for s in speed]
    cnt = [int(math.floor(x)) for x in raw]
    rem = n_items - sum(cnt)
    for i in sorted(range(len(raw)), key=lambda i: raw[i] - cnt[i], reverse=True)[:rem]:
        cnt[i] += 1
    out, a = [], 0
    for c in cnt:
        out.append((a, a + c))
        a += c
    return out


def warmup_split(warmup: Callable[[], float], n_items: int, device) -> tuple[tuple[int, int], list[float]]:
    """Warm-up phase of PAPER.md §3.3: every rank times a few metaheuristic iterations
    (``warmup`` returns seconds), the times are gathered (one all-gather), Percent = t / t_slowest
    (Eq. 1) and each rank takes a share of the items proportional to its speed.  Returns this rank's
    range and the measured times."""
    world, rank = dist.get_world_size(), dist.get_rank()
    t = torch.tensor([float(warmup())], dtype=torch.float64, device=device)
    ts = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(ts, t)
    times = [float(x.item()) for x in ts]
    return shares_from_percent(percent_from_times(times), n_items)[rank], times
