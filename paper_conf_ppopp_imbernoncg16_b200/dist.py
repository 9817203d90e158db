"""Multi-GPU plumbing: one process per GPU, spots dealt by a dynamic queue, one gather.

Spots are independent (§3.1) and independent executions need
no communication; "the final solution is chosen from all independent
executions" (§3.3).  The paper balances heterogeneous GPUs with a
warm-up-measured static split (Eq. 1); its abstract asks for a
"dynamic assignment of jobs" (P:9).  Here:

  * strong scaling: the spot list is cut into a guided schedule of chunks
    (large first, small last, so the tail is short); ranks claim chunk
    indices with an atomic fetch-add on the torch.distributed store, run
    ``vs_run`` on each claimed chunk, and rank 0 gathers the per-spot bests;
  * weak scaling: every rank runs the whole workload as an independent
    metaheuristic execution with its own seed, and rank 0 keeps the
    best of all executions per spot.

The RNG is keyed by the global spot id, so a spot's result does not depend
on which rank or chunk ran it.  The only collectives are one all-gather of
per-rank counts and one gather of fixed-size records {spot, score, pose[7]}.
"""
from __future__ import annotations

import math
from typing import Callable, Sequence

import numpy as np
import torch
import torch.distributed as dist

REC = 9  # spot id, score, w, x, y, z, tx, ty, tz


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


def claim_chunks(store, key: str, schedule: Sequence[tuple[int, int]],
                 work: Callable[[int, int], None]) -> list[int]:
    """Claim chunk indices from the shared counter until the schedule is exhausted."""
    done = []
    while True:
        i = int(store.add(key, 1)) - 1
        if i >= len(schedule):
            return done
        a, b = schedule[i]
        work(a, b)
        done.append(i)


def pack(spot_ids: np.ndarray, pose: np.ndarray, score: np.ndarray) -> np.ndarray:
    rec = np.zeros((len(spot_ids), REC), np.float32)
    rec[:, 0] = spot_ids
    rec[:, 1] = score
    rec[:, 2:] = pose
    return rec


def gather_records(rec: torch.Tensor, device: torch.device) -> torch.Tensor | None:
    """Gather variable-length [n, REC] float32 records to rank 0 (one all-gather of counts,
    one gather of padded records).  Returns the concatenation on rank 0, None elsewhere."""
    world = dist.get_world_size()
    rank = dist.get_rank()
    n = torch.tensor([rec.shape[0]], dtype=torch.int64, device=device)
    counts = [torch.zeros_like(n) for _ in range(world)]
    dist.all_gather(counts, n)
    counts = [int(c.item()) for c in counts]
    mx = max(max(counts), 1)
    pad = torch.full((mx, REC), float("nan"), dtype=torch.float32, device=device)
    pad[: rec.shape[0]] = rec.to(device)
    bufs = [torch.empty_like(pad) for _ in range(world)] if rank == 0 else None
    dist.gather(pad, bufs, dst=0)
    if rank != 0:
        return None
    return torch.cat([b[:c] for b, c in zip(bufs, counts)])


def best_per_spot(records: np.ndarray, n_spots: int) -> tuple[np.ndarray, np.ndarray]:
    """Best (lowest score; ties -> first record) per spot id; NaN score where a spot is missing."""
    score = np.full(n_spots, np.nan, np.float32)
    pose = np.full((n_spots, 7), np.nan, np.float32)
    for r in records:
        s = int(r[0])
        if np.isnan(score[s]) or r[1] < score[s]:
            score[s] = r[1]
            pose[s] = r[2:]
    return pose, score
