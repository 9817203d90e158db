"""Screening sweep: a ligand library docked at every spot of one receptor.

"Given a receptor protein, large libraries of small molecules (ligands) are
explored to search for the structures which best bind to the receptor"
(§1); "a large ligand database is screened against the target
protein over its whole surface simultaneously" (§2.1).

Work units are (ligand, spot chunk).  They are ordered largest ligand first
(longest-processing-time first) with guided chunk sizes, and dealt to the
ranks by the same atomic fetch-add queue as the single-ligand driver
(dist.claim_chunks), mirroring the paper's "dynamic assignment of jobs"
(P:9).  One scoring context per ligand (vs_create) holds that ligand's
per-spot receptor lists; all runs are device-resident (vs_run_async).

Random streams: ligand l uses seed ``ligand_seed(seed, l)``; within a ligand
the Philox counter is keyed by the global spot id, so every (ligand, spot)
result is independent of the rank and chunk that computed it.
"""
from __future__ import annotations

import math
from typing import Sequence

import numpy as np

from . import vs

REC = 10  # ligand id, spot id, score, w, x, y, z, tx, ty, tz


def ligand_seed(seed: int, lig: int) -> int:
    """Distinct 64-bit Philox key per ligand (golden-ratio increment)."""
    return (seed + 0x9E3779B97F4A7C15 * (lig + 1)) & 0xFFFFFFFFFFFFFFFF


def unit_schedule(lig_sizes: Sequence[int], n_spots: int, n_ranks: int, min_chunk: int = 8):
    """(ligand, a, b) units: ligands by decreasing size; each ligand's spots cut into guided chunks
    (large first).  Every (ligand, spot) appears exactly once."""
    order = sorted(range(len(lig_sizes)), key=lambda i: (-lig_sizes[i], i))
    out = []
    for li in order:
        a = 0
        while a < n_spots:
            rem = n_spots - a
            c = rem if n_ranks <= 1 else max(min_chunk, math.ceil(rem / (2 * n_ranks)))
            c = min(c, rem)
            out.append((li, a, a + c))
            a += c
    return out


class Screen:
    """Per-rank state of a screening sweep on one GPU."""

    def __init__(self, rec, spots, ligands, sp: vs.ScoreParams, mp: vs.MHParams, seed: int, device: int = 0):
        self.rec, self.spots, self.ligands = rec, np.ascontiguousarray(spots, np.float32), ligands
        self.sp, self.mp, self.seed, self.device = sp, mp, seed, device
        self.ctx: dict[int, vs.Context] = {}
        self.done: list[tuple[int, int, int]] = []
        self.timing = 0   # vs_set_timing flags given to every context, also those created later (lazily)

    def context(self, li: int) -> vs.Context:
        if li not in self.ctx:
            L = self.ligands[li]
            self.ctx[li] = vs.Context(self.rec.xyz, self.rec.q, self.rec.type, L.xyz, L.q, L.type, self.spots,
                                      self.sp, self.device)
            if self.timing:
                self.ctx[li].set_timing(self.timing)
        return self.ctx[li]

    def set_timing(self, flags: int) -> None:
        self.timing = flags
        for c in self.ctx.values():
            c.set_timing(flags)

    def prepare(self, ligs: Sequence[int]) -> None:
        for li in ligs:
            self.context(li)

    def run_unit(self, li: int, a: int, b: int, pose_out, score_out, stream=None) -> None:
        """vs_run_async for spots [a, b) of ligand li into device tensors pose_out [b-a, 7], score_out [b-a]."""
        ids = np.arange(a, b, dtype=np.int32)
        self.context(li).run_async(self.mp, ligand_seed(self.seed, li), ids, pose_out, score_out, stream)
        self.done.append((li, a, b))

    def stats(self) -> dict:
        tot: dict = {}
        for c in self.ctx.values():
            for k, v in c.stats().items():
                tot[k] = tot.get(k, 0) + v
        return tot

    def reset_stats(self) -> None:
        for c in self.ctx.values():
            c.reset_stats()

    def close(self) -> None:
        for c in self.ctx.values():
            c.close()
        self.ctx.clear()
