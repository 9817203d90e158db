"""compute-sanitizer driver: scoring + vs_run on small problems, both cutoff modes, every code path of the pair
kernel that the round-2 build added.

6 spots (one spot group; latency-bound: KP 1 chunks, coarse item sort) and 24 spots (spot-group streams, PDL chains),
canonical list splits S = 1, 2, 4, the census and launch-interval instrumentation, vs_run_async / vs_score_poses_device
on a caller stream; VS_GRAPHS=0 so the sanitizer sees plain launches.  Contexts are created and destroyed back to back
(device memory cache reuse)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
import torch
from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
for n_spots in (6, 24):
    prob = synth.make_custom(1200, 45, n_spots, seed=3)
    for cutoff in (12.0, 0.0):
        for S in (1, 2, 4):
            ctx = vs.Context.from_problem(prob, vs.score_params(cutoff=cutoff, list_splits=S))
            spot, q, t = synth.make_poses(200, n_spots, 3.0, seed=1)
            s = ctx.score_poses(spot, q, t)
            ctx.set_timing(vs.TIMING_KERNEL | vs.TIMING_CENSUS | vs.TIMING_EVENTS)
            pose, best = ctx.run(vs.mh_preset(3, population=40, generations=2), 7)
            ctx.set_timing(0)
            pose, best = ctx.run(vs.mh_preset(4, population=64, ls_neighbours=3), 7)
            st = torch.cuda.Stream()
            d = [torch.from_numpy(x).cuda() for x in (spot, q, t)]
            out = torch.empty(len(spot), device="cuda")
            bp = torch.empty((n_spots, 7), device="cuda")
            bs = torch.empty(n_spots, device="cuda")
            ctx.score_poses_device(*d, out, st)
            ctx.run_async(vs.mh_preset(3, population=16, generations=1), 3, None, bp, bs, st)
            st.synchronize()
            ctx.stats()
            ctx.close()
print("ok", float(s.sum()), float(best.sum()))
