"""compute-sanitizer driver: scoring + vs_run on small problems, both cutoff modes.

6 spots (one spot group, list splits) and 24 spots (three spot-group streams, PDL chains); VS_GRAPHS=0 so the
sanitizer sees plain launches.  Contexts are created and destroyed back to back (device memory cache reuse)."""
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
for n_spots in (6, 24):
    prob = synth.make_custom(1200, 45, n_spots, seed=3)
    for cutoff in (12.0, 0.0):
        ctx = vs.Context.from_problem(prob, vs.score_params(cutoff=cutoff))
        spot, q, t = synth.make_poses(200, n_spots, 3.0, seed=1)
        s = ctx.score_poses(spot, q, t)
        pose, best = ctx.run(vs.mh_preset(3, population=40, generations=2), 7)
        pose, best = ctx.run(vs.mh_preset(4, population=64, ls_neighbours=3), 7)
        ctx.close()
print("ok", float(s.sum()), float(best.sum()))
