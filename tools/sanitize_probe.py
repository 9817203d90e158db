import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np
from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
prob = synth.make_custom(1200, 45, 6, seed=3)
for cutoff in (12.0, 0.0):
    ctx = vs.Context.from_problem(prob, vs.score_params(cutoff=cutoff))
    spot, q, t = synth.make_poses(200, 6, 3.0, seed=1)
    s = ctx.score_poses(spot, q, t)
    pose, best = ctx.run(vs.mh_preset(3, population=40, generations=2), 7)
    pose, best = ctx.run(vs.mh_preset(4, population=64, ls_neighbours=3), 7)
    ctx.close()
print("ok", float(s.sum()), float(best.sum()))
