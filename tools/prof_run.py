#!/usr/bin/env python
"""Profiling driver: one vs_run of a config for ncu, e.g.

  VS_GRAPHS=0 ncu --set full -k regex:cell_pair_kernel -c 2 -o gpurun_out/pair python tools/prof_run.py --generations 1
  ncu --graph-profiling graph --metrics ... python tools/prof_run.py --generations 10 --graph
      (--graph: a direct run, a captured run, then one replay of the CUDA graph -- the in-run workload of the bench,
       all spot-group streams concurrent -- which ncu profiles as one workload)
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="medium")
    ap.add_argument("--preset", type=int, default=3)
    ap.add_argument("--generations", type=int, default=1)
    ap.add_argument("--score-poses", type=int, default=0, help="also score N random poses via vs_score_poses")
    ap.add_argument("--spots", type=int, default=0, help="run only the first N spots (0: all)")
    ap.add_argument("--splits", type=int, default=0, help="vs_score_params.list_splits (0: the context default)")
    ap.add_argument("--graph", action="store_true", help="direct run, captured run, then one graph replay")
    ap.add_argument("--replay-only", action="store_true",
                    help="with --graph: cudaProfilerStart/Stop around the replay (ncu --profile-from-start off)")
    args = ap.parse_args()
    import torch
    from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
    prob = synth.make_problem(args.config)
    g = vs.Context.from_problem(prob, vs.score_params(**({"list_splits": args.splits} if args.splits else {})), device=0)
    mp = vs.mh_preset(args.preset, population=prob.cfg.population, generations=args.generations)
    import numpy as np
    ids = np.arange(args.spots, dtype=np.int32) if args.spots else None
    g.run(mp, 42, ids)
    if args.graph:
        g.run(mp, 42, ids)     # captured
        torch.cuda.synchronize()
        if args.replay_only:   # ncu --profile-from-start off: only the replayed graph is profiled
            torch.cuda.profiler.start()
        g.run(mp, 42, ids)     # replayed
        torch.cuda.synchronize()
        if args.replay_only:
            torch.cuda.profiler.stop()
    if args.score_poses:
        spot, q, t = synth.make_poses(args.score_poses, prob.cfg.n_spots, 3.0, seed=1)
        g.score_poses(spot, q, t)
    torch.cuda.synchronize()
    print(g.stats())


if __name__ == "__main__":
    main()
