#!/usr/bin/env python
"""Strong-scaling predictor on one GPU: device time of vs_run over the first n spots of a config.

T(n) for n = n_spots / N approximates one rank's time at N GPUs when spots are dealt evenly, so
T(n_spots) / (N T(n_spots / N)) is the best strong-scaling efficiency the per-GPU fill allows.

  python tools/spot_scaling.py --config medium --reps 3
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="medium")
    ap.add_argument("--preset", type=int, default=3)
    ap.add_argument("--generations", type=int, default=None)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--ranks", default="1,2,4,8")
    ap.add_argument("--spots", default=None, help="explicit spot counts instead of n_spots / ranks")
    ap.add_argument("--splits", type=int, default=1, help="vs_score_params.list_splits")
    args = ap.parse_args()
    import numpy as np
    import torch
    from paper_conf_ppopp_imbernoncg16_b200 import synth, vs
    prob = synth.make_problem(args.config)
    G = prob.cfg.generations if args.generations is None else args.generations
    ctx = vs.Context.from_problem(prob, vs.score_params(list_splits=args.splits), device=0)
    mp = vs.mh_preset(args.preset, population=prob.cfg.population, generations=G)
    st = torch.cuda.Stream()
    ns = prob.cfg.n_spots
    out = {}
    counts = ([(ns + N - 1) // N for N in map(int, args.ranks.split(","))] if args.spots is None
              else [int(x) for x in args.spots.split(",")])
    for n in counts:
        N = ns / n
        ids = np.arange(n, dtype=np.int32)
        bp = torch.empty((n, 7), device="cuda")
        bs = torch.empty(n, device="cuda")
        for _ in range(2):      # second identical call captures the graph
            ctx.run_async(mp, 42, ids, bp, bs, st)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for _ in range(args.reps):
            ctx.run_async(mp, 42, ids, bp, bs, st)
        e1.record(st)
        torch.cuda.synchronize()
        out[n] = {"N": N, "ms": e0.elapsed_time(e1) / args.reps}
    if ns in out:
        t1 = out[ns]["ms"]
        for n, v in out.items():
            v["eff"] = t1 / (v["N"] * v["ms"])
    print(json.dumps({"config": args.config, "generations": G, "list_splits": args.splits, "T": out}))
    ctx.close()


if __name__ == "__main__":
    main()
