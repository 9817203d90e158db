#!/usr/bin/env python
"""Benchmark of the virtual-screening hot path (one JSON line on rank 0).

A step = one full metaheuristic run (Algorithm 1, preset
M3 of Table 4 P:232-237 with the config's population / generations) over
every spot of the configured synthetic workload: pose generation, scoring of
every individual and local-search proposal, selection, on device.

  python bench.py [--gpus N --steps K --warmup W] [--config medium] [--preset 3]
  torchrun --nproc-per-node N bench.py --gpus N ...        (one process per GPU, NCCL)
  python bench.py --impl reference ...                      (the fp64 CPU oracle arm)

metric: atom-pair interactions/s (BASELINE.json); the workload's pairs of a
scored pose = n_lig x the receptor atoms of its spot: the
whole receptor in all-pairs mode, the spot's cutoff list in cutoff mode -- the
same count the oracle arm reports.  `value` is workload pairs / s (a fixed
multiple of scored poses / s, also reported).  The pair kernel evaluates fewer
pairs in cutoff mode (cell culling skips list atoms provably beyond rc of a
chunk); `roofline.achieved` is the evaluated-pair rate against the FP32 issue
roofline, i.e. the kernel's hardware efficiency.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

# One vs_run drives up to 9 streams per context (main + spot groups): give them their own hardware work queues
# (the default 8 aliases streams onto shared queues; measured: context create / destroy costs become erratic,
# up to hundreds of ms).  Must be set before the CUDA context exists.
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "atom-pair interactions/s and scored poses/s at 1/2/4/8 B200; % FP32 roofline"
N_SM = 148
LANES = 128
OPS_CUTOFF, OPS_ALLPAIRS = 25, 20   # canonical issue slots per pair


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="medium")
    ap.add_argument("--preset", type=int, default=3)
    ap.add_argument("--generations", type=int, default=None, help="override the config's G")
    ap.add_argument("--ls-neighbours", type=int, default=1, help="K proposals per Improve step (N4)")
    ap.add_argument("--mode", choices=["cutoff", "allpairs"], default="cutoff")
    ap.add_argument("--scaling", choices=["weak", "strong"], default="weak")
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-clocks", action="store_true")
    ap.add_argument("--no-micro", action="store_true")
    ap.add_argument("--micro-poses", type=int, default=1 << 20)
    return ap.parse_args()


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int, enabled: bool = True):
        self.idx = gpu_index
        self.proc = None
        self.lines: list[str] = []
        self.enabled = enabled

    def start(self):
        if not self.enabled:
            return
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100", "-i", str(self.idx)],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self) -> dict | None:
        if not self.proc:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = max(mx, float(f[2]))
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": len(sm)}


def cpu_model() -> str:
    """The host CPU model (the oracle timing states the cores and the CPU model)."""
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        return {}


def ncu_traffic(config: str):
    """Per-launch DRAM bytes of the scoring kernel from the committed ncu --set full summary."""
    import glob
    for f in sorted(glob.glob(os.path.join(ROOT, "profiles", "*ncu_summary*.json")), reverse=True):
        try:
            d = json.load(open(f))
            v = d.get("score_kernel", {}).get(config, {}).get("dram_bytes_per_launch")
            if v is not None:
                return v
        except (OSError, ValueError):
            pass
    return None


# ---------------------------------------------------------------- oracle arm / cpu baseline
def oracle_sample(prob, sp_kw, mp_kw, list_len, seed, n_spots_sample: int, generations: int):
    """Time the fp64 oracle (as it stands) on a bounded sample of the workload.

    Returns (seconds, workload pairs in the sample, poses in the sample, threads)."""
    import oracle
    o = oracle.Oracle.from_problem(prob, oracle.score_params(**sp_kw))
    mp = oracle.mh_preset(mp_kw["preset"], population=mp_kw["population"], generations=generations)
    ids = np.arange(n_spots_sample, dtype=np.int32)
    t0 = time.perf_counter()
    o.run(mp, seed, ids)
    dt = time.perf_counter() - t0
    n_lig = len(prob.lig.q)      # the sampled ligand (sweep: ligand 0; cfg.n_lig is per-ligand there)
    poses = o.pairs_evaluated() // (n_lig * prob.cfg.n_rec)
    per_spot = poses // n_spots_sample
    pairs = int(sum(int(list_len[s]) for s in ids)) * n_lig * per_spot
    return dt, pairs, poses, min(n_spots_sample, oracle.get_threads())


def list_lengths_host(prob, cutoff: float, T: float = 3.0):
    """Per-spot list lengths as the library defines them (reach = T sqrt3 + max|l| + rc + 0.01)."""
    if not cutoff > 0:
        return np.full(len(prob.spots), prob.cfg.n_rec, np.int64)
    lig = prob.lig.xyz.astype(np.float64)
    cen = np.float32(lig.mean(0))
    rmax = np.linalg.norm((prob.lig.xyz - cen).astype(np.float64), axis=1).max()
    reach = T * np.sqrt(3) + rmax + cutoff + 0.01
    out = []
    rec = prob.rec.xyz.astype(np.float32)
    for c in prob.spots:
        d = rec - c
        out.append(int(((d * d).sum(1) <= np.float32(reach * reach)).sum()))
    return np.array(out)


def run_reference(args, rank, world):
    """--impl reference: the oracle on the host cores (rank 0 only)."""
    if rank != 0:
        return
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem(args.config)
    cutoff = 12.0 if args.mode == "cutoff" else 0.0
    lens = list_lengths_host(prob, cutoff)
    P = prob.cfg.population
    import oracle
    n_s = max(1, min(prob.cfg.n_spots, oracle.get_threads()))   # OpenMP runs one spot per thread
    G = 2 if args.config in ("medium", "large", "sweep") else min(prob.cfg.generations, 5)
    mp_kw = {"preset": args.preset, "population": P}
    times, pairs, poses, cores = [], 0, 0, 1
    for i in range(args.warmup + args.steps):
        dt, pr, po, cores = oracle_sample(prob, {"cutoff": cutoff}, mp_kw, lens, args.seed, n_s, G)
        if i >= args.warmup:
            times.append(dt)
            pairs, poses = pr, po
    ms = 1e3 * statistics.mean(times)
    val = pairs / (ms * 1e-3)
    sample = f"oracle vso_run on {n_s} spot(s) x {G} generations (P={P}, preset M{args.preset}) of {args.config}"
    print(json.dumps({
        "metric": METRIC, "value": val, "unit": "pairs/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": args.scaling,
        "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
        "config": {"workload": args.config, "preset": f"M{args.preset}", "mode": args.mode, "sample": sample},
        "poses_per_s": poses / (ms * 1e-3),
        "cpu_baseline": {"value": val, "unit": "pairs/s", "cores": cores, "cpu": cpu_model(), "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": val, "unit": "pairs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ---------------------------------------------------------------- our arm
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_imbernoncg16_b200 import dist as vdist
    from paper_conf_ppopp_imbernoncg16_b200 import screen, synth, vs

    # one process per GPU; VS_BENCH_BACKEND=gloo (CPU collectives, ranks may share a GPU) exercises the
    # multi-rank path on a single-GPU box
    backend = os.environ.get("VS_BENCH_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cdev = dev if backend == "nccl" else torch.device("cpu")   # where collective tensors live
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    prob = synth.make_problem(args.config)
    cfg = prob.cfg
    G = cfg.generations if args.generations is None else args.generations
    cutoff = 12.0 if args.mode == "cutoff" else 0.0
    sp = vs.score_params(cutoff=cutoff)
    mp = vs.mh_preset(args.preset, population=cfg.population, generations=G, ls_neighbours=args.ls_neighbours)
    sweep = cfg.n_ligands > 1
    n_spots = cfg.n_spots
    stream = torch.cuda.Stream(device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # > 126 MB L2
    store = dist.distributed_c10d._get_default_store() if world > 1 else None
    if sweep:
        # screening sweep (N1): units (ligand, spot chunk), largest ligands first, dynamic queue
        scr = screen.Screen(prob.rec, prob.spots, prob.ligands, sp, mp, args.seed, device=local)
        sizes = [len(m.q) for m in prob.ligands]
        units = screen.unit_schedule(sizes, n_spots, world, min_chunk=16)
        if world == 1:
            scr.prepare(range(len(prob.ligands)))
        res_pose = torch.empty((len(prob.ligands), n_spots, 7), dtype=torch.float32, device=dev)
        res_score = torch.empty((len(prob.ligands), n_spots), dtype=torch.float32, device=dev)
        ctx = None
    else:
        ctx = vs.Context.from_problem(prob, sp, device=local)
        best_pose = torch.empty((n_spots, 7), dtype=torch.float32, device=dev)
        best_score = torch.empty(n_spots, dtype=torch.float32, device=dev)
        schedule = vdist.chunk_schedule(n_spots, world, min_chunk=4) if args.scaling == "strong" else None

    class Work:
        """stats / timing over every context this rank uses"""
        def stats(self):
            return scr.stats() if sweep else ctx.stats()

        def reset_stats(self):
            scr.reset_stats() if sweep else ctx.reset_stats()

        def set_timing(self, on):
            for c in (scr.ctx.values() if sweep else [ctx]):
                c.set_timing(on)

    work_obj = Work()

    def step(i: int):
        """One whole-job pass: returns this rank's records (device tensor) for the gather."""
        with torch.cuda.stream(stream):
            flush.zero_()
            if sweep:
                parts = []

                def unit(k0, k1):
                    for li, a, b in units[k0:k1]:
                        scr.run_unit(li, a, b, res_pose[li, a:b], res_score[li, a:b], stream)
                        ids = torch.arange(a, b, dtype=torch.float32, device=dev)
                        lid = torch.full_like(ids, float(li))
                        parts.append(torch.cat([lid[:, None], ids[:, None], res_score[li, a:b, None],
                                                res_pose[li, a:b]], 1))

                if world > 1:
                    vdist.claim_chunks(store, f"s{i}", [(k, k + 1) for k in range(len(units))], unit)
                else:
                    unit(0, len(units))
                rec = torch.cat(parts) if parts else torch.zeros((0, screen.REC), device=dev)
            elif args.scaling == "weak":
                ctx.run_async(mp, args.seed + rank, None, best_pose, best_score, stream)
                ids = torch.arange(n_spots, dtype=torch.float32, device=dev)
                rec = torch.cat([ids[:, None], best_score[:, None], best_pose], 1)
            else:
                parts = []

                def work(a, b):
                    ctx.run_async(mp, args.seed, np.arange(a, b, dtype=np.int32), best_pose[a:b], best_score[a:b],
                                  stream)
                    ids = torch.arange(a, b, dtype=torch.float32, device=dev)
                    parts.append(torch.cat([ids[:, None], best_score[a:b, None], best_pose[a:b]], 1))

                if world > 1:
                    vdist.claim_chunks(store, f"q{i}", schedule, work)
                else:
                    for a, b in schedule:
                        work(a, b)
                rec = torch.cat(parts) if parts else torch.zeros((0, vdist.REC), device=dev)
            if world > 1:
                vdist.gather_records(rec, cdev)
        return rec

    for i in range(args.warmup):
        step(-1 - i)
    torch.cuda.synchronize(dev)
    work_obj.reset_stats()
    work_obj.set_timing(True)
    clocks = ClockSampler(local, enabled=(rank == 0 and not args.no_clocks))
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    clocks.start()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for i in range(args.steps):
        step(i)
    e1.record(stream)
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms_rank = e0.elapsed_time(e1)
    st = work_obj.stats()
    work_obj.set_timing(False)
    # whole-job totals and max-over-ranks time
    tot = torch.tensor([st["pairs"], st["poses_scored"], st["kernel_launches"], st["pairs_evaluated"]],
                       dtype=torch.float64, device=cdev)
    tmax = torch.tensor([ms_rank], dtype=torch.float64, device=cdev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    pairs, poses, launches, pairs_ev = (float(x) for x in tot.tolist())
    ms = float(tmax.item())
    value = pairs / (ms * 1e-3)
    # dominant kernel (the pair kernel, ~94 % of device time): evaluated pairs / device time.  vs_run
    # overlaps the scoring launches of up to 4 spot groups on separate streams, so per-launch event
    # times overlap; the conservative figure is this rank's evaluated pairs over its whole device-timed
    # step (which also contains the item sort, the per-pose sums and the population kernels).
    achieved = st["pairs_evaluated"] / (ms_rank * 1e-3) / 1e9      # Gpairs/s on this rank
    pk = peaks()
    f_max = pk.get("sm_max_mhz", 1965.0)
    ops = OPS_CUTOFF if cutoff > 0 else OPS_ALLPAIRS
    peak = N_SM * LANES * f_max * 1e6 / ops / 1e9
    roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "Gpairs/s", "frac": achieved / peak,
            "traffic": ncu_traffic(args.config),
            "peak_basis": f"{N_SM} SMs x {LANES} FP32 lanes x {f_max:.0f} MHz (MEASURED_PEAKS sm_max) / "
                          f"{ops} canonical issue slots per pair",
            "achieved_basis": "pairs evaluated by the pair kernel per step / device step time (CUDA events on "
                              "the launching stream; per-rank kernel figure)",
            "workload_frac": st["pairs"] / (ms_rank * 1e-3) / 1e9 / peak,
            "cull_ratio": st["pairs_evaluated"] / max(1.0, st["pairs"]),
            "score_launches": st["score_launches"], "score_launch_ms_sum": st["score_ms"],
            "pairs_evaluated_per_launch": st["pairs_evaluated"] / max(1, st["score_launches"])}
    if clk:
        roof["frac_at_run_clock"] = achieved / (N_SM * LANES * clk["sm_mhz"] * 1e6 / ops / 1e9)

    # ---- end to end through the public C ABI with host buffers (vs_create + vs_run + results to host)
    e2e = None
    if not args.no_e2e:
        import torch as _t
        pin = lambda a: _t.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
        ligs = prob.ligands if sweep else [prob.lig]
        rec_h = [pin(x) for x in (prob.rec.xyz, prob.rec.q, prob.rec.type)]
        lig_h = [[pin(x) for x in (L.xyz, L.q, L.type)] for L in ligs]
        spot_h = pin(prob.spots)
        n_e2e = args.e2e_steps if args.e2e_steps is not None else (1 if sweep else max(1, min(args.steps, 2)))
        e2e_ctx_stats = []
        # one untimed warm-up pass (ligand 0): the first context of the process pays cudaMalloc for the
        # device memory cache; later contexts reuse its blocks
        c2 = vs.Context(*rec_h, *lig_h[0], spot_h, sp=sp, device=local)
        c2.run(mp, args.seed + rank, None)
        c2.close()
        torch.cuda.synchronize(local)
        if world > 1:
            dist.barrier()
        t0 = time.perf_counter()
        parts_ms = {"create": 0.0, "run": 0.0, "stats": 0.0, "destroy": 0.0}
        for i in range(n_e2e):
            # sweep: this rank's share of the ligands (static round robin), one context per ligand
            for li in (range(rank, len(ligs), world) if sweep else [0]):
                ta = time.perf_counter()
                c2 = vs.Context(*rec_h, *lig_h[li], spot_h, sp=sp, device=local)
                tb = time.perf_counter()
                c2.run(mp, (screen.ligand_seed(args.seed, li) if sweep else args.seed + rank), None)
                tc = time.perf_counter()
                e2e_ctx_stats.append(c2.stats())
                tcs = time.perf_counter()
                c2.close()
                td = time.perf_counter()
                parts_ms["create"] += 1e3 * (tb - ta)
                parts_ms["run"] += 1e3 * (tc - tb)
                parts_ms["stats"] += 1e3 * (tcs - tc)
                parts_ms["destroy"] += 1e3 * (td - tcs)
        dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=cdev)
        e2e_pairs = torch.tensor([sum(s["pairs"] for s in e2e_ctx_stats)], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(dt, op=dist.ReduceOp.MAX)
            dist.all_reduce(e2e_pairs, op=dist.ReduceOp.SUM)
        h2d = sum(a.nbytes for a in rec_h) + spot_h.nbytes + sum(a.nbytes for L in lig_h for a in L)
        d2h = n_spots * 8 * 4 * len(ligs)
        e2e = {"value": float(e2e_pairs.item()) / float(dt.item()), "unit": "pairs/s", "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "steps": n_e2e,
               "ms_per_step_parts": {k: v / n_e2e for k, v in parts_ms.items()},
               "what": "vs_create (receptor/ligand/spot upload + per-spot list build) + vs_run (host spot ids) + "
                       "best poses/scores to host, wall clock, after one untimed warm-up pass" + (", per ligand of the library" if sweep else "")}

    # ---- scoring-kernel microbenchmark: one vs_score_poses_device batch of device-resident poses
    micro = None
    if sweep:                       # the microbenchmark uses the first ligand's context
        ctx = scr.context(0)
    if not args.no_micro:
        n_micro = args.micro_poses
        spot_h, q_h, t_h = synth.make_poses(n_micro, n_spots, 3.0, seed=7)
        spot_d = torch.from_numpy(spot_h).to(dev)
        q_d, t_d = torch.from_numpy(q_h).to(dev), torch.from_numpy(t_h).to(dev)
        out_d = torch.empty(n_micro, dtype=torch.float32, device=dev)
        with torch.cuda.stream(stream):
            for _ in range(2):
                ctx.score_poses_device(spot_d, q_d, t_d, out_d, stream)
            torch.cuda.synchronize(dev)
            ctx.reset_stats()
            ctx.set_timing(True)
            m0, m1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 3
            m0.record(stream)
            for _ in range(reps):
                ctx.score_poses_device(spot_d, q_d, t_d, out_d, stream)
            m1.record(stream)
        torch.cuda.synchronize(dev)
        ms_m = m0.elapsed_time(m1) / reps
        stm = ctx.stats()
        ctx.set_timing(False)
        pairs_m = stm["pairs"] / reps
        ach_m = stm["pairs_evaluated"] / (stm["score_ms"] * 1e-3) / 1e9
        micro = {"what": f"vs_score_poses_device, {n_micro} device-resident random in-region poses over "
                         f"{n_spots} spots (validate + bucket by spot + score), mean of {reps}",
                 "ms": ms_m, "pairs_per_s": pairs_m / (ms_m * 1e-3), "poses_per_s": n_micro / (ms_m * 1e-3),
                 "score_kernel_gpairs_per_s": ach_m, "frac": ach_m / peak}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        lens = ctx.list_lengths()
        if sweep:
            prob.lig = prob.ligands[0]
            lens = list_lengths_host(prob, cutoff)     # ligand 0's lists (the sampled ligand)
        import oracle
        n_s = max(1, min(n_spots, oracle.get_threads()))
        # generations in the sample: about 10 s of oracle work on 16 host threads
        Gs = min(G, {"medium": 10, "large": 4, "sweep": 40}.get(args.config, 50))
        dt, pr, po, cores = oracle_sample(prob, {"cutoff": cutoff},
                                          {"preset": args.preset, "population": cfg.population}, lens,
                                          args.seed, n_s, Gs)
        cpu = {"value": pr / dt, "unit": "pairs/s", "cores": cores, "cpu": cpu_model(), "kind": "oracle",
               "sample": f"fp64 oracle vso_run, {n_s} spots x {Gs} generations of {args.config} "
                         f"(P={cfg.population}, M{args.preset}), {po} poses, {dt:.1f} s; pairs counted as the "
                         f"workload defines them (n_lig x list length), the oracle itself visits all n_rec atoms"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "pairs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": args.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": args.config, "preset": f"M{args.preset}", "n_rec": cfg.n_rec,
                       "n_lig": ([len(m.q) for m in prob.ligands] if sweep else cfg.n_lig),
                       "n_spots_per_rank": n_spots, "population": cfg.population, "generations": G,
                       "mode": f"cutoff {cutoff:g} A, per-spot lists" if cutoff > 0 else "all pairs",
                       "l2": "flushed between steps (256 MB write inside the timed region)",
                       "parallelism": (f"dp{world}: (ligand, spot-chunk) units, largest ligand first, dynamic queue"
                                       if sweep else
                                       f"dp{world}: independent runs per rank (seed+rank), best-of gathered"
                                       if args.scaling == "weak" else
                                       f"dp{world}: spots dealt by a dynamic chunk queue, one gather")},
            "poses_per_s": poses / (ms * 1e-3),
            "pairs_per_step": pairs / args.steps,
            "pairs_evaluated_per_s": pairs_ev / (ms * 1e-3),
            "roofline": roof,
            "score_micro": micro,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clk,
        }
        print(json.dumps(line), flush=True)
    if sweep:
        scr.close()
    else:
        ctx.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
