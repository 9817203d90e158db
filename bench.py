#!/usr/bin/env python
"""Benchmark of the virtual-screening hot path (one JSON line on rank 0).

A step = one full metaheuristic run (Algorithm 1, preset
M3 of Table 4 P:232-237 with the config's population / generations) over
every spot of the configured synthetic workload: pose generation, scoring of
every individual and local-search proposal, selection, on device, then the
one gather of the per-spot bests.

  python bench.py [--gpus N --steps K --warmup W] [--config medium] [--preset 3]
      N > 1 without torchrun: re-launches itself under torch.distributed.run (one process per GPU, NCCL)
  python bench.py --impl reference ...                      (the fp64 CPU oracle arm)

Metric (BASELINE.json): atom-pair interactions / s.  `value` counts the
interactions that contribute to the scores -- the pairs within the cutoff
(r^2 < rc^2; every pair in all-pairs mode) -- counted exactly by a census run
of the same workload (same seed, so the same poses: a pair-kernel
instantiation that counts them, scores bitwise unchanged), whole job over the
max-over-ranks device time.  Workload pairs (n_lig x list length per pose),
pairs evaluated by the pair kernel and scored poses / s are reported beside it.

Multi-GPU (P:9): `--scaling strong` (default) deals
the spots to the ranks by `--schedule queue` (dynamic chunk queue on the
c10d store, the default), `static` or `warmup` (Eq. 1); rank 0
assembles the gathered per-spot bests and checks them bitwise against a
single-process run of the same spots.  `--scaling replicas`: every rank runs
the whole workload with its own seed (independent executions).
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

# One vs_run drives 13 streams per context (main + spot groups): give them their own hardware work queues (the
# default 8 aliases streams onto shared queues; measured: context create / destroy costs become erratic, up to
# hundreds of ms).  Must be set before the CUDA context exists.
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "atom-pair interactions/s and scored poses/s at 1/2/4/8 B200; % FP32 roofline"
N_SM = 148
LANES = 128
OPS_CUTOFF, OPS_ALLPAIRS = 25, 20   # canonical issue slots per pair
PACKED_PAIRS_PER_CLK_SM = 7.3       # measured ceiling of the packed cutoff pair loop (profiles/r01_notes.md)


def parse(argv=None):
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
    ap.add_argument("--dielectric", type=int, choices=[0, 1], default=0, help="1: constant eps_r (N3)")
    ap.add_argument("--eps-r", type=float, default=1.0)
    ap.add_argument("--scaling", choices=["strong", "replicas"], default="strong")
    ap.add_argument("--schedule", choices=["queue", "static", "warmup"], default="queue")
    ap.add_argument("--chunks-per-rank", type=int, default=1, help="queue: chunks = ranks x this")
    ap.add_argument("--slots", type=int, default=None,
                    help="queue: chunks in flight per rank, one context / stream each (default 1; sweep 2)")
    ap.add_argument("--list-splits", type=int, default=-1,
                    help="vs_score_params.list_splits (-1: by the spots per rank, 0: by the context)")
    ap.add_argument("--hetero", default="", help="injected heterogeneity 'rank:factor,...' (each chunk run factor x)")
    ap.add_argument("--warmup-gens", type=int, default=5, help="schedule warmup: generations timed (P:142: 5-10)")
    ap.add_argument("--seed", type=int, default=42)
    ap.add_argument("--e2e-steps", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-clocks", action="store_true")
    ap.add_argument("--no-micro", action="store_true")
    ap.add_argument("--no-check", action="store_true", help="skip the census / single-process check run")
    ap.add_argument("--micro-poses", type=int, default=1 << 20)
    return ap.parse_args(argv)


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
            # nvidia-smi takes a few hundred ms to start sampling: wait for its first line, so that a short timed
            # region (small config) is sampled too
            t0 = time.perf_counter()
            while not self.lines and time.perf_counter() - t0 < 3.0 and self.proc.poll() is None:
                time.sleep(0.01)
            self.lines.clear()
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
        if not self.lines:  # a region shorter than the 100 ms period: one query right after it
            try:
                r = subprocess.run(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                    "-i", str(self.idx)], capture_output=True, text=True, timeout=20)
                self.lines = [x.strip() for x in r.stdout.splitlines() if x.strip()]
            except (OSError, subprocess.SubprocessError):
                pass
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
    """Per-launch DRAM bytes of the pair kernel from the newest committed ncu --set full summary."""
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


def union_ms(iv) -> float:
    """Length in ms of the union of [start, end) intervals given in ns ([n, 2])."""
    if len(iv) == 0:
        return 0.0
    iv = iv[np.argsort(iv[:, 0], kind="stable")]
    tot, cs, ce = 0, int(iv[0, 0]), int(iv[0, 1])
    for a, b in iv[1:]:
        a, b = int(a), int(b)
        if a > ce:
            tot += ce - cs
            cs, ce = a, b
        elif b > ce:
            ce = b
    return (tot + ce - cs) * 1e-6


def hetero_factor(spec: str, rank: int) -> int:
    """--hetero 'r:f,...': rank r runs each of its chunks f times (an injected per-unit load, same results)."""
    for part in filter(None, spec.split(",")):
        r, f = part.split(":")
        if int(r) == rank:
            return max(1, int(f))
    return 1


def auto_splits(n_spots_per_rank: int) -> int:
    """Canonical list splits for a run of this many spots per GPU: latency-bound runs (few spots) get more
    warps per chunk (profiles/r02_notes.md, medium: 63 spots 105.6 -> 85.2 ms with 4 splits, 125 spots 159.7 ->
    140.3 ms with 2, 250 spots best with 1)."""
    return 4 if n_spots_per_rank <= 96 else (2 if n_spots_per_rank <= 200 else 1)


# ---------------------------------------------------------------- oracle arm / cpu baseline
def oracle_sample(prob, sp_kw, mp_kw, list_len, seed, n_spots_sample: int, generations: int):
    """Time the fp64 oracle (as it stands) on a bounded sample of the workload.

    Returns a dict: seconds, workload pairs, pairs within rc, pairs the oracle visits (n_lig x n_rec per pose),
    poses, threads."""
    import oracle
    o = oracle.Oracle.from_problem(prob, oracle.score_params(**sp_kw))
    mp = oracle.mh_preset(mp_kw["preset"], population=mp_kw["population"], generations=generations)
    ids = np.arange(n_spots_sample, dtype=np.int32)
    t0 = time.perf_counter()
    o.run(mp, seed, ids)
    dt = time.perf_counter() - t0
    n_lig = len(prob.lig.q)      # the sampled ligand (sweep: ligand 0; cfg.n_lig is per-ligand there)
    visited = o.pairs_evaluated()
    poses = visited // (n_lig * prob.cfg.n_rec)
    per_spot = poses // n_spots_sample
    pairs = int(sum(int(list_len[s]) for s in ids)) * n_lig * per_spot
    return {"s": dt, "pairs": pairs, "within": o.pairs_within(), "visited": visited, "poses": poses,
            "cores": min(n_spots_sample, oracle.get_threads())}


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


def oracle_sp_kw(args):
    kw = {"cutoff": 12.0 if args.mode == "cutoff" else 0.0}
    if args.dielectric:
        kw.update(dielectric=1, eps_r=args.eps_r)
    return kw


def run_reference(args, rank, world):
    """--impl reference: the oracle on the host cores (rank 0 only), same metric: pairs within rc / s."""
    if rank != 0:
        return
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem(args.config)
    if prob.cfg.n_ligands > 1:
        prob.lig = prob.ligands[0]
    kw = oracle_sp_kw(args)
    lens = list_lengths_host(prob, kw["cutoff"])
    P = prob.cfg.population
    import oracle
    n_s = max(1, min(prob.cfg.n_spots, oracle.get_threads()))   # OpenMP runs one spot per thread
    G = 2 if args.config in ("medium", "large", "sweep") else min(prob.cfg.generations, 5)
    mp_kw = {"preset": args.preset, "population": P}
    times, last = [], None
    for i in range(args.warmup + args.steps):
        r = oracle_sample(prob, kw, mp_kw, lens, args.seed, n_s, G)
        if i >= args.warmup:
            times.append(r["s"])
            last = r
    ms = 1e3 * statistics.mean(times)
    val = last["within"] / (ms * 1e-3)
    sample = f"oracle vso_run on {n_s} spot(s) x {G} generations (P={P}, preset M{args.preset}) of {args.config}"
    print(json.dumps({
        "metric": METRIC, "value": val, "unit": "pairs/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
        "config": {"workload": args.config, "preset": f"M{args.preset}", "mode": args.mode, "sample": sample},
        "poses_per_s": last["poses"] / (ms * 1e-3),
        "workload_pairs_per_s": last["pairs"] / (ms * 1e-3),
        "visited_pairs_per_s": last["visited"] / (ms * 1e-3),
        "cpu_baseline": {"value": val, "unit": "pairs/s", "cores": last["cores"], "cpu": cpu_model(),
                         "kind": "oracle", "sample": sample,
                         "visited_pairs_per_s": last["visited"] / (ms * 1e-3)},
        "e2e": {"value": val, "unit": "pairs/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# ---------------------------------------------------------------- multi-process launch
def free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def respawn(n: int) -> int:
    """bench.py --gpus N run without torchrun: start N ranks under torch.distributed.run (rank 0 prints)."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)]
    return subprocess.call(cmd + sys.argv[1:], cwd=ROOT)


# ---------------------------------------------------------------- our arm
class Runner:
    """This rank's share of a step: chunks of spots, each one vs_run_async on one of `slots` contexts / streams
    (a context runs one chunk at a time; a slot is reused after its previous chunk finished)."""

    def __init__(self, torch, vs, prob, sp, mp, seed, device, slots, n_lig_index=None):
        self.torch, self.vs, self.mp, self.seed = torch, vs, mp, seed
        self.dev = torch.device("cuda", device)
        self.ctx = [vs.Context.from_problem(prob, sp, device=device) for _ in range(max(1, slots))]
        self.streams = [torch.cuda.Stream(device=self.dev) for _ in self.ctx]
        self.done_ev = [torch.cuda.Event() for _ in self.ctx]
        n = prob.cfg.n_spots
        self.pose = torch.empty((n, 7), dtype=torch.float32, device=self.dev)
        self.score = torch.empty(n, dtype=torch.float32, device=self.dev)
        self.repeat = 1
        self.ran: list[tuple[int, int]] = []

    def launch(self, slot, a, b, seed=None):
        ids = np.arange(a, b, dtype=np.int32)
        for _ in range(self.repeat):
            self.ctx[slot].run_async(self.mp, self.seed if seed is None else seed, ids, self.pose[a:b],
                                     self.score[a:b], self.streams[slot])
        self.done_ev[slot].record(self.streams[slot])
        self.ran.append((a, b))

    def wait(self, slot):
        self.done_ev[slot].synchronize()

    def join(self, main):
        for s in self.streams:
            main.wait_stream(s)

    def fork(self, main):
        for s in self.streams:
            s.wait_stream(main)

    def stats(self):
        tot = {}
        for c in self.ctx:
            for k, v in c.stats().items():
                tot[k] = tot.get(k, 0) + v
        return tot

    def set_timing(self, flags):
        for c in self.ctx:
            c.set_timing(flags)

    def reset_stats(self):
        for c in self.ctx:
            c.reset_stats()

    def close(self):
        for c in self.ctx:
            c.close()


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(respawn(args.gpus))

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_imbernoncg16_b200 import dist as vdist
    from paper_conf_ppopp_imbernoncg16_b200 import screen, synth, vs

    # one process per GPU; VS_BENCH_BACKEND=gloo (CPU collectives, ranks may share a GPU) exercises the
    # multi-rank path on a single-GPU box
    backend = os.environ.get("VS_BENCH_BACKEND", "nccl")
    ndev = max(1, torch.cuda.device_count())
    if backend == "nccl" and world > ndev:
        raise SystemExit(f"{world} ranks but {ndev} GPU(s): NCCL needs one GPU per rank (VS_BENCH_BACKEND=gloo)")
    local = local % ndev
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cdev = dev if backend == "nccl" else torch.device("cpu")   # where collective tensors live
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    store = dist.distributed_c10d._get_default_store() if world > 1 else None

    prob = synth.make_problem(args.config)
    cfg = prob.cfg
    sweep = cfg.n_ligands > 1
    if args.slots is None:   # two ligands in flight: the sweep's P 64 runs are partly latency-bound (r02_notes.md)
        args.slots = 2 if sweep else 1
    G = cfg.generations if args.generations is None else args.generations
    cutoff = 12.0 if args.mode == "cutoff" else 0.0
    n_spots = cfg.n_spots
    per_rank = n_spots if args.scaling == "replicas" else -(-n_spots // world)
    S = auto_splits(per_rank) if args.list_splits < 0 else args.list_splits
    sp_kw = {"cutoff": cutoff, "list_splits": S}
    if args.dielectric:
        sp_kw.update(dielectric=1, eps_r=args.eps_r)
    sp = vs.score_params(**sp_kw)
    mp = vs.mh_preset(args.preset, population=cfg.population, generations=G, ls_neighbours=args.ls_neighbours)
    main_stream = torch.cuda.Stream(device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # > 126 MB L2
    rep = hetero_factor(args.hetero, rank)
    warm = None

    # ---- work units and this rank's runner
    if sweep:
        # screening sweep (N1): units (ligand, spot chunk), largest ligand first, dynamic queue
        scr = screen.Screen(prob.rec, prob.spots, prob.ligands, sp, mp, args.seed, device=local)
        sizes = [len(m.q) for m in prob.ligands]
        units = screen.unit_schedule(sizes, n_spots, world, min_chunk=16)
        if world == 1:
            scr.prepare(range(len(prob.ligands)))
        L = len(prob.ligands)
        res_pose = torch.empty((L, n_spots, 7), dtype=torch.float32, device=dev)
        res_score = torch.empty((L, n_spots), dtype=torch.float32, device=dev)
        sweep_streams = [torch.cuda.Stream(device=dev) for _ in range(max(1, args.slots))]
        sweep_ev = [torch.cuda.Event() for _ in sweep_streams]
        runner = None
    else:
        runner = Runner(torch, vs, prob, sp, mp, args.seed + (rank if args.scaling == "replicas" else 0), local,
                        args.slots if args.schedule == "queue" else 1)
        runner.repeat = rep
        if args.scaling == "replicas":
            schedule, my_range = [(0, n_spots)], (0, n_spots)
        elif args.schedule == "queue":
            schedule = vdist.equal_chunks(n_spots, world * max(1, args.chunks_per_rank))
        elif args.schedule == "static":
            my_range = vdist.equal_chunks(n_spots, world)[rank] if rank < n_spots else (0, 0)
        if args.schedule == "warmup" and args.scaling == "strong":
            # Eq. (1): time a few generations on a fixed sample of spots on every rank (with any
            # injected load), gather, Percent = t / t_slowest, shares proportional to 1 / Percent
            mpw = vs.mh_preset(args.preset, population=cfg.population, generations=args.warmup_gens,
                               ls_neighbours=args.ls_neighbours)
            wn = min(n_spots, 16)
            wp = torch.empty((wn, 7), device=dev)
            ws = torch.empty(wn, device=dev)

            def warm_run():
                ids = np.arange(wn, dtype=np.int32)
                runner.ctx[0].run_async(mpw, args.seed, ids, wp, ws, main_stream)   # untimed: lazy set-up
                torch.cuda.synchronize(dev)
                if world > 1:
                    dist.barrier()  # no rank times its warm-up while another still does its lazy set-up
                t0 = time.perf_counter()
                for _ in range(rep):
                    runner.ctx[0].run_async(mpw, args.seed, ids, wp, ws, main_stream)
                torch.cuda.synchronize(dev)
                return time.perf_counter() - t0

            if world > 1:
                my_range, wtimes = vdist.warmup_split(warm_run, n_spots, cdev)
            else:
                my_range, wtimes = (0, n_spots), [warm_run()]
            warm = {"times_s": wtimes, "percent": vdist.percent_from_times(wtimes),
                    "shares": [b - a for a, b in vdist.shares_from_percent(vdist.percent_from_times(wtimes),
                                                                            n_spots)]}

    def step(i: int):
        """One whole-job pass: this rank's share, then the one gather of the fixed-size record table."""
        with torch.cuda.stream(main_stream):
            flush.zero_()
            rec = vdist.empty_records(n_spots if not sweep else len(prob.ligands) * n_spots, dev)
            if sweep:
                for s in sweep_streams:
                    s.wait_stream(main_stream)

                def launch(slot, li, a, b):
                    for _ in range(rep):
                        scr.run_unit(li, a, b, res_pose[li, a:b], res_score[li, a:b], sweep_streams[slot])
                    sweep_ev[slot].record(sweep_streams[slot])
                    ran.append((li, a, b))

                ran = []
                q = vdist.ChunkQueue(store, f"s{i}", len(units))
                vdist.run_dynamic(q, [(u,) for u in range(len(units))], len(sweep_streams),
                                  lambda s, u: launch(s, *units[u]), lambda s: sweep_ev[s].synchronize())
                for s in sweep_streams:
                    main_stream.wait_stream(s)
                for li, a, b in ran:
                    vdist.fill_records(rec, li * n_spots + a, li * n_spots + b, res_pose[li, a:b], res_score[li, a:b])
                    rec[li * n_spots + a:li * n_spots + b, 0] = torch.arange(a, b, dtype=torch.float32, device=dev)
            else:
                runner.fork(main_stream)
                runner.ran = []
                if args.scaling == "strong" and args.schedule == "queue":
                    q = vdist.ChunkQueue(store, f"q{i}", len(schedule))
                    vdist.run_dynamic(q, schedule, len(runner.ctx), runner.launch, runner.wait)
                elif my_range[1] > my_range[0]:
                    runner.launch(0, *my_range)
                runner.join(main_stream)
                for a, b in runner.ran:
                    vdist.fill_records(rec, a, b, runner.pose[a:b], runner.score[a:b])
            return vdist.gather_fixed(rec, cdev)

    # the pair kernel's launch intervals are recorded in the warm-up steps too: the instrumented launches are what
    # the warm-up captures into the CUDA graphs the timed steps replay
    if sweep:
        scr.set_timing(vs.TIMING_KERNEL)        # also for the contexts the sweep creates lazily
    else:
        runner.set_timing(vs.TIMING_KERNEL)
    for i in range(args.warmup):
        step(-1 - i)
    torch.cuda.synchronize(dev)
    work_ctx = list(scr.ctx.values()) if sweep else runner.ctx   # the sweep creates its contexts lazily
    for c in work_ctx:
        c.reset_stats()
    clocks = ClockSampler(local, enabled=(rank == 0 and not args.no_clocks))
    clocks.start()   # before the barrier: the sampler is running when every rank enters the timed region
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize(dev)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main_stream)
    for i in range(args.steps):
        tables = step(i)
    e1.record(main_stream)
    torch.cuda.synchronize(dev)
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    ms_rank = e0.elapsed_time(e1)
    work_ctx = list(scr.ctx.values()) if sweep else runner.ctx
    st = {}
    ivs = []
    for c in work_ctx:
        for k, v in c.stats().items():
            st[k] = st.get(k, 0) + v
        ivs.append(c.pair_intervals())
    # contexts (slots, ligands) run concurrently: the pair kernel's busy time is the union of all their launch
    # intervals on the device clock, not the sum of the per-context unions
    st["pair_busy_ms"] = union_ms(np.concatenate(ivs)) if ivs else 0.0
    if sweep:
        scr.set_timing(0)
    else:
        runner.set_timing(0)
    # whole-job totals and max-over-ranks time
    tot = torch.tensor([st["pairs"], st["poses_scored"], st["kernel_launches"], st["pairs_evaluated"]],
                       dtype=torch.float64, device=cdev)
    tmax = torch.tensor([ms_rank], dtype=torch.float64, device=cdev)
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
        dist.all_reduce(tmax, op=dist.ReduceOp.MAX)
    pairs, poses, launches, pairs_ev = (float(x) for x in tot.tolist())
    ms = float(tmax.item())

    # ---- census + check (rank 0, untimed): the same workload in one process with the pair kernel counting the
    # pairs within rc (same poses: same seed); its results must equal the assembled multi-rank results bit for bit
    census = {"pairs_within": None}
    check = None
    if not args.no_check:
        if rank == 0:
            if sweep:
                within = 0
                ok = True
                recs = np.concatenate([t.cpu().numpy() for t in tables]) if tables else None
                for li in range(len(prob.ligands)):
                    c = scr.context(li)
                    c.reset_stats()
                    c.set_timing(vs.TIMING_CENSUS)
                    p, s = c.run(mp, screen.ligand_seed(args.seed, li))
                    within += c.stats()["pairs_within"]
                    c.set_timing(0)
                    if recs is not None:
                        gp, gs, _ = vdist.assemble([t.cpu().numpy()[li * n_spots:(li + 1) * n_spots] for t in tables],
                                                   n_spots)
                        ok = ok and np.array_equal(gp, p) and np.array_equal(gs, s)
                census = {"pairs_within": within * (world if args.scaling == "replicas" else 1)}
                check = {"assembled_equals_single_process": bool(ok)}
            else:
                c = runner.ctx[0]
                c.reset_stats()
                c.set_timing(vs.TIMING_CENSUS)
                p, s = c.run(mp, args.seed)
                cs = c.stats()
                c.set_timing(0)
                census = {"pairs_within": cs["pairs_within"] * (world if args.scaling == "replicas" else 1)}
                tabs = [t.cpu().numpy() for t in tables]
                if args.scaling == "replicas":
                    gp, gs = vdist.best_of(tabs)
                    ok = bool(np.all(gs <= s))                      # the best of the replicas beats replica 0
                    check = {"best_of_replicas_not_worse_than_rank0": ok}
                else:
                    gp, gs, owner = vdist.assemble(tabs, n_spots)
                    ok = bool(np.array_equal(gp, p) and np.array_equal(gs, s))
                    check = {"assembled_equals_single_process": ok,
                             "spots_per_rank": np.bincount(owner, minlength=world).tolist()}
            if not all(v for v in check.values() if isinstance(v, bool)):
                print(f"bench: CHECK FAILED {check}", file=sys.stderr, flush=True)
        if world > 1:
            dist.barrier()
    if world > 1:   # every rank needs the census count (roofline, e2e)
        t = torch.tensor([census["pairs_within"] if census["pairs_within"] is not None else -1.0],
                         dtype=torch.float64, device=cdev)
        dist.broadcast(t, 0)
        census["pairs_within"] = None if t.item() < 0 else float(t.item())
    within_step = census["pairs_within"]

    # ---- roofline of the dominant kernel (the pair kernel, this rank): its launch intervals (device globaltimer,
    # also inside replayed CUDA graphs) give the time the pair kernel was running; within-rc pairs of this rank =
    # its evaluated pairs x the census ratio within / evaluated
    pk = peaks()
    f_max = pk.get("sm_max_mhz", 1965.0)
    ops = OPS_CUTOFF if cutoff > 0 else OPS_ALLPAIRS
    peak = N_SM * LANES * f_max * 1e6 / ops / 1e9
    busy_s = max(1e-9, st["pair_busy_ms"] * 1e-3)
    ev_rank = st["pairs_evaluated"]
    # pairs within rc per pair evaluated (the census counts the whole job once per step)
    frac_within = within_step / max(1.0, pairs_ev / args.steps) if within_step is not None else None
    ach_eval = ev_rank / busy_s / 1e9
    ach_within = ev_rank * frac_within / busy_s / 1e9 if frac_within is not None else None
    roof = {"bound": "alu", "achieved": ach_within if ach_within is not None else ach_eval, "peak": peak,
            "unit": "Gpairs/s",
            "frac": (ach_within if ach_within is not None else ach_eval) / peak,
            "traffic": ncu_traffic(args.config),
            "achieved_basis": "pairs within rc processed by the pair kernel (rank 0) / the time the pair kernel was "
                              "running (union of its launch intervals, device globaltimer, in the timed region)",
            "peak_basis": f"R_pair = {N_SM} SMs x {LANES} FP32 lanes x {f_max:.0f} MHz (MEASURED_PEAKS sm_max) / "
                          f"{ops} canonical issue slots per pair (SURVEY.md §8(d))",
            "evaluated_gpairs_per_s": ach_eval, "frac_evaluated": ach_eval / peak,
            "peak_packed": N_SM * PACKED_PAIRS_PER_CLK_SM * f_max * 1e6 / 1e9,
            "peak_packed_basis": f"{PACKED_PAIRS_PER_CLK_SM} pairs/clk/SM, measured packed cutoff pair loop "
                                 "(tools/microbench/pair_loop_cost.cu)",
            "within_over_evaluated": frac_within,
            "pair_kernel_busy_ms_per_step": st["pair_busy_ms"] / args.steps,
            "pair_kernel_share_of_step": st["pair_busy_ms"] / max(1e-9, ms_rank),
            "pair_kernel_launch_ms_sum": st["pair_launch_ms"], "pair_kernel_launches": st["pair_timed_launches"],
            "pair_kernel_warps_per_sm_in_run": st["pair_warp_ms"] / max(1e-9, st["pair_busy_ms"]) / N_SM,
            "pair_kernel_warps_per_sm_max": 20,
            "in_run_basis": "sum over every pair-kernel warp of its globaltimer duration / busy time / 148 SMs: the "
                            "average number of resident pair-kernel warps per SM during the timed steps (one-warp "
                            "CTAs, 96 registers: at most 20)"}
    if clk:
        roof["frac_at_run_clock"] = roof["frac"] * f_max / clk["sm_mhz"]

    # ---- end to end through the public C ABI with host buffers (vs_create + vs_run + results to host), this
    # rank's share by the same schedule
    e2e = None
    if not args.no_e2e:
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
        ligs = prob.ligands if sweep else [prob.lig]
        rec_h = [pin(x) for x in (prob.rec.xyz, prob.rec.q, prob.rec.type)]
        lig_h = [[pin(x) for x in (L_.xyz, L_.q, L_.type)] for L_ in ligs]
        spot_h = pin(prob.spots)
        n_e2e = args.e2e_steps if args.e2e_steps is not None else (1 if sweep else max(1, min(args.steps, 2)))
        # one untimed warm-up pass of this rank's share: the first context of a process pays cudaMalloc for the
        # device memory cache (and the first launch of every kernel its lazy module load)
        c2 = vs.Context(*rec_h, *lig_h[0], spot_h, sp=sp, device=local)
        wa, wb = (0, n_spots) if sweep or args.scaling == "replicas" else \
            (schedule[0] if args.schedule == "queue" and schedule else (my_range if args.schedule != "queue" else (0, 0)))
        if wb > wa:
            c2.run(mp, args.seed, np.arange(wa, wb, dtype=np.int32))
        c2.close()
        torch.cuda.synchronize(local)
        if world > 1:
            dist.barrier()
        parts_ms = {"create": 0.0, "run": 0.0, "destroy": 0.0}
        h2d = d2h = 0
        t0 = time.perf_counter()
        for i in range(n_e2e):
            if sweep:
                q = vdist.ChunkQueue(store, f"e{i}", len(units))
                ctxs = {}  # a rank closes a ligand's context after the ligand's last unit (device memory back to the cache)
                while (u := q.claim()) is not None:
                    li, a, b = units[u]
                    ta = time.perf_counter()
                    if li not in ctxs:
                        ctxs[li] = vs.Context(*rec_h, *lig_h[li], spot_h, sp=sp, device=local)
                        h2d += sum(x.nbytes for x in rec_h) + spot_h.nbytes + sum(x.nbytes for x in lig_h[li])
                    tb = time.perf_counter()
                    ctxs[li].run(mp, screen.ligand_seed(args.seed, li), np.arange(a, b, dtype=np.int32))
                    h2d += 4 * (b - a)
                    d2h += 32 * (b - a)
                    tc = time.perf_counter()
                    parts_ms["create"] += 1e3 * (tb - ta)
                    parts_ms["run"] += 1e3 * (tc - tb)
                    # units are claimed in order (ligands by decreasing size, then chunks): once the queue has moved
                    # past a ligand's last unit no rank can claim more of it
                    if all(units[v][0] != li for v in range(u + 1, len(units))):
                        ctxs.pop(li).close()
                        parts_ms["destroy"] += 1e3 * (time.perf_counter() - tc)
                tc = time.perf_counter()
                for c in ctxs.values():
                    c.close()
                parts_ms["destroy"] += 1e3 * (time.perf_counter() - tc)
            else:
                ta = time.perf_counter()
                c2 = vs.Context(*rec_h, *lig_h[0], spot_h, sp=sp, device=local)
                h2d += sum(x.nbytes for x in rec_h) + spot_h.nbytes + sum(x.nbytes for x in lig_h[0])
                tb = time.perf_counter()
                if args.scaling == "strong" and args.schedule == "queue":
                    q = vdist.ChunkQueue(store, f"e{i}", len(schedule))
                    while (u := q.claim()) is not None:
                        a, b = schedule[u]
                        c2.run(mp, args.seed, np.arange(a, b, dtype=np.int32))
                        h2d += 4 * (b - a)
                        d2h += 32 * (b - a)
                elif my_range[1] > my_range[0]:
                    a, b = my_range
                    c2.run(mp, args.seed + (rank if args.scaling == "replicas" else 0),
                           np.arange(a, b, dtype=np.int32))
                    h2d += 4 * (b - a)
                    d2h += 32 * (b - a)
                tc = time.perf_counter()
                c2.close()
                td = time.perf_counter()
                parts_ms["create"] += 1e3 * (tb - ta)
                parts_ms["run"] += 1e3 * (tc - tb)
                parts_ms["destroy"] += 1e3 * (td - tc)
        dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64, device=cdev)
        byt = torch.tensor([h2d, d2h], dtype=torch.float64, device=cdev)
        if world > 1:
            dist.all_reduce(dt, op=dist.ReduceOp.MAX)
            dist.all_reduce(byt, op=dist.ReduceOp.SUM)
        per_step_s = float(dt.item()) / n_e2e
        e2e_pairs = within_step if within_step is not None else pairs / args.steps
        e2e = {"value": e2e_pairs / per_step_s, "unit": "pairs/s",
               "h2d_bytes_per_step": float(byt[0].item()) / n_e2e, "d2h_bytes_per_step": float(byt[1].item()) / n_e2e,
               "steps": n_e2e, "ms_per_step": 1e3 * per_step_s,
               "ms_per_step_parts_rank0": {k: v / n_e2e for k, v in parts_ms.items()},
               "what": "vs_create (receptor/ligand/spot upload from pinned host memory + per-spot list build) + "
                       "vs_run per claimed chunk (host spot ids in, best poses/scores to host) + vs_destroy, wall "
                       "clock, max over ranks, after one untimed warm-up context"}

    # ---- scoring-kernel microbenchmark (rank 0): one vs_score_poses_device batch of device-resident poses
    micro = None
    if rank == 0 and not args.no_micro:
        ctx = scr.context(0) if sweep else runner.ctx[0]
        n_micro = args.micro_poses
        spot_h, q_h, t_h = synth.make_poses(n_micro, n_spots, 3.0, seed=7)
        spot_d = torch.from_numpy(spot_h).to(dev)
        q_d, t_d = torch.from_numpy(q_h).to(dev), torch.from_numpy(t_h).to(dev)
        out_d = torch.empty(n_micro, dtype=torch.float32, device=dev)
        with torch.cuda.stream(main_stream):
            for _ in range(2):
                ctx.score_poses_device(spot_d, q_d, t_d, out_d, main_stream)
            torch.cuda.synchronize(dev)
            ctx.set_timing(vs.TIMING_CENSUS)
            ctx.reset_stats()
            ctx.score_poses_device(spot_d, q_d, t_d, out_d, main_stream)
            torch.cuda.synchronize(dev)
            within_m = ctx.stats()["pairs_within"]
            ctx.set_timing(vs.TIMING_KERNEL)
            ctx.reset_stats()
            m0, m1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            reps = 3
            m0.record(main_stream)
            for _ in range(reps):
                ctx.score_poses_device(spot_d, q_d, t_d, out_d, main_stream)
            m1.record(main_stream)
        torch.cuda.synchronize(dev)
        ms_m = m0.elapsed_time(m1) / reps
        stm = ctx.stats()
        ctx.set_timing(0)
        kbusy = max(1e-9, stm["pair_busy_ms"] * 1e-3 / reps)
        micro = {"what": f"vs_score_poses_device, {n_micro} device-resident random in-region poses over "
                         f"{n_spots} spots (validate + bucket by spot + score), mean of {reps}",
                 "ms": ms_m, "pairs_within_per_s": within_m / (ms_m * 1e-3), "poses_per_s": n_micro / (ms_m * 1e-3),
                 "workload_pairs_per_s": stm["pairs"] / reps / (ms_m * 1e-3),
                 "pair_kernel_ms": kbusy * 1e3,
                 "pair_kernel_within_gpairs_per_s": within_m / kbusy / 1e9,
                 "pair_kernel_evaluated_gpairs_per_s": stm["pairs_evaluated"] / reps / kbusy / 1e9,
                 "frac": within_m / kbusy / 1e9 / peak,
                 "frac_evaluated": stm["pairs_evaluated"] / reps / kbusy / 1e9 / peak}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        if sweep:
            prob.lig = prob.ligands[0]
        lens = list_lengths_host(prob, cutoff)
        import oracle
        n_s = max(1, min(n_spots, oracle.get_threads()))
        # generations in the sample: about 10 s of oracle work on 16 host threads
        Gs = min(G, {"medium": 10, "large": 4, "sweep": 40}.get(args.config, 50))
        r = oracle_sample(prob, oracle_sp_kw(args), {"preset": args.preset, "population": cfg.population}, lens,
                          args.seed, n_s, Gs)
        cpu = {"value": r["within"] / r["s"], "unit": "pairs/s", "cores": r["cores"], "cpu": cpu_model(),
               "kind": "oracle", "visited_pairs_per_s": r["visited"] / r["s"],
               "workload_pairs_per_s": r["pairs"] / r["s"], "poses_per_s": r["poses"] / r["s"],
               "sample": f"fp64 oracle vso_run, {n_s} spots x {Gs} generations of {args.config} "
                         f"(P={cfg.population}, M{args.preset}), {r['poses']} poses, {r['s']:.1f} s; value counts "
                         f"the pairs within rc like ours; the oracle visits all n_rec atoms per ligand atom "
                         f"(visited_pairs_per_s)"}

    if rank == 0:
        value = (within_step * args.steps if within_step is not None else pairs) / (ms * 1e-3)
        line = {
            "metric": METRIC, "value": value, "unit": "pairs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if args.scaling == "strong" else "weak", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic",
            "config": {"workload": args.config, "preset": f"M{args.preset}", "n_rec": cfg.n_rec,
                       "n_lig": ([len(m.q) for m in prob.ligands] if sweep else cfg.n_lig),
                       "n_spots": n_spots, "population": cfg.population, "generations": G,
                       "mode": (f"cutoff {cutoff:g} A, per-spot lists" if cutoff > 0 else "all pairs") +
                               (f", constant dielectric eps_r {args.eps_r:g}" if args.dielectric else ""),
                       "list_splits": S,
                       "l2": "flushed between steps (256 MB write inside the timed region)",
                       "parallelism": (f"dp{world}: " + ("replicas: every rank the whole workload, seed + rank, "
                                                        "best of gathered" if args.scaling == "replicas" else
                                                        {"queue": f"spots dealt by a dynamic chunk queue "
                                                                  f"({world * args.chunks_per_rank} chunks, "
                                                                  f"{args.slots} in flight per rank)",
                                                         "static": "equal contiguous spot ranges",
                                                         "warmup": "Eq. 1 warm-up split (P:144)"}[args.schedule])
                                       + ", one gather")},
            "value_basis": "pairs within the cutoff (r^2 < rc^2: the interactions that contribute; every pair in "
                           "all-pairs mode) per step, counted by a census run of the same seed, x steps / "
                           "max-over-ranks device time",
            "poses_per_s": poses / (ms * 1e-3),
            "workload_pairs_per_s": pairs / (ms * 1e-3),
            "pairs_evaluated_per_s": pairs_ev / (ms * 1e-3),
            "pairs_within_per_step": within_step,
            "roofline": roof,
            "score_micro": micro,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "check": check,
            "gpu_launches": int(launches),
            "clocks": clk,
        }
        if warm is not None:
            line["warmup_split"] = warm
        if args.hetero:
            line["config"]["hetero"] = args.hetero
        print(json.dumps(line), flush=True)
    if sweep:
        scr.close()
    else:
        runner.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
