"""bench.py contract: one JSON line with the required keys (GPU box), incl. the multi-rank path."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"}


def _run(cmd, env=None):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900, env=e)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_reference_arm_line():
    d = _run([sys.executable, "bench.py", "--impl", "reference", "--config", "tiny", "--steps", "1", "--warmup", "0"])
    assert d["impl"] == "reference" and d["value"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["e2e"]["h2d_bytes_per_step"] == 0
    # value counts the pairs within rc, the oracle visits every receptor atom
    assert d["value"] <= d["workload_pairs_per_s"] <= d["visited_pairs_per_s"]


@pytest.mark.gpu
def test_bench_single_gpu_line():
    d = _run([sys.executable, "bench.py", "--config", "small", "--steps", "2", "--warmup", "3", "--generations", "4"])
    assert KEYS <= set(d)
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] > 0
    assert d["value"] < d["pairs_evaluated_per_s"] < d["workload_pairs_per_s"]
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 1.5 and r["peak"] > 0
    assert 0 < r["pair_kernel_share_of_step"] <= 1.05 and r["pair_kernel_launches"] > 0
    assert d["check"]["assembled_equals_single_process"] is True
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["cpu_baseline"]["cores"] >= 1


@pytest.mark.gpu
@pytest.mark.parametrize("extra", [["--scaling", "replicas"], ["--schedule", "queue", "--chunks-per-rank", "3",
                                                                "--slots", "2"],
                                   ["--schedule", "warmup", "--hetero", "0:2"], ["--schedule", "static"]])
def test_bench_two_ranks_gloo_on_one_gpu(extra):
    """--gpus 2 re-launches itself under torch.distributed.run; gloo collectives let both ranks share one GPU.
    The gathered, assembled per-spot bests must equal a single-process run bit for bit."""
    d = _run([sys.executable, "bench.py", "--gpus", "2", "--config", "small", "--steps", "1", "--warmup", "3",
              "--generations", "3", "--no-micro", "--no-cpu-baseline"] + extra, env={"VS_BENCH_BACKEND": "gloo"})
    assert d["n_gpus"] == 2 and d["value"] > 0
    assert all(v for v in d["check"].values() if isinstance(v, bool)), d["check"]
    if "--scaling" not in extra:
        assert sum(d["check"]["spots_per_rank"]) == 64
    if "warmup" in extra:
        w = d["warmup_split"]
        assert w["times_s"][0] > w["times_s"][1] and w["shares"][0] < w["shares"][1]   # rank 0 is slowed down


@pytest.mark.gpu
def test_bench_sweep_two_ranks_gloo():
    """The screening sweep (N1) through the multi-rank path: (ligand, spot chunk) units dealt by the queue, the
    fixed-size [ligands x spots] record table gathered and checked per ligand against a single-process run."""
    d = _run([sys.executable, "bench.py", "--gpus", "2", "--config", "sweep", "--steps", "1", "--warmup", "1",
              "--generations", "2", "--no-micro", "--no-cpu-baseline", "--no-e2e"], env={"VS_BENCH_BACKEND": "gloo"})
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["check"]["assembled_equals_single_process"] is True


def test_cpu_baseline_sample_sweep_library():
    """The cpu_baseline leg samples ligand 0 of a screening library (cfg.n_lig is 0 there): the pair count is
    n_lig(ligand 0) x list length x poses per spot, and the pose count is population x (1 + generations x steps)."""
    sys.path.insert(0, ROOT)
    import bench
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    prob = synth.make_problem("sweep")
    assert prob.cfg.n_lig == 0
    prob.lig = prob.ligands[0]
    lens = bench.list_lengths_host(prob, 12.0)
    r = bench.oracle_sample(prob, {"cutoff": 12.0}, {"preset": 3, "population": 64}, lens, 0, 2, 1)
    assert r["s"] > 0 and r["cores"] >= 1 and r["poses"] > 0 and r["poses"] % 2 == 0
    assert r["pairs"] == (int(lens[0]) + int(lens[1])) * len(prob.lig.q) * (r["poses"] // 2)
    assert 0 < r["within"] < r["pairs"] < r["visited"]


def test_hetero_and_splits_helpers():
    sys.path.insert(0, ROOT)
    import bench
    assert bench.hetero_factor("0:2,3:4", 0) == 2 and bench.hetero_factor("0:2,3:4", 3) == 4
    assert bench.hetero_factor("", 1) == 1
    import numpy as np
    iv = np.array([[20, 30], [0, 10], [5, 12], [25, 26], [12, 13]], np.uint64) * 1000000
    assert bench.union_ms(iv) == 23.0 and bench.union_ms(np.zeros((0, 2), np.uint64)) == 0.0
    assert bench.auto_splits(500) == 1 and bench.auto_splits(250) == 1 and bench.auto_splits(125) == 2 and bench.auto_splits(63) == 4
