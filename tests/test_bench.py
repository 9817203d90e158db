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


@pytest.mark.gpu
def test_bench_single_gpu_line():
    d = _run([sys.executable, "bench.py", "--config", "small", "--steps", "2", "--warmup", "3", "--generations", "4"])
    assert KEYS <= set(d)
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["gpu_launches"] > 0
    r = d["roofline"]
    assert r["bound"] == "alu" and 0 < r["frac"] < 3 and r["peak"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["cpu_baseline"]["cores"] >= 1


@pytest.mark.gpu
@pytest.mark.parametrize("scaling", ["weak", "strong"])
def test_bench_two_ranks_gloo_on_one_gpu(scaling):
    """The torchrun path (queue, gather, max-over-ranks timing) with gloo collectives on one GPU."""
    d = _run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
              "--master-addr", "127.0.0.1", "--master-port", "29517" if scaling == "weak" else "29519",
              "bench.py", "--gpus", "2", "--config", "small", "--steps", "1", "--warmup", "3", "--generations", "3",
              "--scaling", scaling, "--no-micro", "--no-cpu-baseline"], env={"VS_BENCH_BACKEND": "gloo"})
    assert d["n_gpus"] == 2 and d["scaling"] == scaling and d["value"] > 0


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
    dt, pairs, poses, cores = bench.oracle_sample(prob, {"cutoff": 12.0}, {"preset": 3, "population": 64},
                                                  lens, 0, 2, 1)
    assert dt > 0 and cores >= 1 and poses > 0 and poses % 2 == 0
    assert pairs == (int(lens[0]) + int(lens[1])) * len(prob.lig.q) * (poses // 2)
