"""The library's device Philox4x32-10 (R23) against NVIDIA's cuRAND device implementation (curand_Philox4x32_10):
an implementation the build did not write (SURVEY.md §8(c) "GPU cross-check against cuRAND")."""
import os
import subprocess

import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import vs

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def curand_bin(tmp_path_factory):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    out = str(tmp_path_factory.mktemp("curand") / "curand_philox")
    nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
    subprocess.run([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-o", out,
                    os.path.join(HERE, "cuda", "curand_philox.cu")], check=True)
    return out


@pytest.mark.parametrize("key", [(0, 0), (0xFFFFFFFF, 0xFFFFFFFF), (42, 0), (0x9E3779B9, 0x7F4A7C15)])
def test_device_philox_equals_curand(curand_bin, key):
    rng = np.random.default_rng(key[0] ^ 3)
    ctr = rng.integers(0, 2 ** 32, size=(2048, 4), dtype=np.uint64).astype(np.uint32)
    ctr[:4] = [[0, 0, 0, 0], [0xFFFFFFFF] * 4, [1, 2, 3, (6 << 24) | 5], [7, 0, 100, (1 << 24) | 63]]
    inp = f"{len(ctr)} {key[0]} {key[1]}\n" + "\n".join(" ".join(map(str, r)) for r in ctr)
    r = subprocess.run([curand_bin], input=inp, capture_output=True, text=True, check=True)
    want = np.array([list(map(int, ln.split())) for ln in r.stdout.splitlines()], np.uint64).astype(np.uint32)
    got = vs.debug_philox(ctr, list(key))
    np.testing.assert_array_equal(got, want)
