"""The C-ABI library builds, loads and exports every symbol include/vs.h declares (CPU box)."""
import ctypes as C
import os
import re

import numpy as np
import pytest

from paper_conf_ppopp_imbernoncg16_b200 import vs

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "vs.h")).read()
    return sorted(set(re.findall(r"^VS_API [^(]*?\b(vs_\w+)\(", src, flags=re.M)))


def test_header_and_binding_agree():
    assert declared_symbols() == sorted(vs.EXPORTS)


def test_library_exports_every_declared_symbol():
    L = vs.load()
    for name in declared_symbols():
        assert hasattr(L, name), name
    assert L.vs_abi_version() == 4


def test_library_targets_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", vs.library_path()],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_defaults_and_presets():
    sp = vs.score_params()
    assert sp.cutoff == 12.0 and sp.region_half_width == 3.0 and sp.dielectric == 0
    assert abs(sp.coulomb_k - 332.0636) < 1e-4
    for m, (P, G, f) in {1: (64, 50, 0.0), 2: (64, 50, 1.0), 3: (64, 50, 0.2), 4: (1024, 0, 1.0)}.items():
        mp = vs.mh_preset(m)
        assert (mp.population, mp.generations) == (P, G) and abs(mp.improve_frac - f) < 1e-7
        assert mp.ls_neighbours == 1
    with pytest.raises(vs.VSError) as e:
        vs.mh_preset(5)
    assert e.value.status == vs.ERR_INVALID_ARGUMENT


def test_argument_errors_without_device():
    L = vs.load()
    h = C.c_void_p()
    # NULL arrays are rejected before any CUDA call
    st = L.vs_create(None, None, None, 1, None, None, None, 1, None, 1, None, 0, C.byref(h))
    assert st == vs.ERR_INVALID_ARGUMENT and not h.value
    assert b"NULL" in L.vs_last_error()
    assert L.vs_score_poses(None, 1, None, None, None, None) == vs.ERR_INVALID_ARGUMENT
    L.vs_destroy(None)  # NULL-safe
    assert L.vs_release_cached_memory(1 << 20) == vs.ERR_INVALID_ARGUMENT  # no such device (none at all here)


def test_create_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_ppopp_imbernoncg16_b200 import synth
    p = synth.make_problem("tiny")
    with pytest.raises(vs.VSError) as e:
        vs.Context.from_problem(p)
    assert e.value.status == vs.ERR_CUDA


def test_c_example_compiles_and_links(tmp_path):
    """The boundary is a plain C library: the C example builds against include/vs.h and links libvs.so."""
    import subprocess
    vs.load()
    out = tmp_path / "vs_example"
    r = subprocess.run(["gcc", "-O2", "-Wall", "-Werror", "-I", os.path.join(ROOT, "include"),
                        os.path.join(ROOT, "examples", "vs_example.c"), "-L", os.path.dirname(vs.library_path()),
                        "-lvs", "-lm", "-o", str(out)], capture_output=True, text=True)
    assert r.returncode == 0, r.stderr


def test_product_package_never_touches_the_oracle():
    """Only tests/, __graft_entry__.smoke() and bench.py's oracle legs may use oracle/."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_imbernoncg16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "vso_" not in src and "libvso" not in src, f


@pytest.mark.gpu
def test_c_example_runs_on_gpu(tmp_path):
    import subprocess
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    vs.load()
    out = tmp_path / "vs_example"
    libdir = os.path.dirname(vs.library_path())
    subprocess.run(["gcc", "-O2", "-I", os.path.join(ROOT, "include"), os.path.join(ROOT, "examples", "vs_example.c"),
                    "-L", libdir, "-lvs", f"-Wl,-rpath,{libdir}", "-lm", "-o", str(out)], check=True)
    r = subprocess.run([str(out)], capture_output=True, text=True, timeout=120)
    assert r.returncode == 0, r.stderr
    assert "spot 7 best" in r.stdout and "pairs" in r.stdout
