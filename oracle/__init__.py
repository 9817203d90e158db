"""fp64 CPU oracle of the virtual-screening hot path -- TEST INFRASTRUCTURE.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product package
(paper_conf_ppopp_imbernoncg16_b200) never does, and shares no code with it.

Thin ctypes wrapper over oracle/libvso.so (built from oracle/vso.cpp with
plain g++; see vso.h for what each function computes and which passage of
the paper it follows).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB = os.path.join(HERE, "libvso.so")
SRC = [os.path.join(HERE, "vso.cpp"), os.path.join(HERE, "vso.h")]

OK, ERR_INVALID_ARGUMENT, ERR_POSE_OUT_OF_REGION, ERR_ZERO_QUATERNION, ERR_CUDA, ERR_OUT_OF_MEMORY, ERR_UNSUPPORTED = range(7)


def build(force: bool = False) -> str:
    """Compile libvso.so with plain g++ (no fast-math, no FMA contraction)."""
    stale = not os.path.exists(LIB) or any(os.path.getmtime(s) > os.path.getmtime(LIB) for s in SRC)
    if force or stale:
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared",
                               "-Wall", SRC[0], "-o", tmp])
        os.replace(tmp, LIB)
    return LIB


class ScoreParams(C.Structure):
    _fields_ = [("coulomb_k", C.c_float), ("dielectric", C.c_int), ("eps_r", C.c_float), ("cutoff", C.c_float),
                ("region_half_width", C.c_float), ("hb_eps", C.c_float), ("hb_r0", C.c_float),
                ("r2_min", C.c_float), ("n_types", C.c_int), ("type_sigma", C.POINTER(C.c_float)),
                ("type_eps", C.POINTER(C.c_float)), ("type_hb_role", C.POINTER(C.c_int))]


class MHParams(C.Structure):
    _fields_ = [("population", C.c_int), ("generations", C.c_int), ("ls_steps", C.c_int),
                ("improve_frac", C.c_float), ("p_mut", C.c_float), ("mut_trans", C.c_float),
                ("mut_rot", C.c_float), ("ls_trans", C.c_float), ("ls_rot", C.c_float),
                ("ls_neighbours", C.c_int)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = C.CDLL(build())
        f32p, i32p, f64p, u32p = (C.POINTER(C.c_float), C.POINTER(C.c_int32), C.POINTER(C.c_double),
                                  C.POINTER(C.c_uint32))
        vp = C.c_void_p
        L.vso_score_params_default.argtypes = [C.POINTER(ScoreParams)]
        L.vso_mh_preset.argtypes = [C.c_int, C.POINTER(MHParams)]
        L.vso_create.argtypes = [f32p, f32p, i32p, C.c_int32, f32p, f32p, i32p, C.c_int32, f32p, C.c_int32,
                                 C.POINTER(ScoreParams), C.c_int32, C.POINTER(vp)]
        L.vso_score_poses.argtypes = [vp, C.c_int64, i32p, f32p, f32p, f32p]
        L.vso_score_poses_d.argtypes = [vp, C.c_int64, i32p, f32p, f32p, f64p]
        L.vso_run.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, i32p, f32p, f32p]
        L.vso_run_d.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, i32p, f32p, f64p]
        L.vso_destroy.argtypes = [vp]
        L.vso_last_error.restype = C.c_char_p
        L.vso_set_threads.argtypes = [C.c_int]
        L.vso_philox4x32_10.argtypes = [u32p, u32p, u32p]
        L.vso_u01.argtypes = [C.c_uint32]
        L.vso_u01.restype = C.c_float
        L.vso_v11.argtypes = [C.c_uint32]
        L.vso_v11.restype = C.c_float
        L.vso_score_one.argtypes = [vp, C.c_int32, f32p, f32p]
        L.vso_score_one.restype = C.c_double
        L.vso_ligand_local.argtypes = [vp, f32p]
        L.vso_pairs_evaluated.argtypes = [vp]
        L.vso_pairs_evaluated.restype = C.c_uint64
        L.vso_pairs_within.argtypes = [vp]
        L.vso_pairs_within.restype = C.c_uint64
        L.vso_init_pose.argtypes = [vp, C.c_uint64, C.c_int32, C.c_int32, f32p]
        L.vso_combine_child.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, C.c_int32, C.c_int32,
                                        f32p, f32p]
        L.vso_ls_proposal.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, C.c_int32, C.c_int32,
                                      C.c_int32, f32p, f32p]
        L.vso_ls_proposal_k.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, C.c_int32, C.c_int32,
                                        C.c_int32, C.c_int32, f32p, f32p]
        L.vso_select_parents.argtypes = [C.POINTER(MHParams), C.c_uint64, C.c_int32, C.c_int32, C.c_int32,
                                         i32p, i32p]
        L.vso_improve_count.argtypes = [C.POINTER(MHParams)]
        L.vso_select_improve.argtypes = [f64p, C.c_int32, C.c_int32, i32p]
        L.vso_include.argtypes = [f64p, f64p, C.c_int32, i32p]
        _lib = L
    return _lib


def _p(a, ctype):
    return a.ctypes.data_as(C.POINTER(ctype)) if a is not None else None


class OracleError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"vso status {status}: {msg}")
        self.status = status


def _check(st):
    if st != OK:
        raise OracleError(st, lib().vso_last_error().decode())


def score_params(**kw) -> ScoreParams:
    sp = ScoreParams()
    lib().vso_score_params_default(C.byref(sp))
    for k, v in kw.items():
        setattr(sp, k, v)
    return sp


def mh_preset(m: int, **kw) -> MHParams:
    mp = MHParams()
    _check(lib().vso_mh_preset(m, C.byref(mp)))
    for k, v in kw.items():
        setattr(mp, k, v)
    return mp


def set_threads(n: int) -> None:
    lib().vso_set_threads(n)


def get_threads() -> int:
    return lib().vso_get_threads()


def philox(ctr, key) -> np.ndarray:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    lib().vso_philox4x32_10(_p(c, C.c_uint32), _p(k, C.c_uint32), _p(o, C.c_uint32))
    return o


def u01(w: int) -> float:
    return lib().vso_u01(w)


def v11(w: int) -> float:
    return lib().vso_v11(w)


def improve_count(mp: MHParams) -> int:
    return lib().vso_improve_count(C.byref(mp))


def select_improve(scores, m: int) -> np.ndarray:
    s = np.ascontiguousarray(scores, dtype=np.float64)
    J = np.zeros(m, dtype=np.int32)
    lib().vso_select_improve(_p(s, C.c_double), len(s), m, _p(J, C.c_int32))
    return J


def select_parents(mp: MHParams, seed: int, spot: int, g: int, j: int) -> tuple[int, int]:
    """Select (R13): sorted-population ranks of the two parents of child j."""
    a, b = C.c_int32(), C.c_int32()
    lib().vso_select_parents(C.byref(mp), seed, spot, g, j, C.byref(a), C.byref(b))
    return a.value, b.value


def include(sS, sC) -> np.ndarray:
    a = np.ascontiguousarray(sS, dtype=np.float64)
    b = np.ascontiguousarray(sC, dtype=np.float64)
    o = np.zeros(len(a), dtype=np.int32)
    lib().vso_include(_p(a, C.c_double), _p(b, C.c_double), len(a), _p(o, C.c_int32))
    return o


class Oracle:
    """fp64 oracle context (vso_create ... vso_destroy)."""

    def __init__(self, rec_xyz, rec_q, rec_type, lig_xyz, lig_q, lig_type, spot_xyz, sp: ScoreParams | None = None):
        self.h = None
        self._keep = [np.ascontiguousarray(rec_xyz, np.float32), np.ascontiguousarray(rec_q, np.float32),
                      np.ascontiguousarray(rec_type, np.int32), np.ascontiguousarray(lig_xyz, np.float32),
                      np.ascontiguousarray(lig_q, np.float32), np.ascontiguousarray(lig_type, np.int32),
                      np.ascontiguousarray(spot_xyz, np.float32)]
        rx, rq, rt, lx, lq, lt, sx = self._keep
        self.n_rec, self.n_lig, self.n_spots = len(rq), len(lq), len(sx)
        self.sp = sp if sp is not None else score_params()
        h = C.c_void_p()
        _check(lib().vso_create(_p(rx, C.c_float), _p(rq, C.c_float), _p(rt, C.c_int32), self.n_rec,
                                _p(lx, C.c_float), _p(lq, C.c_float), _p(lt, C.c_int32), self.n_lig,
                                _p(sx, C.c_float), self.n_spots, C.byref(self.sp), 0, C.byref(h)))
        self.h = h

    @classmethod
    def from_problem(cls, prob, sp=None, ligand=None):
        lig = ligand if ligand is not None else prob.lig
        return cls(prob.rec.xyz, prob.rec.q, prob.rec.type, lig.xyz, lig.q, lig.type, prob.spots, sp)

    def close(self):
        if getattr(self, "h", None):
            lib().vso_destroy(self.h)
            self.h = None

    __del__ = close

    def score(self, spot, q, t) -> np.ndarray:
        spot = np.ascontiguousarray(spot, np.int32)
        q = np.ascontiguousarray(q, np.float32)
        t = np.ascontiguousarray(t, np.float32)
        out = np.zeros(len(spot), np.float64)
        _check(lib().vso_score_poses_d(self.h, len(spot), _p(spot, C.c_int32), _p(q, C.c_float), _p(t, C.c_float),
                                       _p(out, C.c_double)))
        return out

    def score_f32(self, spot, q, t) -> np.ndarray:
        spot = np.ascontiguousarray(spot, np.int32)
        q = np.ascontiguousarray(q, np.float32)
        t = np.ascontiguousarray(t, np.float32)
        out = np.zeros(len(spot), np.float32)
        _check(lib().vso_score_poses(self.h, len(spot), _p(spot, C.c_int32), _p(q, C.c_float), _p(t, C.c_float),
                                     _p(out, C.c_float)))
        return out

    def score_one(self, spot: int, q, t) -> float:
        q = np.ascontiguousarray(q, np.float32)
        t = np.ascontiguousarray(t, np.float32)
        return lib().vso_score_one(self.h, spot, _p(q, C.c_float), _p(t, C.c_float))

    def run(self, mp: MHParams, seed: int, spot_ids=None):
        ids = None if spot_ids is None else np.ascontiguousarray(spot_ids, np.int32)
        n = self.n_spots if ids is None else len(ids)
        pose = np.zeros((n, 7), np.float32)
        sc = np.zeros(n, np.float64)
        _check(lib().vso_run_d(self.h, C.byref(mp), seed, 0 if ids is None else n, _p(ids, C.c_int32),
                               _p(pose, C.c_float), _p(sc, C.c_double)))
        return pose, sc

    def ligand_local(self) -> np.ndarray:
        o = np.zeros((self.n_lig, 3), np.float32)
        lib().vso_ligand_local(self.h, _p(o, C.c_float))
        return o

    def pairs_evaluated(self) -> int:
        return lib().vso_pairs_evaluated(self.h)

    def pairs_within(self) -> int:
        """Visited pairs with r^2 < rc^2 (every pair in all-pairs mode): the interactions that contribute."""
        return lib().vso_pairs_within(self.h)

    # ---- lockstep building blocks (pose = 7 floats) ----
    def init_pose(self, seed: int, spot: int, i: int) -> np.ndarray:
        o = np.zeros(7, np.float32)
        lib().vso_init_pose(self.h, seed, spot, i, _p(o, C.c_float))
        return o

    def combine_child(self, mp: MHParams, seed: int, spot: int, g: int, j: int, S_sorted) -> np.ndarray:
        S = np.ascontiguousarray(S_sorted, np.float32).reshape(-1, 7)
        assert len(S) == mp.population
        o = np.zeros(7, np.float32)
        lib().vso_combine_child(self.h, C.byref(mp), seed, spot, g, j, _p(S, C.c_float), _p(o, C.c_float))
        return o

    def ls_proposal(self, mp: MHParams, seed: int, spot: int, g: int, l: int, j: int, pose, k: int = 0) -> np.ndarray:
        p = np.ascontiguousarray(pose, np.float32).reshape(7)
        o = np.zeros(7, np.float32)
        lib().vso_ls_proposal_k(self.h, C.byref(mp), seed, spot, g, l, k, j, _p(p, C.c_float), _p(o, C.c_float))
        return o
