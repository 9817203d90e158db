"""Python binding of the C-ABI library libvs.so (include/vs.h).

Argument marshalling only: every step of the hot path (list building, pose
generation, scoring, local search, selection) runs in the CUDA kernels of
libvs.so.  There is no CPU fallback: if the library cannot be loaded this
module raises.  torch is used only to hand device pointers and streams to the
``*_device`` / ``*_async`` entry points.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import build as _build

OK, ERR_INVALID_ARGUMENT, ERR_POSE_OUT_OF_REGION, ERR_ZERO_QUATERNION, ERR_CUDA, ERR_OUT_OF_MEMORY, ERR_UNSUPPORTED = range(7)
TIMING_EVENTS, TIMING_KERNEL, TIMING_CENSUS = 1, 2, 4   # vs_set_timing flags (include/vs.h)
TRACE_INIT, TRACE_SCORED, TRACE_SELECT, TRACE_LS, TRACE_SORTED, TRACE_COMBINED, TRACE_INCLUDED = range(7)

# every symbol include/vs.h declares (checked by tests/test_abi.py)
EXPORTS = ["vs_score_params_default", "vs_mh_preset", "vs_create", "vs_score_poses", "vs_score_poses_device",
           "vs_run", "vs_run_async", "vs_destroy", "vs_last_error", "vs_abi_version", "vs_set_timing",
           "vs_get_stats", "vs_reset_stats", "vs_list_lengths", "vs_run_trace", "vs_debug_philox",
           "vs_release_cached_memory", "vs_pair_intervals"]


def release_cached_memory(device: int = -1) -> None:
    """Return the device memory cached from destroyed contexts to the driver (vs_release_cached_memory)."""
    L = load()
    st = L.vs_release_cached_memory(device)
    if st != 0:
        raise VSError(st, L.vs_last_error().decode())


class VSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"vs status {status}: {msg}")
        self.status = status


class ScoreParams(C.Structure):
    _fields_ = [("coulomb_k", C.c_float), ("dielectric", C.c_int), ("eps_r", C.c_float), ("cutoff", C.c_float),
                ("region_half_width", C.c_float), ("hb_eps", C.c_float), ("hb_r0", C.c_float),
                ("r2_min", C.c_float), ("n_types", C.c_int), ("type_sigma", C.POINTER(C.c_float)),
                ("type_eps", C.POINTER(C.c_float)), ("type_hb_role", C.POINTER(C.c_int)),
                ("list_splits", C.c_int)]


class MHParams(C.Structure):
    _fields_ = [("population", C.c_int), ("generations", C.c_int), ("ls_steps", C.c_int),
                ("improve_frac", C.c_float), ("p_mut", C.c_float), ("mut_trans", C.c_float),
                ("mut_rot", C.c_float), ("ls_trans", C.c_float), ("ls_rot", C.c_float),
                ("ls_neighbours", C.c_int)]


class Stats(C.Structure):
    _fields_ = [("kernel_launches", C.c_uint64), ("score_launches", C.c_uint64), ("poses_scored", C.c_uint64),
                ("pairs", C.c_uint64), ("score_ms", C.c_double), ("timed_launches", C.c_uint64),
                ("pairs_evaluated", C.c_uint64), ("pairs_within", C.c_uint64), ("pair_busy_ms", C.c_double),
                ("pair_launch_ms", C.c_double), ("pair_timed_launches", C.c_uint64), ("pair_warp_ms", C.c_double)]

    def asdict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


TRACE_FN = C.CFUNCTYPE(None, C.c_void_p, C.c_int32, C.c_int32, C.c_int32, C.c_int32, C.c_int32,
                       C.POINTER(C.c_float), C.POINTER(C.c_int32))

_lib = None


def library_path() -> str:
    return os.environ.get("VS_LIB") or _build.LIB


def load(build_if_stale: bool = True):
    """Load libvs.so (building it with nvcc first if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("VS_LIB") or _build.LIB
    if os.environ.get("VS_LIB"):
        build_if_stale = False
    if build_if_stale:
        try:
            path = _build.build()
        except (OSError, RuntimeError) as e:  # no nvcc here: use the shipped .so if any
            if not os.path.exists(path):
                raise RuntimeError(f"libvs.so is missing and could not be built: {e}") from e
    if not os.path.exists(path):
        raise RuntimeError(f"libvs.so not found at {path}; run paper_conf_ppopp_imbernoncg16_b200/build.py")
    L = C.CDLL(path)
    f32p, i32p, u32p, vp = C.POINTER(C.c_float), C.POINTER(C.c_int32), C.POINTER(C.c_uint32), C.c_void_p
    L.vs_score_params_default.argtypes = [C.POINTER(ScoreParams)]
    L.vs_score_params_default.restype = None
    L.vs_mh_preset.argtypes = [C.c_int, C.POINTER(MHParams)]
    L.vs_create.argtypes = [f32p, f32p, i32p, C.c_int32, f32p, f32p, i32p, C.c_int32, f32p, C.c_int32,
                            C.POINTER(ScoreParams), C.c_int32, C.POINTER(vp)]
    L.vs_score_poses.argtypes = [vp, C.c_int64, i32p, f32p, f32p, f32p]
    L.vs_score_poses_device.argtypes = [vp, C.c_int64, vp, vp, vp, vp, vp]
    L.vs_run.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, i32p, f32p, f32p]
    L.vs_run_async.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, i32p, vp, vp, vp]
    L.vs_run_trace.argtypes = [vp, C.POINTER(MHParams), C.c_uint64, C.c_int32, i32p, f32p, f32p, TRACE_FN, vp]
    L.vs_destroy.argtypes = [vp]
    L.vs_destroy.restype = None
    L.vs_release_cached_memory.argtypes = [C.c_int32]
    L.vs_release_cached_memory.restype = C.c_int
    L.vs_last_error.restype = C.c_char_p
    L.vs_abi_version.restype = C.c_int
    L.vs_set_timing.argtypes = [vp, C.c_int]
    L.vs_get_stats.argtypes = [vp, C.POINTER(Stats)]
    L.vs_reset_stats.argtypes = [vp]
    L.vs_list_lengths.argtypes = [vp, i32p]
    L.vs_pair_intervals.argtypes = [vp, C.POINTER(C.c_uint64), C.c_int64]
    L.vs_pair_intervals.restype = C.c_int64
    L.vs_debug_philox.argtypes = [C.c_int64, u32p, u32p, u32p]
    _lib = L
    return L


def _p(a, ctype):
    return a.ctypes.data_as(C.POINTER(ctype)) if a is not None else None


def _check(st: int):
    if st != OK:
        raise VSError(st, load().vs_last_error().decode())


def score_params(**kw) -> ScoreParams:
    sp = ScoreParams()
    load().vs_score_params_default(C.byref(sp))
    for k, v in kw.items():
        setattr(sp, k, v)
    return sp


def mh_preset(m: int, **kw) -> MHParams:
    mp = MHParams()
    _check(load().vs_mh_preset(m, C.byref(mp)))
    for k, v in kw.items():
        setattr(mp, k, v)
    return mp


def debug_philox(ctr, key) -> np.ndarray:
    c = np.ascontiguousarray(ctr, np.uint32).reshape(-1, 4)
    k = np.ascontiguousarray(key, np.uint32)
    o = np.zeros_like(c)
    _check(load().vs_debug_philox(len(c), _p(c, C.c_uint32), _p(k, C.c_uint32), _p(o, C.c_uint32)))
    return o


def _stream_handle(stream):
    if stream is None:
        import torch
        return C.c_void_p(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return C.c_void_p(stream)
    return C.c_void_p(stream.cuda_stream)


class Context:
    """vs_create ... vs_destroy on one CUDA device."""

    def __init__(self, rec_xyz, rec_q, rec_type, lig_xyz, lig_q, lig_type, spot_xyz,
                 sp: ScoreParams | None = None, device: int = 0):
        self.h = None
        L = load()
        arrs = [np.ascontiguousarray(rec_xyz, np.float32), np.ascontiguousarray(rec_q, np.float32),
                np.ascontiguousarray(rec_type, np.int32), np.ascontiguousarray(lig_xyz, np.float32),
                np.ascontiguousarray(lig_q, np.float32), np.ascontiguousarray(lig_type, np.int32),
                np.ascontiguousarray(spot_xyz, np.float32)]
        rx, rq, rt, lx, lq, lt, sx = arrs
        self.n_rec, self.n_lig, self.n_spots = len(rq), len(lq), len(sx)
        self.sp = sp if sp is not None else score_params()
        self.device = device
        h = C.c_void_p()
        _check(L.vs_create(_p(rx, C.c_float), _p(rq, C.c_float), _p(rt, C.c_int32), self.n_rec,
                           _p(lx, C.c_float), _p(lq, C.c_float), _p(lt, C.c_int32), self.n_lig,
                           _p(sx, C.c_float), self.n_spots, C.byref(self.sp), device, C.byref(h)))
        self.h = h
        # H2D bytes of vs_create (for end-to-end accounting)
        self.create_h2d_bytes = sum(a.nbytes for a in arrs)

    @classmethod
    def from_problem(cls, prob, sp=None, device: int = 0, ligand=None):
        lig = ligand if ligand is not None else prob.lig
        return cls(prob.rec.xyz, prob.rec.q, prob.rec.type, lig.xyz, lig.q, lig.type, prob.spots, sp, device)

    def close(self):
        if getattr(self, "h", None):
            try:
                load().vs_destroy(self.h)
            except TypeError:  # interpreter shutdown: module globals already torn down
                pass
            self.h = None

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ---- scoring
    def score_poses(self, spot, q, t) -> np.ndarray:
        spot = np.ascontiguousarray(spot, np.int32)
        q = np.ascontiguousarray(q, np.float32)
        t = np.ascontiguousarray(t, np.float32)
        out = np.zeros(len(spot), np.float32)
        _check(load().vs_score_poses(self.h, len(spot), _p(spot, C.c_int32), _p(q, C.c_float), _p(t, C.c_float),
                                     _p(out, C.c_float)))
        return out

    def score_poses_device(self, spot, q, t, out, stream=None):
        """torch tensors on this ctx's device: int32 [n], f32 [n,4], f32 [n,3], f32 [n]."""
        n = spot.numel()
        _check(load().vs_score_poses_device(self.h, n, C.c_void_p(spot.data_ptr()), C.c_void_p(q.data_ptr()),
                                            C.c_void_p(t.data_ptr()), C.c_void_p(out.data_ptr()),
                                            _stream_handle(stream)))

    # ---- metaheuristic
    def run(self, mp: MHParams, seed: int, spot_ids=None):
        ids = None if spot_ids is None else np.ascontiguousarray(spot_ids, np.int32)
        n = self.n_spots if ids is None else len(ids)
        pose = np.zeros((n, 7), np.float32)
        sc = np.zeros(n, np.float32)
        _check(load().vs_run(self.h, C.byref(mp), seed, 0 if ids is None else n, _p(ids, C.c_int32),
                             _p(pose, C.c_float), _p(sc, C.c_float)))
        return pose, sc

    def run_async(self, mp: MHParams, seed: int, spot_ids, best_pose, best_score, stream=None):
        """best_pose: f32 [n,7], best_score: f32 [n] torch tensors on the device."""
        ids = None if spot_ids is None else np.ascontiguousarray(spot_ids, np.int32)
        n = self.n_spots if ids is None else len(ids)
        _check(load().vs_run_async(self.h, C.byref(mp), seed, 0 if ids is None else n, _p(ids, C.c_int32),
                                   C.c_void_p(best_pose.data_ptr()), C.c_void_p(best_score.data_ptr()),
                                   _stream_handle(stream)))

    def run_trace(self, mp: MHParams, seed: int, spot_ids, callback):
        """callback(stage, g, l, poses8 [n_sel, count, 8] or None, idx [n_sel, count] or None)."""
        ids = None if spot_ids is None else np.ascontiguousarray(spot_ids, np.int32)
        n = self.n_spots if ids is None else len(ids)
        pose = np.zeros((n, 7), np.float32)
        sc = np.zeros(n, np.float32)

        def _cb(user, stage, g, l, n_sel, count, poses8, idx):
            P = np.ctypeslib.as_array(poses8, (n_sel, count, 8)).copy() if poses8 else None
            I = np.ctypeslib.as_array(idx, (n_sel, count)).copy() if idx else None
            callback(stage, g, l, P, I)

        fn = TRACE_FN(_cb)
        _check(load().vs_run_trace(self.h, C.byref(mp), seed, 0 if ids is None else n, _p(ids, C.c_int32),
                                   _p(pose, C.c_float), _p(sc, C.c_float), fn, None))
        return pose, sc

    # ---- instrumentation
    def set_timing(self, enable=True):
        """enable: bool (CUDA events around un-graphed scoring calls) or an OR of TIMING_* flags."""
        flags = int(enable) if not isinstance(enable, bool) else (TIMING_EVENTS if enable else 0)
        _check(load().vs_set_timing(self.h, flags))

    def stats(self) -> dict:
        s = Stats()
        _check(load().vs_get_stats(self.h, C.byref(s)))
        return s.asdict()

    def reset_stats(self):
        _check(load().vs_reset_stats(self.h))

    def pair_intervals(self) -> np.ndarray:
        """[n, 2] uint64 (start, end) device-globaltimer ns of the pair kernel's launches (VS_TIMING_KERNEL)."""
        L = load()
        n = L.vs_pair_intervals(self.h, None, 0)
        if n < 0:
            raise VSError(ERR_CUDA, L.vs_last_error().decode())
        out = np.zeros((max(n, 1), 2), np.uint64)
        n = L.vs_pair_intervals(self.h, out.ctypes.data_as(C.POINTER(C.c_uint64)), len(out))
        if n < 0:
            raise VSError(ERR_CUDA, L.vs_last_error().decode())
        return out[:min(n, len(out))]

    def list_lengths(self) -> np.ndarray:
        o = np.zeros(self.n_spots, np.int32)
        _check(load().vs_list_lengths(self.h, _p(o, C.c_int32)))
        return o
