"""Thin ctypes binding of libss (include/ss.h).  Argument marshalling only: every step of
the ORB extract + match path runs in the sm_100a kernels of csrc/.  There is no CPU
fallback: if libss.so is missing or no GPU is present, calls raise.

torch is used only for device memory (tensor.data_ptr()) and streams (cuda_stream handles).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libss.so")
MAX_LEVELS = 8
DESC_BYTES = 32

SS_OK, SS_EINVAL, SS_ECAPACITY, SS_ECUDA, SS_EUNSUPPORTED = 0, -1, -2, -3, -4
SS_MATCH_WINDOW, SS_MATCH_BRUTE = 0, 1
SS_DIST_QUADTREE, SS_DIST_GRID_TOPN = 0, 1
_STATUS = {0: "SS_OK", -1: "SS_EINVAL", -2: "SS_ECAPACITY", -3: "SS_ECUDA", -4: "SS_EUNSUPPORTED"}


class SSError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class ss_orb_params(C.Structure):
    _fields_ = [("width", C.c_int32), ("height", C.c_int32), ("n_features", C.c_int32),
                ("n_levels", C.c_int32), ("scale_factor", C.c_float),
                ("ini_th_fast", C.c_int32), ("min_th_fast", C.c_int32),
                ("scale", C.c_float * MAX_LEVELS), ("inv_scale", C.c_float * MAX_LEVELS),
                ("level_w", C.c_int32 * MAX_LEVELS), ("level_h", C.c_int32 * MAX_LEVELS),
                ("n_per_level", C.c_int32 * MAX_LEVELS),
                ("cell_cols", C.c_int32 * MAX_LEVELS), ("cell_rows", C.c_int32 * MAX_LEVELS),
                ("cell_w", C.c_int32 * MAX_LEVELS), ("cell_h", C.c_int32 * MAX_LEVELS),
                ("n_ini", C.c_int32 * MAX_LEVELS), ("level_cap", C.c_int32 * MAX_LEVELS),
                ("kp_capacity", C.c_int32)]

    def as_dict(self) -> dict:
        out = {}
        for name, _ in self._fields_:
            v = getattr(self, name)
            out[name] = list(v) if hasattr(v, "__len__") else v
        return out


class ss_match_cfg(C.Structure):
    _fields_ = [("mode", C.c_int32), ("th", C.c_int32), ("ratio_num", C.c_int32),
                ("ratio_den", C.c_int32), ("dedup", C.c_int32)]


class ss_tick_io(C.Structure):
    """Host-side inputs / outputs of ss_track_tick (ss.h); pointer fields take addresses."""
    _fields_ = [("frames", C.c_void_p), ("frame_stride", C.c_int64), ("pitch", C.c_int32),
                ("bf", C.c_float), ("baseline", C.c_float),
                ("cams", C.c_void_p), ("n_points", C.c_int32), ("points", C.c_void_p),
                ("point_frame", C.c_void_p), ("point_desc", C.c_void_p), ("taken", C.c_void_p),
                ("th", C.c_float), ("d_map_desc", C.c_void_p), ("n_map", C.c_int32),
                ("kps", C.c_void_p), ("desc", C.c_void_p), ("counts", C.c_void_p), ("matches", C.c_void_p),
                ("uright", C.c_void_p), ("depth", C.c_void_p),
                ("lf_offsets", C.c_void_p), ("lf_points", C.c_void_p), ("lf_desc", C.c_void_p),
                ("last_cams", C.c_void_p), ("mb", C.c_float), ("lf_th", C.c_float), ("lf_min_matches", C.c_int32),
                ("lf_matches", C.c_void_p), ("lf_n_matches", C.c_void_p), ("map_resident", C.c_int32),
                ("reuse_graph", C.c_int32), ("out_packed", C.c_void_p), ("in_packed", C.c_void_p)]


# numpy views of the 20-/20-/12-byte records of ss.h
KEYPOINT_DTYPE = np.dtype([("x", "<f4"), ("y", "<f4"), ("angle_deg", "<f4"), ("lx", "<u2"),
                           ("ly", "<u2"), ("level", "u1"), ("response", "u1"), ("reserved", "<u2")])
QUERY_DTYPE = np.dtype([("frame", "<i4"), ("u", "<f4"), ("v", "<f4"), ("pred_level", "<i4"),
                        ("radius", "<f4")])
MATCH_DTYPE = np.dtype([("idx", "<i4"), ("dist", "<i4"), ("dist2", "<i4")])
CAMERA_DTYPE = np.dtype([("R", "<f4", (9,)), ("t", "<f4", (3,)), ("ow", "<f4", (3,)), ("fx", "<f4"),
                         ("fy", "<f4"), ("cx", "<f4"), ("cy", "<f4"), ("min_x", "<f4"), ("max_x", "<f4"),
                         ("min_y", "<f4"), ("max_y", "<f4"), ("pad", "<f4")])
MAP_POINT_DTYPE = np.dtype([("pos", "<f4", (3,)), ("normal", "<f4", (3,)), ("min_dist", "<f4"),
                            ("max_dist", "<f4")])
FRAME_POINT_DTYPE = np.dtype([("pos", "<f4", (3,)), ("angle_deg", "<f4"), ("octave", "<i4"), ("reserved", "<i4")])

_lib = None


def lib():
    """Load libss.so (built by build.py).  Raises if it is missing -- no fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libss.so not built ({LIB_PATH}); run __graft_entry__.build()")
        try:  # load torch's libcudart first so that libss binds to the same CUDA runtime
            import torch  # noqa: F401
        except Exception:
            pass
        L = C.CDLL(LIB_PATH)
        P, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
        L.ss_orb_params_init.argtypes = [i32, i32, i32, i32, C.c_float, i32, i32, C.POINTER(ss_orb_params)]
        L.ss_create.argtypes = [i32, C.POINTER(ss_orb_params), i32, i32, i32, C.POINTER(P)]
        L.ss_destroy.argtypes = [P]
        L.ss_last_error.argtypes = [P]
        L.ss_last_error.restype = C.c_char_p
        L.ss_orb_extract.argtypes = [P, i32, P, i64, i32, P, P, P, P]
        L.ss_match_projection.argtypes = [P, i32, P, P, P, P, i32, P, P, i32, C.POINTER(ss_match_cfg), P, P]
        L.ss_project_points.argtypes = [P, i32, P, i32, P, P, C.c_float, P, P]
        L.ss_stereo_match.argtypes = [P, i32, P, i64, i32, P, P, P, C.c_float, C.c_float, P, P, P]
        L.ss_match_last_frame.argtypes = [P, i32, P, P, C.c_float, P, P, P, P, P, P, P, C.c_float, i32, i32, i32,
                                          P, P, P, P]
        L.ss_match_brute_partial.argtypes = [P, i32, P, P, P, i32, i32, P, P]
        L.ss_match_brute_merge.argtypes = [P, i32, P, i32, P, C.POINTER(ss_match_cfg), P, P]
        L.ss_brute_map_prepare.argtypes = [P, P, i32, P]
        L.ss_orb_extract_frames.argtypes = [P, i32, C.POINTER(P), C.POINTER(i32), P, P, P, P]
        L.ss_track_run.argtypes = [C.POINTER(P), i32, C.POINTER(P), i32, C.POINTER(ss_match_cfg),
                                   C.POINTER(ss_tick_io), i32, i32]
        L.ss_set_distribution.argtypes = [P, i32]
        L.ss_track_tick.argtypes = [P, i32, C.POINTER(ss_match_cfg), C.POINTER(ss_tick_io), P]
        L.ss_tick_packed_layout.argtypes = [P, i32, i32, i64, i32, i32, P]
        L.ss_tick_packed_in_layout.argtypes = [P, i32, i64, P]
        L.ss_debug_level.argtypes = [P, i32, i32, C.POINTER(P), C.POINTER(i32)]
        L.ss_debug_candidates.argtypes = [P, i32, i32, P, P, P, i32, C.POINTER(i32)]
        L.ss_debug_overflow_count.argtypes = [P, C.POINTER(i32)]
        L.ss_debug_distribution_paths.argtypes = [P, C.POINTER(i32), C.POINTER(i32)]
        L.ss_debug_match_lanes.argtypes = [P, i32]
        L.ss_debug_capture_samples.argtypes = [P, P]
        L.ss_profile_events.argtypes = [P, C.POINTER(P), i32]
        L.ss_debug_phase_times.argtypes = [P, i32, i32, P, i32]
        L.ss_profile_next.argtypes = [P, C.POINTER(i32)]
        for fn in ("ss_orb_params_init", "ss_create", "ss_destroy", "ss_orb_extract", "ss_match_projection",
                   "ss_project_points", "ss_stereo_match", "ss_track_tick", "ss_set_distribution",
                   "ss_match_last_frame", "ss_match_brute_partial", "ss_match_brute_merge", "ss_debug_level", "ss_debug_candidates", "ss_debug_overflow_count", "ss_profile_events",
                   "ss_profile_next", "ss_debug_phase_times", "ss_debug_distribution_paths", "ss_debug_match_lanes",
                   "ss_debug_capture_samples", "ss_brute_map_prepare", "ss_orb_extract_frames", "ss_track_run"):
            getattr(L, fn).restype = C.c_int
        _lib = L
    return _lib


EXPORTED = ("ss_orb_params_init", "ss_create", "ss_destroy", "ss_last_error", "ss_orb_extract",
            "ss_match_projection", "ss_project_points", "ss_stereo_match", "ss_track_tick", "ss_set_distribution",
            "ss_match_last_frame", "ss_match_brute_partial", "ss_match_brute_merge", "ss_profile_events", "ss_profile_next", "ss_debug_level",
            "ss_debug_candidates", "ss_debug_overflow_count", "ss_debug_phase_times", "ss_debug_distribution_paths",
            "ss_debug_match_lanes", "ss_debug_capture_samples", "ss_brute_map_prepare", "ss_orb_extract_frames",
            "ss_track_run", "ss_tick_packed_layout", "ss_tick_packed_in_layout")


def _check(status: int, ctx=None):
    if status != SS_OK:
        raise SSError(status, lib().ss_last_error(ctx).decode())


def _ptr(x) -> int | None:
    """Device pointer of a torch tensor (or int / None)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    return x.data_ptr()


def _stream(s) -> int | None:
    if s is None:
        return None
    if isinstance(s, int):
        return s
    return s.cuda_stream


# ---- same names as the C ABI --------------------------------------------------------

def ss_orb_params_init(width, height, n_features=1000, n_levels=8, scale_factor=1.2, ini_th_fast=20,
                       min_th_fast=7) -> ss_orb_params:
    p = ss_orb_params()
    _check(lib().ss_orb_params_init(width, height, n_features, n_levels, scale_factor, ini_th_fast,
                                    min_th_fast, C.byref(p)))
    return p


def ss_create(device: int, p: ss_orb_params, max_frames: int, max_queries: int = 0, max_map: int = 0) -> int:
    ctx = C.c_void_p()
    _check(lib().ss_create(device, C.byref(p), max_frames, max_queries, max_map, C.byref(ctx)))
    return ctx.value


def ss_destroy(ctx: int) -> None:
    _check(lib().ss_destroy(ctx))


def ss_last_error(ctx=None) -> str:
    return lib().ss_last_error(ctx).decode()


def ss_orb_extract(ctx, n_frames, d_frames, frame_stride, pitch, d_kps, d_desc, d_counts, stream=None):
    _check(lib().ss_orb_extract(ctx, n_frames, _ptr(d_frames), frame_stride, pitch, _ptr(d_kps),
                                _ptr(d_desc), _ptr(d_counts), _stream(stream)), ctx)


def ss_match_projection(ctx, n_frames, d_kps, d_desc, d_counts, d_kp_taken, n_queries, d_queries,
                        d_map_desc, n_map, cfg: ss_match_cfg, d_out, stream=None):
    _check(lib().ss_match_projection(ctx, n_frames, _ptr(d_kps), _ptr(d_desc), _ptr(d_counts),
                                     _ptr(d_kp_taken), n_queries, _ptr(d_queries), _ptr(d_map_desc), n_map,
                                     C.byref(cfg), _ptr(d_out), _stream(stream)), ctx)


def ss_set_distribution(ctx, mode: int) -> None:
    _check(lib().ss_set_distribution(ctx, mode), ctx)


def ss_tick_packed_layout(ctx, n_frames, n_points, n_lf, brute=False, stereo=False) -> np.ndarray:
    """Byte offsets of ss_tick_io.out_packed's sections (kps, desc, counts, lf_n_matches,
    lf_matches, matches, uright, depth) and the total (index 8)."""
    out = np.zeros(9, np.int64)
    _check(lib().ss_tick_packed_layout(ctx, n_frames, n_points, n_lf, int(brute), int(stereo), out.ctypes.data), ctx)
    return out


def ss_tick_packed_in_layout(ctx, n_frames, frame_stride) -> np.ndarray:
    """Byte offsets of ss_tick_io.in_packed's sections (frames, cams, lf_offsets) and the total."""
    out = np.zeros(4, np.int64)
    _check(lib().ss_tick_packed_in_layout(ctx, n_frames, frame_stride, out.ctypes.data), ctx)
    return out


def ss_track_tick(ctx, n_frames, cfg: ss_match_cfg, io: ss_tick_io, stream=None):
    _check(lib().ss_track_tick(ctx, n_frames, C.byref(cfg), C.byref(io), _stream(stream)), ctx)


def ss_stereo_match(ctx, n_pairs, d_frames, frame_stride, pitch, d_kps, d_desc, d_counts, bf, baseline, d_uright,
                    d_depth, stream=None):
    _check(lib().ss_stereo_match(ctx, n_pairs, _ptr(d_frames), frame_stride, pitch, _ptr(d_kps), _ptr(d_desc),
                                 _ptr(d_counts), float(bf), float(baseline), _ptr(d_uright), _ptr(d_depth),
                                 _stream(stream)), ctx)


def ss_project_points(ctx, n_frames, d_cams, n_points, d_points, d_point_frame, th, d_queries, stream=None):
    _check(lib().ss_project_points(ctx, n_frames, _ptr(d_cams), n_points, _ptr(d_points), _ptr(d_point_frame),
                                   float(th), _ptr(d_queries), _stream(stream)), ctx)


def ss_match_last_frame(ctx, n_frames, d_cams, d_last_cams, mb, d_kps, d_desc, d_counts, d_kp_taken, d_point_offsets,
                        d_points, d_point_desc, th, th_high, check_orientation, min_matches, d_out, d_n_matches=None,
                        d_kp_matched=None, stream=None):
    _check(lib().ss_match_last_frame(ctx, n_frames, _ptr(d_cams), _ptr(d_last_cams), float(mb), _ptr(d_kps),
                                     _ptr(d_desc), _ptr(d_counts), _ptr(d_kp_taken), _ptr(d_point_offsets),
                                     _ptr(d_points), _ptr(d_point_desc), float(th), int(th_high),
                                     int(check_orientation), int(min_matches), _ptr(d_out), _ptr(d_n_matches),
                                     _ptr(d_kp_matched), _stream(stream)), ctx)


def ss_match_brute_partial(ctx, n_frames, d_desc, d_counts, d_map_desc, n_map, map_offset, d_top2, stream=None):
    _check(lib().ss_match_brute_partial(ctx, n_frames, _ptr(d_desc), _ptr(d_counts), _ptr(d_map_desc), n_map,
                                        map_offset, _ptr(d_top2), _stream(stream)), ctx)


def ss_match_brute_merge(ctx, n_frames, d_counts, n_parts, d_parts, cfg: "ss_match_cfg", d_out, stream=None):
    _check(lib().ss_match_brute_merge(ctx, n_frames, _ptr(d_counts), n_parts, _ptr(d_parts), C.byref(cfg),
                                      _ptr(d_out), _stream(stream)), ctx)


def ss_profile_events(ctx, events) -> None:
    """events: list of torch.cuda.Event (timing enabled) or raw cudaEvent_t ints; [] disables."""
    handles = [e if isinstance(e, int) else e.cuda_event for e in events]
    if any(not h for h in handles):
        raise SSError(SS_EINVAL, "event not created yet (record a torch.cuda.Event once before passing it)")
    arr = (C.c_void_p * max(1, len(handles)))(*handles)
    _check(lib().ss_profile_events(ctx, arr, len(handles)), ctx)


def ss_profile_next(ctx) -> int:
    n = C.c_int32()
    _check(lib().ss_profile_next(ctx, C.byref(n)), ctx)
    return n.value


def extract_kernels(n_levels: int) -> list[str]:
    """Kernel launches of one ss_orb_extract in profiling-event order (include/ss.h)."""
    if os.environ.get("SS_FAST_SPLIT", "0") not in ("", "0"):  # level 0's FAST beside the pyramid (A/B)
        return ["fast_l0", "pyramid", "fast_l1plus", "distribute", "describe"]
    return ["pyramid", "fast", "distribute", "describe"]


def extract_events(n_levels: int) -> int:
    return 1 + 2 * len(extract_kernels(n_levels))


def match_kernels(mode: int, dedup: bool = True) -> list[str]:
    if mode == SS_MATCH_BRUTE:
        return ["brute_expand", "brute_tc", "brute_merge"]
    return ["match_prepare", "match_window"] + (["match_resolve"] if dedup else [])


def match_events(mode: int, dedup: bool = True) -> int:
    return 2 * len(match_kernels(mode, dedup))


def ss_debug_level(ctx, frame, level):
    ptr, pitch = C.c_void_p(), C.c_int32()
    _check(lib().ss_debug_level(ctx, frame, level, C.byref(ptr), C.byref(pitch)), ctx)
    return ptr.value, pitch.value


def ss_debug_candidates(ctx, frame, level, cap=1 << 21):
    lx, ly, sc = (np.zeros(cap, np.int32) for _ in range(3))
    n = C.c_int32()
    _check(lib().ss_debug_candidates(ctx, frame, level, lx.ctypes.data, ly.ctypes.data, sc.ctypes.data, cap,
                                     C.byref(n)), ctx)
    return lx[:n.value].copy(), ly[:n.value].copy(), sc[:n.value].copy()


def ss_debug_phase_times(ctx, frame, level, n=10) -> np.ndarray:
    out = np.zeros(n, np.int64)
    _check(lib().ss_debug_phase_times(ctx, frame, level, out.ctypes.data, n), ctx)
    return out


def ss_debug_overflow_count(ctx) -> int:
    n = C.c_int32()
    _check(lib().ss_debug_overflow_count(ctx, C.byref(n)), ctx)
    return n.value


class TrackRun:
    """Marshalled arguments of ss_track_run (built once, run many times): ctxs / streams [P],
    ios [P][n_io] (ss_tick_io structures)."""

    def __init__(self, ctxs, streams, n_frames: int, cfg: "ss_match_cfg", ios):
        P, n_io = len(ctxs), len(ios[0])
        self.ctxs = (C.c_void_p * P)(*ctxs)
        self.streams = (C.c_void_p * P)(*[_stream(s) for s in streams])
        self.ios = (ss_tick_io * (P * n_io))(*[io for row in ios for io in row])
        self.cfg, self.n_frames, self.P, self.n_io = cfg, n_frames, P, n_io

    def run(self, n_ticks: int) -> None:
        _check(lib().ss_track_run(self.ctxs, self.P, self.streams, self.n_frames, C.byref(self.cfg), self.ios,
                                  self.n_io, n_ticks))


def ss_orb_extract_frames(ctx, frames, d_kps, d_desc, d_counts, stream=None):
    """frames: list of uint8 CUDA tensors [H, pitch] (one per client, separately allocated)."""
    n = len(frames)
    ptrs = (C.c_void_p * max(n, 1))(*[f.data_ptr() for f in frames])
    pitches = (C.c_int32 * max(n, 1))(*[f.stride(0) for f in frames])
    _check(lib().ss_orb_extract_frames(ctx, n, ptrs, pitches, _ptr(d_kps), _ptr(d_desc), _ptr(d_counts),
                                       _stream(stream)), ctx)


def ss_brute_map_prepare(ctx, d_map_desc, n_map: int, stream=None) -> None:
    _check(lib().ss_brute_map_prepare(ctx, _ptr(d_map_desc), n_map, _stream(stream)), ctx)


def ss_debug_distribution_paths(ctx) -> tuple[int, int]:
    """(sort fallbacks, global-memory distributions) of the last extract."""
    a, b = C.c_int32(), C.c_int32()
    _check(lib().ss_debug_distribution_paths(ctx, C.byref(a), C.byref(b)), ctx)
    return a.value, b.value


def ss_debug_match_lanes(ctx, lanes: int) -> None:
    _check(lib().ss_debug_match_lanes(ctx, lanes), ctx)


def ss_debug_capture_samples(ctx, d_samples) -> None:
    """d_samples: uint8 CUDA tensor of n_frames * kp_capacity * 512 bytes, or None to stop."""
    _check(lib().ss_debug_capture_samples(ctx, _ptr(d_samples)), ctx)


def window_cfg(th=100, ratio_num=4, ratio_den=5, dedup=1) -> ss_match_cfg:
    return ss_match_cfg(SS_MATCH_WINDOW, th, ratio_num, ratio_den, dedup)


def brute_cfg(th=50, ratio_num=3, ratio_den=4) -> ss_match_cfg:
    return ss_match_cfg(SS_MATCH_BRUTE, th, ratio_num, ratio_den, 0)
