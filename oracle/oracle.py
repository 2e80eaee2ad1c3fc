"""ctypes wrapper of oracle/ss_oracle.c (TEST INFRASTRUCTURE ONLY -- see oracle/__init__.py).

Every function here is argument marshalling around the C oracle; the arithmetic and its
citations live in ss_oracle.c.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ss_oracle.c")
_LIB_PATH = os.path.join(_HERE, "libss_oracle.so")
MAX_LEVELS = 8


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc (-O2 -ffp-contract=off, no SIMD/OpenMP)."""
    deps = [_SRC, os.path.join(_HERE, "ss_oracle.h"), os.path.join(_HERE, "brief_pattern_ref.inc")]
    if not force and os.path.exists(_LIB_PATH):
        if os.path.getmtime(_LIB_PATH) >= max(os.path.getmtime(d) for d in deps):
            return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-std=c99", "-fPIC", "-shared",
                           "-Wall", "-o", tmp, _SRC, "-lm"])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


class RefParams(C.Structure):
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
assert FRAME_POINT_DTYPE.itemsize == 24
assert CAMERA_DTYPE.itemsize == 96 and MAP_POINT_DTYPE.itemsize == 32
assert KEYPOINT_DTYPE.itemsize == 20 and QUERY_DTYPE.itemsize == 20 and MATCH_DTYPE.itemsize == 12

_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        P = C.c_void_p
        i32, i64 = C.c_int32, C.c_int64
        _lib.ref_params_init.argtypes = [i32, i32, i32, i32, C.c_float, i32, i32, C.POINTER(RefParams)]
        _lib.ref_resize_linear_exact.argtypes = [P, C.c_int, C.c_int, C.c_int, P, C.c_int, C.c_int, C.c_int]
        _lib.ref_pyramid_bytes.argtypes = [C.POINTER(RefParams)]
        _lib.ref_pyramid_bytes.restype = i64
        _lib.ref_pyramid.argtypes = [C.POINTER(RefParams), P, C.c_int, P]
        _lib.ref_fast_M.argtypes = [P, C.c_int, C.c_int, C.c_int, P]
        _lib.ref_cell_candidates.argtypes = [C.POINTER(RefParams), C.c_int, P, P, P, P, C.c_int]
        _lib.ref_distribute.argtypes = [P, P, P, C.c_int, C.c_int, C.c_int, C.c_int, P]
        _lib.ref_moments.argtypes = [P, C.c_int, C.c_int, C.c_int, C.POINTER(i32), C.POINTER(i32)]
        _lib.ref_angle_deg.argtypes = [i32, i32]
        _lib.ref_angle_deg.restype = C.c_float
        _lib.ref_blur.argtypes = [P, C.c_int, C.c_int, C.c_int, P, C.c_int]
        _lib.ref_rhe_div_sqrt.argtypes = [i64, i64]
        _lib.ref_rhe_div_sqrt.restype = i32
        _lib.ref_descriptor.argtypes = [P, C.c_int, C.c_int, C.c_int, i32, i32, P]
        _lib.ref_orb_extract.argtypes = [C.POINTER(RefParams), P, C.c_int, P, P, P]
        _lib.ref_orb_extract_mode.argtypes = [C.POINTER(RefParams), P, C.c_int, C.c_int, P, P, P]
        _lib.ref_distribute_grid.argtypes = [C.POINTER(RefParams), C.c_int, P, P, P, C.c_int, C.c_int, P]
        _lib.ref_hamming.argtypes = [P, P]
        _lib.ref_hamming.restype = i32
        _lib.ref_match_window.argtypes = [C.POINTER(RefParams), C.c_int, P, P, P, P, C.c_int, P, P,
                                          C.c_int, C.c_int, C.c_int, C.c_int, P]
        _lib.ref_match_brute.argtypes = [C.POINTER(RefParams), C.c_int, P, P, C.c_int, P, C.c_int,
                                         C.c_int, C.c_int, C.c_int, C.c_int, P]
        _lib.ref_stereo_match.argtypes = [C.POINTER(RefParams), P, P, C.c_int, P, P, P, P, P, P, C.c_float, C.c_float,
                                          P, P, P]
        _lib.ref_match_last_frame.argtypes = [C.POINTER(RefParams), C.c_int, P, P, C.c_float, P, P, P, P, P, P, P,
                                              C.c_float, C.c_int, C.c_int, C.c_int, P, P]
        _lib.ref_lf_rot_bin.argtypes = [C.c_float, C.c_float]
        _lib.ref_lf_rot_bin.restype = C.c_int
        _lib.ref_project_points.argtypes = [C.POINTER(RefParams), C.c_int, P, C.c_int, P, P, C.c_float, P]
    return _lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"], "oracle arrays must be C-contiguous"
    return a.ctypes.data_as(C.c_void_p)


def params(width, height, n_features=1000, n_levels=8, scale_factor=1.2, ini_th=20, min_th=7) -> RefParams:
    p = RefParams()
    rc = lib().ref_params_init(width, height, n_features, n_levels, scale_factor, ini_th, min_th, C.byref(p))
    if rc != 0:
        raise ValueError(f"ref_params_init rejected {(width, height, n_features, n_levels)}")
    return p


def resize_linear_exact(src: np.ndarray, dw: int, dh: int) -> np.ndarray:
    src = np.ascontiguousarray(src, dtype=np.uint8)
    dst = np.zeros((dh, dw), np.uint8)
    lib().ref_resize_linear_exact(_p(src), src.shape[1], src.shape[0], src.shape[1], _p(dst), dw, dh, dw)
    return dst


def pyramid(p: RefParams, img: np.ndarray) -> list[np.ndarray]:
    img = np.ascontiguousarray(img, dtype=np.uint8)
    buf = np.zeros(lib().ref_pyramid_bytes(C.byref(p)), np.uint8)
    lib().ref_pyramid(C.byref(p), _p(img), img.shape[1], _p(buf))
    out, off = [], 0
    for l in range(p.n_levels):
        w, h = p.level_w[l], p.level_h[l]
        out.append(buf[off:off + w * h].reshape(h, w).copy())
        off += w * h
    return out


def fast_M(img: np.ndarray) -> np.ndarray:
    img = np.ascontiguousarray(img, dtype=np.uint8)
    h, w = img.shape
    out = np.zeros((h, w), np.uint8)
    lib().ref_fast_M(_p(img), w, h, w, _p(out))
    return out


def cell_candidates(p: RefParams, level: int, M: np.ndarray):
    """-> (lx, ly, M) int32 arrays in rank order (cells row-major, then y, then x)."""
    M = np.ascontiguousarray(M, dtype=np.uint8)
    cap = M.size
    lx, ly, sc = (np.zeros(cap, np.int32) for _ in range(3))
    n = lib().ref_cell_candidates(C.byref(p), level, _p(M), _p(lx), _p(ly), _p(sc), cap)
    assert n >= 0
    return lx[:n].copy(), ly[:n].copy(), sc[:n].copy()


def distribute(kx, ky, score, width, height, N) -> np.ndarray:
    """Indices of the kept keys (ORB-SLAM DistributeOctTree reading, S8c O4), sorted."""
    kx, ky, score = (np.ascontiguousarray(a, dtype=np.int32) for a in (kx, ky, score))
    n = len(kx)
    out = np.zeros(max(n, 1), np.int32)
    m = lib().ref_distribute(_p(kx), _p(ky), _p(score), n, width, height, N, _p(out))
    assert m >= 0
    return np.sort(out[:m])


def moments(img: np.ndarray, lx: int, ly: int):
    img = np.ascontiguousarray(img, dtype=np.uint8)
    a, b = C.c_int32(), C.c_int32()
    lib().ref_moments(_p(img), img.shape[1], lx, ly, C.byref(a), C.byref(b))
    return a.value, b.value


def angle_deg(m10: int, m01: int) -> float:
    return float(lib().ref_angle_deg(m10, m01))


def blur(img: np.ndarray) -> np.ndarray:
    img = np.ascontiguousarray(img, dtype=np.uint8)
    h, w = img.shape
    out = np.zeros((h, w), np.uint8)
    lib().ref_blur(_p(img), w, h, w, _p(out), w)
    return out


def rhe_div_sqrt(z: int, r2: int) -> int:
    return int(lib().ref_rhe_div_sqrt(z, r2))


def descriptor(blurred: np.ndarray, lx: int, ly: int, m10: int, m01: int) -> np.ndarray:
    blurred = np.ascontiguousarray(blurred, dtype=np.uint8)
    out = np.zeros(32, np.uint8)
    lib().ref_descriptor(_p(blurred), blurred.shape[1], lx, ly, m10, m01, _p(out))
    return out


def orb_extract(p: RefParams, img: np.ndarray, mode: int = 0):
    """One frame -> (keypoints[kp_capacity] KEYPOINT_DTYPE, desc[kp_capacity,32], counts[L+1]).
    mode 0 = quadtree distribution (O4), 1 = grid top-N (O4g)."""
    img = np.ascontiguousarray(img, dtype=np.uint8)
    kps = np.zeros(p.kp_capacity, KEYPOINT_DTYPE)
    desc = np.zeros((p.kp_capacity, 32), np.uint8)
    counts = np.zeros(p.n_levels + 1, np.int32)
    n = lib().ref_orb_extract_mode(C.byref(p), _p(img), img.shape[1], mode, _p(kps), _p(desc), _p(counts))
    if n < 0:
        raise RuntimeError("oracle extraction exceeded capacity")
    return kps, desc, counts


def orb_extract_batch(p: RefParams, frames: np.ndarray, mode: int = 0):
    """frames [B,H,W] -> kps [B,cap], desc [B,cap,32], counts [B,L+1]."""
    B = frames.shape[0]
    kps = np.zeros((B, p.kp_capacity), KEYPOINT_DTYPE)
    desc = np.zeros((B, p.kp_capacity, 32), np.uint8)
    counts = np.zeros((B, p.n_levels + 1), np.int32)
    for b in range(B):
        kps[b], desc[b], counts[b] = orb_extract(p, frames[b], mode)
    return kps, desc, counts


def hamming(a: np.ndarray, b: np.ndarray) -> int:
    a = np.ascontiguousarray(a, dtype=np.uint8)
    b = np.ascontiguousarray(b, dtype=np.uint8)
    return int(lib().ref_hamming(_p(a), _p(b)))


def match_window(p: RefParams, kps, desc, counts, taken, queries, qdesc, th=100, ratio_num=4,
                 ratio_den=5, dedup=1) -> np.ndarray:
    kps = np.ascontiguousarray(kps)
    desc = np.ascontiguousarray(desc, dtype=np.uint8)
    counts = np.ascontiguousarray(counts, dtype=np.int32)
    queries = np.ascontiguousarray(queries)
    qdesc = np.ascontiguousarray(qdesc, dtype=np.uint8)
    F = kps.shape[0]
    out = np.zeros(len(queries), MATCH_DTYPE)
    tk = None if taken is None else np.ascontiguousarray(taken, dtype=np.uint8)
    lib().ref_match_window(C.byref(p), F, _p(kps), _p(desc), _p(counts),
                           None if tk is None else _p(tk), len(queries), _p(queries), _p(qdesc),
                           th, ratio_num, ratio_den, dedup, _p(out))
    return out


def match_brute(p: RefParams, desc, counts, map_desc, th=50, ratio_num=3, ratio_den=4, k0=0, k1=None):
    """-> MATCH_DTYPE [F, kp_capacity]; only keypoints k in [k0, k1) are evaluated (sampling)."""
    desc = np.ascontiguousarray(desc, dtype=np.uint8)
    counts = np.ascontiguousarray(counts, dtype=np.int32)
    map_desc = np.ascontiguousarray(map_desc, dtype=np.uint8)
    F = desc.shape[0]
    out = np.zeros((F, p.kp_capacity), MATCH_DTYPE)
    out["idx"] = -1
    out["dist"] = 256
    out["dist2"] = 256
    k1 = p.kp_capacity if k1 is None else k1
    lib().ref_match_brute(C.byref(p), F, _p(desc), _p(counts), len(map_desc), _p(map_desc), th,
                          ratio_num, ratio_den, k0, k1, _p(out))
    return out


def project_points(p: RefParams, cams, points, point_frame, th=1.0):
    """O11: -> QUERY_DTYPE [n_points] (pred_level -1 / radius 0 = outside the frustum)."""
    cams = np.ascontiguousarray(cams, dtype=CAMERA_DTYPE)
    points = np.ascontiguousarray(points, dtype=MAP_POINT_DTYPE)
    point_frame = np.ascontiguousarray(point_frame, dtype=np.int32)
    out = np.zeros(len(points), QUERY_DTYPE)
    lib().ref_project_points(C.byref(p), len(cams), _p(cams), len(points), _p(points), _p(point_frame),
                             float(th), _p(out))
    return out


def stereo_match(p: RefParams, left, right, kl, dl, cl, kr, dr, cr, bf, b):
    """O12: one rectified pair -> (uright[cap] f32, depth[cap] f32, sad[cap] i32), -1 = none."""
    left = np.ascontiguousarray(left, dtype=np.uint8)
    right = np.ascontiguousarray(right, dtype=np.uint8)
    assert left.shape == right.shape
    cap = p.kp_capacity
    ur = np.full(cap, -1.0, np.float32)
    dp = np.full(cap, -1.0, np.float32)
    sad = np.full(cap, -1, np.int32)
    args = [np.ascontiguousarray(a) for a in (kl, dl, cl, kr, dr, cr)]
    lib().ref_stereo_match(C.byref(p), _p(left), _p(right), left.shape[1], *[_p(a) for a in args],
                           float(bf), float(b), _p(ur), _p(dp), _p(sad))
    return ur, dp, sad


def distribute_grid(p: RefParams, level: int, lx, ly, score, N: int) -> np.ndarray:
    """O4g: indices (into the rank-ordered candidates) of the keys grid top-N keeps."""
    lx, ly, score = (np.ascontiguousarray(a, dtype=np.int32) for a in (lx, ly, score))
    out = np.zeros(max(len(lx), 1), np.int32)
    n = lib().ref_distribute_grid(C.byref(p), level, _p(lx), _p(ly), _p(score), len(lx), N, _p(out))
    return out[:n]


def match_last_frame(p: RefParams, cams, last_cams, mb, kps, desc, counts, taken, pt_off, points, pdesc, th=15.0,
                     th_high=100, check_orientation=1, min_matches=20):
    """O13: -> (MATCH_DTYPE [n_points], kept matches per frame i32 [F])."""
    cams = np.ascontiguousarray(cams, dtype=CAMERA_DTYPE)
    lc = None if last_cams is None else np.ascontiguousarray(last_cams, dtype=CAMERA_DTYPE)
    kps = np.ascontiguousarray(kps)
    desc = np.ascontiguousarray(desc, dtype=np.uint8)
    counts = np.ascontiguousarray(counts, dtype=np.int32)
    tk = None if taken is None else np.ascontiguousarray(taken, dtype=np.uint8)
    pt_off = np.ascontiguousarray(pt_off, dtype=np.int32)
    points = np.ascontiguousarray(points, dtype=FRAME_POINT_DTYPE)
    pdesc = np.ascontiguousarray(pdesc, dtype=np.uint8).reshape(-1, 32)
    F = len(cams)
    assert len(pt_off) == F + 1 and pt_off[-1] == len(points) == len(pdesc)
    out = np.zeros(len(points), MATCH_DTYPE)
    nm = np.zeros(F, np.int32)
    lib().ref_match_last_frame(C.byref(p), F, _p(cams), None if lc is None else _p(lc), float(mb), _p(kps), _p(desc),
                               _p(counts), None if tk is None else _p(tk), _p(pt_off), _p(points), _p(pdesc),
                               float(th), int(th_high), int(check_orientation), int(min_matches), _p(out), _p(nm))
    return out, nm


def lf_rot_bin(angle_last: float, angle_cur: float) -> int:
    return int(lib().ref_lf_rot_bin(float(angle_last), float(angle_cur)))
