"""Synthetic textured frames and map-point queries (SURVEY.md §8(d) recipe).

Frames: uniform base U(80,170) + bicubic-upsampled value noise (cells 96/24/6 px,
amplitudes 40/30/20) + ~400*(W*H/360960) opaque convex polygons (radius U(5,40), 3-6
vertices, gray U(30,225)) + two flat 100x80 patches (force the minTh fallback) +
N(0,3) pixel noise, rounded and clipped.  Seeds: splitmix64(cfg<<40 | client<<20 | frame)
into numpy PCG64.  KITTI right image = left warped by a piecewise-constant disparity
field (0..48 px) + N(0,2).
"""
from __future__ import annotations

import cv2
import numpy as np

SHAPES = {"euroc": (752, 480), "tum": (640, 480), "kitti": (1241, 376)}
_MASK64 = (1 << 64) - 1


def _splitmix64(x: int) -> int:
    x = (x + 0x9E3779B97F4A7C15) & _MASK64
    z = x
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _MASK64
    return z ^ (z >> 31)


def frame_seed(cfg: int, client: int, frame: int) -> int:
    return _splitmix64((cfg << 40) | (client << 20) | frame)


def _rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def _value_noise(rng, w, h, cell, amp):
    gw, gh = w // cell + 3, h // cell + 3
    g = rng.uniform(-1.0, 1.0, size=(gh, gw)).astype(np.float32)
    up = cv2.resize(g, (gw * cell, gh * cell), interpolation=cv2.INTER_CUBIC)
    return amp * up[:h, :w]


def make_frame(width: int, height: int, seed: int) -> np.ndarray:
    rng = _rng(seed)
    img = np.full((height, width), rng.uniform(80, 170), np.float32)
    for cell, amp in ((96, 40.0), (24, 30.0), (6, 20.0)):
        img += _value_noise(rng, width, height, cell, amp)
    img = np.clip(img, 0, 255)
    n_poly = int(round(400 * width * height / 360960.0))
    for _ in range(n_poly):
        cx, cy = rng.uniform(0, width), rng.uniform(0, height)
        r = rng.uniform(5, 40)
        nv = int(rng.integers(3, 7))
        ang = np.sort(rng.uniform(0, 2 * np.pi, nv))
        pts = np.stack([cx + r * np.cos(ang), cy + r * np.sin(ang)], 1).round().astype(np.int32)
        cv2.fillPoly(img, [pts], float(rng.uniform(30, 225)))
    for _ in range(2):
        x0 = int(rng.integers(0, max(1, width - 100)))
        y0 = int(rng.integers(0, max(1, height - 80)))
        img[y0:y0 + 80, x0:x0 + 100] = rng.uniform(60, 200)
    img += rng.normal(0.0, 3.0, size=img.shape).astype(np.float32)
    return np.clip(np.rint(img), 0, 255).astype(np.uint8)


def make_frames(width: int, height: int, n: int, cfg: int = 0, client0: int = 0, frame0: int = 0,
                per_client: bool = True) -> np.ndarray:
    """n frames: client c = client0 + i (per_client) or frame index frame0 + i."""
    out = np.empty((n, height, width), np.uint8)
    for i in range(n):
        c, f = (client0 + i, frame0) if per_client else (client0, frame0 + i)
        out[i] = make_frame(width, height, frame_seed(cfg, c, f))
    return out


def make_stereo_pair(width: int, height: int, seed: int):
    left = make_frame(width, height, seed)
    rng = _rng(seed ^ 0x5EED)
    right = np.empty_like(left)
    band = 0
    while band < height:
        bh = int(rng.integers(16, 64))
        xs = 0
        while xs < width:
            bw = int(rng.integers(32, 160))
            disp = int(rng.integers(0, 49))
            x1 = min(width, xs + bw)
            src = np.clip(np.arange(xs, x1) + disp, 0, width - 1)
            right[band:band + bh, xs:x1] = left[band:band + bh][:, src]
            xs = x1
        band += bh
    right = np.clip(np.rint(right + rng.normal(0, 2.0, size=right.shape)), 0, 255).astype(np.uint8)
    return left, right


def flip_bits(desc: np.ndarray, p: float, rng: np.random.Generator) -> np.ndarray:
    bits = np.unpackbits(desc, axis=-1, bitorder="little")
    mask = (rng.random(bits.shape) < p).astype(np.uint8)
    return np.packbits(bits ^ mask, axis=-1, bitorder="little")


def make_queries(kps: np.ndarray, desc: np.ndarray, counts: np.ndarray, n_levels: int,
                 scale: np.ndarray, n_per_level: np.ndarray, width: int, height: int,
                 n_queries_per_frame: int, th: float, seed: int, query_dtype, taken_frac=0.10,
                 true_frac=0.60):
    """Map-point queries for the windowed matcher, per frame.

    kps [F,cap] (keypoint records: x, y, level), desc [F,cap,32], counts [F,L+1].
    Returns (queries [F*Q] query_dtype, qdesc [F*Q,32] u8, taken [F,cap] u8)."""
    rng = _rng(seed)
    F, cap = kps.shape
    Q = n_queries_per_frame
    queries = np.zeros(F * Q, query_dtype)
    qdesc = np.zeros((F * Q, 32), np.uint8)
    taken = np.zeros((F, cap), np.uint8)
    pl = np.asarray(n_per_level, np.float64)
    pl = pl / pl.sum()
    scale = np.asarray(scale, np.float32)
    for f in range(F):
        n = int(counts[f, n_levels])
        base = f * Q
        nt = min(int(true_frac * n), Q)
        sel = rng.permutation(n)[:nt] if n else np.zeros(0, np.int64)
        taken[f, :n] = rng.random(n) < taken_frac
        q = queries[base:base + Q]
        q["frame"] = f
        if nt:
            k = kps[f, sel]
            q["u"][:nt] = k["x"] + rng.normal(0, 1.0, nt).astype(np.float32)
            q["v"][:nt] = k["y"] + rng.normal(0, 1.0, nt).astype(np.float32)
            lev = k["level"].astype(np.int32) + (rng.random(nt) >= 0.8)
            q["pred_level"][:nt] = np.minimum(lev, n_levels - 1)
            qdesc[base:base + nt] = flip_bits(desc[f, sel], 0.06, rng)
        nd = Q - nt
        q["u"][nt:] = rng.uniform(0, width, nd).astype(np.float32)
        q["v"][nt:] = rng.uniform(0, height, nd).astype(np.float32)
        q["pred_level"][nt:] = rng.choice(n_levels, size=nd, p=pl)
        hard = rng.random(nd) < 0.5
        rnd = rng.integers(0, 256, size=(nd, 32), dtype=np.uint8)
        if n:
            other = desc[f, rng.integers(0, n, nd)]
            rnd[hard] = flip_bits(other[hard], 0.25, rng)
        qdesc[base + nt:base + Q] = rnd
        fac = np.where(rng.random(Q) < 0.5, 2.5, 4.0).astype(np.float32)
        q["radius"] = np.float32(th) * fac * scale[q["pred_level"]]
        perm = rng.permutation(Q)
        queries[base:base + Q] = q[perm]
        qdesc[base:base + Q] = qdesc[base:base + Q][perm]
    return queries, qdesc, taken


def make_brute_map(desc_list, n_map: int, seed: int, n_from_kps: int | None = None) -> np.ndarray:
    """Shared-map descriptors: perturbed copies of client keypoint descriptors (p=0.06 flips)
    plus uniform random descriptors, shuffled."""
    rng = _rng(seed)
    pool = np.concatenate([d for d in desc_list], 0) if desc_list else np.zeros((0, 32), np.uint8)
    nk = min(len(pool), n_map if n_from_kps is None else n_from_kps)
    part = flip_bits(pool[rng.permutation(len(pool))[:nk]], 0.06, rng) if nk else np.zeros((0, 32), np.uint8)
    rnd = rng.integers(0, 256, size=(n_map - nk, 32), dtype=np.uint8)
    m = np.concatenate([part, rnd], 0)
    return np.ascontiguousarray(m[rng.permutation(n_map)])


# Pinhole intrinsics (fx, fy, cx, cy) of the datasets the shapes stand for (EuRoC cam0, TUM
# fr1, KITTI 00 left) -- input geometry only; the projection itself is the method's (O11).
INTRINSICS = {"euroc": (458.654, 457.296, 367.215, 248.375), "tum": (517.306, 516.469, 318.643, 255.314),
              "kitti": (718.856, 718.856, 607.1928, 185.2157)}
# rectified stereo baseline (m) of the stereo shape (KITTI 00: bf = fx * b = 386.1448)
STEREO_BASELINE = {"kitti": 0.5371657}
CAMERA_DTYPE = np.dtype([("R", "<f4", (9,)), ("t", "<f4", (3,)), ("ow", "<f4", (3,)), ("fx", "<f4"),
                         ("fy", "<f4"), ("cx", "<f4"), ("cy", "<f4"), ("min_x", "<f4"), ("max_x", "<f4"),
                         ("min_y", "<f4"), ("max_y", "<f4"), ("pad", "<f4")])
MAP_POINT_DTYPE = np.dtype([("pos", "<f4", (3,)), ("normal", "<f4", (3,)), ("min_dist", "<f4"),
                            ("max_dist", "<f4")])


def _rotation(rng) -> np.ndarray:
    q = rng.normal(size=4)
    q /= np.linalg.norm(q)
    w, x, y, z = q
    return np.array([[1 - 2 * (y * y + z * z), 2 * (x * y - z * w), 2 * (x * z + y * w)],
                     [2 * (x * y + z * w), 1 - 2 * (x * x + z * z), 2 * (y * z - x * w)],
                     [2 * (x * z - y * w), 2 * (y * z + x * w), 1 - 2 * (x * x + y * y)]])


def _tilt(d: np.ndarray, deg: np.ndarray, rng) -> np.ndarray:
    """Unit vectors at angle deg from the unit rows of d (random azimuth)."""
    a = np.cross(d, rng.normal(size=d.shape))
    a /= np.linalg.norm(a, axis=1, keepdims=True)
    r = np.radians(deg)[:, None]
    return d * np.cos(r) + np.cross(a, d) * np.sin(r)


def make_local_map(kps: np.ndarray, desc: np.ndarray, counts: np.ndarray, n_levels: int, scale_factor: float,
                   n_per_level: np.ndarray, width: int, height: int, shape: str, n_points_per_frame: int,
                   seed: int, taken_frac=0.10, true_frac=0.60):
    """Local-map points for "search local points" (O11 projection -> O9 windowed match), per
    frame (SURVEY §8(d) query statistics, lifted to 3D):

    * a random camera pose per frame, the dataset's intrinsics, bounds [0, W] x [0, H];
    * true points (60 % of the frame's keypoints): the keypoint position + N(0, 1 px)
      back-projected at depth U(2, 20), descriptor = the keypoint's with 6 % bit flips,
      max_dist = dist * sf^(level' - 0.5) with level' = level (80 %) or level + 1 (so the
      predicted level is level'), min_dist = max_dist / sf^(L-1), normal = the viewing ray
      tilted by U(0, 3) deg (half: radius factor 2.5) or U(6, 50) deg (4.0);
    * distractors: positions uniform over the image +-10 % at depth U(-2, 30) (some behind the
      camera or outside the image), levels ~ N_l, tilt U(0, 70) deg (some beyond 60 deg),
      half random descriptors, half hard negatives (another keypoint's, 25 % flips);
    * 10 % of keypoints marked taken.

    kps [F, cap] (x, y, level), desc [F, cap, 32], counts [F, L+1].
    Returns (cams [F], points [F*Q], point_frame [F*Q] i32, qdesc [F*Q, 32] u8, taken [F, cap] u8)."""
    rng = _rng(seed)
    F, cap = kps.shape
    Q = n_points_per_frame
    fx, fy, cx, cy = INTRINSICS[shape]
    cams = np.zeros(F, CAMERA_DTYPE)
    pts = np.zeros(F * Q, MAP_POINT_DTYPE)
    pf = np.repeat(np.arange(F, dtype=np.int32), Q)
    qdesc = np.zeros((F * Q, 32), np.uint8)
    taken = np.zeros((F, cap), np.uint8)
    pl = np.asarray(n_per_level, np.float64)
    pl = pl / pl.sum()
    sf = float(scale_factor)
    for f in range(F):
        R, t = _rotation(rng), rng.normal(0, 3.0, 3)
        ow = -R.T @ t
        c = cams[f]
        c["R"], c["t"], c["ow"] = R.astype(np.float32).ravel(), t.astype(np.float32), ow.astype(np.float32)
        c["fx"], c["fy"], c["cx"], c["cy"] = fx, fy, cx, cy
        c["min_x"], c["max_x"], c["min_y"], c["max_y"] = 0.0, width, 0.0, height
        n = int(counts[f, n_levels])
        nt = min(int(true_frac * n), Q)
        sel = rng.permutation(n)[:nt] if n else np.zeros(0, np.int64)
        taken[f, :n] = rng.random(n) < taken_frac
        u = np.empty(Q)
        v = np.empty(Q)
        lev = np.empty(Q, np.int64)
        k = kps[f, sel]
        u[:nt] = k["x"] + rng.normal(0, 1.0, nt)
        v[:nt] = k["y"] + rng.normal(0, 1.0, nt)
        lev[:nt] = np.minimum(k["level"].astype(np.int64) + (rng.random(nt) >= 0.8), n_levels - 1)
        nd = Q - nt
        u[nt:] = rng.uniform(-0.1 * width, 1.1 * width, nd)
        v[nt:] = rng.uniform(-0.1 * height, 1.1 * height, nd)
        lev[nt:] = rng.choice(n_levels, size=nd, p=pl)
        z = np.concatenate([rng.uniform(2.0, 20.0, nt), rng.uniform(-2.0, 30.0, nd)])
        pc = np.stack([(u - cx) / fx * z, (v - cy) / fy * z, z], 1)
        pw = (pc - t) @ R  # R^T (pc - t), row-wise
        ray = pw - ow
        dist = np.linalg.norm(ray, axis=1)
        tilt = np.where(rng.random(Q) < 0.5, rng.uniform(0, 3, Q), rng.uniform(6, 50, Q))
        tilt[nt:] = rng.uniform(0, 70, nd)
        nrm = _tilt(ray / dist[:, None], tilt, rng)
        p = pts[f * Q:(f + 1) * Q]
        p["pos"] = pw.astype(np.float32)
        p["normal"] = nrm.astype(np.float32)
        p["max_dist"] = (dist * sf ** (lev - 0.5)).astype(np.float32)
        p["min_dist"] = (p["max_dist"].astype(np.float64) / sf ** (n_levels - 1)).astype(np.float32)
        qd = qdesc[f * Q:(f + 1) * Q]
        if nt:
            qd[:nt] = flip_bits(desc[f, sel], 0.06, rng)
        rnd = rng.integers(0, 256, size=(nd, 32), dtype=np.uint8)
        hard = rng.random(nd) < 0.5
        if n:
            other = desc[f, rng.integers(0, n, nd)]
            rnd[hard] = flip_bits(other[hard], 0.25, rng)
        qd[nt:] = rnd
        perm = rng.permutation(Q)
        pts[f * Q:(f + 1) * Q] = p[perm]
        qdesc[f * Q:(f + 1) * Q] = qd[perm]
    return cams, pts, pf, qdesc, taken


FRAME_POINT_DTYPE = np.dtype([("pos", "<f4", (3,)), ("angle_deg", "<f4"), ("octave", "<i4"), ("reserved", "<i4")])


def _camera(c, R, t, shape, width, height):
    fx, fy, cx, cy = INTRINSICS[shape]
    c["R"], c["t"], c["ow"] = R.astype(np.float32).ravel(), t.astype(np.float32), (-R.T @ t).astype(np.float32)
    c["fx"], c["fy"], c["cx"], c["cy"] = fx, fy, cx, cy
    c["min_x"], c["max_x"], c["min_y"], c["max_y"] = 0.0, width, 0.0, height


def make_last_frame(kps: np.ndarray, desc: np.ndarray, counts: np.ndarray, n_levels: int, n_per_level: np.ndarray,
                    width: int, height: int, shape: str, n_points_per_frame: int, seed: int, true_frac=0.70,
                    pos_sigma=1.5, stereo_z=0.0, cams=None):
    """The previous frame's tracked map points for frame-to-frame matching (O13, ORB-SLAM
    TrackWithMotionModel), per frame:

    * the current camera: a random pose (or the given `cams`, e.g. the local map's) and the
      dataset's intrinsics, bounds [0, W] x [0, H];
      the last camera: the current one moved by stereo_z * U(-2, 2) along its optical axis
      (0 = the same pose; the stereo forward / backward gate needs |motion| > baseline);
    * true points (70 % of Q, at most the keypoint count): a keypoint's position +
      N(0, pos_sigma px) back-projected at depth U(2, 20), octave = its level (80 %) or
      level -+ 1 (clamped), angle = the keypoint's + a per-frame in-plane rotation U(-20, 20)
      deg + N(0, 4) deg (mod 360), descriptor with 6 % bit flips;
    * distractors: positions uniform over the image +-10 % at depth U(-2, 30), octave ~ N_l,
      uniform angle, half random descriptors, half hard negatives (25 % flips).

    Returns (cams [F], last_cams [F], pt_off [F+1] i32, points [F*Q] FRAME_POINT_DTYPE,
    pdesc [F*Q, 32] u8); frame f's points are [pt_off[f], pt_off[f+1])."""
    rng = _rng(seed)
    F, cap = kps.shape
    Q = n_points_per_frame
    fx, fy, cx, cy = INTRINSICS[shape]
    given = cams
    cams = np.zeros(F, CAMERA_DTYPE)
    last = np.zeros(F, CAMERA_DTYPE)
    pts = np.zeros(F * Q, FRAME_POINT_DTYPE)
    pdesc = np.zeros((F * Q, 32), np.uint8)
    pl = np.asarray(n_per_level, np.float64)
    pl = pl / pl.sum()
    for f in range(F):
        if given is None:
            R, t = _rotation(rng), rng.normal(0, 3.0, 3)
        else:
            R, t = given[f]["R"].reshape(3, 3).astype(np.float64), given[f]["t"].astype(np.float64)
        if given is None:
            _camera(cams[f], R, t, shape, width, height)
        else:
            cams[f] = given[f]
        tl = t + np.array([0.0, 0.0, stereo_z * rng.uniform(-2.0, 2.0)])
        _camera(last[f], R, tl, shape, width, height)
        n = int(counts[f, n_levels])
        nt = min(int(true_frac * Q), n)
        sel = rng.permutation(n)[:nt] if n else np.zeros(0, np.int64)
        k = kps[f, sel]
        u = np.concatenate([k["x"] + rng.normal(0, pos_sigma, nt), rng.uniform(-0.1 * width, 1.1 * width, Q - nt)])
        v = np.concatenate([k["y"] + rng.normal(0, pos_sigma, nt), rng.uniform(-0.1 * height, 1.1 * height, Q - nt)])
        z = np.concatenate([rng.uniform(2.0, 20.0, nt), rng.uniform(-2.0, 30.0, Q - nt)])
        pc = np.stack([(u - cx) / fx * z, (v - cy) / fy * z, z], 1)
        pw = (pc - t) @ R
        oct_t = k["level"].astype(np.int64) + np.where(rng.random(nt) < 0.8, 0, rng.choice([-1, 1], nt))
        octv = np.concatenate([np.clip(oct_t, 0, n_levels - 1), rng.choice(n_levels, size=Q - nt, p=pl)])
        rot = rng.uniform(-20.0, 20.0)
        ang = np.concatenate([k["angle_deg"] + rot + rng.normal(0, 4.0, nt), rng.uniform(0, 360, Q - nt)])
        pd = np.zeros((Q, 32), np.uint8)
        if nt:
            pd[:nt] = flip_bits(desc[f, sel], 0.06, rng)
        nd = Q - nt
        rnd = rng.integers(0, 256, size=(nd, 32), dtype=np.uint8)
        hard = rng.random(nd) < 0.5
        if n:
            other = desc[f, rng.integers(0, n, nd)]
            rnd[hard] = flip_bits(other[hard], 0.25, rng)
        pd[nt:] = rnd
        p = np.zeros(Q, FRAME_POINT_DTYPE)
        p["pos"] = pw.astype(np.float32)
        p["angle_deg"] = np.mod(ang, 360.0).astype(np.float32) % np.float32(360.0)
        p["octave"] = octv
        perm = rng.permutation(Q)
        pts[f * Q:(f + 1) * Q] = p[perm]
        pdesc[f * Q:(f + 1) * Q] = pd[perm]
    pt_off = (np.arange(F + 1) * Q).astype(np.int32)
    return cams, last, pt_off, pts, pdesc


def make_dotted_frame(width: int, height: int, seed: int, n_clusters: int = 12) -> np.ndarray:
    """Adversarial frame for the quadtree's deep-split path: a flat gray background with
    isolated bright pixels (each one FAST corner) arranged in clusters whose members sit at
    distances 3, 5, 9, ..., 129 px from the cluster centre, so the node count keeps growing
    at every quadtree depth (the kernel's dense-histogram tables stop at depth ~5, and the
    stop rules then need the sort fallback).  No method arithmetic: only pixel placement."""
    rng = _rng(seed)
    img = np.full((height, width), 60, np.uint8)
    for _ in range(n_clusters):
        cx, cy = int(rng.integers(40, width - 40)), int(rng.integers(40, height - 40))
        img[cy, cx] = 200
        for k in range(1, 8):
            a = rng.uniform(0, 2 * np.pi)
            d = 2 ** k + 1
            x, y = int(cx + d * np.cos(a)), int(cy + d * np.sin(a))
            if 20 <= x < width - 20 and 20 <= y < height - 20:
                img[y, x] = 200
    return img
