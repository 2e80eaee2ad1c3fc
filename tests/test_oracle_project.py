"""Pins of the oracle's O11 local-map projection (ORB-SLAM3 isInFrustum + PredictScale +
RadiusByViewingCos [ext]; the per-point step of "search local points", §4.2.1),
against things other than the oracle itself: cv2.projectPoints in f64, closed forms on
the optical axis and under a 90-degree roll, the log-based level formula away from level
boundaries, and one point per culling rule that violates only that rule."""
import math

import cv2
import numpy as np
import pytest

EUROC_K = (458.654, 457.296, 367.215, 248.375)


def camera(R, t, K=EUROC_K, W=752, H=480):
    import oracle
    c = np.zeros(1, oracle.CAMERA_DTYPE)
    R = np.asarray(R, np.float64)
    t = np.asarray(t, np.float64)
    c["R"][0] = R.astype(np.float32).ravel()
    c["t"][0] = t.astype(np.float32)
    c["ow"][0] = (-R.T @ t).astype(np.float32)
    c["fx"], c["fy"], c["cx"], c["cy"] = K
    c["min_x"], c["max_x"], c["min_y"], c["max_y"] = 0.0, W, 0.0, H
    return c


def points(pos, normal=None, dmin=0.1, dmax=100.0, ow=(0, 0, 0)):
    import oracle
    pos = np.asarray(pos, np.float64).reshape(-1, 3)
    p = np.zeros(len(pos), oracle.MAP_POINT_DTYPE)
    p["pos"] = pos.astype(np.float32)
    if normal is None:  # looking straight at the point: viewCos = 1
        d = pos - np.asarray(ow, np.float64)
        normal = d / np.linalg.norm(d, axis=1, keepdims=True)
    p["normal"] = np.asarray(normal, np.float32).reshape(-1, 3)
    p["min_dist"] = dmin
    p["max_dist"] = dmax
    return p


def test_projection_matches_cv2_projectPoints(ref):
    p = ref.params(752, 480)
    rng = np.random.default_rng(5)
    for trial in range(20):
        rvec = rng.normal(0, 0.4, 3)
        R, _ = cv2.Rodrigues(rvec)
        t = rng.normal(0, 2.0, 3)
        cam = camera(R, t)
        ow = (-R.T @ t)
        # points in front of the camera, inside the image
        uv = rng.uniform([5, 5], [747, 475], size=(200, 2))
        z = rng.uniform(0.5, 30.0, 200)
        fx, fy, cx, cy = EUROC_K
        pc = np.stack([(uv[:, 0] - cx) / fx * z, (uv[:, 1] - cy) / fy * z, z], 1)
        pw = (R.T @ (pc - t).T).T
        pts = points(pw, ow=ow)
        got = ref.project_points(p, cam, pts, np.zeros(len(pts), np.int32))
        want, _ = cv2.projectPoints(pts["pos"].astype(np.float64), cv2.Rodrigues(R.astype(np.float32).astype(np.float64))[0],
                                    t.astype(np.float32).astype(np.float64),
                                    np.array([[fx, 0, cx], [0, fy, cy], [0, 0, 1]]), None)
        want = want.reshape(-1, 2)
        inside = (want[:, 0] > 0.01) & (want[:, 0] < 751.99) & (want[:, 1] > 0.01) & (want[:, 1] < 479.99)
        assert (got["pred_level"][inside] >= 0).all(), trial
        np.testing.assert_allclose(got["u"][inside], want[inside, 0], atol=2e-3)
        np.testing.assert_allclose(got["v"][inside], want[inside, 1], atol=2e-3)
        assert (got["frame"] == 0).all()


def test_optical_axis_and_roll(ref):
    p = ref.params(752, 480)
    fx, fy, cx, cy = 400.0, 400.0, 376.0, 240.0
    K = (fx, fy, cx, cy)
    # identity pose: (0, 0, Z) projects to the principal point exactly
    q = ref.project_points(p, camera(np.eye(3), [0, 0, 0], K), points([[0, 0, 7.0]], dmax=7.0), [0])
    assert q["u"][0] == cx and q["v"][0] == cy and q["pred_level"][0] == 0
    # a 90-degree roll about the optical axis maps (X, Y) -> (-Y, X): the projection turns
    # by 90 degrees about the principal point (exact: every product here is exact in f32)
    Rz = np.array([[0, -1, 0], [1, 0, 0], [0, 0, 1]], np.float64)
    P = np.array([[1.0, 0.5, 4.0], [-0.25, 0.75, 2.0]])
    a = ref.project_points(p, camera(np.eye(3), [0, 0, 0], K), points(P), [0, 0])
    b = ref.project_points(p, camera(Rz, [0, 0, 0], K), points(P), [0, 0])
    np.testing.assert_array_equal(b["u"] - cx, -(a["v"] - cy))
    np.testing.assert_array_equal(b["v"] - cy, a["u"] - cx)


def test_each_culling_rule(ref):
    p = ref.params(752, 480)
    cam = camera(np.eye(3), [0, 0, 0], (400.0, 400.0, 376.0, 240.0))
    base = [0.5, 0.25, 5.0]
    dist = math.sqrt(0.25 + 0.0625 + 25.0)
    cases = {
        "visible": (points([base]), True),
        "behind": (points([[0.5, 0.25, -5.0]]), False),
        "left of the image": (points([[-5.0, 0.0, 5.0]]), False),
        "below the image": (points([[0.0, 4.0, 5.0]]), False),
        "nearer than 0.8 min": (points([base], dmin=dist / 0.79), False),
        "farther than 1.2 max": (points([base], dmax=dist / 1.21), False),
        "viewing angle > 60 deg": (points([base], normal=[[1.0, 0.0, 0.0]]), False),
    }
    for name, (pt, vis) in cases.items():
        q = ref.project_points(p, cam, pt, [0])
        assert (q["pred_level"][0] >= 0) == vis, name
        if not vis:
            assert q["radius"][0] == 0 and q["u"][0] == 0 and q["v"][0] == 0, name
    # frame index outside the batch: never visible
    q = ref.project_points(p, cam, points([base]), [3])
    assert q["pred_level"][0] == -1 and q["frame"][0] == 3


def test_predicted_level_matches_log_formula(ref):
    p = ref.params(752, 480)
    cam = camera(np.eye(3), [0, 0, 0], (400.0, 400.0, 376.0, 240.0))
    rng = np.random.default_rng(2)
    dist = rng.uniform(0.5, 20.0, 3000)
    dmax = dist * np.exp(rng.uniform(-0.5, math.log(1.2) * 9, 3000))
    pos = np.stack([np.zeros_like(dist), np.zeros_like(dist), dist], 1)
    pts = points(pos, dmin=0.01, dmax=dmax)
    q = ref.project_points(p, cam, pts, np.zeros(len(pts), np.int32))
    d32 = pts["pos"][:, 2].astype(np.float64)
    ratio = pts["max_dist"].astype(np.float64) / d32
    x = np.log(ratio) / math.log(1.2)
    want = np.clip(np.ceil(x), 0, 7)
    vis = q["pred_level"] >= 0
    assert vis.sum() > 2000
    far = np.abs(x - np.round(x)) > 1e-4  # away from the level boundaries
    np.testing.assert_array_equal(q["pred_level"][vis & far], want[vis & far])


def test_radius_by_viewing_cos(ref):
    p = ref.params(752, 480)
    cam = camera(np.eye(3), [0, 0, 0], (400.0, 400.0, 376.0, 240.0))
    P = [[0.0, 0.0, 5.0]]
    q = ref.project_points(p, cam, points(P, dmax=5.0), [0], th=1.0)
    assert q["radius"][0] == 2.5 and q["pred_level"][0] == 0  # viewCos = 1 > 0.998
    c = math.cos(math.radians(10))  # 0.985 < 0.998
    q = ref.project_points(p, cam, points(P, normal=[[0.0, math.sin(math.radians(10)), c]], dmax=5.0), [0],
                           th=3.0)
    assert q["radius"][0] == 12.0
    # level 3: radius = 2.5 * scale[3] (f32)
    q = ref.project_points(p, cam, points(P, dmax=5.0 * 1.2 ** 2.5), [0], th=1.0)
    assert q["pred_level"][0] == 3 and q["radius"][0] == np.float32(2.5) * np.float32(p.scale[3])
