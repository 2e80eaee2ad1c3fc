"""Pins of oracle O2 (FAST-9 M map) and O3 (per-cell FAST with iniTh/minTh fallback).

O2: cv2.FAST(TYPE_9_16) (library) -- corner at t <=> M > t, response = M - 1 -- and the
exhaustive 2^16 ring-mask x 2 polarity table against "cyclic run >= 9" brute force (E15).
O3: ORB-SLAM's per-cell loop [ext] transcribed with cv2.FAST on each cell ROI (the library
routine ORB-SLAM itself calls), compared with the oracle's M-map + cell-local NMS.
"""
import cv2
import numpy as np
import pytest

import synth

RING = [(0, 3), (1, 3), (2, 2), (3, 1), (3, 0), (3, -1), (2, -2), (1, -3), (0, -3), (-1, -3),
        (-2, -2), (-3, -1), (-3, 0), (-3, 1), (-2, 2), (-1, 3)]


def _cv_fast(img, t, nonmax):
    det = cv2.FastFeatureDetector_create(threshold=t, nonmaxSuppression=nonmax,
                                         type=cv2.FAST_FEATURE_DETECTOR_TYPE_9_16)
    return det.detect(img)


def _blocky(seed, w=160, h=120):
    rng = np.random.default_rng(seed)
    small = rng.integers(0, 256, size=(h // 4 + 1, w // 4 + 1), dtype=np.uint8)
    img = cv2.resize(small, (w // 4 * 4 + 4, h // 4 * 4 + 4), interpolation=cv2.INTER_NEAREST)[:h, :w]
    return np.clip(img.astype(np.int32) + rng.integers(-6, 7, size=img.shape), 0, 255).astype(np.uint8)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("t", [7, 20])
def test_fast_threshold_set_matches_cv2(ref, seed, t):
    img = _blocky(seed)
    M = ref.fast_M(img).astype(np.int32)
    want = {(int(round(k.pt[0])), int(round(k.pt[1]))) for k in _cv_fast(img, t, False)}
    ys, xs = np.nonzero(M > t)
    got = set(zip(xs.tolist(), ys.tolist()))
    assert got == want


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("t", [7, 20])
def test_fast_nonmax_responses_match_cv2(ref, seed, t):
    img = _blocky(seed + 100)
    M = ref.fast_M(img).astype(np.int32)
    kps = _cv_fast(img, t, True)
    assert len(kps) > 20
    for k in kps:
        x, y = int(round(k.pt[0])), int(round(k.pt[1]))
        assert M[y, x] - 1 == int(k.response)
        nb = M[y - 1:y + 2, x - 1:x + 2].copy()
        nb[1, 1] = -1
        nb[nb <= t] = 0
        assert (nb < M[y, x]).all()


def test_fast_exhaustive_ring_masks(ref):
    """Every 16-bit ring mask x {bright, dark}: corner <=> cyclic run >= 9 (E15)."""
    t, c = 20, 100
    masks = np.arange(1 << 16)
    n = 2 * len(masks)
    side = int(np.ceil(np.sqrt(n)))
    img = np.full((side * 7, side * 7), c, np.uint8)
    for pol, delta in enumerate((t + 1, -(t + 1))):
        for bit, (dx, dy) in enumerate(RING):
            on = (masks >> bit) & 1
            idx = pol * len(masks) + masks
            cy, cx = (idx // side) * 7 + 3, (idx % side) * 7 + 3
            img[cy + dy, cx + dx] = np.where(on == 1, c + delta, c).astype(np.uint8)
    M = ref.fast_M(img).astype(np.int32)
    idx = np.arange(n)
    cy, cx = (idx // side) * 7 + 3, (idx % side) * 7 + 3
    got = M[cy, cx] > t
    m2 = np.concatenate([masks, masks])
    bits = ((m2[:, None] >> np.arange(16)) & 1).astype(bool)
    dbl = np.concatenate([bits, bits], 1)
    run = np.zeros(n, bool)
    for s in range(16):
        run |= dbl[:, s:s + 9].all(1)
    np.testing.assert_array_equal(got, run)
    cvset = {(int(round(k.pt[0])), int(round(k.pt[1]))) for k in _cv_fast(img, t, False)}
    cv_at_centres = np.array([(x, y) in cvset for x, y in zip(cx.tolist(), cy.tolist())])
    np.testing.assert_array_equal(cv_at_centres, run)


def orbslam_cells_cv2(lev, p, l):
    """ORB-SLAM ComputeKeyPointsOctTree cell loop [ext] with cv2.FAST on each ROI."""
    h, w = lev.shape
    minB, maxBX, maxBY = 16, w - 16, h - 16
    wc, hc = p.cell_w[l], p.cell_h[l]
    out = []
    for i in range(p.cell_rows[l]):
        iniY = minB + i * hc
        if iniY >= maxBY - 3:
            continue
        maxY = min(iniY + hc + 6, maxBY)
        for j in range(p.cell_cols[l]):
            iniX = minB + j * wc
            if iniX >= maxBX - 6:
                continue
            maxX = min(iniX + wc + 6, maxBX)
            roi = np.ascontiguousarray(lev[iniY:maxY, iniX:maxX])
            ks = _cv_fast(roi, p.ini_th_fast, True)
            if not ks:
                ks = _cv_fast(roi, p.min_th_fast, True)
            cell = sorted((int(round(k.pt[1])), int(round(k.pt[0])), int(k.response)) for k in ks)
            out += [(x + iniX, y + iniY, r) for (y, x, r) in cell]
    return out


@pytest.mark.parametrize("shape,seed", [("euroc", 21), ("tum", 22), ("kitti", 21)])
def test_cell_candidates_match_orbslam_loop(ref, shape, seed):
    w, h = synth.SHAPES[shape]
    img = synth.make_frame(w, h, synth.frame_seed(3, seed, 0))
    p = ref.params(w, h, 1000)
    levels = ref.pyramid(p, img)
    fallback_seen = 0
    for l in range(8):
        M = ref.fast_M(levels[l])
        lx, ly, sc = ref.cell_candidates(p, l, M)
        got = list(zip(lx.tolist(), ly.tolist(), (sc - 1).tolist()))
        want = orbslam_cells_cv2(levels[l], p, l)
        assert got == want, f"level {l}"
        fallback_seen += int((sc <= p.ini_th_fast).sum())
    assert fallback_seen > 0  # the minTh path is exercised by the synthetic frames
