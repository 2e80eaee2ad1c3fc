"""Pins of the oracle's per-level ASSEMBLY of an extraction (S8c O8 wiring of O1, O2, O5, O6,
O7 on every pyramid level, not only level 0) against objects built here with library
routines, independent of the oracle:

* level images: chained cv2.resize(INTER_LINEAR_EXACT) (O1's library pin);
* blurred level images: cv2.GaussianBlur(7x7, sigma 2, REFLECT_101) of each level as a
  standalone image (O6's library pin);
* FAST response = M - 1: cv2.FastFeatureDetector (TYPE_9_16, no NMS) reports (lx, ly) as a
  corner at threshold t = response and not at t = response + 1 (corner at t <=> M > t);
* x, y: one f32 multiply f32(lx) * scale[l], scale = the f32 chain of 1.2 (App. B);
* moments: the 749-px disk sums written out in numpy on the UNBLURRED cv2 level; the angle is
  atan2 of them in f64 (tolerance 1e-4 rad, circular);
* descriptor: ref.descriptor (the O7 primitive, pinned in test_oracle_describe.py) evaluated on
  the cv2-BLURRED level with the numpy moments.

A plausible wiring mistake -- x = lx * inv_scale, moments taken on the blurred level,
descriptor sampled on the unblurred level, the level index off by one, response = M --
fails one of these assertions (the last test shows the blurred-moments one is detectable).
"""
import cv2
import numpy as np
import pytest

import synth

UMAX = [15, 15, 15, 15, 14, 14, 14, 13, 13, 12, 11, 10, 9, 8, 6, 3]


def _cv2_levels(p, img):
    levels = [img]
    for l in range(1, p.n_levels):
        levels.append(cv2.resize(levels[-1], (p.level_w[l], p.level_h[l]), interpolation=cv2.INTER_LINEAR_EXACT))
    return levels


def _cv2_blur(im):
    return cv2.GaussianBlur(im, (7, 7), 2, sigmaY=2, borderType=cv2.BORDER_REFLECT_101)


def _f32_scales(n, sf=1.2):
    s = [np.float32(1.0)]
    for _ in range(1, n):
        s.append(np.float32(s[-1] * np.float32(sf)))
    return s


def _moments(im, lx, ly):
    m10 = m01 = 0
    for v in range(-15, 16):
        u = np.arange(-UMAX[abs(v)], UMAX[abs(v)] + 1)
        row = im[ly + v, lx + u].astype(np.int64)
        m10 += int((u * row).sum())
        m01 += int(v * row.sum())
    return m10, m01


def _fast_corners(im, t):
    det = cv2.FastFeatureDetector_create(threshold=int(t), nonmaxSuppression=False,
                                         type=cv2.FAST_FEATURE_DETECTOR_TYPE_9_16)
    return {(int(round(k.pt[0])), int(round(k.pt[1]))) for k in det.detect(im)}


@pytest.mark.parametrize("shape,nf,seed", [("euroc", 1000, 3), ("kitti", 2000, 4), ("tum", 1000, 5)])
def test_every_level_assembly(ref, shape, nf, seed):
    w, h = synth.SHAPES[shape]
    p = ref.params(w, h, nf)
    img = synth.make_frame(w, h, synth.frame_seed(40, seed, 0))
    kps, desc, counts = ref.orb_extract(p, img)
    levels = _cv2_levels(p, img)
    blurred = [_cv2_blur(im) for im in levels]
    scales = _f32_scales(p.n_levels)
    for l in range(p.n_levels):
        a, b = int(counts[l]), int(counts[l + 1])
        assert b - a > 0, l
        k = kps[a:b]
        assert (k["level"] == l).all()
        order = k["ly"].astype(np.int64) * 4096 + k["lx"]
        assert (np.diff(order) > 0).all(), "canonical (ly, lx) order within a level"
        lx = k["lx"].astype(np.int64)
        ly = k["ly"].astype(np.int64)
        np.testing.assert_array_equal(k["x"].view(np.uint32), (lx.astype(np.float32) * scales[l]).view(np.uint32))
        np.testing.assert_array_equal(k["y"].view(np.uint32), (ly.astype(np.float32) * scales[l]).view(np.uint32))
        # response = M - 1 with M = the largest t at which cv2 still calls the pixel a corner + 1:
        # a corner at t = response, not at t = response + 1
        corners = {int(t): _fast_corners(levels[l], t) for t in np.unique(np.concatenate(
            [k["response"].astype(np.int64), k["response"].astype(np.int64) + 1]))}
        for i in range(b - a):
            x, y = int(lx[i]), int(ly[i])
            r = int(k["response"][i])
            assert (x, y) in corners[r] and (x, y) not in corners[r + 1], (l, x, y, r)
            m10, m01 = _moments(levels[l], x, y)
            ang = np.degrees(np.arctan2(m01, m10)) % 360.0 if (m10 or m01) else 0.0
            da = abs(float(k["angle_deg"][i]) - ang)
            assert np.radians(min(da, 360.0 - da)) <= 1e-4, (l, x, y)
            np.testing.assert_array_equal(desc[a + i], ref.descriptor(blurred[l], x, y, m10, m01),
                                          err_msg=f"level {l} ({x},{y})")


def test_wrong_wiring_is_detected(ref):
    """Sanity of the pin above: moments taken on the BLURRED level give angles that differ by
    more than the 1e-4 rad tolerance for most keypoints, and sampling the UNBLURRED level
    changes descriptors -- so those wiring errors cannot pass test_every_level_assembly."""
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1000)
    img = synth.make_frame(w, h, synth.frame_seed(40, 9, 0))
    kps, desc, counts = ref.orb_extract(p, img)
    levels = _cv2_levels(p, img)
    blurred = [_cv2_blur(im) for im in levels]
    l = 2
    a, b = int(counts[l]), int(counts[l + 1])
    off_angle = same_desc = 0
    for i in range(a, b):
        x, y = int(kps[i]["lx"]), int(kps[i]["ly"])
        m10, m01 = _moments(blurred[l], x, y)
        ang = np.degrees(np.arctan2(m01, m10)) % 360.0
        da = abs(float(kps[i]["angle_deg"]) - ang)
        off_angle += np.radians(min(da, 360.0 - da)) > 1e-4
        t10, t01 = _moments(levels[l], x, y)
        same_desc += bool((ref.descriptor(levels[l], x, y, t10, t01) == desc[i]).all())
    assert off_angle > 0.9 * (b - a)
    assert same_desc < 0.1 * (b - a)
