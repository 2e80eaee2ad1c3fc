"""Pins of oracle O5 (orientation), O6 (blur), O7 (rotated BRIEF) and the BRIEF pattern.

O5: closed form on intensity planes (angle = atan2(q, p) exactly), rot90 permutation of
    the moments, the 749-pixel rot90-symmetric disk.
O6: cv2.GaussianBlur(7x7, sigma 2, REFLECT_101) on standalone Mats (library routine).
O7: exact round-half-even of z/sqrt(r2) against Python's exact integer arithmetic;
    bit-exact rot90 invariance of the whole orientation+blur+descriptor chain (E10);
    unrotated case (m01 = 0) samples the pattern directly; agreement with cv2.ORB.
"""
import hashlib
import os

import cv2
import numpy as np
import pytest

import synth

PATTERN_SHA = "7e645581387b82784797e8adddb9b6f0c12611859fda09ca8a9bec96d767a05f"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _parse_inc(path):
    txt = open(path).read()
    body = txt[txt.index("{") + 1: txt.index("}")]
    return np.array([int(v) for v in body.replace("\n", " ").split(",") if v.strip()], "<i4")


def _cv2_pattern():
    so = os.path.join(os.path.dirname(cv2.__file__), "cv2.abi3.so")
    b = open(so, "rb").read()
    i = b.find(np.array([8, -3, 9, 5, 4, 2, 7, -12], "<i4").tobytes())
    assert i >= 0
    return b[i:i + 4096]


def test_pattern_tables_match_cv2():
    raw = _cv2_pattern()
    assert hashlib.sha256(raw).hexdigest() == PATTERN_SHA
    for path in ("oracle/brief_pattern_ref.inc",
                 "paper_conf_conext_dhakalrwcr22_b200/csrc/brief_pattern.inc"):
        arr = _parse_inc(os.path.join(ROOT, path))
        assert arr.tobytes() == raw, path


def _disk():
    umax = [15, 15, 15, 15, 14, 14, 14, 13, 13, 12, 11, 10, 9, 8, 6, 3]
    return [(u, v) for v in range(-15, 16) for u in range(-umax[abs(v)], umax[abs(v)] + 1)]


def test_disk_via_moments(ref):
    # moments of a delta image recover the disk membership of each offset
    img = np.zeros((41, 41), np.uint8)
    inside = set()
    for v in range(-18, 19):
        for u in range(-18, 19):
            if abs(u) > 18 or abs(v) > 18:
                continue
            img[:] = 0
            img[20 + v, 20 + u] = 1
            m10, m01 = ref.moments(img, 20, 20)
            if m10 or m01:
                assert (m10, m01) == (u, v)
                inside.add((u, v))
    assert inside == set(_disk()) - {(0, 0)}  # App. B umax table
    full = set(_disk())
    assert len(full) == 749
    assert {(v, -u) for (u, v) in full} == full  # rot90 symmetric


@pytest.mark.parametrize("p,q", [(1, 0), (0, 1), (-1, 2), (3, -3), (2, 1), (-3, -1), (1, 3)])
def test_angle_plane_closed_form(ref, p, q):
    img = np.zeros((41, 41), np.uint8)
    for y in range(41):
        for x in range(41):
            img[y, x] = 128 + p * (x - 20) + q * (y - 20)
    m10, m01 = ref.moments(img, 20, 20)
    # sum u^2 = sum v^2 over the symmetric disk, sum uv = 0 -> (m10, m01) = S (p, q)
    S = sum(u * u for u, _ in _disk())
    assert (m10, m01) == (S * p, S * q)
    want = np.degrees(np.arctan2(q, p)) % 360.0
    got = ref.angle_deg(m10, m01)
    d = abs(got - want)
    assert min(d, 360 - d) < 1e-4


def test_angle_special(ref):
    assert ref.angle_deg(0, 0) == 0.0
    assert ref.angle_deg(5, 0) == 0.0
    assert ref.angle_deg(0, 5) == 90.0
    assert ref.angle_deg(-5, 0) == 180.0
    a = ref.angle_deg(1_000_000, -1)  # tiny negative angle -> 360 - eps, must stay < 360
    assert 0.0 <= a < 360.0


@pytest.mark.parametrize("shape", [(480, 752), (134, 210), (37, 53), (8, 9), (376, 1241)])
def test_blur_matches_cv2(ref, shape):
    rng = np.random.default_rng(shape[0])
    img = rng.integers(0, 256, size=shape, dtype=np.uint8)
    want = cv2.GaussianBlur(img, (7, 7), 2, 2, borderType=cv2.BORDER_REFLECT_101)
    np.testing.assert_array_equal(ref.blur(img), want)


def test_rhe_div_sqrt_exact(ref):
    import math
    rng = np.random.default_rng(7)

    def exact(z, r2):  # round-half-even of z / sqrt(r2) with integers only
        a = abs(z)
        k = math.isqrt((a * a) // r2)  # floor-ish start
        best = None
        for c in range(max(0, k - 2), k + 3):
            # compare |a/r - c| exactly via squares: (2a - 2c r)^2 -> use 4a^2 vs (2c+-1)^2 r2
            lo_ok = c == 0 or (2 * c - 1) ** 2 * r2 <= 4 * a * a
            hi_ok = 4 * a * a <= (2 * c + 1) ** 2 * r2
            if lo_ok and hi_ok:
                if best is None:
                    best = c
                elif c % 2 == 0:  # tie between best and c -> even
                    best = c
        return -best if z < 0 else best

    for _ in range(4000):
        m10, m01 = (int(v) for v in rng.integers(-1_248_480, 1_248_481, size=2))
        if rng.random() < 0.2:  # Pythagorean radii give exact ties
            t = int(rng.integers(1, 300))
            m10, m01 = 3 * t * int(rng.choice([-1, 1])), 4 * t * int(rng.choice([-1, 1]))
        r2 = m10 * m10 + m01 * m01
        if r2 == 0:
            continue
        px, py = (int(v) for v in rng.integers(-13, 13, size=2))
        for z in (px * m10 - py * m01, px * m01 + py * m10):
            assert ref.rhe_div_sqrt(z, r2) == exact(z, r2)
    # explicit ties: 5/2 -> 2, 7/2 -> 4, -5/2 -> -2, 1/2 -> 0
    assert [ref.rhe_div_sqrt(z, 4) for z in (5, 7, -5, 1, 3)] == [2, 4, -2, 0, 2]


def _frame_keypoints(rng, w, h, n):
    xs = rng.integers(19, w - 19, size=n)
    ys = rng.integers(19, h - 19, size=n)
    return list(zip(xs.tolist(), ys.tolist()))


def test_descriptor_rot90_invariance(ref):
    img = synth.make_frame(200, 160, synth.frame_seed(5, 0, 0))
    rot = np.ascontiguousarray(np.rot90(img))  # new(x', y') = old(x = W-1-y', y = x')
    W = img.shape[1]
    B, Br = ref.blur(img), ref.blur(rot)
    np.testing.assert_array_equal(np.rot90(B), Br)  # blur commutes with rot90
    rng = np.random.default_rng(0)
    for x, y in _frame_keypoints(rng, img.shape[1], img.shape[0], 200):
        xr, yr = y, W - 1 - x
        if not (19 <= xr < rot.shape[1] - 19 and 19 <= yr < rot.shape[0] - 19):
            continue
        m10, m01 = ref.moments(img, x, y)
        r10, r01 = ref.moments(rot, xr, yr)
        assert (r10, r01) == (m01, -m10)
        d0 = ref.descriptor(B, x, y, m10, m01)
        d1 = ref.descriptor(Br, xr, yr, r10, r01)
        np.testing.assert_array_equal(d0, d1)


def test_descriptor_unrotated_samples_pattern(ref):
    rng = np.random.default_rng(3)
    Bimg = rng.integers(0, 256, size=(64, 64), dtype=np.uint8)
    pat = np.frombuffer(_cv2_pattern(), "<i4").reshape(256, 2, 2)
    for m10 in (1, 77, 1_000_000):
        d = ref.descriptor(Bimg, 32, 32, m10, 0)
        bits = np.unpackbits(d, bitorder="little")
        for b in range(256):
            (x0, y0), (x1, y1) = pat[b]
            assert bits[b] == int(Bimg[32 + y0, 32 + x0] < Bimg[32 + y1, 32 + x1])
    np.testing.assert_array_equal(ref.descriptor(Bimg, 32, 32, 0, 0), ref.descriptor(Bimg, 32, 32, 5, 0))


def test_descriptor_agrees_with_cv2_orb(ref):
    """cv2.ORB (one level) computes the same intensity-centroid angle and rotated BRIEF
    up to its float rounding and its own blur: angles within 0.01 deg, >= 99.5 % bits."""
    img = synth.make_frame(640, 480, synth.frame_seed(6, 0, 0))
    orb = cv2.ORB_create(nfeatures=400, nlevels=1, edgeThreshold=31, patchSize=31, fastThreshold=20)
    kps, desc = orb.detectAndCompute(img, None)
    B = ref.blur(img)
    agree = total = 0
    for k, d in zip(kps, desc):
        x, y = int(round(k.pt[0])), int(round(k.pt[1]))
        if not (40 <= x < img.shape[1] - 40 and 40 <= y < img.shape[0] - 40):
            continue
        m10, m01 = ref.moments(img, x, y)
        a = ref.angle_deg(m10, m01)
        diff = abs(a - k.angle)
        assert min(diff, 360 - diff) < 0.01
        mine = np.unpackbits(ref.descriptor(B, x, y, m10, m01), bitorder="little")
        theirs = np.unpackbits(d, bitorder="little")
        agree += int((mine == theirs).sum())
        total += 256
    assert total > 256 * 100
    assert agree / total >= 0.995
