"""Pins of the oracle's O12 stereo matching (ORB-SLAM2 Frame::ComputeStereoMatches [ext];
SURVEY §8(f) F1) against geometry it must reproduce, not against itself: a right image that
is the left image shifted by an integer disparity d puts every correctly matched level-0
keypoint within half a pixel of uL - d (the SAD minimum is exactly 0 at the true shift and
the parabola offset is below 0.5), with depth = bf / disparity; plus the output invariants
(disparity range, the outlier cut at 2.1 x the median SAD)."""
import numpy as np
import pytest

import synth

FX, BASE = 718.856, 0.537
BF = np.float32(FX * BASE)


def _pair_shift(w, h, d, seed):
    big = synth.make_frame(w + d, h, seed)
    return np.ascontiguousarray(big[:, :w]), np.ascontiguousarray(big[:, d:])  # uR = uL - d


@pytest.mark.parametrize("d", [7, 23])
def test_integer_shift_recovers_disparity(ref, d):
    w, h = 752, 480
    p = ref.params(w, h, 1500)
    L, R = _pair_shift(w, h, d, seed=100 + d)
    kl, dl, cl = ref.orb_extract(p, L)
    kr, dr, cr = ref.orb_extract(p, R)
    ur, dp, sad = ref.stereo_match(p, L, R, kl, dl, cl, kr, dr, cr, BF, BASE)
    n0 = int(cl[1])  # level-0 keypoints
    uL = kl["x"][:n0]
    eligible = uL >= d + 40
    got = ur[:n0] >= 0
    assert (got & eligible).sum() >= 0.5 * eligible.sum(), ((got & eligible).sum(), eligible.sum())
    err = np.abs(ur[:n0][got] - (uL[got] - d))
    assert (err < 0.5).mean() >= 0.9, np.sort(err)[-20:]
    good = got.copy()
    good[got] = err < 0.5
    np.testing.assert_allclose(dp[:n0][good], BF / (uL[good] - ur[:n0][good]), rtol=1e-6)


@pytest.mark.parametrize("d", [7, 23, 36])
def test_integer_shift_on_every_octave(ref, d):
    """O12 on octaves >= 1: the refinement runs on octave o's level at round(uR0 * invScale)
    and maps back with scale[o], so a matched level-o keypoint lands within half a level-o
    pixel (0.5 * scale[o] level-0 px) of uL - d.  Level o of the shifted frame is only
    approximately shifted (resampling), so the pin asks for >= 90 % of all octave >= 1 matches
    and >= 80 % on every octave with >= 20 matches; a refinement on the wrong level or with
    the wrong scale misses by several pixels."""
    w, h = 752, 480
    p = ref.params(w, h, 1500)
    L, R = _pair_shift(w, h, d, seed=100 + d)
    kl, dl, cl = ref.orb_extract(p, L)
    kr, dr, cr = ref.orb_extract(p, R)
    ur, dp, sad = ref.stereo_match(p, L, R, kl, dl, cl, kr, dr, cr, BF, BASE)
    ok_all = n_all = 0
    for o in range(1, p.n_levels):
        a, b = int(cl[o]), int(cl[o + 1])
        got = ur[a:b] >= 0
        if not got.any():
            continue
        err = np.abs(ur[a:b][got] - (kl["x"][a:b][got] - d))
        good = err < 0.5 * p.scale[o]
        ok_all += int(good.sum())
        n_all += int(got.sum())
        if got.sum() >= 20:
            assert good.mean() >= 0.8, (o, good.mean())
        np.testing.assert_allclose(dp[a:b][got], BF / (kl["x"][a:b][got] - ur[a:b][got]), rtol=1e-6)
    assert n_all >= 300 and ok_all >= 0.9 * n_all, (ok_all, n_all)


def test_invariants_on_warped_pairs(ref):
    w, h = synth.SHAPES["kitti"]
    p = ref.params(w, h, 2000)
    maxD = np.float32(BF / np.float32(BASE))
    for seed in (1, 2):
        L, R = synth.make_stereo_pair(w, h, seed=seed)
        kl, dl, cl = ref.orb_extract(p, L)
        kr, dr, cr = ref.orb_extract(p, R)
        ur, dp, sad = ref.stereo_match(p, L, R, kl, dl, cl, kr, dr, cr, BF, BASE)
        n = int(cl[-1])
        ok = ur[:n] >= 0
        assert ok.sum() > 0.15 * n
        disp = kl["x"][:n][ok] - ur[:n][ok]
        assert (disp > 0).all() and (disp < maxD + 1e-3).all()
        assert ((dp[:n] >= 0) == ok).all()
        # the warp's disparities are 0..48 px (+ sub-pixel)
        assert np.median(disp) < 50
        # outlier cut: kept SADs < 2.1 x the median of the accepted SADs, and every accepted
        # SAD at or above it was cut
        acc = sad[:n] >= 0
        med = np.sort(sad[:n][acc])[acc.sum() // 2]
        th = np.float32(np.float32(1.5) * np.float32(1.4)) * np.float32(med)
        assert (sad[:n][ok].astype(np.float32) < th).all()
        assert not (acc & ~ok & (sad[:n].astype(np.float32) < th)).any()


def test_no_keypoints_is_a_no_op(ref):
    w, h = 640, 480
    p = ref.params(w, h, 1000)
    flat = np.full((h, w), 128, np.uint8)
    kl, dl, cl = ref.orb_extract(p, flat)
    ur, dp, sad = ref.stereo_match(p, flat, flat, kl, dl, cl, kl, dl, cl, BF, BASE)
    assert cl[-1] == 0 and (ur == -1).all() and (sad == -1).all()
