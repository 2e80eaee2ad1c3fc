"""Pins of oracle O0 (params) and O1 (pyramid) -- SURVEY.md §8(c), DESIGN.md §3.

O0 is pinned to the App. B tables (tests/golden/params_appB.json); O1 to OpenCV's
bit-exact cv2.resize(INTER_LINEAR_EXACT), a library routine independent of the oracle.
"""
import json
import os

import cv2
import numpy as np
import pytest

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold():
    with open(os.path.join(GOLD, "params_appB.json")) as f:
        return json.load(f)


@pytest.mark.parametrize("shape", ["euroc", "tum", "kitti"])
def test_params_match_appendix_b(ref, shape):
    g = _gold()
    s = g["shapes"][shape]
    p = ref.params(s["w"], s["h"], 1000)
    assert [[p.level_w[l], p.level_h[l]] for l in range(8)] == s["level_wh"]
    assert sum(p.level_w[l] * p.level_h[l] for l in range(8)) == s["px_total"]
    assert [[p.cell_cols[l], p.cell_rows[l], p.cell_w[l], p.cell_h[l]] for l in range(8)] == s["cells"]
    assert p.n_ini[0] == s["nini"]
    np.testing.assert_allclose(list(p.scale), g["scales"], rtol=3e-7)


@pytest.mark.parametrize("nf", [1000, 1250, 2000])
def test_features_per_level(ref, nf):
    p = ref.params(752, 480, nf)
    assert list(p.n_per_level) == _gold()["features_per_level"][str(nf)]
    assert sum(p.n_per_level) == nf
    assert p.kp_capacity == nf + 16  # N_l + 2 per level when N_l + 2 >= 4 nIni


def test_scale_chain_is_f32(ref):
    p = ref.params(752, 480, 1000)
    s = np.float32(1.0)
    for l in range(8):
        assert np.float32(p.scale[l]) == s
        assert np.float32(p.inv_scale[l]) == np.float32(1.0) / s
        s = np.float32(s * np.float32(1.2))
    # App. B: the f32 chain gives 2.985985 (6 d.p.), not the exact 1.2^6 = 2.985984
    assert round(float(p.scale[6]), 6) == 2.985985 and np.float32(p.scale[6]) != np.float32(2.985984)


def test_params_reject(ref):
    with pytest.raises(ValueError):
        ref.params(40, 40, 1000)
    with pytest.raises(ValueError):
        ref.params(752, 480, 1000, n_levels=9)


@pytest.mark.parametrize("seed", range(12))
def test_resize_matches_cv2_linear_exact(ref, seed):
    rng = np.random.default_rng(seed)
    sw, sh = int(rng.integers(20, 900)), int(rng.integers(20, 600))
    dw, dh = max(1, int(sw / rng.uniform(1.05, 1.6))), max(1, int(sh / rng.uniform(1.05, 1.6)))
    src = rng.integers(0, 256, size=(sh, sw), dtype=np.uint8)
    want = cv2.resize(src, (dw, dh), interpolation=cv2.INTER_LINEAR_EXACT)
    np.testing.assert_array_equal(ref.resize_linear_exact(src, dw, dh), want)


def test_resize_adversarial_ties(ref):
    # alternating 0/255 rows & columns make every weight-rounding tie visible (E6)
    for sw in range(40, 140, 7):
        for dw in (sw - 1, int(sw / 1.2), int(sw / 1.2) + 1, sw // 2 + 1):
            src = np.tile(np.array([0, 255], np.uint8), (sw // 2 + 1, sw // 2 + 1))[: sw, : sw]
            want = cv2.resize(src, (dw, dw), interpolation=cv2.INTER_LINEAR_EXACT)
            np.testing.assert_array_equal(ref.resize_linear_exact(src, dw, dw), want)


@pytest.mark.parametrize("shape", ["euroc", "tum", "kitti"])
def test_pyramid_chain_matches_cv2(ref, shape):
    w, h = synth.SHAPES[shape]
    img = synth.make_frame(w, h, synth.frame_seed(9, 1, 2))
    p = ref.params(w, h, 1000)
    levels = ref.pyramid(p, img)
    prev = img
    for l in range(8):
        if l:
            prev = cv2.resize(prev, (p.level_w[l], p.level_h[l]), interpolation=cv2.INTER_LINEAR_EXACT)
        np.testing.assert_array_equal(levels[l], prev, err_msg=f"level {l}")


def test_pyramid_constant_image(ref):
    p = ref.params(752, 480, 1000)
    for v in (0, 1, 128, 255):
        for lev in ref.pyramid(p, np.full((480, 752), v, np.uint8)):
            assert (lev == v).all()
