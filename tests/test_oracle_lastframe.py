"""Pins of oracle O13: frame-to-frame projection matching (ORB-SLAM SearchByProjection of the
last frame's map points, TrackWithMotionModel [ext]; the "ORB-Matching" bar of P:L254 Fig. 8;
DESIGN.md §3 item 14).

Independent of the oracle's code:
* closed forms of the rotation bin (factor 1/30, literally ORB-SLAM's 1.0f/HISTO_LENGTH);
* hand-worked cases whose expected outputs are derived in the comments: three-maxima filter
  (incl. the 0.1 * max1 cut), dedup, TH_HIGH boundary, the level gates (mono and the stereo
  forward / backward rules), the 2*th retry;
* a physical pin: the current frame is the last frame shifted by an integer number of pixels
  (a fronto-parallel plane seen after a sideways camera move), so every level-0 keypoint of
  the last frame reappears with the identical descriptor and angle at (x + dx, y + dy);
* invariants on the synthetic workload and a numpy brute force of the definition.
"""
import numpy as np
import pytest

import synth
from oracle import CAMERA_DTYPE, FRAME_POINT_DTYPE, KEYPOINT_DTYPE

FX, FY, CX, CY = 400.0, 400.0, 376.0, 240.0


def _params(ref):
    return ref.params(752, 480, 1000)


def _cam(t=(0.0, 0.0, 0.0)):
    c = np.zeros(1, CAMERA_DTYPE)
    c["R"] = np.eye(3, dtype=np.float32).ravel()
    c["t"] = np.asarray(t, np.float32)
    c["ow"] = -np.asarray(t, np.float32)
    c["fx"], c["fy"], c["cx"], c["cy"] = FX, FY, CX, CY
    c["min_x"], c["max_x"], c["min_y"], c["max_y"] = 0.0, 752.0, 0.0, 480.0
    return c


def _frame(p, recs, rng):
    """recs: (level, lx, ly, angle) -> canonical-order keypoints of one frame + random descriptors."""
    cap, L = p.kp_capacity, p.n_levels
    recs = sorted(recs, key=lambda r: (r[0], r[2], r[1]))
    kps = np.zeros((1, cap), KEYPOINT_DTYPE)
    counts = np.zeros((1, L + 1), np.int32)
    for k, (l, lx, ly, a) in enumerate(recs):
        kps[0, k]["level"], kps[0, k]["lx"], kps[0, k]["ly"], kps[0, k]["angle_deg"] = l, lx, ly, a
        kps[0, k]["x"] = np.float32(lx) * np.float32(p.scale[l])
        kps[0, k]["y"] = np.float32(ly) * np.float32(p.scale[l])
    for l in range(L):
        counts[0, l + 1] = counts[0, l] + sum(1 for r in recs if r[0] == l)
    desc = np.zeros((1, cap, 32), np.uint8)
    desc[0, :len(recs)] = rng.integers(0, 256, (len(recs), 32), dtype=np.uint8)
    return kps, desc, counts, recs


def _point_at(x, y, octave, angle, Z=10.0):
    """World point that the identity camera projects to (x, y) (up to f32 rounding)."""
    p = np.zeros(1, FRAME_POINT_DTYPE)
    p["pos"] = np.array([(x - CX) * Z / FX, (y - CY) * Z / FY, Z], np.float32)
    p["angle_deg"], p["octave"] = angle, octave
    return p


def _flip(d, nbits, rng):
    d = d.copy()
    bits = rng.permutation(256)[:nbits]
    for b in bits:
        d[b >> 3] ^= np.uint8(1 << (b & 7))
    return d


def _run(ref, p, kps, desc, counts, pts, pdesc, cams=None, last=None, mb=0.0, th=15.0, min_matches=0, check=1,
         taken=None):
    cams = _cam() if cams is None else cams
    pt_off = np.array([0, len(pts)], np.int32)
    return ref.match_last_frame(p, cams, last, mb, kps, desc, counts, taken, pt_off, np.concatenate(pts),
                                np.stack(pdesc), th=th, check_orientation=check, min_matches=min_matches)


def test_rot_bin_closed_forms(ref):
    # bin = round(rot / 30) with rot in [0, 360): 13 bins (0..12), bin 12 = [345, 360) is NOT
    # folded into bin 0 -- ORB-SLAM's factor 1.0f/HISTO_LENGTH taken literally.
    for a in (0.0, 17.5, 180.0, 359.5):
        assert ref.lf_rot_bin(a, a) == 0
    for tenth in range(3600):
        rot = tenth / 10.0
        if abs((rot % 30.0) - 15.0) < 1e-3:
            continue
        assert ref.lf_rot_bin(rot, 0.0) == int(np.floor(rot / 30.0 + 0.5)), rot
    assert ref.lf_rot_bin(10.0, 20.0) == 12       # -10 -> 350 -> 11.67 -> 12
    assert ref.lf_rot_bin(0.0, 359.99) == 0       # -359.99 -> 0.01
    assert ref.lf_rot_bin(15.0, 0.0) == 1         # 15 * f32(1/30) = 0.50000006 -> 1
    assert max(ref.lf_rot_bin(r, 0.0) for r in np.linspace(0, 359.999, 5000)) == 12


def test_three_maxima_hand_worked(ref):
    p = _params(ref)
    rng = np.random.default_rng(3)
    # 16 level-0 keypoints on a 4x4 lattice 60 px apart (windows of r = 15 never overlap),
    # all at angle 0; point i sits on keypoint i with its exact descriptor (d = 0) and a last
    # angle that puts its match in a chosen bin: 10 x bin 0, 3 x bin 2 (60 deg),
    # 1 x bin 5 (150 deg), 1 x bin 7 (210 deg), 1 x bin 12 (350 deg).
    recs = [(0, 100 + 60 * (i % 4), 100 + 60 * (i // 4), 0.0) for i in range(16)]
    kps, desc, counts, recs = _frame(p, recs, rng)
    ang = [0.0] * 10 + [60.0] * 3 + [150.0, 210.0, 350.0]
    pts = [_point_at(float(kps[0, k]["x"]), float(kps[0, k]["y"]), 0, ang[k]) for k in range(16)]
    out, nm = _run(ref, p, kps, desc, counts, pts, [desc[0, k] for k in range(16)])
    assert (out["dist"] == 0).all()
    # ComputeThreeMaxima: max1 = 10 (bin 0), max2 = 3 (bin 2), max3 = 1 (bin 5: the first bin
    # whose count exceeds 0 after bin 2; bins 7 and 12 tie it and lose); 3 >= 1.0 and
    # 1 >= 0.1 * 10 = 1.0, so bins {0, 2, 5} survive and the matches in bins 7, 12 are removed.
    want = list(range(14)) + [-1, -1]
    assert out["idx"].tolist() == want and nm.tolist() == [14]
    # without the orientation check every point keeps its keypoint
    out2, nm2 = _run(ref, p, kps, desc, counts, pts, [desc[0, k] for k in range(16)], check=0)
    assert out2["idx"].tolist() == list(range(16)) and nm2.tolist() == [16]
    # 12 x bin 0, 1 x bin 3: max2 = 1 < 0.1 * 12 = 1.2 -> only bin 0 survives
    ang = [0.0] * 12 + [90.0] + [0.0] * 3
    pts = [_point_at(float(kps[0, k]["x"]), float(kps[0, k]["y"]), 0, ang[k]) for k in range(16)]
    out, nm = _run(ref, p, kps, desc, counts, pts, [desc[0, k] for k in range(16)])
    assert out["idx"].tolist() == [k if k != 12 else -1 for k in range(16)] and nm.tolist() == [15]


def test_dedup_th_high_and_taken(ref):
    p = _params(ref)
    rng = np.random.default_rng(4)
    kps, desc, counts, _ = _frame(p, [(0, 200, 200, 0.0), (0, 400, 300, 0.0)], rng)
    k0, k1 = desc[0, 0], desc[0, 1]
    x0, y0 = float(kps[0, 0]["x"]), float(kps[0, 0]["y"])
    x1, y1 = float(kps[0, 1]["x"]), float(kps[0, 1]["y"])
    pts = [_point_at(x0, y0, 0, 0.0), _point_at(x0 + 2, y0, 0, 0.0), _point_at(x0, y0 - 3, 0, 0.0),
           _point_at(x1, y1, 0, 0.0), _point_at(x1 + 1, y1 + 1, 0, 0.0)]
    # points 0..2 all want keypoint 0 at distances 7, 5, 5: the min (d, point) = (5, 1) wins;
    # point 3 is at distance 100 from keypoint 1 (accepted: <= TH_HIGH), point 4 at 101 (rejected)
    pd = [_flip(k0, 7, rng), _flip(k0, 5, rng), _flip(k0, 5, rng), _flip(k1, 100, rng), _flip(k1, 101, rng)]
    out, nm = _run(ref, p, kps, desc, counts, pts, pd)
    assert out["idx"].tolist() == [-1, 0, -1, 1, -1]
    assert out["dist"].tolist() == [7, 5, 5, 100, 101]
    assert out["dist2"].tolist() == [256] * 5        # one candidate per window
    # a taken keypoint is never a candidate
    taken = np.zeros((1, p.kp_capacity), np.uint8)
    taken[0, 0] = 1
    out, _ = _run(ref, p, kps, desc, counts, pts, pd, taken=taken)
    assert out["idx"].tolist() == [-1, -1, -1, 1, -1] and out["dist"][:3].tolist() == [256] * 3


def _gate_scene(ref, p, rng):
    """One keypoint on every level at (nearly) the same level-0 position; the point's
    descriptor is a copy of the level-l keypoint's with (l + 1) bit flips, so the best
    candidate is the LOWEST level the gate admits."""
    recs = []
    for l in range(p.n_levels):
        s = p.scale[l]
        recs.append((l, int(round(300 / s)), int(round(200 / s)), 0.0))
    kps, desc, counts, recs = _frame(p, recs, rng)
    base = desc[0, 0].copy()
    for l in range(p.n_levels):      # descriptors of level l = base with exactly l+1 flips
        desc[0, l] = _flip(base, l + 1, np.random.default_rng(100 + l))
    return kps, desc, counts, base


@pytest.mark.parametrize("octave,lmin,lmax", [(0, 0, 1), (3, 2, 4), (7, 6, 7)])
def test_level_gate_mono(ref, octave, lmin, lmax):
    p = _params(ref)
    kps, desc, counts, base = _gate_scene(ref, p, np.random.default_rng(5))
    # window r = 40 * scale[octave] >= 40 px covers every level's copy (rounding <= 4 px)
    out, _ = _run(ref, p, kps, desc, counts, [_point_at(300.0, 200.0, octave, 0.0)], [base], th=40.0)
    assert out["idx"][0] == lmin
    # candidates are exactly the levels lmin..lmax: best = lmin (lmin+1 flips), second lmin+1
    assert out["dist"][0] == lmin + 1
    assert out["dist2"][0] == (lmin + 2 if lmax > lmin else 256)


def test_level_gate_stereo_forward_backward(ref):
    p = _params(ref)
    kps, desc, counts, base = _gate_scene(ref, p, np.random.default_rng(6))
    cams = _cam()
    pt = [_point_at(300.0, 200.0, 3, 0.0)]
    mb = 0.5
    # last camera centre at z = -1 (the current camera moved forward by 1 > mb):
    # tlc = R_last * ow_cur + t_last = (0, 0, 1) -> forward -> levels [3, 7]
    fwd = _cam(t=(0.0, 0.0, 1.0))
    out, _ = _run(ref, p, kps, desc, counts, pt, [base], cams=cams, last=fwd, mb=mb, th=40.0)
    assert out["idx"][0] == 3 and out["dist2"][0] == 5
    # moved backward: tlc.z = -1 -> levels [0, 3]
    bwd = _cam(t=(0.0, 0.0, -1.0))
    out, _ = _run(ref, p, kps, desc, counts, pt, [base], cams=cams, last=bwd, mb=mb, th=40.0)
    assert out["idx"][0] == 0 and out["dist2"][0] == 2
    # |tlc.z| = 0.3 <= mb: neither -> [2, 4]; and mono (mb = 0) ignores the motion
    small = _cam(t=(0.0, 0.0, 0.3))
    out, _ = _run(ref, p, kps, desc, counts, pt, [base], cams=cams, last=small, mb=mb, th=40.0)
    assert out["idx"][0] == 2
    out, _ = _run(ref, p, kps, desc, counts, pt, [base], cams=cams, last=fwd, mb=0.0, th=40.0)
    assert out["idx"][0] == 2


def test_window_and_retry(ref):
    p = _params(ref)
    rng = np.random.default_rng(7)
    kps, desc, counts, _ = _frame(p, [(0, 300, 200, 0.0), (0, 500, 300, 0.0)], rng)
    x, y = float(kps[0, 0]["x"]), float(kps[0, 0]["y"])
    # the keypoint lies 20 px left of the projection: outside r = 15, inside r = 30
    pts = [_point_at(x + 20.0, y, 0, 0.0), _point_at(x + 14.0, y + 14.0, 0, 0.0)]
    pd = [desc[0, 0], desc[0, 0]]
    out, nm = _run(ref, p, kps, desc, counts, pts[:1], pd[:1], min_matches=0)
    assert out["idx"][0] == -1 and out["dist"][0] == 256 and nm[0] == 0
    out, nm = _run(ref, p, kps, desc, counts, pts[:1], pd[:1], min_matches=1)
    assert out["idx"][0] == 0 and nm[0] == 1           # retried with 2 * th = 30
    # 14 px diagonal is inside r = 15 (|dx| < r and |dy| < r, a square window)
    out, nm = _run(ref, p, kps, desc, counts, pts[1:], pd[1:], min_matches=0)
    assert out["idx"][0] == 0
    # both points: pass 1 keeps 1 match (< 2) -> retry: both claim keypoint 0 at d = 0,
    # dedup keeps point 0 -> the second pass result (1 match) stands
    out, nm = _run(ref, p, kps, desc, counts, pts, pd, min_matches=2)
    assert out["idx"].tolist() == [0, -1] and nm[0] == 1


def test_shifted_frame_physical_pin(ref):
    """A fronto-parallel textured plane at depth Z, camera moved sideways by (dx*Z/fx, dy*Z/fy):
    the image shifts by exactly (dx, dy) px, so every level-0 keypoint k of the last frame
    whose patch stays inside both images reappears in the current frame at (x+dx, y+dy) with
    the identical descriptor and angle; matched with d = 0 in bin 0."""
    p = _params(ref)
    w, h = 752, 480
    big = synth.make_frame(w + 16, h + 16, synth.frame_seed(13, 0, 0))
    dx, dy = 6, 4
    last = np.ascontiguousarray(big[8:8 + h, 8:8 + w])
    cur = np.ascontiguousarray(big[8 - dy:8 - dy + h, 8 - dx:8 - dx + w])   # cur(x+dx, y+dy) = last(x, y)
    kl, dl, cl = ref.orb_extract_batch(p, last[None])
    kc, dc, cc = ref.orb_extract_batch(p, cur[None])
    n0 = int(cl[0, 1])
    Z = 8.0
    pts = []
    for k in range(n0):
        x, y = float(kl[0, k]["x"]), float(kl[0, k]["y"])
        pts.append(_point_at(x, y, 0, float(kl[0, k]["angle_deg"]), Z=Z))
    cam = _cam(t=(dx * Z / FX, dy * Z / FY, 0.0))
    out, nm = _run(ref, p, kc, dc, cc, pts, [dl[0, k] for k in range(n0)], cams=cam, min_matches=0)
    cur_pos = {(int(kc[0, k]["lx"]), int(kc[0, k]["ly"])): k for k in range(int(cc[0, 1]))}
    have = [k for k in range(n0) if (int(kl[0, k]["lx"]) + dx, int(kl[0, k]["ly"]) + dy) in cur_pos]
    assert len(have) > 0.5 * n0
    hits = sum(out["idx"][k] == cur_pos[(int(kl[0, k]["lx"]) + dx, int(kl[0, k]["ly"]) + dy)] for k in have)
    assert hits >= 0.95 * len(have), (hits, len(have))
    for k in have:
        assert out["dist"][k] == 0
    # every kept match is in the zero-rotation bin
    for k in np.nonzero(out["idx"] >= 0)[0]:
        assert ref.lf_rot_bin(float(kl[0, k]["angle_deg"]), float(kc[0, out["idx"][k]]["angle_deg"])) == 0


def _synthetic(ref, shape="euroc", F=2, Q=500, seed=11, stereo_z=0.0):
    w, h = synth.SHAPES[shape]
    p = ref.params(w, h, 1000)
    frames = synth.make_frames(w, h, F, cfg=21)
    kps, desc, counts = ref.orb_extract_batch(p, frames)
    cams, last, pt_off, pts, pdesc = synth.make_last_frame(kps, desc, counts, p.n_levels, p.n_per_level, w, h, shape,
                                                           Q, seed, stereo_z=stereo_z)
    return p, kps, desc, counts, cams, last, pt_off, pts, pdesc


@pytest.mark.parametrize("mb,stereo_z", [(0.0, 0.0), (0.3, 1.0)])
def test_invariants_synthetic(ref, mb, stereo_z):
    p, kps, desc, counts, cams, last, pt_off, pts, pdesc = _synthetic(ref, stereo_z=stereo_z)
    out, nm = ref.match_last_frame(p, cams, last, mb, kps, desc, counts, None, pt_off, pts, pdesc, th=15.0,
                                   min_matches=20)
    L = p.n_levels
    for f in range(len(cams)):
        o = out[pt_off[f]:pt_off[f + 1]]
        m = o["idx"] >= 0
        assert nm[f] == m.sum() and m.sum() > 0.3 * len(o)
        assert len(set(o["idx"][m].tolist())) == m.sum()               # dedup
        assert (o["dist"][m] <= 100).all() and (o["dist"] <= o["dist2"]).all()
        k = kps[f, o["idx"][m]]
        lp = pts[pt_off[f]:pt_off[f + 1]][m]
        assert (np.abs(k["level"].astype(int) - lp["octave"]) <= (L if mb > 0 else 1)).all()
        bins = {ref.lf_rot_bin(float(a), float(b)) for a, b in zip(lp["angle_deg"], k["angle_deg"])}
        assert len(bins) <= 3
        for kk, d in zip(o["idx"][m], o["dist"][m]):
            assert ref.hamming(pdesc[pt_off[f] + int(np.nonzero((o["idx"] == kk))[0][0])], desc[f, kk]) == d


def test_numpy_bruteforce_no_orientation(ref):
    """Steps 1-4 written out in numpy (float32 arithmetic in the same order) on the synthetic
    workload; orientation check off, no retry."""
    p, kps, desc, counts, cams, last, pt_off, pts, pdesc = _synthetic(ref, F=1, Q=400, seed=12)
    out, _ = ref.match_last_frame(p, cams, None, 0.0, kps, desc, counts, None, pt_off, pts, pdesc, th=15.0,
                                  check_orientation=0, min_matches=0)
    f32 = np.float32
    c = cams[0]
    R, t = c["R"].reshape(3, 3), c["t"]
    n = int(counts[0, p.n_levels])
    kx, ky, kl = kps[0, :n]["x"], kps[0, :n]["y"], kps[0, :n]["level"].astype(int)
    bits = np.unpackbits(desc[0, :n], axis=-1)
    best = []
    for i, pt in enumerate(pts):
        P = pt["pos"]
        pc = [f32(f32(f32(R[r, 0] * P[0]) + f32(R[r, 1] * P[1])) + f32(R[r, 2] * P[2])) + t[r] for r in range(3)]
        pc = [f32(v) for v in pc]
        res = (-1, 256, 256)
        if pc[2] >= 0:
            u = f32(f32(f32(c["fx"] * pc[0]) / pc[2]) + c["cx"])
            v = f32(f32(f32(c["fy"] * pc[1]) / pc[2]) + c["cy"])
            if c["min_x"] <= u <= c["max_x"] and c["min_y"] <= v <= c["max_y"]:
                o = int(pt["octave"])
                r = f32(f32(15.0) * f32(p.scale[o]))
                ok = (kl >= o - 1) & (kl <= o + 1) & (np.abs(f32(kx - u)) < r) & (np.abs(f32(ky - v)) < r)
                d = (bits != np.unpackbits(pdesc[i])).sum(-1)
                cand = sorted((int(d[k]), k) for k in np.nonzero(ok)[0])
                if cand:
                    d1, k1 = cand[0]
                    d2 = cand[1][0] if len(cand) > 1 else 256
                    res = (k1 if d1 <= 100 else -1, d1, d2)
        best.append(res)
    idx = np.array([b[0] for b in best])
    for k in set(idx[idx >= 0].tolist()):          # dedup: min (d, i)
        claim = [i for i in range(len(best)) if idx[i] == k]
        win = min(claim, key=lambda i: (best[i][1], i))
        for i in claim:
            if i != win:
                idx[i] = -1
    assert out["idx"].tolist() == idx.tolist()
    assert out["dist"].tolist() == [b[1] for b in best]
    assert out["dist2"].tolist() == [b[2] for b in best]
