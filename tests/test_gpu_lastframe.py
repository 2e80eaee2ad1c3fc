"""GPU parity of O13 frame-to-frame projection matching (k_lastframe.cu, ss_match_last_frame)
vs the oracle: every (idx, dist, dist2) and every per-frame match count bit-exact.

The keypoints fed to both sides are the ORACLE's extraction (uploaded), so the rotation-bin
decisions see identical angles; the chained GPU-extract -> GPU-match path is checked
separately, where the extraction's angles may differ from the oracle's by <= 1e-4 rad."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import oracle
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    oracle.build()
    return torch, oracle


_cache = {}


def _workload(ref, shape, F, Q, seed, stereo_z=0.0, pos_sigma=1.5):
    key = (shape, F)
    w, h = synth.SHAPES[shape]
    nf = 2000 if shape == "kitti" else 1000
    if key not in _cache:
        p = ref.params(w, h, nf)
        frames = synth.make_frames(w, h, F, cfg=31 + len(_cache))
        _cache[key] = (p, frames) + tuple(ref.orb_extract_batch(p, frames))
    p, frames, kps, desc, counts = _cache[key]
    lf = synth.make_last_frame(kps, desc, counts, p.n_levels, p.n_per_level, w, h, shape, Q, seed,
                               stereo_z=stereo_z, pos_sigma=pos_sigma)
    return (p, frames, kps, desc, counts) + lf


def _gpu_match(torch, p, kps, desc, counts, cams, last, pt_off, pts, pdesc, mb, th, check, min_matches, taken=None,
               max_frames=None):
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_records, to_device_records
    F = kps.shape[0]
    pipe = OrbPipeline(p.width, p.height, p.n_features, p.n_levels, max_frames=max_frames or F, max_queries=1)
    dev = "cuda"
    tk = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(dev)  # noqa: E731
    d_kps = tk(np.ascontiguousarray(kps).view(np.uint8).reshape(F, -1))
    d_desc, d_counts = tk(desc), tk(counts.astype(np.int32))
    d_cams = to_device_records(cams, dev)
    d_last = to_device_records(last, dev) if last is not None else None
    d_off = tk(pt_off.astype(np.int32))
    n = len(pts)
    d_pts = to_device_records(pts, dev) if n else torch.zeros((1, 24), dtype=torch.uint8, device=dev)
    d_pd = tk(pdesc) if n else torch.zeros((1, 32), dtype=torch.uint8, device=dev)
    out = torch.full((max(n, 1), 3), 7, dtype=torch.int32, device=dev)
    nm = torch.full((F,), -5, dtype=torch.int32, device=dev)
    d_taken = tk(taken) if taken is not None else None
    mask = torch.full((F, p.kp_capacity), 9, dtype=torch.uint8, device=dev)
    ss.ss_match_last_frame(pipe.ctx, F, d_cams, d_last, mb, d_kps, d_desc, d_counts, d_taken, d_off, d_pts, d_pd, th,
                           100, check, min_matches, out, nm, mask, torch.cuda.current_stream())
    torch.cuda.synchronize()
    got = match_records(out)[:n]
    pipe.close()
    # matched mask = taken | kept matches
    want_mask = np.zeros((F, p.kp_capacity), np.uint8) if taken is None else (taken != 0).astype(np.uint8)
    for f in range(F):
        o = got[pt_off[f]:pt_off[f + 1]]
        want_mask[f, o["idx"][o["idx"] >= 0]] = 1
    assert (mask.cpu().numpy() == want_mask).all()
    return got, nm.cpu().numpy()


CASES = [  # shape, F, Q, mb, stereo_z, th, check, min_matches, pos_sigma
    ("euroc", 4, 600, 0.0, 0.0, 15.0, 1, 20, 1.5),
    ("euroc", 4, 600, 0.0, 0.0, 15.0, 0, 0, 1.5),
    ("euroc", 4, 600, 0.0, 0.0, 7.0, 1, 10 ** 6, 6.0),     # every frame retried with 2*th
    ("euroc", 4, 900, 0.0, 0.0, 4.0, 1, 250, 5.0),         # some frames retried
    ("tum", 3, 2000, 0.0, 0.0, 15.0, 1, 20, 1.5),         # more points than keypoints: many claims
    ("kitti", 2, 1200, 0.25, 1.0, 7.0, 1, 20, 1.5),        # stereo forward / backward gates
]


@pytest.mark.parametrize("case", CASES, ids=[f"{c[0]}-th{c[5]}-chk{c[6]}-min{c[7]}-mb{c[3]}" for c in CASES])
def test_lastframe_parity(env, case):
    torch, ref = env
    shape, F, Q, mb, sz, th, check, mm, ps = case
    p, frames, kps, desc, counts, cams, last, pt_off, pts, pdesc = _workload(ref, shape, F, Q, 77, sz, ps)
    rng = np.random.default_rng(5)
    taken = (rng.random(counts.shape[:1] + (p.kp_capacity,)) < 0.05).astype(np.uint8)
    want, wn = ref.match_last_frame(p, cams, last, mb, kps, desc, counts, taken, pt_off, pts, pdesc, th=th,
                                    check_orientation=check, min_matches=mm)
    got, gn = _gpu_match(torch, p, kps, desc, counts, cams, last, pt_off, pts, pdesc, mb, th, check, mm, taken)
    assert (wn > 0).all()
    assert (got == want).all(), np.nonzero(got != want)[0][:10]
    assert (gn == wn).all()


def test_lastframe_edge_cases(env):
    torch, ref = env
    p, frames, kps, desc, counts, cams, last, pt_off, pts, pdesc = _workload(ref, "euroc", 4, 300, 78)
    pts = pts.copy()
    pts["octave"][::17] = -1                     # invalid octaves: no candidates
    pts["octave"][5::17] = p.n_levels
    # frame 1 has no points, frame 3 has one; frame 2 gets every other point
    off = np.array([0, 300, 300, 900, 901], np.int32)
    sel = np.concatenate([np.arange(0, 300), np.arange(600, 1200), np.arange(900, 901)])
    P, D = pts[sel], pdesc[sel]
    want, wn = ref.match_last_frame(p, cams, None, 0.0, kps, desc, counts, None, off, P, D, th=15.0, min_matches=20)
    got, gn = _gpu_match(torch, p, kps, desc, counts, cams, None, off, P, D, 0.0, 15.0, 1, 20)
    assert (got == want).all() and (gn == wn).all()
    assert wn[1] == 0
    # zero points in every frame
    z = np.zeros(5, np.int32)
    got, gn = _gpu_match(torch, p, kps, desc, counts, cams, None, z, P[:0], D[:0], 0.0, 15.0, 1, 20)
    assert (gn == 0).all()
    # a frame with no keypoints
    counts0 = counts.copy()
    counts0[2] = 0
    want, wn = ref.match_last_frame(p, cams, None, 0.0, kps, desc, counts0, None, off, P, D, th=15.0, min_matches=20)
    got, gn = _gpu_match(torch, p, kps, desc, counts0, cams, None, off, P, D, 0.0, 15.0, 1, 20)
    assert (got == want).all() and (gn == wn).all() and wn[2] == 0


def test_lastframe_chained_gpu_extract(env):
    """GPU extract -> GPU O13 vs oracle extract -> oracle O13: identical except where a rotation
    bin sits within the angle tolerance (1e-4 rad) of a bin edge."""
    torch, ref = env
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_records, to_device_records
    p, frames, kps, desc, counts, cams, last, pt_off, pts, pdesc = _workload(ref, "euroc", 4, 600, 79)
    F = len(frames)
    want, wn = ref.match_last_frame(p, cams, None, 0.0, kps, desc, counts, None, pt_off, pts, pdesc, th=15.0,
                                    min_matches=20)
    pipe = OrbPipeline(p.width, p.height, p.n_features, p.n_levels, max_frames=F, max_queries=1)
    pipe.extract(torch.from_numpy(frames).cuda())
    out = torch.zeros((len(pts), 3), dtype=torch.int32, device="cuda")
    nm = torch.zeros(F, dtype=torch.int32, device="cuda")
    pipe.match_last_frame(F, to_device_records(cams, "cuda"), torch.from_numpy(pt_off).cuda(),
                          to_device_records(pts, "cuda"), torch.from_numpy(pdesc).cuda(), out, nm)
    gk, gd, gc = pipe.results(F)
    got = match_records(out)
    pipe.close()
    assert (gc == counts).all() and (gd == desc).all()
    # exact: the oracle's O13 on the GPU keypoints (GPU angles, <= 1e-4 rad from the oracle's)
    # takes every rotation-bin decision on the same values as the kernel
    want_g, wn_g = ref.match_last_frame(p, cams, None, 0.0, gk, desc, counts, None, pt_off, pts, pdesc, th=15.0,
                                        min_matches=20)
    assert (got == want_g).all()
    np.testing.assert_array_equal(nm.cpu().numpy(), wn_g)
    # and against the oracle's own extraction: identical except where a rotation bin sits within
    # the angle tolerance of a bin edge
    edge = np.zeros(len(pts), bool)
    for f in range(F):
        for i in range(pt_off[f], pt_off[f + 1]):
            k = want["idx"][i] if want["idx"][i] >= 0 else got["idx"][i]
            if k < 0:
                continue
            rot = (float(pts["angle_deg"][i]) - float(kps[f, k]["angle_deg"])) % 360.0
            if abs((rot % 30.0) - 15.0) < 0.02:
                edge[i] = True
    bad = (got != want) & ~edge
    assert not bad.any(), np.nonzero(bad)[0][:10]
