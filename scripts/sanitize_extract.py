"""Small runs of every kernel for compute-sanitizer (memcheck / racecheck / synccheck): extract
(quadtree and grid top-N), window match, projection, frame-to-frame matching (cluster kernel,
with its 2*th retry), stereo, brute force (tensor cores, replicated and map-sharded; skipped
when SANITIZE_BRUTE=0) and one ss_track_tick.

usage: compute-sanitizer --tool racecheck python scripts/sanitize_extract.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_out, to_device_records  # noqa: E402


def main():
    w, h, B = 320, 240, 2
    frames = synth.make_frames(w, h, B, cfg=7)
    noise = np.random.default_rng(1).integers(0, 256, size=(h, w), dtype=np.uint8)
    frames[1] = noise  # the overflow / fallback paths too
    pipe = OrbPipeline(w, h, 300, 4, max_frames=B, max_queries=512)
    pipe.extract(torch.from_numpy(frames).cuda())
    kps, desc, counts = pipe.results(B)
    q = np.zeros(512, ss.QUERY_DTYPE)
    rng = np.random.default_rng(2)
    q["frame"] = rng.integers(0, B, 512)
    q["u"], q["v"] = rng.uniform(0, w, 512), rng.uniform(0, h, 512)
    q["pred_level"] = rng.integers(0, 4, 512)
    q["radius"] = 12.0
    qd = rng.integers(0, 256, (512, 32), dtype=np.uint8)
    out = match_out(512, "cuda")
    pipe.match_window(B, to_device_records(q, "cuda"), torch.from_numpy(qd).cuda(), out)
    # projection of a small local map, then the projected queries
    cams = np.zeros(B, synth.CAMERA_DTYPE)
    cams["R"] = np.eye(3, dtype=np.float32).ravel()
    cams["fx"], cams["fy"], cams["cx"], cams["cy"] = 300.0, 300.0, w / 2, h / 2
    cams["max_x"], cams["max_y"] = w, h
    pts = np.zeros(512, synth.MAP_POINT_DTYPE)
    pts["pos"] = np.stack([rng.uniform(-2, 2, 512), rng.uniform(-2, 2, 512), rng.uniform(-1, 8, 512)], 1)
    pts["normal"] = [0.0, 0.0, 1.0]
    pts["min_dist"], pts["max_dist"] = 0.5, 6.0
    pf = rng.integers(-1, B + 1, 512).astype(np.int32)
    qb = torch.zeros((512, 20), dtype=torch.uint8, device="cuda")
    pipe.project(B, torch.from_numpy(cams.view(np.uint8).reshape(B, -1).copy()).cuda(),
                 torch.from_numpy(pts.view(np.uint8).reshape(512, -1).copy()).cuda(), torch.from_numpy(pf).cuda(), qb)
    pipe.match_window(B, qb, torch.from_numpy(qd).cuda(), out)
    # frame-to-frame matching (O13): every frame retried (min_matches huge), stereo gates on
    kk, dd, cc = pipe.results(B)
    lcams, llast, loff, lp, ld = synth.make_last_frame(kk, dd, cc, 4, np.array([100, 80, 70, 50]), w, h, "euroc", 200,
                                                       3, stereo_z=1.0)
    lo = match_out(len(lp), "cuda")
    ln = torch.zeros(B, dtype=torch.int32, device="cuda")
    lm = torch.zeros((B, pipe.cap), dtype=torch.uint8, device="cuda")
    for mm, mb in ((20, 0.0), (10 ** 6, 0.3)):
        pipe.match_last_frame(B, to_device_records(lcams, "cuda"), torch.from_numpy(loff).cuda(),
                              to_device_records(lp, "cuda"), torch.from_numpy(ld).cuda(), lo, ln,
                              last_cams=to_device_records(llast, "cuda"), mb=mb, min_matches=mm, matched=lm)
    torch.cuda.synchronize()
    # stereo on the (frame 0, frame 1) pair
    d_frames = torch.from_numpy(frames).cuda()
    ur = torch.zeros((1, pipe.cap), dtype=torch.float32, device="cuda")
    dp = torch.zeros_like(ur)
    pipe.extract(d_frames)
    pipe.stereo(d_frames, 200.0, 0.5, ur, dp)
    # grid top-N distribution
    pipe.set_distribution(ss.SS_DIST_GRID_TOPN)
    pipe.extract(d_frames)
    pipe.set_distribution(ss.SS_DIST_QUADTREE)
    if os.environ.get("SANITIZE_BRUTE", "1") == "1":
        mp = rng.integers(0, 256, (300, 32), dtype=np.uint8)
        bp = OrbPipeline(w, h, 300, 4, max_frames=B, max_map=300)
        bp.extract(d_frames)
        bo = torch.zeros((B * bp.cap, 3), dtype=torch.int32, device="cuda")
        bp.match_brute(B, torch.from_numpy(mp).cuda(), bo)
        parts = torch.zeros((2, B, bp.cap, 2), dtype=torch.int64, device="cuda")  # F4: two shards + merge
        dm = torch.from_numpy(mp).cuda()
        for r, (a, b) in enumerate(((0, 130), (130, 300))):
            ss.ss_match_brute_partial(bp.ctx, B, bp.desc, bp.counts, dm[a:b], b - a, a, parts[r])
        ss.ss_match_brute_merge(bp.ctx, B, bp.counts, 2, parts, ss.brute_cfg(), bo)
        torch.cuda.synchronize()
        bp.close()
    # one tick from host memory
    hf = torch.from_numpy(frames.copy()).pin_memory()
    hk = torch.zeros(B * pipe.cap * 20, dtype=torch.uint8).pin_memory()
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch, io.kps = hf.data_ptr(), h * w, w, hk.data_ptr()
    ss.ss_track_tick(pipe.ctx, B, ss.window_cfg(), io)
    torch.cuda.synchronize()
    print("sanitize run ok", int(counts[:, -1].sum()), "keypoints")


if __name__ == "__main__":
    main()
