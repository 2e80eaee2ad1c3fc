"""Diagnose the end-to-end (host memory) path: host cost per ss_track_tick call and device time
per tick, for P contexts/streams in flight, with and without the copies."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline  # noqa: E402

w, h = synth.SHAPES["euroc"]
B, Q, nf = 4, 20000, 1000
frames = synth.make_frames(w, h, B, cfg=2)
P = int(sys.argv[1]) if len(sys.argv) > 1 else 4
pipes = [OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=Q) for _ in range(P)]
p = pipes[0].params
pipes[0].extract(torch.from_numpy(frames).cuda())
k, d, c = pipes[0].results(B)
cm, pt, pf, qd, tk = synth.make_local_map(k, d, c, 8, p.scale_factor, np.array(p.n_per_level[:8]), w, h, "euroc",
                                          Q // B, seed=1)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).pin_memory()
hin = [pin(a) for a in (frames, cm, pt, pf, qd, tk)]
cap = p.kp_capacity
outs = [{k_: torch.zeros(n, dtype=torch.uint8).pin_memory() for k_, n in
         (("kps", B * cap * 20), ("desc", B * cap * 32), ("counts", B * 9 * 4), ("matches", Q * 12))} for _ in range(P)]
streams = [torch.cuda.Stream() for _ in range(P)]


def mk(q, copies=True):
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch = hin[0].data_ptr(), h * w, w
    io.cams, io.n_points, io.points, io.point_frame = hin[1].data_ptr(), Q, hin[2].data_ptr(), hin[3].data_ptr()
    io.point_desc, io.taken, io.th = hin[4].data_ptr(), hin[5].data_ptr(), 1.0
    if copies:
        for k_ in outs[q]:
            setattr(io, k_, outs[q][k_].data_ptr())
    return io


cfg = ss.window_cfg()
for copies in (True, False):
    ios = [mk(q, copies) for q in range(P)]
    for _ in range(5):
        for q in range(P):
            ss.ss_track_tick(pipes[q].ctx, B, cfg, ios[q], streams[q].cuda_stream)
    torch.cuda.synchronize()
    K = 200
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(streams[0])
    for q in range(1, P):
        streams[q].wait_event(t0)
    h0 = time.perf_counter()
    for s in range(K):
        q = s % P
        ss.ss_track_tick(pipes[q].ctx, B, cfg, ios[q], streams[q].cuda_stream)
    h1 = time.perf_counter()
    for q in range(1, P):
        streams[0].wait_stream(streams[q])
    t1.record(streams[0])
    torch.cuda.synchronize()
    print(f"P={P} copies_out={copies}: host {1e6 * (h1 - h0) / K:.1f} us/call, device {1000 * t0.elapsed_time(t1) / K:.1f} "
          f"us/tick -> {B * K / (t0.elapsed_time(t1) / 1000):.0f} frames/s")
