"""e2e diagnosis with the current tick (O13 + projection + window, map resident in HBM): host cost
per ss_track_tick call and device time per tick, with / without graph reuse and output copies,
plus the raw pinned-copy bandwidths of one tick's frames (H2D) and outputs (D2H)."""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline  # noqa: E402

w, h = synth.SHAPES["euroc"]
B, Qc, nf = 4, 5000, 1000
P = int(sys.argv[1]) if len(sys.argv) > 1 else 4
DISTINCT = len(sys.argv) > 2 and sys.argv[2] == "distinct"  # one pinned frame buffer + map state per context
Q = Qc * B
frames = synth.make_frames(w, h, B, cfg=2)
pipes = [OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=Q) for _ in range(P)]
p = pipes[0].params
cap = p.kp_capacity
pipes[0].extract(torch.from_numpy(frames).cuda())
k, d, c = pipes[0].results(B)
cm, pt, pf, qd, tk = synth.make_local_map(k, d, c, 8, p.scale_factor, np.array(p.n_per_level[:8]), w, h, "euroc",
                                          Qc, seed=1)
_, last, off, lp, ld = synth.make_last_frame(k, d, c, 8, np.array(p.n_per_level[:8]), w, h, "euroc", 600, 2, cams=cm)
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).pin_memory()
hfs = [pin(frames) for _ in range(P if DISTINCT else 1)]
hf, hc, hoff = hfs[0], pin(cm), pin(off)
devs = [[pin(a).cuda() for a in (pt, pf, qd, tk, lp, ld)] for _ in range(P if DISTINCT else 1)]
outs = [{k_: torch.zeros(n, dtype=torch.uint8).pin_memory() for k_, n in
         (("kps", B * cap * 20), ("desc", B * cap * 32), ("counts", B * 9 * 4), ("matches", Q * 12),
          ("lf_matches", len(lp) * 12), ("lf_n_matches", B * 4))} for _ in range(P)]
streams = [torch.cuda.Stream() for _ in range(P)]


def mk(q, copies, reuse):
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch, io.reuse_graph, io.map_resident = hfs[q % len(hfs)].data_ptr(), h * w, w, reuse, 1
    io.cams, io.n_points = hc.data_ptr(), Q
    io.points, io.point_frame, io.point_desc, io.taken, io.lf_points, io.lf_desc = (t.data_ptr() for t in devs[q % len(devs)])
    io.th, io.lf_offsets, io.lf_th, io.lf_min_matches = 1.0, hoff.data_ptr(), 15.0, 20
    if copies:
        for k_ in outs[q]:
            setattr(io, k_, outs[q][k_].data_ptr())
    return io


cfg = ss.window_cfg()
for reuse in (0, 1):
    for copies in (True, False):
        ios = [mk(q, copies, reuse) for q in range(P)]
        for _ in range(5):
            for q in range(P):
                ss.ss_track_tick(pipes[q].ctx, B, cfg, ios[q], streams[q].cuda_stream)
        torch.cuda.synchronize()
        K = 1000
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
        print(f"reuse_graph={reuse} copies_out={copies}: host {1e6 * (h1 - h0) / K:.1f} us/call, device "
              f"{1000 * t0.elapsed_time(t1) / K:.1f} us/tick -> {B * K / (t0.elapsed_time(t1) / 1000):.0f} frames/s")
# raw copies
dh = torch.empty(hf.numel(), dtype=torch.uint8, device="cuda")
ob = sum(t.numel() for t in outs[0].values())
do = torch.empty(ob, dtype=torch.uint8, device="cuda")
ho = torch.empty(ob, dtype=torch.uint8).pin_memory()
for name, fn, nbytes in (("H2D frames", lambda s: dh.copy_(hf, non_blocking=True), hf.numel()),
                         ("D2H outputs (one copy)", lambda s: ho.copy_(do, non_blocking=True), ob)):
    torch.cuda.synchronize()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record()
    for _ in range(200):
        fn(None)
    t1.record()
    torch.cuda.synchronize()
    us = 1000 * t0.elapsed_time(t1) / 200
    print(f"{name}: {nbytes} B in {us:.1f} us = {nbytes / us / 1e3:.1f} GB/s")
