"""ss_track_tick (one C-ABI call per tick from host memory) vs the oracle: keypoints,
descriptors, counts, stereo u_right / depth and window matches (search local points) of a
KITTI-shaped stereo batch, and brute matches of an EuRoC batch, bit-exact (angle <= 1e-4 rad)."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    return torch


def _check_extract(p, kps, desc, counts, frames, ref):
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    out = []
    for f in range(len(frames)):
        rk, rd, rc = ref.orb_extract(p, frames[f])
        n = int(rc[-1])
        gk = np.ascontiguousarray(kps[f]).reshape(-1).view(ss.KEYPOINT_DTYPE)
        np.testing.assert_array_equal(counts[f], rc)
        for fld in ("lx", "ly", "level", "response", "x", "y"):
            np.testing.assert_array_equal(gk[fld][:n], rk[fld][:n], err_msg=fld)
        da = np.radians(np.abs(gk["angle_deg"][:n].astype(np.float64) - rk["angle_deg"][:n]))
        assert np.minimum(da, 2 * np.pi - da).max(initial=0) <= 1e-4
        np.testing.assert_array_equal(desc[f][:n], rd[:n])
        out.append((rk, rd, rc))
    return out


def test_track_tick_stereo_window(torch_cuda, ref):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["kitti"]
    frames = np.stack([im for i in range(2) for im in synth.make_stereo_pair(w, h, seed=90 + i)])
    B, Q, nf = 4, 2000, 2000
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    cm, pt, pf, qd, tk = synth.make_local_map(rk[::2], rd[::2], rc[::2], 8, p.scale_factor,
                                              np.array(p.n_per_level[:8]), w, h, "kitti", Q // 2, seed=9)
    pf = pf * 2
    cams = np.zeros(B, synth.CAMERA_DTYPE)
    cams[::2] = cm
    taken = np.zeros((B, cap), np.uint8)
    taken[::2] = tk
    base = synth.STEREO_BASELINE["kitti"]
    bf = float(np.float32(synth.INTRINSICS["kitti"][0] * base))
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).pin_memory()
    hf, hc, hp, hpf, hqd, htk = (pin(a) for a in (frames, cams, pt, pf, qd, taken))
    o = {k: torch.zeros(n, dtype=torch.uint8).pin_memory()
         for k, n in (("kps", B * cap * 20), ("desc", B * cap * 32), ("counts", B * 9 * 4), ("matches", Q * 12),
                      ("uright", 2 * cap * 4), ("depth", 2 * cap * 4))}
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch, io.bf, io.baseline = hf.data_ptr(), h * w, w, bf, base
    io.cams, io.n_points, io.points, io.point_frame = hc.data_ptr(), Q, hp.data_ptr(), hpf.data_ptr()
    io.point_desc, io.taken, io.th = hqd.data_ptr(), htk.data_ptr(), 1.0
    for k in o:
        setattr(io, k, o[k].data_ptr())
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=Q)
    ss.ss_track_tick(pipe.ctx, B, ss.window_cfg(), io)
    torch.cuda.synchronize()
    kps = o["kps"].numpy().reshape(B, cap, 20)
    desc = o["desc"].numpy().reshape(B, cap, 32)
    counts = o["counts"].numpy().view(np.int32).reshape(B, 9)
    _check_extract(p, kps, desc, counts, frames, ref)
    ur = o["uright"].numpy().view(np.float32).reshape(2, cap)
    dp = o["depth"].numpy().view(np.float32).reshape(2, cap)
    for i in range(2):
        u_w, d_w, _ = ref.stereo_match(p, frames[2 * i], frames[2 * i + 1], rk[2 * i], rd[2 * i], rc[2 * i],
                                       rk[2 * i + 1], rd[2 * i + 1], rc[2 * i + 1], bf, base)
        n = int(rc[2 * i][-1])
        np.testing.assert_array_equal(ur[i, :n].view(np.uint32), u_w[:n].view(np.uint32))
        np.testing.assert_array_equal(dp[i, :n].view(np.uint32), d_w[:n].view(np.uint32))
    q = ref.project_points(p, cams, pt, pf, 1.0)
    want = ref.match_window(p, rk, rd, rc, taken, q, qd)
    got = o["matches"].numpy().view(ref.MATCH_DTYPE).reshape(-1)
    np.testing.assert_array_equal(got, want)
    assert (got["idx"] >= 0).sum() > 100
    pipe.close()


def test_track_tick_brute(torch_cuda, ref):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["euroc"]
    B, nf, n_map = 3, 1250, 3000
    frames = synth.make_frames(w, h, B, cfg=5)
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    mp = synth.make_brute_map([rd[b][: rc[b][-1]] for b in range(B)], n_map, seed=3, n_from_kps=1000)
    d_map = torch.from_numpy(mp).cuda()
    hf = torch.from_numpy(frames.copy()).pin_memory()
    hm = torch.zeros(B * cap * 12, dtype=torch.uint8).pin_memory()
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch = hf.data_ptr(), h * w, w
    io.d_map_desc, io.n_map, io.matches = d_map.data_ptr(), n_map, hm.data_ptr()
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B, max_map=n_map)
    ss.ss_track_tick(pipe.ctx, B, ss.brute_cfg(), io)
    torch.cuda.synchronize()
    got = hm.numpy().view(ref.MATCH_DTYPE).reshape(B, cap)
    want = ref.match_brute(p, rd, rc, mp, 50, 3, 4)
    for b in range(B):
        n = int(rc[b][-1])
        np.testing.assert_array_equal(got[b, :n], want[b, :n])
    pipe.close()


@pytest.mark.parametrize("resident,packed", [(0, 0), (1, 0), (1, 1)])
def test_track_tick_lastframe_window(torch_cuda, ref, resident, packed):
    """Mono tick with frame-to-frame matching (O13) before search local points: the window
    match skips keypoints that are taken or kept by O13.  Oracle chain: extract -> O13 ->
    taken | kept -> O11 -> O9.  packed: every output through ss_tick_io.out_packed (one D2H
    copy; ss_tick_packed_layout's sections) and the frames, cameras and last-frame offsets
    through ss_tick_io.in_packed (one H2D copy), direct and replayed from the cached graph."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["euroc"]
    B, Qm, Qlf, nf = 4, 1500, 600, 1000
    frames = synth.make_frames(w, h, B, cfg=41)
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    cm, pt, pf, qd, tk = synth.make_local_map(rk, rd, rc, 8, p.scale_factor, np.array(p.n_per_level[:8]), w, h,
                                              "euroc", Qm, seed=19)
    _, last, off, lp, ld = synth.make_last_frame(rk, rd, rc, 8, np.array(p.n_per_level[:8]), w, h, "euroc", Qlf,
                                                 seed=20, cams=cm)
    pin = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).pin_memory()
    hf, hc, hp, hpf, hqd, htk, hoff, hlp, hld = (pin(a) for a in (frames, cm, pt, pf, qd, tk, off, lp, ld))
    o = {k: torch.zeros(n, dtype=torch.uint8).pin_memory()
         for k, n in (("kps", B * cap * 20), ("desc", B * cap * 32), ("counts", B * 9 * 4),
                      ("matches", B * Qm * 12), ("lf_matches", B * Qlf * 12), ("lf_n_matches", B * 4))}
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch = hf.data_ptr(), h * w, w
    io.cams, io.n_points, io.points, io.point_frame = hc.data_ptr(), B * Qm, hp.data_ptr(), hpf.data_ptr()
    io.point_desc, io.taken, io.th = hqd.data_ptr(), htk.data_ptr(), 1.0
    io.lf_offsets, io.lf_points, io.lf_desc = hoff.data_ptr(), hlp.data_ptr(), hld.data_ptr()
    io.lf_th, io.lf_min_matches = 15.0, 20
    if resident:  # the map state lives in HBM (server state): device pointers, not copied
        dev = [t.cuda() for t in (hp, hpf, hqd, htk, hlp, hld)]
        io.map_resident = 1
        io.points, io.point_frame, io.point_desc, io.taken, io.lf_points, io.lf_desc = (t.data_ptr() for t in dev)
    for k in o:
        setattr(io, k, o[k].data_ptr())
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=B * Qm)
    if packed:
        lay = ss.ss_tick_packed_layout(pipe.ctx, B, B * Qm, int(off[-1]))
        assert (lay[:8] % 256 == 0).all()
        blk = torch.full((int(lay[8]),), 0xAB, dtype=torch.uint8).pin_memory()
        io.out_packed = blk.data_ptr()
        # inputs too: frames + cams + lf_offsets in one block; the separate pointers are ignored
        ilay = ss.ss_tick_packed_in_layout(pipe.ctx, B, h * w)
        iblk = torch.zeros(int(ilay[3]), dtype=torch.uint8).pin_memory()
        for j, t_ in enumerate((hf, hc, hoff)):
            iblk[int(ilay[j]):int(ilay[j]) + t_.numel()].copy_(t_)
        io.in_packed = iblk.data_ptr()
        io.frames, io.cams, io.lf_offsets = None, None, None
        io.reuse_graph = 1
        st = torch.cuda.Stream()
        for _ in range(3):  # direct, capture, replay: the block is rewritten every time
            blk.fill_(0xAB)
            ss.ss_track_tick(pipe.ctx, B, ss.window_cfg(), io, st)
            torch.cuda.synchronize()
        names = ["kps", "desc", "counts", "lf_n_matches", "lf_matches", "matches"]
        for j, k in enumerate(names):
            o[k] = blk[int(lay[j]):int(lay[j]) + o[k].numel()]
    else:
        ss.ss_track_tick(pipe.ctx, B, ss.window_cfg(), io)
        torch.cuda.synchronize()
    kps = o["kps"].numpy().reshape(B, cap, 20)
    desc = o["desc"].numpy().reshape(B, cap, 32)
    counts = o["counts"].numpy().view(np.int32).reshape(B, 9)
    _check_extract(p, kps, desc, counts, frames, ref)
    # O13's rotation bins are integer decisions taken on the keypoint angles, which may differ
    # from the oracle's by <= 1e-4 rad (checked above; everything else is bit-exact).  Both
    # sides take the decision on the same values: the oracle's O13 runs on the GPU keypoints
    # (GPU angles), so the comparison is exact for any seed.
    gk = np.ascontiguousarray(kps).view(ref.KEYPOINT_DTYPE).reshape(B, cap)
    want_lf, want_n = ref.match_last_frame(p, cm, None, 0.0, gk, rd, rc, tk, off, lp, ld, th=15.0, min_matches=20)
    got_lf = o["lf_matches"].numpy().view(ref.MATCH_DTYPE).reshape(-1)
    np.testing.assert_array_equal(got_lf, want_lf)
    np.testing.assert_array_equal(o["lf_n_matches"].numpy().view(np.int32), want_n)
    assert (want_n > 100).all()
    mask = (tk != 0).astype(np.uint8)
    for f in range(B):
        s = want_lf[off[f]:off[f + 1]]
        mask[f, s["idx"][s["idx"] >= 0]] = 1
    q = ref.project_points(p, cm, pt, pf, 1.0)
    want = ref.match_window(p, rk, rd, rc, mask, q, qd)
    got = o["matches"].numpy().view(ref.MATCH_DTYPE).reshape(-1)
    np.testing.assert_array_equal(got, want)
    assert (got["idx"] >= 0).sum() > 100
    pipe.close()


def test_track_tick_graph_reuse(torch_cuda, ref):
    """io.reuse_graph = 1: the same io (pinned buffers) replayed from the ctx's cached CUDA graph
    follows changes of the buffers' CONTENTS (new frames, new local maps) exactly like direct
    calls -- checked against the oracle on every call."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["euroc"]
    B, Q, nf = 2, 800, 1000
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    hf = torch.zeros(B * h * w, dtype=torch.uint8).pin_memory()
    hc = torch.zeros(B * 96, dtype=torch.uint8).pin_memory()
    hp = torch.zeros(B * Q * 32, dtype=torch.uint8).pin_memory()
    hpf = torch.zeros(B * Q * 4, dtype=torch.uint8).pin_memory()
    hqd = torch.zeros(B * Q * 32, dtype=torch.uint8).pin_memory()
    o = {k: torch.zeros(n, dtype=torch.uint8).pin_memory()
         for k, n in (("kps", B * cap * 20), ("desc", B * cap * 32), ("counts", B * 9 * 4), ("matches", B * Q * 12))}
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch, io.reuse_graph = hf.data_ptr(), h * w, w, 1
    io.cams, io.n_points, io.points, io.point_frame = hc.data_ptr(), B * Q, hp.data_ptr(), hpf.data_ptr()
    io.point_desc, io.th = hqd.data_ptr(), 1.0
    for k in o:
        setattr(io, k, o[k].data_ptr())
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=B * Q)
    st = torch.cuda.Stream()  # a capturable stream (the legacy NULL stream always runs directly)
    for it in range(4):  # call 0 direct, call 1 captures, calls 2, 3 replay
        frames = synth.make_frames(w, h, B, cfg=50 + it)
        rk, rd, rc = ref.orb_extract_batch(p, frames)
        cm, pt, pf, qd, _ = synth.make_local_map(rk, rd, rc, 8, p.scale_factor, np.array(p.n_per_level[:8]), w, h,
                                                 "euroc", Q, seed=60 + it)
        for dst, a in ((hf, frames), (hc, cm), (hp, pt), (hpf, pf), (hqd, qd)):
            dst.copy_(torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1)))
        ss.ss_track_tick(pipe.ctx, B, ss.window_cfg(), io, st)
        torch.cuda.synchronize()
        counts = o["counts"].numpy().view(np.int32).reshape(B, 9)
        np.testing.assert_array_equal(counts, rc)
        desc = o["desc"].numpy().reshape(B, cap, 32)
        for f in range(B):
            np.testing.assert_array_equal(desc[f, :rc[f, -1]], rd[f, :rc[f, -1]])
        q = ref.project_points(p, cm, pt, pf, 1.0)
        want = ref.match_window(p, rk, rd, rc, None, q, qd)
        np.testing.assert_array_equal(o["matches"].numpy().view(ref.MATCH_DTYPE).reshape(-1), want)
    pipe.close()


def test_track_run_native_loop(torch_cuda, ref):
    """ss_track_run (the native tick loop): 6 ticks over 2 contexts x 3 io slots (graph reuse
    on), each slot's outputs equal the oracle's extraction of its frames."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["tum"]
    B, nf, P, NIO = 2, 1000, 2, 3
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    frames = [synth.make_frames(w, h, B, cfg=80 + i) for i in range(NIO)]
    pipes = [OrbPipeline(w, h, nf, 8, max_frames=B) for _ in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    keep, ios = [], []
    for q in range(P):
        row = []
        for i in range(NIO):
            hf = torch.from_numpy(frames[i].reshape(-1).copy()).pin_memory()
            hk = torch.zeros(B * cap * 20, dtype=torch.uint8).pin_memory()
            hc = torch.zeros(B * 9 * 4, dtype=torch.uint8).pin_memory()
            hd = torch.zeros(B * cap * 32, dtype=torch.uint8).pin_memory()
            keep.append((hf, hk, hc, hd))
            io = ss.ss_tick_io()
            io.frames, io.frame_stride, io.pitch, io.reuse_graph = hf.data_ptr(), h * w, w, 1
            io.kps, io.counts, io.desc = hk.data_ptr(), hc.data_ptr(), hd.data_ptr()
            row.append(io)
        ios.append(row)
    run = ss.TrackRun([pp.ctx for pp in pipes], streams, B, ss.brute_cfg(), ios)
    run.run(6)  # ticks t = 0..5: ctx t % 2, slot t % 3 -> every (ctx, slot) pair once
    torch.cuda.synchronize()
    for i in range(NIO):
        rk, rd, rc = ref.orb_extract_batch(p, frames[i])
        for q in range(P):
            hf, hk, hc, hd = keep[q * NIO + i]
            counts = hc.numpy().view(np.int32).reshape(B, 9)
            kps = hk.numpy().reshape(B, cap, 20)
            desc = hd.numpy().reshape(B, cap, 32)
            # every (ctx q, slot i) pair ran exactly once: t < 6 with t % 2 == q, t % 3 == i (CRT)
            _check_extract(p, kps, desc, counts, frames[i], ref)
    for pp in pipes:
        pp.close()
