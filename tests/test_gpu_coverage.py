"""GPU parity for the code paths round 1 left without a test (VERDICT r01 "weak" #2, #3,
"missing" #5):

* every match_window_kernel instance (1, 2, 4, 8 lanes per query) and the c3-sized launch
  (16 TUM frames x 50 k queries = 800 k, where the launcher picks 1 lane) vs ref.match_window;
* brute_tc at the c5 size (8 x 1266 slots x 200 k map) vs ref.match_brute on a keypoint
  sample that straddles a 256-row tile boundary;
* the distribution's in-shared-memory sort fallback (counted by ss_debug_distribution_paths)
  on an adversarial dotted frame, bit-exact;
* the blur at every one of the 512 sample points per keypoint (ss_debug_capture_samples) vs
  ref.blur of the oracle's pyramid level at the exact rotated offsets (O6, O7);
* BRUTE with an empty map (ctx with and without max_map), and a distribution switch between
  graph-replayed ticks.
"""
import os

import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    return torch


def _extract(torch, p, frames, max_queries=0, max_map=0):
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    pipe = OrbPipeline(p.width, p.height, p.n_features, p.n_levels, max_frames=len(frames), max_queries=max_queries,
                       max_map=max_map)
    pipe.extract(torch.from_numpy(np.ascontiguousarray(frames)).cuda())
    return pipe


def _assert_same_extract(pipe, rk, rd, rc):
    gk, gd, gc = pipe.results(len(rk))
    np.testing.assert_array_equal(gc, rc)
    for b in range(len(rk)):
        n = int(rc[b][-1])
        for fld in ("lx", "ly", "level", "response", "x", "y"):
            np.testing.assert_array_equal(gk[b][:n][fld], rk[b][:n][fld], err_msg=fld)
        np.testing.assert_array_equal(gd[b][:n], rd[b][:n])
    return gk, gd, gc


@pytest.mark.parametrize("lanes", [1, 2, 4, 8])
def test_window_every_lane_instance(torch_cuda, ref, lanes):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import match_out, match_records, to_device_records
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1000)
    frames = synth.make_frames(w, h, 4, cfg=61)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    q, qd, tk = synth.make_queries(rk, rd, rc, 8, np.array(p.scale[:8]), np.array(p.n_per_level[:8]), w, h, 5000,
                                   1.0, 62, ref.QUERY_DTYPE)
    pipe = _extract(torch, p, frames, max_queries=len(q))
    _assert_same_extract(pipe, rk, rd, rc)
    ss.ss_debug_match_lanes(pipe.ctx, lanes)
    out = match_out(len(q), "cuda")
    pipe.match_window(4, to_device_records(q, "cuda"), torch.from_numpy(qd).cuda(), out,
                      taken=torch.from_numpy(tk).cuda())
    got = match_records(out)
    want = ref.match_window(p, rk, rd, rc, tk, q, qd)
    np.testing.assert_array_equal(got, want)
    assert (want["idx"] >= 0).sum() > 1000
    ss.ss_debug_match_lanes(pipe.ctx, 0)
    pipe.close()


def test_window_c3_size(torch_cuda, ref):
    """c3: 16 TUM-shaped frames, 50 k map-point queries each (th = 3), the launch the bench
    times (the launcher picks 1 lane per query at 800 k queries)."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import match_out, match_records, to_device_records
    w, h = synth.SHAPES["tum"]
    p = ref.params(w, h, 1000)
    frames = synth.make_frames(w, h, 16, cfg=3)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    q, qd, tk = synth.make_queries(rk, rd, rc, 8, np.array(p.scale[:8]), np.array(p.n_per_level[:8]), w, h, 50000,
                                   3.0, 7, ref.QUERY_DTYPE)
    assert len(q) == 800000
    pipe = _extract(torch, p, frames, max_queries=len(q))
    _assert_same_extract(pipe, rk, rd, rc)
    out = match_out(len(q), "cuda")
    pipe.match_window(16, to_device_records(q, "cuda"), torch.from_numpy(qd).cuda(), out,
                      taken=torch.from_numpy(tk).cuda())
    got = match_records(out)
    want = ref.match_window(p, rk, rd, rc, tk, q, qd)
    np.testing.assert_array_equal(got, want)
    assert (want["idx"] >= 0).sum() > 5000
    pipe.close()


def test_brute_c5_size_sampled(torch_cuda, ref):
    """c5: 8 EuRoC frames x 1266 slots vs a 200 k shared map (the bench's split count);
    keypoints 250..261 of every frame (straddling row 256 of a frame's slots) are checked
    against the oracle over the whole map, and every evaluated slot against invariants."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import match_records
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1250)
    frames = synth.make_frames(w, h, 8, cfg=5)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    mp = synth.make_brute_map([rd[b][: rc[b][-1]] for b in range(8)], 200000, seed=3, n_from_kps=80000)
    pipe = _extract(torch, p, frames, max_map=len(mp))
    _assert_same_extract(pipe, rk, rd, rc)
    out = torch.zeros((8 * p.kp_capacity, 3), dtype=torch.int32, device="cuda")
    pipe.match_brute(8, torch.from_numpy(mp).cuda(), out)
    got = match_records(out).reshape(8, p.kp_capacity)
    k0, k1 = 250, 262
    want = ref.match_brute(p, rd, rc, mp, 50, 3, 4, k0=k0, k1=k1)
    for b in range(8):
        np.testing.assert_array_equal(got[b, k0:k1], want[b, k0:k1])
        n = int(rc[b][-1])
        g = got[b, :n]
        assert (g["dist"] <= g["dist2"]).all()
        ok = g["idx"] >= 0
        assert ((g["dist"][ok] <= 50) & (4 * g["dist"][ok] < 3 * g["dist2"][ok])).all()
        # an accepted match's distance is the Hamming distance to that map row
        for k in np.nonzero(ok)[0][:64]:
            assert ref.hamming(rd[b][k], mp[g["idx"][k]]) == g["dist"][k]
        rest = got[b, n:]
        assert (rest["idx"] == -1).all() and (rest["dist"] == 256).all()
    assert (got["idx"] >= 0).sum() > 1000
    pipe.close()


def test_distribution_sort_fallback(torch_cuda, ref):
    """Dotted frames: the quadtree stop rules need depths beyond the dense tables, so the
    kernel's in-shared-memory sort path runs (counter >= 1); results stay bit-exact."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1000)
    frames = np.stack([synth.make_dotted_frame(w, h, seed=s) for s in range(2)] + [synth.make_frame(w, h, 5)])
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    pipe = _extract(torch, p, frames)
    _assert_same_extract(pipe, rk, rd, rc)
    n_sort, n_global = ss.ss_debug_distribution_paths(pipe.ctx)
    assert n_sort >= 6, (n_sort, n_global)
    pipe.close()


def _pattern():
    from test_oracle_describe import _parse_inc
    return np.asarray(_parse_inc(os.path.join(ROOT, "oracle", "brief_pattern_ref.inc")), np.int64).reshape(256, 2, 2)


@pytest.mark.parametrize("shape", ["euroc", "kitti"])
def test_blur_at_every_sample_point(torch_cuda, ref, shape):
    """S6 bit-exact: the 512 blurred values each descriptor reads == ref.blur(level) at the
    O7 offsets computed here with exact integer round-half-even (ref.rhe_div_sqrt) from the
    oracle's moments; and every descriptor bit is the comparison of its two samples."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES[shape]
    nf = 1000 if shape == "euroc" else 2000
    p = ref.params(w, h, nf)
    B = 2
    frames = synth.make_frames(w, h, B, cfg=71)
    pitch = w if shape == "euroc" else w + 3  # KITTI: an unaligned pitch (describe's byte-load path)
    buf = np.zeros((B, h, pitch), np.uint8)
    buf[:, :, :w] = frames
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B)
    samples = torch.zeros(B * p.kp_capacity * 512, dtype=torch.uint8, device="cuda")
    ss.ss_debug_capture_samples(pipe.ctx, samples)
    pipe.extract(torch.from_numpy(buf).cuda())
    ss.ss_debug_capture_samples(pipe.ctx, None)
    gk, gd, gc = pipe.results(B)
    pipe.close()
    got = samples.cpu().numpy().reshape(B, p.kp_capacity, 256, 2)
    pat = _pattern()
    checked = 0
    for b in range(B):
        levels = ref.pyramid(p, frames[b])
        blurred = [ref.blur(im) for im in levels]
        rk, rd, rc = ref.orb_extract(p, frames[b])
        np.testing.assert_array_equal(gc[b], rc)
        n = int(rc[-1])
        for i in range(n):
            l, lx, ly = int(rk[i]["level"]), int(rk[i]["lx"]), int(rk[i]["ly"])
            m10, m01 = ref.moments(levels[l], lx, ly)
            r2 = m10 * m10 + m01 * m01
            want = np.empty((256, 2), np.int64)
            for bit in range(256):
                for e in range(2):
                    px, py = int(pat[bit, e, 0]), int(pat[bit, e, 1])
                    if r2:
                        ox = ref.rhe_div_sqrt(px * m10 - py * m01, r2)
                        oy = ref.rhe_div_sqrt(px * m01 + py * m10, r2)
                    else:
                        ox, oy = px, py
                    want[bit, e] = blurred[l][ly + oy, lx + ox]
            np.testing.assert_array_equal(got[b, i], want, err_msg=f"frame {b} kp {i} level {l}")
            bits = (got[b, i, :, 0] < got[b, i, :, 1]).astype(np.uint8)
            np.testing.assert_array_equal(np.packbits(bits, bitorder="little"), gd[b][i])
            checked += 1
    assert checked > 1000


@pytest.mark.parametrize("max_map", [0, 4000])
def test_brute_empty_map(torch_cuda, ref, max_map):
    """BRUTE with n_map = 0 (a session's first ticks): every slot {-1, 256, 256}, also right
    after a non-empty match on the same ctx (no stale partials), and with max_map = 0."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import match_records
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1000)
    frames = synth.make_frames(w, h, 2, cfg=17)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    pipe = _extract(torch, p, frames, max_map=max_map)
    out = torch.zeros((2 * p.kp_capacity, 3), dtype=torch.int32, device="cuda")
    if max_map:
        mp = synth.make_brute_map([rd[b][: rc[b][-1]] for b in range(2)], max_map, seed=4)
        pipe.match_brute(2, torch.from_numpy(mp).cuda(), out)
        got = match_records(out).reshape(2, p.kp_capacity)
        want = ref.match_brute(p, rd, rc, mp)
        np.testing.assert_array_equal(got, want)
        assert (got["idx"] >= 0).sum() > 100
    empty = torch.zeros((0, 32), dtype=torch.uint8, device="cuda")
    pipe.match_brute(2, empty, out)
    got = match_records(out)
    assert (got["idx"] == -1).all() and (got["dist"] == 256).all() and (got["dist2"] == 256).all()
    want = ref.match_brute(p, rd, rc, np.zeros((0, 32), np.uint8))
    np.testing.assert_array_equal(got.reshape(2, p.kp_capacity), want)
    pipe.close()


def test_distribution_switch_with_graph_reuse(torch_cuda, ref):
    """ss_set_distribution between graph-replayed ss_track_tick calls takes effect (the ctx
    drops tick graphs captured with the other distribution's kernels)."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["euroc"]
    B, nf = 2, 1000
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    frames = synth.make_frames(w, h, B, cfg=23)
    hf = torch.from_numpy(frames.reshape(-1).copy()).pin_memory()
    hk = torch.zeros(B * cap * 20, dtype=torch.uint8).pin_memory()
    hc = torch.zeros(B * 9 * 4, dtype=torch.uint8).pin_memory()
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch, io.reuse_graph = hf.data_ptr(), h * w, w, 1
    io.kps, io.counts = hk.data_ptr(), hc.data_ptr()
    cfg = ss.brute_cfg()
    pipe = OrbPipeline(w, h, nf, 8, max_frames=B)
    want = {m: ref.orb_extract_batch(p, frames, mode=m) for m in (0, 1)}
    assert not (want[0][2] == want[1][2]).all()
    for mode in (0, 0, 0, 1, 1, 1, 0, 0, 1):  # 2nd call of a key captures, 3rd replays
        pipe.set_distribution(mode)
        ss.ss_track_tick(pipe.ctx, B, cfg, io, torch.cuda.current_stream())
        torch.cuda.synchronize()
        counts = hc.numpy().view(np.int32).reshape(B, 9)
        kps = hk.numpy().reshape(B, cap, 20)
        np.testing.assert_array_equal(counts, want[mode][2], err_msg=f"mode {mode}")
        for b in range(B):
            n = int(counts[b][-1])
            gk = np.ascontiguousarray(kps[b]).reshape(-1).view(ss.KEYPOINT_DTYPE)[:n]
            np.testing.assert_array_equal(gk["lx"], want[mode][0][b][:n]["lx"])
            np.testing.assert_array_equal(gk["ly"], want[mode][0][b][:n]["ly"])
    pipe.close()


def test_brute_prepared_map(torch_cuda, ref):
    """ss_brute_map_prepare: the map expanded once, then BRUTE calls with a NULL map (direct,
    map-sharded partial and ss_track_tick) expand only their keypoints -- bit-exact with the
    oracle; a call with an explicit map forgets the preparation; a NULL map without a matching
    preparation is rejected."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import match_records
    w, h = synth.SHAPES["euroc"]
    B, nf, n_map = 3, 1250, 20000
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    frames = synth.make_frames(w, h, B, cfg=29)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    mp = synth.make_brute_map([rd[b][: rc[b][-1]] for b in range(B)], n_map, seed=31, n_from_kps=3000)
    want = ref.match_brute(p, rd, rc, mp, 50, 3, 4)
    pipe = _extract(torch, p, frames, max_map=n_map)
    d_map = torch.from_numpy(mp).cuda()
    out = torch.zeros((B * cap, 3), dtype=torch.int32, device="cuda")
    st = torch.cuda.current_stream()
    with pytest.raises(ss.SSError):  # nothing prepared yet
        ss.ss_match_projection(pipe.ctx, B, pipe.kps, pipe.desc, pipe.counts, None, 0, None, None, n_map,
                               ss.brute_cfg(), out, st)
    pipe.prepare_map(d_map)
    d_map.zero_()  # the preparation is a snapshot: later changes of the source are not seen
    pipe.match_brute(B, None, out)
    got = match_records(out).reshape(B, cap)
    for b in range(B):
        n = int(rc[b][-1])
        np.testing.assert_array_equal(got[b, :n], want[b, :n])
    # sharded partial over the prepared map == top-2 of the direct result
    top2 = torch.zeros((B, cap, 2), dtype=torch.int64, device="cuda")
    ss.ss_match_brute_partial(pipe.ctx, B, pipe.desc, pipe.counts, None, n_map, 0, top2, torch.cuda.current_stream())
    out2 = torch.zeros_like(out)
    ss.ss_match_brute_merge(pipe.ctx, B, pipe.counts, 1, top2, ss.brute_cfg(), out2, torch.cuda.current_stream())
    got2 = match_records(out2).reshape(B, cap)
    for b in range(B):
        n = int(rc[b][-1])
        np.testing.assert_array_equal(got2[b, :n], want[b, :n])
    # ss_track_tick with io.d_map_desc = NULL
    hf = torch.from_numpy(frames.reshape(-1).copy()).pin_memory()
    hm = torch.zeros(B * cap * 12, dtype=torch.uint8).pin_memory()
    io = ss.ss_tick_io()
    io.frames, io.frame_stride, io.pitch = hf.data_ptr(), h * w, w
    io.d_map_desc, io.n_map, io.matches = None, n_map, hm.data_ptr()
    ss.ss_track_tick(pipe.ctx, B, ss.brute_cfg(), io, torch.cuda.current_stream())
    torch.cuda.synchronize()
    got3 = hm.numpy().view(ref.MATCH_DTYPE).reshape(B, cap)
    for b in range(B):
        n = int(rc[b][-1])
        np.testing.assert_array_equal(got3[b, :n], want[b, :n])
    with pytest.raises(ss.SSError):
        ss.ss_match_projection(pipe.ctx, B, pipe.kps, pipe.desc, pipe.counts, None, 0, None, None, n_map - 1,
                               ss.brute_cfg(), out, torch.cuda.current_stream())  # row count differs
    # an explicit map replaces the prepared one
    d_map2 = torch.from_numpy(mp).cuda()
    pipe.match_brute(B, d_map2, out)
    with pytest.raises(ss.SSError):
        ss.ss_match_projection(pipe.ctx, B, pipe.kps, pipe.desc, pipe.counts, None, 0, None, None, n_map,
                               ss.brute_cfg(), out, st)
    pipe.close()


def test_extract_separately_allocated_frames(torch_cuda, ref):
    """ss_orb_extract_frames (SURVEY §8(b)'s d_frames[] / pitches[] boundary): independently
    allocated client frames with different pitches give the oracle's results bit for bit."""
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["tum"]
    p = ref.params(w, h, 1000)
    frames = synth.make_frames(w, h, 3, cfg=33)
    rk, rd, rc = ref.orb_extract_batch(p, frames)
    bufs = []
    for b, pitch in enumerate((w, w + 7, w + 64)):
        t = torch.zeros((h, pitch), dtype=torch.uint8, device="cuda")
        t[:, :w] = torch.from_numpy(frames[b]).cuda()
        bufs.append(t)
    pipe = OrbPipeline(w, h, 1000, 8, max_frames=3)
    ss.ss_orb_extract_frames(pipe.ctx, bufs, pipe.kps, pipe.desc, pipe.counts, torch.cuda.current_stream())
    _assert_same_extract(pipe, rk, rd, rc)
    pipe.close()
