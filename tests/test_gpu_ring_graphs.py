"""The configuration bench.py times, checked against the oracle: each tick captured as a CUDA
graph (extract -> O13 frame-to-frame matching -> search local points, with the local-map
projection on a forked branch beside O13, programmatic dependent launches throughout), one
graph per (context, input slot), several contexts replaying their graphs concurrently on
their own streams (ticks in flight).  Every tick's keypoints, descriptors, O13 matches and
window matches are compared with the oracle chain (bit-exact; angle <= 1e-4 rad)."""
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


def test_ring_graphs_in_flight(torch_cuda, ref):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    w, h = synth.SHAPES["euroc"]
    B, nf, Qf, NLf = 4, 1000, 1200, 600  # c2's batch and features; fewer map points per frame
    P, S = 3, 2                          # contexts (ticks in flight), input slots per context
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    dev = torch.device("cuda")
    u8 = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.uint8).reshape(-1).copy()).to(dev)

    # per slot: frames, local map, last-frame points; the oracle's extraction
    slots = []
    for s in range(S):
        frames = synth.make_frames(w, h, B, cfg=70 + s)
        rk, rd, rc = ref.orb_extract_batch(p, frames)
        cm, pt, pf, qd, tk = synth.make_local_map(rk, rd, rc, 8, p.scale_factor, np.array(p.n_per_level[:8]), w, h,
                                                  "euroc", Qf, seed=80 + s)
        _, last, off, lp, ld = synth.make_last_frame(rk, rd, rc, 8, np.array(p.n_per_level[:8]), w, h, "euroc", NLf,
                                                     seed=90 + s, cams=cm)
        slots.append(dict(frames=frames, rk=rk, rd=rd, rc=rc, cm=cm, pt=pt, pf=pf, qd=qd, tk=tk, off=off, lp=lp, ld=ld,
                          d_frames=torch.from_numpy(frames).to(dev), d_cams=u8(cm).view(B, -1),
                          d_pts=u8(pt).view(len(pt), -1), d_pf=torch.from_numpy(pf.astype(np.int32)).to(dev),
                          d_qd=u8(qd).view(len(qd), 32), d_tk=torch.from_numpy(tk).to(dev),
                          d_off=torch.from_numpy(off.astype(np.int32)).to(dev), d_lp=u8(lp).view(len(lp), -1),
                          d_ld=u8(ld).view(len(ld), 32)))
    Q, NLF = len(slots[0]["pt"]), int(slots[0]["off"][-1])
    assert all(len(sl["pt"]) == Q and int(sl["off"][-1]) == NLF for sl in slots)

    pipes = [OrbPipeline(w, h, nf, 8, max_frames=B, max_queries=max(Q, NLF)) for _ in range(P)]
    streams = [torch.cuda.Stream(dev) for _ in range(P)]
    aux = [torch.cuda.Stream(dev) for _ in range(P)]
    outs = [torch.zeros((Q, 3), dtype=torch.int32, device=dev) for _ in range(P)]
    qbufs = [torch.zeros((Q, 20), dtype=torch.uint8, device=dev) for _ in range(P)]
    lf_out = [torch.zeros((NLF, 3), dtype=torch.int32, device=dev) for _ in range(P)]
    lf_n = [torch.zeros(B, dtype=torch.int32, device=dev) for _ in range(P)]
    lf_mask = [torch.zeros((B, cap), dtype=torch.uint8, device=dev) for _ in range(P)]

    def tick(q, sl, capture_stream):
        pp, st = pipes[q], capture_stream
        pp.extract(sl["d_frames"], stream=st)
        ev0, ev1 = torch.cuda.Event(), torch.cuda.Event()
        ev0.record(st)
        aux[q].wait_event(ev0)  # the projection beside O13 (bench.py --fork-project 2)
        pp.project(B, sl["d_cams"], sl["d_pts"], sl["d_pf"], qbufs[q], th=1.0, stream=aux[q])
        ev1.record(aux[q])
        pp.match_last_frame(B, sl["d_cams"], sl["d_off"], sl["d_lp"], sl["d_ld"], lf_out[q], lf_n[q], th=15.0,
                            min_matches=20, taken=sl["d_tk"], matched=lf_mask[q], stream=st)
        st.wait_event(ev1)
        pp.match_window(B, qbufs[q], sl["d_qd"], outs[q], taken=lf_mask[q], stream=st)

    for q in range(P):  # first calls outside capture (kernel attributes), as bench.py does
        tick(q, slots[0], streams[q])
    torch.cuda.synchronize()
    graphs = []
    for q in range(P):
        row = []
        for s in range(S):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=streams[q]):
                tick(q, slots[s], streams[q])
            row.append(g)
        graphs.append(row)
    torch.cuda.synchronize()

    for rnd in range(2 * S):
        s = rnd % S
        for q in range(P):  # P ticks in flight, each context on its own stream
            with torch.cuda.stream(streams[q]):
                graphs[q][s].replay()
        torch.cuda.synchronize()
        sl = slots[s]
        for q in range(P):
            gk, gd, gc = pipes[q].results(B)
            np.testing.assert_array_equal(gc, sl["rc"], err_msg=f"counts ctx {q} slot {s}")
            for f in range(B):
                n = int(sl["rc"][f][-1])
                for fld in ("lx", "ly", "level", "response", "x", "y"):
                    np.testing.assert_array_equal(gk[f][:n][fld], sl["rk"][f][:n][fld], err_msg=f"{fld} ctx {q} slot {s}")
                da = np.radians(np.abs(gk[f][:n]["angle_deg"].astype(np.float64) - sl["rk"][f][:n]["angle_deg"]))
                assert np.minimum(da, 2 * np.pi - da).max(initial=0) <= 1e-4
                np.testing.assert_array_equal(gd[f][:n], sl["rd"][f][:n], err_msg=f"desc ctx {q} slot {s}")
            # O13 on the GPU keypoints (its rotation bins are decided on the GPU angles), then
            # taken | kept -> O11 -> O9, as the tick does
            gk_ref = np.ascontiguousarray(gk).view(ref.KEYPOINT_DTYPE).reshape(B, cap)
            want_lf, want_n = ref.match_last_frame(p, sl["cm"], None, 0.0, gk_ref, sl["rd"], sl["rc"], sl["tk"], sl["off"],
                                                   sl["lp"], sl["ld"], th=15.0, min_matches=20)
            got_lf = lf_out[q].cpu().numpy().view(ref.MATCH_DTYPE).reshape(-1)
            np.testing.assert_array_equal(got_lf, want_lf, err_msg=f"O13 ctx {q} slot {s}")
            np.testing.assert_array_equal(lf_n[q].cpu().numpy(), want_n)
            mask = (sl["tk"] != 0).astype(np.uint8)
            for f in range(B):
                seg = want_lf[sl["off"][f]:sl["off"][f + 1]]
                mask[f, seg["idx"][seg["idx"] >= 0]] = 1
            qq = ref.project_points(p, sl["cm"], sl["pt"], sl["pf"], 1.0)
            want = ref.match_window(p, sl["rk"], sl["rd"], sl["rc"], mask, qq, sl["qd"])
            got = outs[q].cpu().numpy().view(ref.MATCH_DTYPE).reshape(-1)
            np.testing.assert_array_equal(got, want, err_msg=f"window ctx {q} slot {s}")
            assert (got["idx"] >= 0).sum() > 100
    for pp in pipes:
        pp.close()
