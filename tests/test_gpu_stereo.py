"""GPU parity of O12 stereo matching (k_stereo.cu, ss_stereo_match) vs the oracle: u_right and
depth bit-exact for every left keypoint, on KITTI-shaped warped pairs and on integer-shift
pairs, after a GPU extraction of the interleaved (left, right) frames."""
import numpy as np
import pytest

import synth

pytestmark = pytest.mark.gpu

FX, BASE = 718.856, 0.537
BF = float(np.float32(FX * BASE))


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    return torch


def _pairs(kind, w, h, n):
    out = []
    for i in range(n):
        if kind == "warp":
            out += list(synth.make_stereo_pair(w, h, seed=40 + i))
        else:
            d = 5 + 9 * i
            big = synth.make_frame(w + d, h, 70 + i)
            out += [np.ascontiguousarray(big[:, :w]), np.ascontiguousarray(big[:, d:])]
    return np.stack(out)


@pytest.mark.parametrize("kind,w,h,nf,n", [("warp", 1241, 376, 2000, 3), ("shift", 752, 480, 1000, 2)])
def test_stereo_bit_exact(torch_cuda, ref, kind, w, h, nf, n):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    frames = _pairs(kind, w, h, n)
    p = ref.params(w, h, nf)
    pipe = OrbPipeline(w, h, nf, 8, max_frames=2 * n)
    d_frames = torch.from_numpy(frames).cuda()
    pipe.extract(d_frames)
    ur = torch.zeros((n, p.kp_capacity), dtype=torch.float32, device="cuda")
    dp = torch.zeros_like(ur)
    pipe.stereo(d_frames, BF, BASE, ur, dp)
    gk, gd, gc = pipe.results(2 * n)
    ur_g, dp_g = ur.cpu().numpy(), dp.cpu().numpy()
    total = 0
    for i in range(n):
        kl, dl, cl = ref.orb_extract(p, frames[2 * i])
        kr, dr, cr = ref.orb_extract(p, frames[2 * i + 1])
        assert (gc[2 * i] == cl).all() and (gc[2 * i + 1] == cr).all()
        u_w, d_w, _ = ref.stereo_match(p, frames[2 * i], frames[2 * i + 1], kl, dl, cl, kr, dr, cr, BF, BASE)
        m = int(cl[-1])
        np.testing.assert_array_equal(ur_g[i, :m].view(np.uint32), u_w[:m].view(np.uint32), err_msg=f"uright {i}")
        np.testing.assert_array_equal(dp_g[i, :m].view(np.uint32), d_w[:m].view(np.uint32), err_msg=f"depth {i}")
        total += int((u_w[:m] >= 0).sum())
    assert total > 200
    pipe.close()
