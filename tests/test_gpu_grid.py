"""GPU parity of the grid top-N distribution (O4g, k_grid.cu) inside a full extraction vs the
oracle's extract in mode 1: keypoints, descriptors and counts bit-exact (angle <= 1e-4 rad),
on EuRoC / TUM / KITTI shapes and an adversarial noise frame (thousands of candidates)."""
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


@pytest.mark.parametrize("shape,nf", [("euroc", 1000), ("tum", 1000), ("kitti", 2000), ("noise", 1000)])
def test_grid_extract_bit_exact(torch_cuda, ref, shape, nf):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    if shape == "noise":
        w, h = 640, 480
        frames = np.random.default_rng(3).integers(0, 256, size=(2, h, w), dtype=np.uint8)
    else:
        w, h = synth.SHAPES[shape]
        frames = synth.make_frames(w, h, 3, cfg=8)
    p = ref.params(w, h, nf)
    pipe = OrbPipeline(w, h, nf, 8, max_frames=len(frames))
    pipe.set_distribution(ss.SS_DIST_GRID_TOPN)
    pipe.extract(torch.from_numpy(frames).cuda())
    gk, gd, gc = pipe.results(len(frames))
    for b in range(len(frames)):
        rk, rd, rc = ref.orb_extract(p, frames[b], mode=1)
        np.testing.assert_array_equal(gc[b], rc)
        n = int(rc[-1])
        for fld in ("lx", "ly", "level", "response", "x", "y"):
            np.testing.assert_array_equal(gk[b][:n][fld], rk[:n][fld], err_msg=fld)
        da = np.radians(np.abs(gk[b][:n]["angle_deg"].astype(np.float64) - rk[:n]["angle_deg"]))
        assert np.minimum(da, 2 * np.pi - da).max(initial=0) <= 1e-4
        np.testing.assert_array_equal(gd[b][:n], rd[:n])
    # switching back gives the quadtree result again
    pipe.set_distribution(ss.SS_DIST_QUADTREE)
    pipe.extract(torch.from_numpy(frames).cuda())
    gk, gd, gc = pipe.results(len(frames))
    rk, rd, rc = ref.orb_extract(p, frames[0])
    np.testing.assert_array_equal(gc[0], rc)
    pipe.close()
