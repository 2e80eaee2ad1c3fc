"""GPU parity of the O11 local-map projection (k_project.cu) vs the oracle: every field of
every query bit-exact, on random poses with points spread over the culling boundaries
(behind the camera, outside the image, at the distance gates, grazing viewing angles)."""
import math

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    return torch


def _rot(rng):
    q = rng.normal(size=4)
    q /= np.linalg.norm(q)
    w, x, y, z = q
    return np.array([[1 - 2 * (y * y + z * z), 2 * (x * y - z * w), 2 * (x * z + y * w)],
                     [2 * (x * y + z * w), 1 - 2 * (x * x + z * z), 2 * (y * z - x * w)],
                     [2 * (x * z - y * w), 2 * (y * z + x * w), 1 - 2 * (x * x + y * y)]])


def make_case(ss, F, n, seed, W=752, H=480):
    rng = np.random.default_rng(seed)
    cams = np.zeros(F, ss.CAMERA_DTYPE)
    pts = np.zeros(n, ss.MAP_POINT_DTYPE)
    pf = rng.integers(-1, F + 1, n).astype(np.int32)  # includes out-of-batch frame indices
    for f in range(F):
        R, t = _rot(rng), rng.normal(0, 3, 3)
        cams[f]["R"] = R.astype(np.float32).ravel()
        cams[f]["t"] = t.astype(np.float32)
        cams[f]["ow"] = (-R.T @ t).astype(np.float32)
        cams[f]["fx"], cams[f]["fy"] = 458.654, 457.296
        cams[f]["cx"], cams[f]["cy"] = 367.215, 248.375
        cams[f]["min_x"], cams[f]["max_x"], cams[f]["min_y"], cams[f]["max_y"] = 0, W, 0, H
    for i in range(n):
        f = min(max(pf[i], 0), F - 1)
        c = cams[f]
        R = c["R"].reshape(3, 3).astype(np.float64)
        t = c["t"].astype(np.float64)
        uv = rng.uniform([-60, -60], [W + 60, H + 60])
        z = rng.uniform(-2.0, 40.0)
        pc = np.array([(uv[0] - c["cx"]) / c["fx"] * z, (uv[1] - c["cy"]) / c["fy"] * z, z])
        pw = R.T @ (pc - t)
        d = pw - c["ow"].astype(np.float64)
        dist = np.linalg.norm(d)
        ang = rng.uniform(0, 75) if rng.random() < 0.8 else rng.uniform(0, 4)
        axis = np.cross(d, rng.normal(size=3))
        axis /= np.linalg.norm(axis)
        dn = d / dist
        nrm = dn * math.cos(math.radians(ang)) + np.cross(axis, dn) * math.sin(math.radians(ang))
        pts[i]["pos"] = pw.astype(np.float32)
        pts[i]["normal"] = nrm.astype(np.float32)
        pts[i]["max_dist"] = dist * math.exp(rng.uniform(-0.3, 2.2))
        pts[i]["min_dist"] = pts[i]["max_dist"] / 1.2 ** 7 * rng.uniform(0.2, 3.0)
    return cams, pts, pf


@pytest.mark.parametrize("F,n,th", [(1, 1, 1.0), (4, 5000, 1.0), (16, 20011, 3.0)])
def test_project_bit_exact(torch_cuda, ref, F, n, th):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
    p = ref.params(752, 480)
    cams, pts, pf = make_case(ss, F, n, seed=F * 1000 + n)
    want = ref.project_points(p, cams, pts, pf, th)
    pipe = OrbPipeline(752, 480, 1000, 8, max_frames=max(F, 1))
    d_cams = torch.from_numpy(cams.view(np.uint8).reshape(F, -1).copy()).cuda()
    d_pts = torch.from_numpy(pts.view(np.uint8).reshape(n, -1).copy()).cuda()
    d_pf = torch.from_numpy(pf).cuda()
    out = torch.zeros((n, 20), dtype=torch.uint8, device="cuda")
    pipe.project(F, d_cams, d_pts, d_pf, out, th=th)
    got = out.cpu().numpy().view(ss.QUERY_DTYPE).reshape(-1)
    vis = want["pred_level"] >= 0
    if n > 100:
        assert 0.1 < vis.mean() < 0.9, vis.mean()
    for fld in ("frame", "pred_level"):
        np.testing.assert_array_equal(got[fld], want[fld], err_msg=fld)
    for fld in ("u", "v", "radius"):  # bit patterns, not values
        np.testing.assert_array_equal(got[fld].view(np.uint32), want[fld].view(np.uint32), err_msg=fld)
    pipe.close()
