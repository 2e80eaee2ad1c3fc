"""GPU parity of the map-sharded brute force (ss_match_brute_partial +
ss_match_brute_merge): shards of uneven size (incl. an empty one and one smaller than a
128-row tile) merged in any order == the oracle's O10 over the whole map == the unsharded
ss_match_projection BRUTE, bit-exact; each shard's top-2 == its brute-force definition."""
import numpy as np
import pytest

from test_gpu_brute_tc import _case
from test_multirank_cpu import _np_shard_top2

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_conext_dhakalrwcr22_b200 import build as b
    b.build()
    return torch


@pytest.mark.parametrize("F,counts,n_map,cuts", [
    (2, [1266, 700], 3000, [0, 1000, 1000, 1057, 3000]),
    (3, [1266, 0, 1266], 20000, [0, 7000, 20000]),
    (1, [300], 129, [0, 129]),
])
def test_brute_shard_bit_exact(torch_cuda, ref, F, counts, n_map, cuts):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200 import ss
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_records
    w, h, nf = 752, 480, 1250
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    rng = np.random.default_rng(2000 + n_map)
    desc, mp = _case(rng, F, cap, counts, n_map, n_map // 10)
    cnt = np.zeros((F, p.n_levels + 1), np.int32)
    cnt[:, -1] = counts
    pipe = OrbPipeline(w, h, nf, 8, max_frames=F, max_map=n_map)
    pipe.desc[:F].copy_(torch.from_numpy(desc))
    pipe.counts[:F].copy_(torch.from_numpy(cnt))
    d_map = torch.from_numpy(mp).cuda()
    R = len(cuts) - 1
    parts = torch.zeros((R, F, cap, 2), dtype=torch.int64, device="cuda")
    for r in range(R):
        lo, hi = cuts[r], cuts[r + 1]
        ss.ss_match_brute_partial(pipe.ctx, F, pipe.desc, pipe.counts, d_map[lo:hi] if hi > lo else d_map, hi - lo, lo,
                                  parts[r], torch.cuda.current_stream())
    out = torch.zeros((F * cap, 3), dtype=torch.int32, device="cuda")
    perm = torch.from_numpy(np.random.default_rng(1).permutation(R)).cuda()
    ss.ss_match_brute_merge(pipe.ctx, F, pipe.counts, R, parts[perm].contiguous(), ss.brute_cfg(), out,
                            torch.cuda.current_stream())
    ref_out = torch.zeros_like(out)
    pipe.match_brute(F, d_map, ref_out)
    torch.cuda.synchronize()
    got = match_records(out).reshape(F, cap)
    np.testing.assert_array_equal(got, match_records(ref_out).reshape(F, cap))
    want = ref.match_brute(p, desc, cnt, mp, 50, 3, 4)
    for f in range(F):
        np.testing.assert_array_equal(got[f, :counts[f]], want[f, :counts[f]], err_msg=f"frame {f}")
    # every shard's top-2 against its definition, on a sample of keypoints
    pt = parts.cpu().numpy().view(np.uint64)
    sub = np.zeros((F, 40, 32), np.uint8)
    sub[:, :] = desc[:, :40]
    sc = np.zeros((F, 2), np.int32)
    sc[:, 1] = np.minimum(counts, 40)
    for r in range(R):
        want_t = _np_shard_top2(sub, sc, mp[cuts[r]:cuts[r + 1]], cuts[r])
        np.testing.assert_array_equal(pt[r, :, :40], want_t)
    pipe.close()
