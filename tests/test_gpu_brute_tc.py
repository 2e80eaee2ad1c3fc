"""GPU parity of the brute-force matcher (S10, DESIGN.md §3 O10) on the tensor-core path
(k_brute_tc.cu): the C ABI vs the oracle's plain top-2 scan, bit-exact, on synthetic
descriptors chosen to exercise the tiling (partial 256-keypoint blocks, partial 128-row map
tiles, several map splits) and the tie rules (duplicate map rows: equal distances resolve to
the lowest map index; exact copies d = 0; complements d = 256)."""
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


def _case(rng, F, cap, counts, n_map, n_dup):
    desc = rng.integers(0, 256, size=(F, cap, 32), dtype=np.uint8)
    mp = rng.integers(0, 256, size=(n_map, 32), dtype=np.uint8)
    flat = desc.reshape(-1, 32)
    if n_map >= 8:
        # near copies of keypoints (accepted matches), exact copies, complements, duplicates
        k = min(n_map // 4, len(flat))
        src = rng.choice(len(flat), size=k, replace=False)
        dst = rng.choice(n_map, size=k, replace=False)
        flips = (rng.random((k, 256)) < 0.05)
        mp[dst] = flat[src] ^ np.packbits(flips, axis=1, bitorder="little")
        mp[dst[: k // 8]] = flat[src[: k // 8]]
        mp[dst[k // 8: k // 4]] = ~flat[src[k // 8: k // 4]]
    if n_dup:
        a = rng.choice(n_map, size=n_dup)
        b = rng.choice(n_map, size=n_dup)
        mp[b] = mp[a]
    return desc, mp


@pytest.mark.parametrize("F,counts,n_map,n_dup", [
    (1, [1266], 1, 0),
    (1, [5], 127, 10),
    (2, [1266, 700], 128, 20),
    (3, [1266, 0, 1000], 129, 30),
    (3, [1266, 1266, 1266], 4097, 400),
    (2, [1266, 1], 50000, 3000),
])
def test_brute_tc_bit_exact(torch_cuda, ref, F, counts, n_map, n_dup):
    torch = torch_cuda
    from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_records
    w, h, nf = 752, 480, 1250
    p = ref.params(w, h, nf)
    cap = p.kp_capacity
    rng = np.random.default_rng(1000 + n_map)
    desc, mp = _case(rng, F, cap, counts, n_map, n_dup)
    cnt = np.zeros((F, p.n_levels + 1), np.int32)
    cnt[:, -1] = counts
    pipe = OrbPipeline(w, h, nf, 8, max_frames=F, max_map=n_map)
    pipe.desc[:F].copy_(torch.from_numpy(desc))
    pipe.counts[:F].copy_(torch.from_numpy(cnt))
    out = torch.zeros((F * cap, 3), dtype=torch.int32, device="cuda")
    pipe.match_brute(F, torch.from_numpy(mp).cuda(), out)
    got = match_records(out).reshape(F, cap)
    want = ref.match_brute(p, desc, cnt, mp, 50, 3, 4)
    for f in range(F):
        n = counts[f]
        np.testing.assert_array_equal(got[f, :n], want[f, :n], err_msg=f"frame {f}")
    pipe.close()
