"""Pins of oracle O9 (windowed "search local points") and O10 (brute force).

Both are definitions (top-2 by (distance, index) + threshold/ratio rules), so the pin is
brute force written independently here with numpy bit counts; plus the integer ratio
rules equal ORB-SLAM's float forms for all distances (E12), and Hamming vs a naive count.
"""
import numpy as np
import pytest

from oracle import KEYPOINT_DTYPE, QUERY_DTYPE


def _popcount_rows(a, b):
    return np.unpackbits(np.bitwise_xor(a, b), axis=-1).sum(-1).astype(np.int64)


def test_hamming_naive(ref):
    rng = np.random.default_rng(1)
    for _ in range(300):
        a = rng.integers(0, 256, 32, dtype=np.uint8)
        b = rng.integers(0, 256, 32, dtype=np.uint8)
        assert ref.hamming(a, b) == sum(bin(int(x) ^ int(y)).count("1") for x, y in zip(a, b))
    a = rng.integers(0, 256, 32, dtype=np.uint8)
    assert ref.hamming(a, a) == 0 and ref.hamming(a, ~a) == 256


def test_ratio_rules_equal_float_forms():
    f = np.float32
    for b in range(257):
        for s in range(257):
            assert (f(b) <= f(0.8) * f(s)) == (5 * b <= 4 * s)
            assert (f(b) < f(0.75) * f(s)) == (4 * b < 3 * s)
            assert (f(b) < f(0.7) * f(s)) == (10 * b < 7 * s)


def _random_frame_set(rng, p, F, n_per_frame):
    cap, L = p.kp_capacity, p.n_levels
    kps = np.zeros((F, cap), KEYPOINT_DTYPE)
    desc = np.zeros((F, cap, 32), np.uint8)
    counts = np.zeros((F, L + 1), np.int32)
    for f in range(F):
        n = n_per_frame[f]
        lev = np.sort(rng.integers(0, L, n))
        recs = []
        for l in range(L):
            m = int((lev == l).sum())
            ly = rng.integers(19, p.level_h[l] - 19, m)
            lx = rng.integers(19, p.level_w[l] - 19, m)
            o = np.lexsort((lx, ly))
            recs += [(l, int(lx[i]), int(ly[i])) for i in o]
            counts[f, l + 1] = counts[f, l] + m
        for k, (l, lx, ly) in enumerate(recs):
            kps[f, k]["level"], kps[f, k]["lx"], kps[f, k]["ly"] = l, lx, ly
            kps[f, k]["x"] = np.float32(lx) * np.float32(p.scale[l])
            kps[f, k]["y"] = np.float32(ly) * np.float32(p.scale[l])
        base = rng.integers(0, 256, (4, 32), dtype=np.uint8)  # few prototypes -> many ties
        desc[f, :n] = base[rng.integers(0, 4, n)] ^ (rng.random((n, 32)) < 0.02).astype(np.uint8) * 1
    return kps, desc, counts


def _naive_window(p, kps, desc, counts, taken, qs, qd, th, num, den, dedup):
    L, out = p.n_levels, []
    for i, q in enumerate(qs):
        f = int(q["frame"])
        cands = []
        if 0 <= f < len(kps):
            for k in range(counts[f, L]):
                kp = kps[f, k]
                if not (q["pred_level"] - 1 <= kp["level"] <= q["pred_level"]):
                    continue
                if taken is not None and taken[f, k]:
                    continue
                dx = np.float32(kp["x"]) - np.float32(q["u"])
                dy = np.float32(kp["y"]) - np.float32(q["v"])
                if abs(dx) < q["radius"] and abs(dy) < q["radius"]:
                    cands.append((int(_popcount_rows(qd[i], desc[f, k])), k))
        cands.sort()
        d1, k1 = cands[0] if cands else (256, -1)
        d2, k2 = cands[1] if len(cands) > 1 else (256, -1)
        acc = False
        if k1 >= 0 and d1 <= th:
            l1 = kps[f, k1]["level"]
            l2 = kps[f, k2]["level"] if k2 >= 0 else -1
            acc = l1 != l2 or den * d1 <= num * d2
        out.append([k1 if acc else -1, d1, d2])
    out = np.array(out, np.int64).reshape(-1, 3)
    if dedup:
        claims = {}
        for i in range(len(qs)):
            if out[i, 0] >= 0:
                key = (int(qs[i]["frame"]), int(out[i, 0]))
                claims.setdefault(key, []).append((int(out[i, 1]), i))
        for key, lst in claims.items():
            win = min(lst)[1]
            for _, i in lst:
                if i != win:
                    out[i, 0] = -1
    return out


@pytest.mark.parametrize("seed", range(6))
def test_window_match_vs_naive(ref, seed):
    rng = np.random.default_rng(seed)
    p = ref.params(320, 240, 150, n_levels=4)
    F = 3
    kps, desc, counts = _random_frame_set(rng, p, F, [int(rng.integers(0, p.kp_capacity + 1)) for _ in range(F)])
    nq = 400
    qs = np.zeros(nq, QUERY_DTYPE)
    qs["frame"] = rng.integers(-1, F + 1, nq)  # includes invalid frames
    qs["u"] = rng.uniform(0, 320, nq)
    qs["v"] = rng.uniform(0, 240, nq)
    qs["pred_level"] = rng.integers(0, 4, nq)
    qs["radius"] = rng.choice([2.5, 4.0, 12.0, 40.0], nq).astype(np.float32)
    # exact-boundary radii: place some queries exactly r away from a keypoint
    for i in range(0, nq, 7):
        f = int(rng.integers(0, F))
        if counts[f, -1]:
            k = int(rng.integers(0, counts[f, -1]))
            qs[i]["frame"], qs[i]["u"], qs[i]["v"] = f, kps[f, k]["x"] + 4.0, kps[f, k]["y"]
            qs[i]["radius"], qs[i]["pred_level"] = 4.0, kps[f, k]["level"]
    qd = np.zeros((nq, 32), np.uint8)
    for i in range(nq):
        f = int(np.clip(qs[i]["frame"], 0, F - 1))
        n = counts[f, -1]
        qd[i] = desc[f, int(rng.integers(0, n))] if n and rng.random() < 0.7 else rng.integers(0, 256, 32)
    taken = (rng.random((F, p.kp_capacity)) < 0.1).astype(np.uint8)
    for dedup in (0, 1):
        for tk in (None, taken):
            got = ref.match_window(p, kps, desc, counts, tk, qs, qd, 100, 4, 5, dedup)
            want = _naive_window(p, kps, desc, counts, tk, qs, qd, 100, 4, 5, dedup)
            np.testing.assert_array_equal(np.stack([got["idx"], got["dist"], got["dist2"]], 1), want)


@pytest.mark.parametrize("seed", range(4))
def test_brute_match_vs_naive(ref, seed):
    rng = np.random.default_rng(50 + seed)
    p = ref.params(320, 240, 120, n_levels=4)
    F = 2
    kps, desc, counts = _random_frame_set(rng, p, F, [p.kp_capacity - 3, 17])
    n_map = int(rng.integers(1, 700))
    mp = rng.integers(0, 256, (n_map, 32), dtype=np.uint8)
    # plant near-duplicates so that some matches pass th=50 and equal-distance ties occur
    for f in range(F):
        for k in range(0, counts[f, -1], 3):
            mp[rng.integers(0, n_map)] = desc[f, k] ^ (rng.random(32) < 0.03).astype(np.uint8)
    got = ref.match_brute(p, desc, counts, mp, 50, 3, 4)
    for f in range(F):
        for k in range(p.kp_capacity):
            g = got[f, k]
            if k >= counts[f, -1]:
                assert (g["idx"], g["dist"], g["dist2"]) == (-1, 256, 256)
                continue
            d = _popcount_rows(desc[f, k][None], mp)
            order = np.lexsort((np.arange(n_map), d))
            d1, m1 = int(d[order[0]]), int(order[0])
            d2 = int(d[order[1]]) if n_map > 1 else 256
            acc = d1 <= 50 and 4 * d1 < 3 * d2
            assert (g["idx"], g["dist"], g["dist2"]) == (m1 if acc else -1, d1, d2)
