"""CPU check of the GPU distribution algorithm's *reformulation* (k_distribute.cu) against
the oracle's literal DistributeOctTree transcription (S8c O4).

The kernel never builds the node list: it sorts per-key quadtree path codes once, derives
every depth's node count S_r and multi-key count E_r from two histograms of neighbour
separation rounds, replays ORB-SLAM's phase-1/phase-2 stop rules on those counts, and
only orders nodes for the final partial phase-2 round.  This file is a line-by-line
Python model of that kernel (not of the oracle) and asserts it keeps exactly the keys the
oracle keeps on synthetic frames and on random / clustered / degenerate key sets."""
import numpy as np
import pytest

import synth

ROUNDS = 13


def f32(x):
    return np.float32(x)


def gpu_model(kx, ky, sc, width, height, N):
    n = len(kx)
    if n == 0:
        return []
    nini = int(np.floor(abs(f32(f32(width) / f32(height))) + 0.5))
    hX = f32(f32(width) / f32(nini))

    def root(ri):
        return int(f32(hX * f32(ri))), int(f32(hX * f32(ri + 1)))

    keys = []
    for i in range(n):
        ri = min(int(f32(f32(kx[i]) / hX)), nini - 1)
        ulx, urx = root(ri)
        uly, bly, path = 0, height, 0
        for _ in range(ROUNDS):
            hx, hy = (urx - ulx + 1) >> 1, (bly - uly + 1) >> 1
            right, down = int(kx[i] >= ulx + hx), int(ky[i] >= uly + hy)
            path = (path << 2) | (down * 2 + right)
            ulx, urx = (ulx + hx, urx) if right else (ulx, ulx + hx)
            uly, bly = (uly + hy, bly) if down else (uly, uly + hy)
        keys.append((ri << 26) | path)
    order = sorted(range(n), key=lambda i: (keys[i], i))  # stable radix sort by key
    K = [keys[i] for i in order]
    R = order

    def sep(a, b):
        x = a ^ b
        if x >> 26:
            return 0
        if x == 0:
            return 14
        return ((32 - x.bit_length() - 6) >> 1) + 1

    dd = [0] + [sep(K[i - 1], K[i]) for i in range(1, n)]
    H, G = [0] * 16, [0] * 17
    for i in range(n):
        lo = dd[i] if i else -1
        hi = dd[i + 1] if i + 1 < n else -1
        if i:
            H[lo] += 1
        G[max(lo, hi) + 1] += 1
    S, E = [0] * 15, [0] * 15
    s, single = 1, G[0]
    for r in range(14):
        s += H[r]
        single += G[r + 1]
        S[r], E[r] = s, s - single
    S[14], E[14] = S[13], E[13]
    D, partial, r = 1, False, 0
    while True:
        nx = S[min(r + 1, 14)]
        if nx >= N or nx == S[r]:
            D = r + 1
            break
        if nx + 3 * E[min(r + 1, 14)] > N:
            d = r + 1
            while True:
                s2 = S[min(d + 1, 14)]
                if s2 >= N:
                    D, partial = d, True
                    break
                if s2 == S[min(d, 14)]:
                    D = d + 1
                    break
                d += 1
            break
        r += 1
    D = min(D, 14)
    dlim = min(D, 13)
    split = set()
    if partial:
        recs = []
        for i in range(n):
            if i != 0 and dd[i] > D:
                continue
            size, c, mr, j = 1, 1, R[i], i + 1
            while j < n and dd[j] > D:
                size, mr, c, j = size + 1, min(mr, R[j]), c + (dd[j] == D + 1), j + 1
            if size > 1:
                ri = K[i] >> 26
                ulx, urx = root(ri)
                uly, bly = 0, height
                for rr in range(1, D + 1):
                    q = (K[i] >> (26 - 2 * rr)) & 3
                    hx, hy = (urx - ulx + 1) >> 1, (bly - uly + 1) >> 1
                    ulx, urx = (ulx + hx, urx) if q & 1 else (ulx, ulx + hx)
                    uly, bly = (uly + hy, bly) if q & 2 else (uly, uly + hy)
                recs.append(((0x1FFFFF - size) << 43 | uly << 32 | ulx << 20 | mr, i, c))
        recs.sort()
        acc = S[D]
        for _, h, c in recs:
            if acc >= N:
                break
            acc += c - 1
            split.add(h)
    kept = []
    for i in range(n):
        if i != 0 and dd[i] > dlim:
            continue
        sp = partial and i in split
        best_m, best_r, j = -1, 0, i
        while j < n and (j == i or dd[j] > dlim):
            if j != i and sp and dd[j] == D + 1:
                kept.append(best_r)
                best_m = -1
            rr_ = R[j]
            if sc[rr_] > best_m or (sc[rr_] == best_m and rr_ < best_r):
                best_m, best_r = sc[rr_], rr_
            j += 1
        kept.append(best_r)
    return sorted(kept)


@pytest.mark.parametrize("w,h,L,nf", [(200, 160, 3, 150), (752, 480, 8, 1000), (1241, 376, 8, 2000),
                                      (640, 480, 8, 1000)])
def test_reformulation_on_frames(ref, w, h, L, nf):
    p = ref.params(w, h, nf, n_levels=L)
    for seed in range(2):
        img = synth.make_frame(w, h, synth.frame_seed(13, seed, 0))
        levs = ref.pyramid(p, img)
        for l in range(L):
            lx, ly, sc = ref.cell_candidates(p, l, ref.fast_M(levs[l]))
            args = (lx - 16, ly - 16, sc, p.level_w[l] - 32, p.level_h[l] - 32, p.n_per_level[l])
            assert gpu_model(*[a.tolist() if hasattr(a, "tolist") else a for a in args]) == \
                ref.distribute(*args).tolist(), (w, h, seed, l)


@pytest.mark.parametrize("seed", range(30))
def test_reformulation_random(ref, seed):
    from test_oracle_quadtree import _random_keys
    rng = np.random.default_rng(500 + seed)
    width = int(rng.choice([720, 608, 1209, 178, 147, 314, 300, 97, 1000]))
    height = int(rng.choice([448, 368, 344, 102, 73, 61, 200]))
    if round(width / height) < 1:
        width = height
    kx, ky, sc = _random_keys(rng, width, height, int(rng.integers(0, 1500)), clustered=bool(seed % 2))
    for N in (0, 1, 5, 60, 217, 434, max(1, len(kx) // 2), 3 * len(kx) + 1):
        want = ref.distribute(kx, ky, sc, width, height, N).tolist()
        assert gpu_model(kx.tolist(), ky.tolist(), sc.tolist(), width, height, N) == want, (seed, N)


def dense_model(kx, ky, sc, width, height, N, bins=4096):
    """Model of the kernel's dense fast path: per-depth prefix histograms instead of a sort.
    Returns None when the stop rules need a depth beyond R (the kernel then falls back)."""
    n = len(kx)
    if n == 0:
        return []
    nini = int(np.floor(abs(f32(f32(width) / f32(height))) + 0.5))
    R = 0
    while R < 6 and nini << (2 * (R + 1)) <= bins:
        R += 1
    hX = f32(f32(width) / f32(nini))
    keys = []
    for i in range(n):
        ri = min(int(f32(f32(kx[i]) / hX)), nini - 1)
        ulx, urx = int(f32(hX * f32(ri))), int(f32(hX * f32(ri + 1)))
        uly, bly, path = 0, height, 0
        for _ in range(ROUNDS):
            hx, hy = (urx - ulx + 1) >> 1, (bly - uly + 1) >> 1
            right, down = int(kx[i] >= ulx + hx), int(ky[i] >= uly + hy)
            path = (path << 2) | (down * 2 + right)
            ulx, urx = (ulx + hx, urx) if right else (ulx, ulx + hx)
            uly, bly = (uly + hy, bly) if down else (uly, uly + hy)
        keys.append((ri << 26) | path)
    cnt = [dict() for _ in range(R + 1)]
    for k in keys:
        for r in range(R + 1):
            b = k >> (26 - 2 * r)
            cnt[r][b] = cnt[r].get(b, 0) + 1
    S = [len(c) for c in cnt]
    E = [sum(v > 1 for v in c.values()) for c in cnt]
    D, partial, r = None, False, 0
    while True:
        if r + 1 > R:
            return None
        nx = S[r + 1]
        if nx >= N or nx == S[r]:
            D = r + 1
            break
        if nx + 3 * E[r + 1] > N:
            d = r + 1
            while True:
                if d + 1 > R:
                    return None
                if S[d + 1] >= N:
                    partial = True
                    break
                if S[d + 1] == S[d]:
                    d += 1
                    break
                d += 1
            D = d
            break
        r += 1
    split = set()
    if partial:
        first = {}
        for i, k in enumerate(keys):
            b = k >> (26 - 2 * D)
            first[b] = min(first.get(b, n), i)
        recs = []
        for b, c in cnt[D].items():
            if c > 1:
                ch = sum(((b << 2) | q) in cnt[D + 1] for q in range(4))
                kk = b << (26 - 2 * D)
                ri = kk >> 26
                ulx, urx = int(f32(hX * f32(ri))), int(f32(hX * f32(ri + 1)))
                uly, bly = 0, height
                for rr in range(1, D + 1):
                    q = (kk >> (26 - 2 * rr)) & 3
                    hx, hy = (urx - ulx + 1) >> 1, (bly - uly + 1) >> 1
                    ulx, urx = (ulx + hx, urx) if q & 1 else (ulx, ulx + hx)
                    uly, bly = (uly + hy, bly) if q & 2 else (uly, uly + hy)
                recs.append(((0x1FFFFF - c) << 43 | uly << 32 | ulx << 20 | first[b], b, ch))
        recs.sort()
        acc = S[D]
        for _, b, ch in recs:
            if acc >= N:
                break
            acc += ch - 1
            split.add(b)
    best = {}
    for i, k in enumerate(keys):
        b = k >> (26 - 2 * D)
        node = (1, k >> (26 - 2 * (D + 1))) if b in split else (0, b)
        v = (sc[i] << 20) | (0xFFFFF - i)
        best[node] = max(best.get(node, 0), v)
    return sorted(0xFFFFF - (v & 0xFFFFF) for v in best.values())


@pytest.mark.parametrize("seed", range(30))
def test_dense_fast_path_equals_oracle_or_falls_back(ref, seed):
    from test_oracle_quadtree import _random_keys
    rng = np.random.default_rng(900 + seed)
    width = int(rng.choice([720, 608, 1209, 178, 147, 314, 300, 97, 1000]))
    height = int(rng.choice([448, 368, 344, 102, 73, 61, 200]))
    if round(width / height) < 1:
        width = height
    kx, ky, sc = _random_keys(rng, width, height, int(rng.integers(1, 3000)), clustered=bool(seed % 2))
    fell_back = 0
    for N in (0, 1, 5, 60, 217, 434, max(1, len(kx) // 2), 3 * len(kx) + 1):
        got = dense_model(kx.tolist(), ky.tolist(), sc.tolist(), width, height, N)
        if got is None:
            fell_back += 1
            continue
        assert got == ref.distribute(kx, ky, sc, width, height, N).tolist(), (seed, N)
    assert fell_back < 8


def test_dense_fast_path_taken_on_frames(ref):
    p = ref.params(752, 480, 1000)
    img = synth.make_frame(752, 480, synth.frame_seed(13, 0, 0))
    levs = ref.pyramid(p, img)
    for l in range(8):
        lx, ly, sc = ref.cell_candidates(p, l, ref.fast_M(levs[l]))
        args = (lx - 16, ly - 16, sc, p.level_w[l] - 32, p.level_h[l] - 32, p.n_per_level[l])
        got = dense_model(*[a.tolist() if hasattr(a, "tolist") else a for a in args])
        assert got is not None, l  # synthetic frames never need the sort fallback
        assert got == ref.distribute(*args).tolist()


def test_dotted_frame_needs_sort_fallback(ref):
    """The adversarial frame the GPU test uses to drive distribute_kernel into its sort path
    (tests/test_gpu_coverage.py): its level candidates need quadtree depths beyond the dense
    tables on several levels, and the sort-path model still equals the oracle there."""
    p = ref.params(752, 480, 1000)
    img = synth.make_dotted_frame(752, 480, seed=0)
    levs = ref.pyramid(p, img)
    fell = 0
    for l in range(8):
        lx, ly, sc = ref.cell_candidates(p, l, ref.fast_M(levs[l]))
        args = (lx - 16, ly - 16, sc, p.level_w[l] - 32, p.level_h[l] - 32, p.n_per_level[l])
        lists = [a.tolist() if hasattr(a, "tolist") else a for a in args]
        want = ref.distribute(*args).tolist()
        if dense_model(*lists) is None:
            fell += 1
        assert gpu_model(*lists) == want, l
    assert fell >= 3
