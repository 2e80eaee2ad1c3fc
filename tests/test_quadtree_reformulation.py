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
