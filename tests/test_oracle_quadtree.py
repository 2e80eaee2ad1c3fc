"""Pins of oracle O4 (quadtree keypoint distribution, ORB-SLAM DistributeOctTree reading).

No library or paper value exists for this step (the paper never describes it and
ORB-SLAM's own tie-break is heap-address order), so O4 is "parity unpinned" against
ORB-SLAM itself.  What pins the oracle here:
  * hand-worked cases (tests/golden/quadtree_cases.json), re-derived
    by hand below;
  * invariants (count bound, one key per leaf, leaf maxima);
  * an independent list-based transcription written in this file from the C++ algorithm
    (S8c O4), compared on random inputs, including degenerate geometries.
"""
import json
import math
import os

import numpy as np
import pytest

GOLD = os.path.join(os.path.dirname(__file__), "golden")


# ex1 (100x50, N=3): nIni=round(2.0)=2, hX=50 -> roots [0,50),[50,100). Round 1: root 0 keeps
#   (10,10),(12,12) together in TL; root 1 sends (60,40)->BL, (70,5)->TL, (90,45)->BR. 4 >= 3:
#   stop; the 2-key node keeps its max (12,12,9).
# ex2 (100x100, N=5): both keys land in TL of the single root -> node count 1 == prev: stop.
# ex3 (64x64, 9 keys in 4 tight clusters of 3/2/2/2, N = 5, 6, 7): nIni = 1; round 1 puts one
#   cluster in each 32x32 quadrant -> 4 nodes (< N, 4 + 3*4 = 16 > N) -> phase 2.  Its first round
#   splits each 32x32 node at 16 px, but every cluster lies inside one 16x16 child (TL keys
#   x,y < 16; TR x in [32,48), y < 16; BL x < 16, y in [32,48); BR x,y >= 48), so each split
#   yields ONE child: node count 4 == prev -> no-progress stop with 4 outputs for every N.
#   Kept = each cluster's max score: TL (5,6,9) and (7,5,9) tie -> the smaller rank (5,6);
#   TR (42,2,7); BL (10,40,6); BR (52,53,8).
# ex4 (64x64): round 1 gives four 2-key nodes (4 < N, 4+12 > N) -> phase 2 in order
#   TL (UL 0,0), TR (UL 32,0), BL (UL 0,32), BR (UL 32,32), each split separating its pair.
def test_hand_worked_cases(ref):
    with open(os.path.join(GOLD, "quadtree_cases.json")) as f:
        cases = json.load(f)["cases"]
    for c in cases:
        k = np.array(c["keys"], np.int32)
        idx = ref.distribute(k[:, 0], k[:, 1], k[:, 2], c["width"], c["height"], c["N"])
        got = sorted(map(tuple, k[idx, :2].tolist()))
        assert got == sorted(map(tuple, c["expect"])), c["name"]


def _f32(x):
    return float(np.float32(x))


def transcription(kx, ky, score, width, height, N):
    """Independent list-based transcription of DistributeOctTree [ext] (S8c O4 reading)."""
    n = len(kx)
    if n == 0:
        return []
    nIni = int(math.floor(abs(_f32(_f32(width) / _f32(height))) + 0.5))
    hX = _f32(_f32(width) / _f32(nIni))

    def node(ul, ur_x, bl_y, keys):
        return {"ul": ul, "urx": ur_x, "bly": bl_y, "keys": keys, "nomore": len(keys) == 1}

    roots = [node((int(_f32(hX * i)), 0), int(_f32(hX * (i + 1))), height, []) for i in range(nIni)]
    for k in range(n):
        r = min(int(_f32(_f32(kx[k]) / hX)), nIni - 1)
        roots[r]["keys"].append(k)
    nodes = [r for r in roots if r["keys"]]
    for r in nodes:
        r["nomore"] = len(r["keys"]) == 1

    def divide(nd):
        ulx, uly = nd["ul"]
        hx = math.ceil((nd["urx"] - ulx) / 2)
        hy = math.ceil((nd["bly"] - uly) / 2)
        geo = [((ulx, uly), ulx + hx, uly + hy), ((ulx + hx, uly), nd["urx"], uly + hy),
               ((ulx, uly + hy), ulx + hx, nd["bly"]), ((ulx + hx, uly + hy), nd["urx"], nd["bly"])]
        ch = [node(g[0], g[1], g[2], []) for g in geo]
        for k in nd["keys"]:
            right = kx[k] >= ulx + hx
            down = ky[k] >= uly + hy
            ch[2 * down + right]["keys"].append(k)
        out = [c for c in ch if c["keys"]]
        for c in out:
            c["nomore"] = len(c["keys"]) == 1
        return out

    finish = False
    while not finish:
        prev = len(nodes)
        new, expand = [], []
        for nd in nodes:
            if nd["nomore"]:
                new.append(nd)
                continue
            for c in divide(nd):
                new.append(c)
                if len(c["keys"]) > 1:
                    expand.append(c)
        nodes = new
        if len(nodes) >= N or len(nodes) == prev:
            finish = True
        elif len(nodes) + 3 * len(expand) > N:
            while not finish:
                prev = len(nodes)
                order = sorted(expand, key=lambda c: (-len(c["keys"]), c["ul"][1], c["ul"][0], c["keys"][0]))
                expand = []
                for nd in order:
                    nodes = [m for m in nodes if m is not nd]
                    for c in divide(nd):
                        nodes.append(c)
                        if len(c["keys"]) > 1:
                            expand.append(c)
                    if len(nodes) >= N:
                        break
                if len(nodes) >= N or len(nodes) == prev:
                    finish = True
    out = []
    for nd in nodes:
        best = nd["keys"][0]
        for k in nd["keys"][1:]:
            if score[k] > score[best]:
                best = k
        out.append(best)
    return sorted(out)


def _random_keys(rng, width, height, n, clustered):
    if clustered:
        cx = rng.integers(0, width, size=max(1, n // 8))
        cy = rng.integers(0, height, size=max(1, n // 8))
        pick = rng.integers(0, len(cx), size=n)
        xs = np.clip(cx[pick] + rng.integers(-6, 7, size=n), 0, width - 1)
        ys = np.clip(cy[pick] + rng.integers(-6, 7, size=n), 0, height - 1)
    else:
        xs = rng.integers(0, width, size=n)
        ys = rng.integers(0, height, size=n)
    pos = np.unique(ys.astype(np.int64) * 4096 + xs)
    rng.shuffle(pos)
    ky, kx = (pos // 4096).astype(np.int32), (pos % 4096).astype(np.int32)
    sc = rng.integers(8, 60, size=len(kx)).astype(np.int32)  # many equal scores -> tie rule
    return kx, ky, sc


@pytest.mark.parametrize("seed", range(40))
def test_oracle_equals_transcription(ref, seed):
    rng = np.random.default_rng(seed)
    width = int(rng.choice([720, 608, 1209, 178, 147, 314, 300, 97]))
    height = int(rng.choice([448, 368, 344, 102, 73, 61, 200]))
    if round(width / height) < 1:
        width = height
    n = int(rng.integers(0, 900))
    kx, ky, sc = _random_keys(rng, width, height, n, clustered=bool(seed % 2))
    for N in (1, 5, 60, 217, 434, max(1, n // 2), 3 * n + 1):
        got = ref.distribute(kx, ky, sc, width, height, N).tolist()
        assert got == transcription(kx.tolist(), ky.tolist(), sc.tolist(), width, height, N), (seed, N)


@pytest.mark.parametrize("seed", range(12))
def test_invariants(ref, seed):
    rng = np.random.default_rng(1000 + seed)
    width, height = 720, 448
    kx, ky, sc = _random_keys(rng, width, height, int(rng.integers(1, 3000)), clustered=True)
    nIni = round(width / height)
    for N in (60, 217, 500):
        idx = ref.distribute(kx, ky, sc, width, height, N)
        assert len(idx) <= max(N + 2, 4 * nIni)
        assert len(set(idx.tolist())) == len(idx)
        # every kept key beats or ties (with lower rank) keys at the same position class:
        # the global max-score key with the lowest rank is always kept (it wins its leaf)
        best = max(range(len(kx)), key=lambda k: (sc[k], -k))
        assert best in set(idx.tolist())


def test_empty_and_single(ref):
    e = np.zeros(0, np.int32)
    assert len(ref.distribute(e, e, e, 720, 448, 217)) == 0
    one = np.array([5], np.int32)
    assert ref.distribute(one, one, one, 720, 448, 217).tolist() == [0]
