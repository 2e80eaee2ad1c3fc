"""Pins of the oracle's O4g grid top-N distribution (DESIGN.md §3 item 13; the north_star's
"grid top-N" alternative to the quadtree).  The rule is our own reading, so
there is no external implementation: it is pinned by hand-worked cases (cell quota
q = ceil(N / non-empty cells), ties by rank, the global trim to N) and by invariants on
real frames (per-cell quota, count = min(N, sum of capped cells), the trim keeps the best)."""
import numpy as np

import synth


def _cell_xy(p, l, i, j, dx=0, dy=0):
    # a pixel inside cell (i, j)'s detect window: window origin = 16 + 3 + cell size * index
    return 19 + j * p.cell_w[l] + dx, 19 + i * p.cell_h[l] + dy


def test_hand_worked_quota_and_trim(ref):
    p = ref.params(752, 480)
    # three cells: (0,0) has scores 50, 40, 40, 30 (ranks 0-3); (0,1) has 45 (rank 4);
    # (1,0) has 60, 20 (ranks 5, 6).  K = 3.
    pts = [(0, 0, 1, 1, 50), (0, 0, 2, 1, 40), (0, 0, 3, 1, 40), (0, 0, 4, 1, 30), (0, 1, 1, 1, 45),
           (1, 0, 1, 1, 60), (1, 0, 2, 1, 20)]
    lx, ly, sc = [], [], []
    for i, j, dx, dy, s in pts:
        x, y = _cell_xy(p, 0, i, j, dx, dy)
        lx.append(x), ly.append(y), sc.append(s)
    # N = 3 -> q = 1: best of each cell -> ranks {0, 4, 5}; pool 3 <= N
    assert sorted(ref.distribute_grid(p, 0, lx, ly, sc, 3)) == [0, 4, 5]
    # N = 4 -> q = 2: cell0 {0, 1} (40 tie -> lower rank 1), cell1 {4}, cell2 {5, 6}: pool 5 > 4,
    # trim by (score desc, rank): 60(5), 50(0), 45(4), 40(1) -> drops 20(6)
    assert sorted(ref.distribute_grid(p, 0, lx, ly, sc, 4)) == [0, 1, 4, 5]
    # N = 6 -> q = 2: same pool of 5 <= 6
    assert sorted(ref.distribute_grid(p, 0, lx, ly, sc, 6)) == [0, 1, 4, 5, 6]
    # N = 9 -> q = 3: cell0 {0, 1, 2}, pool 6
    assert sorted(ref.distribute_grid(p, 0, lx, ly, sc, 9)) == [0, 1, 2, 4, 5, 6]
    # N = 2 -> q = 1: pool {0, 4, 5} trimmed to the best two: 60(5), 50(0)
    assert sorted(ref.distribute_grid(p, 0, lx, ly, sc, 2)) == [0, 5]
    assert len(ref.distribute_grid(p, 0, [], [], [], 5)) == 0


def test_invariants_on_frames(ref):
    for shape in ("euroc", "kitti"):
        w, h = synth.SHAPES[shape]
        p = ref.params(w, h, 1000)
        img = synth.make_frame(w, h, 31)
        pyr = ref.pyramid(p, img)
        for l in range(p.n_levels):
            M = ref.fast_M(pyr[l])
            lx, ly, sc = ref.cell_candidates(p, l, M)
            N = p.n_per_level[l]
            keep = ref.distribute_grid(p, l, lx, ly, sc, N)
            cell = ((ly - 19) // p.cell_h[l]) * p.cell_cols[l] + (lx - 19) // p.cell_w[l]
            cells, cnt = np.unique(cell, return_counts=True)
            q = -(-N // len(cells)) if len(cells) else 0
            assert len(keep) == min(N, int(np.minimum(cnt, q).sum()))
            assert len(set(keep.tolist())) == len(keep)
            kc = np.bincount(np.searchsorted(cells, cell[keep]), minlength=len(cells))
            assert (kc <= q).all()
            # inside a cell, nothing dropped beats a kept one
            key = sc.astype(np.int64) * 10 ** 7 - np.arange(len(sc))
            kept = np.zeros(len(sc), bool)
            kept[keep] = True
            for c in cells:
                m = cell == c
                if kept[m].sum() == q and (~kept[m]).any():  # at quota: its best q were kept
                    assert key[m & ~kept].max() < key[m & kept].min()
            # trimmed: every cell-quota survivor that was dropped is worse than every kept key
            pool = np.zeros(len(sc), bool)
            for c in cells:
                idx = np.where(cell == c)[0]
                order = idx[np.lexsort((idx, -sc[idx]))]
                pool[order[:q]] = True
            if pool.sum() > N:
                assert key[pool & ~kept].max() < key[kept].min()
            else:
                assert (pool == kept).all()


def test_extract_mode_grid_counts(ref):
    w, h = synth.SHAPES["euroc"]
    p = ref.params(w, h, 1000)
    img = synth.make_frame(w, h, 5)
    k, d, c = ref.orb_extract(p, img, mode=1)
    per_level = np.diff(c)
    assert (per_level <= np.array(p.n_per_level[:p.n_levels])).all()
    assert per_level.sum() > 0.9 * 1000
    lv = k["level"][: c[-1]]
    key = lv.astype(np.int64) << 40 | k["ly"][: c[-1]].astype(np.int64) << 20 | k["lx"][: c[-1]]
    assert (np.diff(key) > 0).all()  # canonical (level, ly, lx) order
