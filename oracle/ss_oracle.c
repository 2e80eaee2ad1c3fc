/*
 * ss_oracle.c -- CPU ORACLE (TEST INFRASTRUCTURE ONLY; see ss_oracle.h).
 *
 * Plain, single-threaded, obviously-correct C following the definitions the
 * product must reproduce.  The paper (SLAM-Share, CoNEXT'22) moves ORB-SLAM3's
 * FAST detection and "search local points" onto a GPU (§4.2.1)
 * but prints no arithmetic; every step below therefore follows the reading in
 * SURVEY.md §8(c) (rows O0..O10), each of which DESIGN.md §3 lists.
 *
 * Build: gcc -O2 -ffp-contract=off -fPIC -shared (no SIMD intrinsics, no OpenMP).
 * Nothing here is shared with the CUDA path.
 *
 * Parity pins (tests/test_oracle_*.py):
 *   O0 params      : App. B tables of SURVEY.md (tests/golden/params_*.json)
 *   O1 pyramid     : cv2.resize(INTER_LINEAR_EXACT), chained
 *   O2 FAST M      : cv2.FAST(TYPE_9_16) thresholds/responses; exhaustive ring masks
 *   O3 cells       : ORB-SLAM's per-cell cv2.FAST loop with iniTh/minTh fallback
 *   O4 quadtree    : hand-worked cases (tests/golden/quadtree_cases.json) + invariants
 *                    + an independent std::list-style transcription.  NO external
 *                    reference exists (ORB-SLAM's tie-break is heap-address order):
 *                    "parity unpinned" against ORB-SLAM itself, see DESIGN.md.
 *   O5 orientation : closed form on intensity planes; rot90 permutation
 *   O6 blur        : cv2.GaussianBlur(7x7, sigma 2, REFLECT_101)
 *   O7 descriptor  : rot90 invariance (bit-exact); unrotated case = pattern lookups
 *   O9/O10 match   : brute-force definitions in Python on small inputs
 *   O12 stereo     : right image = left shifted by an integer disparity (uR within 0.5 px
 *                    of uL - d, depth ~ bf/d); invariants (level gate, Hamming < 75,
 *                    disparity range, outlier cut at 2.1 x the median SAD)
 *   O11 projection : cv2.projectPoints (f64) on random poses; closed forms (optical axis,
 *                    rot90 about z, viewCos = 1 along the normal); predicted level vs
 *                    ceil(log(ratio)/log(1.2)) away from level boundaries; each culling
 *                    rule isolated by a point that violates only it
 *   O13 last frame : integer image shift of a fronto-parallel plane (every level-0 keypoint
 *                    matched to its shifted twin at d = 0, rotation bin 0); hand-worked
 *                    three-maxima / dedup / TH_HIGH / level-gate / retry cases; rotation-bin
 *                    closed forms; numpy brute force of steps 1-4
 */
#include "ss_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

#include "brief_pattern_ref.inc"

#define EDGE_THRESHOLD 19
#define MIN_BORDER (EDGE_THRESHOLD - 3) /* 16 */
#define CELL_W 30                       /* north_star: "per 30-px grid cell" */
#define HALF_PATCH 15

static int imin(int a, int b) { return a < b ? a : b; }
static int imax(int a, int b) { return a > b ? a : b; }

/* ---------------------------------------------------------------- O0 params */
/* S8c O0: f32 scale chain, rne level sizes, ORB-SLAM per-level feature split. */
int ref_params_init(int32_t w, int32_t h, int32_t nf, int32_t L, float sf, int32_t ini, int32_t mn,
                    ref_params* p) {
  if (!p || L < 1 || L > REF_MAX_LEVELS || w < 64 || h < 64 || w > 2048 || h > 2048 || nf < 1 ||
      !(sf > 1.0f) || ini < 1 || mn < 1 || ini > 254 || mn > 254)
    return -1;
  memset(p, 0, sizeof(*p));
  p->width = w; p->height = h; p->n_features = nf; p->n_levels = L; p->scale_factor = sf;
  p->ini_th_fast = ini; p->min_th_fast = mn;
  p->scale[0] = 1.0f;
  for (int l = 1; l < L; l++) p->scale[l] = p->scale[l - 1] * sf;
  for (int l = 0; l < L; l++) p->inv_scale[l] = 1.0f / p->scale[l];
  for (int l = 0; l < L; l++) {
    float fw = (float)w * p->inv_scale[l];
    float fh = (float)h * p->inv_scale[l];
    p->level_w[l] = (int32_t)lrintf(fw);
    p->level_h[l] = (int32_t)lrintf(fh);
  }
  float factor = 1.0f / sf;
  float nd = (float)nf * (1.0f - factor) / (1.0f - (float)pow((double)factor, (double)L));
  int sum = 0;
  for (int l = 0; l < L - 1; l++) {
    p->n_per_level[l] = (int32_t)lrintf(nd);
    sum += p->n_per_level[l];
    nd *= factor;
  }
  p->n_per_level[L - 1] = imax(nf - sum, 0);
  int cap = 0;
  for (int l = 0; l < L; l++) {
    int lw = p->level_w[l], lh = p->level_h[l];
    int maxBX = lw - EDGE_THRESHOLD + 3, maxBY = lh - EDGE_THRESHOLD + 3;
    float width = (float)(maxBX - MIN_BORDER), height = (float)(maxBY - MIN_BORDER);
    int ncols = (int)(width / (float)CELL_W), nrows = (int)(height / (float)CELL_W);
    if (ncols < 1 || nrows < 1) return -1;
    p->cell_cols[l] = ncols; p->cell_rows[l] = nrows;
    p->cell_w[l] = (int)ceilf(width / (float)ncols);
    p->cell_h[l] = (int)ceilf(height / (float)nrows);
    int nini = (int)roundf(width / height); /* std::round: half away from zero */
    if (nini < 1 || nini > 62) return -1;
    p->n_ini[l] = nini;
    /* S8c O4: <= N+2 after phase 1/2, but the first unconditional split can give 4*nIni. */
    p->level_cap[l] = imax(p->n_per_level[l] + 2, 4 * nini);
    cap += p->level_cap[l];
  }
  p->kp_capacity = cap;
  return 0;
}

/* ---------------------------------------------------------------- O1 pyramid */
/* S8c O1: bit-exact INTER_LINEAR_EXACT (8-bit weights, f64 source mapping, rne weights). */
static void linear_coeffs(int d, int sn, int dn, int* s0, int* s1, int* w1) {
  double f = ((double)d + 0.5) * ((double)sn / (double)dn) - 0.5;
  double fl = floor(f);
  int s = (int)fl;
  double a = f - fl;
  if (s < 0) { s = 0; a = 0.0; }
  if (s >= sn - 1) { s = sn - 1; a = 0.0; }
  *s0 = s;
  *s1 = imin(s + 1, sn - 1);
  *w1 = (int)lrint(a * 256.0); /* round half even */
}

void ref_resize_linear_exact(const uint8_t* src, int sw, int sh, int sp, uint8_t* dst, int dw, int dh,
                             int dp) {
  for (int y = 0; y < dh; y++) {
    int y0, y1, wy1;
    linear_coeffs(y, sh, dh, &y0, &y1, &wy1);
    int wy0 = 256 - wy1;
    for (int x = 0; x < dw; x++) {
      int x0, x1, wx1;
      linear_coeffs(x, sw, dw, &x0, &x1, &wx1);
      int wx0 = 256 - wx1;
      int h0 = wx0 * src[y0 * sp + x0] + wx1 * src[y0 * sp + x1];
      int h1 = wx0 * src[y1 * sp + x0] + wx1 * src[y1 * sp + x1];
      int v = wy0 * h0 + wy1 * h1;
      dst[y * dp + x] = (uint8_t)((v + (1 << 15)) >> 16);
    }
  }
}

int64_t ref_pyramid_bytes(const ref_params* p) {
  int64_t s = 0;
  for (int l = 0; l < p->n_levels; l++) s += (int64_t)p->level_w[l] * p->level_h[l];
  return s;
}

void ref_pyramid(const ref_params* p, const uint8_t* img, int pitch, uint8_t* out) {
  int64_t off = 0, prev = 0;
  for (int l = 0; l < p->n_levels; l++) {
    int w = p->level_w[l], h = p->level_h[l];
    if (l == 0) {
      for (int y = 0; y < h; y++) memcpy(out + (int64_t)y * w, img + (int64_t)y * pitch, (size_t)w);
    } else {
      ref_resize_linear_exact(out + prev, p->level_w[l - 1], p->level_h[l - 1], p->level_w[l - 1],
                              out + off, w, h, w);
    }
    prev = off;
    off += (int64_t)w * h;
  }
}

/* ---------------------------------------------------------------- O2 FAST */
/* OpenCV offsets16 order, (dx, dy). FAST-9/16 [38]. */
static const int RING[16][2] = {{0, 3},  {1, 3},   {2, 2},   {3, 1},   {3, 0},  {3, -1},
                                {2, -2}, {1, -3},  {0, -3},  {-1, -3}, {-2, -2}, {-3, -1},
                                {-3, 0}, {-3, 1},  {-2, 2},  {-1, 3}};

/* M(p) = max_s max( min_{k<9} d_{s+k}, min_{k<9} -d_{s+k} ),  d_k = I(p) - I(p + R_k).
 * corner at threshold t  <=>  M > t ;  OpenCV response = M - 1. */
static int fast_M_at(const uint8_t* img, int pitch, int x, int y) {
  int c = img[y * pitch + x];
  int d[16];
  for (int k = 0; k < 16; k++) d[k] = c - img[(y + RING[k][1]) * pitch + x + RING[k][0]];
  int best = -1000;
  for (int s = 0; s < 16; s++) {
    int mn = 1000, mx = 1000;
    for (int k = 0; k < 9; k++) {
      int v = d[(s + k) & 15];
      if (v < mn) mn = v;
      if (-v < mx) mx = -v;
    }
    if (mn > best) best = mn;
    if (mx > best) best = mx;
  }
  return best;
}

void ref_fast_M(const uint8_t* img, int w, int h, int pitch, uint8_t* out) {
  memset(out, 0, (size_t)w * h);
  for (int y = 3; y < h - 3; y++)
    for (int x = 3; x < w - 3; x++) {
      int m = fast_M_at(img, pitch, x, y);
      out[y * w + x] = (uint8_t)(m < 0 ? 0 : m);
    }
}

/* ---------------------------------------------------------------- O3 cells */
/* ORB-SLAM's per-cell FAST (cv::FAST on the cell ROI, nonmax on) with the iniTh ->
 * minTh fallback [ext], restated: in the detect window D of the cell, keep p with
 * M(p) > t that beats every 8-neighbour inside D (S8c O3). Rank = cell row-major, y, x. */
int ref_cell_candidates(const ref_params* p, int l, const uint8_t* M, int32_t* lx, int32_t* ly,
                        int32_t* score, int cap) {
  int w = p->level_w[l], h = p->level_h[l];
  int maxBX = w - EDGE_THRESHOLD + 3, maxBY = h - EDGE_THRESHOLD + 3;
  int wc = p->cell_w[l], hc = p->cell_h[l];
  int n = 0;
  (void)h;
  for (int i = 0; i < p->cell_rows[l]; i++) {
    int iniY = MIN_BORDER + i * hc;
    if (iniY >= maxBY - 3) continue;
    int maxY = imin(iniY + hc + 6, maxBY);
    for (int j = 0; j < p->cell_cols[l]; j++) {
      int iniX = MIN_BORDER + j * wc;
      if (iniX >= maxBX - 6) continue;
      int maxX = imin(iniX + wc + 6, maxBX);
      int x0 = iniX + 3, x1 = maxX - 3, y0 = iniY + 3, y1 = maxY - 3;
      int thr[2] = {p->ini_th_fast, p->min_th_fast};
      for (int pass = 0; pass < 2; pass++) {
        int found = 0;
        for (int y = y0; y < y1; y++)
          for (int x = x0; x < x1; x++) {
            int m = M[y * w + x];
            if (m <= thr[pass]) continue;
            int keep = 1;
            for (int dy = -1; dy <= 1 && keep; dy++)
              for (int dx = -1; dx <= 1; dx++) {
                if (!dx && !dy) continue;
                int qx = x + dx, qy = y + dy;
                if (qx < x0 || qx >= x1 || qy < y0 || qy >= y1) continue; /* outside D: ignored */
                if (M[qy * w + qx] >= m) { keep = 0; break; }
              }
            if (!keep) continue;
            if (n >= cap) return -1;
            lx[n] = x; ly[n] = y; score[n] = m; n++;
            found++;
          }
        if (found) break;
      }
    }
  }
  return n;
}

/* ---------------------------------------------------------------- O4 quadtree */
/* Literal transcription of ORB-SLAM's DistributeOctTree [ext] (S8c O4): f32 root
 * geometry, ceil halving, phase 1 (split every multi-key node) and phase 2 (split
 * largest nodes first until N), "no progress" stop, per-node max response with ties to
 * the first key in parent order.  Reading: equal-size nodes in phase 2 are ordered by
 * (UL.y, UL.x, first-key rank) instead of heap address.  parity unpinned vs ORB-SLAM. */
typedef struct {
  int ulx, uly, urx, blx, bly; /* UR.y == UL.y, BR = (UR.x, BL.y) */
  int* keys;                   /* indices into the input, in parent order */
  int n;
  int nomore;
} qnode;

typedef struct {
  qnode* v;
  int n, cap;
} qlist;

static void qpush(qlist* L, qnode nd) {
  if (L->n == L->cap) {
    L->cap = L->cap ? 2 * L->cap : 64;
    L->v = (qnode*)realloc(L->v, sizeof(qnode) * (size_t)L->cap);
  }
  L->v[L->n++] = nd;
}

static void qdivide(const qnode* nd, const int32_t* kx, const int32_t* ky, qnode ch[4]) {
  int halfX = (int)ceilf((float)(nd->urx - nd->ulx) / 2);
  int halfY = (int)ceilf((float)(nd->bly - nd->uly) / 2);
  /* n1 TL, n2 TR, n3 BL, n4 BR (ORB-SLAM ExtractorNode::DivideNode) */
  ch[0].ulx = nd->ulx;         ch[0].uly = nd->uly;         ch[0].urx = nd->ulx + halfX;
  ch[0].blx = nd->ulx;         ch[0].bly = nd->uly + halfY;
  ch[1].ulx = nd->ulx + halfX; ch[1].uly = nd->uly;         ch[1].urx = nd->urx;
  ch[1].blx = nd->ulx + halfX; ch[1].bly = nd->uly + halfY;
  ch[2].ulx = nd->ulx;         ch[2].uly = nd->uly + halfY; ch[2].urx = nd->ulx + halfX;
  ch[2].blx = nd->blx;         ch[2].bly = nd->bly;
  ch[3].ulx = nd->ulx + halfX; ch[3].uly = nd->uly + halfY; ch[3].urx = nd->urx;
  ch[3].blx = nd->ulx + halfX; ch[3].bly = nd->bly;
  for (int c = 0; c < 4; c++) {
    ch[c].keys = (int*)malloc(sizeof(int) * (size_t)(nd->n > 0 ? nd->n : 1));
    ch[c].n = 0;
    ch[c].nomore = 0;
  }
  int midx = nd->ulx + halfX, midy = nd->uly + halfY;
  for (int i = 0; i < nd->n; i++) {
    int k = nd->keys[i];
    int c;
    if (kx[k] < midx) c = (ky[k] < midy) ? 0 : 2;
    else c = (ky[k] < midy) ? 1 : 3;
    ch[c].keys[ch[c].n++] = k;
  }
  for (int c = 0; c < 4; c++)
    if (ch[c].n == 1) ch[c].nomore = 1;
}

/* phase-2 order: size desc, UL.y asc, UL.x asc, first-key rank asc (reading) */
static const qnode* g_sort_base;
static int cmp_phase2(const void* a, const void* b) {
  const qnode* A = &g_sort_base[*(const int*)a];
  const qnode* B = &g_sort_base[*(const int*)b];
  if (A->n != B->n) return A->n > B->n ? -1 : 1;
  if (A->uly != B->uly) return A->uly < B->uly ? -1 : 1;
  if (A->ulx != B->ulx) return A->ulx < B->ulx ? -1 : 1;
  return A->keys[0] < B->keys[0] ? -1 : (A->keys[0] > B->keys[0] ? 1 : 0);
}

/* Splits node index `idx` of *nodes (marking it dead, n = -1) and appends the non-empty
 * children; indices of children with > 1 key are appended to *expand. Returns #children. */
static int split_node(qlist* nodes, int idx, const int32_t* kx, const int32_t* ky, int** expand,
                      int* nexp, int* expcap) {
  qnode ch[4];
  qnode parent = nodes->v[idx];
  qdivide(&parent, kx, ky, ch);
  free(parent.keys);
  nodes->v[idx].keys = NULL;
  nodes->v[idx].n = -1; /* dead */
  int made = 0;
  for (int c = 0; c < 4; c++) {
    if (ch[c].n > 0) {
      qpush(nodes, ch[c]);
      made++;
      if (ch[c].n > 1) {
        if (*nexp == *expcap) {
          *expcap = *expcap ? 2 * *expcap : 64;
          *expand = (int*)realloc(*expand, sizeof(int) * (size_t)*expcap);
        }
        (*expand)[(*nexp)++] = nodes->n - 1;
      }
    } else {
      free(ch[c].keys);
    }
  }
  return made;
}

int ref_distribute(const int32_t* kx, const int32_t* ky, const int32_t* score, int n, int width,
                   int height, int N, int32_t* out_idx) {
  if (n <= 0) return 0;
  int nIni = (int)roundf((float)width / (float)height);
  if (nIni < 1) return -1;
  float hX = (float)width / (float)nIni;
  qlist nodes = {0, 0, 0};
  int alive = 0;
  /* roots */
  int root0 = 0;
  for (int i = 0; i < nIni; i++) {
    qnode r;
    r.ulx = (int)(hX * (float)i);
    r.uly = 0;
    r.urx = (int)(hX * (float)(i + 1));
    r.blx = r.ulx;
    r.bly = height;
    r.keys = (int*)malloc(sizeof(int) * (size_t)n);
    r.n = 0;
    r.nomore = 0;
    qpush(&nodes, r);
  }
  for (int k = 0; k < n; k++) {
    int ri = (int)((float)kx[k] / hX);
    if (ri > nIni - 1) ri = nIni - 1; /* unreachable for widths <= 2048; kept defined */
    nodes.v[root0 + ri].keys[nodes.v[root0 + ri].n++] = k;
  }
  for (int i = 0; i < nIni; i++) {
    qnode* r = &nodes.v[i];
    if (r->n == 0) { free(r->keys); r->keys = NULL; r->n = -1; }
    else { if (r->n == 1) r->nomore = 1; alive++; }
  }
  int* expand = NULL;
  int nexp = 0, expcap = 0;
  int finish = 0;
  while (!finish) {
    int prevSize = alive;
    int nToExpand;
    nexp = 0;
    int cur = nodes.n;
    for (int i = 0; i < cur; i++) {
      if (nodes.v[i].n < 0 || nodes.v[i].nomore) continue;
      int made = split_node(&nodes, i, kx, ky, &expand, &nexp, &expcap);
      alive += made - 1;
    }
    nToExpand = nexp;
    if (alive >= N || alive == prevSize) {
      finish = 1;
    } else if (alive + nToExpand * 3 > N) {
      while (!finish) {
        prevSize = alive;
        int nprev = nexp;
        int* prev = (int*)malloc(sizeof(int) * (size_t)(nprev > 0 ? nprev : 1));
        memcpy(prev, expand, sizeof(int) * (size_t)nprev);
        nexp = 0;
        g_sort_base = nodes.v;
        qsort(prev, (size_t)nprev, sizeof(int), cmp_phase2);
        for (int j = 0; j < nprev; j++) {
          int made = split_node(&nodes, prev[j], kx, ky, &expand, &nexp, &expcap);
          alive += made - 1;
          g_sort_base = nodes.v; /* nodes.v may have been reallocated */
          if (alive >= N) break;
        }
        free(prev);
        if (alive >= N || alive == prevSize) finish = 1;
      }
    }
  }
  /* retain the best key of each node: max score, ties -> first key (smallest rank) */
  int m = 0;
  for (int i = 0; i < nodes.n; i++) {
    qnode* nd = &nodes.v[i];
    if (nd->n < 0) continue;
    int best = nd->keys[0];
    for (int t = 1; t < nd->n; t++)
      if (score[nd->keys[t]] > score[best]) best = nd->keys[t];
    out_idx[m++] = best;
    free(nd->keys);
  }
  free(nodes.v);
  free(expand);
  return m;
}

/* ---------------------------------------------------------------- O5 orientation */
/* umax built as ORB-SLAM's ORBextractor constructor does [ext]; 749-px disk. */
static void build_umax(int umax[HALF_PATCH + 1]) {
  int vmax = (int)floor(HALF_PATCH * sqrt(2.f) / 2 + 1);
  int vmin = (int)ceil(HALF_PATCH * sqrt(2.f) / 2);
  const double hp2 = HALF_PATCH * HALF_PATCH;
  int v, v0;
  for (v = 0; v <= vmax; ++v) umax[v] = (int)lrint(sqrt(hp2 - v * v));
  for (v = HALF_PATCH, v0 = 0; v >= vmin; --v) {
    while (umax[v0] == umax[v0 + 1]) ++v0;
    umax[v] = v0;
    ++v0;
  }
}

/* "Oriented FAST": intensity-centroid moments over the disk (S8c O5). */
void ref_moments(const uint8_t* img, int pitch, int lx, int ly, int32_t* m10, int32_t* m01) {
  int umax[HALF_PATCH + 1];
  build_umax(umax);
  int64_t a = 0, b = 0;
  for (int v = -HALF_PATCH; v <= HALF_PATCH; v++) {
    int d = umax[v < 0 ? -v : v];
    for (int u = -d; u <= d; u++) {
      int I = img[(ly + v) * pitch + lx + u];
      a += (int64_t)u * I;
      b += (int64_t)v * I;
    }
  }
  *m10 = (int32_t)a;
  *m01 = (int32_t)b;
}

/* angle = atan2(m01, m10) in degrees, [0, 360); (0,0) -> 0 (S8c O5 reading). */
float ref_angle_deg(int32_t m10, int32_t m01) {
  if (m10 == 0 && m01 == 0) return 0.0f;
  double a = atan2((double)m01, (double)m10) * (180.0 / 3.14159265358979323846);
  if (a < 0) a += 360.0;
  float f = (float)a;
  if (f >= 360.0f) f = 0.0f;
  return f;
}

/* ---------------------------------------------------------------- O6 blur */
/* GaussianBlur(7x7, sigma=2, REFLECT_101) bit-exact fixed point: Q8 taps, exact
 * horizontal sum, vertical (sum + 2^15) >> 16 (S8c O6). */
static const int BLUR_K[7] = {18, 34, 48, 56, 48, 34, 18};

static int reflect101(int i, int n) {
  while (i < 0 || i >= n) {
    if (i < 0) i = -i;
    if (i >= n) i = 2 * n - 2 - i;
  }
  return i;
}

void ref_blur(const uint8_t* img, int w, int h, int pitch, uint8_t* out, int opitch) {
  int* hs = (int*)malloc(sizeof(int) * (size_t)w * h);
  for (int y = 0; y < h; y++)
    for (int x = 0; x < w; x++) {
      int s = 0;
      for (int j = 0; j < 7; j++) s += BLUR_K[j] * img[y * pitch + reflect101(x + j - 3, w)];
      hs[y * w + x] = s;
    }
  for (int y = 0; y < h; y++)
    for (int x = 0; x < w; x++) {
      int64_t s = 0;
      for (int i = 0; i < 7; i++) s += (int64_t)BLUR_K[i] * hs[reflect101(y + i - 3, h) * w + x];
      out[y * opitch + x] = (uint8_t)((s + (1 << 15)) >> 16);
    }
  free(hs);
}

/* ---------------------------------------------------------------- O7 descriptor */
/* Exact round-half-even of z / sqrt(r2), r2 > 0, by plain integer search (S8c O7). */
int32_t ref_rhe_div_sqrt(int64_t z, int64_t r2) {
  int neg = z < 0;
  int64_t a = neg ? -z : z;
  int64_t A = 4 * a * a; /* (2a)^2 */
  int64_t k = 0;
  while ((2 * k + 1) * (2 * k + 1) * r2 < A) k++; /* a/r in (k-1/2, k+1/2] */
  if ((2 * k + 1) * (2 * k + 1) * r2 == A && (k & 1)) k++; /* a/r == k+1/2: to even */
  return (int32_t)(neg ? -k : k);
}

/* Rotated BRIEF: offsets (x cos - y sin, x sin + y cos) with cos = m10/r,
 * sin = m01/r, exactly rounded; bit b = B(p_2b) < B(p_2b+1), LSB first. */
void ref_descriptor(const uint8_t* B, int pitch, int lx, int ly, int32_t m10, int32_t m01,
                    uint8_t out[32]) {
  int64_t r2 = (int64_t)m10 * m10 + (int64_t)m01 * m01;
  memset(out, 0, 32);
  for (int b = 0; b < 256; b++) {
    int v[2];
    for (int e = 0; e < 2; e++) {
      int px = REF_BRIEF_PATTERN[4 * b + 2 * e], py = REF_BRIEF_PATTERN[4 * b + 2 * e + 1];
      int ox, oy;
      if (r2 == 0) { ox = px; oy = py; }
      else {
        ox = ref_rhe_div_sqrt((int64_t)px * m10 - (int64_t)py * m01, r2);
        oy = ref_rhe_div_sqrt((int64_t)px * m01 + (int64_t)py * m10, r2);
      }
      v[e] = B[(ly + oy) * pitch + lx + ox];
    }
    if (v[0] < v[1]) out[b >> 3] |= (uint8_t)(1u << (b & 7));
  }
}

/* ---------------------------------------------------------------- O1..O8 */
/* ------------------------------------------------ O4g grid top-N distribution */
/* The north_star's alternative to the quadtree ("a per-level quadtree (or grid top-N)
 * distribution"), reading (DESIGN.md §3 item 13): on level l with N
 * = n_per_level[l] and the O3 candidates in rank order,
 *   K = number of FAST cells with at least one candidate, q = ceil(N / K);
 *   every cell keeps its q best candidates by (score desc, rank asc);
 *   if more than N remain, the N best of them by (score desc, rank asc) are kept.
 * A candidate's cell is (i, j) = ((ly - 16 - 3) / cell_h, (lx - 16 - 3) / cell_w), the O3
 * detect-window tiling.  Returns the number kept (<= N); out_idx = indices into the input.
 * Parity: no external reference exists (the definition is ours): hand-worked cases and
 * invariants in tests/test_oracle_grid.py. */
typedef struct { int score, rank, cell; } gcand;
static int cmp_gcand(const void* a, const void* b) {  /* cell, then score desc, then rank */
  const gcand* A = (const gcand*)a; const gcand* B = (const gcand*)b;
  if (A->cell != B->cell) return A->cell < B->cell ? -1 : 1;
  if (A->score != B->score) return A->score > B->score ? -1 : 1;
  return A->rank < B->rank ? -1 : (A->rank > B->rank);
}
static int cmp_gbest(const void* a, const void* b) {  /* score desc, then rank */
  const gcand* A = (const gcand*)a; const gcand* B = (const gcand*)b;
  if (A->score != B->score) return A->score > B->score ? -1 : 1;
  return A->rank < B->rank ? -1 : (A->rank > B->rank);
}

int ref_distribute_grid(const ref_params* p, int l, const int32_t* lx, const int32_t* ly, const int32_t* score,
                        int n, int N, int32_t* out_idx) {
  if (n <= 0 || N <= 0) return 0;
  gcand* c = (gcand*)malloc(sizeof(gcand) * (size_t)n);
  for (int i = 0; i < n; i++) {
    int ci = (ly[i] - MIN_BORDER - 3) / p->cell_h[l], cj = (lx[i] - MIN_BORDER - 3) / p->cell_w[l];
    c[i].score = score[i]; c[i].rank = i; c[i].cell = ci * p->cell_cols[l] + cj;
  }
  qsort(c, (size_t)n, sizeof(gcand), cmp_gcand);
  int K = 0;
  for (int i = 0; i < n; i++) if (i == 0 || c[i].cell != c[i - 1].cell) K++;
  int q = (N + K - 1) / K;
  gcand* pool = (gcand*)malloc(sizeof(gcand) * (size_t)n);
  int np = 0, run = 0;
  for (int i = 0; i < n; i++) {
    run = (i > 0 && c[i].cell == c[i - 1].cell) ? run + 1 : 0;
    if (run < q) pool[np++] = c[i];
  }
  if (np > N) {
    qsort(pool, (size_t)np, sizeof(gcand), cmp_gbest);
    np = N;
  }
  for (int i = 0; i < np; i++) out_idx[i] = pool[i].rank;
  free(pool); free(c);
  return np;
}

typedef struct { int lx, ly, score; } selkp;
static int cmp_yx(const void* a, const void* b) {
  const selkp* A = (const selkp*)a; const selkp* B = (const selkp*)b;
  if (A->ly != B->ly) return A->ly < B->ly ? -1 : 1;
  return A->lx < B->lx ? -1 : (A->lx > B->lx ? 1 : 0);
}

int ref_orb_extract_mode(const ref_params* p, const uint8_t* img, int pitch, int mode, ref_keypoint* kps,
                         uint8_t* desc, int32_t* counts) {
  int64_t pb = ref_pyramid_bytes(p);
  uint8_t* pyr = (uint8_t*)malloc((size_t)pb);
  ref_pyramid(p, img, pitch, pyr);
  int64_t off = 0;
  int total = 0;
  counts[0] = 0;
  for (int l = 0; l < p->n_levels; l++) {
    int w = p->level_w[l], h = p->level_h[l];
    const uint8_t* lev = pyr + off;
    uint8_t* M = (uint8_t*)malloc((size_t)w * h);
    ref_fast_M(lev, w, h, w, M);
    int cap = w * h;
    int32_t* cx = (int32_t*)malloc(sizeof(int32_t) * (size_t)cap * 3);
    int32_t *cy = cx + cap, *cs = cx + 2 * cap;
    int nc = ref_cell_candidates(p, l, M, cx, cy, cs, cap);
    int32_t* kx = (int32_t*)malloc(sizeof(int32_t) * (size_t)(nc > 0 ? nc : 1) * 3);
    int32_t *ky = kx + (nc > 0 ? nc : 1), *sel = kx + 2 * (nc > 0 ? nc : 1);
    for (int i = 0; i < nc; i++) { kx[i] = cx[i] - MIN_BORDER; ky[i] = cy[i] - MIN_BORDER; }
    int maxBX = w - EDGE_THRESHOLD + 3, maxBY = h - EDGE_THRESHOLD + 3;
    int ns = mode == 1 ? ref_distribute_grid(p, l, cx, cy, cs, nc, p->n_per_level[l], sel)
                       : ref_distribute(kx, ky, cs, nc, maxBX - MIN_BORDER, maxBY - MIN_BORDER,
                                        p->n_per_level[l], sel);
    if (ns > p->level_cap[l] || total + ns > p->kp_capacity) { ns = -1; }
    if (ns < 0) { free(kx); free(cx); free(M); free(pyr); return -1; }
    selkp* s = (selkp*)malloc(sizeof(selkp) * (size_t)(ns > 0 ? ns : 1));
    for (int i = 0; i < ns; i++) { s[i].lx = cx[sel[i]]; s[i].ly = cy[sel[i]]; s[i].score = cs[sel[i]]; }
    qsort(s, (size_t)ns, sizeof(selkp), cmp_yx);
    uint8_t* blur = (uint8_t*)malloc((size_t)w * h);
    ref_blur(lev, w, h, w, blur, w);
    for (int i = 0; i < ns; i++) {
      ref_keypoint* k = &kps[total + i];
      int32_t m10, m01;
      ref_moments(lev, w, s[i].lx, s[i].ly, &m10, &m01);
      k->x = (float)s[i].lx * p->scale[l];
      k->y = (float)s[i].ly * p->scale[l];
      k->angle_deg = ref_angle_deg(m10, m01);
      k->lx = (uint16_t)s[i].lx; k->ly = (uint16_t)s[i].ly;
      k->level = (uint8_t)l; k->response = (uint8_t)(s[i].score - 1);
      k->reserved = 0;
      ref_descriptor(blur, w, s[i].lx, s[i].ly, m10, m01, desc + (size_t)(total + i) * 32);
    }
    total += ns;
    counts[l + 1] = total;
    free(blur); free(s); free(kx); free(cx); free(M);
    off += (int64_t)w * h;
  }
  free(pyr);
  return total;
}

int ref_orb_extract(const ref_params* p, const uint8_t* img, int pitch, ref_keypoint* kps,
                    uint8_t* desc, int32_t* counts) {
  return ref_orb_extract_mode(p, img, pitch, 0, kps, desc, counts);
}

/* ---------------------------------------------------------------- O9 / O10 */
int32_t ref_hamming(const uint8_t* a, const uint8_t* b) {
  int d = 0;
  for (int i = 0; i < 32; i++) {
    uint8_t x = a[i] ^ b[i];
    for (int j = 0; j < 8; j++) d += (x >> j) & 1;
  }
  return d;
}

/* ORB-SLAM SearchByProjection (local map points) [ext], the paper's "search local
 * points": window + level gate + taken mask -> Hamming top-2 by (d, k) ->
 * d <= th and (levels differ or den*d1 <= num*d2); dedup keeps min (d, q) (S8c O9). */
void ref_match_window(const ref_params* p, int F, const ref_keypoint* kps, const uint8_t* desc,
                      const int32_t* counts, const uint8_t* taken, int nq, const ref_query* q,
                      const uint8_t* qdesc, int th, int num, int den, int dedup, ref_match* out) {
  int L = p->n_levels, cap = p->kp_capacity;
  for (int i = 0; i < nq; i++) {
    int d1 = 256, d2 = 256, k1 = -1, k2 = -1;
    int f = q[i].frame;
    if (f >= 0 && f < F) {
      int n = counts[f * (L + 1) + L];
      for (int k = 0; k < n; k++) {
        const ref_keypoint* kp = &kps[(size_t)f * cap + k];
        if (kp->level < q[i].pred_level - 1 || kp->level > q[i].pred_level) continue;
        if (taken && taken[(size_t)f * cap + k]) continue;
        float dx = kp->x - q[i].u, dy = kp->y - q[i].v;
        if (!(fabsf(dx) < q[i].radius && fabsf(dy) < q[i].radius)) continue;
        int d = ref_hamming(qdesc + (size_t)i * 32, desc + ((size_t)f * cap + k) * 32);
        /* keep the two smallest (d, k); k increases so ties keep the earlier k */
        if (d < d1) { d2 = d1; k2 = k1; d1 = d; k1 = k; }
        else if (d < d2) { d2 = d; k2 = k; }
      }
    }
    int accept = 0;
    if (k1 >= 0 && d1 <= th) {
      int lev1 = kps[(size_t)f * cap + k1].level;
      int lev2 = k2 >= 0 ? kps[(size_t)f * cap + k2].level : -1;
      if (lev1 != lev2 || den * d1 <= num * d2) accept = 1;
    }
    out[i].idx = accept ? k1 : -1;
    out[i].dist = d1;
    out[i].dist2 = d2;
  }
  if (!dedup) return;
  /* winner[f][k] = the claimant query with the smallest (dist, query index) */
  int* winner = (int*)malloc(sizeof(int) * (size_t)(F > 0 ? F : 1) * (size_t)cap);
  for (size_t t = 0; t < (size_t)F * cap; t++) winner[t] = -1;
  for (int i = 0; i < nq; i++) {
    if (out[i].idx < 0) continue;
    size_t slot = (size_t)q[i].frame * cap + out[i].idx;
    int w = winner[slot];
    if (w < 0 || out[i].dist < out[w].dist || (out[i].dist == out[w].dist && i < w)) winner[slot] = i;
  }
  for (int i = 0; i < nq; i++) {
    if (out[i].idx < 0) continue;
    if (winner[(size_t)q[i].frame * cap + out[i].idx] != i) out[i].idx = -1;
  }
  free(winner);
}

/* Brute force keypoint -> map (ORB-SLAM relocalisation thresholds [ext], S8c O10):
 * top-2 by (d, m); accept iff d1 <= th and den*d1 < num*d2. */
void ref_match_brute(const ref_params* p, int F, const uint8_t* desc, const int32_t* counts, int n_map,
                     const uint8_t* map_desc, int th, int num, int den, int k0, int k1,
                     ref_match* out) {
  int L = p->n_levels, cap = p->kp_capacity;
  for (int f = 0; f < F; f++) {
    int n = counts[f * (L + 1) + L];
    for (int k = k0; k < k1 && k < cap; k++) {
      ref_match* o = &out[(size_t)f * cap + k];
      o->idx = -1; o->dist = 256; o->dist2 = 256;
      if (k >= n) continue;
      const uint8_t* a = desc + ((size_t)f * cap + k) * 32;
      int d1 = 256, d2 = 256, m1 = -1;
      for (int m = 0; m < n_map; m++) {
        int d = ref_hamming(a, map_desc + (size_t)m * 32);
        if (d < d1) { d2 = d1; d1 = d; m1 = m; }
        else if (d < d2) { d2 = d; }
      }
      o->dist = d1; o->dist2 = d2;
      if (m1 >= 0 && d1 <= th && den * d1 < num * d2) o->idx = m1;
    }
  }
}

/* --------------------------------------------------------- O11 projection */
/* ORB-SLAM3 Frame::isInFrustum + MapPoint::PredictScale + ORBmatcher::RadiusByViewingCos
 * [ext]: the per-map-point step of "search local points" (§4.2.1) before the
 * windowed match (O9).  f32 throughout, every operation rounded once in the order written
 * (built with -ffp-contract=off; sums left to right).  Readings (DESIGN.md §3 item 11):
 * the predicted level is the smallest n in [0, L-1] with ratio <= scale[n] (the f32 scale
 * chain of O0), i.e. ceil(log(ratio)/log(sf)) clamped, decided by comparisons instead of a
 * libm log; radius = f32(f32(rv * th) * scale[level]) with rv = 2.5 if viewCos > 0.998
 * else 4.0; viewing-cosine limit 0.5; distance gate [0.8*min_dist, 1.2*max_dist]. */
static float dot3(const float* a, const float* b) {
  float s = a[0] * b[0];
  s = s + a[1] * b[1];
  s = s + a[2] * b[2];
  return s;
}

void ref_project_points(const ref_params* p, int F, const ref_camera* cams, int n, const ref_map_point* pts,
                        const int32_t* point_frame, float th, ref_query* out) {
  int L = p->n_levels;
  for (int i = 0; i < n; i++) {
    ref_query* o = &out[i];
    int f = point_frame[i];
    o->frame = f; o->u = 0.0f; o->v = 0.0f; o->pred_level = -1; o->radius = 0.0f;
    if (f < 0 || f >= F) continue;
    const ref_camera* c = &cams[f];
    const float* P = pts[i].pos;
    float pc[3];
    for (int r = 0; r < 3; r++) pc[r] = dot3(&c->R[3 * r], P) + c->t[r];
    if (pc[2] < 0.0f) continue;                          /* behind the camera */
    float u = c->fx * pc[0] / pc[2] + c->cx;              /* Pinhole::project */
    float v = c->fy * pc[1] / pc[2] + c->cy;
    if (u < c->min_x || u > c->max_x) continue;
    if (v < c->min_y || v > c->max_y) continue;
    float po[3] = {P[0] - c->ow[0], P[1] - c->ow[1], P[2] - c->ow[2]};
    float dist = sqrtf(dot3(po, po));
    float min_d = 0.8f * pts[i].min_dist, max_d = 1.2f * pts[i].max_dist;
    if (dist < min_d || dist > max_d) continue;
    float view_cos = dot3(po, pts[i].normal) / dist;
    if (view_cos < 0.5f) continue;
    float ratio = pts[i].max_dist / dist;                 /* PredictScale */
    int level = L - 1;
    for (int l = 0; l < L; l++)
      if (ratio <= p->scale[l]) { level = l; break; }
    float rv = view_cos > 0.998f ? 2.5f : 4.0f;           /* RadiusByViewingCos */
    float r = rv * th;
    o->u = u; o->v = v; o->pred_level = level; o->radius = r * p->scale[level];
  }
}

/* ------------------------------------------------------------- O12 stereo */
/* ORB-SLAM2 Frame::ComputeStereoMatches [ext] (the stereo tracking input of P:L163/L246;
 * SURVEY §8(f) F1), step by step in ORB-SLAM's order:
 *  1. every right keypoint iR is listed on rows floor(y - r) .. ceil(y + r), r = 2*scale[oct];
 *  2. per left keypoint: candidates = the list of row (int)vL, in iR order; keep those on
 *     octaves [oct-1, oct+1] with uL - maxD <= uR <= uL (maxD = bf/b, minD = 0); best =
 *     first minimum Hamming distance below TH_HIGH = 100;
 *  3. if best < (TH_HIGH + TH_LOW)/2 = 75: 11x11 SAD of the left window (centre-subtracted)
 *     against right windows at scaleduR0 + inc, inc in [-5, 5] (centre-subtracted), on the
 *     octave's pyramid level; rounded coordinates round(v * invScale[oct]) (half away from
 *     zero); skip if iniu = scaleduR0 < 0 or endu = scaleduR0 + 11 >= level width (ORB-SLAM's
 *     check, literally); first minimum SAD; reject inc = +-5; parabola
 *     deltaR = (d1 - d3) / (2 (d1 + d3 - 2 d2)), reject |deltaR| > 1;
 *     uR = scale[oct] * ((float)scaleduR0 + (float)inc + deltaR); disparity = uL - uR,
 *     accept 0 <= disparity < maxD (<= 0 -> 0.01, uR = uL - 0.01 in double); depth = bf/disparity;
 *  4. outliers: median = the SAD of element size/2 of the accepted (SAD, iL) sorted
 *     ascending; reject every accepted match with SAD >= 1.5f*1.4f*median.
 * Keypoint indices are the canonical (level, ly, lx) order.  SADs are exact integers. */
static const uint8_t* ref_level_ptr(const ref_params* p, const uint8_t* pyr, int l) {
  int64_t off = 0;
  for (int i = 0; i < l; i++) off += (int64_t)p->level_w[i] * p->level_h[i];
  return pyr + off;
}

static int cmp_pair(const void* a, const void* b) {
  const int32_t* x = (const int32_t*)a;
  const int32_t* y = (const int32_t*)b;
  if (x[0] != y[0]) return x[0] < y[0] ? -1 : 1;
  return x[1] < y[1] ? -1 : (x[1] > y[1]);
}

void ref_stereo_match(const ref_params* p, const uint8_t* left, const uint8_t* right, int pitch,
                      const ref_keypoint* kl, const uint8_t* dl, const int32_t* cl,
                      const ref_keypoint* kr, const uint8_t* dr, const int32_t* cr, float bf, float b,
                      float* uright, float* depth, int32_t* sad) {
  const int L = p->n_levels, H = p->height;
  const int nl = cl[L], nr = cr[L];
  int64_t pb = ref_pyramid_bytes(p);
  uint8_t* pyl = (uint8_t*)malloc((size_t)pb);
  uint8_t* pyr = (uint8_t*)malloc((size_t)pb);
  ref_pyramid(p, left, pitch, pyl);
  ref_pyramid(p, right, pitch, pyr);
  /* 1. row lists */
  int* rcount = (int*)calloc((size_t)H, sizeof(int));
  int* rstart = (int*)malloc(sizeof(int) * (size_t)(H + 1));
  for (int i = 0; i < nr; i++) {
    float ky = kr[i].y, r = 2.0f * p->scale[kr[i].level];
    int maxr = (int)ceilf(ky + r), minr = (int)floorf(ky - r);
    for (int yi = minr; yi <= maxr; yi++)
      if (yi >= 0 && yi < H) rcount[yi]++;
  }
  rstart[0] = 0;
  for (int y = 0; y < H; y++) rstart[y + 1] = rstart[y] + rcount[y];
  int* rlist = (int*)malloc(sizeof(int) * (size_t)(rstart[H] > 0 ? rstart[H] : 1));
  memset(rcount, 0, sizeof(int) * (size_t)H);
  for (int i = 0; i < nr; i++) {
    float ky = kr[i].y, r = 2.0f * p->scale[kr[i].level];
    int maxr = (int)ceilf(ky + r), minr = (int)floorf(ky - r);
    for (int yi = minr; yi <= maxr; yi++) {
      if (yi < 0 || yi >= H) continue;
      rlist[rstart[yi] + rcount[yi]++] = i;
    }
  }
  const float minD = 0.0f, maxD = bf / b;
  const int thOrb = (100 + 50) / 2;
  int32_t* acc = (int32_t*)malloc(sizeof(int32_t) * 2 * (size_t)(nl > 0 ? nl : 1));
  int nacc = 0;
  for (int iL = 0; iL < nl; iL++) {
    uright[iL] = -1.0f; depth[iL] = -1.0f; sad[iL] = -1;
    const ref_keypoint* k = &kl[iL];
    const int lev = k->level;
    const float vL = k->y, uL = k->x;
    const int row = (int)vL;
    if (row < 0 || row >= H || rcount[row] == 0) continue;
    const float minU = uL - maxD, maxU = uL - minD;
    if (maxU < 0) continue;
    int bestDist = 100, bestIdxR = 0;
    for (int c = 0; c < rcount[row]; c++) {
      int iR = rlist[rstart[row] + c];
      const ref_keypoint* q = &kr[iR];
      if (q->level < lev - 1 || q->level > lev + 1) continue;
      const float uR = q->x;
      if (uR >= minU && uR <= maxU) {
        int dist = ref_hamming(dl + (size_t)iL * 32, dr + (size_t)iR * 32);
        if (dist < bestDist) { bestDist = dist; bestIdxR = iR; }
      }
    }
    if (bestDist >= thOrb) continue;
    /* 3. sub-pixel refinement by SAD on the octave's level */
    const float uR0 = kr[bestIdxR].x;
    const float sf = p->inv_scale[lev];
    const int su = (int)roundf(uL * sf), sv = (int)roundf(vL * sf), su0 = (int)roundf(uR0 * sf);
    const int w = 5, Lr = 5;
    const int lw = p->level_w[lev];
    const uint8_t* IL = ref_level_ptr(p, pyl, lev);
    const uint8_t* IR = ref_level_ptr(p, pyr, lev);
    const int iniu = su0 + Lr - w, endu = su0 + Lr + w + 1;
    if (iniu < 0 || endu >= lw) continue;
    float vd[11];
    float best = 3.0e38f;
    int bestinc = 0;
    const int cL = IL[(size_t)sv * lw + su];
    for (int inc = -Lr; inc <= Lr; inc++) {
      const int cR = IR[(size_t)sv * lw + su0 + inc];
      double s1 = 0.0;
      for (int dy = -w; dy <= w; dy++)
        for (int dx = -w; dx <= w; dx++) {
          int a = IL[(size_t)(sv + dy) * lw + su + dx] - cL;
          int bb = IR[(size_t)(sv + dy) * lw + su0 + inc + dx] - cR;
          s1 += fabs((double)(a - bb));
        }
      float dist = (float)s1;
      if (dist < best) { best = dist; bestinc = inc; }
      vd[Lr + inc] = dist;
    }
    if (bestinc == -Lr || bestinc == Lr) continue;
    const float d1 = vd[Lr + bestinc - 1], d2 = vd[Lr + bestinc], d3 = vd[Lr + bestinc + 1];
    const float deltaR = (d1 - d3) / (2.0f * (d1 + d3 - 2.0f * d2));
    if (deltaR < -1 || deltaR > 1) continue;
    float bestuR = p->scale[lev] * ((float)su0 + (float)bestinc + deltaR);
    float disparity = uL - bestuR;
    if (disparity >= minD && disparity < maxD) {
      if (disparity <= 0) {
        disparity = 0.01;
        bestuR = (float)((double)uL - 0.01);
      }
      depth[iL] = bf / disparity;
      uright[iL] = bestuR;
      sad[iL] = (int32_t)best;
      acc[2 * nacc] = (int32_t)best;
      acc[2 * nacc + 1] = iL;
      nacc++;
    }
  }
  /* 4. outlier cut */
  if (nacc > 0) {
    qsort(acc, (size_t)nacc, 2 * sizeof(int32_t), cmp_pair);
    const int median = acc[2 * (nacc / 2)];
    const float thDist = 1.5f * 1.4f * (float)median;
    for (int i = nacc - 1; i >= 0; i--) {
      if ((float)acc[2 * i] < thDist) break;
      uright[acc[2 * i + 1]] = -1.0f;
      depth[acc[2 * i + 1]] = -1.0f;
    }
  }
  free(acc); free(rlist); free(rstart); free(rcount); free(pyl); free(pyr);
}

/* ------------------------------------------- O13 frame-to-frame projection matching */
/* ORB-SLAM2/3 ORBmatcher::SearchByProjection(CurrentFrame, LastFrame, th, bMono) as called by
 * Tracking::TrackWithMotionModel [ext]: the "ORB-Matching" step of the paper's tracking-time
 * breakdown (§5, Fig. 8: "feature extraction (ORB-Extraction), feature matching
 * (ORB-Matching), pose prediction, and finally search local point").  SURVEY §8(f) F2;
 * readings in DESIGN.md §3 item 14.  Per frame f, its last-frame points
 * [pt_off[f], pt_off[f+1]) (a map point seen in the previous frame: world position, the
 * previous keypoint's octave and angle), in ORB-SLAM's order:
 *  1. Pc = R*Pw + t (O11's arithmetic); skip if Pc.z < 0; u = fx*X/Z + cx, v = fy*Y/Z + cy;
 *     skip if outside [min_x, max_x] x [min_y, max_y];
 *  2. radius = f32(th * scale[octave]); stereo direction (only when mb > 0 and last cameras
 *     are given): tlc = R_last * ow_cur + t_last, forward iff tlc.z > mb, backward iff
 *     -tlc.z > mb; level gate: forward [octave, L-1], backward [0, octave], else
 *     [octave-1, octave+1] (GetFeaturesInArea(u, v, r, minLevel, maxLevel));
 *  3. candidates: keypoints of frame f in the gate with |x-u| < r and |y-v| < r (f32), not
 *     taken; best / second by (Hamming, keypoint index); accept iff best <= th_high
 *     (TH_HIGH = 100; no ratio test in this matcher);
 *  4. reading of ORB-SLAM's sequential claim (a keypoint matched by an earlier point is
 *     skipped by later ones): every point is evaluated independently, then a keypoint claimed
 *     by several accepted points keeps the min (distance, point index) (as O9);
 *  5. rotation consistency (mbCheckOrientation): rot = angle_last - angle_cur (f32), +360 if
 *     negative, bin = roundf(rot * f32(1/30)) (HISTO_LENGTH = 30, factor = 1.0f/HISTO_LENGTH,
 *     literally), 30 -> 0; ComputeThreeMaxima (strict >, earlier bin wins ties; drop the 2nd /
 *     3rd maximum when below 0.1f * max1); matches in other bins are removed;
 *  6. if min_matches > 0 and the frame kept fewer than min_matches matches, the whole frame is
 *     matched again from step 1 with radius factor 2*th (TrackWithMotionModel's retry), and
 *     the second result stands.
 * Output per point: idx = keypoint index or -1, dist / dist2 = best / second distance of the
 * last pass that evaluated it (256 = none).  Points whose octave is outside [0, L-1] have no
 * candidates. */
#define HISTO_LENGTH 30

static void lf_three_maxima(const int* hist, int* ind1, int* ind2, int* ind3) {
  int max1 = 0, max2 = 0, max3 = 0;
  *ind1 = *ind2 = *ind3 = -1;
  for (int i = 0; i < HISTO_LENGTH; i++) {
    int s = hist[i];
    if (s > max1) { max3 = max2; max2 = max1; max1 = s; *ind3 = *ind2; *ind2 = *ind1; *ind1 = i; }
    else if (s > max2) { max3 = max2; max2 = s; *ind3 = *ind2; *ind2 = i; }
    else if (s > max3) { max3 = s; *ind3 = i; }
  }
  if ((float)max2 < 0.1f * (float)max1) { *ind2 = -1; *ind3 = -1; }
  else if ((float)max3 < 0.1f * (float)max1) { *ind3 = -1; }
}

int ref_lf_rot_bin(float angle_last, float angle_cur) {
  const float factor = 1.0f / HISTO_LENGTH;
  float rot = angle_last - angle_cur;
  if (rot < 0.0f) rot = rot + 360.0f;
  float t = rot * factor;
  int bin = (int)roundf(t);
  if (bin == HISTO_LENGTH) bin = 0;
  return bin;
}

/* one pass over frame f's points with window factor th; returns the kept match count */
static int lf_frame_pass(const ref_params* p, int f, const ref_camera* c, int dir, const ref_keypoint* kps,
                         const uint8_t* desc, const int32_t* counts, const uint8_t* taken, int i0, int i1,
                         const ref_frame_point* pts, const uint8_t* pdesc, float th, int th_high,
                         int check_orientation, ref_match* out, int* winner) {
  int L = p->n_levels, cap = p->kp_capacity;
  int n = counts[f * (L + 1) + L];
  const ref_keypoint* fk = &kps[(size_t)f * cap];
  for (int i = i0; i < i1; i++) {
    out[i].idx = -1; out[i].dist = 256; out[i].dist2 = 256;
    int o = pts[i].octave;
    if (o < 0 || o >= L) continue;
    const float* P = pts[i].pos;
    float pc[3];
    for (int r = 0; r < 3; r++) pc[r] = dot3(&c->R[3 * r], P) + c->t[r];
    if (pc[2] < 0.0f) continue;
    float u = c->fx * pc[0] / pc[2] + c->cx;
    float v = c->fy * pc[1] / pc[2] + c->cy;
    if (u < c->min_x || u > c->max_x) continue;
    if (v < c->min_y || v > c->max_y) continue;
    float radius = th * p->scale[o];
    int lmin, lmax;
    if (dir == 1) { lmin = o; lmax = L - 1; }
    else if (dir == 2) { lmin = 0; lmax = o; }
    else { lmin = o - 1; lmax = o + 1; }
    int d1 = 256, d2 = 256, k1 = -1;
    for (int k = 0; k < n; k++) {
      if (fk[k].level < lmin || fk[k].level > lmax) continue;
      if (taken && taken[(size_t)f * cap + k]) continue;
      float dx = fk[k].x - u, dy = fk[k].y - v;
      if (!(fabsf(dx) < radius && fabsf(dy) < radius)) continue;
      int d = ref_hamming(pdesc + (size_t)i * 32, desc + ((size_t)f * cap + k) * 32);
      if (d < d1) { d2 = d1; d1 = d; k1 = k; }
      else if (d < d2) { d2 = d; }
    }
    out[i].dist = d1; out[i].dist2 = d2;
    if (k1 >= 0 && d1 <= th_high) out[i].idx = k1;
  }
  /* step 4: dedup, min (distance, point index) per keypoint */
  for (int k = 0; k < cap; k++) winner[k] = -1;
  for (int i = i0; i < i1; i++) {
    int k = out[i].idx;
    if (k < 0) continue;
    int w = winner[k];
    if (w < 0 || out[i].dist < out[w].dist || (out[i].dist == out[w].dist && i < w)) winner[k] = i;
  }
  for (int i = i0; i < i1; i++)
    if (out[i].idx >= 0 && winner[out[i].idx] != i) out[i].idx = -1;
  /* step 5: rotation consistency */
  if (check_orientation) {
    int hist[HISTO_LENGTH] = {0};
    for (int i = i0; i < i1; i++)
      if (out[i].idx >= 0) hist[ref_lf_rot_bin(pts[i].angle_deg, fk[out[i].idx].angle_deg)]++;
    int a, b, d;
    lf_three_maxima(hist, &a, &b, &d);
    for (int i = i0; i < i1; i++) {
      if (out[i].idx < 0) continue;
      int bin = ref_lf_rot_bin(pts[i].angle_deg, fk[out[i].idx].angle_deg);
      if (bin != a && bin != b && bin != d) out[i].idx = -1;
    }
  }
  int kept = 0;
  for (int i = i0; i < i1; i++) kept += out[i].idx >= 0;
  return kept;
}

void ref_match_last_frame(const ref_params* p, int F, const ref_camera* cams, const ref_camera* last_cams, float mb,
                          const ref_keypoint* kps, const uint8_t* desc, const int32_t* counts, const uint8_t* taken,
                          const int32_t* pt_off, const ref_frame_point* pts, const uint8_t* pdesc, float th,
                          int th_high, int check_orientation, int min_matches, ref_match* out, int32_t* n_matches) {
  int cap = p->kp_capacity;
  int* winner = (int*)malloc(sizeof(int) * (size_t)(cap > 0 ? cap : 1));
  for (int f = 0; f < F; f++) {
    const ref_camera* c = &cams[f];
    int dir = 0;
    if (mb > 0.0f && last_cams) {
      const ref_camera* cl = &last_cams[f];
      float tz = dot3(&cl->R[6], c->ow) + cl->t[2];
      if (tz > mb) dir = 1;
      else if (-tz > mb) dir = 2;
    }
    int kept = lf_frame_pass(p, f, c, dir, kps, desc, counts, taken, pt_off[f], pt_off[f + 1], pts, pdesc, th,
                             th_high, check_orientation, out, winner);
    if (min_matches > 0 && kept < min_matches)
      kept = lf_frame_pass(p, f, c, dir, kps, desc, counts, taken, pt_off[f], pt_off[f + 1], pts, pdesc,
                           2.0f * th, th_high, check_orientation, out, winner);
    if (n_matches) n_matches[f] = kept;
  }
  free(winner);
}
