// match_common.cuh -- device helpers shared by the matchers (k_match.cu, k_lastframe.cu):
// 256-bit Hamming distance, the per-(frame, level, row) keypoint row index, packed top-2.
#pragma once
#include "ss_internal.h"

namespace ss {

__device__ __forceinline__ int hamming256(const uint4 a0, const uint4 a1, const uint4 b0, const uint4 b1) {
  return __popc(a0.x ^ b0.x) + __popc(a0.y ^ b0.y) + __popc(a0.z ^ b0.z) + __popc(a0.w ^ b0.w) +
         __popc(a1.x ^ b1.x) + __popc(a1.y ^ b1.y) + __popc(a1.z ^ b1.z) + __popc(a1.w ^ b1.w);
}

__host__ __device__ __forceinline__ int row_off(const Geom& g, int l) {  // start of level l in a frame's row index
  return l < g.L ? g.row_off[l] : g.row_off[g.L - 1] + g.h[g.L - 1] + 1;
}

// A frame's segment of the global keypoint index (stride match_index_stride): the row index
// ([row_off(g, L)] entries), then from lx_off(g) (16-B aligned) every keypoint's lx as u16 in
// canonical order, which the window matcher prefilters eight at a time.
__host__ __device__ __forceinline__ int lx_off(const Geom& g) { return (row_off(g, g.L) + 7) & ~7; }

// Row-index entries owned by slot k of one frame (keypoints in canonical (level, ly, lx)
// order): ri_l[r] = index of the first keypoint of level l with ly >= r, r in [0, h_l].
// Slot k < L also fills the rows of an empty level k.  fk = the frame's keypoints, cnt = its
// prefix counts, fr = its row index.
__device__ __forceinline__ void rowidx_fill(const Geom& g, const ss_keypoint* __restrict__ fk,
                                            const int32_t* __restrict__ cnt, uint16_t* __restrict__ fr, int k,
                                            uint16_t* __restrict__ flx = nullptr) {
  const int L = g.L;
  if (k < L && cnt[k] == cnt[k + 1]) {  // empty level k: every row points at its (empty) range
    uint16_t* ri = fr + row_off(g, k);
    for (int r = 0; r <= g.h[k]; r++) ri[r] = (uint16_t)cnt[k];
  }
  if (k >= cnt[L]) return;
  const ss_keypoint kp = fk[k];
  const int l = kp.level, ly = kp.ly;
  if (flx) flx[k] = kp.lx;
  uint16_t* ri = fr + row_off(g, l);
  const int prev = k > cnt[l] ? (int)fk[k - 1].ly : -1;
  for (int r = prev + 1; r <= ly; r++) ri[r] = (uint16_t)k;
  if (k == cnt[l + 1] - 1)
    for (int r = ly + 1; r <= g.h[l]; r++) ri[r] = (uint16_t)(k + 1);
}

// Rows [rlo, rhi) of level l (clamped to [0, h_l]) that can hold |y - v| < r, widened by one
// row each side; the exact test on each keypoint decides, so the bounds only need to be a
// superset: (v -+ r) * f32(1/scale) is within 1e-3 rows of the real quotient (rows < 2048),
// far inside the one-row margin that also covers y = f32(ly * scale) rounding.
__device__ __forceinline__ void window_rows(const Geom& g, int l, float v, float r, int* rlo, int* rhi) {
  const float is_l = g.inv_scale[l];
  const int hl = g.h[l];
  *rlo = max(0, min(hl, (int)floorf(__fsub_rn(v, r) * is_l) - 1));
  *rhi = max(0, min(hl, (int)ceilf(__fadd_rn(v, r) * is_l) + 2));
}

// Columns [lo, hi] of level l (lo | hi << 16) that can hold |x - u| < r: floor / ceil of
// (u -+ r) / scale, widened by one column (a superset, as window_rows is for the rows); the
// exact f32 test decides.
__device__ __forceinline__ unsigned col_range(const Geom& g, int l, float u, float r) {  // lo | hi << 16
  const float is_l = g.inv_scale[l];
  const float lo = fminf(fmaxf(floorf(__fsub_rn(u, r) * is_l) - 1.0f, 0.0f), 65535.0f);
  const float hi = fminf(fmaxf(ceilf(__fadd_rn(u, r) * is_l) + 1.0f, 0.0f), 65535.0f);
  return (unsigned)lo | ((unsigned)hi << 16);
}

// top-2 of two packed (distance << 32 | index) pairs
__device__ __forceinline__ void merge_top2(unsigned long long& a1, unsigned long long& a2, unsigned long long b1,
                                           unsigned long long b2) {
  const unsigned long long lo = a1 < b1 ? a1 : b1, hi = a1 < b1 ? b1 : a1;
  const unsigned long long s2 = a2 < b2 ? a2 : b2;
  a1 = lo;
  a2 = hi < s2 ? hi : s2;
}

}  // namespace ss
