// k_pyramid.cu -- S1: image pyramid, level l = bilinear resize of level l-1 (DESIGN.md §3 O1).
//
// Fixed-point definition (bit-exact INTER_LINEAR_EXACT semantics): per destination column
// the host precomputes (x0, wx1, x1-x0) with wx1 = rne(frac * 256); then
//   out = ((256-wy1)*(wx0*s[y0][x0] + wx1*s[y0][x1]) + wy1*(...row y1...) + 2^15) >> 16.
//
// One launch per level (levels are chained), all frames at once, 128x32 output tiles: the
// CTA stages the source rectangle the tile reads (<= 48 x 208 B) in shared memory with
// 16-byte coalesced loads and writes 4 output pixels per thread with one 32-bit store.
// The chain runs on the main stream while level 0's FAST and distribution run on a second
// stream (ss_api.cpp), so its latency is off the critical path.
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int TW = 128, TH = 32, PT = 256;
constexpr int SRC_ROWS = 48, SRC_PITCH = 208;  // >= TH*scale+2 rows, >= TW*scale+2+15 (aligned) cols

__global__ void __launch_bounds__(PT) pyramid_level_kernel(Geom g, int l, FrameSrc src, const uint32_t* __restrict__ xtab,
                                                           const uint32_t* __restrict__ ytab) {
  pdl_wait();
  pdl_trigger();
  __shared__ __align__(16) uint8_t s_src[SRC_ROWS * SRC_PITCH];
  __shared__ uint32_t s_x[TW];
  const int f = blockIdx.z;
  const int dw = g.w[l], dh = g.h[l];
  const int tx0 = blockIdx.x * TW, ty0 = blockIdx.y * TH;
  const int tx1 = min(tx0 + TW, dw), ty1 = min(ty0 + TH, dh);
  const uint8_t* s;
  int sp;
  if (l == 1) {
    s = src.frames + (int64_t)f * src.stride;
    sp = src.pitch;
  } else {
    s = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l - 1];
    sp = g.pitch[l - 1];
  }
  // source rectangle: rows [sy0, sy1], columns [sx0, sx1] (sx0 aligned down to 16)
  const uint32_t cy0 = __ldg(ytab + ty0), cy1 = __ldg(ytab + ty1 - 1);
  const int sy0 = (int)(cy0 & 0xFFFF), sy1 = (int)(cy1 & 0xFFFF) + (int)(cy1 >> 25);
  const uint32_t cx0 = __ldg(xtab + tx0), cx1 = __ldg(xtab + tx1 - 1);
  const int sx0 = (int)(cx0 & 0xFFFF) & ~15, sx1 = (int)(cx1 & 0xFFFF) + (int)(cx1 >> 25);
  // columns past the level edge reuse the last column's coefficients (computed, never stored)
  if (threadIdx.x < TW) s_x[threadIdx.x] = __ldg(xtab + min(tx0 + (int)threadIdx.x, dw - 1));
  const int nrows = sy1 - sy0 + 1;
  if ((sp & 15) == 0 && (reinterpret_cast<uintptr_t>(s) & 15) == 0) {
    const int nch = (sx1 - sx0 + 16) >> 4;
    for (int i = threadIdx.x; i < nrows * nch; i += PT) {
      const int r = i / nch, c = i - r * nch;
      *reinterpret_cast<uint4*>(s_src + r * SRC_PITCH + 16 * c) =
          __ldg(reinterpret_cast<const uint4*>(s + (int64_t)(sy0 + r) * sp + sx0) + c);
    }
  } else {
    const int ncol = sx1 - sx0 + 1;
    for (int i = threadIdx.x; i < nrows * ncol; i += PT) {
      const int r = i / ncol, c = i - r * ncol;
      s_src[r * SRC_PITCH + c] = __ldg(s + (int64_t)(sy0 + r) * sp + sx0 + c);
    }
  }
  __syncthreads();
  uint8_t* d = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
  const int dp = g.pitch[l];
  const int gx = (threadIdx.x & 31) * 4;  // 32 threads x 4 px = one 128-px tile row
  for (int y = ty0 + (threadIdx.x >> 5); y < ty1; y += PT / 32) {
    const uint32_t cy = __ldg(ytab + y);
    const int y0 = (int)(cy & 0xFFFF) - sy0, wy1 = (int)((cy >> 16) & 0x1FF), y1 = y0 + (int)(cy >> 25);
    const uint8_t* r0 = s_src + y0 * SRC_PITCH - sx0;
    const uint8_t* r1 = s_src + y1 * SRC_PITCH - sx0;
    uint32_t packed = 0;
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const uint32_t cx = s_x[gx + q];
      const int x0 = (int)(cx & 0xFFFF), wx1 = (int)((cx >> 16) & 0x1FF), x1 = x0 + (int)(cx >> 25);
      const int wx0 = 256 - wx1;
      const int h0 = wx0 * r0[x0] + wx1 * r0[x1];
      const int h1 = wx0 * r1[x0] + wx1 * r1[x1];
      packed |= (uint32_t)(((256 - wy1) * h0 + wy1 * h1 + (1 << 15)) >> 16) << (8 * q);
    }
    const int x = tx0 + gx;
    if (x >= tx1) continue;
    uint8_t* drow = d + (int64_t)y * dp;
    if (x + 4 <= tx1) {
      *reinterpret_cast<uint32_t*>(drow + x) = packed;  // pitch is a multiple of 16
    } else {
      for (int q = 0; x + q < tx1; q++) drow[x + q] = (uint8_t)(packed >> (8 * q));
    }
  }
}

}  // namespace

// Whether every 128x32 tile's source rectangle fits the kernel's shared-memory staging.
bool pyramid_tiles_fit(int dst_w, int dst_h, const uint32_t* xt, const uint32_t* yt) {
  for (int ty0 = 0; ty0 < dst_h; ty0 += TH) {
    const int ty1 = (ty0 + TH < dst_h ? ty0 + TH : dst_h) - 1;
    const int rows = (int)(yt[ty1] & 0xFFFF) + (int)(yt[ty1] >> 25) - (int)(yt[ty0] & 0xFFFF) + 1;
    if (rows > SRC_ROWS) return false;
  }
  for (int tx0 = 0; tx0 < dst_w; tx0 += TW) {
    const int tx1 = (tx0 + TW < dst_w ? tx0 + TW : dst_w) - 1;
    const int cols = (int)(xt[tx1] & 0xFFFF) + (int)(xt[tx1] >> 25) - ((int)(xt[tx0] & 0xFFFF) & ~15) + 1;
    if (((cols + 15) & ~15) > SRC_PITCH) return false;
  }
  return true;
}

cudaError_t launch_pyramid_level(const Geom& g, int l, int n_frames, FrameSrc src, const uint32_t* xytab, PyrTabs tabs,
                                 cudaStream_t s) {
  dim3 grid((g.w[l] + TW - 1) / TW, (g.h[l] + TH - 1) / TH, n_frames);
  cudaError_t e = launch_pdl(pyramid_level_kernel, grid, dim3(PT), 0, s, g, l, src, xytab + tabs.xoff[l],
                             xytab + tabs.yoff[l]);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_pyramid(const Geom& g, int n_frames, FrameSrc src, const uint32_t* xytab, PyrTabs tabs,
                           cudaStream_t s) {
  for (int l = 1; l < g.L; l++) {
    dim3 grid((g.w[l] + TW - 1) / TW, (g.h[l] + TH - 1) / TH, n_frames);
    cudaError_t e = launch_pdl(pyramid_level_kernel, grid, dim3(PT), 0, s, g, l, src, xytab + tabs.xoff[l], xytab + tabs.yoff[l]);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace ss
