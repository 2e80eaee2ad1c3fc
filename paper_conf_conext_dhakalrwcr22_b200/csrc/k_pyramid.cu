// k_pyramid.cu -- S1: image pyramid, level l = bilinear resize of level l-1 (DESIGN.md §3 O1).
//
// Fixed-point definition (bit-exact INTER_LINEAR_EXACT semantics): per destination column
// the host precomputes (x0, wx1, x1-x0) with wx1 = rne(frac * 256); the kernel evaluates
//   out = ((256-wy1)*(wx0*s[y0][x0] + wx1*s[y0][x1]) + wy1*(...row y1...) + 2^15) >> 16.
// HBM-bound streaming kernel: each CTA stages nothing (source rows are read twice by
// neighbouring threads and hit L1), one byte out per thread, 4 output pixels per thread
// packed into one 32-bit store.
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int PX_PER_THREAD = 4;

__global__ void __launch_bounds__(256) pyramid_level_kernel(Geom g, int l, FrameSrc src,
                                                           const uint32_t* __restrict__ xtab,
                                                           const uint32_t* __restrict__ ytab) {
  const int f = blockIdx.z;
  const int dw = g.w[l], dh = g.h[l];
  const int y = blockIdx.y * blockDim.y + threadIdx.y;
  const int xb = (blockIdx.x * blockDim.x + threadIdx.x) * PX_PER_THREAD;
  if (y >= dh || xb >= dw) return;
  const uint8_t* s;
  int sp;
  if (l == 1) {
    s = src.frames + (int64_t)f * src.stride;
    sp = src.pitch;
  } else {
    s = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l - 1];
    sp = g.pitch[l - 1];
  }
  uint8_t* d = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l] + (int64_t)y * g.pitch[l];
  const uint32_t cy = __ldg(ytab + y);
  const int y0 = cy & 0xFFFF, wy1 = (cy >> 16) & 0x1FF, y1 = y0 + (int)(cy >> 25);
  const uint8_t* r0 = s + (int64_t)y0 * sp;
  const uint8_t* r1 = s + (int64_t)y1 * sp;
  uint32_t packed = 0;
#pragma unroll
  for (int i = 0; i < PX_PER_THREAD; i++) {
    const int x = xb + i;
    if (x < dw) {
      const uint32_t cx = __ldg(xtab + x);
      const int x0 = cx & 0xFFFF, wx1 = (cx >> 16) & 0x1FF, x1 = x0 + (int)(cx >> 25);
      const int wx0 = 256 - wx1;
      const int h0 = wx0 * __ldg(r0 + x0) + wx1 * __ldg(r0 + x1);
      const int h1 = wx0 * __ldg(r1 + x0) + wx1 * __ldg(r1 + x1);
      const int v = (256 - wy1) * h0 + wy1 * h1;
      packed |= (uint32_t)((v + (1 << 15)) >> 16) << (8 * i);
    }
  }
  if (xb + PX_PER_THREAD <= dw) {
    *reinterpret_cast<uint32_t*>(d + xb) = packed;  // pitch is a multiple of 16
  } else {
    for (int i = 0; xb + i < dw; i++) d[xb + i] = (uint8_t)(packed >> (8 * i));
  }
}

}  // namespace

cudaError_t launch_pyramid_level(const Geom& g, int level, int n_frames, FrameSrc src, const uint32_t* xtab,
                                 const uint32_t* ytab, cudaStream_t s) {
  dim3 block(32, 8);
  dim3 grid((g.w[level] + 32 * PX_PER_THREAD - 1) / (32 * PX_PER_THREAD), (g.h[level] + 7) / 8, n_frames);
  pyramid_level_kernel<<<grid, block, 0, s>>>(g, level, src, xtab, ytab);
  return cudaGetLastError();
}

}  // namespace ss
