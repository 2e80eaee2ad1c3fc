// k_pyramid.cu -- S1: image pyramid, level l = bilinear resize of level l-1 (DESIGN.md §3 O1).
//
// Fixed-point definition (bit-exact INTER_LINEAR_EXACT semantics): per destination column
// the host precomputes (x0, wx1, x1-x0) with wx1 = rne(frac * 256); then
//   out = ((256-wy1)*(wx0*s[y0][x0] + wx1*s[y0][x1]) + wy1*(...row y1...) + 2^15) >> 16.
//
// The chain level 1 -> ... -> level L-1 is latency-bound (7 dependent steps over ~1 MB per
// frame), so one launch builds every level of every frame, one CTA per (vertical strip,
// frame), entirely in shared memory: the CTA stages the level-0 columns its strip's
// dependency cone needs, then computes each level over the cone (its own strip widened by
// the source columns the next level reads) from the previous level in shared memory,
// writing only its own strip to HBM.  Strips are independent -- cone columns are recomputed
// by neighbours, never read from them -- so no inter-CTA synchronisation is needed.
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int PT = 1024;

__global__ void __launch_bounds__(PT) pyramid_strips_kernel(Geom g, FrameSrc src, const PyrStrip* __restrict__ strips,
                                                            const uint32_t* __restrict__ xytab, PyrTabs tabs,
                                                            int buf_bytes) {
  extern __shared__ __align__(16) uint8_t sm[];
  __shared__ PyrStrip st;
  const int f = blockIdx.y;
  if (threadIdx.x < (int)(sizeof(PyrStrip) / 4))
    reinterpret_cast<int32_t*>(&st)[threadIdx.x] = reinterpret_cast<const int32_t*>(strips + blockIdx.x)[threadIdx.x];
  __syncthreads();
  uint8_t* A = sm;               // level l-1 cone, staged columns [a, a + pa)
  uint8_t* Bf = sm + buf_bytes;  // level l cone
  // ---- stage the level-0 cone (all rows): columns [a, c1_0) with a = c0_0 rounded down to 16 ----
  int a = st.c0[0] & ~15;
  int pa = ((st.c1[0] - a) + 15) & ~15;  // staged pitch
  {
    const uint8_t* s0 = src.frames + (int64_t)f * src.stride;
    const int h = g.h[0];
    if ((src.pitch & 15) == 0 && (reinterpret_cast<uintptr_t>(s0) & 15) == 0) {
      const int nch = pa >> 4;
      for (int i = threadIdx.x; i < h * nch; i += PT) {
        const int r = i / nch, c = i - r * nch;
        *reinterpret_cast<uint4*>(A + r * pa + 16 * c) =
            __ldg(reinterpret_cast<const uint4*>(s0 + (int64_t)r * src.pitch + a) + c);
      }
    } else {
      const int wdt = st.c1[0] - a;
      for (int i = threadIdx.x; i < h * wdt; i += PT) {
        const int r = i / wdt, c = i - r * wdt;
        A[r * pa + c] = __ldg(s0 + (int64_t)r * src.pitch + a + c);
      }
    }
  }
  __syncthreads();
  for (int l = 1; l < g.L; l++) {
    const int c0 = st.c0[l], wdt = st.c1[l] - c0;
    const int pb = (wdt + 3) & ~3;
    const uint32_t* xtab = xytab + tabs.xoff[l];
    const uint32_t* ytab = xytab + tabs.yoff[l];
    const int hl = g.h[l];
    uint8_t* dst = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    const int dp = g.pitch[l];
    const int p0 = st.p0[l], p1 = st.p1[l];
    // thread = one column of the cone (coefficients loaded once), rows strided by the
    // number of column groups the CTA covers at once
    const int nx = wdt < PT ? wdt : PT;
    const int rstep = PT / nx;
    const int ty = threadIdx.x / nx;
    if (ty < rstep) {
      for (int xx = threadIdx.x - ty * nx; xx < wdt; xx += nx) {
        const int x = c0 + xx;
        const uint32_t cx = __ldg(xtab + x);
        const int x0 = (int)(cx & 0xFFFF) - a, wx1 = (int)((cx >> 16) & 0x1FF), x1 = x0 + (int)(cx >> 25);
        const int wx0 = 256 - wx1;
        const bool own = x >= p0 && x < p1;
        for (int y = ty; y < hl; y += rstep) {
          const uint32_t cy = __ldg(ytab + y);
          const int y0 = (int)(cy & 0xFFFF), wy1 = (int)((cy >> 16) & 0x1FF), y1 = y0 + (int)(cy >> 25);
          const uint8_t* r0 = A + y0 * pa;
          const uint8_t* r1 = A + y1 * pa;
          const int h0 = wx0 * r0[x0] + wx1 * r0[x1];
          const int h1 = wx0 * r1[x0] + wx1 * r1[x1];
          const int v = ((256 - wy1) * h0 + wy1 * h1 + (1 << 15)) >> 16;
          Bf[y * pb + xx] = (uint8_t)v;
          if (own) dst[(int64_t)y * dp + x] = (uint8_t)v;
        }
      }
    }
    __syncthreads();
    uint8_t* t = A;
    A = Bf;
    Bf = t;
    a = c0;
    pa = pb;
  }
}

}  // namespace

cudaError_t launch_pyramid(const Geom& g, int n_frames, FrameSrc src, const PyrStrip* strips, int n_strips,
                           const uint32_t* xytab, PyrTabs tabs, int buf_bytes, cudaStream_t s) {
  if (g.L < 2) return cudaSuccess;
  static bool attr_set = false;
  if (!attr_set) {
    // dynamic + static shared memory must stay <= 227 KB
    cudaError_t e = cudaFuncSetAttribute(pyramid_strips_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 224 * 1024);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  dim3 grid(n_strips, n_frames);
  pyramid_strips_kernel<<<grid, PT, 2 * (size_t)buf_bytes, s>>>(g, src, strips, xytab, tabs, buf_bytes);
  return cudaGetLastError();
}

}  // namespace ss
