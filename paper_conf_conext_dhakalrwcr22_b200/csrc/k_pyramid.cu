// k_pyramid.cu -- S1: image pyramid, level l = bilinear resize of level l-1 (DESIGN.md §3 O1).
//
// Fixed-point definition (bit-exact INTER_LINEAR_EXACT semantics): per destination column
// the host precomputes (x0, wx1, x1-x0) with wx1 = rne(frac * 256); then
//   out = ((256-wy1)*(wx0*s[y0][x0] + wx1*s[y0][x1]) + wy1*(...row y1...) + 2^15) >> 16.
//
// ONE launch builds every level of every frame.  Levels are chained (level l reads level
// l-1), so instead of one launch per level (7 dependent launches, each a few microseconds
// of launch + drain for a few hundred KB of work) each CTA owns a block of the frame and
// carries it through all levels in shared memory: at level l it owns the rectangle O_l
// (the level is cut into Gx x Gy blocks at columns i*w_l/Gx, rows j*h_l/Gy, so the owned
// rectangles partition every level exactly) and computes the larger rectangle N_l that the
// deeper levels' footprints need (N_{L-1} = O_{L-1}, N_{l-1} = bbox(O_{l-1}, footprint of
// N_l)).  Halo pixels are recomputed by the neighbouring CTAs with the same integer formula,
// so the result is identical to the level-by-level definition.  Only O_l is stored to HBM.
// The host (pyramid_plan) computes every rectangle once at ss_create.
#include "ss_internal.h"

namespace ss {

namespace {

#ifndef SS_PYR_THREADS
#define SS_PYR_THREADS 256
#endif
constexpr int PT = SS_PYR_THREADS;  // threads per CTA (a block of every level per CTA)

// Four destination pixels of one row.  Per thread the four columns are fixed: their source
// bytes x0_q, x1_q lie in [x0_0, x0_0 + 6) (x1_3 - x0_0 <= 5 for scale <= 4/3), read as three
// aligned words from a = x0_0 & ~3 and funnel-shifted by sh = 8 * (x0_0 & 3).  Horizontal
// first: one byte permute gathers (s[x0_q], s[x1_q]) of two pixels into the bytes of one
// register and one IDP.2A per pixel forms h_q = wx0_q * s[x0_q] + wx1_q * s[x1_q] (weights as a
// 16x2 pair, wx0 + wx1 = 256, h <= 65280); then vertical per pixel with two IMADs,
// acc = wy0 * h(y0) + wy1 * h(y1) + 2^15 < 2^24, whose byte 2 is the output (>> 16), picked by
// byte permutes.  Exact integer arithmetic: the order of the two passes does not change the
// result (INTER_LINEAR_EXACT, DESIGN.md §3 O1).
__device__ __forceinline__ void window8(const uint8_t* row, uint32_t sh, uint32_t* lo, uint32_t* hi) {
  const uint32_t* w = reinterpret_cast<const uint32_t*>(row);
  const uint32_t w0 = w[0], w1 = w[1], w2 = w[2];
  *lo = __funnelshift_r(w0, w1, sh);
  *hi = __funnelshift_r(w1, w2, sh);
}

// h_q of one source row (sel: byte gathers (x0_0, x1_0, x0_1, x1_1) | (x0_2, x1_2, x0_3, x1_3) << 16)
__device__ __forceinline__ void hrow4(const uint8_t* row, uint32_t sh, uint32_t sel, const uint32_t (&W)[4],
                                      uint32_t (&h)[4]) {
  uint32_t lo, hi;
  window8(row, sh, &lo, &hi);
  const uint32_t g01 = __byte_perm(lo, hi, sel & 0xFFFF), g23 = __byte_perm(lo, hi, sel >> 16);
  h[0] = __dp2a_lo(W[0], g01, 0u);
  h[1] = __dp2a_hi(W[1], g01, 0u);
  h[2] = __dp2a_lo(W[2], g23, 0u);
  h[3] = __dp2a_hi(W[3], g23, 0u);
}

__device__ __forceinline__ uint32_t lerp4(const uint8_t* r0, const uint8_t* r1, uint32_t sh, uint32_t sel,
                                          const uint32_t (&W)[4], uint32_t wy1) {
  uint32_t h0[4], h1[4];
  hrow4(r0, sh, sel, W, h0);
  hrow4(r1, sh, sel, W, h1);
  const uint32_t wy0 = 256 - wy1;
  uint32_t a[4];
#pragma unroll
  for (int q = 0; q < 4; q++) a[q] = h0[q] * wy0 + (h1[q] * wy1 + (1u << 15));  // < 2^24
  // byte 2 of each accumulator = (acc >> 16)
  return __byte_perm(__byte_perm(a[0], a[1], 0x0062), __byte_perm(a[2], a[3], 0x0062), 0x5410);
}

// the level whose start lets the dependent grid (FAST) launch: <= 1 = the kernel's start (FAST's
// level-0 CTAs run beside the pyramid; its other CTAs sit resident until the pyramid ends),
// k = once levels < k are built, > L - 1 = only at exit
#ifndef SS_PYR_TRIGGER
#define SS_PYR_TRIGGER 3
#endif
#ifndef SS_PYR_MINB
#define SS_PYR_MINB 1
#endif
__global__ void __launch_bounds__(PT, SS_PYR_MINB) pyramid_fused_kernel(const __grid_constant__ Geom g, FrameSrc src,
                                                              const uint4* __restrict__ gtab,
                                                              const uint32_t* __restrict__ ytab,
                                                              const PyrLvl* __restrict__ plan, int buf0_bytes,
                                                              int buf1_bytes) {
  pdl_wait();
  if (SS_PYR_TRIGGER <= 1) pdl_trigger();
  extern __shared__ __align__(16) uint8_t smem[];
  // [buffer 0 | pad | buffer 1 | pad | plan | group coefficients | row coefficients]; level l
  // lives in buffer l & 1; the pads absorb the source windows' over-read past a buffer's
  // last row (bytes never used).
  uint8_t* const buf0 = smem;
  uint8_t* const buf1 = smem + buf0_bytes + 16;
  const int L = g.L;
  int4* const s_plan = reinterpret_cast<int4*>(buf1 + buf1_bytes + 16);
  uint4* const s_g = reinterpret_cast<uint4*>(s_plan + 4 * L);
  const int f = blockIdx.y;
  const PyrLvl* P = plan + (int64_t)blockIdx.x * L;
  const int tid = threadIdx.x;

  // ---- plan + every level's coefficients into shared memory (all loads in flight at once)
  if (tid < 4 * L) s_plan[tid] = __ldg(reinterpret_cast<const int4*>(P) + tid);
  {
    uint32_t* const s_y = reinterpret_cast<uint32_t*>(s_g) + __ldg(&P[0].soff);  // entry 0: s_y base
#pragma unroll
    for (int l = 1; l < kMaxLevels; l++) {
      if (l < L) {
        const int ngx = __ldg(&P[l].ngx), rows = __ldg(&P[l].rows), so = __ldg(&P[l].soff);
        if (tid < ngx) {
          s_g[(so & 0xFFFF) + tid] = __ldg(gtab + __ldg(&P[l].gg) + tid);
        } else if (tid < ngx + rows) {
          s_y[(so >> 16) + tid - ngx] = __ldg(ytab + __ldg(&P[l].yg) + tid - ngx);
        }
      }
    }
  }

  // ---- stage the level-0 footprint (x0 aligned down to 16) ----
  {
    const PyrLvl r = P[0];
    const int rows = r.rows, pitch = r.dpitch;
    const uint8_t* s = src.frames + (int64_t)f * src.stride + (int64_t)r.ny0 * src.pitch + r.nx0;
    const int sp = src.pitch;
    if ((sp & 15) == 0 && (reinterpret_cast<uintptr_t>(s) & 15) == 0) {
      const int nch = pitch >> 4;
      for (int i = tid; i < rows * nch; i += PT) {
        const int y = i / nch, c = i - y * nch;
        *reinterpret_cast<uint4*>(buf0 + y * pitch + 16 * c) =
            __ldg(reinterpret_cast<const uint4*>(s + (int64_t)y * sp) + c);
      }
    } else {
      const int ncol = r.ngx;  // entry 0: staged width
      for (int i = tid; i < rows * ncol; i += PT) {
        const int y = i / ncol, c = i - y * ncol;
        buf0[y * pitch + c] = __ldg(s + (int64_t)y * sp + c);
      }
    }
  }

  const uint32_t* const s_y = reinterpret_cast<const uint32_t*>(s_g) + P[0].soff;
  for (int l = 1; l < L; l++) {
    __syncthreads();  // staged / the previous level's buffer complete
    if (l == SS_PYR_TRIGGER && l > 1) pdl_trigger();
    const int4 A = s_plan[4 * l], B = s_plan[4 * l + 1], C = s_plan[4 * l + 2], D = s_plan[4 * l + 3];
    const int nx0 = A.x, ngx = A.y, ny0 = A.z, rows = A.w;
    const int ry = (int)(((uint32_t)tid * (uint32_t)(D.x & 0x1FFFFF)) >> 20);  // tid / ngx (host-verified)
    if (ry >= (D.x >> 21)) continue;                                             // rows in parallel
    const int cx = tid - ry * ngx;
    const uint8_t* sb = (l & 1) ? buf0 : buf1;
    uint8_t* db = (l & 1) ? buf1 : buf0;
    const int spitch = C.z, dpitch = C.w;
    // this thread's four columns (host-built: source window, gather selectors, weights)
    const uint4 gq = s_g[(D.y & 0xFFFF) + cx];
    const uint32_t sh = gq.x >> 16, sel = gq.y;
    // (wx0, wx1) = (256 - wx1, wx1) as a 16x2 pair: wx1 * 65535 + 256
    const uint32_t W[4] = {(gq.z & 0xFFFF) * 0xFFFFu + 256u, (gq.z >> 16) * 0xFFFFu + 256u,
                           (gq.w & 0xFFFF) * 0xFFFFu + 256u, (gq.w >> 16) * 0xFFFFu + 256u};
    const uint8_t* const sa = sb + (int)(gq.x & 0xFFFF) - C.x;
    uint8_t* const da = db + 4 * cx;
    // owned columns come in whole groups of 4 (cuts are multiples of 4); only the level's
    // last group can pass its right edge
    const int x = nx0 + 4 * cx;
    const bool own_x = x >= B.x && x < B.y;
    uint8_t* const d = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l] + x;
    const int gp = g.pitch[l];
    const uint32_t* const yc = s_y + (D.y >> 16);
    for (int r = ry; r < rows; r += (D.x >> 21)) {
      const uint32_t cy = yc[r];
      const int y0 = (int)(cy & 0xFFFF) - C.y, y1 = y0 + (int)(cy >> 25);
      const uint32_t packed = lerp4(sa + y0 * spitch, sa + y1 * spitch, sh, sel, W, (cy >> 16) & 0x1FF);
      *reinterpret_cast<uint32_t*>(da + r * dpitch) = packed;
      const int y = ny0 + r;
      if (own_x && y >= B.z && y < B.w)  // x and the pitch are multiples of 4 and x < w <= pitch:
        // the level's last group may write up to 3 bytes of the row's pitch padding, which no
        // reader uses (FAST and stereo stay inside the level; describe's TMA boxes are bounded
        // by the level width)
        *reinterpret_cast<uint32_t*>(d + (int64_t)y * gp) = packed;
    }
  }
}

// footprint of destination rows/columns [a, b) in the source: [lo, hi) (tab = coefficients)
void footprint(const uint32_t* tab, int n, int a, int b, int* lo, int* hi) {
  const uint32_t c0 = tab[a < n ? a : n - 1], c1 = tab[(b - 1) < n ? b - 1 : n - 1];
  *lo = (int)(c0 & 0xFFFF);
  *hi = (int)(c1 & 0xFFFF) + (int)(c1 >> 25) + 1;
}

}  // namespace

bool pyramid_groups(const Geom& g, const uint32_t* tab, const int64_t* xoff, std::vector<uint4>* gtab,
                    std::vector<int64_t>* goff) {
  // per level l >= 1 and 4-column group G: source window, gather selectors and weights
  const int L = g.L;
  goff->assign(L, 0);
  gtab->clear();
  for (int l = 1; l < L; l++) {
    (*goff)[l] = (int64_t)gtab->size();
    const uint32_t* xt = tab + xoff[l];
    for (int x = 0; x < g.w[l]; x += 4) {
      uint32_t c[4];
      for (int q = 0; q < 4; q++) c[q] = xt[x + q < g.w[l] ? x + q : g.w[l] - 1];
      const uint32_t x00 = c[0] & 0xFFFF;
      uint32_t sel = 0;  // byte gathers: (x0_q, x1_q) of pixel q in bytes 2(q%2), 2(q%2)+1 of word q/2
      for (int q = 0; q < 4; q++) {
        const uint32_t k = (c[q] & 0xFFFF) - x00;
        if (k + (c[q] >> 25) > 5) return false;  // the kernel's 6-byte window (scale <= 4/3)
        sel |= (k | (k + (c[q] >> 25)) << 4) << (8 * q);
      }
      uint4 e;
      e.x = (x00 & ~3u) | ((8u * (x00 & 3)) << 16);
      e.y = sel;
      e.z = ((c[0] >> 16) & 0x1FF) | (((c[1] >> 16) & 0x1FF) << 16);
      e.w = ((c[2] >> 16) & 0x1FF) | (((c[3] >> 16) & 0x1FF) << 16);
      gtab->push_back(e);
    }
  }
  return true;
}

bool pyramid_plan(const Geom& g, const uint32_t* tab, const int64_t* xoff, const int64_t* yoff,
                  const std::vector<int64_t>& goff, int gx, int gy, std::vector<PyrLvl>* out, int* buf0, int* buf1,
                  int* smem) {
  const int L = g.L;
  out->assign((size_t)gx * gy * L, PyrLvl{});
  std::vector<PyrRect> R(L);
  int b0 = 0, b1 = 0, max_g = 0, max_y = 0;
  for (int j = 0; j < gy; j++) {
    for (int i = 0; i < gx; i++) {
      for (int l = 1; l < L; l++) {
        // column cuts on multiples of 4 so every 4-pixel group has one owner
        R[l].ox0 = (int16_t)(i == 0 ? 0 : (int)(((int64_t)i * g.w[l] / gx + 2) & ~3));
        R[l].ox1 = (int16_t)(i + 1 == gx ? g.w[l] : (int)(((int64_t)(i + 1) * g.w[l] / gx + 2) & ~3));
        R[l].oy0 = (int16_t)((int64_t)j * g.h[l] / gy);
        R[l].oy1 = (int16_t)((int64_t)(j + 1) * g.h[l] / gy);
      }
      // needed rectangles, deepest level first
      int nx0 = R[L - 1].ox0, nx1 = R[L - 1].ox1, ny0 = R[L - 1].oy0, ny1 = R[L - 1].oy1;
      for (int l = L - 1; l >= 1; l--) {
        nx0 &= ~3;
        nx1 = (nx1 + 3) & ~3;  // may pass the level edge: those columns are computed, never stored
        R[l].nx0 = (int16_t)nx0;
        R[l].nx1 = (int16_t)nx1;
        R[l].ny0 = (int16_t)ny0;
        R[l].ny1 = (int16_t)ny1;
        int fx0, fx1, fy0, fy1;
        footprint(tab + xoff[l], g.w[l], nx0, nx1 < g.w[l] ? nx1 : g.w[l], &fx0, &fx1);
        footprint(tab + yoff[l], g.h[l], ny0, ny1, &fy0, &fy1);
        if (l - 1 >= 1) {
          nx0 = fx0 < R[l - 1].ox0 ? fx0 : R[l - 1].ox0;
          nx1 = fx1 > R[l - 1].ox1 ? fx1 : R[l - 1].ox1;
          ny0 = fy0 < R[l - 1].oy0 ? fy0 : R[l - 1].oy0;
          ny1 = fy1 > R[l - 1].oy1 ? fy1 : R[l - 1].oy1;
        } else {
          R[0].nx0 = (int16_t)(fx0 & ~15);
          R[0].nx1 = (int16_t)fx1;
          R[0].ny0 = (int16_t)fy0;
          R[0].ny1 = (int16_t)fy1;
        }
      }
      PyrLvl* P = out->data() + (size_t)(j * gx + i) * L;
      int sg = 0, sy = 0;
      for (int l = 0; l < L; l++) {
        const int w = R[l].nx1 - R[l].nx0, h = R[l].ny1 - R[l].ny0;
        const int pitch = (w + 15) & ~15;
        int& b = (l & 1) ? b1 : b0;
        if (pitch * h > b) b = pitch * h;
        PyrLvl& v = P[l];
        v.nx0 = R[l].nx0;
        v.ny0 = R[l].ny0;
        v.rows = h;
        v.dpitch = pitch;
        if (l == 0) {
          v.ngx = w;  // staged width
          continue;
        }
        const int ngx = w / 4;
        if (ngx < 1 || ngx + h > PT) return false;  // one coefficient load per thread per level
        const uint32_t magic = (uint32_t)(((1u << 20) + ngx - 1) / ngx);
        for (int t = 0; t < PT; t++)
          if ((int)((t * magic) >> 20) != t / ngx) return false;
        v.ngx = ngx;
        v.ox0 = R[l].ox0;
        v.ox1 = R[l].ox1;
        v.oy0 = R[l].oy0;
        v.oy1 = R[l].oy1;
        v.sx0 = R[l - 1].nx0;
        v.sy0 = R[l - 1].ny0;
        v.spitch = P[l - 1].dpitch;
        v.mr = (int32_t)(magic | ((uint32_t)(PT / ngx) << 21));
        v.soff = sg | (sy << 16);
        v.gg = (int32_t)(goff[l] + R[l].nx0 / 4);
        v.yg = (int32_t)(yoff[l] + R[l].ny0);
        sg += ngx;
        sy += h;
      }
      if (sg > max_g) max_g = sg;
      if (sy > max_y) max_y = sy;
    }
  }
  for (size_t b = 0; b < out->size(); b += L) (*out)[b].soff = 4 * max_g;  // s_y base, words after s_g
  *buf0 = (b0 + 15) & ~15;
  *buf1 = (b1 + 15) & ~15;
  *smem = *buf0 + 16 + *buf1 + 16 + L * (int)sizeof(PyrLvl) + 16 * max_g + 4 * max_y;
  return *smem <= kPyrSmemMax && max_g < 16384 && max_y < 65536;
}

cudaError_t pyramid_init() {  // ss_create, per device; pyramid_plan keeps every plan within kPyrSmemMax
  cudaError_t e = carveout_from_env(pyramid_fused_kernel);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(pyramid_fused_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kPyrSmemMax);
}

cudaError_t launch_pyramid(const Geom& g, int n_frames, FrameSrc src, const uint4* gtab, const uint32_t* ytab,
                           const PyrLvl* plan, int n_blocks, int buf0, int buf1, int smem, cudaStream_t s) {
  dim3 grid(n_blocks, n_frames);
  cudaError_t e = launch_pdl(pyramid_fused_kernel, grid, dim3(PT), (size_t)smem, s, g, src, gtab, ytab, plan, buf0, buf1);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
