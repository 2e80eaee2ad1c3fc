// k_fast.cu -- S2+S3: FAST-9 score map + per-cell non-max suppression with the
// iniThFAST -> minThFAST fallback (DESIGN.md §3 O2, O3; "parallelization of
// FAST corner detection ... with the GPU").
//
// One warp per 30-px FAST cell (all levels and frames of the call in one launch): the
// cell's input region (detect window D + 3-px ring halo) is staged in shared memory, M(p)
// is computed for every pixel of D (cardinal pre-test at minTh, then the full arc test on
// packed 16x2 lanes with the sm_90+/sm_100 DPX three-way min/max), cell-local strict
// maxima are flagged with warp ballots, and the survivors of the threshold the cell uses
// (iniTh if any survive it, else minTh) are compacted into the cell's slots in raster
// order with ballot prefix counts.  No block-level synchronisation: warps are independent.
//
//   M(p) = max_s max( min_{k<9} d_{s+k}, min_{k<9} -d_{s+k} ),  d_k = I(p) - I(p + R_k)
//   corner at t <=> M > t; pixels with M <= minTh are stored as 0 (they can neither be
//   candidates nor suppress one: a candidate has M > minTh).
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int FAST_WARPS = 8;

__device__ __forceinline__ uint32_t swap16(uint32_t v) { return __byte_perm(v, 0, 0x1032); }

// c points at the centre pixel inside the staged region (row pitch p).
__device__ __forceinline__ int fast_score(const uint8_t* c, int p, int tmin) {
  const int cv = c[0];
  const int r0 = c[3 * p], r4 = c[3], r8 = c[-3 * p], r12 = c[-3];
  const int hi = cv + tmin, lo = cv - tmin;
  const unsigned b = (unsigned)(r0 > hi) | ((unsigned)(r4 > hi) << 1) | ((unsigned)(r8 > hi) << 2) |
                     ((unsigned)(r12 > hi) << 3);
  const unsigned d = (unsigned)(r0 < lo) | ((unsigned)(r4 < lo) << 1) | ((unsigned)(r8 < lo) << 2) |
                     ((unsigned)(r12 < lo) << 3);
  // an arc of 9 of the 16 ring pixels always contains two cyclically adjacent cardinals
  const unsigned pb = b & ((b >> 1) | ((b & 1u) << 3));
  const unsigned pd = d & ((d >> 1) | ((d & 1u) << 3));
  if (!(pb | pd)) return 0;
  // ring in OpenCV offsets16 order: (0,3) (1,3) (2,2) (3,1) (3,0) (3,-1) (2,-2) (1,-3) ...
  const int r1 = c[3 * p + 1], r2 = c[2 * p + 2], r3 = c[p + 3];
  const int r5 = c[-p + 3], r6 = c[-2 * p + 2], r7 = c[-3 * p + 1];
  const int r9 = c[-3 * p - 1], r10 = c[-2 * p - 2], r11 = c[-p - 3];
  const int r13 = c[p - 3], r14 = c[2 * p - 2], r15 = c[3 * p - 1];
  // biased differences d'_k = cv - r_k + 256 in [1, 511], packed (d'_k, d'_{k+8})
  const uint32_t cc = (uint32_t)(cv + 256) * 0x10001u;
  uint32_t q[16];
  q[0] = cc - ((uint32_t)r0 | ((uint32_t)r8 << 16));
  q[1] = cc - ((uint32_t)r1 | ((uint32_t)r9 << 16));
  q[2] = cc - ((uint32_t)r2 | ((uint32_t)r10 << 16));
  q[3] = cc - ((uint32_t)r3 | ((uint32_t)r11 << 16));
  q[4] = cc - ((uint32_t)r4 | ((uint32_t)r12 << 16));
  q[5] = cc - ((uint32_t)r5 | ((uint32_t)r13 << 16));
  q[6] = cc - ((uint32_t)r6 | ((uint32_t)r14 << 16));
  q[7] = cc - ((uint32_t)r7 | ((uint32_t)r15 << 16));
#pragma unroll
  for (int k = 0; k < 8; k++) q[k + 8] = swap16(q[k]);
  // windows of 9: lo half = window s, hi half = window s+8
  uint32_t mn3[14], mx3[14];
#pragma unroll
  for (int k = 0; k < 14; k++) {
    mn3[k] = __vimin3_u16x2(q[k], q[k + 1], q[k + 2]);
    mx3[k] = __vimax3_u16x2(q[k], q[k + 1], q[k + 2]);
  }
  uint32_t mn9[8], mx9[8];
#pragma unroll
  for (int s = 0; s < 8; s++) {
    mn9[s] = __vimin3_u16x2(mn3[s], mn3[s + 3], mn3[s + 6]);
    mx9[s] = __vimax3_u16x2(mx3[s], mx3[s + 3], mx3[s + 6]);
  }
  uint32_t a = __vimax3_u16x2(__vimax3_u16x2(mn9[0], mn9[1], mn9[2]), __vimax3_u16x2(mn9[3], mn9[4], mn9[5]),
                              __vimax3_u16x2(mn9[6], mn9[7], mn9[7]));
  uint32_t z = __vimin3_u16x2(__vimin3_u16x2(mx9[0], mx9[1], mx9[2]), __vimin3_u16x2(mx9[3], mx9[4], mx9[5]),
                              __vimin3_u16x2(mx9[6], mx9[7], mx9[7]));
  const int maxmin = max((int)(a & 0xFFFF), (int)(a >> 16));  // max_s min9(d') (dark ring)
  const int minmax = min((int)(z & 0xFFFF), (int)(z >> 16));  // min_s max9(d') (bright ring)
  const int M = max(maxmin - 256, 256 - minmax);
  return M > tmin ? M : 0;
}

__global__ void __launch_bounds__(FAST_WARPS * 32) fast_cells_kernel(Geom g, FrameSrc src,
                                                                     const CellInfo* __restrict__ cells,
                                                                     uint32_t* __restrict__ slots,
                                                                     int32_t* __restrict__ cell_counts,
                                                                     int rp, int per_warp) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ci = blockIdx.x * FAST_WARPS + warp;
  const int f = blockIdx.y;
  if (ci >= g.total_cells) return;  // warp-uniform; no block barriers below
  const CellInfo c = cells[ci];
  const int l = c.level;
  const uint8_t* img;
  int ip;
  if (l == 0) {
    img = src.frames + (int64_t)f * src.stride;
    ip = src.pitch;
  } else {
    img = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    ip = g.pitch[l];
  }
  uint8_t* reg = smem + warp * per_warp;
  const int Dw = c.x1 - c.x0, Dh = c.y1 - c.y0;
  const int RW = Dw + 6, RH = Dh + 6;
  const int MW = Dw + 2;
  uint8_t* Mt = reg + RH * rp;
  uint32_t* ball = reinterpret_cast<uint32_t*>(Mt + ((((Dh + 2) * MW) + 15) & ~15));
  // stage the input region (D + 3-px halo)
  const uint8_t* src0 = img + (int64_t)(c.y0 - 3) * ip + (c.x0 - 3);
  for (int r = 0; r < RH; r++)
    for (int x = lane; x < RW; x += 32) reg[r * rp + x] = __ldg(src0 + (int64_t)r * ip + x);
  for (int i = lane; i < (Dh + 2) * MW; i += 32) Mt[i] = 0;
  __syncwarp();
  const int npx = Dw * Dh;
  const int tmin = g.min_th, tini = g.ini_th;
  for (int base = 0; base < npx; base += 32) {
    const int idx = base + lane;
    if (idx < npx) {
      const int y = idx / Dw, x = idx - y * Dw;
      const int m = fast_score(reg + (y + 3) * rp + (x + 3), rp, tmin);
      Mt[(y + 1) * MW + x + 1] = (uint8_t)m;
    }
  }
  __syncwarp();
  bool any_ini = false;
  int nch = 0;
  for (int base = 0; base < npx; base += 32, nch++) {
    const int idx = base + lane;
    bool kmin = false, kini = false;
    if (idx < npx) {
      const int y = idx / Dw, x = idx - y * Dw;
      const uint8_t* p = Mt + (y + 1) * MW + x + 1;
      const int m = p[0];
      if (m > tmin) {
        const bool mx = m > p[-MW - 1] && m > p[-MW] && m > p[-MW + 1] && m > p[-1] && m > p[1] &&
                        m > p[MW - 1] && m > p[MW] && m > p[MW + 1];
        kmin = mx;
        kini = mx && m > tini;
      }
    }
    const unsigned bmin = __ballot_sync(0xFFFFFFFFu, kmin);
    const unsigned bini = __ballot_sync(0xFFFFFFFFu, kini);
    if (lane == 0) {
      ball[2 * nch] = bmin;
      ball[2 * nch + 1] = bini;
    }
    any_ini |= (bini != 0u);
  }
  __syncwarp();
  const int sel = any_ini ? 1 : 0;
  uint32_t* out = slots + (int64_t)f * g.slots_per_frame + c.slot_off;
  const unsigned lt = (1u << lane) - 1u;
  int cnt = 0;
  for (int ch = 0; ch < nch; ch++) {
    const unsigned b = ball[2 * ch + sel];
    if ((b >> lane) & 1u) {
      const int idx = ch * 32 + lane;
      const int y = idx / Dw, x = idx - y * Dw;
      out[cnt + __popc(b & lt)] = pack_key(c.x0 + x, c.y0 + y, Mt[(y + 1) * MW + x + 1]);
    }
    cnt += __popc(b);
  }
  if (lane == 0) cell_counts[(int64_t)f * g.total_cells + ci] = cnt;
}

}  // namespace

cudaError_t launch_fast_cells(const Geom& g, int n_frames, FrameSrc src, const CellInfo* cells, uint32_t* slots,
                              int32_t* cell_counts, cudaStream_t s) {
  const int rp = (g.max_rw + 3) & ~3;
  const int dmax_w = g.max_rw - 6, dmax_h = g.max_rh - 6;
  const int mbytes = (((dmax_h + 2) * (dmax_w + 2)) + 15) & ~15;
  const int nch = (dmax_w * dmax_h + 31) / 32;
  int per_warp = g.max_rh * rp + mbytes + nch * 8;
  per_warp = (per_warp + 15) & ~15;
  const size_t smem = (size_t)per_warp * FAST_WARPS;
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(fast_cells_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    attr_set = true;
  }
  dim3 grid((g.total_cells + FAST_WARPS - 1) / FAST_WARPS, n_frames);
  fast_cells_kernel<<<grid, FAST_WARPS * 32, smem, s>>>(g, src, cells, slots, cell_counts, rp, per_warp);
  return cudaGetLastError();
}

}  // namespace ss
