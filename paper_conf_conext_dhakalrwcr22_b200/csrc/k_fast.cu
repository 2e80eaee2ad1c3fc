// k_fast.cu -- S2+S3: FAST-9 score map + per-cell non-max suppression with the
// iniThFAST -> minThFAST fallback (DESIGN.md §3 O2, O3; "parallelization of
// FAST corner detection ... with the GPU").
//
// One CTA per *band* = one row of 30-px FAST cells of one level of one frame (the cells of a
// row share their detect rows, and their detect windows tile [x0, x1) without gaps):
//  1. stage the band + 3-px ring halo in shared memory with 16-byte coalesced loads;
//  2. every warp walks band rows 32 pixels at a time: an 8-point pre-test (any 9-arc of the
//     ring contains 4 consecutive even ring positions) rejects ~80 % of pixels; survivors are
//     compacted into a per-warp queue with ballots and scored 32 at a time by the full arc test
//     on packed 16x2 lanes (DPX VIMNMX3.U16x2) -> M map of the band in shared memory;
//  3. one warp per cell: strict 8-neighbour maxima inside the cell's window (neighbours in the
//     next cell are ignored: per-cell ROI semantics), the cell's threshold (iniTh if any
//     survivor beats it, else minTh), compaction in raster order by ballot prefix counts.
//
//   M(p) = max_s max( min_{k<9} d_{s+k}, min_{k<9} -d_{s+k} ),  d_k = I(p) - I(p + R_k)
//   corner at t <=> M > t; pixels with M <= minTh are stored as 0 (they can neither be
//   candidates nor suppress one: a candidate has M > minTh).
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int FB_WARPS = 16;
constexpr int QCAP = 64;  // per-warp queue of pre-test survivors

__device__ __forceinline__ uint32_t swap16(uint32_t v) { return __byte_perm(v, 0, 0x1032); }

// 8-point necessary condition for M > t: four cyclically consecutive even ring positions
// all brighter than I+t or all darker than I-t.
__device__ __forceinline__ bool pretest8(const uint8_t* c, int p, int t) {
  const int cv = c[0];
  const int e0 = c[3 * p], e1 = c[2 * p + 2], e2 = c[3], e3 = c[-2 * p + 2];
  const int e4 = c[-3 * p], e5 = c[-2 * p - 2], e6 = c[-3], e7 = c[2 * p - 2];
  const int hi = cv + t, lo = cv - t;
  unsigned b = (unsigned)(e0 > hi) | ((unsigned)(e1 > hi) << 1) | ((unsigned)(e2 > hi) << 2) |
               ((unsigned)(e3 > hi) << 3) | ((unsigned)(e4 > hi) << 4) | ((unsigned)(e5 > hi) << 5) |
               ((unsigned)(e6 > hi) << 6) | ((unsigned)(e7 > hi) << 7);
  unsigned d = (unsigned)(e0 < lo) | ((unsigned)(e1 < lo) << 1) | ((unsigned)(e2 < lo) << 2) |
               ((unsigned)(e3 < lo) << 3) | ((unsigned)(e4 < lo) << 4) | ((unsigned)(e5 < lo) << 5) |
               ((unsigned)(e6 < lo) << 6) | ((unsigned)(e7 < lo) << 7);
  b |= b << 8;
  d |= d << 8;
  const unsigned rb = b & (b >> 1) & (b >> 2) & (b >> 3);
  const unsigned rd = d & (d >> 1) & (d >> 2) & (d >> 3);
  return ((rb | rd) & 0xFFu) != 0u;
}

// Full arc test: M clamped to 0 when <= tmin.  c = centre pixel in the staged band (pitch p).
__device__ __forceinline__ int fast_M(const uint8_t* c, int p, int tmin) {
  const int cv = c[0];
  // ring in OpenCV offsets16 order: (0,3) (1,3) (2,2) (3,1) (3,0) (3,-1) (2,-2) (1,-3) ...
  const int r0 = c[3 * p], r1 = c[3 * p + 1], r2 = c[2 * p + 2], r3 = c[p + 3];
  const int r4 = c[3], r5 = c[-p + 3], r6 = c[-2 * p + 2], r7 = c[-3 * p + 1];
  const int r8 = c[-3 * p], r9 = c[-3 * p - 1], r10 = c[-2 * p - 2], r11 = c[-p - 3];
  const int r12 = c[-3], r13 = c[p - 3], r14 = c[2 * p - 2], r15 = c[3 * p - 1];
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
  const uint32_t a = __vimax3_u16x2(__vimax3_u16x2(mn9[0], mn9[1], mn9[2]), __vimax3_u16x2(mn9[3], mn9[4], mn9[5]),
                                    __vimax3_u16x2(mn9[6], mn9[7], mn9[7]));
  const uint32_t z = __vimin3_u16x2(__vimin3_u16x2(mx9[0], mx9[1], mx9[2]), __vimin3_u16x2(mx9[3], mx9[4], mx9[5]),
                                    __vimin3_u16x2(mx9[6], mx9[7], mx9[7]));
  const int maxmin = max((int)(a & 0xFFFF), (int)(a >> 16));  // max_s min9(d') (dark ring)
  const int minmax = min((int)(z & 0xFFFF), (int)(z >> 16));  // min_s max9(d') (bright ring)
  const int M = max(maxmin - 256, 256 - minmax);
  return M > tmin ? M : 0;
}

__global__ void __launch_bounds__(FB_WARPS * 32) fast_bands_kernel(Geom g, FrameSrc src,
                                                                   const BandInfo* __restrict__ bands,
                                                                   const CellInfo* __restrict__ cells,
                                                                   uint32_t* __restrict__ slots,
                                                                   int32_t* __restrict__ cell_counts, int rp, int mbw,
                                                                   int region_bytes, int mband_bytes, int nball) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const BandInfo bd = bands[blockIdx.x];
  const int f = blockIdx.y;
  const int l = bd.level;
  const uint8_t* img;
  int ip;
  if (l == 0) {
    img = src.frames + (int64_t)f * src.stride;
    ip = src.pitch;
  } else {
    img = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    ip = g.pitch[l];
  }
  uint8_t* reg = smem;                                   // [RH][rp] staged band + halo
  uint8_t* Mb = smem + region_bytes;                     // [Dh + 2][mbw] M map (zero border rows)
  uint32_t* queue = reinterpret_cast<uint32_t*>(Mb + mband_bytes) + warp * QCAP;
  uint32_t* ball = reinterpret_cast<uint32_t*>(Mb + mband_bytes) + FB_WARPS * QCAP + warp * nball;
  const int Dw = bd.x1 - bd.x0, Dh = bd.y1 - bd.y0;
  const int RH = Dh + 6;
  const int xs = bd.x0 - 3;       // first staged column
  const int xa = xs & ~15;        // 16-byte aligned start
  const int shift = xs - xa;      // staged column of level column x = x - xa
  const int nchunk = (shift + Dw + 6 + 15) >> 4;
  const uint8_t* row0 = img + (int64_t)(bd.y0 - 3) * ip;
  // ---- 1. stage the band + halo (coalesced 16-B loads when the rows are 16-B aligned) ----
  if ((ip & 15) == 0 && (reinterpret_cast<uintptr_t>(img) & 15) == 0) {
    for (int i = threadIdx.x; i < RH * nchunk; i += blockDim.x) {
      const int r = i / nchunk, c = i - r * nchunk;
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(row0 + (int64_t)r * ip + xa) + c);
      *reinterpret_cast<uint4*>(reg + r * rp + 16 * c) = v;
    }
  } else {
    for (int i = threadIdx.x; i < RH * (Dw + 6); i += blockDim.x) {
      const int r = i / (Dw + 6), c = i - r * (Dw + 6);
      reg[r * rp + shift + c] = __ldg(row0 + (int64_t)r * ip + xs + c);
    }
  }
  for (int i = threadIdx.x; i < mband_bytes / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(Mb)[i] = 0u;
  __syncthreads();
  // ---- 2. M map: 8-point pre-test, warp-queue compaction, full arc test ----
  const int tmin = g.min_th, tini = g.ini_th;
  const unsigned lt = (1u << lane) - 1u;
  int qn = 0;
  auto drain = [&](int cnt) {  // score queue entries [0, cnt)
    if (lane < cnt) {
      const uint32_t e = queue[lane];
      const int x = (int)(e & 0xFFFF), y = (int)(e >> 16);  // band-relative D coordinates
      const int m = fast_M(reg + (y + 3) * rp + (x + 3 + shift), rp, tmin);
      Mb[(y + 1) * mbw + x + 1] = (uint8_t)m;
    }
  };
  for (int y = warp; y < Dh; y += FB_WARPS) {
    const uint8_t* rowc = reg + (y + 3) * rp + 3 + shift;
    for (int xc = 0; xc < Dw; xc += 32) {
      const int x = xc + lane;
      const bool pass = x < Dw && pretest8(rowc + x, rp, tmin);
      const unsigned msk = __ballot_sync(0xFFFFFFFFu, pass);
      if (pass) queue[qn + __popc(msk & lt)] = ((uint32_t)y << 16) | (uint32_t)x;
      qn += __popc(msk);
      __syncwarp();
      if (qn >= 32) {
        drain(32);
        __syncwarp();
        if (lane < qn - 32) queue[lane] = queue[32 + lane];
        qn -= 32;
        __syncwarp();
      }
    }
  }
  drain(qn);
  __syncthreads();
  // ---- 3. per cell: strict maxima inside the cell window, threshold choice, compaction ----
  for (int j = warp; j < bd.ncells; j += FB_WARPS) {
    const int ci = bd.cell_first + j;
    const CellInfo c = cells[ci];
    const int cx0 = c.x0 - bd.x0, cx1 = c.x1 - bd.x0;  // band-relative cell columns
    const int cw = cx1 - cx0;
    const int nxc = (cw + 31) >> 5;
    bool any_ini = false;
    int nch = 0;
    for (int y = 0; y < Dh; y++) {
      for (int xc = 0; xc < cw; xc += 32, nch++) {
        const int x = cx0 + xc + lane;
        bool kmin = false, kini = false;
        if (xc + lane < cw) {
          const uint8_t* p = Mb + (y + 1) * mbw + x + 1;
          const int m = p[0];
          if (m > tmin) {
            const bool lok = x > cx0, rok = x < cx1 - 1;  // neighbours in other cells are ignored
            bool mx = m > p[-mbw] && m > p[mbw];
            if (lok) mx = mx && m > p[-mbw - 1] && m > p[-1] && m > p[mbw - 1];
            if (rok) mx = mx && m > p[-mbw + 1] && m > p[1] && m > p[mbw + 1];
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
    }
    __syncwarp();
    const int sel = any_ini ? 1 : 0;
    uint32_t* out = slots + (int64_t)f * g.slots_per_frame + c.slot_off;
    int cnt = 0;
    for (int ch = 0; ch < nch; ch++) {
      const unsigned b = ball[2 * ch + sel];
      if ((b >> lane) & 1u) {
        const int y = ch / nxc, xc = (ch - y * nxc) * 32;
        const int x = cx0 + xc + lane;
        out[cnt + __popc(b & lt)] = pack_key(bd.x0 + x, bd.y0 + y, Mb[(y + 1) * mbw + x + 1]);
      }
      cnt += __popc(b);
    }
    if (lane == 0) cell_counts[(int64_t)f * g.total_cells + ci] = cnt;
    __syncwarp();
  }
}

}  // namespace

size_t fast_smem_bytes(const Geom& g, int* rp, int* mbw, int* region_bytes, int* mband_bytes, int* nball) {
  // widest band + halo, 16-B aligned staging with up to 15 B of lead-in
  *rp = ((g.max_band_w + 6 + 15 + 15) / 16) * 16;
  *region_bytes = ((g.max_band_h + 6) * *rp + 15) & ~15;
  *mbw = (g.max_band_w + 2 + 3) & ~3;
  *mband_bytes = ((g.max_band_h + 2) * *mbw + 15) & ~15;
  *nball = 2 * g.max_band_h * ((g.max_cell_w + 31) / 32);
  return (size_t)*region_bytes + *mband_bytes + (size_t)FB_WARPS * QCAP * 4 + (size_t)FB_WARPS * *nball * 4;
}

cudaError_t launch_fast_bands(const Geom& g, int n_frames, FrameSrc src, const BandInfo* bands,
                              const CellInfo* cells, uint32_t* slots, int32_t* cell_counts, cudaStream_t s) {
  int rp, mbw, rb, mb, nb;
  const size_t smem = fast_smem_bytes(g, &rp, &mbw, &rb, &mb, &nb);
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(fast_bands_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr_set = true;
  }
  dim3 grid(g.total_bands, n_frames);
  fast_bands_kernel<<<grid, FB_WARPS * 32, smem, s>>>(g, src, bands, cells, slots, cell_counts, rp, mbw, rb, mb, nb);
  return cudaGetLastError();
}

}  // namespace ss
