// k_fast.cu -- S2+S3: FAST-9 score map + per-cell non-max suppression with the
// iniThFAST -> minThFAST fallback (DESIGN.md §3 O2, O3; "parallelization of
// FAST corner detection ... with the GPU").
//
// ONE launch for every level of every frame (levels >= 1 wait for the pyramid; level 0 reads
// only the caller's frames and runs beside it), one CTA per *segment* = up to 8 consecutive
// 30-px FAST cells of one cell row of one level of one frame (the cells of a row share their
// detect rows and their detect windows tile [x0, x1) without gaps), largest segments first:
//  1. stage the band + ring halo in shared memory with 16-byte coalesced loads;
//  2. the score M of EVERY band pixel, four horizontally adjacent pixels per thread: the band
//     is staged as I - 128 (bytes XOR 0x80); each ring value PAIR of pixels (0, 2) or (1, 3)
//     is one sign-replicating byte permute of a sliding 7-row x 3-word register window (3
//     shared loads per row step) into two signed 16-bit lanes, and the cyclic min / max over
//     the 16 arcs of 9 of the RAW ring values runs on DPX three-way min/max (VIMNMX3.S16x2);
//     the centre enters only at the end (min_k (c - r_k) = c - max_k r_k) -- no pre-test, no
//     divergence, one 32-bit store of 4 scores;
//  3. strict 8-neighbour maxima above minTh / iniTh, every thread on 4-pixel groups (the score
//     tasks' layout): each row's horizontal 3-max and left/right max per 16x2 half, with
//     neighbours in another cell masked to 0 by a cell-start column bitmap (per-cell ROI
//     semantics), into two shared-memory bit planes;
//  4. one warp per cell, one lane per cell row: the row's 64-bit masks from the bit planes, the
//     cell's threshold (iniTh if any maximum beats it, else minTh), and the survivors written
//     in raster order (warp prefix sum of the row counts).
//
//   M(p) = max_s max( min_{k<9} d_{s+k}, min_{k<9} -d_{s+k} ),  d_k = I(p) - I(p + R_k)
//        = max( I(p) - min_s max_{k<9} I(p + R_{s+k}),  max_s min_{k<9} I(p + R_{s+k}) - I(p) )
//   corner at t <=> M > t (stored clamped to >= 0; scores <= minTh can neither be candidates
//   nor suppress one, so no thresholding is needed before the NMS).
#include "ss_internal.h"

namespace ss {

#ifdef SS_FAST_PHASES  // per-CTA phase timestamps (scripts/fast_phases.py; instrumented builds only)
__device__ unsigned long long g_fast_ts[2][4096][8];
#define FAST_TS(i)                                                                                     \
  do {                                                                                                 \
    if (threadIdx.x == 0 && blockIdx.y * gridDim.x + blockIdx.x < 4096) {                              \
      unsigned long long t_;                                                                           \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                                           \
      g_fast_ts[bd.level != 0][blockIdx.y * gridDim.x + blockIdx.x][i] = t_;                           \
    }                                                                                                  \
  } while (0)
#else
#define FAST_TS(i) \
  do {             \
  } while (0)
#endif

namespace {

#ifndef SS_FAST_WARPS
#define SS_FAST_WARPS 8
#endif
#ifndef SS_FAST_ROWS
#define SS_FAST_ROWS 8
#endif
constexpr int FB_WARPS = SS_FAST_WARPS;
constexpr int FB_THREADS = FB_WARPS * 32;
constexpr int ROWS_PER_TASK = SS_FAST_ROWS;  // rows per score task (sliding 7-row window)
// when the dependent grid (the distribution: 32 CTAs of 215 KB shared memory at c2, resident from
// then until this grid ends) may launch: 0 = the CTA's start, 2 = after its scores, 3 = after
// its NMS, -1 = at exit (measured: exit -3.5 % at c2)
#ifndef SS_FAST_TRIGGER
#define SS_FAST_TRIGGER 0
#endif
#ifndef SS_FAST_MINB
#define SS_FAST_MINB (24 / FB_WARPS > 1 ? 24 / FB_WARPS : 1)
#endif
constexpr int FB_MIN_BLOCKS = SS_FAST_MINB;  // 3: 80 registers

// The band is staged with every byte XOR 0x80, so a byte read as a signed char is I - 128
// (order preserving).  A PRMT whose selector nibbles set the sign-replicate bit turns two
// bytes of a 64-bit window straight into two signed 16-bit lanes, so every ring value of a
// pixel pair is ONE byte permute of the row's words (no separate unpack and no subtraction).
//
// For a pair of pixels (16x2 lanes, values v = I - 128) with ring values r[0..15] and
// centre c, using min_k (c - r_k) = c - max_k r_k and min_k (r_k - c) = min_k r_k - c:
//   M = max( max_s min9(r)[s] - c,  c - min_s max9(r)[s],  0 ).
// Returns M + 256 in both lanes (the low byte of each lane is M).
__device__ __forceinline__ uint32_t arc_score2(const uint32_t (&r)[16], uint32_t c) {
  // the bright side (min over arcs, max over starts) first, then the dark side, so only one
  // side's 16 three-way partials are live at a time (register pressure: 4 CTAs per SM)
  uint32_t maxmin, minmax;
  {
    uint32_t mn3[16];
#pragma unroll
    for (int k = 0; k < 16; k++) mn3[k] = __vimin3_s16x2(r[k], r[(k + 1) & 15], r[(k + 2) & 15]);
    uint32_t mn9[16];
#pragma unroll
    for (int s = 0; s < 16; s++) mn9[s] = __vimin3_s16x2(mn3[s], mn3[(s + 3) & 15], mn3[(s + 6) & 15]);
    const uint32_t a1 = __vimax3_s16x2(__vimax3_s16x2(mn9[0], mn9[1], mn9[2]), __vimax3_s16x2(mn9[3], mn9[4], mn9[5]),
                                       __vimax3_s16x2(mn9[6], mn9[7], mn9[8]));
    const uint32_t a2 = __vimax3_s16x2(__vimax3_s16x2(mn9[9], mn9[10], mn9[11]),
                                       __vimax3_s16x2(mn9[12], mn9[13], mn9[14]), mn9[15]);
    maxmin = __vimax3_s16x2(a1, a2, a2) ^ 0x80008000u;  // max_s min9(r), offset-binary
  }
  {
    uint32_t mx3[16];
#pragma unroll
    for (int k = 0; k < 16; k++) mx3[k] = __vimax3_s16x2(r[k], r[(k + 1) & 15], r[(k + 2) & 15]);
    uint32_t mx9[16];
#pragma unroll
    for (int s = 0; s < 16; s++) mx9[s] = __vimax3_s16x2(mx3[s], mx3[(s + 3) & 15], mx3[(s + 6) & 15]);
    const uint32_t z1 = __vimin3_s16x2(__vimin3_s16x2(mx9[0], mx9[1], mx9[2]), __vimin3_s16x2(mx9[3], mx9[4], mx9[5]),
                                       __vimin3_s16x2(mx9[6], mx9[7], mx9[8]));
    const uint32_t z2 = __vimin3_s16x2(__vimin3_s16x2(mx9[9], mx9[10], mx9[11]),
                                       __vimin3_s16x2(mx9[12], mx9[13], mx9[14]), mx9[15]);
    minmax = __vimin3_s16x2(z1, z2, z2) ^ 0x80008000u;  // min_s max9(r), offset-binary
  }
  // offset-binary (s16 + 32768, order preserving) makes the differences lane-local:
  // (x + 32768) + 256 - (y + 32768) = x - y + 256 in [1, 511], never borrowing across lanes
  const uint32_t cb = c ^ 0x80008000u;
  const uint32_t bright = maxmin + 0x01000100u - cb;                 // 256 + max_s min9(r) - c
  const uint32_t dark = cb + 0x01000100u - minmax;                   // 256 + c - min_s max9(r)
  return __vimax3_u16x2(bright, dark, 0x01000100u);
}

// Sign-replicating byte-permute selector: lanes = bytes (i, j) of the 8-byte window {b:a},
// each sign-extended to 16 bits.
__host__ __device__ constexpr uint32_t sx_sel(int i, int j) {
  return (uint32_t)i | (uint32_t)(i | 8) << 4 | (uint32_t)j << 8 | (uint32_t)(j | 8) << 12;
}
// PTX prmt: a selector nibble with bit 3 set replicates the sign of the selected byte (the
// __byte_perm intrinsic masks bit 3 away, so this is inline PTX)
template <uint32_t SEL>
__device__ __forceinline__ uint32_t prmt_sx(uint32_t a, uint32_t b) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "n"(SEL));
  return r;
}

// Ring value pair of ring offset dx for pixels (q, q + 2) (q = 0: pixels 0, 2; q = 1: 1, 3)
// from one row's words w0..w2 (bytes 0..11 <-> columns gx-4 .. gx+7): bytes 4+q+dx, 6+q+dx.
template <int Q, int DX>
__device__ __forceinline__ uint32_t ring_pair(uint32_t w0, uint32_t w1, uint32_t w2) {
  constexpr int b = 4 + Q + DX;  // first byte, 1..8
  if constexpr (b <= 3) return prmt_sx<sx_sel(b, b + 2)>(w0, w1);
  else if constexpr (b <= 7) return prmt_sx<sx_sel(b - 4, b - 2)>(w1, w2);
  else return prmt_sx<sx_sel(b - 8, b - 6)>(w2, w2);
}

// M of 4 horizontally adjacent pixels from the 7-row window W[dy + 3][0..2] (columns
// gx-4 .. gx+7 of rows y-3 .. y+3, bytes XOR 0x80), packed as 4 bytes (pixel i in byte i).
template <int Q>
__device__ __forceinline__ uint32_t fast_M2(const uint32_t (&W)[7][3]) {
  uint32_t r[16];
  // OpenCV offsets16 order: (dx, dy)
  r[0] = ring_pair<Q, 0>(W[6][0], W[6][1], W[6][2]);    // ( 0, 3)
  r[1] = ring_pair<Q, 1>(W[6][0], W[6][1], W[6][2]);    // ( 1, 3)
  r[2] = ring_pair<Q, 2>(W[5][0], W[5][1], W[5][2]);    // ( 2, 2)
  r[3] = ring_pair<Q, 3>(W[4][0], W[4][1], W[4][2]);    // ( 3, 1)
  r[4] = ring_pair<Q, 3>(W[3][0], W[3][1], W[3][2]);    // ( 3, 0)
  r[5] = ring_pair<Q, 3>(W[2][0], W[2][1], W[2][2]);    // ( 3,-1)
  r[6] = ring_pair<Q, 2>(W[1][0], W[1][1], W[1][2]);    // ( 2,-2)
  r[7] = ring_pair<Q, 1>(W[0][0], W[0][1], W[0][2]);    // ( 1,-3)
  r[8] = ring_pair<Q, 0>(W[0][0], W[0][1], W[0][2]);    // ( 0,-3)
  r[9] = ring_pair<Q, -1>(W[0][0], W[0][1], W[0][2]);   // (-1,-3)
  r[10] = ring_pair<Q, -2>(W[1][0], W[1][1], W[1][2]);  // (-2,-2)
  r[11] = ring_pair<Q, -3>(W[2][0], W[2][1], W[2][2]);  // (-3,-1)
  r[12] = ring_pair<Q, -3>(W[3][0], W[3][1], W[3][2]);  // (-3, 0)
  r[13] = ring_pair<Q, -3>(W[4][0], W[4][1], W[4][2]);  // (-3, 1)
  r[14] = ring_pair<Q, -2>(W[5][0], W[5][1], W[5][2]);  // (-2, 2)
  r[15] = ring_pair<Q, -1>(W[6][0], W[6][1], W[6][2]);  // (-1, 3)
  return arc_score2(r, ring_pair<Q, 0>(W[3][0], W[3][1], W[3][2]));
}

__device__ __forceinline__ uint32_t fast_M4(const uint32_t (&W)[7][3]) {
  const uint32_t slo = fast_M2<0>(W);  // pixels 0, 2 (M + 256 per lane)
  const uint32_t shi = fast_M2<1>(W);  // pixels 1, 3
  return __byte_perm(slo, shi, 0x6240);
}

// 4-bit column mask of one NMS step from the two 16x2 half results (bit 15 / 31 of h0 =
// pixels 0 / 2, of h1 = pixels 1 / 3): bits 0..3 = pixels 0..3
__device__ __forceinline__ uint32_t nibble4(uint32_t h0, uint32_t h1) {
  const uint32_t t = (h0 >> 15) | (h1 >> 14);  // bits 0, 16 (pixels 0, 2) and 1, 17 (pixels 1, 3)
  return (t | (t >> 14)) & 0xFu;
}

// Scores of a staged band: task t = (4-pixel group t % ng, rows [ROWS * (t / ng), + ROWS)),
// a sliding 7-row register window per task (3 shared loads per row step).
template <int ROWS>
__device__ __forceinline__ void score_band(const uint8_t* reg, int rp, uint8_t* Mb, int mbw, int g0, int ng, int Dh) {
  const int nrt = (Dh + ROWS - 1) / ROWS;
  for (int t = threadIdx.x; t < ng * nrt; t += FB_THREADS) {
    const int gc = g0 + 4 * (t % ng);
    const int ys = (t / ng) * ROWS;
    uint32_t W[7][3];
    // staged row of band row y is y + 3; rows y-3..y+3 -> staged rows y..y+6
#pragma unroll
    for (int r = 0; r < 6; r++) {
      const uint32_t* p = reinterpret_cast<const uint32_t*>(reg + (ys + r) * rp + gc - 4);
      W[r + 1][0] = p[0];
      W[r + 1][1] = p[1];
      W[r + 1][2] = p[2];
    }
#pragma unroll
    for (int i = 0; i < ROWS; i++) {  // fully unrolled: the window shift is renaming
      const int y = ys + i;
      if (y >= Dh) break;
#pragma unroll
      for (int r = 0; r < 6; r++) {
        W[r][0] = W[r + 1][0];
        W[r][1] = W[r + 1][1];
        W[r][2] = W[r + 1][2];
      }
      const uint32_t* p = reinterpret_cast<const uint32_t*>(reg + (y + 6) * rp + gc - 4);
      W[6][0] = p[0];
      W[6][1] = p[1];
      W[6][2] = p[2];
      *reinterpret_cast<uint32_t*>(Mb + (y + 1) * mbw + gc) = fast_M4(W);
    }
  }
}

// Strict 8-neighbour maxima of a band's score map into the bit planes (same task layout as
// score_band): see step 3 of the kernel.
template <int ROWS>
__device__ __forceinline__ void nms_band(const uint8_t* Mb, int mbw, uint32_t* bits, int bw, const uint32_t* starts,
                                         int g0, int ng, int Dh, int tmin, int tini) {
  const int nrt = (Dh + ROWS - 1) / ROWS;
  const uint32_t tmin1 = (uint32_t)(tmin + 1) * 0x10001u, tini1 = (uint32_t)(tini + 1) * 0x10001u;
  for (int t = threadIdx.x; t < ng * nrt; t += FB_THREADS) {
    const int gc = g0 + 4 * (t % ng);
    const int ys = (t / ng) * ROWS;
    // cell starts at columns gc .. gc + 4 -> lane masks of valid left / right neighbours
    const uint32_t sw5 = (uint32_t)(__funnelshift_r(starts[gc >> 5], starts[(gc >> 5) + 1], gc & 31)) & 0x1Fu;
    uint32_t mL[2], mR[2];
#pragma unroll
    for (int hv = 0; hv < 2; hv++) {  // pixels (hv, hv + 2)
      mL[hv] = ((sw5 >> hv) & 1u ? 0u : 0xFFFFu) | ((sw5 >> (hv + 2)) & 1u ? 0u : 0xFFFF0000u);
      mR[hv] = ((sw5 >> (hv + 1)) & 1u ? 0u : 0xFFFFu) | ((sw5 >> (hv + 3)) & 1u ? 0u : 0xFFFF0000u);
    }
    // per half: hf / hlr of rows y - 1 and y, the centre of row y
    uint32_t hfp[2], hf0[2], hl0[2], c0[2];
    auto rowq = [&](int y, uint32_t (&hf)[2], uint32_t (&hl)[2], uint32_t (&cc)[2]) {
      const uint32_t* pr = reinterpret_cast<const uint32_t*>(Mb + (y + 1) * mbw + gc - 4);
      const uint32_t wp = pr[0], wc = pr[1], wn = pr[2];
      const uint32_t Lw = __byte_perm(wp, wc, 0x6543), Rw = __byte_perm(wc, wn, 0x4321);
#pragma unroll
      for (int hv = 0; hv < 2; hv++) {
        const uint32_t sel = hv ? 0x7371u : 0x7270u;
        const uint32_t Ch = __byte_perm(wc, 0, sel);
        const uint32_t Lh = __byte_perm(Lw, 0, sel) & mL[hv], Rh = __byte_perm(Rw, 0, sel) & mR[hv];
        hl[hv] = __vmaxu2(Lh, Rh);
        hf[hv] = __vimax3_u16x2(Lh, Rh, Ch);
        cc[hv] = Ch;
      }
    };
    {
      uint32_t dummy[2];
      rowq(ys - 1, hfp, dummy, dummy);  // row -1 reads the zero row
      rowq(ys, hf0, hl0, c0);
    }
    uint32_t* bmin = bits + gc / 32;
    const int bsh = gc & 31;
#pragma unroll
    for (int i = 0; i < ROWS; i++) {
      const int y = ys + i;
      if (y >= Dh) break;
      uint32_t hfn[2], hln[2], cn[2];
      rowq(y + 1, hfn, hln, cn);  // row Dh reads the zero row
      uint32_t ok[2], oi[2];
#pragma unroll
      for (int hv = 0; hv < 2; hv++) {
        const uint32_t nb = __vimax3_u16x2(hfp[hv], hl0[hv], hfn[hv]);
        const uint32_t C = c0[hv] | 0x80008000u;
        ok[hv] = (C - nb - 0x00010001u) & (C - tmin1) & 0x80008000u;  // > neighbours, > minTh
        oi[hv] = ok[hv] & (C - tini1);                                // and > iniTh
        hfp[hv] = hf0[hv];
        hf0[hv] = hfn[hv];
        hl0[hv] = hln[hv];
        c0[hv] = cn[hv];
      }
      const uint32_t km = nibble4(ok[0], ok[1]), ki = nibble4(oi[0], oi[1]);
      if (km) atomicOr(bmin + y * bw, km << bsh);
      if (ki) atomicOr(bmin + (Dh + y) * bw, ki << bsh);
    }
  }
}

__global__ void __launch_bounds__(FB_THREADS, FB_MIN_BLOCKS) fast_bands_kernel(const __grid_constant__ Geom g, FrameSrc src,
                                                                const BandInfo* __restrict__ bands,
                                                                const CellInfo* __restrict__ cells,
                                                                uint32_t* __restrict__ slots,
                                                                int32_t* __restrict__ cell_counts, int rp, int mbw,
                                                                int region_bytes, int bits_off, int flat_frames) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // 2-D grid (band, frame), or flat band-major (flat_frames = F: CTA i = band i / F, frame i % F,
  // so the band order -- longest first -- holds across frames too)
  const int bi = flat_frames ? (int)blockIdx.x / flat_frames : (int)blockIdx.x;
  const BandInfo bd = bands[bi];  // static (ss_create): readable before the dependency wait
  // Level 0 reads only the caller's frames, which are complete before the pyramid (the kernel
  // this one depends on) passed its own dependency wait -- and this grid launches only after
  // the pyramid's trigger -- so level-0 CTAs run beside the pyramid; the other levels wait for
  // it (as level 0's separate launch on a side branch did in round 1, without the extra launch).
  if (bd.level != 0) pdl_wait();
  if (SS_FAST_TRIGGER == 0) pdl_trigger();
  const int f = flat_frames ? (int)blockIdx.x % flat_frames : (int)blockIdx.y;
  FAST_TS(0);
  const int l = bd.level;
  const int tmin = g.min_th, tini = g.ini_th;
  const uint8_t* img;
  int ip;
  if (l == 0) {
    img = src.frames + (int64_t)f * src.stride;
    ip = src.pitch;
  } else {
    img = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    ip = g.pitch[l];
  }
  uint8_t* reg = smem;                 // [Dh + 6][rp] staged band; staged column s <-> level column xa + s
  uint8_t* Mb = smem + region_bytes;   // [Dh + 2][mbw] scores; same columns, zero rows above/below
  const int Dh = bd.y1 - bd.y0;
  const int xa = ((bd.x0 - 3) & ~15) - 16;              // >= 0: x0 >= 19
  const int g0 = ((bd.x0 - xa) & ~3), g1 = (bd.x1 - xa + 3) & ~3;  // 4-px groups covering [x0, x1)
  const int sw = (g1 + 4 + 15) & ~15;                   // staged columns [0, sw)
  const uint8_t* row0 = img + (int64_t)(bd.y0 - 3) * ip + xa;
  // ---- 1. stage rows y0-3 .. y1+2, columns xa .. xa+sw-1 (all inside the level row) ----
  const int nchunk = sw >> 4;
  // NMS bit planes: [2][Dh][bw] words (bit s of row y = staged column s is a maximum above
  // minTh / above iniTh), then the cell-start columns [bw]; zeroed here, set by atomicOr
  const int bw = (mbw + 31) / 32 + 2;
  uint32_t* bits = reinterpret_cast<uint32_t*>(smem + bits_off);
  uint32_t* starts = bits + 2 * Dh * bw;
  for (int i = threadIdx.x; i < (2 * Dh + 1) * bw; i += FB_THREADS) bits[i] = 0u;
  if ((ip & 15) == 0 && (reinterpret_cast<uintptr_t>(img) & 15) == 0) {
    const uint32_t inv = 0xFFFFFFFFu / (uint32_t)nchunk + 1u;  // i / nchunk = umulhi(i, inv) for i < 2^16
    for (int i = threadIdx.x; i < (Dh + 6) * nchunk; i += FB_THREADS) {
      const int r = (int)__umulhi((uint32_t)i, inv), c = i - r * nchunk;
      uint4 v = __ldg(reinterpret_cast<const uint4*>(row0 + (int64_t)r * ip) + c);
      v.x ^= 0x80808080u, v.y ^= 0x80808080u, v.z ^= 0x80808080u, v.w ^= 0x80808080u;  // bytes as I - 128
      *reinterpret_cast<uint4*>(reg + r * rp + 16 * c) = v;
    }
  } else {
    for (int i = threadIdx.x; i < (Dh + 6) * sw; i += FB_THREADS) {
      const int r = i / sw, c = i - r * sw;
      reg[r * rp + c] = __ldg(row0 + (int64_t)r * ip + c) ^ 0x80;
    }
  }
  // zero border rows of the score map
  for (int i = threadIdx.x; i < mbw / 4; i += FB_THREADS) {
    reinterpret_cast<uint32_t*>(Mb)[i] = 0u;
    reinterpret_cast<uint32_t*>(Mb + (Dh + 1) * mbw)[i] = 0u;
  }
  __syncthreads();
  FAST_TS(1);
  // cell-start columns (and the band's end): a pixel's left neighbour is in its cell unless its
  // column starts a cell, its right neighbour unless the next column does
  if (threadIdx.x <= bd.ncells) {
    const int sc = (threadIdx.x < bd.ncells ? cells[bd.cell_first + threadIdx.x].x0 : bd.x1) - xa;
    atomicOr(&starts[sc >> 5], 1u << (sc & 31));
  }
  // ---- 2. scores of all band pixels, 4 per thread, ROWS rows per task: 8, or 4 when 8-row
  // tasks would leave half the CTA's threads without one (level-0 segments of <= 4 cells) ----
  {
    const int ng = (g1 - g0) >> 2;
    if (ng * ((Dh + 7) / 8) * 2 <= FB_THREADS)
      score_band<4>(reg, rp, Mb, mbw, g0, ng, Dh);
    else
      score_band<ROWS_PER_TASK>(reg, rp, Mb, mbw, g0, ng, Dh);
  }
  __syncthreads();
  FAST_TS(2);
  if (SS_FAST_TRIGGER == 2) pdl_trigger();
  // ---- 3. strict 8-neighbour maxima above minTh / iniTh, every thread on 4-pixel groups of
  // ROWS_PER_TASK rows (the score tasks' layout), into the bit planes: per 16x2 half (pixels
  // 0, 2 or 1, 3) the horizontal 3-max hf and left/right max hlr of each row are formed once
  // (neighbours in another cell masked to 0: per-cell ROI semantics; rows -1 and Dh are the
  // score map's zero rows) and row y tests C > max(hf(y-1), hlr(y), hf(y+1)) ----
  {
    const int ng = (g1 - g0) >> 2;
    if (ng * ((Dh + 7) / 8) * 2 <= FB_THREADS)
      nms_band<4>(Mb, mbw, bits, bw, starts, g0, ng, Dh, tmin, tini);
    else
      nms_band<ROWS_PER_TASK>(Mb, mbw, bits, bw, starts, g0, ng, Dh, tmin, tini);
  }
  __syncthreads();
  FAST_TS(3);
  if (SS_FAST_TRIGGER == 3) pdl_trigger();
  // ---- 4. per cell (warp), per row (lane): the cell's threshold (iniTh if any maximum beats
  // it, else minTh) and the survivors in raster order (warp prefix sum of the row counts) ----
  for (int j = warp; j < bd.ncells; j += FB_WARPS) {
    const int ci = bd.cell_first + j;
    const CellInfo c = cells[ci];
    const int cx0 = c.x0 - xa, cw = c.x1 - c.x0;  // staged columns [cx0, cx0 + cw), cw < 64
    const unsigned long long cm = cw >= 64 ? ~0ull : (1ull << cw) - 1ull;
    unsigned long long kmin[2] = {0ull, 0ull}, kini[2] = {0ull, 0ull};
#pragma unroll
    for (int hh = 0; hh < 2; hh++) {
      const int y = lane + 32 * hh;
      if (y < Dh) {
        const uint32_t* r0 = bits + y * bw + (cx0 >> 5);
        const uint32_t* r1 = bits + (Dh + y) * bw + (cx0 >> 5);
        const int sh = cx0 & 31;
        kmin[hh] = (((unsigned long long)__funnelshift_r(r0[1], r0[2], sh) << 32) | __funnelshift_r(r0[0], r0[1], sh)) & cm;
        kini[hh] = (((unsigned long long)__funnelshift_r(r1[1], r1[2], sh) << 32) | __funnelshift_r(r1[0], r1[1], sh)) & cm;
      }
    }
    const bool any_ini = __any_sync(0xFFFFFFFFu, (kini[0] | kini[1]) != 0ull);
    uint32_t* out = slots + (int64_t)f * g.slots_per_frame + c.slot_off;
    int base = 0;
#pragma unroll
    for (int hh = 0; hh < 2; hh++) {
      unsigned long long sel = any_ini ? kini[hh] : kmin[hh];
      const int cnt = __popcll(sel);
      int incl = cnt;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(0xFFFFFFFFu, incl, o);
        if (lane >= o) incl += v;
      }
      int pos = base + incl - cnt;
      const int y = lane + 32 * hh;
      while (sel) {
        const int x = __ffsll((long long)sel) - 1;
        sel &= sel - 1;
        out[pos++] = pack_key(c.x0 + x, bd.y0 + y, Mb[(y + 1) * mbw + cx0 + x]);
      }
      base += __shfl_sync(0xFFFFFFFFu, incl, 31);
    }
    if (lane == 0) cell_counts[(int64_t)f * g.total_cells + ci] = base;
  }
#ifdef SS_FAST_PHASES
  __syncthreads();
  FAST_TS(4);
  if (threadIdx.x == 0 && blockIdx.y * gridDim.x + blockIdx.x < 4096) {
    unsigned smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    g_fast_ts[bd.level != 0][blockIdx.y * gridDim.x + blockIdx.x][5] = smid;
  }
#endif
}

}  // namespace

size_t fast_smem_bytes(const Geom& g, int* rp, int* mbw, int* region_bytes, int* mband_bytes, int* nball) {
  // staged columns: up to 16 + 15 lead-in, the band, 4-px group round-up and a 4-B right guard
  const int sw = ((g.max_band_w + 31 + 3 + 4 + 4) + 15) & ~15;
  *rp = sw + 16;
  *region_bytes = ((g.max_band_h + 6) * *rp + 15) & ~15;
  int m = (sw + 8 + 3) & ~3;  // + 8: the NMS reads 8 scores per step past a cell's last column
  if (((m >> 2) & 1) == 0) m += 4;  // odd word pitch: lane-per-row reads hit distinct banks
  *mbw = m;
  *mband_bytes = ((g.max_band_h + 2) * m + 16 + 15) & ~15;  // + 16: the NMS word reads pass the last row
  const int bw = (m + 31) / 32 + 2;  // bit-plane words per row (+ 2: the 64-bit cell reads)
  *nball = *region_bytes + *mband_bytes;  // bit planes [2][max_band_h][bw] + cell starts [bw]
  return (size_t)*nball + (size_t)(2 * g.max_band_h + 1) * bw * 4;
}

#ifdef SS_FAST_PHASES
extern "C" int ss_dbg_fast_ts(unsigned long long* out) {  // [2][4096][8]
  return (int)cudaMemcpyFromSymbol(out, g_fast_ts, sizeof(g_fast_ts));
}
#endif

cudaError_t fast_init() {  // ss_create, per device; ss_create rejects bands above 227 KB
  cudaError_t e = carveout_from_env(fast_bands_kernel);
  if (e != cudaSuccess) return e;
  return set_max_dynamic_smem(fast_bands_kernel);
}

cudaError_t launch_fast_bands(const Geom& g, int n_frames, FrameSrc src, const BandInfo* bands, int n_bands,
                              const CellInfo* cells, uint32_t* slots, int32_t* cell_counts, cudaStream_t s,
                              bool flat) {
  if (n_bands <= 0) return cudaSuccess;
  int rp, mbw, rb, mb, nb;
  const size_t smem = fast_smem_bytes(g, &rp, &mbw, &rb, &mb, &nb);
  const dim3 grid = flat ? dim3(n_bands * n_frames) : dim3(n_bands, n_frames);
  cudaError_t e = launch_pdl(fast_bands_kernel, grid, dim3(FB_THREADS), smem, s, g, src, bands, cells, slots,
                             cell_counts, rp, mbw, rb, nb, flat ? n_frames : 0);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
