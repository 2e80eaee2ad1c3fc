// k_describe.cu -- S5+S6+S7+S8: orientation, 7x7 blur, rotated BRIEF and output packing
// (DESIGN.md §3 O5-O8; "Oriented FAST and Rotated BRIEF").
//
// One warp per output keypoint slot.  The warp stages the 43x43 raw patch around the
// keypoint (REFLECT_101 at the level border, which the blur needs) in shared memory and
// derives everything from it: intensity-centroid moments over the 749-px disk (unblurred),
// the vertical blur pass over the patch (Q8 taps [18,34,48,56,48,34,18], exact sums, two
// columns per register), and the 256 comparisons at the pattern points rotated by
// (cos, sin) = (m10, m01)/sqrt(m10^2 + m01^2), each offset rounded half-to-even EXACTLY (f32
// estimate; int64 test only within 1e-4 of a tie), with the horizontal blur pass and the
// (sum + 2^15) >> 16 rounding evaluated at the 512 sample points only.  Blurring only what
// the samples read replaces a whole-level blur pass and its HBM round trip.  Output
// position = the keypoint's canonical index, so the per-level counts of the distribution
// become the prefix offsets written to d_counts.
#include <cudaTypedefs.h>  // PFN_cuTensorMapEncodeTiled

#include "brief_pattern.inc"
#include "ss_internal.h"

namespace ss {

#ifdef SS_DESC_PHASES  // per-warp phase timestamps (scripts/desc_phases.py; instrumented builds only)
__device__ unsigned long long g_desc_ts[16384][8];
#define DESC_TS(i)                                                                   \
  do {                                                                               \
    const int w_ = (blockIdx.y * gridDim.x + blockIdx.x) * DESC_WARPS + (threadIdx.x >> 5); \
    if ((threadIdx.x & 31) == 0 && w_ < 16384) {                                     \
      unsigned long long t_;                                                         \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                         \
      g_desc_ts[w_][i] = t_;                                                         \
    }                                                                                \
  } while (0)
#define DESC_PATH(v)                                                                 \
  do {                                                                               \
    const int w_ = (blockIdx.y * gridDim.x + blockIdx.x) * DESC_WARPS + (threadIdx.x >> 5); \
    if ((threadIdx.x & 31) == 0 && w_ < 16384) g_desc_ts[w_][7] = (v) | ((unsigned long long)l << 8); \
  } while (0)
#else
#define DESC_TS(i) \
  do {             \
  } while (0)
#define DESC_PATH(v) \
  do {               \
  } while (0)
#endif

namespace {

#ifndef SS_DESC_WARPS
#define SS_DESC_WARPS 4  // 4 vs 6 vs 8: c2 describe 18.9 / 19.6 / 19.8 us (scripts/ab_descwarps.sh)
#endif
constexpr int DESC_WARPS = SS_DESC_WARPS;  // warps (keypoints in flight) per CTA
constexpr int PR = 43;  // raw patch: radius 21 (18 max sample offset + 3 blur taps)
constexpr int PP = 64;  // raw patch pitch: a 16-B aligned 64-B window covers the 43 B row
constexpr int BR = 37;  // blurred patch: radius 18
constexpr int VP = 46;  // pitch (u16) of the vertical pass V[37][43]: 23 words (odd) per row
constexpr int PER_WARP = ((PR * PP + BR * VP * 2) + 127) & ~127;

__constant__ int c_umax[16] = {15, 15, 15, 15, 14, 14, 14, 13, 13, 12, 11, 10, 9, 8, 6, 3};

__device__ __forceinline__ int reflect101(int i, int n) {
  i = i < 0 ? -i : i;
  return i >= n ? 2 * n - 2 - i : i;
}

// Exact round-half-even of z / sqrt(r2), r2 > 0, |z| < 2^31.  Fast path: t = z * (1/r) in
// f32 is within 4e-6 of z/r (|z/r| <= 19), so rint(t) is the exact answer unless t lies
// within 1e-4 of a half-integer; then the integer test (2k-1)^2 r2 < 4 z^2 <= (2k+1)^2 r2
// selects k and a tie 4z^2 == (2k+1)^2 r2 goes to even.
__device__ __noinline__ int rhe_exact(long long z, long long r2, int k) {
  const long long a = z < 0 ? -z : z;
  const long long A = 4 * a * a;
  k = k < 0 ? -k : k;
  while (k > 0 && (long long)(2 * k - 1) * (2 * k - 1) * r2 >= A) k--;
  while ((long long)(2 * k + 1) * (2 * k + 1) * r2 < A) k++;
  if ((k & 1) && (long long)(2 * k + 1) * (2 * k + 1) * r2 == A) k++;
  return z < 0 ? -k : k;
}

// round-half-even of (a * m_a + b * m_b) / r for the rotated pattern offsets, r^2 = r2 > 0:
// t = a * ca + b * cb in f32 (ca = m_a / r, cb = m_b / r; |t| <= 19, error < 1e-5), rounded
// with the 1.5 * 2^23 trick (round-to-nearest-even, no conversion instructions); within 1e-4
// of a half-integer the exact integer test decides.
__device__ __forceinline__ int rhe_rot(int a, int b, float ca, float cb, int ma, int mb, long long r2) {
  const float t = __fmaf_rn((float)a, ca, __fmul_rn((float)b, cb));
  const float big = __fadd_rn(t, 12582912.0f);
  const int k = __float_as_int(big) - 0x4B400000;
  const float d = __fsub_rn(t, __fsub_rn(big, 12582912.0f));
  if (fabsf(fabsf(d) - 0.5f) > 1e-4f) return k;
  return rhe_exact((long long)a * ma + (long long)b * mb, r2, k);
}

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// A 43-row x 64-byte box (rows y.., columns x.., x a multiple of 16) of frame f's level by one
// TMA tensor copy into the warp's buffer (lane 0 issues; the warp waits on its mbarrier).
__device__ __forceinline__ void tma_patch(const CUtensorMap* map, uint8_t* dst, uint64_t* bar, int x, int y, int f,
                                          int lane) {
  const uint32_t b = smem_addr(bar);
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(kPatchBoxW * kPatchBoxH)
                 : "memory");
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
        "[%5];" ::"r"(smem_addr(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(f), "r"(b)
        : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "TMA_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t"
      "@!P1 bra TMA_WAIT_%=;\n}" ::"r"(b)
      : "memory");
}

// SAMPLES (test hook, ss_debug_capture_samples): also write the blurred value of every sample
// point the comparisons read, samples[slot][b][e] for bit b = 8 * lane + t, point e
template <bool SAMPLES>
__global__ void __launch_bounds__(DESC_WARPS * 32, 32 / DESC_WARPS) describe_kernel(Geom g, FrameSrc src,
                                                                   const uint32_t* __restrict__ selected,
                                                                   const int32_t* __restrict__ sel_counts,
                                                                   const int8_t* __restrict__ pattern,
                                                                   ss_keypoint* __restrict__ kps,
                                                                   uint8_t* __restrict__ desc,
                                                                   int32_t* __restrict__ counts,
                                                                   uint8_t* __restrict__ samples,
                                                                   const __grid_constant__ PatchMaps maps) {
#ifndef SS_DESC_LATE_TRIGGER
  pdl_trigger();
#endif
  DESC_TS(0);
  extern __shared__ __align__(128) uint8_t sm_raw[];  // DESC_WARPS * PER_WARP + 128
  // 128-B aligned warp buffers (TMA destinations)
  uint8_t* const sm = sm_raw + ((128 - (smem_addr(sm_raw) & 127)) & 127);
  __shared__ __align__(8) uint64_t s_bar[DESC_WARPS];
  __shared__ int off[kMaxLevels + 1];
  __shared__ __align__(16) uint32_t s_wmask[16 * 8], s_wu[16 * 8];  // per |v|: 32 byte weights
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int f = blockIdx.y;
  const int L = g.L;
  // Constant inputs (set at ss_create) are read before the dependency wait, overlapping the
  // predecessor kernel's tail.  Lane = output byte: its 8 pairs are the 32 pattern bytes
  // 32 * lane .. 32 * lane + 31, one word (px0, py0, px1, py1) per bit, held in registers.
  // the lane's 16 pattern points as floats in shared memory, point j of lane at [j][lane]
  // (conflict-free LDS.64): point 2t + e of output byte `lane` is pattern point 16 lane + j
  __shared__ float2 s_pat[16 * 32];
  for (int i = threadIdx.x; i < 16 * 32; i += DESC_WARPS * 32) {
    const int ln = i & 31, j = i >> 5, pt = 16 * ln + j;
    s_pat[i] = make_float2((float)__ldg(pattern + 2 * pt), (float)__ldg(pattern + 2 * pt + 1));
  }
  for (int it = threadIdx.x; it < 256; it += DESC_WARPS * 32) {  // byte j = u + 15 of row |v|: inside the disk -> (1, u + 15), else 0
    const int t = it >> 7, av = (it >> 3) & 15, k = it & 7;
    uint32_t word = 0;
    for (int b = 0; b < 4; b++) {
      const int j = 4 * k + b, u = j - 15;
      if (j <= 30 && u >= -c_umax[av] && u <= c_umax[av]) word |= (uint32_t)(t ? j : 1) << (8 * b);
    }
    (t ? s_wu : s_wmask)[(it & 127)] = word;
  }
  pdl_wait();
  DESC_TS(1);
  if (warp == 0) {  // level offsets: the L counts loaded at once, inclusive warp scan
    int s = lane < L ? sel_counts[f * L + lane] : 0;
#pragma unroll
    for (int o = 1; o < kMaxLevels; o <<= 1) {
      const int v = __shfl_up_sync(0xFFFFFFFFu, s, o);
      if (lane >= o) s += v;
    }
    if (lane < L) off[lane + 1] = s;
    if (lane == 0) off[0] = 0;
  }
  __syncthreads();
  if (blockIdx.x == 0 && threadIdx.x <= L) counts[f * (L + 1) + threadIdx.x] = off[threadIdx.x];
  const int i = blockIdx.x * DESC_WARPS + warp;
  if (i >= off[L]) return;  // warp-uniform; only warp-level sync below
  DESC_TS(2);
  int l = 0;
  while (i >= off[l + 1]) l++;
  const uint32_t packed = selected[(int64_t)f * g.kp_capacity + g.cap_off[l] + (i - off[l])];
  const int lx = key_lx(packed), ly = key_ly(packed), M = key_m(packed);
  const uint8_t* img;
  int ip;
  if (l == 0) {
    img = src.frames + (int64_t)f * src.stride;
    ip = src.pitch;
  } else {
    img = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    ip = g.pitch[l];
  }
  const int w = g.w[l], h = g.h[l];
  uint8_t* Pw = sm + warp * PER_WARP;
  uint16_t* V = reinterpret_cast<uint16_t*>(Pw + PR * PP);
  const uint8_t* p0 = img + (int64_t)(ly - 21) * ip + (lx - 21);
  const int sh = (int)(reinterpret_cast<uintptr_t>(p0) & 15);
  const uint8_t* P;  // P[r * PP + c] = raw patch pixel (ly - 21 + r, lx - 21 + c)
  if (((maps.valid >> l) & 1u) && lx >= 21 && lx + 21 < w && ly >= 21 && ly + 21 < h) {
    // the patch lies inside the level (no REFLECT_101 needed): one TMA tensor copy of 43 rows
    // x 64 columns from the 16-B aligned column at or left of lx - 21 (a u8 tile's innermost
    // coordinate must be 16-B aligned: measured, scripts/micro/tma_probe2.cu); columns past the
    // level edge arrive as zeros and are never read
    const int x0 = lx - 21;
    tma_patch(&maps.level[l], Pw, &s_bar[warp], x0 & ~15, ly - 21, f, lane);
    P = Pw + (x0 & 15);
    DESC_PATH(1);
  } else if ((ip & 15) == 0 && lx >= 21 && lx + 21 < w && lx - 21 - sh + 64 <= ip) {
    // columns inside the level: 43 rows x four aligned 16-B chunks, rows mapped by REFLECT_101
    // (identity away from the top/bottom border); all six loads of a lane are issued before
    // the first store (one global latency, not six)
    const uint8_t* cb = img + (lx - 21 - sh);
    const bool rows_in = ly >= 21 && ly + 21 < h;
    constexpr int NCH = (PR * 4 + 31) / 32;
    uint4 chunk[NCH];
#pragma unroll
    for (int k = 0; k < NCH; k++) {
      const int i = lane + 32 * k;
      if (i < PR * 4) {
        const int r = i >> 2, sr = rows_in ? ly - 21 + r : reflect101(ly - 21 + r, h);
        chunk[k] = __ldg(reinterpret_cast<const uint4*>(cb + (int64_t)sr * ip) + (i & 3));
      }
    }
#pragma unroll
    for (int k = 0; k < NCH; k++) {
      const int i = lane + 32 * k;
      if (i < PR * 4) *reinterpret_cast<uint4*>(Pw + (i >> 2) * PP + 16 * (i & 3)) = chunk[k];
    }
    P = Pw + sh;
    DESC_PATH(2);
  } else if ((ip & 15) == 0 && w >= 22) {
    // near the left/right level border (round 2; was per-byte REFLECT_101 loads in 8 dependent
    // batches, the describe launch's slowest warps): the 16-B chunks of the aligned 64-column
    // window from the patch's first in-level column (chunks past the row's end skipped), rows
    // mapped by REFLECT_101, stored 16 B to the right when the patch starts left of column 0;
    // then the <= 3 reflected columns per row are copied in shared memory (a row's slot is
    // 64 B: the shifted row's unused last columns and the next row's left pad overlap)
    const int a0 = max(lx - 21, 0) & ~15;
    const int sft = lx < 21 ? 16 : 0;
    const uint8_t* cb = img + a0;
    constexpr int NCH = (PR * 4 + 31) / 32;
    uint4 chunk[NCH];
#pragma unroll
    for (int k = 0; k < NCH; k++) {
      const int i = lane + 32 * k;
      if (i < PR * 4 && a0 + 16 * (i & 3) < ip)
        chunk[k] = __ldg(reinterpret_cast<const uint4*>(cb + (int64_t)reflect101(ly - 21 + (i >> 2), h) * ip) + (i & 3));
    }
#pragma unroll
    for (int k = 0; k < NCH; k++) {
      const int i = lane + 32 * k;
      if (i < PR * 4 && a0 + 16 * (i & 3) < ip) *reinterpret_cast<uint4*>(Pw + (i >> 2) * PP + sft + 16 * (i & 3)) = chunk[k];
    }
    __syncwarp();
    for (int r = lane; r < PR; r += 32) {
      uint8_t* row = Pw + r * PP + sft - a0;  // row[x] = pixel column x of this patch row
      for (int x = lx - 21; x < 0; x++) row[x] = row[-x];                     // REFLECT_101, left
      for (int x = w; x <= lx + 21; x++) row[x] = row[2 * w - 2 - x];        // REFLECT_101, right
    }
    __syncwarp();
    P = Pw + sft + (lx - 21 - a0);
    DESC_PATH(3);
  } else {
    // tiny levels or an unaligned pitch: REFLECT_101 (the blur's border rule) byte loads, 8 per
    // lane in flight per batch
    constexpr int BB = 8;
#pragma unroll 1
    for (int i0 = 0; i0 < PR * PR; i0 += 32 * BB) {
      uint32_t v[BB];
#pragma unroll
      for (int k = 0; k < BB; k++) {
        const int i = i0 + lane + 32 * k;
        if (i < PR * PR) {
          const int r = i / PR, c = i - r * PR;
          v[k] = __ldg(img + (int64_t)reflect101(ly - 21 + r, h) * ip + reflect101(lx - 21 + c, w));
        }
      }
#pragma unroll
      for (int k = 0; k < BB; k++) {
        const int i = i0 + lane + 32 * k;
        if (i < PR * PR) Pw[(i / PR) * PP + (i % PR)] = (uint8_t)v[k];
      }
    }
    P = Pw;
  }
  __syncwarp();
  DESC_TS(3);
  // moments over the disk |u| <= umax[|v|] (always inside the level: 19 <= lx < w-19):
  // lane = row v; the row's 31 pixels (plus one zero-weight byte) as 8 words, dotted 4 bytes
  // at a time with the disk mask (S0 = sum I) and with weights u + 15 (S1); m10 = sum of
  // S1 - 15 S0, m01 = sum of v S0
  int m10 = 0, m01 = 0;
  {
    if (lane < 31) {
      const int v = lane - 15, av = v < 0 ? -v : v;
      const uint8_t* rp = P + (21 + v) * PP + 6;  // column u = -15
      const uint32_t* wa = reinterpret_cast<const uint32_t*>(reinterpret_cast<uintptr_t>(rp) & ~(uintptr_t)3);
      const uint32_t shb = 8u * (uint32_t)(reinterpret_cast<uintptr_t>(rp) & 3);
      const uint4* wm = reinterpret_cast<const uint4*>(s_wmask + 8 * av);
      const uint4* wu = reinterpret_cast<const uint4*>(s_wu + 8 * av);
      const uint4 m0 = wm[0], m1 = wm[1], u0 = wu[0], u1 = wu[1];
      const uint32_t mk[8] = {m0.x, m0.y, m0.z, m0.w, m1.x, m1.y, m1.z, m1.w};
      const uint32_t uk[8] = {u0.x, u0.y, u0.z, u0.w, u1.x, u1.y, u1.z, u1.w};
      uint32_t w[9];
#pragma unroll
      for (int k = 0; k < 9; k++) w[k] = wa[k];
      unsigned s0 = 0, s1 = 0;
#pragma unroll
      for (int k = 0; k < 8; k++) {
        const uint32_t x = __funnelshift_r(w[k], w[k + 1], shb);
        s0 = __dp4a(x, mk[k], s0);
        s1 = __dp4a(x, uk[k], s1);
      }
      m10 = (int)s1 - 15 * (int)s0;
      m01 = v * (int)s0;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      m10 += __shfl_xor_sync(0xFFFFFFFFu, m10, o);
      m01 += __shfl_xor_sync(0xFFFFFFFFu, m01, o);
    }
  }
  // separable blur; all sums are exact integers until the final rounding, so the vertical
  // pass may come first: V[r][x] = sum_i k_i P[r + i][x] (lane = column, sliding over rows),
  // then B[r][c] = (sum_j k_j V[r][c + j] + 2^15) >> 16 at the sample points (below)
  // pass 1 on packed column pairs: lane covers columns 2*lane, 2*lane + 1 as two 16-bit lanes
  // of one register (a weighted sum is <= 255 * 256, so the halves never carry)
  // column pairs start at an even address: V column x' holds patch column x' - podd
  const int podd = (int)(reinterpret_cast<uintptr_t>(P) & 1);
  if (lane < (PR + 2) / 2) {
    const uint16_t* pc = reinterpret_cast<const uint16_t*>(P - podd) + lane;
    auto ld2 = [&](int r) -> uint32_t {  // bytes (r, 2 lane - podd), (r, 2 lane + 1 - podd) -> (lo16, hi16)
      return __byte_perm((uint32_t)pc[r * (PP / 2)], 0, 0x7170);
    };
    uint32_t q0 = ld2(0), q1 = ld2(1), q2 = ld2(2), q3 = ld2(3), q4 = ld2(4), q5 = ld2(5);
    uint32_t* V32 = reinterpret_cast<uint32_t*>(V) + lane;
#pragma unroll
    for (int r = 0; r < BR; r++) {  // fully unrolled: the window shift is register renaming
      const uint32_t q6 = ld2(r + 6);
      V32[r * (VP / 2)] = 18u * (q0 + q6) + 34u * (q1 + q5) + 48u * (q2 + q4) + 56u * q3;
      q0 = q1; q1 = q2; q2 = q3; q3 = q4; q4 = q5; q5 = q6;
    }
  }
  __syncwarp();  // V complete
  DESC_TS(4);
  // rotated BRIEF: lane = output byte; bit t compares points 2b, 2b+1 with b = 8*lane + t.
  // The blurred value is needed only at the 512 sample points, so the horizontal pass runs
  // there alone: B(oy, ox) = (sum_j k_j V[18 + oy][18 + ox + j] + 2^15) >> 16.
  const long long r2 = (long long)m10 * m10 + (long long)m01 * m01;
  // 1/r in f32: r2 < 2^49 converts with relative error <= 2^-24 and rsqrtf is within 2 ulp,
  // so cs, sn carry < 4e-7 relative error and |t| <= 19 stays within 1e-5 of the exact
  // quotient -- far inside the 1e-4 band that sends a near-tie to the exact integer test
  const float inv_r = r2 ? rsqrtf((float)r2) : 0.f;
  // r2 == 0 (no rotation): (cs, sn) = (1, 0) gives t = px, py exactly, never near a tie
  const float cs = r2 ? (float)m10 * inv_r : 1.f, sn = r2 ? (float)m01 * inv_r : 0.f;  // |m| < 2^24: exact
  // horizontal pass at one sample: the 7 V values v0..v6 from the 4 words covering them
  // (funnel shift by 16 when they start at an odd u16; V is word aligned, the 4th word may be
  // the padding after V), weighted by dp2a on 16-bit pairs (v <= 65280, weights < 256)
  const uint32_t* V32 = reinterpret_cast<const uint32_t*>(V);
  auto blurred = [&](int ox, int oy) -> int {
    const int idx = (18 + oy) * VP + 18 + ox + podd;
    const uint32_t* wv = V32 + (idx >> 1);
    const uint32_t s = 16u * (uint32_t)(idx & 1);
    const uint32_t w0 = wv[0], w1 = wv[1], w2 = wv[2], w3 = wv[3];
    uint32_t sum = __dp2a_lo(__funnelshift_r(w0, w1, s), 18u | 34u << 8, 1u << 15);  // 18 v0 + 34 v1
    sum = __dp2a_lo(__funnelshift_r(w1, w2, s), 48u | 56u << 8, sum);               // 48 v2 + 56 v3
    sum = __dp2a_lo(__funnelshift_r(w2, w3, s), 48u | 34u << 8, sum);               // 48 v4 + 34 v5
    sum = __dp2a_lo(__funnelshift_r(w3, w3, s), 18u, sum);                          // 18 v6
    return (int)(sum >> 16);
  };
  // fast pass, branch-free: every offset from the f32 estimate rounded half-to-even with the
  // 1.5 * 2^23 trick; an estimate within 1e-4 of a half-integer only raises `near`
  const int64_t o = (int64_t)f * g.kp_capacity + i;
  uint8_t* smp = SAMPLES ? samples + o * 512 + 16 * lane : nullptr;
  uint32_t byte = 0;
  uint32_t near = 0;  // bit t: pair t had an estimate within 1e-4 of a half-integer
#pragma unroll
  for (int t = 0; t < 8; t++) {
    int v[2];
    bool nr = false;
#pragma unroll
    for (int e = 0; e < 2; e++) {
      const float2 pp = s_pat[(2 * t + e) * 32 + lane];  // exact small integers
      const float tx = __fmaf_rn(pp.x, cs, __fmul_rn(-pp.y, sn));  // (px m10 - py m01) / r
      const float ty = __fmaf_rn(pp.x, sn, __fmul_rn(pp.y, cs));   // (px m01 + py m10) / r
      const float bx = __fadd_rn(tx, 12582912.0f), by = __fadd_rn(ty, 12582912.0f);
      const float dx = __fsub_rn(tx, __fsub_rn(bx, 12582912.0f)), dy = __fsub_rn(ty, __fsub_rn(by, 12582912.0f));
      // |d| <= 1/2 always (t minus its nearest integer): a near-tie is |d| >= 1/2 - 1e-4
      nr |= (fabsf(dx) >= 0.4999f) | (fabsf(dy) >= 0.4999f);
      v[e] = blurred(__float_as_int(bx) - 0x4B400000, __float_as_int(by) - 0x4B400000);
      if (SAMPLES) smp[2 * t + e] = (uint8_t)v[e];
    }
    byte |= (uint32_t)(v[0] < v[1]) << t;
    near |= (uint32_t)nr << t;
  }
  // rare: only the pairs with a near-tie estimate are redone with the exact tie test (round
  // 1 redid all 16 samples of every lane of the warp: those warps were the launch's slowest)
  while (near) {
    const int t = __ffs(near) - 1;
    near &= near - 1;
    int v[2];
#pragma unroll
    for (int e = 0; e < 2; e++) {
      const float2 pp = s_pat[(2 * t + e) * 32 + lane];
      const int px = (int)pp.x, py = (int)pp.y;
      int ox = px, oy = py;
      if (r2) {
        ox = rhe_rot(px, -py, cs, sn, m10, m01, r2);
        oy = rhe_rot(px, py, sn, cs, m01, m10, r2);
      }
      v[e] = blurred(ox, oy);
      if (SAMPLES) smp[2 * t + e] = (uint8_t)v[e];
    }
    byte = (byte & ~(1u << t)) | ((uint32_t)(v[0] < v[1]) << t);
  }
  desc[o * SS_DESC_BYTES + lane] = (uint8_t)byte;
  DESC_TS(5);
  if (lane == 0) {
    float ang = 0.f;
    if (m10 != 0 || m01 != 0) {
      // f32 atan2 of exactly representable moments: |error| < 1e-6 rad (budget 1e-4)
      float a = atan2f((float)m01, (float)m10) * 57.29577951308232f;
      if (a < 0.f) a += 360.0f;
      ang = a >= 360.0f ? 0.0f : a;
    }
    ss_keypoint kp;
    kp.x = __fmul_rn((float)lx, g.scale[l]);
    kp.y = __fmul_rn((float)ly, g.scale[l]);
    kp.angle_deg = ang;
    kp.lx = (uint16_t)lx;
    kp.ly = (uint16_t)ly;
    kp.level = (uint8_t)l;
    kp.response = (uint8_t)(M - 1);
    kp.reserved = 0;
    kps[o] = kp;
  }
  DESC_TS(6);
}

}  // namespace

#ifdef SS_DESC_PHASES
extern "C" int ss_dbg_desc_ts(unsigned long long* out) { return (int)cudaMemcpyFromSymbol(out, g_desc_ts, sizeof(g_desc_ts)); }
#endif

const int* brief_pattern_host() { return SS_BRIEF_PATTERN_HOST; }

cudaError_t describe_init() {  // ss_create, per device (never under stream capture)
  cudaError_t e = carveout_from_env(describe_kernel<false>);
  if (e == cudaSuccess) e = carveout_from_env(describe_kernel<true>);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(describe_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       (int)(DESC_WARPS * PER_WARP + 128));
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(describe_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              (int)(DESC_WARPS * PER_WARP + 128));
}

bool encode_patch_map(CUtensorMap* m, const void* base, int w, int h, int frames, int64_t pitch, int64_t fstride) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  static bool tried = false;
  if (!tried) {  // the driver entry point through the runtime (no -lcuda link)
    tried = true;
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }
  if (!encode || !base || w < kPatchBoxW || h < kPatchBoxH || frames < 1) return false;
  if ((reinterpret_cast<uintptr_t>(base) & 15) || (pitch & 15)) return false;
  if (frames == 1) fstride = ((int64_t)pitch * h + 15) & ~(int64_t)15;  // unused dimension
  if (fstride & 15) return false;
  const cuuint64_t dims[3] = {(cuuint64_t)w, (cuuint64_t)h, (cuuint64_t)frames};
  const cuuint64_t strides[2] = {(cuuint64_t)pitch, (cuuint64_t)fstride};
  const cuuint32_t box[3] = {(cuuint32_t)kPatchBoxW, (cuuint32_t)kPatchBoxH, 1u};
  const cuuint32_t estr[3] = {1u, 1u, 1u};
  return encode(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, const_cast<void*>(base), dims, strides, box, estr,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t launch_describe(const Geom& g, int n_frames, FrameSrc src, const uint32_t* selected,
                            const int32_t* sel_counts, const int8_t* pattern, ss_keypoint* kps, uint8_t* desc,
                            int32_t* counts, uint8_t* samples, const PatchMaps& maps, cudaStream_t s) {
  const size_t smem = (size_t)DESC_WARPS * PER_WARP + 128;
  dim3 grid((g.kp_capacity + DESC_WARPS - 1) / DESC_WARPS, n_frames);
  cudaError_t e = samples ? launch_pdl(describe_kernel<true>, grid, dim3(DESC_WARPS * 32), smem, s, g, src, selected,
                                       sel_counts, pattern, kps, desc, counts, samples, maps)
                          : launch_pdl(describe_kernel<false>, grid, dim3(DESC_WARPS * 32), smem, s, g, src, selected,
                                       sel_counts, pattern, kps, desc, counts, samples, maps);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
