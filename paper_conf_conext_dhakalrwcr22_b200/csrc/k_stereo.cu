// k_stereo.cu -- O12: stereo matching of rectified pairs (ORB-SLAM2 Frame::ComputeStereoMatches
// [ext]; the stereo input of the paper's stereo tracking, P:L163 / P:L246; SURVEY §8(f) F1;
// DESIGN.md §3 item 12, include/ss.h ss_stereo_match).
//
// stereo_match_kernel: one warp per left keypoint.
//  1. candidates: right keypoints on octaves [oct-1, oct+1] whose row span
//     [floor(y - 2 scale), ceil(y + 2 scale)] holds row (int)vL -- a contiguous run of each
//     level's (ly, lx)-ordered keypoints found through the matcher's row index (a superset
//     widened by a row, then the exact f32 test) -- with uL - maxD <= uR <= uL; best = the
//     smallest (Hamming, canonical index) below 100 (warp min over packed keys), kept if < 75;
//  2. refinement: the 11x11 left window and the 11x21 right strip of the octave's level are
//     staged in shared memory; lane i < 11 computes the centre-subtracted SAD at shift i - 5;
//     first minimum (packed warp min), parabola sub-pixel offset, disparity range, depth =
//     bf / disparity -- every f32 op an explicit round-to-nearest intrinsic in ORB-SLAM's
//     order, so the result is bit-identical to the oracle;
// stereo_outlier_kernel: one CTA per pair: the median accepted SAD (two-pass radix select
// over the 16-bit SAD values), then every accepted match with SAD >= 1.5f * 1.4f * median is
// dropped.
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int ST_WARPS = 8;
constexpr int ST_W = 5;   // half window (11 x 11)
constexpr int ST_L = 5;   // shift range [-5, 5]
constexpr int ST_RW = 2 * (ST_W + ST_L) + 1;  // right strip width: 21

__device__ __forceinline__ int row_offset(const Geom& g, int l) {  // the matcher's row-index layout
  int o = 0;
  for (int i = 0; i < l; i++) o += g.h[i] + 1;
  return o;
}

__device__ __forceinline__ int hamming256(const uint4 a0, const uint4 a1, const uint4 b0, const uint4 b1) {
  return __popc(a0.x ^ b0.x) + __popc(a0.y ^ b0.y) + __popc(a0.z ^ b0.z) + __popc(a0.w ^ b0.w) +
         __popc(a1.x ^ b1.x) + __popc(a1.y ^ b1.y) + __popc(a1.z ^ b1.z) + __popc(a1.w ^ b1.w);
}

__device__ __forceinline__ const uint8_t* level_ptr(const Geom& g, const FrameSrc& src, int f, int l, int* pitch) {
  if (l == 0) {
    *pitch = src.pitch;
    return src.frames + (int64_t)f * src.stride;
  }
  *pitch = g.pitch[l];
  return src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
}

__global__ void __launch_bounds__(ST_WARPS * 32) stereo_match_kernel(Geom g, int n_pairs, FrameSrc src,
                                                                      const ss_keypoint* __restrict__ kps,
                                                                      const uint8_t* __restrict__ desc,
                                                                      const int32_t* __restrict__ counts,
                                                                      const uint16_t* __restrict__ rowidx,
                                                                      int index_stride, float bf, float maxD,
                                                                      float* __restrict__ uright,
                                                                      float* __restrict__ depth,
                                                                      int32_t* __restrict__ sad) {
  pdl_wait();
  pdl_trigger();
  __shared__ uint8_t sL[ST_WARPS][2 * ST_W + 1][2 * ST_W + 1];
  __shared__ uint8_t sR[ST_WARPS][2 * ST_W + 1][ST_RW];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cap = g.kp_capacity, L = g.L;
  const int64_t gw = (int64_t)blockIdx.x * ST_WARPS + warp;  // global left-keypoint slot
  if (gw >= (int64_t)n_pairs * cap) return;
  const int pr = (int)(gw / cap), iL = (int)(gw - (int64_t)pr * cap);
  const int fl = 2 * pr, fr = 2 * pr + 1;
  if (iL >= counts[fl * (L + 1) + L]) return;
  const ss_keypoint kl = kps[(int64_t)fl * cap + iL];
  const int lev = kl.level;
  const float uL = kl.x, vL = kl.y;
  const int row = (int)vL;
  const float minU = __fsub_rn(uL, maxD), maxU = __fsub_rn(uL, 0.0f);
  float out_u = -1.0f, out_d = -1.0f;
  int out_s = -1;
  // ---- 1. best Hamming candidate ----
  uint32_t best = 0xFFFFFFFFu;  // (distance << 16) | right index
  if (!(maxU < 0.0f)) {
    const uint4* dl = reinterpret_cast<const uint4*>(desc + ((int64_t)fl * cap + iL) * SS_DESC_BYTES);
    const uint4 a0 = dl[0], a1 = dl[1];
    const ss_keypoint* kr = kps + (int64_t)fr * cap;
    const uint4* dr = reinterpret_cast<const uint4*>(desc + (int64_t)fr * cap * SS_DESC_BYTES);
    const uint16_t* fri = rowidx + (int64_t)fr * index_stride;
    for (int lr = max(lev - 1, 0); lr <= min(lev + 1, L - 1); lr++) {
      const float s = g.scale[lr], r = __fmul_rn(2.0f, s);
      const int hl = g.h[lr];
      // rows ly with f32(ly) * s within (row - 1 - r, row + 1 + r), widened by a row
      const int rlo = max(0, min(hl, (int)floorf((float)(row - 1) / s - r / s) - 1));
      const int rhi = max(0, min(hl, (int)ceilf((float)(row + 1) / s + r / s) + 2));
      const uint16_t* ri = fri + row_offset(g, lr);
      const int kb = ri[rlo], ke = ri[rhi];
      for (int k = kb + lane; k < ke; k += 32) {
        const ss_keypoint q = kr[k];
        const float ky = q.y;
        if ((int)floorf(__fsub_rn(ky, r)) > row || (int)ceilf(__fadd_rn(ky, r)) < row) continue;
        const float uR = q.x;
        if (!(uR >= minU && uR <= maxU)) continue;
        const int d = hamming256(a0, a1, dr[2 * k], dr[2 * k + 1]);
        if (d < 100) best = min(best, ((uint32_t)d << 16) | (uint32_t)k);
      }
    }
  }
  best = __reduce_min_sync(0xFFFFFFFFu, best);
  if (best != 0xFFFFFFFFu && (int)(best >> 16) < 75) {
    // ---- 2. SAD refinement on the octave's level ----
    const int iR = (int)(best & 0xFFFFu);
    const float uR0 = kps[(int64_t)fr * cap + iR].x;
    const float sf = g.inv_scale[lev];
    const int su = (int)roundf(__fmul_rn(uL, sf)), sv = (int)roundf(__fmul_rn(vL, sf));
    const int su0 = (int)roundf(__fmul_rn(uR0, sf));
    const int lw = g.w[lev];
    const int iniu = su0 + ST_L - ST_W, endu = su0 + ST_L + ST_W + 1;
    if (!(iniu < 0 || endu >= lw)) {
      int pl, prr;
      const uint8_t* IL = level_ptr(g, src, fl, lev, &pl);
      const uint8_t* IR = level_ptr(g, src, fr, lev, &prr);
      for (int i = lane; i < 11 * 11; i += 32) {
        const int y = i / 11, x = i - 11 * (i / 11);
        sL[warp][y][x] = IL[(int64_t)(sv - ST_W + y) * pl + su - ST_W + x];
      }
      for (int i = lane; i < 11 * ST_RW; i += 32) {
        const int y = i / ST_RW, x = i - ST_RW * (i / ST_RW);
        sR[warp][y][x] = IR[(int64_t)(sv - ST_W + y) * prr + su0 - ST_L - ST_W + x];
      }
      __syncwarp();
      uint32_t key = 0xFFFFFFFFu;
      int dist = 0;
      if (lane < 2 * ST_L + 1) {
        const int cL = sL[warp][ST_W][ST_W], cR = sR[warp][ST_W][lane + ST_W];
        for (int y = 0; y < 11; y++)
#pragma unroll
          for (int x = 0; x < 11; x++) dist += abs(((int)sL[warp][y][x] - cL) - ((int)sR[warp][y][lane + x] - cR));
        key = ((uint32_t)dist << 4) | (uint32_t)lane;  // first minimum: lowest shift on ties
      }
      const uint32_t kmin = __reduce_min_sync(0xFFFFFFFFu, key);
      const int bi = (int)(kmin & 15u), bestd = (int)(kmin >> 4);
      const int d1i = __shfl_sync(0xFFFFFFFFu, dist, max(bi - 1, 0));
      const int d3i = __shfl_sync(0xFFFFFFFFu, dist, min(bi + 1, 2 * ST_L));
      const int inc = bi - ST_L;
      if (inc != -ST_L && inc != ST_L) {
        const float d1 = (float)d1i, d2 = (float)bestd, d3 = (float)d3i;
        const float deltaR =
            __fdiv_rn(__fsub_rn(d1, d3), __fmul_rn(2.0f, __fsub_rn(__fadd_rn(d1, d3), __fmul_rn(2.0f, d2))));
        if (!(deltaR < -1.0f || deltaR > 1.0f)) {
          float bestuR = __fmul_rn(g.scale[lev], __fadd_rn(__fadd_rn((float)su0, (float)inc), deltaR));
          float disparity = __fsub_rn(uL, bestuR);
          if (disparity >= 0.0f && disparity < maxD) {
            if (disparity <= 0.0f) {
              disparity = 0.01f;
              bestuR = __double2float_rn(__dsub_rn((double)uL, 0.01));
            }
            out_d = __fdiv_rn(bf, disparity);
            out_u = bestuR;
            out_s = bestd;
          }
        }
      }
    }
  }
  if (lane == 0) {
    const int64_t o = (int64_t)pr * cap + iL;
    uright[o] = out_u;
    depth[o] = out_d;
    sad[o] = out_s;
  }
}

// One CTA per pair: median of the accepted SADs (element size/2 of the ascending order), then
// the cut at 1.5f * 1.4f * median.
__global__ void __launch_bounds__(1024) stereo_outlier_kernel(Geom g, const int32_t* __restrict__ counts,
                                                              const int32_t* __restrict__ sad,
                                                              float* __restrict__ uright, float* __restrict__ depth) {
  pdl_wait();
  pdl_trigger();
  __shared__ int hist[256];
  __shared__ int s_n, s_bin, s_rank;
  const int pr = blockIdx.x, cap = g.kp_capacity, L = g.L;
  const int n = counts[(2 * pr) * (L + 1) + L];
  const int32_t* sd = sad + (int64_t)pr * cap;
  if (threadIdx.x < 256) hist[threadIdx.x] = 0;
  if (threadIdx.x == 0) s_n = 0;
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const int v = sd[i];
    if (v >= 0) {
      atomicAdd(&hist[(v >> 8) & 255], 1);
      atomicAdd(&s_n, 1);
    }
  }
  __syncthreads();
  const int nacc = s_n;
  if (nacc == 0) return;
  if (threadIdx.x == 0) {  // high byte of the element of rank nacc / 2
    int k = nacc / 2, b = 0;
    while (k >= hist[b]) k -= hist[b++];
    s_bin = b;
    s_rank = k;
  }
  __syncthreads();
  const int hb = s_bin;
  if (threadIdx.x < 256) hist[threadIdx.x] = 0;
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const int v = sd[i];
    if (v >= 0 && (v >> 8) == hb) atomicAdd(&hist[v & 255], 1);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    int k = s_rank, b = 0;
    while (k >= hist[b]) k -= hist[b++];
    s_bin = (hb << 8) | b;
  }
  __syncthreads();
  const float th = __fmul_rn(__fmul_rn(1.5f, 1.4f), (float)s_bin);
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const int v = sd[i];
    if (v >= 0 && !((float)v < th)) {
      uright[(int64_t)pr * cap + i] = -1.0f;
      depth[(int64_t)pr * cap + i] = -1.0f;
    }
  }
}

}  // namespace

cudaError_t launch_stereo(const Geom& g, int n_pairs, FrameSrc src, const ss_keypoint* kps, const uint8_t* desc,
                          const int32_t* counts, const uint16_t* rowidx, int index_stride, float bf, float maxD,
                          float* uright, float* depth, int32_t* sad, cudaStream_t s) {
  if (n_pairs <= 0) return cudaSuccess;
  const int64_t warps = (int64_t)n_pairs * g.kp_capacity;
  cudaError_t e = launch_pdl(stereo_match_kernel, dim3((unsigned)((warps + ST_WARPS - 1) / ST_WARPS)),
                             dim3(ST_WARPS * 32), 0, s, g, n_pairs, src, kps, desc, counts, rowidx, index_stride,
                             bf, maxD, uright, depth, sad);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_stereo_outliers(const Geom& g, int n_pairs, const int32_t* counts, const int32_t* sad,
                                   float* uright, float* depth, cudaStream_t s) {
  if (n_pairs <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(stereo_outlier_kernel, dim3(n_pairs), dim3(1024), 0, s, g, counts, sad, uright, depth);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
