// k_lastframe.cu -- O13: frame-to-frame projection matching, ORB-SLAM's
// SearchByProjection(CurrentFrame, LastFrame) in TrackWithMotionModel [ext] -- the
// "ORB-Matching" step of the paper's tracking breakdown (§5, Fig. 8;
// DESIGN.md §3 item 14, include/ss.h ss_match_last_frame).
//
// ONE launch for the whole step: one 1024-thread CTA per frame (kCluster = 1, the default; a
// build with SS_LF_CLUSTER=8 spreads a frame over a thread-block cluster of 8 x 512 threads
// with DSMEM histograms instead).  The step has three frame-wide dependencies (the dedup of
// keypoints claimed by several points, the rotation histogram's three maxima, and the "fewer
// than min_matches -> redo with 2*th" retry), which are block (or cluster) barriers here
// instead of kernel boundaries:
//   P0  every CTA stages the frame's keypoint positions and builds its row index (first
//       keypoint per (level, row)) in shared memory; claims reset; the cluster also writes
//       the window matcher's global row index and resets its claims (match_prepare's work,
//       so the following search-local-points match skips that launch); | cluster.sync
//   P1  four lanes per point: pose transform + pinhole projection + bounds (single-rounded
//       f32 ops in the oracle's order), octave-scaled window, level gate, exact |x-u| < r,
//       |y-v| < r, 8 x POPC Hamming over the candidate runs of the row index, shuffle merge
//       of packed (d << 32 | k) top-2; accepted -> atomicMin claim (pass tag | d | point);
//                                                                              | cluster.sync
//   P2  claim lost -> rejected; else rotation bin -> histogram in the leader CTA's shared
//       memory (DSMEM atomics);                                                | cluster.sync
//   P3  ComputeThreeMaxima of the 30 bins (each CTA once), other bins rejected, survivors
//       counted in the leader's shared memory;                                 | cluster.sync
//   retry: if the count is below min_matches, P1-P3 again with 2*th.  Pass-2 claim keys
//   carry a smaller tag, so they win over stale pass-1 claims without a reset barrier.
// Latency-bound (a few hundred points per frame, a handful of candidates each).
#include <cooperative_groups.h>

#include "match_common.cuh"

namespace cg = cooperative_groups;

namespace ss {

namespace {

#ifndef SS_LF_CLUSTER
#define SS_LF_CLUSTER 1
#endif
constexpr int kCluster = SS_LF_CLUSTER;           // CTAs per frame (1: one CTA, block barriers)
#ifndef SS_LF_THREADS
#define SS_LF_THREADS 1024
#endif
constexpr int kThreads = SS_LF_THREADS;  // per CTA
#ifndef SS_LF_LANES
#define SS_LF_LANES 1
#endif
constexpr int kLanes = SS_LF_LANES;  // lanes per point in P1
constexpr int kHisto = 30;     // ORB-SLAM HISTO_LENGTH
constexpr size_t kLfSmemMax = 200 * 1024;

__device__ __forceinline__ float dot3r(const float* a, float b0, float b1, float b2) {
  float s = __fmul_rn(a[0], b0);
  s = __fadd_rn(s, __fmul_rn(a[1], b1));
  return __fadd_rn(s, __fmul_rn(a[2], b2));
}

// rot = angle_last - angle_cur (+360 if negative); bin = roundf(rot * f32(1/30)); 30 -> 0
__device__ __forceinline__ int rot_bin(float al, float ac) {
  float rot = __fsub_rn(al, ac);
  if (rot < 0.0f) rot = __fadd_rn(rot, 360.0f);
  int bin = (int)roundf(__fmul_rn(rot, 1.0f / kHisto));
  return bin == kHisto ? 0 : bin;
}

struct LfArgs {
  Geom g;
  int F;
  const ss_camera* cams;
  const ss_camera* last_cams;
  float mb;
  const ss_keypoint* kps;
  const uint8_t* desc;
  const int32_t* counts;
  const uint8_t* taken;
  const int32_t* pt_off;
  const ss_frame_point* pts;
  const uint8_t* pdesc;
  float th;
  int th_high, check_orientation, min_matches;
  ss_match* out;
  int32_t* n_matches;
  uint8_t* matched;
  unsigned long long* claim;       // this matcher's dedup claims [F][cap]
  uint16_t* rowidx;                // if set: the window matcher's global row index, built here too
  unsigned long long* win_claim;   // ... and its dedup claims, reset here (match_prepare's work)
  int rows_per_frame;              // row-index entries (the shared-memory copy)
  int index_stride;                // per-frame stride of the global index (rows + lx section)
};

// frame-wide barrier: the cluster's when a frame spans several CTAs, else the block's
__device__ __forceinline__ void frame_sync() {
  if constexpr (kCluster > 1) cg::this_cluster().sync();
  else __syncthreads();
}

__global__ void __launch_bounds__(kThreads) lastframe_kernel(const LfArgs a) {
  __shared__ int s_hist[2][32];
  __shared__ int s_count[2];
  __shared__ int s_keep[3];
  __shared__ int s_roff[kMaxLevels];
  const int rank = kCluster > 1 ? (int)cg::this_cluster().block_rank() : 0;
  const int f = blockIdx.x / kCluster;
  const int ct = rank * kThreads + threadIdx.x, nct = kCluster * kThreads;
  const Geom& g = a.g;
  const int L = g.L, cap = g.kp_capacity;
  if (threadIdx.x < 64) (&s_hist[0][0])[threadIdx.x] = 0;
  if (threadIdx.x < 2) s_count[threadIdx.x] = 0;
  if (threadIdx.x < kMaxLevels) s_roff[threadIdx.x] = threadIdx.x < a.g.L ? row_off(a.g, threadIdx.x) : 0;
  pdl_wait();
  pdl_trigger();
  int* lead_hist = &s_hist[0][0];
  int* lead_count = &s_count[0];
  if constexpr (kCluster > 1) {
    lead_hist = cg::this_cluster().map_shared_rank(&s_hist[0][0], 0);
    lead_count = cg::this_cluster().map_shared_rank(&s_count[0], 0);
  }

  const ss_keypoint* fk = a.kps + (int64_t)f * cap;
  const int32_t* cnt = a.counts + f * (L + 1);
  // every CTA keeps its own copy of the frame's keypoint positions and row index in shared
  // memory; with one CTA per frame also the descriptors and the taken mask, so the window
  // walk of P1 never waits on global memory (a cluster CTA reads descriptors from L2)
  extern __shared__ __align__(16) uint4 s_dyn[];
  const int cap8 = (cap + 7) & ~7;
  uint4* s_desc = s_dyn;                                                          // [cap][2] (kCluster == 1)
  uint16_t* s_lx = reinterpret_cast<uint16_t*>(s_dyn + (kCluster == 1 ? 2 * cap : 0));  // [cap8] keypoint lx
  float2* s_xy = reinterpret_cast<float2*>(s_lx + cap8);                          // [cap]
  uint16_t* fri = reinterpret_cast<uint16_t*>(s_xy + cap);                        // [rows_per_frame]
  uint8_t* s_taken = reinterpret_cast<uint8_t*>(fri + a.rows_per_frame);          // [cap] (kCluster == 1)
  unsigned long long* fclaim = a.claim + (int64_t)f * cap;
  uint8_t* fmask = a.matched ? a.matched + (int64_t)f * cap : nullptr;
  const int nk = cnt[L];
  const uint4* gdesc = reinterpret_cast<const uint4*>(a.desc + (int64_t)f * cap * SS_DESC_BYTES);
  for (int k = threadIdx.x; k < cap; k += kThreads) {  // P0
    rowidx_fill(g, fk, cnt, fri, k);
    if (k < nk) {
      const ss_keypoint kp = fk[k];
      s_xy[k] = make_float2(kp.x, kp.y);
      s_lx[k] = (uint16_t)kp.lx;
    }
    if constexpr (kCluster == 1) {
      if (k < nk) {
        s_desc[2 * k] = gdesc[2 * k];
        s_desc[2 * k + 1] = gdesc[2 * k + 1];
      }
      s_taken[k] = a.taken ? a.taken[(int64_t)f * cap + k] : 0;
    }
  }
  for (int k = ct; k < cap; k += nct) {
    fclaim[k] = ~0ull;
    if (fmask) fmask[k] = (a.taken && a.taken[(int64_t)f * cap + k]) ? 1 : 0;
    if (a.rowidx) {  // the following search-local-points match reuses this index (no match_prepare)
      uint16_t* gri = a.rowidx + (int64_t)f * a.index_stride;
      rowidx_fill(g, fk, cnt, gri, k, gri + lx_off(g));
      a.win_claim[(int64_t)f * cap + k] = ~0ull;
    }
  }
  frame_sync();

  const ss_camera& c = a.cams[f];
  int dir = 0;  // 1 = forward [o, L-1], 2 = backward [0, o], 0 = [o-1, o+1]
  if (a.mb > 0.0f && a.last_cams) {
    const ss_camera& cl = a.last_cams[f];
    const float tz = __fadd_rn(dot3r(cl.R + 6, c.ow[0], c.ow[1], c.ow[2]), cl.t[2]);
    dir = tz > a.mb ? 1 : (-tz > a.mb ? 2 : 0);
  }
  const int i0 = a.pt_off[f], i1 = a.pt_off[f + 1];
  const uint4* fd = kCluster == 1 ? s_desc : gdesc;
  const uint8_t* ft = kCluster == 1 ? (a.taken ? s_taken : nullptr) : (a.taken ? a.taken + (int64_t)f * cap : nullptr);
  const int sub = threadIdx.x % kLanes;
  const unsigned gmask = ((1u << kLanes) - 1u) << ((threadIdx.x & 31) & ~(kLanes - 1));
  int kept = 0;

  for (int pass = 0; pass < 2; pass++) {
    const float th = pass ? __fmul_rn(2.0f, a.th) : a.th;
    const unsigned long long tag = pass ? 0ull : (1ull << 62);
    // P1: search (all lanes of a group run the same trip count)
    for (int i = i0 + ct / kLanes; i < i1; i += nct / kLanes) {
      const ss_frame_point P = a.pts[i];
      unsigned long long b1 = ~0ull, b2 = ~0ull;
      const int o = P.octave;
      if (o >= 0 && o < L) {
        const float X = __fadd_rn(dot3r(c.R, P.pos[0], P.pos[1], P.pos[2]), c.t[0]);
        const float Y = __fadd_rn(dot3r(c.R + 3, P.pos[0], P.pos[1], P.pos[2]), c.t[1]);
        const float Z = __fadd_rn(dot3r(c.R + 6, P.pos[0], P.pos[1], P.pos[2]), c.t[2]);
        const float u = __fadd_rn(__fdiv_rn(__fmul_rn(c.fx, X), Z), c.cx);
        const float v = __fadd_rn(__fdiv_rn(__fmul_rn(c.fy, Y), Z), c.cy);
        if (!(Z < 0.0f) && !(u < c.min_x || u > c.max_x) && !(v < c.min_y || v > c.max_y)) {
          const float r = __fmul_rn(th, g.scale[o]);
          const int l0 = dir == 1 ? o : (dir == 2 ? 0 : max(o - 1, 0));
          const int l1 = dir == 1 ? L - 1 : (dir == 2 ? o : min(o + 1, L - 1));
          const uint4* qd = reinterpret_cast<const uint4*>(a.pdesc + (int64_t)i * SS_DESC_BYTES);
          const uint4 qa = qd[0], qb = qd[1];
          for (int l = l0; l <= l1; l++) {
            int rlo, rhi;
            window_rows(g, l, v, r, &rlo, &rhi);
            const uint16_t* ri = fri + s_roff[l];
            const int kb = ri[rlo], ke = ri[rhi];
            // the rows' keypoints in 8-keypoint chunks of the lx array, prefiltered against the
            // level's column range (a superset of |x - u| < r); survivors take the exact tests
            const unsigned cr = col_range(g, l, u, r);
            const unsigned lo = cr & 0xFFFFu, span = (cr >> 16) - lo;
            for (int ch = (kb >> 3) + sub; ch < (ke + 7) >> 3; ch += kLanes) {
              const int k0 = ch * 8;
              const uint4 x8 = reinterpret_cast<const uint4*>(s_lx)[ch];
              unsigned m = ((x8.x & 0xFFFFu) - lo <= span ? 0x01u : 0u) | ((x8.x >> 16) - lo <= span ? 0x02u : 0u) |
                           ((x8.y & 0xFFFFu) - lo <= span ? 0x04u : 0u) | ((x8.y >> 16) - lo <= span ? 0x08u : 0u) |
                           ((x8.z & 0xFFFFu) - lo <= span ? 0x10u : 0u) | ((x8.z >> 16) - lo <= span ? 0x20u : 0u) |
                           ((x8.w & 0xFFFFu) - lo <= span ? 0x40u : 0u) | ((x8.w >> 16) - lo <= span ? 0x80u : 0u);
              m &= (0xFFu << max(kb - k0, 0)) & (0xFFu >> max(k0 + 8 - ke, 0));
              while (m) {
                const int k = k0 + __ffs(m) - 1;
                m &= m - 1;
                const float2 xy = s_xy[k];
                const float dx = __fsub_rn(xy.x, u), dy = __fsub_rn(xy.y, v);
                if (!(fabsf(dx) < r && fabsf(dy) < r)) continue;
                if (ft && ft[k]) continue;
                const int d = hamming256(qa, qb, fd[2 * k], fd[2 * k + 1]);
                const unsigned long long key = ((unsigned long long)d << 32) | (unsigned)k;
                if (key < b1) {
                  b2 = b1;
                  b1 = key;
                } else if (key < b2) {
                  b2 = key;
                }
              }
            }
          }
        }
      }
#pragma unroll
      for (int s = kLanes / 2; s > 0; s >>= 1) {
        const unsigned long long o1 = __shfl_xor_sync(gmask, b1, s), o2 = __shfl_xor_sync(gmask, b2, s);
        merge_top2(b1, b2, o1, o2);
      }
      if (sub == 0) {
        ss_match m;
        m.dist = b1 == ~0ull ? 256 : (int)(b1 >> 32);
        m.dist2 = b2 == ~0ull ? 256 : (int)(b2 >> 32);
        m.idx = (b1 != ~0ull && m.dist <= a.th_high) ? (int)(b1 & 0xFFFFFFFFu) : -1;
        a.out[i] = m;
        if (m.idx >= 0)
          atomicMin(fclaim + m.idx, tag | ((unsigned long long)m.dist << 32) | (unsigned)(i - i0));
      }
    }
    frame_sync();
    // P2: dedup (min (distance, point) per keypoint) + rotation histogram
    for (int i = i0 + ct; i < i1; i += nct) {
      const ss_match m = a.out[i];
      if (m.idx < 0) continue;
      const unsigned long long mine = tag | ((unsigned long long)m.dist << 32) | (unsigned)(i - i0);
      if (fclaim[m.idx] != mine) {
        a.out[i].idx = -1;
      } else if (a.check_orientation) {
        atomicAdd(lead_hist + pass * 32 + rot_bin(a.pts[i].angle_deg, fk[m.idx].angle_deg), 1);
      } else {
        atomicAdd(lead_count + pass, 1);
      }
    }
    frame_sync();
    // P3: ComputeThreeMaxima, reject the other bins, count the survivors
    if (a.check_orientation) {
      if (threadIdx.x == 0) {
        int max1 = 0, max2 = 0, max3 = 0, ind1 = -1, ind2 = -1, ind3 = -1;
        for (int b = 0; b < kHisto; b++) {
          const int s = lead_hist[pass * 32 + b];
          if (s > max1) {
            max3 = max2; max2 = max1; max1 = s;
            ind3 = ind2; ind2 = ind1; ind1 = b;
          } else if (s > max2) {
            max3 = max2; max2 = s;
            ind3 = ind2; ind2 = b;
          } else if (s > max3) {
            max3 = s;
            ind3 = b;
          }
        }
        const float cut = __fmul_rn(0.1f, (float)max1);
        if ((float)max2 < cut) {
          ind2 = -1;
          ind3 = -1;
        } else if ((float)max3 < cut) {
          ind3 = -1;
        }
        s_keep[0] = ind1;
        s_keep[1] = ind2;
        s_keep[2] = ind3;
      }
      __syncthreads();
      const int k1 = s_keep[0], k2 = s_keep[1], k3 = s_keep[2];
      for (int i = i0 + ct; i < i1; i += nct) {
        const int idx = a.out[i].idx;
        if (idx < 0) continue;
        const int bin = rot_bin(a.pts[i].angle_deg, fk[idx].angle_deg);
        if (bin != k1 && bin != k2 && bin != k3)
          a.out[i].idx = -1;
        else
          atomicAdd(lead_count + pass, 1);
      }
      frame_sync();
    }
    kept = lead_count[pass];
    if (a.min_matches <= 0 || kept >= a.min_matches) break;  // uniform over the cluster
  }
  if (a.n_matches && rank == 0 && threadIdx.x == 0) a.n_matches[f] = kept;
  if (fmask)  // kept matches are unique per keypoint (dedup), so these stores never collide
    for (int i = i0 + ct; i < i1; i += nct) {
      const int idx = a.out[i].idx;
      if (idx >= 0) fmask[idx] = 1;
    }
  frame_sync();  // the leader's shared memory must outlive every remote access
}

}  // namespace

cudaError_t lastframe_init() {  // at ss_create (never inside a stream capture)
  return cudaFuncSetAttribute(lastframe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kLfSmemMax);
}

size_t lastframe_smem_bytes(const Geom& g) {
  const size_t base = sizeof(float2) * (size_t)g.kp_capacity + sizeof(uint16_t) * (size_t)match_rows_per_frame(g) +
                      sizeof(uint16_t) * (size_t)((g.kp_capacity + 7) & ~7);
  return kCluster == 1 ? base + (size_t)SS_DESC_BYTES * g.kp_capacity + (size_t)g.kp_capacity : base;
}

cudaError_t launch_lastframe(const Geom& g, int n_frames, const ss_camera* cams, const ss_camera* last_cams, float mb,
                             const ss_keypoint* kps, const uint8_t* desc, const int32_t* counts, const uint8_t* taken,
                             const int32_t* pt_off, const ss_frame_point* pts, const uint8_t* pdesc, float th,
                             int th_high, int check_orientation, int min_matches, ss_match* out, int32_t* n_matches,
                             uint8_t* matched, unsigned long long* claim, uint16_t* rowidx,
                             unsigned long long* win_claim, int n_sm, cudaStream_t s, void (*mark)(void*),
                             void* mark_arg) {
  (void)n_sm;
  if (n_frames <= 0) return cudaSuccess;
  LfArgs a{g,     n_frames, cams,    last_cams,         mb,          kps, desc, counts,
           taken, pt_off,   pts,     pdesc,             th,          th_high, check_orientation,
           min_matches, out, n_matches, matched, claim, rowidx, win_claim, match_rows_per_frame(g),
           match_index_stride(g)};
  const size_t smem = lastframe_smem_bytes(g);
  if (smem > kLfSmemMax) return cudaErrorInvalidValue;
  if (mark) mark(mark_arg);
  cudaError_t e;
  if constexpr (kCluster > 1) {  // a thread-block cluster per frame (+ programmatic serialisation)
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(n_frames * kCluster);
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = kCluster;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 2;
    e = cudaLaunchKernelEx(&cfg, lastframe_kernel, a);
  } else {
    e = launch_pdl(lastframe_kernel, dim3(n_frames), dim3(kThreads), smem, s, a);
  }
  if (mark) mark(mark_arg);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
