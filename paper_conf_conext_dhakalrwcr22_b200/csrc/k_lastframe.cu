// k_lastframe.cu -- O13: frame-to-frame projection matching, ORB-SLAM's
// SearchByProjection(CurrentFrame, LastFrame) in TrackWithMotionModel [ext] -- the
// "ORB-Matching" step of the paper's tracking breakdown (§5, Fig. 8;
// DESIGN.md §3 item 14, include/ss.h ss_match_last_frame).
//
// ONE launch for the whole step: one 1024-thread CTA per frame.  The step has three
// frame-wide dependencies (the dedup of keypoints claimed by several points, the rotation
// histogram's three maxima, and the "fewer than min_matches -> redo with 2*th" retry), which
// are block barriers here instead of kernel boundaries:
//   P0  stage the frame's keypoint positions, lx, angles, descriptors and taken mask and its
//       row index (first keypoint per (level, row)) in shared memory; write the window
//       matcher's global row index and reset its claims (match_prepare's work, so the
//       following search-local-points match skips that launch); reset this matcher's claims;
//       each thread's first point is loaded meanwhile;                   | barrier
//   P1  one thread per point: pose transform + pinhole projection + bounds (single-rounded
//       f32 ops in the oracle's order), octave-scaled window, level gate, the window rows'
//       keypoints in 8-keypoint lx chunks prefiltered against the level's column range, exact
//       |x-u| < r, |y-v| < r, taken mask, 8 x POPC Hamming, top-2 of packed (d << 32 | k);
//       accepted -> atomicMin claim (pass tag | d | point); the match index and the point's
//       angle stay in shared memory for P2 / P3;                         | barrier
//   P2  claim lost -> rejected; else rotation bin -> histogram;          | barrier
//   P3  ComputeThreeMaxima of the 30 bins, other bins rejected, survivors counted; | barrier
//   retry: if the count is below min_matches, P1-P3 again with 2*th.  Pass-2 claim keys
//   carry a smaller tag, so they win over stale pass-1 claims without a reset barrier.
// Latency-bound (a few hundred points per frame, a handful of candidates each).  Round 1 also
// had a thread-block-cluster form (8 x 512 threads per frame, DSMEM histograms): slower with
// ticks in flight, removed in round 2.
#include "match_common.cuh"

namespace ss {

#ifdef SS_LF_PHASES  // phase timestamps per frame CTA + per-warp P1 ends (scripts/lf_phases.py; instrumented builds)
__device__ unsigned long long g_lf_ts[64][8];
__device__ unsigned long long g_lf_w[64][32];
__device__ unsigned long long g_lf_w2[64][32][2];
#define LF_WTS2(q)                                                                        \
  do {                                                                                    \
    if ((threadIdx.x & 31) == 0 && blockIdx.x < 64) {                                     \
      unsigned long long t_;                                                              \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                              \
      g_lf_w2[blockIdx.x][threadIdx.x >> 5][q] = t_;                                      \
    }                                                                                     \
  } while (0)
#define LF_TS(i)                                                   \
  do {                                                             \
    if (threadIdx.x == 0 && blockIdx.x < 64) {                     \
      unsigned long long t_;                                       \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));       \
      g_lf_ts[blockIdx.x][i] = t_;                                 \
    }                                                              \
  } while (0)
#define LF_WTS()                                                                          \
  do {                                                                                    \
    if ((threadIdx.x & 31) == 0 && blockIdx.x < 64) {                                     \
      unsigned long long t_;                                                              \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                              \
      g_lf_w[blockIdx.x][threadIdx.x >> 5] = t_;                                          \
    }                                                                                     \
  } while (0)
extern "C" int ss_dbg_lf_ts(unsigned long long* out) {
  cudaError_t e = cudaMemcpyFromSymbol(out, g_lf_ts, sizeof(g_lf_ts));
  if (e == cudaSuccess) e = cudaMemcpyFromSymbol(out + 64 * 8, g_lf_w, sizeof(g_lf_w));
  if (e == cudaSuccess) e = cudaMemcpyFromSymbol(out + 64 * 8 + 64 * 32, g_lf_w2, sizeof(g_lf_w2));
  return (int)e;
}
#else
#define LF_TS(i) \
  do {           \
  } while (0)
#define LF_WTS() \
  do {           \
  } while (0)
#define LF_WTS2(q) \
  do {             \
  } while (0)
#endif

namespace {

// when the dependent grid (the window matcher) may launch: 0 = after the dependency wait, 1 = after
// the first pass's search (P1), -1 = at exit; its CTAs sit resident from then until this ends
#ifndef SS_LF_TRIGGER
#define SS_LF_TRIGGER 0
#endif
constexpr int kThreads = 1024;   // per CTA (one CTA per frame)
constexpr int kPtCache = 2048;   // points per frame whose P1 results stay in shared memory
constexpr int kHisto = 30;       // ORB-SLAM HISTO_LENGTH
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

__global__ void __launch_bounds__(kThreads) lastframe_kernel(const LfArgs a) {
  __shared__ int s_hist[2][32];
  __shared__ int s_count[2];
  __shared__ int s_keep[3];
  __shared__ int s_roff[kMaxLevels];
  __shared__ int s_midx[kPtCache];    // P1's match index of local point j (-1: none / rejected)
  __shared__ float s_pang[kPtCache];  // the point's angle
  __shared__ uint8_t s_bin[kPtCache]; // its rotation bin (P2)
  const int f = blockIdx.x, tid = threadIdx.x;
  const Geom& g = a.g;
  const int L = g.L, cap = g.kp_capacity;
  if (tid < 64) (&s_hist[0][0])[tid] = 0;
  if (tid < 2) s_count[tid] = 0;
  if (tid < kMaxLevels) s_roff[tid] = tid < a.g.L ? row_off(a.g, tid) : 0;
  LF_TS(0);
  pdl_wait();
  if (SS_LF_TRIGGER == 0) pdl_trigger();
  LF_TS(1);
  const ss_keypoint* fk = a.kps + (int64_t)f * cap;
  const int32_t* cnt = a.counts + f * (L + 1);
  const int i0 = a.pt_off[f], i1 = a.pt_off[f + 1];
  // the thread's first point, loaded while P0 stages the frame
  ss_frame_point P0v;
  uint4 qa0 = make_uint4(0, 0, 0, 0), qb0 = qa0;
  if (i0 + tid < i1) {
    P0v = a.pts[i0 + tid];
    const uint4* qd = reinterpret_cast<const uint4*>(a.pdesc + (int64_t)(i0 + tid) * SS_DESC_BYTES);
    qa0 = qd[0];
    qb0 = qd[1];
  }
  // the frame's keypoints, descriptors, taken mask and row index in shared memory, so the
  // window walk of P1 never waits on global memory
  extern __shared__ __align__(16) uint4 s_dyn[];
  const int cap8 = (cap + 7) & ~7;
  uint4* s_desc = s_dyn;                                                      // [cap][2]
  uint16_t* s_lx = reinterpret_cast<uint16_t*>(s_dyn + 2 * cap);              // [cap8] keypoint lx
  float2* s_xy = reinterpret_cast<float2*>(s_lx + cap8);                      // [cap]
  float* s_ang = reinterpret_cast<float*>(s_xy + cap);                        // [cap] keypoint angle
  uint16_t* fri = reinterpret_cast<uint16_t*>(s_ang + cap);                   // [rows_per_frame]
  uint8_t* s_taken = reinterpret_cast<uint8_t*>(fri + a.rows_per_frame);      // [cap]
  unsigned long long* fclaim = a.claim + (int64_t)f * cap;
  uint8_t* fmask = a.matched ? a.matched + (int64_t)f * cap : nullptr;
  const int nk = cnt[L];
  const uint4* gdesc = reinterpret_cast<const uint4*>(a.desc + (int64_t)f * cap * SS_DESC_BYTES);
  for (int k = tid; k < cap; k += kThreads) {  // P0
    rowidx_fill(g, fk, cnt, fri, k);
    if (k < nk) {
      const ss_keypoint kp = fk[k];
      s_xy[k] = make_float2(kp.x, kp.y);
      s_lx[k] = (uint16_t)kp.lx;
      s_ang[k] = kp.angle_deg;
      s_desc[2 * k] = gdesc[2 * k];
      s_desc[2 * k + 1] = gdesc[2 * k + 1];
    }
    const uint8_t tk = a.taken ? a.taken[(int64_t)f * cap + k] : 0;
    s_taken[k] = tk;
    fclaim[k] = ~0ull;
    if (fmask) fmask[k] = tk ? 1 : 0;
    if (a.rowidx) {  // the following search-local-points match reuses this index (no match_prepare)
      uint16_t* gri = a.rowidx + (int64_t)f * a.index_stride;
      rowidx_fill(g, fk, cnt, gri, k, gri + lx_off(g));
      a.win_claim[(int64_t)f * cap + k] = ~0ull;
    }
  }
  __syncthreads();
  LF_TS(2);

  const ss_camera& c = a.cams[f];
  int dir = 0;  // 1 = forward [o, L-1], 2 = backward [0, o], 0 = [o-1, o+1]
  if (a.mb > 0.0f && a.last_cams) {
    const ss_camera& cl = a.last_cams[f];
    const float tz = __fadd_rn(dot3r(cl.R + 6, c.ow[0], c.ow[1], c.ow[2]), cl.t[2]);
    dir = tz > a.mb ? 1 : (-tz > a.mb ? 2 : 0);
  }
  const uint8_t* ft = a.taken ? s_taken : nullptr;
  int kept = 0;

  for (int pass = 0; pass < 2; pass++) {
    const float th = pass ? __fmul_rn(2.0f, a.th) : a.th;
    const unsigned long long tag = pass ? 0ull : (1ull << 62);
    // P1: search
    for (int i = i0 + tid; i < i1; i += kThreads) {
      const int j = i - i0;
      ss_frame_point P;
      uint4 qa, qb;
      if (pass == 0 && j == tid) {
        P = P0v;
        qa = qa0;
        qb = qb0;
      } else {
        P = a.pts[i];
        const uint4* qd = reinterpret_cast<const uint4*>(a.pdesc + (int64_t)i * SS_DESC_BYTES);
        qa = qd[0];
        qb = qd[1];
      }
      unsigned b1 = ~0u, b2 = ~0u;  // top-2 keys (distance << 16 | keypoint), keypoints < 65536
      const int o = P.octave;
      if (o >= 0 && o < L) {
        const float X = __fadd_rn(dot3r(c.R, P.pos[0], P.pos[1], P.pos[2]), c.t[0]);
        const float Y = __fadd_rn(dot3r(c.R + 3, P.pos[0], P.pos[1], P.pos[2]), c.t[1]);
        const float Z = __fadd_rn(dot3r(c.R + 6, P.pos[0], P.pos[1], P.pos[2]), c.t[2]);
        const float u = __fadd_rn(__fdiv_rn(__fmul_rn(c.fx, X), Z), c.cx);
        const float v = __fadd_rn(__fdiv_rn(__fmul_rn(c.fy, Y), Z), c.cy);
        if (pass == 0 && j == tid) LF_WTS2(0);
        if (!(Z < 0.0f) && !(u < c.min_x || u > c.max_x) && !(v < c.min_y || v > c.max_y)) {
          const float r = __fmul_rn(th, g.scale[o]);
          const int l0 = dir == 1 ? o : (dir == 2 ? 0 : max(o - 1, 0));
          const int l1 = dir == 1 ? L - 1 : (dir == 2 ? o : min(o + 1, L - 1));
          for (int l = l0; l <= l1; l++) {
            int rlo, rhi;
            window_rows(g, l, v, r, &rlo, &rhi);
            const uint16_t* ri = fri + s_roff[l];
            const int kb = ri[rlo], ke = ri[rhi];
            // the rows' keypoints in 8-keypoint chunks of the lx array, prefiltered against the
            // level's column range (a superset of |x - u| < r); survivors take the exact tests
            const unsigned cr = col_range(g, l, u, r);
            const unsigned lo = cr & 0xFFFFu, span = (cr >> 16) - lo;
            // two chunks per step: both lx loads in flight before either's survivors are tested
            const uint4* lx4 = reinterpret_cast<const uint4*>(s_lx);
            auto pref = [&](const uint4 x8, int k0) -> unsigned {
              const unsigned mm = ((x8.x & 0xFFFFu) - lo <= span ? 0x01u : 0u) | ((x8.x >> 16) - lo <= span ? 0x02u : 0u) |
                                  ((x8.y & 0xFFFFu) - lo <= span ? 0x04u : 0u) | ((x8.y >> 16) - lo <= span ? 0x08u : 0u) |
                                  ((x8.z & 0xFFFFu) - lo <= span ? 0x10u : 0u) | ((x8.z >> 16) - lo <= span ? 0x20u : 0u) |
                                  ((x8.w & 0xFFFFu) - lo <= span ? 0x40u : 0u) | ((x8.w >> 16) - lo <= span ? 0x80u : 0u);
              return mm & (0xFFu << max(kb - k0, 0)) & (0xFFu >> max(k0 + 8 - ke, 0));
            };
            auto survivors = [&](unsigned m, int k0) {
              while (m) {
                const int k = k0 + __ffs(m) - 1;
                m &= m - 1;
                const float2 xy = s_xy[k];
                const float dx = __fsub_rn(xy.x, u), dy = __fsub_rn(xy.y, v);
                if (!(fabsf(dx) < r && fabsf(dy) < r)) continue;
                if (ft && ft[k]) continue;
                const unsigned key = ((unsigned)hamming256(qa, qb, s_desc[2 * k], s_desc[2 * k + 1]) << 16) | (unsigned)k;
                if (key < b1) {
                  b2 = b1;
                  b1 = key;
                } else if (key < b2) {
                  b2 = key;
                }
              }
            };
            const int ce = (ke + 7) >> 3;
            for (int ch = kb >> 3; ch < ce; ch += 2) {
              const bool two = ch + 1 < ce;
              const uint4 xa = lx4[ch];
              const uint4 xb = two ? lx4[ch + 1] : make_uint4(0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu);
              const unsigned ma = pref(xa, ch * 8), mb = two ? pref(xb, ch * 8 + 8) : 0u;
              survivors(ma, ch * 8);
              survivors(mb, ch * 8 + 8);
            }
          }
        }
      }
      if (pass == 0 && j == tid) LF_WTS2(1);
      ss_match m;
      m.dist = b1 == ~0u ? 256 : (int)(b1 >> 16);
      m.dist2 = b2 == ~0u ? 256 : (int)(b2 >> 16);
      m.idx = (b1 != ~0u && m.dist <= a.th_high) ? (int)(b1 & 0xFFFFu) : -1;
      a.out[i] = m;
      if (j < kPtCache) {
        s_midx[j] = m.idx;
        s_pang[j] = P.angle_deg;
      }
      if (m.idx >= 0) atomicMin(fclaim + m.idx, tag | ((unsigned long long)m.dist << 32) | (unsigned)j);
    }
    if (pass == 0) LF_WTS();
    __syncthreads();
    if (pass == 0 && SS_LF_TRIGGER == 1) pdl_trigger();
    if (pass == 0) LF_TS(3);
    // P2: dedup (min (distance, point) per keypoint) + rotation histogram
    for (int i = i0 + tid; i < i1; i += kThreads) {
      const int j = i - i0;
      const bool cached = j < kPtCache;
      const int idx = cached ? s_midx[j] : a.out[i].idx;
      if (idx < 0) continue;
      const int dist = a.out[i].dist;
      const unsigned long long mine = tag | ((unsigned long long)dist << 32) | (unsigned)j;
      if (fclaim[idx] != mine) {
        a.out[i].idx = -1;
        if (cached) s_midx[j] = -1;
      } else if (a.check_orientation) {
        const int bin = rot_bin(cached ? s_pang[j] : a.pts[i].angle_deg, s_ang[idx]);
        if (cached) s_bin[j] = (uint8_t)bin;
        atomicAdd(&s_hist[pass][bin], 1);
      } else {
        atomicAdd(&s_count[pass], 1);
      }
    }
    __syncthreads();
    // P3: ComputeThreeMaxima, reject the other bins, count the survivors
    if (a.check_orientation) {
      if (tid == 0) {
        int max1 = 0, max2 = 0, max3 = 0, ind1 = -1, ind2 = -1, ind3 = -1;
        for (int b = 0; b < kHisto; b++) {
          const int s = s_hist[pass][b];
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
      for (int i = i0 + tid; i < i1; i += kThreads) {
        const int j = i - i0;
        const bool cached = j < kPtCache;
        const int idx = cached ? s_midx[j] : a.out[i].idx;
        if (idx < 0) continue;
        const int bin = cached ? (int)s_bin[j] : rot_bin(a.pts[i].angle_deg, s_ang[idx]);
        if (bin != k1 && bin != k2 && bin != k3) {
          a.out[i].idx = -1;
          if (cached) s_midx[j] = -1;
        } else {
          atomicAdd(&s_count[pass], 1);
        }
      }
      __syncthreads();
    }
    if (pass == 0) LF_TS(4);
    kept = s_count[pass];
    if (a.min_matches <= 0 || kept >= a.min_matches) break;  // uniform over the CTA
  }
  if (a.n_matches && tid == 0) a.n_matches[f] = kept;
  if (fmask)  // kept matches are unique per keypoint (dedup), so these stores never collide
    for (int i = i0 + tid; i < i1; i += kThreads) {
      const int j = i - i0;
      const int idx = j < kPtCache ? s_midx[j] : a.out[i].idx;
      if (idx >= 0) fmask[idx] = 1;
    }
  LF_TS(5);
}

}  // namespace

cudaError_t lastframe_init() {  // at ss_create (never inside a stream capture)
  cudaError_t e = carveout_from_env(lastframe_kernel);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(lastframe_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kLfSmemMax);
}

size_t lastframe_smem_bytes(const Geom& g) {  // dynamic part (static: ~19 KB)
  const size_t cap = (size_t)g.kp_capacity;
  return (size_t)SS_DESC_BYTES * cap + sizeof(uint16_t) * ((cap + 7) & ~(size_t)7) + sizeof(float2) * cap +
         sizeof(float) * cap + sizeof(uint16_t) * (size_t)match_rows_per_frame(g) + cap;
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
  e = launch_pdl(lastframe_kernel, dim3(n_frames), dim3(kThreads), smem, s, a);
  if (mark) mark(mark_arg);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
