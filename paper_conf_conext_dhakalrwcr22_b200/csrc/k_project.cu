// k_project.cu -- O11: local-map point projection, the per-point half of "search local
// points" (§4.2.1; ORB-SLAM3 Frame::isInFrustum + MapPoint::PredictScale +
// ORBmatcher::RadiusByViewingCos [ext]; DESIGN.md §3 item 11, include/ss.h).
//
// One thread per map point: camera transform, pinhole projection, bounds, distance gate,
// viewing cosine, predicted level (smallest n with max_dist / dist <= scale[n], the f32 scale
// chain, instead of a libm log) and window radius.  Every f32 operation is an explicit
// round-to-nearest intrinsic in the documented order (no FMA contraction), so the result is
// bit-identical to the oracle's plain C.  HBM-bound: 36 B read + 20 B written per point.
#include "ss_internal.h"

namespace ss {

namespace {

__device__ __forceinline__ float dot3(float a0, float a1, float a2, float b0, float b1, float b2) {
  float s = __fmul_rn(a0, b0);
  s = __fadd_rn(s, __fmul_rn(a1, b1));
  return __fadd_rn(s, __fmul_rn(a2, b2));
}

struct LevelScales {
  float s[kMaxLevels];
};

__global__ void __launch_bounds__(256) project_kernel(int L, LevelScales sc, int F, const ss_camera* __restrict__ cams,
                                                      int n, const ss_map_point* __restrict__ pts,
                                                      const int32_t* __restrict__ point_frame, float th,
                                                      ss_mp_query* __restrict__ out) {
  pdl_wait();
  pdl_trigger();
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int f = point_frame[i];
  ss_mp_query o;
  o.frame = f;
  o.u = 0.0f;
  o.v = 0.0f;
  o.pred_level = -1;
  o.radius = 0.0f;
  if (f >= 0 && f < F) {
    const ss_camera& c = cams[f];
    const ss_map_point mp = pts[i];
    const float px = mp.pos[0], py = mp.pos[1], pz = mp.pos[2];
    const float X = __fadd_rn(dot3(c.R[0], c.R[1], c.R[2], px, py, pz), c.t[0]);
    const float Y = __fadd_rn(dot3(c.R[3], c.R[4], c.R[5], px, py, pz), c.t[1]);
    const float Z = __fadd_rn(dot3(c.R[6], c.R[7], c.R[8], px, py, pz), c.t[2]);
    bool vis = !(Z < 0.0f);
    const float u = __fadd_rn(__fdiv_rn(__fmul_rn(c.fx, X), Z), c.cx);
    const float v = __fadd_rn(__fdiv_rn(__fmul_rn(c.fy, Y), Z), c.cy);
    vis = vis && !(u < c.min_x || u > c.max_x) && !(v < c.min_y || v > c.max_y);
    const float ox = __fsub_rn(px, c.ow[0]), oy = __fsub_rn(py, c.ow[1]), oz = __fsub_rn(pz, c.ow[2]);
    const float dist = __fsqrt_rn(dot3(ox, oy, oz, ox, oy, oz));
    const float min_d = __fmul_rn(0.8f, mp.min_dist), max_d = __fmul_rn(1.2f, mp.max_dist);
    vis = vis && !(dist < min_d || dist > max_d);
    const float view_cos = __fdiv_rn(dot3(ox, oy, oz, mp.normal[0], mp.normal[1], mp.normal[2]), dist);
    vis = vis && !(view_cos < 0.5f);
    if (vis) {
      const float ratio = __fdiv_rn(mp.max_dist, dist);
      int level = L - 1;
      for (int l = L - 1; l >= 0; l--)
        if (ratio <= sc.s[l]) level = l;
      const float r = __fmul_rn(view_cos > 0.998f ? 2.5f : 4.0f, th);
      o.u = u;
      o.v = v;
      o.pred_level = level;
      o.radius = __fmul_rn(r, sc.s[level]);
    }
  }
  out[i] = o;
}

}  // namespace

cudaError_t launch_project(const Geom& g, int n_frames, const ss_camera* cams, int n_points, const ss_map_point* pts,
                           const int32_t* point_frame, float th, ss_mp_query* out, cudaStream_t s) {
  if (n_points <= 0) return cudaSuccess;
  LevelScales sc;
  for (int l = 0; l < kMaxLevels; l++) sc.s[l] = l < g.L ? g.scale[l] : 0.0f;
  cudaError_t e = launch_pdl(project_kernel, dim3((n_points + 255) / 256), dim3(256), 0, s, g.L, sc, n_frames, cams,
                             n_points, pts, point_frame, th, out);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
