/*
 * ss_oracle.h -- CPU ORACLE for the SLAM-Share tracking hot path (TEST INFRASTRUCTURE ONLY).
 *
 * This is the plain, slow, single-threaded reference that the CUDA path is checked
 * against.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares NO code, header, table or constant
 * generator with paper_conf_conext_dhakalrwcr22_b200/ (the product); structs here
 * are declared independently and merely have the same byte layout as include/ss.h
 * so that the tests can compare outputs field by field.
 *
 * Citations: "P:Lnnn §x" = /root/reference/PAPER.md line nnn, section x;
 * "S8c Ox" = SURVEY.md §8(c) row Ox (the readings DESIGN.md adopts).
 * Parity status of each function is stated at its definition in ss_oracle.c.
 */
#ifndef SS_ORACLE_H
#define SS_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define REF_MAX_LEVELS 8

typedef struct {
  int32_t width, height, n_features, n_levels;
  float scale_factor;
  int32_t ini_th_fast, min_th_fast;
  float scale[REF_MAX_LEVELS], inv_scale[REF_MAX_LEVELS];
  int32_t level_w[REF_MAX_LEVELS], level_h[REF_MAX_LEVELS], n_per_level[REF_MAX_LEVELS];
  int32_t cell_cols[REF_MAX_LEVELS], cell_rows[REF_MAX_LEVELS];
  int32_t cell_w[REF_MAX_LEVELS], cell_h[REF_MAX_LEVELS];
  int32_t n_ini[REF_MAX_LEVELS];
  int32_t level_cap[REF_MAX_LEVELS];
  int32_t kp_capacity;
} ref_params;

typedef struct {            /* 20 bytes, same layout as ss_keypoint */
  float x, y, angle_deg;
  uint16_t lx, ly;
  uint8_t level, response;
  uint16_t reserved;
} ref_keypoint;

typedef struct { int32_t frame; float u, v; int32_t pred_level; float radius; } ref_query;  /* 20 B */
typedef struct { int32_t idx; int32_t dist; int32_t dist2; } ref_match;                    /* 12 B */

/* O0 */
int ref_params_init(int32_t w, int32_t h, int32_t n_features, int32_t n_levels, float scale_factor,
                    int32_t ini_th, int32_t min_th, ref_params* out);
/* O1 */
void ref_resize_linear_exact(const uint8_t* src, int sw, int sh, int spitch,
                             uint8_t* dst, int dw, int dh, int dpitch);
/* level l stored at out + sum_{l'<l} level_w*level_h, pitch level_w */
int64_t ref_pyramid_bytes(const ref_params* p);
void ref_pyramid(const ref_params* p, const uint8_t* img, int pitch, uint8_t* out);
/* O2: M(p) for 3<=x<w-3, 3<=y<h-3, clamped to >=0; 0 elsewhere.  out is w*h. */
void ref_fast_M(const uint8_t* img, int w, int h, int pitch, uint8_t* out);
/* O3: candidates of one level in rank order; returns count (or -1 if > cap). score = M. */
int ref_cell_candidates(const ref_params* p, int level, const uint8_t* M,
                        int32_t* lx, int32_t* ly, int32_t* score, int cap);
/* O4: indices (into the input) of the keys the quadtree keeps; returns count. */
int ref_distribute(const int32_t* kx, const int32_t* ky, const int32_t* score, int n,
                   int width, int height, int N, int32_t* out_idx);
/* O5 */
void ref_moments(const uint8_t* img, int pitch, int lx, int ly, int32_t* m10, int32_t* m01);
float ref_angle_deg(int32_t m10, int32_t m01);
/* O6 */
void ref_blur(const uint8_t* img, int w, int h, int pitch, uint8_t* out, int opitch);
/* O7 */
int32_t ref_rhe_div_sqrt(int64_t z, int64_t r2);
void ref_descriptor(const uint8_t* blurred, int pitch, int lx, int ly, int32_t m10, int32_t m01,
                    uint8_t out[32]);
/* O1..O8 for one frame.  kps[kp_capacity], desc[kp_capacity*32], counts[n_levels+1] (prefix). */
/* O4g grid top-N (mode 1 of ref_orb_extract_mode): indices of the kept candidates. */
int ref_distribute_grid(const ref_params* p, int level, const int32_t* lx, const int32_t* ly,
                        const int32_t* score, int n, int N, int32_t* out_idx);
/* O1..O8 with distribution mode 0 = quadtree (O4), 1 = grid top-N (O4g). */
int ref_orb_extract_mode(const ref_params* p, const uint8_t* img, int pitch, int mode,
                         ref_keypoint* kps, uint8_t* desc, int32_t* counts);
int ref_orb_extract(const ref_params* p, const uint8_t* img, int pitch,
                    ref_keypoint* kps, uint8_t* desc, int32_t* counts);
int32_t ref_hamming(const uint8_t* a, const uint8_t* b);
/* O9 */
void ref_match_window(const ref_params* p, int n_frames, const ref_keypoint* kps, const uint8_t* desc,
                      const int32_t* counts, const uint8_t* taken, int n_queries, const ref_query* q,
                      const uint8_t* qdesc, int th, int ratio_num, int ratio_den, int dedup,
                      ref_match* out);
/* O10: out[n_frames*kp_capacity]; map_desc[n_map*32]; k0/k1 restrict to keypoints [k0,k1) (sampling) */
void ref_match_brute(const ref_params* p, int n_frames, const uint8_t* desc, const int32_t* counts,
                     int n_map, const uint8_t* map_desc, int th, int ratio_num, int ratio_den,
                     int k0, int k1, ref_match* out);

/* O11 (S9's input): local-map point -> frame projection ("isInFrustum").
 * Camera: Pc = R*Pw + t (R row-major), pinhole fx, fy, cx, cy, bounds [min_x, max_x] x
 * [min_y, max_y], camera centre ow.  96 bytes, same layout as ss_camera. */
typedef struct {
  float R[9], t[3], ow[3];
  float fx, fy, cx, cy;
  float min_x, max_x, min_y, max_y;
  float pad;
} ref_camera;
/* 32 bytes, same layout as ss_map_point: world position, unit mean viewing direction,
 * ORB-SLAM mfMinDistance / mfMaxDistance (scale-invariance distances). */
typedef struct { float pos[3], normal[3], min_dist, max_dist; } ref_map_point;
/* out[i]: frame = point_frame[i]; u, v, pred_level, radius when point i is in frame
 * point_frame[i]'s frustum, else pred_level = -1, radius = 0, u = v = 0 (never matches). */
void ref_project_points(const ref_params* p, int n_frames, const ref_camera* cams, int n_points,
                        const ref_map_point* pts, const int32_t* point_frame, float th, ref_query* out);

/* O12: ORB-SLAM2 Frame::ComputeStereoMatches for one rectified pair.
 * left/right: level-0 images (pitch), keypoints/descriptors/counts of each image (O1..O8);
 * bf = baseline x fx, b = baseline (maxD = bf / b).  Out: uright[kp_capacity],
 * depth[kp_capacity] per LEFT keypoint (-1 = no stereo match; slots >= count untouched), and
 * sad[kp_capacity] = the SAD of accepted matches before the outlier cut (-1 otherwise). */
void ref_stereo_match(const ref_params* p, const uint8_t* left, const uint8_t* right, int pitch,
                      const ref_keypoint* kl, const uint8_t* dl, const int32_t* cl,
                      const ref_keypoint* kr, const uint8_t* dr, const int32_t* cr, float bf, float b,
                      float* uright, float* depth, int32_t* sad);

/* O13 ("ORB-Matching" of P:L254 Fig. 8): ORB-SLAM SearchByProjection of the
 * last frame's map points into the current frame (TrackWithMotionModel).  24 bytes, same
 * layout as ss_frame_point: world position, the last keypoint's angle (deg) and octave. */
typedef struct { float pos[3]; float angle_deg; int32_t octave; int32_t reserved; } ref_frame_point;
/* Points of frame f = [pt_off[f], pt_off[f+1]); last_cams may be NULL (mono); mb > 0 enables the
 * stereo forward/backward level gate.  out[pt_off[F]]; n_matches[F] (may be NULL) = kept per frame. */
void ref_match_last_frame(const ref_params* p, int n_frames, const ref_camera* cams, const ref_camera* last_cams,
                          float mb, const ref_keypoint* kps, const uint8_t* desc, const int32_t* counts,
                          const uint8_t* taken, const int32_t* pt_off, const ref_frame_point* pts,
                          const uint8_t* pdesc, float th, int th_high, int check_orientation, int min_matches,
                          ref_match* out, int32_t* n_matches);
/* the rotation-histogram bin of step 5 */
int ref_lf_rot_bin(float angle_last, float angle_cur);

#ifdef __cplusplus
}
#endif
#endif
