/*
 * ss.h -- C ABI of libss: batched ORB extraction + tracking-time descriptor matching on
 * B200 (sm_100a), the data-parallel hot path of SLAM-Share's GPU tracking
 * (Dhakal et al., CoNEXT'22): "the parallelization of FAST corner detection ... with the
 * GPU" (§4.2.1) and the "local tracking CUDA kernel" that parallelises
 * search-local-points (L168), run for many clients at once ("spatio-temporal sharing of
 * the GPU ... on the data received from multiple client updates", L170).
 *
 * The paper fixes no arithmetic; each entry point cites the DESIGN.md §3 reading
 * (= SURVEY.md §8(c) row O0..O10) that defines it.
 *
 * Conventions
 *  - Every function returns ss_status; nothing aborts or throws across the ABI.
 *  - "device pointer" = CUDA global memory of the ctx's device; "host pointer" = CPU memory.
 *  - Calls taking a stream only ENQUEUE work on it (no host synchronisation, no allocation);
 *    outputs are valid once the stream reaches the call.  Inputs must stay valid until then.
 *  - The caller owns every input/output buffer; an ss_ctx owns only its scratch, sized at
 *    ss_create.  One ctx may be used by one host thread / stream at a time.
 *  - Argument and capacity errors are detected synchronously (SS_EINVAL / SS_ECAPACITY),
 *    before anything is enqueued.  SS_ECUDA = a CUDA API or launch error (message in
 *    ss_last_error).  Kernels never write outside the documented output extents.
 */
#ifndef SS_H
#define SS_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SS_OK = 0,
  SS_EINVAL = -1,       /* bad argument / shape / params mismatch                       */
  SS_ECAPACITY = -2,    /* more frames / queries / map entries than the ctx was sized for */
  SS_ECUDA = -3,        /* CUDA runtime or launch error                                   */
  SS_EUNSUPPORTED = -4  /* valid request this build does not implement                   */
} ss_status;

typedef struct ss_ctx ss_ctx; /* opaque */
typedef void* ss_stream_t;    /* a cudaStream_t (NULL = legacy default stream) */

#define SS_MAX_LEVELS 8
#define SS_DESC_BYTES 32

/* ORB parameters (DESIGN.md §3 O0).  Fill with ss_orb_params_init, then treat read-only:
 * scale[l] = f32(scale[l-1]*scale_factor); inv_scale[l] = f32(1/scale[l]);
 * level_w/h[l] = rne(f32(W*inv_scale[l])); n_per_level = ORB-SLAM's geometric split of
 * n_features; cells = 30-px FAST grid of each level (cols, rows, cell w, cell h);
 * n_ini = quadtree root count; level_cap[l] = max(n_per_level[l]+2, 4*n_ini[l]) = the most
 * keypoints the distribution can keep on level l; kp_capacity = sum of level_cap. */
typedef struct {
  int32_t width, height, n_features, n_levels;
  float scale_factor;
  int32_t ini_th_fast, min_th_fast;
  float scale[SS_MAX_LEVELS], inv_scale[SS_MAX_LEVELS];
  int32_t level_w[SS_MAX_LEVELS], level_h[SS_MAX_LEVELS], n_per_level[SS_MAX_LEVELS];
  int32_t cell_cols[SS_MAX_LEVELS], cell_rows[SS_MAX_LEVELS];
  int32_t cell_w[SS_MAX_LEVELS], cell_h[SS_MAX_LEVELS];
  int32_t n_ini[SS_MAX_LEVELS];
  int32_t level_cap[SS_MAX_LEVELS];
  int32_t kp_capacity;
} ss_orb_params;

/* One ORB keypoint, 20 bytes.  Per frame, keypoints are in canonical order
 * (level, ly, lx) (DESIGN.md §3 O8). */
typedef struct {
  float x, y;            /* level-0 coordinates: f32(lx) * scale[level] (one f32 multiply)   */
  float angle_deg;       /* intensity-centroid angle atan2(m01, m10) in [0, 360) (O5)        */
  uint16_t lx, ly;       /* integer pixel on its pyramid level                              */
  uint8_t level;         /* pyramid level                                                   */
  uint8_t response;      /* FAST score = M - 1 (O2)                                         */
  uint16_t reserved;     /* 0                                                               */
} ss_keypoint;

/* A local-map point projected into a frame (the caller's frustum test, ORB-SLAM
 * isInFrustum): frame index, predicted position (level-0 px), predicted level, window
 * half-size r (level-0 px).  20 bytes. */
typedef struct {
  int32_t frame;
  float u, v;
  int32_t pred_level;
  float radius;
} ss_mp_query;

/* A camera pose + pinhole intrinsics for ss_project_points (DESIGN.md §3 O11), 96 bytes:
 * camera coordinates Pc = R * Pw + t (R row-major), camera centre ow = -R^T t (given, not
 * recomputed), projection u = fx * Pc.x / Pc.z + cx, v = fy * Pc.y / Pc.z + cy, image bounds
 * [min_x, max_x] x [min_y, max_y] (ORB-SLAM mnMinX..mnMaxY, level-0 px). */
typedef struct {
  float R[9], t[3], ow[3];
  float fx, fy, cx, cy;
  float min_x, max_x, min_y, max_y;
  float pad;
} ss_camera;

/* A local-map point for ss_project_points (O11), 32 bytes: world position, unit mean viewing
 * direction (ORB-SLAM mNormalVector), scale-invariance distances mfMinDistance /
 * mfMaxDistance. */
typedef struct {
  float pos[3], normal[3];
  float min_dist, max_dist;
} ss_map_point;

/* A match: idx = keypoint index within its frame (WINDOW) or map index (BRUTE), -1 = none;
 * dist / dist2 = best / second-best Hamming distance over the candidates (256 = none). */
typedef struct {
  int32_t idx;
  int32_t dist;
  int32_t dist2;
} ss_match;

#define SS_MATCH_WINDOW 0 /* one result per query: search local points (O9)       */
#define SS_MATCH_BRUTE 1  /* one result per frame keypoint vs the whole map (O10) */

typedef struct {
  int32_t mode;      /* SS_MATCH_WINDOW or SS_MATCH_BRUTE                                       */
  int32_t th;        /* accept only d1 <= th (WINDOW: ORB-SLAM TH_HIGH 100; BRUTE: TH_LOW 50)   */
  int32_t ratio_num; /* ratio = num/den; WINDOW: den*d1 <= num*d2 unless the two best lie on   */
  int32_t ratio_den; /*   different levels (4/5); BRUTE: den*d1 < num*d2 (3/4)                  */
  int32_t dedup;     /* WINDOW: 1 = a keypoint claimed by several queries keeps min (d, query)  */
} ss_match_cfg;

/* O0.  Validates 64 <= w,h <= 2048, 1 <= n_levels <= 8, scale_factor > 1, 1 <= thresholds
 * <= 254, every level >= 30 px of FAST grid in each direction and 1 <= n_ini <= 62.
 * Host only; never touches the GPU.  Returns SS_EINVAL (out untouched) on rejection. */
ss_status ss_orb_params_init(int32_t width, int32_t height, int32_t n_features, int32_t n_levels,
                             float scale_factor, int32_t ini_th_fast, int32_t min_th_fast,
                             ss_orb_params* out);

/* Create a context on `device` for frames of shape p (p must equal what
 * ss_orb_params_init returns for its own first seven fields, else SS_EINVAL).
 * max_frames bounds n_frames per call, max_queries the WINDOW query count and max_map the
 * BRUTE map size (0 = that mode unused).  Allocates all scratch here (none per call).
 * SS_EUNSUPPORTED when this build's kernels cannot serve p: scale_factor above 4/3 (the
 * pyramid kernel's source window), kp_capacity above 65535, a FAST band / pyramid block
 * that does not fit in shared memory, or max_map >= 2^23 (larger maps: shard them, see
 * ss_match_brute_partial). */
ss_status ss_create(int32_t device, const ss_orb_params* p, int32_t max_frames, int32_t max_queries,
                    int32_t max_map, ss_ctx** out);
ss_status ss_destroy(ss_ctx* ctx);

/* Message of the last failing call on this host thread (ctx may be NULL).  Never NULL. */
const char* ss_last_error(const ss_ctx* ctx);

/* O1..O8 for n_frames frames of the ctx's shape (FAST on the GPU; the rest
 * of ORB, L87, on the GPU as well).  Device pointers:
 *   d_frames : u8 gray frames, frame f row y at d_frames + f*frame_stride + y*pitch
 *              (pitch >= width, frame_stride >= height*pitch)
 *   d_kps    : [n_frames][kp_capacity] ss_keypoint      (slots >= count are left untouched)
 *   d_desc   : [n_frames][kp_capacity][32] u8, bit b of byte i = comparison 8i+b   (O7)
 *   d_counts : [n_frames][n_levels+1] i32 prefix offsets: level l is [counts[l], counts[l+1])
 * Bit-exact with the oracle except angle_deg (|err| <= 1e-4 rad).  Deterministic. */
ss_status ss_orb_extract(ss_ctx* ctx, int32_t n_frames, const uint8_t* d_frames, int64_t frame_stride,
                         int32_t pitch, ss_keypoint* d_kps, uint8_t* d_desc, int32_t* d_counts,
                         ss_stream_t stream);

/* ss_orb_extract for n_frames independently allocated client frames (SURVEY.md §8(b)'s
 * d_frames[] / pitches[] form): d_frames = HOST array of n_frames DEVICE pointers, pitches =
 * HOST array of their row pitches (>= width).  The frames are packed into the ctx's frame
 * staging buffer by one device-side 2-D copy each (enqueued on `stream`), then extracted as
 * one batch; outputs, results and errors as ss_orb_extract (plus SS_EINVAL for a NULL frame
 * pointer or a pitch < width).  The staging buffer is shared with ss_track_tick: the two must
 * not be in flight on one ctx at the same time.  Stereo pairs (ss_stereo_match reads level 0
 * from the buffer it is given) use ss_orb_extract's single-buffer form or ss_track_tick. */
ss_status ss_orb_extract_frames(ss_ctx* ctx, int32_t n_frames, const uint8_t* const* d_frames, const int32_t* pitches,
                                ss_keypoint* d_kps, uint8_t* d_desc, int32_t* d_counts, ss_stream_t stream);

/* O9 / O10 on the outputs of ss_orb_extract (same layouts).  Device pointers:
 * WINDOW ("search local points"):
 *   d_kp_taken [n_frames][kp_capacity] u8 (non-zero = keypoint already matched; may be NULL),
 *   d_queries [n_queries], d_map_desc [n_queries][32] (the map points' descriptors),
 *   d_out [n_queries]: candidates = keypoints of frame q.frame with level in
 *   [pred_level-1, pred_level], |x-u| < r and |y-v| < r (f32), not taken; top-2 by
 *   (distance, index); accepted as in ss_match_cfg; queries with an out-of-range frame
 *   get {-1, 256, 256}.
 * BRUTE: d_kp_taken and d_queries ignored (n_queries must be 0); d_map_desc [n_map][32], or
 *   NULL to use the map prepared by ss_brute_map_prepare (its n_map must equal the prepared
 *   row count, else SS_EINVAL); d_out [n_frames][kp_capacity]: per keypoint, top-2 over the
 *   map by (distance, index); slots >= the frame's count get {-1, 256, 256}; n_map = 0 (an
 *   empty map) gives {-1, 256, 256} everywhere.  A non-NULL d_map_desc overwrites (forgets)
 *   the prepared map. */
ss_status ss_match_projection(ss_ctx* ctx, int32_t n_frames, const ss_keypoint* d_kps,
                              const uint8_t* d_desc, const int32_t* d_counts,
                              const uint8_t* d_kp_taken, int32_t n_queries,
                              const ss_mp_query* d_queries, const uint8_t* d_map_desc, int32_t n_map,
                              const ss_match_cfg* cfg, ss_match* d_out, ss_stream_t stream);

/* Map-sharded brute force (DESIGN.md §3 item 15): O10 with the map
 * partitioned across ranks.  Each rank runs ss_match_brute_partial for the frames to match
 * (typically every rank's frames, all-gathered) against its shard, the partial results are
 * exchanged (all-to-all), and the frames' owner runs ss_match_brute_merge over the parts.
 * For shards that partition [0, M) (map_offset = the shard's first global index), the merge is
 * bit-identical to ss_match_projection BRUTE over the whole map.  Device pointers:
 *   ss_match_brute_partial: d_desc / d_counts as ss_orb_extract writes them; d_map_desc
 *     [n_map][32] (the shard); d_top2 [n_frames][kp_capacity][2] u64: per keypoint the two
 *     smallest (distance << 32 | (map_offset + m)) over the shard, UINT64_MAX = none (also for
 *     slots >= the frame's count).  SS_ECAPACITY if n_frames > max_frames or n_map > max_map;
 *     SS_EINVAL for negative sizes / offset, map_offset + n_map > 2^31 - 1 or NULL buffers.
 *   ss_match_brute_merge: d_parts [n_parts][n_frames][kp_capacity][2] (the shards' d_top2,
 *     any order), cfg as BRUTE (th, ratio); d_out [n_frames][kp_capacity] as
 *     ss_match_projection BRUTE (idx = global map index or -1).  n_parts >= 1. */
ss_status ss_match_brute_partial(ss_ctx* ctx, int32_t n_frames, const uint8_t* d_desc, const int32_t* d_counts,
                                 const uint8_t* d_map_desc, int32_t n_map, int32_t map_offset, uint64_t* d_top2,
                                 ss_stream_t stream);
ss_status ss_match_brute_merge(ss_ctx* ctx, int32_t n_frames, const int32_t* d_counts, int32_t n_parts,
                               const uint64_t* d_parts, const ss_match_cfg* cfg, ss_match* d_out, ss_stream_t stream);

/* BRUTE map preparation (O10; the shared map of C5 is server state that changes rarely):
 * enqueues on `stream` the one-time expansion of d_map_desc [n_map][32] (DEVICE) into the
 * ctx's tensor-core operand scratch (s8 +-1 rows in the UMMA K-major layout, 256 B per row),
 * so BRUTE calls with d_map_desc = NULL and the same n_map (ss_match_projection,
 * ss_match_brute_partial, ss_track_tick's io->d_map_desc) expand only their keypoints.  The
 * prepared copy is a snapshot: after changing the map's contents, call again.  Any BRUTE call
 * with a non-NULL map replaces the scratch and forgets the preparation.  SS_EINVAL for
 * n_map < 1 or a NULL map, SS_ECAPACITY for n_map > max_map. */
ss_status ss_brute_map_prepare(ss_ctx* ctx, const uint8_t* d_map_desc, int32_t n_map, ss_stream_t stream);

/* O11: the per-map-point half of "search local points" (ORB-SLAM3
 * Frame::isInFrustum + MapPoint::PredictScale + ORBmatcher::RadiusByViewingCos): map point
 * i is tested against the camera of frame d_point_frame[i] and written as WINDOW query i.
 * Device pointers: d_cams [n_frames] ss_camera, d_points [n_points] ss_map_point,
 * d_point_frame [n_points] i32, d_queries [n_points] ss_mp_query (output).  In the frustum
 * (Pc.z >= 0, u, v inside the bounds, 0.8*min_dist <= |Pw - ow| <= 1.2*max_dist, viewing
 * cosine >= 0.5): {frame, u, v, level, radius} with level = the smallest n in [0, L-1]
 * with max_dist / dist <= scale[n] (else L-1) and radius = f32(f32(rv * th) * scale[level]),
 * rv = 2.5 if the viewing cosine > 0.998 else 4.0.  Otherwise (or a frame index outside
 * [0, n_frames)) {frame, 0, 0, -1, 0}, which ss_match_projection never matches.  Every f32
 * operation is rounded once in the documented order (no contraction): bit-exact with the
 * oracle.  The map points' descriptors are the queries' descriptors (same index).
 * SS_EINVAL for negative sizes or NULL buffers with n_points > 0. */
ss_status ss_project_points(ss_ctx* ctx, int32_t n_frames, const ss_camera* d_cams, int32_t n_points,
                            const ss_map_point* d_points, const int32_t* d_point_frame, float th,
                            ss_mp_query* d_queries, ss_stream_t stream);

/* O12: stereo matching of rectified pairs (ORB-SLAM2 Frame::ComputeStereoMatches; the input
 * of the paper's stereo tracking, PAPER.md L163 / L246), run after ss_orb_extract on the
 * SAME ctx and frames: pair i = extracted frames 2i (left) and 2i+1 (right); d_frames,
 * frame_stride, pitch, d_kps, d_desc, d_counts are that call's arguments (the pyramid levels
 * >= 1 are read from the ctx's scratch, so no other ss_orb_extract may run on the ctx in
 * between).  Per left keypoint iL (slot iL of pair i): d_uright[i][iL] = the right-image x
 * coordinate (level-0 px, sub-pixel) and d_depth[i][iL] = bf / disparity, or -1 for both when
 * there is no stereo match (slots >= the left count are left untouched).  Matching: right
 * keypoints on octaves [o-1, o+1] whose row span [floor(y - 2 s), ceil(y + 2 s)] holds
 * (int)vL, with uL - bf/baseline <= uR <= uL; smallest Hamming (lowest index on ties) below
 * 100, kept if < 75; 11x11 centre-subtracted SAD over shifts [-5, 5] on octave o's level,
 * parabola sub-pixel offset, disparity in [0, bf/baseline); then every match whose SAD is
 * >= 1.5f*1.4f*(median accepted SAD) is dropped.  Bit-exact with the oracle (DESIGN.md §3
 * item 12).  SS_EINVAL for bad sizes, pitches, NULL buffers or bf / baseline <= 0;
 * SS_ECAPACITY if 2*n_pairs > max_frames. */
ss_status ss_stereo_match(ss_ctx* ctx, int32_t n_pairs, const uint8_t* d_frames, int64_t frame_stride, int32_t pitch,
                          const ss_keypoint* d_kps, const uint8_t* d_desc, const int32_t* d_counts, float bf,
                          float baseline, float* d_uright, float* d_depth, ss_stream_t stream);

/* A map point seen in the previous frame, for ss_match_last_frame (O13), 24 bytes: world
 * position, the angle (deg, [0, 360)) and octave of the previous frame's keypoint it was matched
 * to (ORB-SLAM LastFrame.mvKeysUn[i].angle / .octave). */
typedef struct {
  float pos[3];
  float angle_deg;
  int32_t octave;
  int32_t reserved;
} ss_frame_point;

/* O13: frame-to-frame projection matching, ORB-SLAM SearchByProjection(CurrentFrame,
 * LastFrame, th, bMono) as run by TrackWithMotionModel -- the "ORB-Matching" step of the
 * paper's tracking-time breakdown (§5, Fig. 8); DESIGN.md §3 item 14.  Run after
 * ss_orb_extract (same layouts).  Device pointers:
 *   d_cams [n_frames]        current camera of each frame (the motion-model pose)
 *   d_last_cams [n_frames]   previous camera of each frame, or NULL (only read when mb > 0)
 *   d_kp_taken               [n_frames][kp_capacity] u8 or NULL (non-zero = not a candidate)
 *   d_point_offsets [n_frames+1] i32: frame f's points are [off[f], off[f+1]), off[0] = 0,
 *                            non-decreasing (the host never reads it: no synchronisation)
 *   d_points / d_point_desc  [off[n_frames]] ss_frame_point / [off[n_frames]][32] u8
 *   d_out [off[n_frames]]    per point: idx = keypoint index in its frame or -1; dist / dist2 =
 *                            best / second Hamming distance over its candidates (256 = none)
 *   d_n_matches [n_frames]   kept matches per frame, or NULL
 *   d_kp_matched             [n_frames][kp_capacity] u8 or NULL: 1 where d_kp_taken is non-zero
 *                            or a kept match claims the keypoint, else 0 -- the d_kp_taken of
 *                            the following search-local-points ss_match_projection (ORB-SLAM's
 *                            SearchLocalPoints skips keypoints the motion model already matched)
 * Per point: Pc = R*Pw + t, skip if Pc.z < 0, u = fx*X/Z + cx, v = fy*Y/Z + cy inside the
 * bounds; window r = th * scale[octave] (|x-u| < r and |y-v| < r, f32); levels [o-1, o+1], or,
 * when mb > 0 (stereo baseline) and the current camera centre seen from the last camera has
 * z > mb, [o, L-1] (forward), or z < -mb, [0, o] (backward); best by (distance, index),
 * accepted iff <= th_high (TH_HIGH = 100).  A keypoint claimed by several points keeps the
 * min (distance, point).  check_orientation != 0: rotation histogram of (angle_last -
 * angle_cur) with ORB-SLAM's bin = roundf(rot * (1.0f/30)), matches outside the three
 * largest bins (ComputeThreeMaxima, 10 % rule) rejected.  min_matches > 0: a frame keeping
 * fewer matches is redone with window factor 2*th (TrackWithMotionModel's retry).  Points
 * with an octave outside [0, L-1] get {-1, 256, 256}.  Bit-exact with the oracle.
 * SS_EINVAL for negative sizes, NULL buffers, th <= 0; SS_ECAPACITY if n_frames > max_frames.
 * Uses the ctx's matcher scratch (row index, claims): not concurrently with another match
 * call on the same ctx.  It also prepares the WINDOW matcher's row index and claims for these
 * keypoints, so a following ss_match_projection WINDOW on the same d_kps / d_counts (no
 * ss_orb_extract or ss_stereo_match in between) skips its match_prepare kernel. */
ss_status ss_match_last_frame(ss_ctx* ctx, int32_t n_frames, const ss_camera* d_cams, const ss_camera* d_last_cams,
                              float mb, const ss_keypoint* d_kps, const uint8_t* d_desc, const int32_t* d_counts,
                              const uint8_t* d_kp_taken, const int32_t* d_point_offsets,
                              const ss_frame_point* d_points, const uint8_t* d_point_desc, float th,
                              int32_t th_high, int32_t check_orientation, int32_t min_matches, ss_match* d_out,
                              int32_t* d_n_matches, uint8_t* d_kp_matched, ss_stream_t stream);

/* Keypoint distribution of the following ss_orb_extract calls on ctx (default quadtree):
 * SS_DIST_QUADTREE = ORB-SLAM's DistributeOctTree reading (O4); SS_DIST_GRID_TOPN = grid
 * top-N (O4g: K = FAST cells with a candidate, q = ceil(N_l / K), each cell keeps its q best
 * by (score desc, rank asc), then the N_l best of those; <= N_l keypoints per level).
 * SS_EINVAL for an unknown mode.  Host only. */
#define SS_DIST_QUADTREE 0
#define SS_DIST_GRID_TOPN 1
ss_status ss_set_distribution(ss_ctx* ctx, int32_t mode);

/* ---- one tracking tick from host memory (the native executor of a client batch) ---- */

/* Inputs and outputs of ss_track_tick, all HOST pointers (page-locked memory makes the copies
 * asynchronous; pageable memory works but the copies then block).  NULL = unused. */
typedef struct {
  /* n_frames frames, frame f row y at frames + f*frame_stride + y*pitch (pitch >= width) */
  const uint8_t* frames;
  int64_t frame_stride;
  int32_t pitch;
  /* stereo (O12): bf > 0 and baseline > 0 match pairs (2i, 2i+1); 0 = no stereo */
  float bf, baseline;
  /* WINDOW (search local points, O11 + O9): cams [n_frames], points / point_frame /
   * point_desc [n_points], taken [n_frames][kp_capacity] (may be NULL), projection th */
  const ss_camera* cams;
  int32_t n_points;
  const ss_map_point* points;
  const int32_t* point_frame;
  const uint8_t* point_desc;
  const uint8_t* taken;
  float th;
  /* BRUTE (O10): a DEVICE-resident map [n_map][32] (a shared map is uploaded once), or NULL
   * for the map prepared on this ctx by ss_brute_map_prepare */
  const uint8_t* d_map_desc;
  int32_t n_map;
  /* outputs: kps [n_frames][kp_capacity], desc [n_frames][kp_capacity][32], counts
   * [n_frames][n_levels+1], matches [n_points] (WINDOW) or [n_frames][kp_capacity] (BRUTE),
   * uright / depth [n_frames/2][kp_capacity] (stereo).  Any output may be NULL (not copied). */
  ss_keypoint* kps;
  uint8_t* desc;
  int32_t* counts;
  ss_match* matches;
  float* uright;
  float* depth;
  /* O13 frame-to-frame matching (ss_match_last_frame), run before the WINDOW match when
   * lf_offsets != NULL: lf_offsets [n_frames+1], lf_points / lf_desc [lf_offsets[n_frames]]
   * (<= max_queries), current cameras = cams, last_cams [n_frames] (read when mb > 0);
   * outputs lf_matches [lf_offsets[n_frames]], lf_n_matches [n_frames] (may be NULL).  The
   * WINDOW match then skips keypoints that are taken OR kept by O13 (ORB-SLAM's
   * SearchLocalPoints skips the motion model's matches). */
  const int32_t* lf_offsets;
  const ss_frame_point* lf_points;
  const uint8_t* lf_desc;
  const ss_camera* last_cams;
  float mb, lf_th;
  int32_t lf_min_matches;
  ss_match* lf_matches;
  int32_t* lf_n_matches;
  /* 1 = the map state is DEVICE-resident (the server's map, kept in HBM across ticks):
   * points, point_frame, point_desc, taken, lf_points, lf_desc and last_cams are device
   * pointers and are not copied; frames, cams and lf_offsets stay host inputs. */
  int32_t map_resident;
  /* 1 = replay from a CUDA graph: the ctx caches (LRU, 16 entries) an instantiated graph of
   * the tick per distinct argument set (every pointer and size in io, cfg, n_frames and
   * lf_offsets[n_frames]); the second call with the same arguments captures it, later ones
   * launch it (one launch instead of ~30 API calls).  Requires every HOST buffer of io to be
   * page-locked and to stay allocated while the ctx lives (a ring of pinned buffers).  The
   * buffers' CONTENTS may change freely between calls.  Ignored while profiling events are
   * installed or when the stream is already capturing. */
  int32_t reuse_graph;
  /* NULL, or ONE host block (page-locked) that receives every output of the tick in a single
   * device-to-host copy instead of one copy per output (each copy costs the DMA engine a few
   * microseconds whatever its size: c2 end to end 75k -> 92k frames/s).  When set, the
   * separate output pointers above (kps ... lf_n_matches) are ignored and the block holds, in
   * this order and packed: kps [n_frames][kp_capacity], desc [n_frames][kp_capacity][32],
   * counts [n_frames][n_levels+1], lf_n_matches [n_frames], lf_matches
   * [lf_offsets[n_frames]] (0 without O13), matches [n_points] (WINDOW) or
   * [n_frames][kp_capacity] (BRUTE), uright / depth [n_frames/2][kp_capacity] (stereo only),
   * each section starting on a 256-byte boundary; ss_tick_packed_layout gives the offsets. */
  void* out_packed;
  /* NULL, or ONE host block (page-locked) holding the tick's per-tick host inputs, copied in a
   * single host-to-device copy: frames [n_frames][frame_stride] (dense: frame_stride = height
   * * pitch, pitch a multiple of 16 and <= the width rounded up to 16), cams [n_frames], and
   * lf_offsets [n_frames+1] (read only with O13), each section on a 256-byte boundary
   * (ss_tick_packed_in_layout).  When set, frames, cams and lf_offsets above are ignored; the
   * other inputs (the map state, last_cams) are unchanged. */
  const void* in_packed;
} ss_tick_io;

/* Byte offsets of ss_tick_io.in_packed's sections for n_frames frames of frame_stride bytes:
 * offsets[0..2] = frames, cams, lf_offsets; offsets[3] = total bytes.  Host only. */
ss_status ss_tick_packed_in_layout(const ss_ctx* ctx, int32_t n_frames, int64_t frame_stride, int64_t* offsets);

/* Byte offsets of the sections of ss_tick_io.out_packed for a tick: offsets[0..7] = kps,
 * desc, counts, lf_n_matches, lf_matches, matches, uright, depth; offsets[8] = total bytes.
 * n_lf = lf_offsets[n_frames] (0 without O13), brute = 1 for a BRUTE tick (matches per
 * keypoint slot), stereo = 1 when bf > 0 and baseline > 0.  Host only; SS_EINVAL on NULL or
 * negative sizes. */
ss_status ss_tick_packed_layout(const ss_ctx* ctx, int32_t n_frames, int32_t n_points, int64_t n_lf, int32_t brute,
                                int32_t stereo, int64_t* offsets);

/* One tick of the hot path for a batch of client frames, enqueued on `stream` from a single
 * call: host -> device copies into ctx-owned staging buffers (sized at ss_create: max_frames
 * frames, max_queries points), ss_orb_extract, ss_stereo_match (if io->bf > 0),
 * ss_match_last_frame (if io->lf_offsets, WINDOW only), ss_project_points +
 * ss_match_projection WINDOW (cfg->mode == SS_MATCH_WINDOW, n_points > 0) or
 * ss_match_projection BRUTE (cfg->mode == SS_MATCH_BRUTE), device -> host copies of the
 * outputs.  Asynchronous: outputs are valid once the stream reaches the end of the call; the
 * caller must not reuse the ctx for another tick before then.  Same results and errors as
 * the individual calls (SS_ECAPACITY when n_frames > max_frames or n_points > max_queries). */
ss_status ss_track_tick(ss_ctx* ctx, int32_t n_frames, const ss_match_cfg* cfg, const ss_tick_io* io,
                        ss_stream_t stream);

/* A server's tick loop in native code: n_ticks calls of ss_track_tick, tick t on ctxs[t %
 * n_ctx] and streams[t % n_ctx] with ios[(t % n_ctx) * n_io + t % n_io] (HOST arrays; each
 * ctx owns its own staging, so consecutive ticks on different ctxs / streams overlap: one
 * tick's copies with another's kernels).  Same requirements, results and errors as the
 * individual calls (stops at the first failing tick).  Asynchronous like ss_track_tick. */
ss_status ss_track_run(ss_ctx* const* ctxs, int32_t n_ctx, const ss_stream_t* streams, int32_t n_frames,
                       const ss_match_cfg* cfg, const ss_tick_io* ios, int32_t n_io, int32_t n_ticks);

/* ---- profiling hook (bench.py; does not synchronise) ---- */

/* When n_events > 0, every following ss_orb_extract / ss_match_projection records the
 * caller's events (cudaEvent_t handles created with timing enabled; host array copied) on
 * its stream: the next unused event before its first operation, then one after every
 * kernel it launches, continuing across calls until the next ss_profile_events call
 * (n_events = 0 disables; events beyond n_events are not recorded).  One extract records a
 * start event, then a (before, after) pair around every kernel launch, in this order:
 * fast(level 0), pyramid (levels 1..L-1, one launch), fast(levels >= 1), distribute (all
 * levels, one launch), describe -- 11 events (while events are installed the level-0
 * branch runs in line on `stream` instead of on its side stream, so each kernel is timed
 * alone).  WINDOW match: a pair per kernel
 * (match_prepare, match_window[, match_resolve if dedup]; the match_prepare pair encloses
 * no work when ss_match_last_frame already prepared the index); BRUTE: brute_expand, brute_tc,
 * brute_merge; ss_project_points: project; ss_stereo_match: stereo_prepare, stereo, stereo_outliers;
 * ss_match_last_frame: lastframe; ss_match_brute_partial: brute_expand, brute_tc, brute_shard_top2;
 * ss_match_brute_merge: brute_parts_merge.
 * Works under CUDA-graph stream capture (the records become graph event nodes).
 * *next_index (may be NULL) receives the index of the next event to be recorded. */
ss_status ss_profile_events(ss_ctx* ctx, void* const* events, int32_t n_events);
ss_status ss_profile_next(ss_ctx* ctx, int32_t* next_index);

/* ---- debug / test hooks (synchronise the ctx's device; not for the hot path) ---- */

/* Device pointer + pitch of pyramid level `level` (>= 1) of frame slot `frame` as left by the
 * last ss_orb_extract (level 0 is the caller's frame). */
ss_status ss_debug_level(ss_ctx* ctx, int32_t frame, int32_t level, const uint8_t** d_ptr,
                         int32_t* pitch);

/* FAST candidates (O3) of (frame, level) from the last ss_orb_extract, in rank order
 * (cells row-major, then y, then x), copied to host arrays of capacity `cap`
 * (h_lx, h_ly: pixel; h_score: M).  *n = count; SS_ECAPACITY if count > cap. */
ss_status ss_debug_candidates(ss_ctx* ctx, int32_t frame, int32_t level, int32_t* h_lx, int32_t* h_ly,
                              int32_t* h_score, int32_t cap, int32_t* n);

/* Global-timer timestamps (ns) of the distribution phases of (frame, level) in the last
 * ss_orb_extract: [0] start, [1] candidate count known, [2] candidates gathered, [3] dense
 * tables cleared, [4] keys + per-depth node counts, [5] stop rules evaluated, [6] partial round,
 * [7] best keys, [8] kept keys listed, [9] written (dense path; unused slots unspecified). */
ss_status ss_debug_phase_times(ss_ctx* ctx, int32_t frame, int32_t level, int64_t* h_ns, int32_t n);

/* Number of (frame, level) distributions of the last ss_orb_extract that exceeded the
 * in-shared-memory capacity and took the global-memory path (for tests/benchmarks). */
ss_status ss_debug_overflow_count(ss_ctx* ctx, int32_t* n);

/* Which quadtree paths the (frame, level) distributions of the last ss_orb_extract took
 * (DESIGN.md §5 distribute_kernel): *n_sort_smem = how many fell back from the dense-histogram
 * fast path to the in-shared-memory sort path (the stop rules needed a depth beyond the dense
 * tables), *n_global = how many ran on global scratch (> 8192 candidates).  Either may be NULL. */
ss_status ss_debug_distribution_paths(ss_ctx* ctx, int32_t* n_sort_smem, int32_t* n_global);

/* Lanes per query of the following WINDOW matches on ctx (1, 2, 4 or 8; 0 = chosen per launch
 * from the query count, the default).  Results are identical for every value; tests use this
 * to cover each kernel instance.  SS_EINVAL for other values.  Host only. */
ss_status ss_debug_match_lanes(ss_ctx* ctx, int32_t lanes);

/* Blurred-sample capture (S6 blur parity): while d_samples != NULL, every following
 * ss_orb_extract also writes, per output keypoint slot, the 512 blurred values (u8) its 256
 * comparisons read -- d_samples[f][slot][2b + e] = B_level(ly + oy, lx + ox) at point e of
 * comparison b, (ox, oy) the rotated pattern offset (O6, O7) -- into the caller's DEVICE buffer
 * of n_frames * kp_capacity * 512 bytes (slots >= the frame's count untouched).  The capture
 * runs a second instance of the descriptor kernel; NULL (the default) restores the product
 * kernel.  Host only (the pointer is stored, nothing is enqueued). */
ss_status ss_debug_capture_samples(ss_ctx* ctx, uint8_t* d_samples);

#ifdef __cplusplus
}
#endif
#endif /* SS_H */
