// ss_api.cpp -- host side of libss: parameter derivation, validation, scratch ownership and
// the launch sequence of each C-ABI entry point (include/ss.h).  No per-call allocation,
// no host synchronisation on the hot path; every entry point returns a status.
#include <climits>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <utility>
#include <vector>

#include "ss_internal.h"

using namespace ss;

namespace {

thread_local std::string g_err = "no error";

ss_status fail(ss_status st, const std::string& msg) {
  g_err = msg;
  return st;
}

#define SS_CUDA_TRY(expr)                                                                    \
  do {                                                                                       \
    cudaError_t _e = (expr);                                                                 \
    if (_e != cudaSuccess) return fail(SS_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(_e)); \
  } while (0)

int imax(int a, int b) { return a > b ? a : b; }
int imin(int a, int b) { return a < b ? a : b; }

// O0: ORB-SLAM's ORBextractor constructor quantities in f32 (see ss.h).
ss_status params_init(int32_t W, int32_t H, int32_t nf, int32_t L, float sf, int32_t ini, int32_t mn,
                      ss_orb_params* p) {
  if (L < 1 || L > SS_MAX_LEVELS) return fail(SS_EINVAL, "n_levels must be in [1, 8]");
  if (W < 64 || H < 64 || W > 2048 || H > 2048) return fail(SS_EINVAL, "width/height must be in [64, 2048]");
  if (nf < 1) return fail(SS_EINVAL, "n_features must be >= 1");
  if (!(sf > 1.0f)) return fail(SS_EINVAL, "scale_factor must be > 1");
  if (ini < 1 || mn < 1 || ini > 254 || mn > 254) return fail(SS_EINVAL, "FAST thresholds must be in [1, 254]");
  ss_orb_params q;
  std::memset(&q, 0, sizeof(q));
  q.width = W;
  q.height = H;
  q.n_features = nf;
  q.n_levels = L;
  q.scale_factor = sf;
  q.ini_th_fast = ini;
  q.min_th_fast = mn;
  volatile float s = 1.0f;  // keep every product a separate f32 rounding
  q.scale[0] = 1.0f;
  for (int l = 1; l < L; l++) {
    s = s * sf;
    q.scale[l] = s;
  }
  for (int l = 0; l < L; l++) {
    volatile float inv = 1.0f / q.scale[l];
    q.inv_scale[l] = inv;
    volatile float fw = (float)W * q.inv_scale[l];
    volatile float fh = (float)H * q.inv_scale[l];
    q.level_w[l] = (int32_t)std::nearbyint((float)fw);  // round half even (default mode)
    q.level_h[l] = (int32_t)std::nearbyint((float)fh);
  }
  const float factor = 1.0f / sf;
  volatile float num = (float)nf * (1.0f - factor);
  volatile float den = 1.0f - (float)std::pow((double)factor, (double)L);
  volatile float per = num / den;
  int sum = 0;
  for (int l = 0; l < L - 1; l++) {
    q.n_per_level[l] = (int32_t)std::nearbyint((float)per);
    sum += q.n_per_level[l];
    per = per * factor;
  }
  q.n_per_level[L - 1] = imax(nf - sum, 0);
  int cap = 0;
  for (int l = 0; l < L; l++) {
    const int maxbx = q.level_w[l] - kEdgeThreshold + 3, maxby = q.level_h[l] - kEdgeThreshold + 3;
    const float width = (float)(maxbx - kMinBorder), height = (float)(maxby - kMinBorder);
    const int cols = (int)(width / (float)kCellPx), rows = (int)(height / (float)kCellPx);
    if (cols < 1 || rows < 1) return fail(SS_EINVAL, "a pyramid level is smaller than one FAST cell");
    q.cell_cols[l] = cols;
    q.cell_rows[l] = rows;
    q.cell_w[l] = (int)std::ceil(width / (float)cols);
    q.cell_h[l] = (int)std::ceil(height / (float)rows);
    const int nini = (int)std::round(width / height);  // half away from zero
    if (nini < 1 || nini > 62) return fail(SS_EINVAL, "level aspect ratio outside the quadtree's root range");
    q.n_ini[l] = nini;
    q.level_cap[l] = imax(q.n_per_level[l] + 2, 4 * nini);
    cap += q.level_cap[l];
  }
  q.kp_capacity = cap;
  *p = q;
  return SS_OK;
}

// Bilinear source coordinate of destination index d (INTER_LINEAR_EXACT): packed
// x0 | wx1 << 16 | (x1 - x0) << 25 with wx1 = rne(frac * 256).
uint32_t lin_coef(int d, int sn, int dn) {
  volatile double ratio = (double)sn / (double)dn;
  volatile double fx = ((double)d + 0.5) * ratio;
  double f = fx - 0.5;
  double fl = std::floor(f);
  int x0 = (int)fl;
  double frac = f - fl;
  if (x0 < 0) { x0 = 0; frac = 0.0; }
  if (x0 >= sn - 1) { x0 = sn - 1; frac = 0.0; }
  const int w1 = (int)std::nearbyint(frac * 256.0);
  const int x1 = imin(x0 + 1, sn - 1);
  return (uint32_t)x0 | ((uint32_t)w1 << 16) | ((uint32_t)(x1 - x0) << 25);
}

}  // namespace

struct ss_ctx {
  int device = 0;
  ss_orb_params p{};
  Geom g{};
  int max_frames = 0, max_queries = 0, max_map = 0, max_splits = 0;
  std::vector<CellInfo> cells_h;
  std::vector<BandInfo> bands_h;
  // device scratch
  CellInfo* cells = nullptr;
  BandInfo* bands = nullptr;
  uint32_t* xytab = nullptr;  // per level l >= 1: xtab [w_l], ytab [h_l]
  uint32_t* qtab = nullptr;   // quadtree key tables (launch_distribute_tables)
  PyrLvl* pyr_plan = nullptr;   // [pyr_blocks][L] fused-pyramid block records
  uint4* pyr_gtab = nullptr;    // per level >= 1: 4-column group coefficients
  int pyr_blocks = 0, pyr_buf0 = 0, pyr_buf1 = 0, pyr_smem = 0;
  std::vector<int64_t> xoff, yoff;
  uint8_t* pyr = nullptr;
  uint32_t* slots = nullptr;
  int32_t* cell_counts = nullptr;
  uint32_t* selected = nullptr;
  int32_t* sel_counts = nullptr;
  uint8_t* ovf = nullptr;
  int64_t ovf_frame_bytes = 0;
  int64_t* ovf_level_off = nullptr;
  int32_t* ovf_counter = nullptr;  // [0] overflowed levels, [1] capacity violations, [2] sort fallbacks
  int8_t* pattern = nullptr;
  unsigned long long* claim = nullptr;
  unsigned long long* claim_lf = nullptr;  // O13's own dedup claims
  uint16_t* rowidx = nullptr;  // WINDOW matcher: first keypoint per (frame, level, row)
  // rowidx + claim already prepared (by ss_match_last_frame) for these keypoints: the next
  // WINDOW match skips match_prepare.  Cleared by every ss_orb_extract.
  bool win_ready = false;
  const ss_keypoint* win_kps = nullptr;
  const int32_t* win_counts = nullptr;
  int win_nf = 0;
  uint64_t* phase_ts = nullptr;  // distribution phase timestamps [max_frames][L][16] (debug hook)
  unsigned long long* partial = nullptr;
  int dist_mode = SS_DIST_QUADTREE;  // ss_set_distribution
  PatchMaps maps{};                  // TMA maps of the describe kernel (levels >= 1 at ss_create)
  // test hooks: lanes per WINDOW query (0 = chosen per launch), blurred-sample capture buffer
  int win_lanes = 0;
  int fast_flat = 0;         // SS_FAST_FLAT (A/B): flat band-major FAST grid, 2 = level 0 first
  bool fast_split = false;  // SS_FAST_SPLIT=1: level 0's FAST on a side branch beside the pyramid (A/B)
  bool tick_fork = true;  // ss_track_tick: local-map projection on the aux branch (SS_TICK_FORK=0: serial)
  uint8_t* dbg_samples = nullptr;
  int32_t* stereo_sad = nullptr;  // O12: accepted SAD per left keypoint [max_frames/2][cap]
  // ss_track_tick staging (device copies of the host inputs / outputs of a tick)
  uint8_t* io_frames = nullptr;   // [max_frames][H][io_pitch]
  uint8_t* io_frames_lin = nullptr;  // [max_frames][H][W]: dense frames with an unaligned pitch land here first
  int32_t io_pitch = 0;
  ss_keypoint* io_kps = nullptr;
  uint8_t* io_desc = nullptr;
  int32_t* io_counts = nullptr;
  ss_camera* io_cams = nullptr;
  ss_map_point* io_points = nullptr;
  int32_t* io_pf = nullptr;
  uint8_t* io_pdesc = nullptr;
  uint8_t* io_taken = nullptr;
  ss_mp_query* io_queries = nullptr;
  ss_match* io_matches = nullptr;
  float* io_uright = nullptr;
  float* io_depth = nullptr;
  int32_t* io_lf_off = nullptr;  // O13 staging
  ss_frame_point* io_lf_pts = nullptr;
  uint8_t* io_lf_desc = nullptr;
  ss_camera* io_last_cams = nullptr;
  ss_match* io_lf_matches = nullptr;
  int32_t* io_lf_n = nullptr;
  uint8_t* io_packed = nullptr;  // ss_tick_io.out_packed: every output of a tick, packed (one D2H copy)
  uint8_t* io_inpacked = nullptr;  // ss_tick_io.in_packed: frames + cams + lf_offsets (one H2D copy)
  uint8_t* io_lf_mask = nullptr;
  // ss_track_tick graph cache (io->reuse_graph): LRU of instantiated tick graphs by argument key
  struct TickGraph {
    std::vector<unsigned char> key;
    cudaGraphExec_t exec;
    uint64_t last_use;
  };
  static constexpr size_t kTickGraphs = 16;
  std::vector<TickGraph> tick_graphs;
  uint64_t tick_clock = 0;
  int8_t* brute_qexp = nullptr;  // BRUTE: keypoint descriptors expanded to s8 +-1 (k_brute_tc.cu)
  int8_t* brute_mexp = nullptr;  // BRUTE: map descriptors expanded to s8 +-1
  int prepared_map = -1;         // rows of the map brute_mexp holds from ss_brute_map_prepare (-1: none)
  int n_sm = 148;
  // per-extract DAG: level 0's FAST + distribution on side stream 0 right away; level l >= 1's
  // on side stream 1 + (l % kSideLevel) as soon as the pyramid (caller's stream) has level l
  static constexpr int kSide = 4, kSideLevel = 3;
  cudaStream_t side[kSide] = {};
  cudaEvent_t ev_fork = nullptr, ev_level[kMaxLevels] = {}, ev_join[kSide] = {};
  // ss_track_tick: the local-map projection runs on its own branch, concurrently with extraction
  cudaStream_t aux = nullptr;
  cudaEvent_t ev_aux0 = nullptr, ev_aux1 = nullptr;
  // profiling hook
  std::vector<cudaEvent_t> prof;
  size_t prof_next = 0;
  // last extract (debug hooks)
  const uint8_t* last_frames = nullptr;
  int64_t last_stride = 0;
  int32_t last_pitch = 0;
  int last_n = 0;
};

namespace {

// Clears any stale error left in this thread by unrelated runtime calls, so that the launch
// checks report only our own launches.  (No stream query here: it is illegal while the caller
// captures the stream into a CUDA graph.)
cudaError_t check_stream(cudaStream_t) {
  (void)cudaGetLastError();
  return cudaSuccess;
}

inline void prof_mark(ss_ctx* c, cudaStream_t s) {
  // External: under stream capture the record becomes a real graph event node (a plain
  // record would only be a capture-internal dependency and could not be timed).
  if (c->prof_next < c->prof.size()) cudaEventRecordWithFlags(c->prof[c->prof_next++], s, cudaEventRecordExternal);
}

void free_ctx(ss_ctx* c) {
  if (!c) return;
  cudaSetDevice(c->device);
  void* ptrs[] = {c->cells, c->bands, c->xytab, c->qtab, c->pyr_plan, c->pyr_gtab, c->pyr, c->slots, c->cell_counts, c->selected, c->sel_counts, c->ovf,
                  c->ovf_level_off, c->ovf_counter, c->pattern, c->claim, c->claim_lf, c->partial, c->rowidx, c->phase_ts,
                  c->brute_qexp, c->brute_mexp, c->stereo_sad, c->io_frames, c->io_frames_lin, c->io_kps, c->io_desc, c->io_counts,
                  c->io_cams, c->io_points, c->io_pf, c->io_pdesc, c->io_taken, c->io_queries, c->io_matches,
                  c->io_uright, c->io_depth, c->io_lf_off, c->io_lf_pts, c->io_lf_desc, c->io_last_cams,
                  c->io_lf_matches, c->io_lf_n, c->io_lf_mask, c->io_packed, c->io_inpacked};
  for (void* q : ptrs)
    if (q) cudaFree(q);
  for (ss_ctx::TickGraph& tg : c->tick_graphs)
    if (tg.exec) cudaGraphExecDestroy(tg.exec);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_aux0) cudaEventDestroy(c->ev_aux0);
  if (c->ev_aux1) cudaEventDestroy(c->ev_aux1);
  if (c->aux) cudaStreamDestroy(c->aux);
  for (cudaEvent_t e : c->ev_level)
    if (e) cudaEventDestroy(e);
  for (cudaEvent_t e : c->ev_join)
    if (e) cudaEventDestroy(e);
  for (cudaStream_t q : c->side)
    if (q) cudaStreamDestroy(q);
  delete c;
}

// Byte offsets of a tick's packed outputs (ss_tick_io.out_packed; ss.h documents the order):
// o[0..7] = kps, desc, counts, lf_n, lf_matches, matches, uright, depth; o[8] = total.
void packed_layout(const Geom& g, int64_t n_frames, int64_t n_match, int64_t n_lf, bool stereo, int64_t* o) {
  const int64_t cap = g.kp_capacity;
  const int64_t ns = stereo ? (n_frames / 2) * cap : 0;
  const int64_t len[8] = {(int64_t)sizeof(ss_keypoint) * n_frames * cap, n_frames * cap * SS_DESC_BYTES,
                          4 * n_frames * (g.L + 1), 4 * n_frames, (int64_t)sizeof(ss_match) * n_lf,
                          (int64_t)sizeof(ss_match) * n_match, 4 * ns, 4 * ns};
  int64_t b = 0;
  for (int i = 0; i < 8; i++) {  // every section starts on a 256-byte boundary (vector loads of desc)
    o[i] = b;
    b = (b + len[i] + 255) & ~(int64_t)255;
  }
  o[8] = o[7] + len[7];
}

// Byte offsets of a tick's packed host inputs (ss_tick_io.in_packed): frames, cams,
// lf_offsets (each on a 256-byte boundary); o[3] = total.
void packed_in_layout(int64_t n_frames, int64_t frame_stride, int64_t* o) {
  const int64_t len[3] = {n_frames * frame_stride, (int64_t)sizeof(ss_camera) * n_frames, 4 * (n_frames + 1)};
  int64_t b = 0;
  for (int i = 0; i < 3; i++) {
    o[i] = b;
    b = (b + len[i] + 255) & ~(int64_t)255;
  }
  o[3] = o[2] + len[2];
}

int64_t packed_capacity(const Geom& g, int64_t F, int64_t Qm) {
  int64_t o[9];
  packed_layout(g, F, std::max<int64_t>(Qm, F * g.kp_capacity), Qm, true, o);
  return o[8] + 256;
}

template <typename T>
cudaError_t dalloc(T** p, size_t bytes) {
  return cudaMalloc(reinterpret_cast<void**>(p), bytes > 0 ? bytes : 16);
}

}  // namespace

extern "C" {

ss_status ss_orb_params_init(int32_t width, int32_t height, int32_t n_features, int32_t n_levels, float scale_factor,
                             int32_t ini_th_fast, int32_t min_th_fast, ss_orb_params* out) {
  if (!out) return fail(SS_EINVAL, "out is NULL");
  return params_init(width, height, n_features, n_levels, scale_factor, ini_th_fast, min_th_fast, out);
}

const char* ss_last_error(const ss_ctx*) { return g_err.c_str(); }

ss_status ss_create(int32_t device, const ss_orb_params* p, int32_t max_frames, int32_t max_queries, int32_t max_map,
                    ss_ctx** out) {
  if (!p || !out) return fail(SS_EINVAL, "NULL argument");
  *out = nullptr;
  if (max_frames < 1 || max_queries < 0 || max_map < 0) return fail(SS_EINVAL, "bad capacities");
  if (max_map >= (1 << 23))  // the brute kernel's running top-2 packs (distance << 23 | map row)
    return fail(SS_EUNSUPPORTED, "max_map must be below 2^23 (8388608) map descriptors per ctx / shard");
  ss_orb_params q;
  ss_status st = params_init(p->width, p->height, p->n_features, p->n_levels, p->scale_factor, p->ini_th_fast,
                             p->min_th_fast, &q);
  if (st != SS_OK) return st;
  if (std::memcmp(&q, p, sizeof(q)) != 0) return fail(SS_EINVAL, "params differ from ss_orb_params_init's");
  int ndev = 0;
  SS_CUDA_TRY(cudaGetDeviceCount(&ndev));
  if (device < 0 || device >= ndev) return fail(SS_EINVAL, "no such device");
  SS_CUDA_TRY(cudaSetDevice(device));
  ss_ctx* c = new (std::nothrow) ss_ctx();
  if (!c) return fail(SS_ECUDA, "host allocation failed");
  c->device = device;
  c->p = q;
  if (const char* e = std::getenv("SS_TICK_FORK")) c->tick_fork = std::atoi(e) != 0;
  c->max_frames = max_frames;
  c->max_queries = max_queries;
  c->max_map = max_map;
  Geom& g = c->g;
  const int L = q.n_levels;
  g.L = L;
  g.W = q.width;
  g.H = q.height;
  g.ini_th = q.ini_th_fast;
  g.min_th = q.min_th_fast;
  int64_t poff = 0;
  int cap_off = 0, slot_off = 0, max_rw = 0, max_rh = 0;
  for (int l = 0; l < L; l++) {
    g.w[l] = q.level_w[l];
    g.h[l] = q.level_h[l];
    g.scale[l] = q.scale[l];
    g.inv_scale[l] = q.inv_scale[l];
    g.row_off[l] = l == 0 ? 0 : g.row_off[l - 1] + g.h[l - 1] + 1;
    g.pitch[l] = (g.w[l] + 15) & ~15;
    g.lvl_off[l] = 0;
    if (l >= 1) {
      g.lvl_off[l] = poff;
      poff += ((int64_t)g.pitch[l] * g.h[l] + 127) & ~(int64_t)127;
    }
    g.N[l] = q.n_per_level[l];
    g.cap[l] = q.level_cap[l];
    g.cap_off[l] = cap_off;
    cap_off += q.level_cap[l];
    g.nini[l] = q.n_ini[l];
    const int maxbx = g.w[l] - kEdgeThreshold + 3, maxby = g.h[l] - kEdgeThreshold + 3;
    g.qw[l] = maxbx - kMinBorder;
    g.qh[l] = maxby - kMinBorder;
    volatile float hx = (float)g.qw[l] / (float)g.nini[l];
    g.hX[l] = hx;
    g.qrounds[l] = kQuadRounds;
    g.qtab_off[l] = l == 0 ? 0 : g.qtab_off[l - 1] + g.qw[l - 1] + 1 + g.qh[l - 1] + 1;
    g.qtab_total = g.qtab_off[l] + g.qw[l] + 1 + g.qh[l] + 1;
    {
      int R = 0;
      while (R < 6 && (g.nini[l] << (2 * (R + 1))) <= 4096) R++;
      g.dense_r[l] = R;
    }
    // active FAST cells, row-major (DESIGN.md §3 O3)
    g.cell_first[l] = (int)c->cells_h.size();
    g.level_slot_off[l] = slot_off;
    const int wc = q.cell_w[l], hc = q.cell_h[l];
    for (int i = 0; i < q.cell_rows[l]; i++) {
      const int iniY = kMinBorder + i * hc;
      if (iniY >= maxby - 3) continue;
      const int maxY = imin(iniY + hc + 6, maxby);
      for (int j = 0; j < q.cell_cols[l]; j++) {
        const int iniX = kMinBorder + j * wc;
        if (iniX >= maxbx - 6) continue;
        const int maxX = imin(iniX + wc + 6, maxbx);
        CellInfo ci;
        ci.level = l;
        ci.x0 = iniX + 3;
        ci.y0 = iniY + 3;
        ci.x1 = maxX - 3;
        ci.y1 = maxY - 3;
        const int dw = ci.x1 - ci.x0, dh = ci.y1 - ci.y0;
        ci.slot_off = slot_off;
        ci.slot_cap = ((dw + 1) / 2) * ((dh + 1) / 2);
        ci.pad = 0;
        slot_off += ci.slot_cap;
        max_rw = imax(max_rw, dw + 6);
        max_rh = imax(max_rh, dh + 6);
        c->cells_h.push_back(ci);
      }
    }
    g.ncells[l] = (int)c->cells_h.size() - g.cell_first[l];
    g.level_slots[l] = slot_off - g.level_slot_off[l];
    if (g.ncells[l] > 4608) {
      free_ctx(c);
      return fail(SS_EUNSUPPORTED, "more than 4608 FAST cells on one level");
    }
  }
  g.pyr_frame_bytes = poff;
  g.total_cells = (int)c->cells_h.size();
  // FAST work units: runs of <= kSegCells consecutive cells of one row (same level and detect
  // rows; their windows tile [x0, x1)), biggest levels first in the grid.  8 measured best
  // on B200 (c2: 2..24 swept; smaller runs pay more halo, larger ones lose parallelism).
  // Level 0 too since FAST is one launch for all levels (round 2: 8-cell level-0 runs give
  // fewer, longer CTAs after the levels >= 1 ones; c2 fast 30.4 -> 28.1 us, 92.0k -> 94-96k
  // frames/s on one box, scripts/sweep_seg.sh; the 4-cell runs had paid off only while level 0
  // was a launch of its own beside the pyramid).
  int kSegCells = 8, kSegCells0 = 8;  // levels >= 1 / level 0 (SS_SEG / SS_SEG0 override: experiments)
  if (const char* e = std::getenv("SS_SEG")) kSegCells = imax(1, std::atoi(e));
  if (const char* e = std::getenv("SS_SEG0")) kSegCells0 = imax(1, std::atoi(e));
  g.max_band_w = g.max_band_h = g.max_cell_w = 0;
  // a row of n cells is cut into nseg = ceil(n / S) near-equal runs: cell k of the row goes
  // to run floor(k * nseg / n)
  std::vector<int> run_of(c->cells_h.size());
  for (size_t r0 = 0; r0 < c->cells_h.size();) {
    size_t r1 = r0;
    while (r1 < c->cells_h.size() && c->cells_h[r1].level == c->cells_h[r0].level && c->cells_h[r1].y0 == c->cells_h[r0].y0)
      r1++;
    const int n = (int)(r1 - r0), S = c->cells_h[r0].level == 0 ? kSegCells0 : kSegCells;
    const int nseg = (n + S - 1) / S;
    for (int k = 0; k < n; k++) run_of[r0 + k] = (int)((int64_t)k * nseg / n);
    r0 = r1;
  }
  for (size_t i = 0; i < c->cells_h.size(); i++) {
    const CellInfo& ci = c->cells_h[i];
    g.max_cell_w = imax(g.max_cell_w, ci.x1 - ci.x0);
    if (c->bands_h.empty() || c->bands_h.back().level != ci.level || c->bands_h.back().y0 != ci.y0 ||
        run_of[i] != run_of[i - 1]) {
      BandInfo b;
      b.level = ci.level;
      b.y0 = ci.y0;
      b.y1 = ci.y1;
      b.x0 = ci.x0;
      b.x1 = ci.x1;
      b.cell_first = (int)i;
      b.ncells = 0;
      b.pad = 0;
      c->bands_h.push_back(b);
    }
    BandInfo& b = c->bands_h.back();
    if (ci.x0 != b.x1 && b.ncells > 0) {
      free_ctx(c);
      return fail(SS_EUNSUPPORTED, "FAST cell windows of a row do not tile");
    }
    b.x1 = ci.x1;
    b.ncells++;
    g.max_band_w = imax(g.max_band_w, b.x1 - b.x0);
    g.max_band_h = imax(g.max_band_h, b.y1 - b.y0);
  }
  g.total_bands = (int)c->bands_h.size();
  g.level0_bands = 0;
  for (int l = 0; l < kMaxLevels; l++) g.band_first[l] = g.band_count[l] = 0;
  for (size_t i = 0; i < c->bands_h.size(); i++) {
    const int l = c->bands_h[i].level;
    if (g.band_count[l] == 0) g.band_first[l] = (int)i;
    g.band_count[l]++;
  }
  g.level0_bands = g.band_count[0];
  {
    int rp, mbw, rb, mb, nb;
    if (fast_smem_bytes(g, &rp, &mbw, &rb, &mb, &nb) > 227 * 1024) {
      free_ctx(c);
      return fail(SS_EUNSUPPORTED, "a FAST band does not fit in shared memory");
    }
  }
  g.slots_per_frame = slot_off;
  g.kp_capacity = q.kp_capacity;
  if (g.kp_capacity > 65535) {  // keypoint indices are 16-bit in the matcher's row index
    free_ctx(c);
    return fail(SS_EUNSUPPORTED, "kp_capacity above 65535");
  }
  g.max_rw = max_rw;
  g.max_rh = max_rh;
  // coefficient tables for levels >= 1
  std::vector<uint32_t> tab;
  c->xoff.assign(L, 0);
  c->yoff.assign(L, 0);
  for (int l = 1; l < L; l++) {
    c->xoff[l] = (int64_t)tab.size();
    for (int x = 0; x < g.w[l]; x++) tab.push_back(lin_coef(x, g.w[l - 1], g.w[l]));
    c->yoff[l] = (int64_t)tab.size();
    for (int y = 0; y < g.h[l]; y++) tab.push_back(lin_coef(y, g.h[l - 1], g.h[l]));
  }
  std::vector<PyrLvl> plan;
  std::vector<uint4> gtab;
  std::vector<int64_t> goff;
  if (L > 1 && !pyramid_groups(g, tab.data(), c->xoff.data(), &gtab, &goff)) {
    free_ctx(c);
    return fail(SS_EUNSUPPORTED, "scale_factor above 4/3 is not supported by the pyramid kernel");
  }
  // fused pyramid: blocks of about 128 x 96 level-0 pixels (more, smaller blocks if a
  // block does not fit).  One 1024-thread CTA per SM: while a full batch (max_frames) still
  // fits in one wave, smaller blocks shorten the launch (at most 2x the blocks per axis; c2:
  // 6x5 -> 6x6 blocks for 4 frames, 17.9 -> 16.3 us, scripts/sweep_pyr.sh)
  if (L > 1) {
    int gx = (g.w[0] + 127) / 128, gy = (g.h[0] + 95) / 96;
    {
      int nsm = 0;
      if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device) != cudaSuccess || nsm < 1) nsm = 148;
      const int gx0 = gx, gy0 = gy;
      for (;;) {
        const int nx = gy >= gx ? gx + 1 : gx, ny = gy >= gx ? gy : gy + 1;
        if ((int64_t)max_frames * nx * ny > nsm || nx > 2 * gx0 || ny > 2 * gy0) break;
        gx = nx;
        gy = ny;
      }
    }
    if (const char* e = std::getenv("SS_PYR_GX")) gx = imax(1, std::atoi(e));  // experiments
    if (const char* e = std::getenv("SS_PYR_GY")) gy = imax(1, std::atoi(e));
    while (!pyramid_plan(g, tab.data(), c->xoff.data(), c->yoff.data(), goff, gx, gy, &plan, &c->pyr_buf0,
                         &c->pyr_buf1, &c->pyr_smem)) {
      if (gx >= g.w[L - 1] / 4 || gy >= g.h[L - 1]) {
        free_ctx(c);
        return fail(SS_EUNSUPPORTED, "no pyramid block plan fits shared memory");
      }
      if (gx <= gy) gx++; else gy++;
    }
    c->pyr_blocks = gx * gy;
  }
  // overflow scratch layout
  std::vector<int64_t> ovf_off(L, 0);
  int64_t ob = 0;
  for (int l = 0; l < L; l++) {
    ovf_off[l] = ob;
    ob += distribute_ovf_bytes(g.level_slots[l]);
  }
  c->ovf_frame_bytes = ob;
  c->max_splits = 64;
  {
    int nsm = 0;
    if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, device) == cudaSuccess && nsm > 0) c->n_sm = nsm;
  }
  std::vector<int8_t> pat(1024);
  const int* ph = brief_pattern_host();
  for (int i = 0; i < 1024; i++) pat[i] = (int8_t)ph[i];
  const int64_t F = max_frames;
  cudaError_t e = cudaSuccess;
#define ALLOC(ptr, bytes)                          \
  if (e == cudaSuccess) e = dalloc(&(ptr), (bytes));
  ALLOC(c->cells, sizeof(CellInfo) * c->cells_h.size());
  ALLOC(c->bands, sizeof(BandInfo) * c->bands_h.size() * 2);  // [ordered by level | merged-launch order]
  ALLOC(c->xytab, sizeof(uint32_t) * tab.size());
  ALLOC(c->qtab, sizeof(uint32_t) * g.qtab_total);
  if (!plan.empty()) ALLOC(c->pyr_plan, sizeof(PyrLvl) * plan.size());
  if (!gtab.empty()) ALLOC(c->pyr_gtab, sizeof(uint4) * gtab.size());
  ALLOC(c->pyr, F * g.pyr_frame_bytes);
  ALLOC(c->slots, sizeof(uint32_t) * F * g.slots_per_frame);
  ALLOC(c->cell_counts, sizeof(int32_t) * F * g.total_cells);
  ALLOC(c->selected, sizeof(uint32_t) * F * g.kp_capacity);
  ALLOC(c->sel_counts, sizeof(int32_t) * F * L);
  ALLOC(c->ovf, F * c->ovf_frame_bytes);
  ALLOC(c->ovf_level_off, sizeof(int64_t) * L);
  ALLOC(c->ovf_counter, sizeof(int32_t) * 4);
  ALLOC(c->pattern, 1024);
  ALLOC(c->claim, sizeof(unsigned long long) * F * g.kp_capacity);
  ALLOC(c->claim_lf, sizeof(unsigned long long) * F * g.kp_capacity);
  ALLOC(c->rowidx, sizeof(uint16_t) * F * match_index_stride(g));
  ALLOC(c->phase_ts, sizeof(uint64_t) * F * L * 16);
  ALLOC(c->stereo_sad, sizeof(int32_t) * ((F + 1) / 2) * g.kp_capacity);
  c->io_pitch = (g.W + 15) & ~15;
  {
    const int64_t Qm = std::max<int64_t>(max_queries, 1);
    ALLOC(c->io_frames, (size_t)F * g.H * c->io_pitch);
    ALLOC(c->io_frames_lin, (size_t)F * g.H * c->io_pitch);
    ALLOC(c->io_kps, sizeof(ss_keypoint) * F * g.kp_capacity);
    ALLOC(c->io_desc, (size_t)F * g.kp_capacity * SS_DESC_BYTES);
    ALLOC(c->io_counts, sizeof(int32_t) * F * (L + 1));
    ALLOC(c->io_cams, sizeof(ss_camera) * F);
    ALLOC(c->io_points, sizeof(ss_map_point) * Qm);
    ALLOC(c->io_pf, sizeof(int32_t) * Qm);
    ALLOC(c->io_pdesc, (size_t)Qm * SS_DESC_BYTES);
    ALLOC(c->io_taken, (size_t)F * g.kp_capacity);
    ALLOC(c->io_queries, sizeof(ss_mp_query) * Qm);
    ALLOC(c->io_matches, sizeof(ss_match) * std::max<int64_t>(Qm, F * g.kp_capacity));
    ALLOC(c->io_uright, sizeof(float) * ((F + 1) / 2) * g.kp_capacity);
    ALLOC(c->io_depth, sizeof(float) * ((F + 1) / 2) * g.kp_capacity);
    ALLOC(c->io_lf_off, sizeof(int32_t) * (F + 1));
    ALLOC(c->io_lf_pts, sizeof(ss_frame_point) * Qm);
    ALLOC(c->io_lf_desc, (size_t)Qm * SS_DESC_BYTES);
    ALLOC(c->io_last_cams, sizeof(ss_camera) * F);
    ALLOC(c->io_lf_matches, sizeof(ss_match) * Qm);
    ALLOC(c->io_lf_n, sizeof(int32_t) * F);
    ALLOC(c->io_packed, packed_capacity(g, F, Qm));
    {
      int64_t o[4];
      packed_in_layout(F, (int64_t)g.H * c->io_pitch, o);
      ALLOC(c->io_inpacked, o[3] + 256);
    }
    ALLOC(c->io_lf_mask, (size_t)F * g.kp_capacity);
  }
  if (max_map > 0) {
    ALLOC(c->partial, sizeof(unsigned long long) * F * g.kp_capacity * c->max_splits * 4);  // [slot][2 splits][2]
    ALLOC(c->brute_qexp, brute_tc_query_bytes(F * g.kp_capacity));
    ALLOC(c->brute_mexp, brute_tc_map_bytes(max_map));
  }
#undef ALLOC
  if (e == cudaSuccess) e = lastframe_init();
  if (e == cudaSuccess) e = fast_init();
  if (e == cudaSuccess) e = distribute_init();
  if (e == cudaSuccess) e = describe_init();
  if (e == cudaSuccess) e = pyramid_init();
  if (e == cudaSuccess) e = brute_tc_init();
  if (e == cudaSuccess) e = grid_init();
  if (e == cudaSuccess) e = cudaMemcpy(c->cells, c->cells_h.data(), sizeof(CellInfo) * c->cells_h.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c->bands, c->bands_h.data(), sizeof(BandInfo) * c->bands_h.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) {
    // the one-launch FAST order: larger work units (detect pixels of the segment) first, so
    // the CTAs that start last are the short ones (longest-processing-time first)
    // SS_FAST_FLAT (A/B): 1 = a flat band-major grid (the order holds across frames), 2 = that
    // with level 0's bands first (they need not wait for the pyramid)
    const char* ff = std::getenv("SS_FAST_FLAT");
    c->fast_flat = ff ? std::atoi(ff) : 0;
    const bool l0first = c->fast_flat == 2;
    std::vector<BandInfo> mo(c->bands_h.begin(), c->bands_h.end());
    std::stable_sort(mo.begin(), mo.end(), [l0first](const BandInfo& x, const BandInfo& y) {
      if (l0first && (x.level == 0) != (y.level == 0)) return x.level == 0;
      return (int64_t)(x.x1 - x.x0) * (x.y1 - x.y0) > (int64_t)(y.x1 - y.x0) * (y.y1 - y.y0);
    });
    e = cudaMemcpy(c->bands + c->bands_h.size(), mo.data(), sizeof(BandInfo) * mo.size(), cudaMemcpyHostToDevice);
  }
  c->fast_split = std::getenv("SS_FAST_SPLIT") && std::atoi(std::getenv("SS_FAST_SPLIT")) != 0;
  if (e == cudaSuccess && !tab.empty()) e = cudaMemcpy(c->xytab, tab.data(), sizeof(uint32_t) * tab.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess && !plan.empty())
    e = cudaMemcpy(c->pyr_plan, plan.data(), sizeof(PyrLvl) * plan.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess && !gtab.empty())
    e = cudaMemcpy(c->pyr_gtab, gtab.data(), sizeof(uint4) * gtab.size(), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c->ovf_level_off, ovf_off.data(), sizeof(int64_t) * L, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(c->pattern, pat.data(), 1024, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemset(c->ovf_counter, 0, sizeof(int32_t) * 4);
  if (e == cudaSuccess) e = launch_distribute_tables(g, c->qtab, 0);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  for (int i = 0; i < ss_ctx::kSide && e == cudaSuccess; i++) {
    e = cudaStreamCreateWithFlags(&c->side[i], cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_join[i], cudaEventDisableTiming);
  }
  for (int l = 0; l < kMaxLevels && e == cudaSuccess; l++)
    e = cudaEventCreateWithFlags(&c->ev_level[l], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&c->aux, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_aux0, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->ev_aux1, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaMemset(c->sel_counts, 0, sizeof(int32_t) * F * L);
  if (e == cudaSuccess) {
    c->maps.valid = 0;
    for (int l = 1; l < L; l++)
      if (encode_patch_map(&c->maps.level[l], c->pyr + g.lvl_off[l], g.w[l], g.h[l], max_frames, g.pitch[l],
                           g.pyr_frame_bytes))
        c->maps.valid |= 1u << l;
  }
  if (e != cudaSuccess) {
    std::string m = std::string("ss_create: ") + cudaGetErrorString(e);
    free_ctx(c);
    return fail(SS_ECUDA, m);
  }
  *out = c;
  return SS_OK;
}

ss_status ss_destroy(ss_ctx* ctx) {
  if (!ctx) return fail(SS_EINVAL, "NULL ctx");
  free_ctx(ctx);
  return SS_OK;
}

ss_status ss_orb_extract(ss_ctx* c, int32_t n_frames, const uint8_t* d_frames, int64_t frame_stride, int32_t pitch,
                         ss_keypoint* d_kps, uint8_t* d_desc, int32_t* d_counts, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_frames < 0) return fail(SS_EINVAL, "n_frames < 0");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (n_frames == 0) return SS_OK;
  if (!d_frames || !d_kps || !d_desc || !d_counts) return fail(SS_EINVAL, "NULL buffer");
  if (pitch < c->g.W) return fail(SS_EINVAL, "pitch < width");
  if (n_frames > 1 && frame_stride < (int64_t)pitch * c->g.H) return fail(SS_EINVAL, "frame_stride < height*pitch");
  c->win_ready = false;  // new keypoints: any prepared window index is stale
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  const Geom& g = c->g;
  FrameSrc src{d_frames, frame_stride, pitch, c->pyr};
  // The chain: pyramid (levels 1..L-1, one launch), FAST of all levels (one launch; its grid
  // fills the GPU better than two launches of which level 0's ran beside the pyramid), the
  // distribution of all levels (one launch, one (level, frame) CTA each), describe.  With
  // SS_FAST_SPLIT=1 level 0's FAST runs on side stream 0 beside the pyramid instead (A/B).
  // Profiling events: start, then a (before, after) pair around every launch in this order:
  // pyramid, fast (all levels), distribute, describe; with SS_FAST_SPLIT: fast l0, pyramid,
  // fast l>=1, distribute, describe.
  prof_mark(c, s);
  SS_CUDA_TRY(cudaMemsetAsync(c->ovf_counter, 0, sizeof(int32_t) * 4, s));
  if (c->fast_split) {
    SS_CUDA_TRY(cudaEventRecord(c->ev_fork, s));
    // with profiling events installed the level-0 branch runs in line on `stream`, so every
    // kernel is timed alone (the fork/join only changes overlap, not any kernel's work)
    cudaStream_t q = c->prof.empty() ? c->side[0] : s;
    if (q != s) SS_CUDA_TRY(cudaStreamWaitEvent(q, c->ev_fork, 0));
    prof_mark(c, q);
    SS_CUDA_TRY(launch_fast_bands(g, n_frames, src, c->bands, g.band_count[0], c->cells, c->slots, c->cell_counts, q));
    prof_mark(c, q);
    if (q != s) SS_CUDA_TRY(cudaEventRecord(c->ev_join[0], q));
    prof_mark(c, s);
    if (g.L > 1)
      SS_CUDA_TRY(launch_pyramid(g, n_frames, src, c->pyr_gtab, c->xytab, c->pyr_plan, c->pyr_blocks, c->pyr_buf0,
                                 c->pyr_buf1, c->pyr_smem, s));
    prof_mark(c, s);
    prof_mark(c, s);
    SS_CUDA_TRY(launch_fast_bands(g, n_frames, src, c->bands + g.band_count[0], g.total_bands - g.band_count[0],
                                  c->cells, c->slots, c->cell_counts, s));
    prof_mark(c, s);
    if (q != s) SS_CUDA_TRY(cudaStreamWaitEvent(s, c->ev_join[0], 0));
  } else {
    prof_mark(c, s);
    if (g.L > 1)
      SS_CUDA_TRY(launch_pyramid(g, n_frames, src, c->pyr_gtab, c->xytab, c->pyr_plan, c->pyr_blocks, c->pyr_buf0,
                                 c->pyr_buf1, c->pyr_smem, s));
    prof_mark(c, s);
    prof_mark(c, s);
    SS_CUDA_TRY(launch_fast_bands(g, n_frames, src, c->bands + g.total_bands, g.total_bands, c->cells, c->slots,
                                  c->cell_counts, s, c->fast_flat != 0));
    prof_mark(c, s);
  }
  prof_mark(c, s);
  if (c->dist_mode == SS_DIST_GRID_TOPN)
    SS_CUDA_TRY(launch_distribute_grid(g, n_frames, 0, g.L, c->cells, c->slots, c->cell_counts, c->selected,
                                       c->sel_counts, s));
  else
    SS_CUDA_TRY(launch_distribute(g, n_frames, 0, g.L, c->cells, c->qtab, c->slots, c->cell_counts, c->selected,
                                  c->sel_counts, c->ovf, c->ovf_frame_bytes, c->ovf_level_off, c->ovf_counter,
                                  c->phase_ts, s));
  prof_mark(c, s);
  prof_mark(c, s);
  // level 0: the caller's frames, encoded for this call (TMA when 16-B aligned, else LDG)
  c->maps.valid &= ~1u;
  if (encode_patch_map(&c->maps.level[0], d_frames, g.W, g.H, n_frames, pitch, frame_stride)) c->maps.valid |= 1u;
  SS_CUDA_TRY(launch_describe(g, n_frames, src, c->selected, c->sel_counts, c->pattern, d_kps, d_desc, d_counts,
                              c->dbg_samples, c->maps, s));
  prof_mark(c, s);
  c->last_frames = d_frames;
  c->last_stride = frame_stride;
  c->last_pitch = pitch;
  c->last_n = n_frames;
  return SS_OK;
}

ss_status ss_orb_extract_frames(ss_ctx* c, int32_t n_frames, const uint8_t* const* d_frames, const int32_t* pitches,
                                ss_keypoint* d_kps, uint8_t* d_desc, int32_t* d_counts, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_frames < 0) return fail(SS_EINVAL, "n_frames < 0");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (n_frames == 0) return SS_OK;
  if (!d_frames || !pitches) return fail(SS_EINVAL, "NULL frame / pitch array");
  for (int f = 0; f < n_frames; f++) {
    if (!d_frames[f]) return fail(SS_EINVAL, "NULL frame pointer");
    if (pitches[f] < c->g.W) return fail(SS_EINVAL, "pitch < width");
  }
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  // independently allocated client frames are packed into the ctx's frame staging buffer (one
  // device-side 2-D copy per frame, 16-B aligned pitch), then extracted as one batch
  const int P = c->io_pitch;
  const int64_t fstride = (int64_t)c->g.H * P;
  for (int f = 0; f < n_frames; f++)
    SS_CUDA_TRY(cudaMemcpy2DAsync(c->io_frames + f * fstride, P, d_frames[f], pitches[f], c->g.W, c->g.H,
                                  cudaMemcpyDeviceToDevice, s));
  return ss_orb_extract(c, n_frames, c->io_frames, fstride, P, d_kps, d_desc, d_counts, stream);
}

ss_status ss_match_projection(ss_ctx* c, int32_t n_frames, const ss_keypoint* d_kps, const uint8_t* d_desc,
                              const int32_t* d_counts, const uint8_t* d_kp_taken, int32_t n_queries,
                              const ss_mp_query* d_queries, const uint8_t* d_map_desc, int32_t n_map,
                              const ss_match_cfg* cfg, ss_match* d_out, ss_stream_t stream) {
  if (!c || !cfg) return fail(SS_EINVAL, "NULL ctx/cfg");
  if (n_frames < 0 || n_queries < 0 || n_map < 0) return fail(SS_EINVAL, "negative size");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (cfg->ratio_den <= 0 || cfg->ratio_num < 0) return fail(SS_EINVAL, "bad ratio");
  if (!d_kps || !d_desc || !d_counts || !d_out) return fail(SS_EINVAL, "NULL buffer");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  if (cfg->mode == SS_MATCH_WINDOW) {
    if (n_queries > c->max_queries) return fail(SS_ECAPACITY, "n_queries exceeds the ctx's max_queries");
    if (n_queries > 0 && (!d_queries || !d_map_desc)) return fail(SS_EINVAL, "NULL queries");
    if (n_queries == 0) return SS_OK;
    prof_mark(c, s);
    if (!(c->win_ready && d_kps == c->win_kps && d_counts == c->win_counts && n_frames <= c->win_nf))
      SS_CUDA_TRY(launch_match_prepare(c->g, n_frames, d_kps, d_counts, c->rowidx, c->claim, cfg->dedup, s));
    c->win_ready = false;  // the claims are consumed by this match
    prof_mark(c, s);
    prof_mark(c, s);
    SS_CUDA_TRY(launch_match_window(c->g, n_frames, d_kps, d_desc, d_counts, d_kp_taken, n_queries, d_queries,
                                    d_map_desc, *cfg, c->claim, d_out, c->rowidx, c->win_lanes, s));
    prof_mark(c, s);
    if (cfg->dedup) {
      prof_mark(c, s);
      SS_CUDA_TRY(launch_match_resolve(c->g, n_queries, d_queries, c->claim, d_out, s));
      prof_mark(c, s);
    }
    return SS_OK;
  }
  if (cfg->mode == SS_MATCH_BRUTE) {
    if (n_queries != 0) return fail(SS_EINVAL, "BRUTE mode takes no queries");
    if (n_map > c->max_map) return fail(SS_ECAPACITY, "n_map exceeds the ctx's max_map");
    const bool prepared = n_map > 0 && !d_map_desc;
    if (prepared && c->prepared_map != n_map)
      return fail(SS_EINVAL, "NULL map and no map of n_map rows prepared by ss_brute_map_prepare");
    if (n_frames == 0) return SS_OK;
    const int n_slots = n_frames * c->g.kp_capacity;
    if (n_map == 0) {
      // an empty map (e.g. at session start): no candidates, every slot gets {-1, 256, 256}
      // (the merge with zero partials; c->partial may not even exist when max_map == 0)
      for (int i = 0; i < 4; i++) prof_mark(c, s);
      prof_mark(c, s);
      SS_CUDA_TRY(launch_brute_merge(c->g, n_frames, d_counts, 0, nullptr, *cfg, d_out, s));
      prof_mark(c, s);
      return SS_OK;
    }
    const int splits = brute_tc_splits(n_slots, n_map, c->max_splits, c->n_sm);
    if (!prepared) c->prepared_map = -1;  // the expansion below overwrites the prepared map
    prof_mark(c, s);
    SS_CUDA_TRY(launch_brute_expand(n_slots, d_desc, n_map, prepared ? nullptr : d_map_desc, c->brute_qexp,
                                    c->brute_mexp, s));
    prof_mark(c, s);
    prof_mark(c, s);
    SS_CUDA_TRY(launch_brute_tc(n_slots, n_map, c->brute_qexp, c->brute_mexp, splits, c->partial, s));
    prof_mark(c, s);
    prof_mark(c, s);
    // brute_tc writes one partial top-2 per (split, column half of the pair's 256-row tiles)
    SS_CUDA_TRY(launch_brute_merge(c->g, n_frames, d_counts, 2 * splits, c->partial, *cfg, d_out, s));
    prof_mark(c, s);
    return SS_OK;
  }
  return fail(SS_EINVAL, "unknown match mode");
}

ss_status ss_match_brute_partial(ss_ctx* c, int32_t n_frames, const uint8_t* d_desc, const int32_t* d_counts,
                                 const uint8_t* d_map_desc, int32_t n_map, int32_t map_offset, uint64_t* d_top2,
                                 ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_frames < 0 || n_map < 0 || map_offset < 0) return fail(SS_EINVAL, "negative size / offset");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (n_map > c->max_map) return fail(SS_ECAPACITY, "n_map exceeds the ctx's max_map");
  if ((int64_t)map_offset + n_map > INT32_MAX) return fail(SS_EINVAL, "map_offset + n_map exceeds 2^31 - 1");
  if (n_frames == 0) return SS_OK;
  if (!d_desc || !d_counts || !d_top2) return fail(SS_EINVAL, "NULL buffer");
  const bool prepared = n_map > 0 && !d_map_desc;
  if (prepared && c->prepared_map != n_map)
    return fail(SS_EINVAL, "NULL map and no map of n_map rows prepared by ss_brute_map_prepare");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  const int n_slots = n_frames * c->g.kp_capacity;
  unsigned long long* top2 = reinterpret_cast<unsigned long long*>(d_top2);
  if (n_map == 0) {  // an empty shard contributes nothing
    SS_CUDA_TRY(cudaMemsetAsync(top2, 0xFF, sizeof(unsigned long long) * 2 * n_slots, s));
    return SS_OK;
  }
  const int splits = brute_tc_splits(n_slots, n_map, c->max_splits, c->n_sm);
  if (!prepared) c->prepared_map = -1;
  prof_mark(c, s);
  SS_CUDA_TRY(launch_brute_expand(n_slots, d_desc, n_map, prepared ? nullptr : d_map_desc, c->brute_qexp,
                                  c->brute_mexp, s));
  prof_mark(c, s);
  prof_mark(c, s);
  SS_CUDA_TRY(launch_brute_tc(n_slots, n_map, c->brute_qexp, c->brute_mexp, splits, c->partial, s));
  prof_mark(c, s);
  prof_mark(c, s);
  SS_CUDA_TRY(launch_brute_shard_top2(c->g, n_frames, d_counts, 2 * splits, c->partial, map_offset, top2, s));
  prof_mark(c, s);
  return SS_OK;
}

ss_status ss_brute_map_prepare(ss_ctx* c, const uint8_t* d_map_desc, int32_t n_map, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_map < 1 || !d_map_desc) return fail(SS_EINVAL, "n_map < 1 or NULL map");
  if (n_map > c->max_map) return fail(SS_ECAPACITY, "n_map exceeds the ctx's max_map");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  SS_CUDA_TRY(launch_brute_expand(0, nullptr, n_map, d_map_desc, c->brute_qexp, c->brute_mexp, s));
  c->prepared_map = n_map;
  return SS_OK;
}

ss_status ss_match_brute_merge(ss_ctx* c, int32_t n_frames, const int32_t* d_counts, int32_t n_parts,
                               const uint64_t* d_parts, const ss_match_cfg* cfg, ss_match* d_out, ss_stream_t stream) {
  if (!c || !cfg) return fail(SS_EINVAL, "NULL ctx/cfg");
  if (n_frames < 0 || n_parts < 1) return fail(SS_EINVAL, "n_frames < 0 or n_parts < 1");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (cfg->ratio_den <= 0 || cfg->ratio_num < 0) return fail(SS_EINVAL, "bad ratio");
  if (n_frames == 0) return SS_OK;
  if (!d_counts || !d_parts || !d_out) return fail(SS_EINVAL, "NULL buffer");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  prof_mark(c, s);
  SS_CUDA_TRY(launch_brute_parts_merge(c->g, n_frames, d_counts, n_parts,
                                       reinterpret_cast<const unsigned long long*>(d_parts), *cfg, d_out, s));
  prof_mark(c, s);
  return SS_OK;
}

ss_status ss_stereo_match(ss_ctx* c, int32_t n_pairs, const uint8_t* d_frames, int64_t frame_stride, int32_t pitch,
                          const ss_keypoint* d_kps, const uint8_t* d_desc, const int32_t* d_counts, float bf,
                          float baseline, float* d_uright, float* d_depth, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_pairs < 0) return fail(SS_EINVAL, "negative size");
  if (2 * (int64_t)n_pairs > c->max_frames) return fail(SS_ECAPACITY, "2 * n_pairs exceeds the ctx's max_frames");
  if (n_pairs == 0) return SS_OK;
  if (!d_frames || !d_kps || !d_desc || !d_counts || !d_uright || !d_depth) return fail(SS_EINVAL, "NULL buffer");
  if (pitch < c->g.W || frame_stride < (int64_t)c->g.H * pitch) return fail(SS_EINVAL, "bad pitch / frame stride");
  if (!(bf > 0.0f) || !(baseline > 0.0f)) return fail(SS_EINVAL, "bf and baseline must be > 0");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  const float maxD = bf / baseline;  // ORB-SLAM: maxD = mbf / minZ, minZ = mb
  c->win_ready = false;               // its prepare rewrites the shared row index
  FrameSrc src{d_frames, frame_stride, pitch, c->pyr};
  prof_mark(c, s);
  SS_CUDA_TRY(launch_match_prepare(c->g, 2 * n_pairs, d_kps, d_counts, c->rowidx, c->claim, 0, s));
  prof_mark(c, s);
  prof_mark(c, s);
  SS_CUDA_TRY(launch_stereo(c->g, n_pairs, src, d_kps, d_desc, d_counts, c->rowidx, match_index_stride(c->g), bf,
                            maxD, d_uright, d_depth, c->stereo_sad, s));
  prof_mark(c, s);
  prof_mark(c, s);
  SS_CUDA_TRY(launch_stereo_outliers(c->g, n_pairs, d_counts, c->stereo_sad, d_uright, d_depth, s));
  prof_mark(c, s);
  return SS_OK;
}

ss_status ss_project_points(ss_ctx* c, int32_t n_frames, const ss_camera* d_cams, int32_t n_points,
                            const ss_map_point* d_points, const int32_t* d_point_frame, float th,
                            ss_mp_query* d_queries, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_frames < 0 || n_points < 0) return fail(SS_EINVAL, "negative size");
  if (n_points == 0) return SS_OK;
  if (!d_points || !d_point_frame || !d_queries || (n_frames > 0 && !d_cams)) return fail(SS_EINVAL, "NULL buffer");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  prof_mark(c, s);
  SS_CUDA_TRY(launch_project(c->g, n_frames, d_cams, n_points, d_points, d_point_frame, th, d_queries, s));
  prof_mark(c, s);
  return SS_OK;
}

ss_status ss_match_last_frame(ss_ctx* c, int32_t n_frames, const ss_camera* d_cams, const ss_camera* d_last_cams,
                              float mb, const ss_keypoint* d_kps, const uint8_t* d_desc, const int32_t* d_counts,
                              const uint8_t* d_kp_taken, const int32_t* d_point_offsets,
                              const ss_frame_point* d_points, const uint8_t* d_point_desc, float th,
                              int32_t th_high, int32_t check_orientation, int32_t min_matches, ss_match* d_out,
                              int32_t* d_n_matches, uint8_t* d_kp_matched, ss_stream_t stream) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (n_frames < 0) return fail(SS_EINVAL, "negative size");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (!(th > 0.0f)) return fail(SS_EINVAL, "th must be > 0");
  if (lastframe_smem_bytes(c->g) > 200 * 1024)
    return fail(SS_EUNSUPPORTED, "kp_capacity too large for the frame-to-frame matcher's shared memory");
  if (n_frames == 0) return SS_OK;
  if (!d_cams || !d_kps || !d_desc || !d_counts || !d_point_offsets || !d_points || !d_point_desc || !d_out)
    return fail(SS_EINVAL, "NULL buffer");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  SS_CUDA_TRY(check_stream(s));
  std::pair<ss_ctx*, cudaStream_t> pm{c, s};
  SS_CUDA_TRY(launch_lastframe(c->g, n_frames, d_cams, mb > 0.0f ? d_last_cams : nullptr, mb, d_kps, d_desc, d_counts,
                               d_kp_taken, d_point_offsets, d_points, d_point_desc, th, th_high, check_orientation,
                               min_matches, d_out, d_n_matches, d_kp_matched, c->claim_lf, c->rowidx, c->claim, c->n_sm, s,
                               [](void* p) {
                                 auto* q = static_cast<std::pair<ss_ctx*, cudaStream_t>*>(p);
                                 prof_mark(q->first, q->second);
                               },
                               &pm));
  c->win_ready = true;
  c->win_kps = d_kps;
  c->win_counts = d_counts;
  c->win_nf = n_frames;
  return SS_OK;
}

ss_status ss_set_distribution(ss_ctx* c, int32_t mode) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (mode != SS_DIST_QUADTREE && mode != SS_DIST_GRID_TOPN) return fail(SS_EINVAL, "unknown distribution mode");
  if (mode == SS_DIST_GRID_TOPN && grid_smem_bytes(c->g) > 200 * 1024)
    return fail(SS_EUNSUPPORTED, "n_per_level too large for the grid top-N kernel's shared memory");
  if (mode != c->dist_mode) {
    // cached tick graphs were captured with the other distribution's kernels
    cudaSetDevice(c->device);
    for (ss_ctx::TickGraph& tg : c->tick_graphs)
      if (tg.exec) cudaGraphExecDestroy(tg.exec);
    c->tick_graphs.clear();
  }
  c->dist_mode = mode;
  return SS_OK;
}

namespace {

// Everything one tick enqueues on s (ss_track_tick after validation): copies in, the hot path,
// copies out.  Captured into a CUDA graph when io->reuse_graph is set (see ss_track_tick).
ss_status tick_enqueue(ss_ctx* c, int32_t n_frames, const ss_match_cfg* cfg, const ss_tick_io* io, cudaStream_t s,
                       bool stereo, bool window, bool lastf, int64_t n_lf) {
  const Geom& g = c->g;
  ss_stream_t stream = reinterpret_cast<ss_stream_t>(s);
  const int cap = g.kp_capacity, L = g.L;
  // outputs: the ctx's buffers, or sections of the packed block (ss_tick_io.out_packed: one D2H)
  const bool packed = io->out_packed != nullptr;
  int64_t po[9];
  packed_layout(g, n_frames, window ? io->n_points : (int64_t)n_frames * cap, lastf ? n_lf : 0, stereo, po);
  ss_keypoint* o_kps = packed ? reinterpret_cast<ss_keypoint*>(c->io_packed + po[0]) : c->io_kps;
  uint8_t* o_desc = packed ? c->io_packed + po[1] : c->io_desc;
  int32_t* o_counts = packed ? reinterpret_cast<int32_t*>(c->io_packed + po[2]) : c->io_counts;
  int32_t* o_lf_n = packed ? reinterpret_cast<int32_t*>(c->io_packed + po[3]) : c->io_lf_n;
  ss_match* o_lf_matches = packed ? reinterpret_cast<ss_match*>(c->io_packed + po[4]) : c->io_lf_matches;
  ss_match* o_matches = packed ? reinterpret_cast<ss_match*>(c->io_packed + po[5]) : c->io_matches;
  float* o_uright = packed ? reinterpret_cast<float*>(c->io_packed + po[6]) : c->io_uright;
  float* o_depth = packed ? reinterpret_cast<float*>(c->io_packed + po[7]) : c->io_depth;
  // host -> device.  Frames stored densely (pitch <= the staging pitch, frame_stride = H *
  // pitch) go in ONE linear copy and keep their pitch; anything else is repacked by 2-D
  // copies (a 2-D copy moves row by row, several times slower for 0.3-0.5 MB frames).
  int P = c->io_pitch;
  int64_t fstride = (int64_t)g.H * P;
  const bool dense = io->pitch <= c->io_pitch && (n_frames == 1 || io->frame_stride == (int64_t)io->pitch * g.H);
  // device copies of the per-tick host inputs: the ctx's buffers, or sections of the packed
  // input block (ss_tick_io.in_packed: frames + cams + lf_offsets in ONE copy)
  uint8_t* d_frames_in = c->io_frames;
  ss_camera* d_cams_in = c->io_cams;
  int32_t* d_lfoff_in = c->io_lf_off;
  if (io->in_packed) {
    int64_t o[4];
    packed_in_layout(n_frames, io->frame_stride, o);
    P = io->pitch;
    fstride = io->frame_stride;
    SS_CUDA_TRY(cudaMemcpyAsync(c->io_inpacked, io->in_packed, (size_t)o[3], cudaMemcpyHostToDevice, s));
    d_frames_in = c->io_inpacked + o[0];
    d_cams_in = reinterpret_cast<ss_camera*>(c->io_inpacked + o[1]);
    d_lfoff_in = reinterpret_cast<int32_t*>(c->io_inpacked + o[2]);
  } else if (dense && io->pitch % 16 == 0) {
    P = io->pitch;
    fstride = (int64_t)g.H * P;
    SS_CUDA_TRY(cudaMemcpyAsync(c->io_frames, io->frames, (size_t)fstride * n_frames, cudaMemcpyHostToDevice, s));
  } else if (dense) {
    // a pitch that is not a multiple of 16 B (e.g. KITTI's 1241) would send FAST's band staging
    // and describe's patch loads down their per-byte paths: one linear H2D into the lead-in
    // staging buffer, then one device-side 2-D copy to the 16-B aligned staging pitch
    const int64_t lin = (int64_t)g.H * io->pitch * n_frames;
    SS_CUDA_TRY(cudaMemcpyAsync(c->io_frames_lin, io->frames, (size_t)lin, cudaMemcpyHostToDevice, s));
    SS_CUDA_TRY(cudaMemcpy2DAsync(c->io_frames, P, c->io_frames_lin, io->pitch, g.W, (size_t)g.H * n_frames,
                                  cudaMemcpyDeviceToDevice, s));
  } else {
    for (int f = 0; f < n_frames; f++)
      SS_CUDA_TRY(cudaMemcpy2DAsync(c->io_frames + f * fstride, P, io->frames + f * io->frame_stride, io->pitch, g.W,
                                    g.H, cudaMemcpyHostToDevice, s));
  }
  // map state: host copies staged into the ctx, or (map_resident) the caller's device buffers
  const bool res = io->map_resident != 0;
  const ss_map_point* d_points = res ? io->points : c->io_points;
  const int32_t* d_pf = res ? io->point_frame : c->io_pf;
  const uint8_t* d_pdesc = res ? io->point_desc : c->io_pdesc;
  const uint8_t* d_taken = io->taken ? (res ? io->taken : c->io_taken) : nullptr;
  const ss_frame_point* d_lf_pts = res ? io->lf_points : c->io_lf_pts;
  const uint8_t* d_lf_desc = res ? io->lf_desc : c->io_lf_desc;
  const ss_camera* d_last = res ? io->last_cams : c->io_last_cams;
  if (window) {
    const int64_t n = io->n_points;
    if (!io->in_packed)
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_cams, io->cams, sizeof(ss_camera) * n_frames, cudaMemcpyHostToDevice, s));
    if (!res) {
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_points, io->points, sizeof(ss_map_point) * n, cudaMemcpyHostToDevice, s));
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_pf, io->point_frame, sizeof(int32_t) * n, cudaMemcpyHostToDevice, s));
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_pdesc, io->point_desc, (size_t)n * SS_DESC_BYTES, cudaMemcpyHostToDevice, s));
      if (io->taken)
        SS_CUDA_TRY(cudaMemcpyAsync(c->io_taken, io->taken, (size_t)n_frames * cap, cudaMemcpyHostToDevice, s));
    }
  }
  if (lastf) {
    if (!io->in_packed)
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_lf_off, io->lf_offsets, sizeof(int32_t) * (n_frames + 1), cudaMemcpyHostToDevice, s));
    if (n_lf > 0 && !res) {
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_lf_pts, io->lf_points, sizeof(ss_frame_point) * n_lf, cudaMemcpyHostToDevice, s));
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_lf_desc, io->lf_desc, (size_t)n_lf * SS_DESC_BYTES, cudaMemcpyHostToDevice, s));
    }
    if (io->mb > 0.0f && !res)
      SS_CUDA_TRY(cudaMemcpyAsync(c->io_last_cams, io->last_cams, sizeof(ss_camera) * n_frames, cudaMemcpyHostToDevice, s));
  }
  // the hot path.  The local-map projection needs only the cameras and map points, so (unless
  // profiling events are installed, which time every kernel alone on `stream`) it forks onto
  // the ctx's aux stream after the extraction and overlaps the frame-to-frame matcher (one CTA
  // per frame: most SMs are free); the WINDOW match joins it.
  ss_status st;
  const bool fork_project = window && c->prof.empty() && c->tick_fork;
  st = ss_orb_extract(c, n_frames, d_frames_in, fstride, P, o_kps, o_desc, o_counts, stream);
  if (st != SS_OK) return st;
  if (stereo) {
    st = ss_stereo_match(c, n_frames / 2, d_frames_in, fstride, P, o_kps, o_desc, o_counts, io->bf,
                         io->baseline, o_uright, o_depth, stream);
    if (st != SS_OK) return st;
  }
  if (fork_project) {
    SS_CUDA_TRY(cudaEventRecord(c->ev_aux0, s));
    SS_CUDA_TRY(cudaStreamWaitEvent(c->aux, c->ev_aux0, 0));
    st = ss_project_points(c, n_frames, d_cams_in, io->n_points, d_points, d_pf, io->th, c->io_queries,
                           reinterpret_cast<ss_stream_t>(c->aux));
    if (st != SS_OK) return st;
    SS_CUDA_TRY(cudaEventRecord(c->ev_aux1, c->aux));
  }
  int64_t n_matches = 0;
  const uint8_t* win_taken = d_taken;
  if (lastf) {
    st = ss_match_last_frame(c, n_frames, d_cams_in, io->mb > 0.0f ? d_last : nullptr, io->mb, o_kps,
                             o_desc, o_counts, win_taken, d_lfoff_in, d_lf_pts, d_lf_desc,
                             io->lf_th, 100, 1, io->lf_min_matches, o_lf_matches, o_lf_n, c->io_lf_mask,
                             stream);
    if (st != SS_OK) return st;
    win_taken = c->io_lf_mask;
  }
  if (window) {
    if (fork_project) {
      SS_CUDA_TRY(cudaStreamWaitEvent(s, c->ev_aux1, 0));
    } else {
      st = ss_project_points(c, n_frames, d_cams_in, io->n_points, d_points, d_pf, io->th, c->io_queries, stream);
      if (st != SS_OK) return st;
    }
    st = ss_match_projection(c, n_frames, o_kps, o_desc, o_counts, win_taken, io->n_points, c->io_queries,
                             d_pdesc, 0, cfg, o_matches, stream);
    if (st != SS_OK) return st;
    n_matches = io->n_points;
  } else if (cfg->mode == SS_MATCH_BRUTE) {
    st = ss_match_projection(c, n_frames, o_kps, o_desc, o_counts, nullptr, 0, nullptr, io->d_map_desc,
                             io->n_map, cfg, o_matches, stream);
    if (st != SS_OK) return st;
    n_matches = (int64_t)n_frames * cap;
  }
  // device -> host
  if (packed) {  // every output in ONE copy
    SS_CUDA_TRY(cudaMemcpyAsync(io->out_packed, c->io_packed, (size_t)po[8], cudaMemcpyDeviceToHost, s));
    return SS_OK;
  }
  if (io->kps)
    SS_CUDA_TRY(cudaMemcpyAsync(io->kps, c->io_kps, sizeof(ss_keypoint) * n_frames * cap, cudaMemcpyDeviceToHost, s));
  if (io->desc)
    SS_CUDA_TRY(cudaMemcpyAsync(io->desc, c->io_desc, (size_t)n_frames * cap * SS_DESC_BYTES, cudaMemcpyDeviceToHost, s));
  if (io->counts)
    SS_CUDA_TRY(cudaMemcpyAsync(io->counts, c->io_counts, sizeof(int32_t) * n_frames * (L + 1), cudaMemcpyDeviceToHost, s));
  if (io->matches && n_matches > 0)
    SS_CUDA_TRY(cudaMemcpyAsync(io->matches, c->io_matches, sizeof(ss_match) * n_matches, cudaMemcpyDeviceToHost, s));
  if (lastf && io->lf_matches && n_lf > 0)
    SS_CUDA_TRY(cudaMemcpyAsync(io->lf_matches, c->io_lf_matches, sizeof(ss_match) * n_lf, cudaMemcpyDeviceToHost, s));
  if (lastf && io->lf_n_matches)
    SS_CUDA_TRY(cudaMemcpyAsync(io->lf_n_matches, c->io_lf_n, sizeof(int32_t) * n_frames, cudaMemcpyDeviceToHost, s));
  if (stereo && io->uright)
    SS_CUDA_TRY(cudaMemcpyAsync(io->uright, c->io_uright, sizeof(float) * (n_frames / 2) * cap, cudaMemcpyDeviceToHost, s));
  if (stereo && io->depth)
    SS_CUDA_TRY(cudaMemcpyAsync(io->depth, c->io_depth, sizeof(float) * (n_frames / 2) * cap, cudaMemcpyDeviceToHost, s));
  return SS_OK;
}


// Graph-cache key of a tick: every argument the enqueued work depends on (host pointers and
// sizes of io, the match cfg, the last-frame point count read from the host offsets).
std::vector<unsigned char> tick_key(int32_t n_frames, const ss_match_cfg* cfg, const ss_tick_io* io, int64_t n_lf) {
  std::vector<unsigned char> k;
  auto put = [&k](const void* p, size_t n) {
    const unsigned char* b = static_cast<const unsigned char*>(p);
    k.insert(k.end(), b, b + n);
  };
  auto ptr = [&put](const void* p) { put(&p, sizeof(p)); };
  put(&n_frames, 4);
  put(&cfg->mode, 4); put(&cfg->th, 4); put(&cfg->ratio_num, 4); put(&cfg->ratio_den, 4); put(&cfg->dedup, 4);
  ptr(io->frames); put(&io->frame_stride, 8); put(&io->pitch, 4); put(&io->bf, 4); put(&io->baseline, 4);
  ptr(io->cams); put(&io->n_points, 4); ptr(io->points); ptr(io->point_frame); ptr(io->point_desc); ptr(io->taken);
  put(&io->th, 4); ptr(io->d_map_desc); put(&io->n_map, 4);
  ptr(io->kps); ptr(io->desc); ptr(io->counts); ptr(io->matches); ptr(io->uright); ptr(io->depth);
  ptr(io->lf_offsets); ptr(io->lf_points); ptr(io->lf_desc); ptr(io->last_cams); put(&io->mb, 4); put(&io->lf_th, 4);
  put(&io->lf_min_matches, 4); ptr(io->lf_matches); ptr(io->lf_n_matches); put(&io->map_resident, 4);
  ptr(io->out_packed); ptr(io->in_packed);
  put(&n_lf, 8);
  return k;
}

}  // namespace

ss_status ss_tick_packed_layout(const ss_ctx* c, int32_t n_frames, int32_t n_points, int64_t n_lf, int32_t brute,
                                int32_t stereo, int64_t* offsets) {
  if (!c || !offsets) return fail(SS_EINVAL, "NULL ctx/offsets");
  if (n_frames < 0 || n_points < 0 || n_lf < 0) return fail(SS_EINVAL, "negative size");
  packed_layout(c->g, n_frames, brute ? (int64_t)n_frames * c->g.kp_capacity : n_points, n_lf, stereo != 0, offsets);
  return SS_OK;
}

ss_status ss_tick_packed_in_layout(const ss_ctx* c, int32_t n_frames, int64_t frame_stride, int64_t* offsets) {
  if (!c || !offsets) return fail(SS_EINVAL, "NULL ctx/offsets");
  if (n_frames < 0 || frame_stride < 0) return fail(SS_EINVAL, "negative size");
  packed_in_layout(n_frames, frame_stride, offsets);
  return SS_OK;
}

ss_status ss_track_tick(ss_ctx* c, int32_t n_frames, const ss_match_cfg* cfg, const ss_tick_io* io,
                        ss_stream_t stream) {
  if (!c || !cfg || !io) return fail(SS_EINVAL, "NULL ctx/cfg/io");
  if (n_frames < 0 || io->n_points < 0 || io->n_map < 0) return fail(SS_EINVAL, "negative size");
  if (n_frames > c->max_frames) return fail(SS_ECAPACITY, "n_frames exceeds the ctx's max_frames");
  if (n_frames == 0) return SS_OK;
  const Geom& g = c->g;
  // packed host inputs: frames, cams and lf_offsets are sections of io->in_packed (one H2D
  // copy, tick_enqueue); O13 then runs when lf_points is set
  ss_tick_io eff = *io;
  if (io->in_packed) {
    if (io->pitch % 16 != 0 || io->pitch > c->io_pitch || io->pitch < g.W || io->frame_stride != (int64_t)io->pitch * g.H)
      return fail(SS_EINVAL, "in_packed needs dense frames (frame_stride = height * pitch, pitch a multiple of 16, "
                             "<= width rounded up to 16)");
    int64_t o[4];
    packed_in_layout(n_frames, io->frame_stride, o);
    const uint8_t* b = static_cast<const uint8_t*>(io->in_packed);
    eff.frames = b + o[0];
    eff.cams = reinterpret_cast<const ss_camera*>(b + o[1]);
    eff.lf_offsets = io->lf_points ? reinterpret_cast<const int32_t*>(b + o[2]) : nullptr;
  }
  io = &eff;
  if (!io->frames) return fail(SS_EINVAL, "NULL frames");
  if (io->pitch < g.W || (n_frames > 1 && io->frame_stride < (int64_t)io->pitch * g.H))
    return fail(SS_EINVAL, "bad pitch / frame stride");
  const bool stereo = io->bf > 0.0f;
  if (stereo && (n_frames & 1)) return fail(SS_EINVAL, "stereo needs an even frame count");
  const bool window = cfg->mode == SS_MATCH_WINDOW && io->n_points > 0;
  if (window) {
    if (io->n_points > c->max_queries) return fail(SS_ECAPACITY, "n_points exceeds the ctx's max_queries");
    if (!io->cams || !io->points || !io->point_frame || !io->point_desc) return fail(SS_EINVAL, "NULL window input");
  }
  const bool lastf = window && io->lf_offsets;
  int64_t n_lf = 0;
  if (lastf) {
    for (int f = 0; f < n_frames; f++)
      if (io->lf_offsets[f + 1] < io->lf_offsets[f]) return fail(SS_EINVAL, "lf_offsets must be non-decreasing");
    if (io->lf_offsets[0] != 0) return fail(SS_EINVAL, "lf_offsets[0] must be 0");
    n_lf = io->lf_offsets[n_frames];
    if (n_lf > c->max_queries) return fail(SS_ECAPACITY, "last-frame points exceed the ctx's max_queries");
    if (n_lf > 0 && (!io->lf_points || !io->lf_desc)) return fail(SS_EINVAL, "NULL last-frame input");
    if (io->mb > 0.0f && !io->last_cams) return fail(SS_EINVAL, "mb > 0 needs last_cams");
    if (!(io->lf_th > 0.0f)) return fail(SS_EINVAL, "lf_th must be > 0");
  }
  SS_CUDA_TRY(cudaSetDevice(c->device));
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  SS_CUDA_TRY(cudaStreamIsCapturing(s, &cs));
  // (the legacy default stream cannot be captured: such ticks always run directly)
  if (!io->reuse_graph || !c->prof.empty() || cs != cudaStreamCaptureStatusNone || s == nullptr ||
      s == cudaStreamLegacy)
    return tick_enqueue(c, n_frames, cfg, io, s, stereo, window, lastf, n_lf);
  // graph reuse: a tick seen before with identical arguments is replayed from a CUDA graph
  // (one launch instead of ~30 API calls); the second occurrence of a key is captured (the
  // first runs directly, so lazily-set kernel attributes are never set under capture)
  std::vector<unsigned char> key = tick_key(n_frames, cfg, io, n_lf);
  c->tick_clock++;
  for (ss_ctx::TickGraph& tg : c->tick_graphs) {
    if (tg.key != key) continue;
    tg.last_use = c->tick_clock;
    if (tg.exec) {
      SS_CUDA_TRY(cudaGraphLaunch(tg.exec, s));
      return SS_OK;
    }
    cudaGraph_t graph = nullptr;
    SS_CUDA_TRY(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    ss_status st = tick_enqueue(c, n_frames, cfg, io, s, stereo, window, lastf, n_lf);
    cudaError_t e = cudaStreamEndCapture(s, &graph);
    if (st != SS_OK) {
      if (graph) cudaGraphDestroy(graph);
      return st;
    }
    SS_CUDA_TRY(e);
    e = cudaGraphInstantiate(&tg.exec, graph, 0);
    cudaGraphDestroy(graph);
    SS_CUDA_TRY(e);
    SS_CUDA_TRY(cudaGraphLaunch(tg.exec, s));
    return SS_OK;
  }
  if (c->tick_graphs.size() >= ss_ctx::kTickGraphs) {  // evict the least recently used
    size_t lru = 0;
    for (size_t i = 1; i < c->tick_graphs.size(); i++)
      if (c->tick_graphs[i].last_use < c->tick_graphs[lru].last_use) lru = i;
    if (c->tick_graphs[lru].exec) cudaGraphExecDestroy(c->tick_graphs[lru].exec);
    c->tick_graphs.erase(c->tick_graphs.begin() + lru);
  }
  c->tick_graphs.push_back({key, nullptr, c->tick_clock});
  return tick_enqueue(c, n_frames, cfg, io, s, stereo, window, lastf, n_lf);
}

ss_status ss_track_run(ss_ctx* const* ctxs, int32_t n_ctx, const ss_stream_t* streams, int32_t n_frames,
                       const ss_match_cfg* cfg, const ss_tick_io* ios, int32_t n_io, int32_t n_ticks) {
  if (!ctxs || !streams || !cfg || !ios || n_ctx < 1 || n_io < 1 || n_ticks < 0)
    return fail(SS_EINVAL, "bad ss_track_run arguments");
  for (int32_t t = 0; t < n_ticks; t++) {
    const int q = t % n_ctx, i = t % n_io;
    const ss_status st = ss_track_tick(ctxs[q], n_frames, cfg, &ios[(int64_t)q * n_io + i], streams[q]);
    if (st != SS_OK) return st;
  }
  return SS_OK;
}

ss_status ss_profile_events(ss_ctx* c, void* const* events, int32_t n_events) {
  if (!c || n_events < 0 || (n_events > 0 && !events)) return fail(SS_EINVAL, "bad profiling events");
  for (int i = 0; i < n_events; i++)
    if (!events[i]) return fail(SS_EINVAL, "NULL event handle (torch creates events lazily: record once first)");
  c->prof.assign(n_events, nullptr);
  for (int i = 0; i < n_events; i++) c->prof[i] = reinterpret_cast<cudaEvent_t>(events[i]);
  c->prof_next = 0;
  return SS_OK;
}

ss_status ss_profile_next(ss_ctx* c, int32_t* next_index) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (next_index) *next_index = (int32_t)c->prof_next;
  return SS_OK;
}

ss_status ss_debug_level(ss_ctx* c, int32_t frame, int32_t level, const uint8_t** d_ptr, int32_t* pitch) {
  if (!c || !d_ptr || !pitch) return fail(SS_EINVAL, "NULL argument");
  if (frame < 0 || frame >= c->max_frames || level < 1 || level >= c->g.L) return fail(SS_EINVAL, "bad frame/level");
  *d_ptr = c->pyr + (int64_t)frame * c->g.pyr_frame_bytes + c->g.lvl_off[level];
  *pitch = c->g.pitch[level];
  return SS_OK;
}

ss_status ss_debug_candidates(ss_ctx* c, int32_t frame, int32_t level, int32_t* h_lx, int32_t* h_ly, int32_t* h_score,
                              int32_t cap, int32_t* n) {
  if (!c || !n) return fail(SS_EINVAL, "NULL argument");
  if (frame < 0 || frame >= c->max_frames || level < 0 || level >= c->g.L) return fail(SS_EINVAL, "bad frame/level");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  SS_CUDA_TRY(cudaDeviceSynchronize());
  const Geom& g = c->g;
  const int c0 = g.cell_first[level], nc = g.ncells[level];
  std::vector<int32_t> cnt(nc);
  SS_CUDA_TRY(cudaMemcpy(cnt.data(), c->cell_counts + (int64_t)frame * g.total_cells + c0, sizeof(int32_t) * nc,
                         cudaMemcpyDeviceToHost));
  std::vector<uint32_t> sl(g.level_slots[level]);
  SS_CUDA_TRY(cudaMemcpy(sl.data(), c->slots + (int64_t)frame * g.slots_per_frame + g.level_slot_off[level],
                         sizeof(uint32_t) * sl.size(), cudaMemcpyDeviceToHost));
  int k = 0;
  for (int i = 0; i < nc; i++) {
    const CellInfo& ci = c->cells_h[c0 + i];
    for (int j = 0; j < cnt[i]; j++) {
      if (k < cap) {
        const uint32_t v = sl[ci.slot_off - g.level_slot_off[level] + j];
        if (h_lx) h_lx[k] = key_lx(v);
        if (h_ly) h_ly[k] = key_ly(v);
        if (h_score) h_score[k] = key_m(v);
      }
      k++;
    }
  }
  *n = k;
  if (k > cap) return fail(SS_ECAPACITY, "more candidates than cap");
  return SS_OK;
}

ss_status ss_debug_phase_times(ss_ctx* c, int32_t frame, int32_t level, int64_t* h_ns, int32_t n) {
  if (!c || !h_ns || n < 0 || n > 16) return fail(SS_EINVAL, "bad argument");
  if (frame < 0 || frame >= c->max_frames || level < 0 || level >= c->g.L) return fail(SS_EINVAL, "bad frame/level");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  SS_CUDA_TRY(cudaDeviceSynchronize());
  SS_CUDA_TRY(cudaMemcpy(h_ns, c->phase_ts + ((int64_t)frame * c->g.L + level) * 16, sizeof(int64_t) * n,
                         cudaMemcpyDeviceToHost));
  return SS_OK;
}

ss_status ss_debug_overflow_count(ss_ctx* c, int32_t* n) {
  if (!c || !n) return fail(SS_EINVAL, "NULL argument");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  SS_CUDA_TRY(cudaDeviceSynchronize());
  int32_t v[2];
  SS_CUDA_TRY(cudaMemcpy(v, c->ovf_counter, sizeof(v), cudaMemcpyDeviceToHost));
  *n = v[0];
  if (v[1] != 0) return fail(SS_ECAPACITY, "a level kept more keypoints than its level_cap (bug)");
  return SS_OK;
}

ss_status ss_debug_distribution_paths(ss_ctx* c, int32_t* n_sort_smem, int32_t* n_global) {
  if (!c) return fail(SS_EINVAL, "NULL argument");
  SS_CUDA_TRY(cudaSetDevice(c->device));
  SS_CUDA_TRY(cudaDeviceSynchronize());
  int32_t v[3];
  SS_CUDA_TRY(cudaMemcpy(v, c->ovf_counter, sizeof(v), cudaMemcpyDeviceToHost));
  if (n_global) *n_global = v[0];
  if (n_sort_smem) *n_sort_smem = v[2];
  return SS_OK;
}

ss_status ss_debug_match_lanes(ss_ctx* c, int32_t lanes) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  if (lanes != 0 && lanes != 1 && lanes != 2 && lanes != 4 && lanes != 8) return fail(SS_EINVAL, "lanes must be 0, 1, 2, 4 or 8");
  c->win_lanes = lanes;
  return SS_OK;
}

ss_status ss_debug_capture_samples(ss_ctx* c, uint8_t* d_samples) {
  if (!c) return fail(SS_EINVAL, "NULL ctx");
  c->dbg_samples = d_samples;
  return SS_OK;
}

}  // extern "C"
