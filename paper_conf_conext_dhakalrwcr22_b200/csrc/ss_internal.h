// ss_internal.h -- product-internal types shared by the host layer (ss_api.cpp) and the
// sm_100a kernels.  Nothing here is shared with oracle/ (the CPU checker).
#pragma once
#include <cuda.h>  // CUtensorMap (TMA descriptors; encoded through the runtime's driver entry point)
#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdlib>
#include <vector>

#include "../../include/ss.h"

namespace ss {

constexpr int kMaxLevels = SS_MAX_LEVELS;
constexpr int kEdgeThreshold = 19;  // ORB-SLAM EDGE_THRESHOLD [ext]
constexpr int kMinBorder = kEdgeThreshold - 3;
constexpr int kCellPx = 30;         // FAST grid cell (north_star "per 30-px grid cell")
constexpr int kQuadRounds = 13;     // quadtree path depth stored per key (levels <= 2048 px)

// One FAST cell: detect window D = [x0,x1) x [y0,y1) of its level (DESIGN.md §3 O3) and
// the range of its candidate slots inside a frame's slot array.
struct CellInfo {
  int32_t level;
  int32_t x0, y0, x1, y1;
  int32_t slot_off;  // entries from the start of the frame's slot array
  int32_t slot_cap;  // ceil(Dw/2)*ceil(Dh/2): strict 8-neighbour maxima per 2x2 block <= 1
  int32_t pad;
};

// One row of FAST cells of one level ("band"): the cells' detect windows share rows
// [y0, y1) and tile columns [x0, x1); cells [cell_first, cell_first + ncells) of the table.
struct BandInfo {
  int32_t level;
  int32_t y0, y1;
  int32_t x0, x1;
  int32_t cell_first;
  int32_t ncells;
  int32_t pad;
};

// Everything the kernels need to know about the frame shape, by value in kernel params.
struct Geom {
  int32_t L, W, H;
  int32_t ini_th, min_th;
  int32_t w[kMaxLevels], h[kMaxLevels];
  int32_t pitch[kMaxLevels];        // pyramid scratch pitch of level l (l >= 1)
  int64_t lvl_off[kMaxLevels];      // byte offset of level l in a frame's pyramid scratch
  int64_t pyr_frame_bytes;
  float scale[kMaxLevels];
  float inv_scale[kMaxLevels];      // f32(1 / scale[l]) (O0)
  int32_t row_off[kMaxLevels];      // start of level l in a frame's keypoint row index (sum of h + 1)
  int32_t cell_first[kMaxLevels];   // first active cell of level l in the cell table
  int32_t ncells[kMaxLevels];       // active cells of level l (row-major, skipped cells removed)
  int32_t total_cells;              // per frame
  int32_t slots_per_frame;          // candidate slot entries per frame
  int32_t level_slot_off[kMaxLevels], level_slots[kMaxLevels];
  int32_t N[kMaxLevels];            // distribution target n_per_level
  int32_t cap[kMaxLevels];          // level_cap
  int32_t cap_off[kMaxLevels];      // offset of level l in a frame's selected-key scratch
  int32_t kp_capacity;
  int32_t nini[kMaxLevels];
  float hX[kMaxLevels];             // f32(qw / nIni)
  int32_t qw[kMaxLevels], qh[kMaxLevels];  // quadtree box (maxBorder - minBorder)
  int32_t qrounds[kMaxLevels];      // quadtree rounds that can still separate keys on level l
  int32_t max_rw, max_rh;           // largest FAST input region (D + 3-px halo) of any cell
  int32_t total_bands;              // FAST work units (cell-row segments) over all levels, per frame
  int32_t level0_bands;             // ... of which on level 0 (they come first)
  int32_t band_first[kMaxLevels], band_count[kMaxLevels];  // FAST work units of level l
  int32_t max_band_w, max_band_h;   // widest band (detect columns) / tallest band (detect rows)
  int32_t max_cell_w;               // widest cell detect window
  // quadtree key tables (k_distribute.cu): level l's x part (root + right bits) for kx in
  // [0, qw] at qtab_off[l], its y part (down bits) for ky in [0, qh] right after
  int32_t qtab_off[kMaxLevels];
  int32_t qtab_total;
  int32_t dense_r[kMaxLevels];      // deepest dense-histogram depth R of level l (nIni * 4^R <= 4096)
};

// Where the frames of one call live.  Level 0 is the caller's frame (no copy).
struct FrameSrc {
  const uint8_t* frames;
  int64_t stride;
  int32_t pitch;
  uint8_t* pyr;  // pyramid scratch (levels >= 1)
};

// TMA tensor maps of the descriptor kernel's 43-row x 64-byte patch loads, one per pyramid
// level: 3-D u8 [frames][h_l][w_l] with the level's row pitch and frame stride (level 0 = the
// caller's frames, encoded per ss_orb_extract call; levels >= 1 = the pyramid scratch, encoded
// at ss_create).  Bit l of `valid`: level l may be loaded by TMA (16-B aligned base / pitch /
// stride), else the kernel uses its LDG path.
constexpr int kPatchBoxW = 64, kPatchBoxH = 43;
struct PatchMaps {
  CUtensorMap level[kMaxLevels];
  uint32_t valid;
};
// Encode one level's map; false if the layout is not TMA-addressable (alignment).
bool encode_patch_map(CUtensorMap* m, const void* base, int w, int h, int frames, int64_t pitch, int64_t fstride);

// Candidate / selected key: (ly << 19) | (lx << 8) | M  (lx, ly < 2048, M = FAST score + 1).
__host__ __device__ inline uint32_t pack_key(int lx, int ly, int m) {
  return ((uint32_t)ly << 19) | ((uint32_t)lx << 8) | (uint32_t)m;
}
__host__ __device__ inline int key_lx(uint32_t k) { return (int)((k >> 8) & 0x7FF); }
__host__ __device__ inline int key_ly(uint32_t k) { return (int)(k >> 19); }
__host__ __device__ inline int key_m(uint32_t k) { return (int)(k & 0xFF); }

// ---- Programmatic Dependent Launch (sm_90+): every kernel of the chain is launched with
// programmatic stream serialisation, lets its dependents launch as soon as all its CTAs are
// resident (pdl_trigger) and waits for its predecessor's completion + memory (pdl_wait)
// before touching its inputs.  This hides the launch latency between dependent kernels. ----
#ifdef __CUDACC__
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s,
                              Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, static_cast<KArgs>(args)...);
}

// Opt a kernel into the largest dynamic shared memory the current device allows next to its
// static shared memory (the launch itself passes what it needs).
template <typename K>
inline cudaError_t set_max_dynamic_smem(K kernel) {
  int dev = 0, optin = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  cudaFuncAttributes fa;
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&fa, kernel);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, optin - (int)fa.sharedSizeBytes);
}
// Shared-memory carveout (percent of the unified L1/shared array) from SS_CARVEOUT, for the
// A/B of one fixed carveout across the extraction kernels (no reconfiguration between them);
// unset = the driver's choice.
template <typename K>
inline cudaError_t carveout_from_env(K kernel) {
  const char* e = std::getenv("SS_CARVEOUT");
  if (!e) return cudaSuccess;
  return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, std::atoi(e));
}
#endif

// ---- launchers (one per kernel; each returns cudaGetLastError()) ----
// Fused pyramid plan (k_pyramid.cu).  Host-side rectangles per (block, level), half-open:
// N = computed (owned + the halo deeper levels need), O = owned (stored).  Level 0: N only
// (the staged footprint, x0 aligned down to 16).
struct PyrRect {
  int16_t nx0, nx1, ny0, ny1, ox0, ox1, oy0, oy1;
};
// Device-side per (block, level >= 1) record, read as four int4 (entry 0: the staged
// footprint nx0/ny0/rows, ngx = staged width, dpitch = staged pitch, soff = s_y base).
struct __align__(16) PyrLvl {
  int32_t nx0, ngx, ny0, rows;        // computed rectangle: x0, 4-column groups, y0, rows
  int32_t ox0, ox1, oy0, oy1;         // owned rectangle
  int32_t sx0, sy0, spitch, dpitch;   // source rectangle origin + pitches of the smem buffers
  int32_t mr, soff, gg, yg;           // ceil(2^20/ngx) | rows-in-parallel << 21; s_g | s_y << 16
                                      // offsets; first group / row coefficient in the tables
};
constexpr int kPyrSmemMax = 200 * 1024;
// Per 4-column group coefficient table of every level >= 1 (goff[l] = level l's first
// entry); false if scale_factor > 4/3 (a group's source bytes exceed the 6-byte window).
bool pyramid_groups(const Geom& g, const uint32_t* tab, const int64_t* xoff, std::vector<uint4>* gtab,
                    std::vector<int64_t>* goff);
// Plan gx x gy blocks per frame; false if a block does not fit (shared memory, one
// coefficient load per thread per level).
bool pyramid_plan(const Geom& g, const uint32_t* tab, const int64_t* xoff, const int64_t* yoff,
                  const std::vector<int64_t>& goff, int gx, int gy, std::vector<PyrLvl>* plan, int* buf0, int* buf1,
                  int* smem);
// Levels 1..L-1 of all frames in one launch (grid: n_blocks x n_frames).
cudaError_t launch_pyramid(const Geom& g, int n_frames, FrameSrc src, const uint4* gtab, const uint32_t* ytab,
                           const PyrLvl* plan, int n_blocks, int buf0, int buf1, int smem, cudaStream_t s);
cudaError_t launch_fast_bands(const Geom& g, int n_frames, FrameSrc src, const BandInfo* bands, int n_bands,
                              const CellInfo* cells, uint32_t* slots, int32_t* cell_counts, cudaStream_t s,
                              bool flat = false);
size_t fast_smem_bytes(const Geom& g, int* rp, int* mbw, int* region_bytes, int* mband_bytes, int* nball);
cudaError_t launch_distribute(const Geom& g, int n_frames, int level0, int n_levels, const CellInfo* cells,
                              const uint32_t* qtab, const uint32_t* slots, const int32_t* cell_counts, uint32_t* selected,
                              int32_t* sel_counts, uint8_t* ovf, int64_t ovf_frame_bytes,
                              const int64_t* ovf_level_off, int32_t* ovf_counter, uint64_t* phase_ts,
                              cudaStream_t s);
cudaError_t launch_describe(const Geom& g, int n_frames, FrameSrc src, const uint32_t* selected,
                            const int32_t* sel_counts, const int8_t* pattern, ss_keypoint* kps, uint8_t* desc,
                            int32_t* counts, uint8_t* samples, const PatchMaps& maps,
                            cudaStream_t s);  // samples: test hook or NULL
// The rotated-BRIEF pattern (1024 ints: 256 pairs x 2 points x (x, y)), host copy.
const int* brief_pattern_host();
// Row index of the keypoints (first keypoint per (frame, level, row)) + dedup claim reset.
int match_rows_per_frame(const Geom& g);
// per-frame stride of the global index buffer: the row index, then the keypoints' lx (u16)
int match_index_stride(const Geom& g);
cudaError_t launch_match_prepare(const Geom& g, int n_frames, const ss_keypoint* kps, const int32_t* counts,
                                 uint16_t* rowidx, unsigned long long* claim, int dedup, cudaStream_t s);
cudaError_t launch_match_window(const Geom& g, int n_frames, const ss_keypoint* kps, const uint8_t* desc,
                                const int32_t* counts, const uint8_t* taken, int n_queries,
                                const ss_mp_query* q, const uint8_t* qdesc, ss_match_cfg cfg,
                                unsigned long long* claim, ss_match* out, const uint16_t* rowidx,
                                int lanes, cudaStream_t s);  // lanes per query: 0 = chosen per launch
cudaError_t launch_match_resolve(const Geom& g, int n_queries, const ss_mp_query* q,
                                 const unsigned long long* claim, ss_match* out, cudaStream_t s);
cudaError_t launch_brute_merge(const Geom& g, int n_frames, const int32_t* counts, int splits,
                               const unsigned long long* partial, ss_match_cfg cfg, ss_match* out,
                               cudaStream_t s);
// Map-sharded brute force (F4): one shard's top-2 with global indices, and the merge of the
// shards' top-2 lists + the accept rule.
cudaError_t launch_brute_shard_top2(const Geom& g, int n_frames, const int32_t* counts, int splits,
                                    const unsigned long long* partial, int map_offset, unsigned long long* top2,
                                    cudaStream_t s);
cudaError_t launch_brute_parts_merge(const Geom& g, int n_frames, const int32_t* counts, int n_parts,
                                     const unsigned long long* parts, ss_match_cfg cfg, ss_match* out, cudaStream_t s);
// Tensor-core brute matcher (k_brute_tc.cu): expanded-operand scratch sizes, the map split
// count (whole waves of one CTA per SM), and expand + tcgen05 partial top-2 (per-split partial
// top-2, reduced by launch_brute_merge).
int64_t brute_tc_query_bytes(int64_t n_slots);
int64_t brute_tc_map_bytes(int64_t n_map);
int brute_tc_splits(int n_slots, int n_map, int max_splits, int n_sm);
// desc == NULL: map rows only; map_desc == NULL: keypoint rows only (prepared map)
cudaError_t launch_brute_expand(int n_slots, const uint8_t* desc, int n_map, const uint8_t* map_desc, int8_t* qexp,
                                int8_t* mexp, cudaStream_t s);
cudaError_t launch_brute_tc(int n_slots, int n_map, const int8_t* qexp, const int8_t* mexp, int splits,
                            unsigned long long* partial, cudaStream_t s);

// O11 local-map projection (k_project.cu): one thread per map point.
cudaError_t launch_project(const Geom& g, int n_frames, const ss_camera* cams, int n_points, const ss_map_point* pts,
                           const int32_t* point_frame, float th, ss_mp_query* out, cudaStream_t s);

// O4g grid top-N distribution (k_grid.cu), same outputs as launch_distribute.
cudaError_t launch_distribute_grid(const Geom& g, int n_frames, int level0, int n_levels, const CellInfo* cells,
                                   const uint32_t* slots, const int32_t* cell_counts, uint32_t* selected,
                                   int32_t* sel_counts, cudaStream_t s);

// O12 stereo matching (k_stereo.cu): one warp per left keypoint, then the per-pair outlier cut.
cudaError_t launch_stereo(const Geom& g, int n_pairs, FrameSrc src, const ss_keypoint* kps, const uint8_t* desc,
                          const int32_t* counts, const uint16_t* rowidx, int index_stride, float bf, float maxD,
                          float* uright, float* depth, int32_t* sad, cudaStream_t s);
cudaError_t launch_stereo_outliers(const Geom& g, int n_pairs, const int32_t* counts, const int32_t* sad,
                                   float* uright, float* depth, cudaStream_t s);

// O13 frame-to-frame projection matching (k_lastframe.cu): one CTA (or cluster) per frame;
// dynamic shared memory per CTA (keypoint positions + lx + row index [+ descriptors]), <= 200 KB.
size_t lastframe_smem_bytes(const Geom& g);
cudaError_t lastframe_init();  // kernel attributes (ss_create)
// Kernel attributes (the >48 KB dynamic shared-memory opt-in) of the other kernels.  Attributes
// are per device, so ss_create sets them on its device every time (cheap; never under capture).
cudaError_t fast_init();
cudaError_t distribute_init();
cudaError_t describe_init();
cudaError_t pyramid_init();
cudaError_t brute_tc_init();
cudaError_t grid_init();
size_t grid_smem_bytes(const Geom& g);  // dynamic shared memory of the grid top-N kernel
cudaError_t launch_lastframe(const Geom& g, int n_frames, const ss_camera* cams, const ss_camera* last_cams, float mb,
                             const ss_keypoint* kps, const uint8_t* desc, const int32_t* counts, const uint8_t* taken,
                             const int32_t* pt_off, const ss_frame_point* pts, const uint8_t* pdesc, float th,
                             int th_high, int check_orientation, int min_matches, ss_match* out, int32_t* n_matches,
                             uint8_t* matched, unsigned long long* claim, uint16_t* rowidx,
                             unsigned long long* win_claim, int n_sm, cudaStream_t s, void (*mark)(void*),
                             void* mark_arg);  // mark: profiling-event hook before / after each launch

// Quadtree key tables of every level (ss_create, once): qtab[g.qtab_total] u32.
cudaError_t launch_distribute_tables(const Geom& g, uint32_t* qtab, cudaStream_t s);
// Overflow scratch bytes the distribution needs for a level with `slots` candidate slots.
int64_t distribute_ovf_bytes(int64_t slots);

}  // namespace ss
