// k_pyramid.cu -- S1: image pyramid, level l = bilinear resize of level l-1 (DESIGN.md §3 O1).
//
// Fixed-point definition (bit-exact INTER_LINEAR_EXACT semantics): per destination column
// the host precomputes (x0, wx1, x1-x0) with wx1 = rne(frac * 256); then
//   out = ((256-wy1)*(wx0*s[y0][x0] + wx1*s[y0][x1]) + wy1*(...row y1...) + 2^15) >> 16.
//
// One launch builds all levels of all frames as a dataflow over row tiles: a persistent grid
// takes tiles (level, frame, 8-row band) from a global ticket counter in level order; a tile
// waits (acquire) until the bands of level l-1 it reads are published, stages those source rows
// in shared memory with 16-B L2 loads (ld.global.cg: never stale L1 lines), writes its rows 4
// pixels per thread (one 32-bit store) and publishes its band (release).  Every tile depends
// only on tiles with smaller tickets, all held by running CTAs, so the wait cannot deadlock.
// This replaces 7 dependent launches (each latency-bound on the small levels) by one.
#include "ss_internal.h"

namespace ss {

namespace {

constexpr int PT = 256;        // threads per CTA
constexpr int BAND_ROWS = 8;   // output rows per tile
constexpr int MAX_SRC_ROWS = 16;  // source rows one 8-row tile may read (checked at ss_create)
constexpr int kSrcPitchMax = 2080;

__device__ __forceinline__ int ld_acquire(const int* p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
  asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

struct PyrTables {
  const uint32_t* xtab[kMaxLevels];
  const uint32_t* ytab[kMaxLevels];
  int32_t nbands[kMaxLevels];     // 8-row bands of level l
  int32_t band_first[kMaxLevels]; // flag index of level l's first band (per frame)
  int32_t tile_first[kMaxLevels]; // first ticket of level l (for n_frames frames)
  int32_t total_tiles;
  int32_t flags_per_frame;
};

__global__ void __launch_bounds__(PT) pyramid_dataflow_kernel(Geom g, FrameSrc src, PyrTables t, int n_frames,
                                                              int* __restrict__ ticket, int* __restrict__ flags) {
  __shared__ __align__(16) uint8_t srows[MAX_SRC_ROWS * kSrcPitchMax];
  __shared__ int s_tile;
  for (;;) {
    if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1);
    __syncthreads();
    const int tile = s_tile;
    if (tile >= t.total_tiles) return;
    int l = 1;
    while (l + 1 < g.L && tile >= t.tile_first[l + 1]) l++;
    const int k = tile - t.tile_first[l];
    const int f = k / t.nbands[l], band = k - f * t.nbands[l];
    const int dw = g.w[l], dh = g.h[l], sw = g.w[l - 1];
    const int r0 = band * BAND_ROWS, r1 = min(r0 + BAND_ROWS, dh);
    const uint32_t* ytab = t.ytab[l];
    const uint32_t* xtab = t.xtab[l];
    const int sy0 = (int)(__ldg(ytab + r0) & 0xFFFF);
    const uint32_t cyl = __ldg(ytab + r1 - 1);
    const int sy1 = (int)(cyl & 0xFFFF) + (int)(cyl >> 25);  // last source row read
    const uint8_t* s;
    int sp;
    if (l == 1) {
      s = src.frames + (int64_t)f * src.stride;
      sp = src.pitch;
    } else {
      s = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l - 1];
      sp = g.pitch[l - 1];
      if (threadIdx.x == 0) {  // wait for the source bands of level l-1
        const int* fl = flags + (int64_t)f * t.flags_per_frame + t.band_first[l - 1];
        for (int b = sy0 / BAND_ROWS; b <= sy1 / BAND_ROWS; b++)
          while (ld_acquire(fl + b) == 0) __nanosleep(64);
      }
      __syncthreads();
    }
    // stage source rows sy0..sy1 (16-B chunks through L2)
    const int nrows = sy1 - sy0 + 1;
    const int spp = (sw + 15 + 15) & ~15;  // staged row pitch
    if ((sp & 15) == 0 && (reinterpret_cast<uintptr_t>(s) & 15) == 0) {
      const int nch = (sw + 15) >> 4;
      for (int i = threadIdx.x; i < nrows * nch; i += PT) {
        const int r = i / nch, c = i - r * nch;
        *reinterpret_cast<uint4*>(srows + r * spp + 16 * c) =
            __ldcg(reinterpret_cast<const uint4*>(s + (int64_t)(sy0 + r) * sp) + c);
      }
    } else {
      for (int i = threadIdx.x; i < nrows * sw; i += PT) {
        const int r = i / sw, c = i - r * sw;
        srows[r * spp + c] = __ldcg(s + (int64_t)(sy0 + r) * sp + c);
      }
    }
    __syncthreads();
    uint8_t* d = src.pyr + (int64_t)f * g.pyr_frame_bytes + g.lvl_off[l];
    const int dp = g.pitch[l];
    const int ngx = (dw + 3) >> 2;
    for (int i = threadIdx.x; i < (r1 - r0) * ngx; i += PT) {
      const int yy = i / ngx, gx = (i - yy * ngx) * 4;
      const int y = r0 + yy;
      const uint32_t cy = __ldg(ytab + y);
      const int y0 = (int)(cy & 0xFFFF), wy1 = (int)((cy >> 16) & 0x1FF), y1 = y0 + (int)(cy >> 25);
      const uint8_t* a0 = srows + (y0 - sy0) * spp;
      const uint8_t* a1 = srows + (y1 - sy0) * spp;
      uint32_t packed = 0;
#pragma unroll
      for (int q = 0; q < 4; q++) {
        const int x = gx + q;
        if (x < dw) {
          const uint32_t cx = __ldg(xtab + x);
          const int x0 = (int)(cx & 0xFFFF), wx1 = (int)((cx >> 16) & 0x1FF), x1 = x0 + (int)(cx >> 25);
          const int wx0 = 256 - wx1;
          const int h0 = wx0 * a0[x0] + wx1 * a0[x1];
          const int h1 = wx0 * a1[x0] + wx1 * a1[x1];
          const int v = (256 - wy1) * h0 + wy1 * h1;
          packed |= (uint32_t)((v + (1 << 15)) >> 16) << (8 * q);
        }
      }
      uint8_t* drow = d + (int64_t)y * dp;
      if (gx + 4 <= dw) {
        *reinterpret_cast<uint32_t*>(drow + gx) = packed;  // pitch is a multiple of 16
      } else {
        for (int q = 0; gx + q < dw; q++) drow[gx + q] = (uint8_t)(packed >> (8 * q));
      }
    }
    __syncthreads();  // all rows of the tile written (and srows free for the next tile)
    if (threadIdx.x == 0) {
      __threadfence();
      st_release(flags + (int64_t)f * t.flags_per_frame + t.band_first[l] + band, 1);
    }
  }
}

}  // namespace

int pyramid_max_src_rows() { return MAX_SRC_ROWS; }
int pyramid_band_rows() { return BAND_ROWS; }

int pyramid_flags_per_frame(const Geom& g) {
  int n = 0;
  for (int l = 0; l < g.L; l++) n += (g.h[l] + BAND_ROWS - 1) / BAND_ROWS;
  return n;
}

cudaError_t launch_pyramid(const Geom& g, int n_frames, FrameSrc src, const uint32_t* xytab, const int64_t* xoff,
                           const int64_t* yoff, int* ticket_and_flags, cudaStream_t s) {
  if (g.L < 2) return cudaSuccess;
  PyrTables t;
  int band_first = 0, tiles = 0;
  for (int l = 0; l < kMaxLevels; l++) {
    t.xtab[l] = t.ytab[l] = nullptr;
    t.nbands[l] = t.band_first[l] = t.tile_first[l] = 0;
  }
  for (int l = 0; l < g.L; l++) {
    t.nbands[l] = (g.h[l] + BAND_ROWS - 1) / BAND_ROWS;
    t.band_first[l] = band_first;
    band_first += t.nbands[l];
    if (l >= 1) {
      t.xtab[l] = xytab + xoff[l];
      t.ytab[l] = xytab + yoff[l];
      t.tile_first[l] = tiles;
      tiles += t.nbands[l] * n_frames;
    }
  }
  t.total_tiles = tiles;
  t.flags_per_frame = band_first;
  const size_t flag_bytes = sizeof(int) * (1 + (size_t)n_frames * band_first);
  cudaError_t e = cudaMemsetAsync(ticket_and_flags, 0, flag_bytes, s);
  if (e != cudaSuccess) return e;
  const int grid = tiles < 148 * 4 ? tiles : 148 * 4;
  pyramid_dataflow_kernel<<<grid, PT, 0, s>>>(g, src, t, n_frames, ticket_and_flags, ticket_and_flags + 1);
  return cudaGetLastError();
}

}  // namespace ss
