// k_grid.cu -- S4 alternative: grid top-N keypoint distribution (the north_star's "grid
// top-N" option next to the quadtree; DESIGN.md §3 item 13, the O4g
// reading): on level l with N = n_per_level[l], K = FAST cells holding a candidate,
// q = ceil(N / K), every cell keeps its q best candidates by (score desc, rank asc), and if
// more than N remain the N best of them (same order) are kept.  Selected via
// ss_set_distribution(ctx, SS_DIST_GRID_TOPN).
//
// One 1024-thread CTA per (level, frame), candidates read in place from the FAST cell slots:
//  1. per-cell candidate offsets (block scan of the cell counts), K;
//  2. a candidate's rank inside its cell = #{cell members with a better (score, rank)} (cells
//     hold tens of candidates, so the cell-local loop is cheap); pool = rank < q;
//  3. if the pool exceeds N: a 256-bin score histogram gives the threshold score s*, and the
//     members with score s* are admitted in rank order by a block-wide exclusive scan;
//  4. the kept keys are written in canonical (ly, lx) order (rank by counting, <= N keys).
#include <cub/block/block_reduce.cuh>
#include <cub/block/block_scan.cuh>

#include "ss_internal.h"

namespace ss {

namespace {

constexpr int GT = 1024;
constexpr int GMAX_CELLS = 4608;
typedef cub::BlockScan<int, GT> GScan;
typedef cub::BlockReduce<int, GT> GReduce;

struct GridShared {
  union {
    typename GScan::TempStorage scan;
    typename GReduce::TempStorage reduce;
  };
  int hist[256];
  int n, K, pool, thr, need, nk, run;
};

__global__ void __launch_bounds__(GT, 1)
    distribute_grid_kernel(const __grid_constant__ Geom g, const CellInfo* __restrict__ cells,
                           const uint32_t* __restrict__ slots, const int32_t* __restrict__ cell_counts,
                           uint32_t* __restrict__ selected, int32_t* __restrict__ sel_counts, int level0) {
  pdl_wait();
  pdl_trigger();
  extern __shared__ __align__(16) uint8_t sm[];
  __shared__ GridShared S;
  const int l = level0 + blockIdx.x, f = blockIdx.y, tid = threadIdx.x;
  const int ncells = g.ncells[l], c0 = g.cell_first[l];
  int32_t* coff = reinterpret_cast<int32_t*>(sm);  // [ncells + 1] candidate offsets (rank order)
  int32_t* cslot = coff + GMAX_CELLS + 1;          // [ncells] slot offsets in the frame's slot array
  uint32_t* kept = reinterpret_cast<uint32_t*>(cslot + GMAX_CELLS);  // [<= N]
  const int32_t* cc = cell_counts + (int64_t)f * g.total_cells + c0;
  const uint32_t* fs = slots + (int64_t)f * g.slots_per_frame;
  const int N = g.N[l];

  // ---- 1. offsets, n, K ----
  {
    const int cpt = (ncells + GT - 1) / GT;  // <= 5
    int cnt[5];
    int s = 0, k = 0;
#pragma unroll
    for (int j = 0; j < 5; j++) {
      const int c = tid * cpt + j;
      cnt[j] = (j < cpt && c < ncells) ? cc[c] : 0;
      s += cnt[j];
      k += cnt[j] > 0;
    }
    int ex, tot;
    GScan(S.scan).ExclusiveSum(s, ex, tot);
#pragma unroll
    for (int j = 0; j < 5; j++) {
      const int c = tid * cpt + j;
      if (j < cpt && c < ncells) {
        coff[c] = ex;
        cslot[c] = cells[c0 + c].slot_off;
        ex += cnt[j];
      }
    }
    __syncthreads();
    const int K = GReduce(S.reduce).Sum(k);
    if (tid == 0) {
      coff[ncells] = tot;
      S.n = tot;
      S.K = K;
      S.nk = 0;
      S.run = 0;
    }
    if (tid < 256) S.hist[tid] = 0;
    __syncthreads();
  }
  const int n = S.n, K = S.K;
  if (n == 0 || N <= 0) {
    if (tid == 0) sel_counts[f * g.L + l] = 0;
    return;
  }
  const int q = (N + K - 1) / K;
  // candidate i -> (key, pool flag); cell-local rank by (score desc, rank asc)
  auto fetch = [&](int i, uint32_t* key) -> bool {
    int lo = 0, hi = ncells - 1;  // last cell with coff[c] <= i
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (coff[mid] <= i) lo = mid; else hi = mid - 1;
    }
    const int b = coff[lo], e = coff[lo + 1];
    const uint32_t* cs = fs + cslot[lo] - b;
    const uint32_t k = cs[i];
    const int m = key_m(k);
    int better = 0;
    for (int j = b; j < e && better < q; j++) {
      const int mj = key_m(cs[j]);
      better += (mj > m) || (mj == m && j < i);
    }
    *key = k;
    return better < q;
  };
  // ---- 2. pool size + score histogram ----
  int mine = 0;
  for (int i = tid; i < n; i += GT) {
    uint32_t k;
    if (fetch(i, &k)) {
      mine++;
      atomicAdd(&S.hist[key_m(k)], 1);
    }
  }
  const int pool = GReduce(S.reduce).Sum(mine);
  if (tid == 0) {
    S.pool = pool;
    S.thr = -1;  // keep the whole pool
    S.need = 0;
    if (pool > N) {
      int cum = 0, s = 255;
      for (; s >= 0; s--) {
        if (cum + S.hist[s] >= N) break;
        cum += S.hist[s];
      }
      S.thr = s;          // scores > s all kept, need of the score-s members (in rank order)
      S.need = N - cum;
    }
  }
  __syncthreads();
  const int thr = S.thr, need = S.need;
  // ---- 3. admit (rank order for the threshold score) ----
  for (int i0 = 0; i0 < n; i0 += GT) {
    const int i = i0 + tid;
    uint32_t k = 0;
    bool in = false;
    if (i < n) in = fetch(i, &k);
    const int m = key_m(k);
    const int tie = (in && thr >= 0 && m == thr) ? 1 : 0;
    int ex, tot;
    GScan(S.scan).ExclusiveSum(tie, ex, tot);
    const int base = S.run;
    bool keep = in && (thr < 0 || m > thr || (tie && base + ex < need));
    if (keep) kept[atomicAdd(&S.nk, 1)] = k;
    __syncthreads();
    if (tid == 0) S.run = base + tot;
    __syncthreads();
  }
  // ---- 4. canonical (ly, lx) order ----
  const int nk = S.nk;
  uint32_t* out = selected + (int64_t)f * g.kp_capacity + g.cap_off[l];
  for (int t = tid; t < nk; t += GT) {
    const uint32_t k = kept[t] >> 8;
    int pos = 0;
    for (int u = 0; u < nk; u++) pos += (kept[u] >> 8) < k;
    out[pos] = kept[t];
  }
  if (tid == 0) sel_counts[f * g.L + l] = nk;
}

}  // namespace

size_t grid_smem_bytes(const Geom& g) {
  int capmax = 0;
  for (int l = 0; l < g.L; l++) capmax = capmax > g.N[l] ? capmax : g.N[l];
  return (size_t)(2 * GMAX_CELLS + 1) * 4 + (size_t)capmax * 4 + 16;
}

cudaError_t grid_init() {  // ss_create, per device (ss_set_distribution checks grid_smem_bytes vs 200 KB)
  return set_max_dynamic_smem(distribute_grid_kernel);
}

cudaError_t launch_distribute_grid(const Geom& g, int n_frames, int level0, int n_levels, const CellInfo* cells,
                                   const uint32_t* slots, const int32_t* cell_counts, uint32_t* selected,
                                   int32_t* sel_counts, cudaStream_t s) {
  if (n_levels <= 0) return cudaSuccess;
  const size_t smem = grid_smem_bytes(g);
  cudaError_t e = launch_pdl(distribute_grid_kernel, dim3(n_levels, n_frames), dim3(GT), smem, s, g, cells, slots, cell_counts,
                 selected, sel_counts, level0);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
