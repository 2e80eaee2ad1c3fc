// k_distribute.cu -- S4: per-(frame, level) quadtree keypoint distribution
// (ORB-SLAM DistributeOctTree reading, DESIGN.md §3 O4), one 1024-thread CTA per
// (level, frame), round-synchronous reformulation:
//
//  * Each candidate's quadtree path is a function of its position only: the root is
//    trunc(f32 kx / hX) and at every round the child is chosen against the node's ceil
//    half-split.  We precompute 13 rounds of 2-bit quadrant codes per key
//    (key = root << 26 | path) and radix-sort the keys once (stable, CUB, in shared
//    memory).  Every depth-r node is then a contiguous run of keys sharing an r-prefix.
//  * dd_i = the round at which sorted neighbours i-1, i separate.  Histograms of dd and of
//    max(dd_i, dd_i+1) give, for every depth r at once, S_r = #nodes and E_r = #nodes
//    with > 1 key -- exactly the quantities ORB-SLAM's phase-1/phase-2 stop rules test
//    (splitting a 1-key node never changes the node count, so phase 1 after r rounds is
//    "group by r-prefix").
//  * Only the last, partial phase-2 round needs an order: its multi-key nodes are ranked
//    by (size desc, UL.y, UL.x, first-key rank) and split in that order until >= N nodes.
//  * Each final node keeps its max-score key (ties -> lowest rank); the kept keys are
//    written in canonical (ly, lx) order.
// Levels with more candidates than fit in shared memory (adversarial noise images) run
// the same code on global scratch with a 1-bit-per-pass LSD split sort (slow, correct,
// never truncated).
#include <cub/block/block_radix_sort.cuh>
#include <cub/block/block_scan.cuh>

#include "ss_internal.h"

namespace ss {

namespace {

constexpr int DT = 1024;
constexpr int DIPT = 8;
constexpr int DCAP = DT * DIPT;
constexpr int MAX_CELLS = 4608;
constexpr int REC_CAP_SMEM = DCAP / 2;

typedef cub::BlockRadixSort<uint32_t, DT, DIPT, uint32_t> BRS;
typedef cub::BlockScan<int, DT> BScan;

struct Arr {
  uint32_t* cand;   // [n] packed candidates, rank order
  uint32_t* key;    // [n] sorted keys (later: unsorted kept keys)
  uint32_t* rank;   // [n] rank of the i-th sorted key
  uint8_t* dd;      // [n] separation round of sorted neighbours (i >= 1)
  uint8_t* splitf;  // [n] at depth-d heads: child count | 0x80 if split
  uint64_t* rec;    // [rec_cap] partial-round order keys
  int32_t* rec_head;
  int32_t* order;
  uint32_t* key2;   // overflow path: ping-pong buffers of the split sort
  uint32_t* rank2;
};

constexpr size_t kSmemCells = MAX_CELLS * 4;
constexpr size_t kSmemArrays = (size_t)DCAP * 12;
constexpr size_t kUnionPost = (size_t)DCAP * 2 + (size_t)REC_CAP_SMEM * 16;
constexpr size_t kUnion = sizeof(typename BRS::TempStorage) > kUnionPost ? sizeof(typename BRS::TempStorage) : kUnionPost;
constexpr size_t kSmemTotal = kSmemCells + kSmemArrays + kUnion;
static_assert(kSmemTotal <= 227 * 1024, "distribution smem budget");

__device__ __forceinline__ void root_geom(const Geom& g, int l, int ri, int& ulx, int& urx) {
  ulx = __float2int_rz(__fmul_rn(g.hX[l], (float)ri));
  urx = __float2int_rz(__fmul_rn(g.hX[l], (float)(ri + 1)));
}

__device__ __forceinline__ uint32_t make_key(const Geom& g, int l, uint32_t packed) {
  const int kx = key_lx(packed) - kMinBorder, ky = key_ly(packed) - kMinBorder;
  int ri = __float2int_rz(__fdiv_rn((float)kx, g.hX[l]));
  ri = min(ri, g.nini[l] - 1);
  int ulx, urx;
  root_geom(g, l, ri, ulx, urx);
  int uly = 0, bly = g.qh[l];
  uint32_t path = 0;
#pragma unroll
  for (int r = 0; r < kQuadRounds; r++) {
    const int hx = (urx - ulx + 1) >> 1, hy = (bly - uly + 1) >> 1;  // ceil(w/2), w >= 0
    const int right = kx >= ulx + hx, down = ky >= uly + hy;
    path = (path << 2) | (uint32_t)(down * 2 + right);
    if (right) ulx += hx; else urx = ulx + hx;
    if (down) uly += hy; else bly = uly + hy;
  }
  return ((uint32_t)ri << 26) | path;
}

// Upper-left corner of the depth-d node holding `key`.
__device__ __forceinline__ void node_ul(const Geom& g, int l, uint32_t key, int d, int& ulx, int& uly) {
  const int ri = (int)(key >> 26);
  int urx;
  root_geom(g, l, ri, ulx, urx);
  uly = 0;
  int bly = g.qh[l];
  for (int r = 1; r <= d; r++) {
    const int q = (int)(key >> (26 - 2 * r)) & 3;
    const int hx = (urx - ulx + 1) >> 1, hy = (bly - uly + 1) >> 1;
    if (q & 1) ulx += hx; else urx = ulx + hx;
    if (q & 2) uly += hy; else bly = uly + hy;
  }
}

__device__ __forceinline__ int sep_round(uint32_t a, uint32_t b) {
  const uint32_t x = a ^ b;
  if (x >> 26) return 0;         // different roots
  if (x == 0) return 14;         // never separated (cannot happen for distinct pixels)
  return ((__clz((int)x) - 6) >> 1) + 1;
}

// Stable LSD split sort of (k, v) on bits [b0, b1), ping-ponging with (k2, v2); on return
// (k, v) name the sorted buffers.  Used only for levels that overflow shared memory.
__device__ void split_sort_global(uint32_t*& k, uint32_t*& v, uint32_t*& k2, uint32_t*& v2, int n, int b0,
                                  int b1, BScan::TempStorage& tmp) {
  const int tid = threadIdx.x;
  for (int b = b0; b < b1; b++) {
    int z = 0;
    for (int i = tid; i < n; i += DT) z += !((k[i] >> b) & 1u);
    int ex, total_zeros;
    BScan(tmp).ExclusiveSum(z, ex, total_zeros);
    __syncthreads();
    int run0 = 0;
    for (int base = 0; base < n; base += DT) {
      const int i = base + tid;
      const int zf = (i < n) ? !((k[i] >> b) & 1u) : 0;
      int pre, tile;
      BScan(tmp).ExclusiveSum(zf, pre, tile);
      if (i < n) {
        const int dst = zf ? run0 + pre : total_zeros + (base - run0) + (tid - pre);
        k2[dst] = k[i];
        v2[dst] = v[i];
      }
      run0 += tile;
      __syncthreads();
    }
    uint32_t* t = k; k = k2; k2 = t;
    t = v; v = v2; v2 = t;
  }
}

__global__ void __launch_bounds__(DT, 1)
    distribute_kernel(Geom g, const CellInfo* __restrict__ cells, const uint32_t* __restrict__ slots,
                      const int32_t* __restrict__ cell_counts, uint32_t* __restrict__ selected,
                      int32_t* __restrict__ sel_counts, uint8_t* ovf, int64_t ovf_frame_bytes,
                      const int64_t* __restrict__ ovf_level_off, int32_t* ovf_counter) {
  extern __shared__ __align__(16) uint8_t sm[];
  __shared__ typename BScan::TempStorage scan_tmp;
  __shared__ int sh[8];
  __shared__ int H[16], G[17], S[15], E[15];
  const int l = blockIdx.x, f = blockIdx.y, tid = threadIdx.x;
  const int warp = tid >> 5, lane = tid & 31;
  const int ncells = g.ncells[l];
  const int c0 = g.cell_first[l];
  const int N = g.N[l];
  int32_t* cell_off = reinterpret_cast<int32_t*>(sm);
  const int32_t* cc = cell_counts + (int64_t)f * g.total_cells + c0;

  // ---- 1. candidate offsets per cell (rank order = cells row-major, then raster) ----
  {
    const int cpt = (ncells + DT - 1) / DT;
    int s = 0;
    for (int j = 0; j < cpt; j++) {
      const int c = tid * cpt + j;
      if (c < ncells) s += cc[c];
    }
    int ex, tot;
    BScan(scan_tmp).ExclusiveSum(s, ex, tot);
    for (int j = 0; j < cpt; j++) {
      const int c = tid * cpt + j;
      if (c < ncells) {
        cell_off[c] = ex;
        ex += cc[c];
      }
    }
    if (tid == 0) {
      sh[0] = tot;
      for (int i = 0; i < 15; i++) H[i] = 0;
      H[15] = 0;
      for (int i = 0; i < 17; i++) G[i] = 0;
      sh[1] = 0;  // partial-round record count
      sh[2] = 0;  // kept keys
    }
    __syncthreads();
  }
  const int n = sh[0];
  uint32_t* sel_out = selected + (int64_t)f * g.kp_capacity + g.cap_off[l];
  if (n == 0) {
    if (tid == 0) sel_counts[f * g.L + l] = 0;
    return;
  }
  const bool big = n > DCAP;
  Arr a;
  if (!big) {
    uint8_t* p = sm + kSmemCells;
    a.cand = reinterpret_cast<uint32_t*>(p);
    a.key = a.cand + DCAP;
    a.rank = a.key + DCAP;
    uint8_t* u = reinterpret_cast<uint8_t*>(a.rank + DCAP);
    a.rec = reinterpret_cast<uint64_t*>(u);
    a.rec_head = reinterpret_cast<int32_t*>(a.rec + REC_CAP_SMEM);
    a.order = a.rec_head + REC_CAP_SMEM;
    a.dd = reinterpret_cast<uint8_t*>(a.order + REC_CAP_SMEM);
    a.splitf = a.dd + DCAP;
    a.key2 = a.rank2 = nullptr;
  } else {
    uint8_t* p = ovf + (int64_t)f * ovf_frame_bytes + ovf_level_off[l];
    const int64_t cap = g.level_slots[l];
    a.cand = reinterpret_cast<uint32_t*>(p);
    a.key = a.cand + cap;
    a.rank = a.key + cap;
    a.key2 = a.rank + cap;
    a.rank2 = a.key2 + cap;
    a.rec = reinterpret_cast<uint64_t*>(a.rank2 + cap + (cap & 1));
    a.rec_head = reinterpret_cast<int32_t*>(a.rec + (cap / 2 + 1));
    a.order = a.rec_head + (cap / 2 + 1);
    a.dd = reinterpret_cast<uint8_t*>(a.order + (cap / 2 + 1));
    a.splitf = a.dd + cap;
    if (tid == 0) atomicAdd(ovf_counter, 1);
  }

  // ---- 2. gather candidates into rank order (one warp per cell) ----
  {
    const uint32_t* fs = slots + (int64_t)f * g.slots_per_frame;
    for (int c = warp; c < ncells; c += DT / 32) {
      const int cnt = cc[c];
      const int off = cell_off[c];
      const uint32_t* src = fs + cells[c0 + c].slot_off;
      for (int j = lane; j < cnt; j += 32) a.cand[off + j] = src[j];
    }
    __syncthreads();
  }

  // ---- 3. quadtree keys + stable sort by key (value = rank) ----
  const int end_bit = 26 + (32 - __clz(max(g.nini[l] - 1, 1)));
  const int begin_bit = 0;
  if (!big) {
    uint32_t kk[DIPT], vv[DIPT];
#pragma unroll
    for (int i = 0; i < DIPT; i++) {
      const int idx = tid * DIPT + i;
      kk[i] = idx < n ? make_key(g, l, a.cand[idx]) : 0xFFFFFFFFu;
      vv[i] = (uint32_t)idx;
    }
    __syncthreads();
    BRS(*reinterpret_cast<typename BRS::TempStorage*>(sm + kSmemCells + kSmemArrays)).Sort(kk, vv, begin_bit, end_bit);
    __syncthreads();
#pragma unroll
    for (int i = 0; i < DIPT; i++) {
      const int idx = tid * DIPT + i;
      if (idx < n) {
        a.key[idx] = kk[i];
        a.rank[idx] = vv[i];
      }
    }
    __syncthreads();
  } else {
    for (int i = tid; i < n; i += DT) {
      a.key[i] = make_key(g, l, a.cand[i]);
      a.rank[i] = (uint32_t)i;
    }
    __syncthreads();
    split_sort_global(a.key, a.rank, a.key2, a.rank2, n, begin_bit, end_bit, scan_tmp);
  }

  // ---- 4. separation rounds + histograms -> S_r, E_r for every depth ----
  for (int i = tid; i < n; i += DT) a.dd[i] = i ? (uint8_t)sep_round(a.key[i - 1], a.key[i]) : 0;
  __syncthreads();
  for (int i = tid; i < n; i += DT) {
    const int lo = i ? (int)a.dd[i] : -1;
    const int hi = (i + 1 < n) ? (int)a.dd[i + 1] : -1;
    if (i) atomicAdd(&H[lo], 1);
    atomicAdd(&G[max(lo, hi) + 1], 1);
  }
  __syncthreads();
  if (tid == 0) {
    int s = 1, single = G[0];
    for (int r = 0; r <= 13; r++) {
      s += H[r];
      single += G[r + 1];
      S[r] = s;
      E[r] = s - single;
    }
    S[14] = S[13];
    E[14] = E[13];
    // ORB-SLAM's loop, on node counts only (phase 1 then phase 2 stop rules)
    int D = 1, partial = 0, r = 0;
    for (;;) {
      const int nx = S[min(r + 1, 14)];
      if (nx >= N || nx == S[r]) { D = r + 1; break; }
      if (nx + 3 * E[min(r + 1, 14)] > N) {
        int d = r + 1;
        for (;;) {
          const int s2 = S[min(d + 1, 14)];
          if (s2 >= N) { D = d; partial = 1; break; }
          if (s2 == S[min(d, 14)]) { D = d + 1; break; }
          d++;
        }
        break;
      }
      r++;
    }
    sh[3] = min(D, 14);
    sh[4] = partial;
  }
  __syncthreads();
  const int D = sh[3];
  const bool partial = sh[4] != 0;
  const int dlim = min(D, 13);

  // ---- 5. partial phase-2 round at depth D: order the multi-key nodes, split a prefix ----
  if (partial) {
    for (int i = tid; i < n; i += DT) {
      if (i != 0 && a.dd[i] > D) continue;  // not a depth-D node head
      int size = 1, c = 1;
      uint32_t minrank = a.rank[i];
      for (int j = i + 1; j < n && a.dd[j] > D; j++) {
        size++;
        minrank = min(minrank, a.rank[j]);
        c += (a.dd[j] == D + 1);
      }
      a.splitf[i] = 0;
      if (size > 1) {
        const int e = atomicAdd(&sh[1], 1);
        int ulx, uly;
        node_ul(g, l, a.key[i], D, ulx, uly);
        a.rec[e] = ((uint64_t)(0x1FFFFF - size) << 43) | ((uint64_t)uly << 32) | ((uint64_t)ulx << 20) |
                   (uint64_t)minrank;
        a.rec_head[e] = i;
        a.splitf[i] = (uint8_t)c;
      }
    }
    __syncthreads();
    const int ne = sh[1];
    for (int e = tid; e < ne; e += DT) {
      const uint64_t k = a.rec[e];
      int pos = 0;
      for (int e2 = 0; e2 < ne; e2++) pos += a.rec[e2] < k;
      a.order[pos] = e;
    }
    __syncthreads();
    if (tid == 0) {
      int acc = S[D];
      for (int t = 0; t < ne && acc < N; t++) {
        const int h = a.rec_head[a.order[t]];
        acc += (a.splitf[h] & 0x7F) - 1;
        a.splitf[h] |= 0x80;
      }
    }
    __syncthreads();
  }

  // ---- 6. one key per final node: max score, ties -> lowest rank ----
  uint32_t* kept = a.key;  // keys are no longer needed
  __syncthreads();
  for (int i = tid; i < n; i += DT) {
    if (i != 0 && a.dd[i] > dlim) continue;  // not a final node head
    const bool split = partial && (a.splitf[i] & 0x80);
    int best_m = -1;
    uint32_t best_r = 0;
    for (int j = i; j < n && (j == i || a.dd[j] > dlim); j++) {
      if (j != i && split && a.dd[j] == D + 1) {
        const int p = atomicAdd(&sh[2], 1);
        kept[p] = a.cand[best_r];
        best_m = -1;
      }
      const uint32_t r = a.rank[j];
      const int m = key_m(a.cand[r]);
      if (m > best_m || (m == best_m && r < best_r)) {
        best_m = m;
        best_r = r;
      }
    }
    const int p = atomicAdd(&sh[2], 1);
    kept[p] = a.cand[best_r];
  }
  __syncthreads();
  const int nk = sh[2];
  const int nk_w = min(nk, g.cap[l]);
  // ---- 7. canonical (ly, lx) order, into the frame's selected scratch ----
  for (int t = tid; t < nk; t += DT) {
    const uint32_t k = kept[t] >> 8;
    int pos = 0;
    for (int u = 0; u < nk; u++) pos += (kept[u] >> 8) < k;
    if (pos < nk_w) sel_out[pos] = kept[t];
  }
  if (tid == 0) {
    sel_counts[f * g.L + l] = nk_w;
    if (nk > g.cap[l]) atomicAdd(ovf_counter + 1, 1);  // impossible by the O4 bound; reported
  }
}

}  // namespace

int64_t distribute_ovf_bytes(int64_t slots) {
  // cand, key, rank, key2, rank2 (u32) + rec (u64) / rec_head / order (i32) + dd, splitf (u8)
  const int64_t rc = slots / 2 + 1;
  int64_t b = slots * 4 * 5 + 4 * (slots & 1) + rc * 16 + slots * 2;
  return (b + 255) & ~(int64_t)255;
}

cudaError_t launch_distribute(const Geom& g, int n_frames, const CellInfo* cells, const uint32_t* slots,
                              const int32_t* cell_counts, uint32_t* selected, int32_t* sel_counts, uint8_t* ovf,
                              int64_t ovf_frame_bytes, const int64_t* ovf_level_off, int32_t* ovf_counter,
                              cudaStream_t s) {
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(distribute_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemTotal);
    attr_set = true;
  }
  dim3 grid(g.L, n_frames);
  distribute_kernel<<<grid, DT, kSmemTotal, s>>>(g, cells, slots, cell_counts, selected, sel_counts, ovf,
                                                 ovf_frame_bytes, ovf_level_off, ovf_counter);
  return cudaGetLastError();
}

}  // namespace ss
