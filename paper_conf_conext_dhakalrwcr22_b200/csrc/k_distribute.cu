// k_distribute.cu -- S4: per-(frame, level) quadtree keypoint distribution
// (ORB-SLAM DistributeOctTree reading, DESIGN.md §3 O4), ONE launch for all levels, one
// 1024-thread CTA per (level, frame), round-synchronous reformulation:
//
//  * Each candidate's quadtree path is a function of its position only: the root is
//    trunc(f32 kx / hX) and at every round the child is chosen against the node's ceil
//    half-split; the x decisions depend on kx alone and the y decisions on ky alone, so the
//    13-round key (key = root << 26 | path of 2-bit quadrant codes) is X[kx] | Y[ky] from two
//    per-level tables built once by make_key (distribute_tables_kernel, at ss_create).
//  * Dense fast path (dense_body, the usual case): the depth-r node of a key is the dense
//    index key >> (26 - 2r), so per-depth node counts are shared-memory histograms -- S_r and
//    E_r below without any sort; the kept keys are ordered by row buckets.
//  * Sort fallback (a stop rule needs a depth beyond the dense table, or > 8192 candidates):
//    the keys radix-sorted once (stable, CUB, in shared memory); every depth-r node is then a
//    contiguous run of keys sharing an r-prefix, and:
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
// never truncated).  tests/test_quadtree_reformulation.py is a CPU model of this kernel.
#include <cub/block/block_radix_sort.cuh>
#include <cub/block/block_scan.cuh>

#include "ss_internal.h"

namespace ss {

namespace {

constexpr int DT = 1024;
constexpr int DCAP = DT * 8;
constexpr int MAX_CELLS = 4608;
constexpr int REC_CAP_SMEM = DCAP / 2;

typedef cub::BlockRadixSort<uint32_t, DT, 2, uint32_t> BRS2;
typedef cub::BlockRadixSort<uint32_t, DT, 4, uint32_t> BRS4;
typedef cub::BlockRadixSort<uint32_t, DT, 8, uint32_t> BRS8;
typedef cub::BlockScan<int, DT> BScan;

constexpr size_t cmax(size_t a, size_t b) { return a > b ? a : b; }
constexpr size_t kSmemCells = ((size_t)(MAX_CELLS + 1) * 4 * 2 + 127) & ~(size_t)127;  // offsets + slot offsets
constexpr size_t kSmemArrays = (size_t)DCAP * 12;                // cand, key, rank
constexpr size_t kUnionPost = (size_t)DCAP * 2 + (size_t)REC_CAP_SMEM * 16;
constexpr size_t kUnion = cmax(cmax(sizeof(BRS8::TempStorage), sizeof(BRS4::TempStorage)),
                               cmax(sizeof(BRS2::TempStorage), kUnionPost));
constexpr size_t kSmemTotal = kSmemCells + kSmemArrays + kUnion;
static_assert(kSmemTotal <= 220 * 1024, "distribution smem budget");
constexpr int kRowsMax = 2048;  // level rows (ss_create: H <= 2048)
constexpr int kTabMax = 2048;   // quadtree key-table entries per axis (qw + 1, qh + 1 <= 2017)
// dense fast-path workspace (dense_body): per-depth bins, best0 / best1 / first, the partial
// round's records, the canonical-order row counts / cursors and the key tables
constexpr size_t kDenseWs = (size_t)(5464 + 4096 * 2 + 1024) * 4 + 1024 * (8 + 4 + 4 + 1) + 1024 +
                            (size_t)kRowsMax * 8 + (size_t)kTabMax * 8;
static_assert((size_t)DCAP * 4 + kUnion >= kDenseWs, "dense fast-path workspace must fit in the rank + union region");

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Where the CTA lets the dependent grid (describe) launch: at phase SS_DIST_TRIGGER of the
// dense path (0 = right after the dependency wait; -1 = only at exit).  Describe's ~1000 CTAs
// become resident as soon as every distribution CTA has triggered and then wait, holding their
// shared memory, for the whole distribution -- SM space other ticks in flight could use.
#ifndef SS_DIST_TRIGGER
#define SS_DIST_TRIGGER 8
#endif
#define DIST_TRIGGER_AT(k)                  \
  do {                                      \
    if (SS_DIST_TRIGGER == (k)) pdl_trigger(); \
  } while (0)
// phase timestamps of one (frame, level) CTA (debug hook ss_debug_phase_times), thread 0 only
#define SS_PHASE(i)                                  \
  do {                                               \
    if (phase_ts && threadIdx.x == 0) phase_ts[i] = gtimer(); \
  } while (0)

struct Shared {
  BScan::TempStorage scan;
  int sh[8];
  int H[16], G[17], S[15], E[15];
  int W[DT / 32][8];  // dense path: per-warp packed (non-empty, multi-key) bin counts per depth
};

__device__ __forceinline__ void root_geom(const Geom& g, int l, int ri, int& ulx, int& urx) {
  ulx = __float2int_rz(__fmul_rn(g.hX[l], (float)ri));
  urx = __float2int_rz(__fmul_rn(g.hX[l], (float)(ri + 1)));
}

// key = root << 26 | quadrant path; `rounds` < 13 leaves the deeper path bits zero (the dense
// path needs only depths <= R + 1)
__device__ __forceinline__ uint32_t make_key(const Geom& g, int l, uint32_t packed, int rounds = kQuadRounds) {
  const int kx = key_lx(packed) - kMinBorder, ky = key_ly(packed) - kMinBorder;
  int ri = __float2int_rz(__fdiv_rn((float)kx, g.hX[l]));
  ri = min(ri, g.nini[l] - 1);
  int ulx, urx;
  root_geom(g, l, ri, ulx, urx);
  int uly = 0, bly = g.qh[l];
  uint32_t path = 0;
  for (int r = 0; r < rounds; r++) {
    const int hx = (urx - ulx + 1) >> 1, hy = (bly - uly + 1) >> 1;  // ceil(w/2), w >= 0
    const int right = kx >= ulx + hx, down = ky >= uly + hy;
    path = (path << 2) | (uint32_t)(down * 2 + right);
    if (right) ulx += hx; else urx = ulx + hx;
    if (down) uly += hy; else bly = uly + hy;
  }
  return ((uint32_t)ri << 26) | (path << (2 * (kQuadRounds - rounds)));
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
  if (x >> 26) return 0;  // different roots
  if (x == 0) return 14;  // never separated (cannot happen for distinct pixels)
  return ((__clz((int)x) - 6) >> 1) + 1;
}

// warp-aggregated shared-memory histogram increment (bin < 0: no-op); whole warp calls
__device__ __forceinline__ void hist_add(int* hist, int bin) {
  const unsigned act = __ballot_sync(0xFFFFFFFFu, bin >= 0);
  if (bin >= 0) {
    const unsigned peers = __match_any_sync(act, bin);
    if ((int)(threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&hist[bin], __popc(peers));
  }
}

// Stable LSD split sort of (k, v) on bits [b0, b1), ping-ponging with (k2, v2); on return
// (k, v) name the sorted buffers.  Used only for levels that overflow shared memory.
__device__ void split_sort_global(uint32_t*& k, uint32_t*& v, uint32_t*& k2, uint32_t*& v2, int n, int b0, int b1,
                                  BScan::TempStorage& tmp) {
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

template <int ITEMS, typename BRS>
__device__ __forceinline__ void block_sort(const Geom& g, int l, const uint32_t* cand, uint32_t* key, uint32_t* rank,
                                           int n, int end_bit, void* tmp) {
  uint32_t kk[ITEMS], vv[ITEMS];
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    const int idx = threadIdx.x * ITEMS + i;
    kk[i] = idx < n ? make_key(g, l, cand[idx]) : 0xFFFFFFFFu;
    vv[i] = (uint32_t)idx;
  }
  BRS(*reinterpret_cast<typename BRS::TempStorage*>(tmp)).Sort(kk, vv, 0, end_bit);
  __syncthreads();
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    const int idx = threadIdx.x * ITEMS + i;
    if (idx < n) {
      key[idx] = kk[i];
      rank[idx] = vv[i];
    }
  }
}

// Everything after the cell-offset scan.  SMEM selects shared-memory arrays (compile-time,
// so the compiler emits LDS/STS) or the global overflow scratch.
template <bool SMEM>
__device__ __forceinline__ void distribute_body(const Geom& g, int l, int f, int n, uint8_t* sm, Shared& S_,
                                                const int32_t* cell_off, const int32_t* cell_slot,
                                                const uint32_t* __restrict__ slots, uint32_t* __restrict__ selected,
                                                int32_t* __restrict__ sel_counts, uint8_t* ovf_base,
                                                int32_t* ovf_counter, bool gathered) {
  const int tid = threadIdx.x;
  const int ncells = g.ncells[l];
  const int N = g.N[l];
  uint32_t *cand, *key, *rank, *key2 = nullptr, *rank2 = nullptr;
  uint8_t *dd, *splitf;
  uint64_t* rec;
  int32_t *rec_head, *order;
  void* sort_tmp = nullptr;
  if (SMEM) {
    uint8_t* p = sm + kSmemCells;
    cand = reinterpret_cast<uint32_t*>(p);
    key = cand + DCAP;
    rank = key + DCAP;
    uint8_t* u = reinterpret_cast<uint8_t*>(rank + DCAP);
    sort_tmp = u;
    rec = reinterpret_cast<uint64_t*>(u);
    rec_head = reinterpret_cast<int32_t*>(rec + REC_CAP_SMEM);
    order = rec_head + REC_CAP_SMEM;
    dd = reinterpret_cast<uint8_t*>(order + REC_CAP_SMEM);
    splitf = dd + DCAP;
  } else {
    const int64_t cap = g.level_slots[l];
    const int64_t rc = cap / 2 + 1;
    cand = reinterpret_cast<uint32_t*>(ovf_base);
    key = cand + cap;
    rank = key + cap;
    key2 = rank + cap;
    rank2 = key2 + cap;
    rec = reinterpret_cast<uint64_t*>(rank2 + cap + (cap & 1));
    rec_head = reinterpret_cast<int32_t*>(rec + rc);
    order = rec_head + rc;
    dd = reinterpret_cast<uint8_t*>(order + rc);
    splitf = dd + cap;
    if (tid == 0) atomicAdd(ovf_counter, 1);
  }

  // ---- 2. gather candidates into rank order (cells row-major, raster inside a cell) ----
  if (!gathered) {
    const uint32_t* fs = slots + (int64_t)f * g.slots_per_frame;
    for (int i = tid; i < n; i += DT) {
      int lo = 0, hi = ncells - 1;  // last cell with cell_off[c] <= i
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (cell_off[mid] <= i) lo = mid; else hi = mid - 1;
      }
      cand[i] = fs[cell_slot[lo] + (i - cell_off[lo])];
    }
    __syncthreads();
  }

  // ---- 3. quadtree keys + stable sort by key (value = rank) ----
  const int end_bit = 26 + (32 - __clz(max(g.nini[l] - 1, 1)));
  if (SMEM) {
    if (n <= DT * 2) block_sort<2, BRS2>(g, l, cand, key, rank, n, end_bit, sort_tmp);
    else if (n <= DT * 4) block_sort<4, BRS4>(g, l, cand, key, rank, n, end_bit, sort_tmp);
    else block_sort<8, BRS8>(g, l, cand, key, rank, n, end_bit, sort_tmp);
    __syncthreads();
  } else {
    for (int i = tid; i < n; i += DT) {
      key[i] = make_key(g, l, cand[i]);
      rank[i] = (uint32_t)i;
    }
    __syncthreads();
    split_sort_global(key, rank, key2, rank2, n, 0, end_bit, S_.scan);
  }

  // ---- 4. separation rounds + histograms -> S_r, E_r for every depth ----
  for (int i = tid; i < n; i += DT) dd[i] = i ? (uint8_t)sep_round(key[i - 1], key[i]) : 0;
  __syncthreads();
  for (int base = 0; base < n; base += DT) {
    const int i = base + tid;
    int hb = -1, gb = -1;
    if (i < n) {
      const int lo = i ? (int)dd[i] : -1;
      const int hi = (i + 1 < n) ? (int)dd[i + 1] : -1;
      hb = lo;
      gb = max(lo, hi) + 1;
    }
    hist_add(S_.H, hb);
    hist_add(S_.G, gb);
  }
  __syncthreads();
  if (tid == 0) {
    int s = 1, single = S_.G[0];
    for (int r = 0; r <= 13; r++) {
      s += S_.H[r];
      single += S_.G[r + 1];
      S_.S[r] = s;
      S_.E[r] = s - single;
    }
    S_.S[14] = S_.S[13];
    S_.E[14] = S_.E[13];
    // ORB-SLAM's loop, on node counts only (phase 1 then phase 2 stop rules)
    int D = 1, partial = 0, r = 0;
    for (;;) {
      const int nx = S_.S[min(r + 1, 14)];
      if (nx >= N || nx == S_.S[r]) { D = r + 1; break; }
      if (nx + 3 * S_.E[min(r + 1, 14)] > N) {
        int d = r + 1;
        for (;;) {
          const int s2 = S_.S[min(d + 1, 14)];
          if (s2 >= N) { D = d; partial = 1; break; }
          if (s2 == S_.S[min(d, 14)]) { D = d + 1; break; }
          d++;
        }
        break;
      }
      r++;
    }
    S_.sh[3] = min(D, 14);
    S_.sh[4] = partial;
  }
  __syncthreads();
  const int D = S_.sh[3];
  const bool partial = S_.sh[4] != 0;
  const int dlim = min(D, 13);

  // ---- 5. partial phase-2 round at depth D: order the multi-key nodes, split a prefix ----
  if (partial) {
    for (int i = tid; i < n; i += DT) {
      if (i != 0 && dd[i] > D) continue;  // not a depth-D node head
      int size = 1, c = 1;
      uint32_t minrank = rank[i];
      for (int j = i + 1; j < n && dd[j] > D; j++) {
        size++;
        minrank = min(minrank, rank[j]);
        c += (dd[j] == D + 1);
      }
      splitf[i] = 0;
      if (size > 1) {
        const int e = atomicAdd(&S_.sh[1], 1);
        int ulx, uly;
        node_ul(g, l, key[i], D, ulx, uly);
        rec[e] = ((uint64_t)(0x1FFFFF - size) << 43) | ((uint64_t)uly << 32) | ((uint64_t)ulx << 20) |
                 (uint64_t)minrank;
        rec_head[e] = i;
        splitf[i] = (uint8_t)c;
      }
    }
    __syncthreads();
    const int ne = S_.sh[1];
    for (int e = tid; e < ne; e += DT) {
      const uint64_t k = rec[e];
      int pos = 0;
      for (int e2 = 0; e2 < ne; e2++) pos += rec[e2] < k;
      order[pos] = e;
    }
    __syncthreads();
    if (tid == 0) {
      int acc = S_.S[D];
      for (int t = 0; t < ne && acc < N; t++) {
        const int h = rec_head[order[t]];
        acc += (splitf[h] & 0x7F) - 1;
        splitf[h] |= 0x80;
      }
    }
    __syncthreads();
  }

  // ---- 6. one key per final node: max score, ties -> lowest rank ----
  uint32_t* kept = key;  // keys are no longer needed
  __syncthreads();
  for (int i = tid; i < n; i += DT) {
    if (i != 0 && dd[i] > dlim) continue;  // not a final node head
    const bool split = partial && (splitf[i] & 0x80);
    int best_m = -1;
    uint32_t best_r = 0;
    for (int j = i; j < n && (j == i || dd[j] > dlim); j++) {
      if (j != i && split && dd[j] == D + 1) {
        const int p = atomicAdd(&S_.sh[2], 1);
        kept[p] = cand[best_r];
        best_m = -1;
      }
      const uint32_t r = rank[j];
      const int m = key_m(cand[r]);
      if (m > best_m || (m == best_m && r < best_r)) {
        best_m = m;
        best_r = r;
      }
    }
    const int p = atomicAdd(&S_.sh[2], 1);
    kept[p] = cand[best_r];
  }
  __syncthreads();
  const int nk = S_.sh[2];
  const int nk_w = min(nk, g.cap[l]);
  // ---- 7. canonical (ly, lx) order, into the frame's selected scratch ----
  uint32_t* sel_out = selected + (int64_t)f * g.kp_capacity + g.cap_off[l];
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

// Fast path for the usual case (n <= DCAP and the stop rules settle at depth <= R, R = the
// deepest level whose nIni * 4^R node grid fits a dense table): the depth-r node of a key is
// the dense index key >> (26 - 2r), so node counts per depth are shared-memory histograms
// (no sort at all); ORB-SLAM's stop rules run on S_r = #non-empty bins, E_r = #bins >= 2;
// the partial phase-2 round ranks the multi-key bins; the best key of every final node is
// an atomicMax of (score << 20 | ~rank).  Returns false (nothing written) when the rules
// need a depth beyond R -- the caller then runs the sort-based body on the same candidates.
constexpr int DENSE_BINS = 4096;      // nIni * 4^R <= DENSE_BINS
constexpr int DENSE_TOTAL = 5464;     // sum_{r<=R} nIni * 4^r <= 4/3 DENSE_BINS
constexpr int DENSE_REC = 1024;       // multi-key bins at the partial depth (<= DENSE_BINS / 4 = DT)

// The dense path's workspace (starts right after the key array; kDenseWs bytes).
struct DenseWs {
  uint32_t* cnt;      // [DENSE_TOTAL] per-depth bins; depth r starts at nini (4^r - 1) / 3
  uint32_t* best0;    // [DENSE_BINS] depth D
  uint32_t* best1;    // [DENSE_BINS] depth D + 1
  uint32_t* first;    // [DENSE_BINS / 4] first rank, depth D
  uint64_t* rec;      // [DENSE_REC]
  int32_t* recnode;   // [DENSE_REC]
  int32_t* order;     // [DENSE_REC]
  uint8_t* recch;     // [DENSE_REC]
  uint8_t* split;     // [DENSE_BINS / 4]
  uint32_t* rowcnt;   // [kRowsMax] kept keys per level row
  uint32_t* rowpos;   // [kRowsMax] row start, then the row's scatter cursor
  uint32_t* tabx;     // [kTabMax] quadtree key table, x part
  uint32_t* taby;     // [kTabMax] ... y part
  __device__ explicit DenseWs(uint8_t* ws) {
    cnt = reinterpret_cast<uint32_t*>(ws);
    best0 = cnt + DENSE_TOTAL;
    best1 = best0 + DENSE_BINS;
    first = best1 + DENSE_BINS;
    rec = reinterpret_cast<uint64_t*>(first + DENSE_BINS / 4);
    recnode = reinterpret_cast<int32_t*>(rec + DENSE_REC);
    order = recnode + DENSE_REC;
    recch = reinterpret_cast<uint8_t*>(order + DENSE_REC);
    split = recch + DENSE_REC;
    rowcnt = reinterpret_cast<uint32_t*>(split + DENSE_BINS / 4);
    rowpos = rowcnt + kRowsMax;
    tabx = rowpos + kRowsMax;
    taby = tabx + kTabMax;
  }
};

__device__ bool dense_body(const Geom& g, int l, int f, int n, uint32_t* cand, uint32_t* key, uint8_t* ws_bytes,
                           Shared& S_, uint32_t* __restrict__ selected, int32_t* __restrict__ sel_counts,
                           int32_t* ovf_counter, uint64_t* phase_ts) {
  typedef cub::BlockScan<int, DT> Scan;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int N = g.N[l];
  const int nini = g.nini[l];
  const int R = g.dense_r[l];
  const DenseWs w(ws_bytes);
  uint32_t* cnt = w.cnt;
  // bins of depth r start at off(r) = nini (4^r - 1) / 3
  auto off = [&](int r) { return nini * (((1 << (2 * r)) - 1) / 3); };
  // the bins, rows and tables were set up at the kernel's start, before its first barrier
  SS_PHASE(3);
  // one pass over the keys: key = X[kx] | Y[ky] (two table reads), one increment at depth R;
  // the value an increment returns says whether it opened a bin (S_R) or made it multi-key
  // (E_R).  Lane j of a warp takes candidate j * P + w (P odd: conflict-free shared reads),
  // so the lanes of one atomic are spread over the level instead of sharing a cell's bins.
  // Depths r_lo .. R-1 are sums of their 4 children, formed level by level afterwards, and
  // the few shallow bins (depth < r_lo) by warp 0.
  const int r_lo = R < 3 ? R : 3;
  {
    int nz[7] = {0, 0, 0, 0, 0, 0, 0}, mu[7] = {0, 0, 0, 0, 0, 0, 0};
    const int P = ((n + 31) >> 5) | 1;
    const int offR = off(R), shR = 26 - 2 * R;
    int nzR = 0, muR = 0;
    for (int wi = warp; wi < P; wi += DT / 32) {
      const int i = lane * P + wi;
      if (i < n) {
        const uint32_t c = cand[i];
        const uint32_t k = w.tabx[key_lx(c) - kMinBorder] | w.taby[key_ly(c) - kMinBorder];
        key[i] = k;
        const uint32_t old = atomicAdd(&cnt[offR + (int)(k >> shR)], 1u);
        nzR += old == 0u;
        muR += old == 1u;
      }
    }
#pragma unroll
    for (int r = 0; r < 7; r++)
      if (r == R) {
        nz[r] = nzR;
        mu[r] = muR;
      }
    __syncthreads();
#pragma unroll
    for (int r = 5; r >= 0; r--) {  // depths R-1 .. r_lo, block-parallel
      if (r >= R || r < r_lo) continue;
      const int sz = nini << (2 * r);
      for (int b = tid; b < sz; b += DT) {
        const uint32_t* ch = cnt + off(r + 1) + 4 * b;  // off(r) is not 16-B aligned for every nini
        const uint32_t c = ch[0] + ch[1] + ch[2] + ch[3];
        cnt[off(r) + b] = c;
        nz[r] += c > 0u;
        mu[r] += c > 1u;
      }
      __syncthreads();
    }
    // the few shallow bins (nini * (1 + 4 + 16)) by warp 0 alone, depth by depth with warp
    // syncs instead of three block barriers; the barrier after the partials orders them
    if (tid < 32) {
#pragma unroll
      for (int r = 2; r >= 0; r--) {  // r < r_lo <= 3; compile-time r keeps nz / mu in registers
        if (r >= r_lo) continue;
        const int sz = nini << (2 * r);
        for (int b = lane; b < sz; b += 32) {
          const uint32_t* ch = cnt + off(r + 1) + 4 * b;
          const uint32_t c = ch[0] + ch[1] + ch[2] + ch[3];
          cnt[off(r) + b] = c;
          nz[r] += c > 0u;
          mu[r] += c > 1u;
        }
        __syncwarp();
      }
    }
    // per-warp partials, one warp reduction (REDUX) per depth of the packed (a | m << 16)
#pragma unroll
    for (int r = 0; r < 7; r++) {
      if (r > R) break;
      const unsigned s = __reduce_add_sync(0xFFFFFFFFu, (unsigned)(nz[r] | (mu[r] << 16)));  // a, m <= 8192
      if (lane == 0) S_.W[warp][r] = (int)s;
    }
  }
  __syncthreads();
  // warp r sums depth r's 32 warp partials (no same-address shared atomics across 32 warps)
  if (warp <= R) {
    const unsigned s = __reduce_add_sync(0xFFFFFFFFu, (unsigned)S_.W[lane][warp]);
    if (lane == 0) {
      S_.H[warp] = (int)(s & 0xFFFFu);
      S_.G[warp] = (int)(s >> 16);
    }
  }
  __syncthreads();
  SS_PHASE(4);
  // ORB-SLAM's loop on node counts (as in the sort path); -1 = a depth > R is needed.  Every
  // thread evaluates it (a handful of shared reads) instead of thread 0 + a barrier.
  int D = -1, partial_i = 0;
  {
    int r = 0;
    for (;;) {
      if (r + 1 > R) break;
      const int nx = S_.H[r + 1];
      if (nx >= N || nx == S_.H[r]) { D = r + 1; break; }
      if (nx + 3 * S_.G[r + 1] > N) {
        int d = r + 1;
        for (;;) {
          if (d + 1 > R) { d = -1; break; }
          const int s2 = S_.H[d + 1];
          if (s2 >= N) { partial_i = 1; break; }
          if (s2 == S_.H[d]) { d = d + 1; break; }
          d++;
        }
        D = d;
        break;
      }
      r++;
    }
  }
  SS_PHASE(5);
  if (D < 0) return false;
  const bool partial = partial_i != 0;
  const int szD = nini << (2 * D);
  const int shD = 26 - 2 * D;
  // best0 / best1 / first / split were initialised at the kernel's start (S_.sh[1], [2] = 0 too)
  if (partial) {
    for (int i = tid; i < n; i += DT) atomicMin(&w.first[key[i] >> shD], (uint32_t)i);
    __syncthreads();
    // the multi-key nodes at depth D, ordered by (size desc, UL.y, UL.x, first-key rank)
    const uint32_t* cD = cnt + off(D);
    const uint32_t* cD1 = cnt + off(D + 1);
    for (int b = tid; b < szD; b += DT) {
      const uint32_t c = cD[b];
      if (c > 1u) {
        const uint32_t* q = cD1 + 4 * b;
        const int ch = (q[0] > 0u) + (q[1] > 0u) + (q[2] > 0u) + (q[3] > 0u);
        int ulx, uly;
        node_ul(g, l, (uint32_t)b << shD, D, ulx, uly);
        const int e = atomicAdd(&S_.sh[1], 1);
        w.rec[e] = ((uint64_t)(0x1FFFFF - c) << 43) | ((uint64_t)uly << 32) | ((uint64_t)ulx << 20) | (uint64_t)w.first[b];
        w.recnode[e] = b;
        w.recch[e] = (uint8_t)ch;
      }
    }
    __syncthreads();
    const int ne = S_.sh[1];
    {  // rank = #smaller records; G = DT / ne rounded down to a power of two (<= 32) lanes
       // per record, each counting a 1/G share of the list (shuffle-summed)
      int G = 1;
      while (G < 32 && 2 * G * ne <= DT) G *= 2;
      const int part = tid & (G - 1);
      for (int e0 = 0; e0 < ne; e0 += DT / G) {
        const int e = e0 + tid / G;
        const bool act = e < ne;
        const uint64_t k = act ? w.rec[e] : 0ull;
        int pos = 0;
        if (act)
          for (int e2 = part; e2 < ne; e2 += G) pos += w.rec[e2] < k;
        for (int o = 1; o < G; o <<= 1) pos += __shfl_xor_sync(0xFFFFFFFFu, pos, o);
        if (act && part == 0) w.order[pos] = e;
      }
    }
    __syncthreads();
    // split the prefix of that order that first brings the node count to >= N: an inclusive
    // scan of (children - 1) over the sorted nodes (ne <= DENSE_REC = DT)
    {
      const int e = tid < ne ? w.order[tid] : 0;
      const int inc = tid < ne ? (int)w.recch[e] - 1 : 0;
      int ex, tot;
      Scan(S_.scan).ExclusiveSum(inc, ex, tot);
      // node t is split iff the nodes before it have not yet reached N
      if (tid < ne && S_.H[D] + ex < N) w.split[w.recnode[e]] = 1;
    }
  }
  __syncthreads();
  SS_PHASE(6);
  DIST_TRIGGER_AT(6);
  // best key of every final node: max score, ties -> lowest rank
  for (int i = tid; i < n; i += DT) {
    const uint32_t k = key[i];
    const uint32_t v = ((uint32_t)key_m(cand[i]) << 20) | (0xFFFFFu - (uint32_t)i);
    const int b = (int)(k >> shD);
    if (partial && w.split[b]) atomicMax(&w.best1[k >> (shD - 2)], v);
    else atomicMax(&w.best0[b], v);
  }
  __syncthreads();
  SS_PHASE(7);
  DIST_TRIGGER_AT(7);
  // kept keys (in no particular order) + their level rows' counts
  uint32_t* kept = key;  // keys are no longer needed
  {
    const uint32_t* cD = cnt + off(D);
    for (int b = tid; b < szD; b += DT) {
      if (cD[b] == 0u) continue;
      if (partial && w.split[b]) {
        const uint4 q = *reinterpret_cast<const uint4*>(w.best1 + 4 * b);  // best1: 16-B aligned
        const uint32_t v4[4] = {q.x, q.y, q.z, q.w};
#pragma unroll
        for (int j = 0; j < 4; j++)
          if (v4[j]) {
            const uint32_t c = cand[0xFFFFFu - (v4[j] & 0xFFFFFu)];
            kept[atomicAdd(&S_.sh[2], 1)] = c;
            atomicAdd(&w.rowcnt[key_ly(c)], 1u);
          }
      } else {
        const uint32_t c = cand[0xFFFFFu - (w.best0[b] & 0xFFFFFu)];
        kept[atomicAdd(&S_.sh[2], 1)] = c;
        atomicAdd(&w.rowcnt[key_ly(c)], 1u);
      }
    }
  }
  __syncthreads();
  const int nk = S_.sh[2];
  const int nk_w = min(nk, g.cap[l]);
  SS_PHASE(8);
  DIST_TRIGGER_AT(8);
  // canonical (ly, lx) order: row starts by a block scan of the row counts, keys scattered
  // into their row's bucket, then ranked by lx among the (few) keys of the same row
  {
    const int h = g.h[l];
    const int y0 = 2 * tid;
    const int a0 = y0 < h ? (int)w.rowcnt[y0] : 0, a1 = y0 + 1 < h ? (int)w.rowcnt[y0 + 1] : 0;
    int ex, tot;
    Scan(S_.scan).ExclusiveSum(a0 + a1, ex, tot);
    if (y0 < h) w.rowpos[y0] = (uint32_t)ex;
    if (y0 + 1 < h) w.rowpos[y0 + 1] = (uint32_t)(ex + a0);
  }
  __syncthreads();
  uint32_t* bucket = cand;  // candidates are no longer needed
  for (int t = tid; t < nk; t += DT) {
    const uint32_t k = kept[t];
    bucket[atomicAdd(&w.rowpos[key_ly(k)], 1u)] = k;
  }
  __syncthreads();
  uint32_t* sel_out = selected + (int64_t)f * g.kp_capacity + g.cap_off[l];
  for (int t = tid; t < nk; t += DT) {
    const uint32_t k = bucket[t];
    const int y = key_ly(k);
    const int e = (int)w.rowpos[y], s0 = e - (int)w.rowcnt[y];  // the row's bucket [s0, e)
    int pos = s0;
    for (int u = s0; u < e; u++) pos += (bucket[u] >> 8) < (k >> 8);
    if (pos < nk_w) sel_out[pos] = k;
  }
  if (tid == 0) {
    sel_counts[f * g.L + l] = nk_w;
    if (nk > g.cap[l]) atomicAdd(ovf_counter + 1, 1);
  }
  SS_PHASE(9);
  return true;
}

__global__ void __launch_bounds__(DT, 1)
    distribute_kernel(const __grid_constant__ Geom g, const CellInfo* __restrict__ cells, const uint32_t* __restrict__ qtab,
                      const uint32_t* __restrict__ slots, const int32_t* __restrict__ cell_counts,
                      uint32_t* __restrict__ selected, int32_t* __restrict__ sel_counts, uint8_t* ovf,
                      int64_t ovf_frame_bytes, const int64_t* __restrict__ ovf_level_off, int32_t* ovf_counter,
                      int level0, uint64_t* phase_base) {
  extern __shared__ __align__(16) uint8_t sm[];
  __shared__ Shared S_;
  const int l = level0 + blockIdx.x, f = blockIdx.y, tid = threadIdx.x;
  uint64_t* phase_ts = phase_base ? phase_base + ((int64_t)f * g.L + l) * 16 : nullptr;
  const int ncells = g.ncells[l];
  const int c0 = g.cell_first[l];
  int32_t* cell_off = reinterpret_cast<int32_t*>(sm);
  int32_t* cell_slot = cell_off + MAX_CELLS + 1;
  uint32_t* cand = reinterpret_cast<uint32_t*>(sm + kSmemCells);
  uint32_t* key = cand + DCAP;
  uint8_t* ws = reinterpret_cast<uint8_t*>(key + DCAP);
  const int32_t* cc = cell_counts + (int64_t)f * g.total_cells + c0;
  SS_PHASE(10);  // kernel entry
  // Work that does not depend on the FAST kernel runs before the dependency wait, overlapping
  // its tail: the static cell table's slot offsets, the key tables and the dense path's
  // table initialisation (its region is past the candidate / key arrays; other paths
  // overwrite it).
  const int cpt = (ncells + DT - 1) / DT;  // <= 5 (MAX_CELLS)
  int slot[5];
#pragma unroll
  for (int j = 0; j < 5; j++) {
    const int c = tid * cpt + j;
    slot[j] = j < cpt && c < ncells ? cells[c0 + c].slot_off : 0;
  }
  if (tid < 16) S_.H[tid] = 0;
  if (tid < 17) S_.G[tid] = 0;
  if (tid == 0) {
    S_.sh[1] = 0;  // partial-round record count
    S_.sh[2] = 0;  // kept keys
  }
  {
    const DenseWs w(ws);
    const int R = g.dense_r[l];
    const int o = g.nini[l] * (((1 << (2 * (R + 1))) - 1) / 3);
    for (int i = tid; i < o; i += DT) w.cnt[i] = 0u;
    for (int i = tid; i < 2 * DENSE_BINS; i += DT) w.best0[i] = 0u;  // best0, best1
    for (int i = tid; i < DENSE_BINS / 4; i += DT) {
      w.first[i] = 0xFFFFFFFFu;
      w.split[i] = 0;
    }
    for (int i = tid; i < g.h[l]; i += DT) w.rowcnt[i] = 0u;
    const uint32_t* qt = qtab + g.qtab_off[l];
    const int nx = g.qw[l] + 1, ny = g.qh[l] + 1;
    for (int i = tid; i < nx; i += DT) w.tabx[i] = __ldg(qt + i);
    for (int i = tid; i < ny; i += DT) w.taby[i] = __ldg(qt + nx + i);
  }
  SS_PHASE(11);  // static set-up issued
  pdl_wait();
  DIST_TRIGGER_AT(0);
  SS_PHASE(0);

  // ---- 1. candidate counts per cell, their offsets (rank order = cells row-major, then
  // raster inside a cell) and, for the usual case, the gather: every thread copies its own
  // cells' candidates (no per-candidate search for its cell) ----
  {
    int cnt[5];
    int s = 0;
#pragma unroll
    for (int j = 0; j < 5; j++) {
      const int c = tid * cpt + j;
      cnt[j] = j < cpt && c < ncells ? cc[c] : 0;
      s += cnt[j];
    }
    int ex, tot;
    BScan(S_.scan).ExclusiveSum(s, ex, tot);
    if (tot <= DCAP) {
      const uint32_t* fs = slots + (int64_t)f * g.slots_per_frame;
#pragma unroll
      for (int j = 0; j < 5; j++) {
        if (j >= cpt) break;
        const uint32_t* src = fs + slot[j];
        uint32_t* dst = cand + ex;
        const int cn = cnt[j];
        int q = 0;
        for (; q + 4 <= cn; q += 4) {  // four independent loads in flight
          const uint32_t v0 = src[q], v1 = src[q + 1], v2 = src[q + 2], v3 = src[q + 3];
          dst[q] = v0;
          dst[q + 1] = v1;
          dst[q + 2] = v2;
          dst[q + 3] = v3;
        }
        for (; q < cn; q++) dst[q] = src[q];
        ex += cn;
      }
    } else {
#pragma unroll
      for (int j = 0; j < 5; j++) {
        const int c = tid * cpt + j;
        if (j < cpt && c < ncells) {
          cell_off[c] = ex;
          cell_slot[c] = slot[j];
          ex += cnt[j];
        }
      }
    }
    if (tid == 0) S_.sh[0] = tot;
    __syncthreads();
  }
  const int n = S_.sh[0];
  SS_PHASE(1);
  if (n == 0) {
    if (tid == 0) sel_counts[f * g.L + l] = 0;
    return;
  }
  if (n <= DCAP) {
    SS_PHASE(2);
    if (dense_body(g, l, f, n, cand, key, ws, S_, selected, sel_counts, ovf_counter, phase_ts)) return;
    if (tid == 0) atomicAdd(ovf_counter + 2, 1);  // counted for the tests (ss_debug_distribution_paths)
    __syncthreads();
    if (tid < 16) S_.H[tid] = 0;
    if (tid < 17) S_.G[tid] = 0;
    if (tid == 0) {
      S_.sh[1] = 0;
      S_.sh[2] = 0;
    }
    __syncthreads();
    distribute_body<true>(g, l, f, n, sm, S_, cell_off, cell_slot, slots, selected, sel_counts, nullptr, ovf_counter,
                          true);
  } else {
    distribute_body<false>(g, l, f, n, sm, S_, cell_off, cell_slot, slots, selected, sel_counts,
                           ovf + (int64_t)f * ovf_frame_bytes + ovf_level_off[l], ovf_counter, false);
  }
}

}  // namespace

int64_t distribute_ovf_bytes(int64_t slots) {
  // cand, key, rank, key2, rank2 (u32) + rec (u64) / rec_head / order (i32) + dd, splitf (u8)
  const int64_t rc = slots / 2 + 1;
  int64_t b = slots * 4 * 5 + 4 * (slots & 1) + rc * 16 + slots * 2;
  return (b + 255) & ~(int64_t)255;
}

// Quadtree key tables: make_key's x decisions depend on kx only and its y decisions on ky
// only (the node's x interval evolves with the "right" bits alone, its y interval with the
// "down" bits), so key = X[kx] | Y[ky] with X = root << 26 | the right bits (bit 0 of every
// 2-bit quadrant code) and Y = the down bits (bit 1).  Built once per ctx by make_key itself.
__global__ void distribute_tables_kernel(const __grid_constant__ Geom g, uint32_t* qtab) {
  const int l = blockIdx.y;
  if (l >= g.L) return;
  const int nx = g.qw[l] + 1, ny = g.qh[l] + 1;
  uint32_t* t = qtab + g.qtab_off[l];
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nx + ny; i += gridDim.x * blockDim.x) {
    if (i < nx)
      t[i] = make_key(g, l, pack_key(i + kMinBorder, kMinBorder, 0)) & 0xFD555555u;  // root (bits 26+) + right bits
    else
      t[i] = make_key(g, l, pack_key(kMinBorder, i - nx + kMinBorder, 0)) & 0x02AAAAAAu;  // down bits
  }
}

cudaError_t launch_distribute_tables(const Geom& g, uint32_t* qtab, cudaStream_t s) {
  distribute_tables_kernel<<<dim3(8, g.L), 256, 0, s>>>(g, qtab);
  return cudaGetLastError();
}

cudaError_t distribute_init() {  // ss_create, per device
  cudaError_t e = carveout_from_env(distribute_kernel);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(distribute_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemTotal);
}

cudaError_t launch_distribute(const Geom& g, int n_frames, int level0, int n_levels, const CellInfo* cells,
                              const uint32_t* qtab, const uint32_t* slots, const int32_t* cell_counts, uint32_t* selected, int32_t* sel_counts,
                              uint8_t* ovf, int64_t ovf_frame_bytes, const int64_t* ovf_level_off, int32_t* ovf_counter,
                              uint64_t* phase_ts, cudaStream_t s) {
  if (n_levels <= 0) return cudaSuccess;
  dim3 grid(n_levels, n_frames);
  cudaError_t e = launch_pdl(distribute_kernel, grid, dim3(DT), kSmemTotal, s, g, cells, qtab, slots, cell_counts, selected,
                             sel_counts, ovf, ovf_frame_bytes, ovf_level_off, ovf_counter, level0, phase_ts);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
