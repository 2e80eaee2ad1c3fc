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
static_assert((size_t)DCAP * 4 + kUnion >= (5464 + 4096 * 2 + 1024) * 4 + 1024 * (8 + 4 + 4 + 1) + 1024,
              "dense fast-path workspace must fit in the rank + union region");

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
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

__device__ bool dense_body(const Geom& g, int l, int f, int n, const uint32_t* cand, uint32_t* key, uint8_t* ws,
                           Shared& S_, uint32_t* __restrict__ selected, int32_t* __restrict__ sel_counts,
                           int32_t* ovf_counter, uint64_t* phase_ts) {
  typedef cub::BlockScan<int, DT> Scan;
  const int tid = threadIdx.x, lane = tid & 31;
  const int N = g.N[l];
  const int nini = g.nini[l];
  int R = 0;
  while (R < 6 && nini << (2 * (R + 1)) <= DENSE_BINS) R++;
  uint32_t* cnt = reinterpret_cast<uint32_t*>(ws);          // [DENSE_TOTAL] per-depth bins
  uint32_t* best0 = cnt + DENSE_TOTAL;                        // [DENSE_BINS] depth D
  uint32_t* best1 = best0 + DENSE_BINS;                       // [DENSE_BINS] depth D + 1
  uint32_t* first = best1 + DENSE_BINS;                       // [DENSE_BINS / 4] first rank, depth D
  uint64_t* rec = reinterpret_cast<uint64_t*>(first + DENSE_BINS / 4);  // [DENSE_REC]
  int32_t* recnode = reinterpret_cast<int32_t*>(rec + DENSE_REC);
  int32_t* order = recnode + DENSE_REC;
  uint8_t* recch = reinterpret_cast<uint8_t*>(order + DENSE_REC);
  uint8_t* split = recch + DENSE_REC;                         // [DENSE_BINS / 4]
  // bins of depth r start at off(r) = nini (4^r - 1) / 3
  auto off = [&](int r) { return nini * (((1 << (2 * r)) - 1) / 3); };
  // the bins were zeroed (and S_.H / S_.G reset) at the kernel's start, before its first barrier
  SS_PHASE(3);
  // one pass over the keys in a scattered order (consecutive candidates share cells, hence
  // bins): key to depth R (+1 spare round), one increment per depth >= r_lo; the value an
  // increment returns says whether it opened a bin (S_r) or made it multi-key (E_r).  The few
  // shallow bins (depth < r_lo) are sums of their 4 children, formed afterwards.
  const int r_lo = R < 3 ? R : 3;
  {
    int nz[7] = {0, 0, 0, 0, 0, 0, 0}, mu[7] = {0, 0, 0, 0, 0, 0, 0};
    uint32_t stride = 1031u;
    while ((uint32_t)n % stride == 0u) stride += 2u;  // an odd prime-ish step coprime with n
    // only the deepest depth R takes atomics (its bins are sparse, so they rarely collide);
    // depths r_lo .. R-1 are sums of their 4 children, formed level by level afterwards
    int nzR = 0, muR = 0;
    for (int j = tid; j < n; j += DT) {
      const int i = (int)(((uint32_t)j * stride) % (uint32_t)n);  // j < 8192: no overflow
      const uint32_t k = make_key(g, l, cand[i], R + 1);
      key[i] = k;
      const uint32_t old = atomicAdd(&cnt[off(R) + (int)(k >> (26 - 2 * R))], 1u);
      nzR += old == 0u;
      muR += old == 1u;
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
        const uint32_t* ch = cnt + off(r + 1) + 4 * b;
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
#pragma unroll
    for (int r = 0; r < 7; r++) {
      if (r > R) break;
      int a = nz[r], m = mu[r];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        a += __shfl_xor_sync(0xFFFFFFFFu, a, o);
        m += __shfl_xor_sync(0xFFFFFFFFu, m, o);
      }
      if (lane == 0) S_.W[tid >> 5][r] = a | (m << 16);  // per-warp partials (a, m <= 8192)
    }
  }
  __syncthreads();
  // warp r sums depth r's 32 warp partials (no same-address shared atomics across 32 warps)
  if ((tid >> 5) <= R) {
    int s = S_.W[lane][tid >> 5];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xFFFFFFFFu, s, o);
    if (lane == 0) {
      S_.H[tid >> 5] = s & 0xFFFF;
      S_.G[tid >> 5] = s >> 16;
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
  // best0 / best1 / first / split were initialised at the kernel's start (S_.sh[1], [2] = 0 too)
  if (partial) {
    for (int i = tid; i < n; i += DT) atomicMin(&first[key[i] >> (26 - 2 * D)], (uint32_t)i);
    __syncthreads();
    // the multi-key nodes at depth D, ordered by (size desc, UL.y, UL.x, first-key rank)
    const uint32_t* cD = cnt + off(D);
    const uint32_t* cD1 = cnt + off(D + 1);
    for (int b = tid; b < szD; b += DT) {
      const uint32_t c = cD[b];
      if (c > 1u) {
        const int ch = (cD1[4 * b] > 0u) + (cD1[4 * b + 1] > 0u) + (cD1[4 * b + 2] > 0u) + (cD1[4 * b + 3] > 0u);
        int ulx, uly;
        node_ul(g, l, (uint32_t)b << (26 - 2 * D), D, ulx, uly);
        const int e = atomicAdd(&S_.sh[1], 1);
        rec[e] = ((uint64_t)(0x1FFFFF - c) << 43) | ((uint64_t)uly << 32) | ((uint64_t)ulx << 20) | (uint64_t)first[b];
        recnode[e] = b;
        recch[e] = (uint8_t)ch;
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
    // split the prefix of that order that first brings the node count to >= N: an inclusive
    // scan of (children - 1) over the sorted nodes (ne <= DENSE_REC = DT)
    {
      const int e = tid < ne ? order[tid] : 0;
      const int inc = tid < ne ? (int)recch[e] - 1 : 0;
      int ex, tot;
      Scan(S_.scan).ExclusiveSum(inc, ex, tot);
      // node t is split iff the nodes before it have not yet reached N
      if (tid < ne && S_.H[D] + ex < N) split[recnode[e]] = 1;
    }
  }
  __syncthreads();
  SS_PHASE(6);
  // best key of every final node: max score, ties -> lowest rank
  for (int i = tid; i < n; i += DT) {
    const uint32_t k = key[i];
    const uint32_t v = ((uint32_t)key_m(cand[i]) << 20) | (0xFFFFFu - (uint32_t)i);
    const int b = (int)(k >> (26 - 2 * D));
    if (partial && split[b]) atomicMax(&best1[k >> (26 - 2 * (D + 1))], v);
    else atomicMax(&best0[b], v);
  }
  __syncthreads();
  SS_PHASE(7);
  uint32_t* kept = key;  // keys are no longer needed
  const uint32_t* cD = cnt + off(D);
  for (int b = tid; b < szD; b += DT) {
    if (cD[b] == 0u) continue;
    if (partial && split[b]) {
      for (int q = 0; q < 4; q++) {
        const uint32_t v = best1[4 * b + q];
        if (v) kept[atomicAdd(&S_.sh[2], 1)] = cand[0xFFFFFu - (v & 0xFFFFFu)];
      }
    } else {
      kept[atomicAdd(&S_.sh[2], 1)] = cand[0xFFFFFu - (best0[b] & 0xFFFFFu)];
    }
  }
  __syncthreads();
  const int nk = S_.sh[2];
  const int nk_w = min(nk, g.cap[l]);
  SS_PHASE(8);
  uint32_t* sel_out = selected + (int64_t)f * g.kp_capacity + g.cap_off[l];
  // rank of each kept key = #smaller keys; 4 lanes per key each count a quarter of the list
  for (int t0 = 0; t0 < nk; t0 += DT / 4) {
    const int t = t0 + (tid >> 2), part = tid & 3;
    const bool act = t < nk;
    const uint32_t k = act ? kept[t] >> 8 : 0u;
    int pos = 0;
    if (act)
      for (int u = part; u < nk; u += 4) pos += (kept[u] >> 8) < k;
    pos += __shfl_xor_sync(0xFFFFFFFFu, pos, 1);
    pos += __shfl_xor_sync(0xFFFFFFFFu, pos, 2);
    if (act && part == 0 && pos < nk_w) sel_out[pos] = kept[t];
  }
  if (tid == 0) {
    sel_counts[f * g.L + l] = nk_w;
    if (nk > g.cap[l]) atomicAdd(ovf_counter + 1, 1);
  }
  SS_PHASE(9);
  return true;
}

__global__ void __launch_bounds__(DT, 1)
    distribute_kernel(const __grid_constant__ Geom g, const CellInfo* __restrict__ cells, const uint32_t* __restrict__ slots,
                      const int32_t* __restrict__ cell_counts, uint32_t* __restrict__ selected,
                      int32_t* __restrict__ sel_counts, uint8_t* ovf, int64_t ovf_frame_bytes,
                      const int64_t* __restrict__ ovf_level_off, int32_t* ovf_counter, int level0,
                      uint64_t* phase_base) {
  extern __shared__ __align__(16) uint8_t sm[];
  __shared__ Shared S_;
  const int l = level0 + blockIdx.x, f = blockIdx.y, tid = threadIdx.x;
  uint64_t* phase_ts = phase_base ? phase_base + ((int64_t)f * g.L + l) * 16 : nullptr;
  const int ncells = g.ncells[l];
  const int c0 = g.cell_first[l];
  int32_t* cell_off = reinterpret_cast<int32_t*>(sm);
  int32_t* cell_slot = cell_off + MAX_CELLS + 1;
  const int32_t* cc = cell_counts + (int64_t)f * g.total_cells + c0;
  // Work that does not depend on the FAST kernel runs before the dependency wait, overlapping
  // its tail: the static cell table's slot offsets and the dense path's table initialisation.
  const int cpt = (ncells + DT - 1) / DT;  // <= 5 (MAX_CELLS)
  int slot[5];
#pragma unroll
  for (int j = 0; j < 5; j++) {
    const int c = tid * cpt + j;
    slot[j] = j < cpt && c < ncells ? cells[c0 + c].slot_off : 0;
  }
  if (tid < 16) S_.H[tid] = 0;
  if (tid < 17) S_.G[tid] = 0;
  {  // the dense path's per-depth bins, zeroed here so its first phase needs no barrier of
     // its own (the region is past the candidate / key arrays; other paths overwrite it)
    int R = 0;
    while (R < 6 && g.nini[l] << (2 * (R + 1)) <= DENSE_BINS) R++;
    uint32_t* bins = reinterpret_cast<uint32_t*>(sm + kSmemCells) + 2 * DCAP;
    const int o = g.nini[l] * (((1 << (2 * (R + 1))) - 1) / 3);
    for (int i = tid; i < o; i += DT) bins[i] = 0u;
    // best0 [DENSE_BINS], best1 [DENSE_BINS], first [DENSE_BINS / 4] (= none), split bytes
    uint32_t* b0 = bins + DENSE_TOTAL;
    for (int i = tid; i < 2 * DENSE_BINS; i += DT) b0[i] = 0u;
    for (int i = tid; i < DENSE_BINS / 4; i += DT) b0[2 * DENSE_BINS + i] = 0xFFFFFFFFu;
    // split = recch + DENSE_REC, recch = order + DENSE_REC ... as laid out in dense_body
    const uint64_t* rec = reinterpret_cast<const uint64_t*>(b0 + 2 * DENSE_BINS + DENSE_BINS / 4);
    const int32_t* recnode = reinterpret_cast<const int32_t*>(rec + DENSE_REC);
    const int32_t* order = recnode + DENSE_REC;
    uint8_t* spl = const_cast<uint8_t*>(reinterpret_cast<const uint8_t*>(order + DENSE_REC)) + DENSE_REC;
    for (int i = tid; i < DENSE_BINS / 4; i += DT) spl[i] = 0;
  }
  pdl_wait();
  pdl_trigger();
  SS_PHASE(0);

  // ---- 1. candidate offsets per cell (rank order = cells row-major, then raster) ----
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
#pragma unroll
    for (int j = 0; j < 5; j++) {
      const int c = tid * cpt + j;
      if (j < cpt && c < ncells) {
        cell_off[c] = ex;
        cell_slot[c] = slot[j];
        ex += cnt[j];
      }
    }
    if (tid == 0) {
      S_.sh[0] = tot;
      S_.sh[1] = 0;  // partial-round record count
      S_.sh[2] = 0;  // kept keys
    }
    __syncthreads();
  }
  const int n = S_.sh[0];
  SS_PHASE(1);
  if (n == 0) {
    if (tid == 0) sel_counts[f * g.L + l] = 0;
    return;
  }
  if (n <= DCAP) {
    uint32_t* cand = reinterpret_cast<uint32_t*>(sm + kSmemCells);
    uint32_t* key = cand + DCAP;
    {  // gather candidates into rank order (cells row-major, raster inside a cell)
      const uint32_t* fs = slots + (int64_t)f * g.slots_per_frame;
      auto src = [&](int i) {  // slot of rank i: last cell with cell_off[c] <= i
        int lo = 0, hi = ncells - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (cell_off[mid] <= i) lo = mid; else hi = mid - 1;
        }
        return cell_slot[lo] + (i - cell_off[lo]);
      };
      for (int i = tid; i < n; i += 2 * DT) {  // two independent global loads in flight per thread
        const int i1 = i + DT;
        const uint32_t v0 = fs[src(i)];
        const uint32_t v1 = i1 < n ? fs[src(i1)] : 0u;
        cand[i] = v0;
        if (i1 < n) cand[i1] = v1;
      }
      __syncthreads();
    }
    SS_PHASE(2);
    if (dense_body(g, l, f, n, cand, key, reinterpret_cast<uint8_t*>(key + DCAP), S_, selected, sel_counts,
                   ovf_counter, phase_ts))
      return;
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

cudaError_t distribute_init() {  // ss_create, per device
  return cudaFuncSetAttribute(distribute_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemTotal);
}

cudaError_t launch_distribute(const Geom& g, int n_frames, int level0, int n_levels, const CellInfo* cells,
                              const uint32_t* slots, const int32_t* cell_counts, uint32_t* selected, int32_t* sel_counts,
                              uint8_t* ovf, int64_t ovf_frame_bytes, const int64_t* ovf_level_off, int32_t* ovf_counter,
                              uint64_t* phase_ts, cudaStream_t s) {
  if (n_levels <= 0) return cudaSuccess;
  dim3 grid(n_levels, n_frames);
  cudaError_t e = launch_pdl(distribute_kernel, grid, dim3(DT), kSmemTotal, s, g, cells, slots, cell_counts, selected,
                             sel_counts, ovf, ovf_frame_bytes, ovf_level_off, ovf_counter, level0, phase_ts);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
