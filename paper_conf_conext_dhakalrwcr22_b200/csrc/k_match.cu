// k_match.cu -- S9 windowed matcher ("search local points") and S10
// brute-force matcher (DESIGN.md §3 O9, O10).
//
// WINDOW: 1-8 lanes per map-point query (fewer when there are many queries).  Keypoints are in canonical (level, ly, lx)
// order, so on each level of the gate [l-1, l] the rows with |y - v| < r (f32) form one
// contiguous run found by two binary searches on the exact predicate; the run is scanned
// with the exact |x - u| < r test, the taken mask, and a 256-bit Hamming distance
// (8 x POPC over 2 x 16-byte loads); the lanes split the run and merge their packed
// (distance << 32 | index) top-2 by shuffles, i.e. top-2 by (distance, index); ORB-SLAM's
// accept rule; a keypoint claimed by several accepted
// queries keeps the min (distance, query) (atomicMin on packed u64, then a resolve pass).
// BRUTE: the per-split partial top-2 comes from the tensor-core kernel (k_brute_tc.cu);
// match_brute_merge takes the two smallest (distance << 32 | map index) and applies the rule.
#include "match_common.cuh"

namespace ss {

namespace {


// Per frame and level: rowidx[r] = index of the first keypoint with ly >= r (r in [0, h_l]),
// from the canonical (level, ly, lx) order, and every keypoint's lx; plus the dedup claim
// table reset.
__global__ void __launch_bounds__(256) match_prepare(Geom g, int F, const ss_keypoint* __restrict__ kps,
                                                     const int32_t* __restrict__ counts, uint16_t* __restrict__ rowidx,
                                                     int index_stride, unsigned long long* __restrict__ claim,
                                                     int dedup) {
  pdl_wait();
  pdl_trigger();
  const int cap = g.kp_capacity, L = g.L;
  const int gt = blockIdx.x * blockDim.x + threadIdx.x;
  if (gt >= F * cap) return;
  if (dedup) claim[gt] = ~0ull;
  const int f = gt / cap, k = gt - f * cap;
  uint16_t* fr = rowidx + (int64_t)f * index_stride;
  rowidx_fill(g, kps + (int64_t)f * cap, counts + f * (L + 1), fr, k, fr + lx_off(g));
}

// One warp takes QW consecutive queries (QW = 32 / lanes).  A query's candidates are its gate's
// row runs (one per level, contiguous in the canonical (level, ly, lx) order); the runs are cut
// into 8-keypoint chunks aligned to the frame's u16 lx array, and the warp concatenates its QW
// queries' chunk lists (warp prefix sum) and walks them 32 chunks per round, so every lane has
// work whatever the spread of run lengths (~10x with the level and the row).  The owner of
// chunk t is the query whose list starts at the last start <= t: a warp OR of the list starts
// inside the round plus a 32-entry owner table.  A chunk is one 16-B load of eight lx values,
// each tested against the owner's column range on that level -- a superset of |x - u| < r
// (floor/ceil of (u -+ r) / scale, widened by one column, as window_rows does for the rows) --
// so only the few keypoints near the column range take the exact f32 tests |x - u| < r,
// |y - v| < r, the taken mask and the Hamming distance (the row runs span whole image rows:
// ~24 keypoints per query on c3, ~2 survive the prefilter).  Survivors are queued per warp and
// tested 32 at a time, on full warps.  A match enters the owner's top-2 by shared-memory
// atomicMin on packed (distance << 16 | index) keys (index < 65536): b1 takes min(b1, key), b2
// takes min(b2, max(old b1, key)) -- keys are distinct (the index), so b1 ends as the minimum
// and b2 as the second (the minimum is never the larger of a pair).

template <int QW>
__global__ void __launch_bounds__(256) match_window_kernel(Geom g, int F, const ss_keypoint* __restrict__ kps,
                                                           const uint8_t* __restrict__ desc,
                                                           const int32_t* __restrict__ counts,
                                                           const uint8_t* __restrict__ taken, int nq,
                                                           const ss_mp_query* __restrict__ q,
                                                           const uint8_t* __restrict__ qdesc, ss_match_cfg cfg,
                                                           unsigned long long* __restrict__ claim,
                                                           ss_match* __restrict__ out,
                                                           const uint16_t* __restrict__ rowidx, int index_stride) {
  constexpr int WPB = 8;  // warps per block
  __shared__ unsigned s_b1[WPB][QW], s_b2[WPB][QW];  // top-2 keys (distance << 16 | index)
  __shared__ unsigned s_cand[WPB][32 + 256];          // survivor queue: < 32 left + one round's
  __shared__ int4 s_rng[WPB][QW];   // (list start in the concatenation, chunks on level a, first chunk a, b)
  __shared__ int4 s_kr[WPB][QW];    // keypoint runs [ka, ea) on level a, [kb, eb) on level b
  __shared__ uint2 s_col[WPB][QW];  // column range (lo | hi << 16) on levels a, b
  __shared__ float4 s_qp[WPB][QW];  // (u, v, r, frame bits)
  __shared__ uint8_t s_own[WPB][32];  // list starting at position p of the round -> its query lane
  pdl_wait();
  pdl_trigger();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int qbase = (blockIdx.x * WPB + w) * QW;
  if (qbase >= nq) return;  // warp-uniform
  const int qi = qbase + lane;
  const bool isq = lane < QW && qi < nq;
  const int L = g.L, cap = g.kp_capacity, xo = lx_off(g);
  int n = 0, f = -1;
  if (isq) {
    const ss_mp_query Q = q[qi];
    f = Q.frame;
    s_b1[w][lane] = ~0u;
    s_b2[w][lane] = ~0u;
    int4 kr = make_int4(0, 0, 0, 0);
    uint2 col = make_uint2(0, 0);
    int n0 = 0, c0 = 0, c1 = 0;
    if (f >= 0 && f < F) {
      // gate [pred_level - 1, pred_level] clamped to the pyramid: levels a = l0 and b = l0 + 1
      const int l0 = max(Q.pred_level - 1, 0), l1 = min(Q.pred_level, L - 1);
      const uint16_t* fri = rowidx + (int64_t)f * index_stride;
      int rlo, rhi;
      if (l0 <= l1) {
        // rows that can hold |y - v| < r, widened by one row each side (f32 rounding); the exact
        // test decides, so the superset only costs a few extra candidates
        window_rows(g, l0, Q.v, Q.radius, &rlo, &rhi);
        kr.x = fri[row_off(g, l0) + rlo];
        kr.y = fri[row_off(g, l0) + rhi];
        col.x = col_range(g, l0, Q.u, Q.radius);
        if (kr.y > kr.x) {  // rhi < rlo for a radius < 0 (or NaN)
          c0 = kr.x >> 3;
          n0 = ((kr.y + 7) >> 3) - c0;
        }
      }
      n = n0;
      if (l0 + 1 <= l1) {
        window_rows(g, l0 + 1, Q.v, Q.radius, &rlo, &rhi);
        kr.z = fri[row_off(g, l0 + 1) + rlo];
        kr.w = fri[row_off(g, l0 + 1) + rhi];
        col.y = col_range(g, l0 + 1, Q.u, Q.radius);
        if (kr.w > kr.z) {
          c1 = kr.z >> 3;
          n += ((kr.w + 7) >> 3) - c1;
        }
      }
    }
    s_kr[w][lane] = kr;
    s_col[w][lane] = col;
    s_qp[w][lane] = make_float4(Q.u, Q.v, Q.radius, __int_as_float(f));
    s_rng[w][lane] = make_int4(0, n0, c0, c1);
  }
  int incl = n;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int t = __shfl_up_sync(0xFFFFFFFFu, incl, o);
    if (lane >= o) incl += t;
  }
  const int excl = incl - n, total = __shfl_sync(0xFFFFFFFFu, incl, 31);
  if (isq) s_rng[w][lane].x = excl;
  __syncwarp();
  // exact tests of one queued survivor: |x - u| < r, |y - v| < r, the taken mask, then the
  // Hamming distance into the owner's top-2 (packed distance << 16 | index, index < 65536)
  auto survivor = [&](unsigned e) {
    const int o = (int)(e >> 16), k = (int)(e & 0xFFFFu);
    const float4 qp = s_qp[w][o];
    const int64_t fk = (int64_t)__float_as_int(qp.w) * cap + k;
    const float dx = __fsub_rn(kps[fk].x, qp.x), dy = __fsub_rn(kps[fk].y, qp.y);
    if (!(fabsf(dx) < qp.z && fabsf(dy) < qp.z)) return;
    if (taken && taken[fk]) return;
    const uint4* qd = reinterpret_cast<const uint4*>(qdesc + (int64_t)(qbase + o) * SS_DESC_BYTES);
    const uint4* kd = reinterpret_cast<const uint4*>(desc + fk * SS_DESC_BYTES);
    const unsigned key = ((unsigned)hamming256(qd[0], qd[1], kd[0], kd[1]) << 16) | (unsigned)k;
    const unsigned old = atomicMin(&s_b1[w][o], key);
    atomicMin(&s_b2[w][o], old > key ? old : key);
  };
  int carry = 0, qn = 0;
  for (int base = 0; base < total; base += 32) {
    const bool st = n > 0 && excl >= base && excl < base + 32;  // lists are non-empty: distinct starts
    const unsigned M = __reduce_or_sync(0xFFFFFFFFu, st ? 1u << (excl - base) : 0u);  // list starts in the round
    if (st) s_own[w][excl - base] = (uint8_t)lane;
    __syncwarp();
    const unsigned mm = M & (0xFFFFFFFFu >> (31 - lane));
    const int o = mm ? s_own[w][31 - __clz(mm)] : carry;
    carry = M ? s_own[w][31 - __clz(M)] : carry;
    const int t = base + lane;
    unsigned cand = 0;
    int ck0 = 0, co = 0;
    if (t < total) {
      const int4 rg = s_rng[w][o];
      const int i = t - rg.x;
      const bool lb = i >= rg.y;  // chunk on level b
      const int c = lb ? rg.w + (i - rg.y) : rg.z + i;
      const int4 kr = s_kr[w][o];
      const int k0 = c * 8;
      const int kb = max(lb ? kr.z : kr.x, k0) - k0, ke = min(lb ? kr.w : kr.y, k0 + 8) - k0;  // [kb, ke) of 8
      const unsigned cr = lb ? s_col[w][o].y : s_col[w][o].x;
      const unsigned lo = cr & 0xFFFFu, span = (cr >> 16) - lo;
      const int fo = __float_as_int(s_qp[w][o].w);
      const uint4 x8 = *reinterpret_cast<const uint4*>(rowidx + (int64_t)fo * index_stride + xo + k0);
      unsigned m = 0;
      m |= ((x8.x & 0xFFFFu) - lo <= span) ? 0x01u : 0u;
      m |= ((x8.x >> 16) - lo <= span) ? 0x02u : 0u;
      m |= ((x8.y & 0xFFFFu) - lo <= span) ? 0x04u : 0u;
      m |= ((x8.y >> 16) - lo <= span) ? 0x08u : 0u;
      m |= ((x8.z & 0xFFFFu) - lo <= span) ? 0x10u : 0u;
      m |= ((x8.z >> 16) - lo <= span) ? 0x20u : 0u;
      m |= ((x8.w & 0xFFFFu) - lo <= span) ? 0x40u : 0u;
      m |= ((x8.w >> 16) - lo <= span) ? 0x80u : 0u;
      m &= (0xFFu << kb) & (0xFFu >> (8 - ke));
      cand = m;
      ck0 = k0;
      co = o;
    }
    // queue the chunk's prefilter survivors (owner << 16 | k); process them 32 at a time so
    // the exact tests run on full warps
    const int ns = __popc(cand);
    int si = ns;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int v = __shfl_up_sync(0xFFFFFFFFu, si, d);
      if (lane >= d) si += v;
    }
    int pos = qn + si - ns;
    qn += __shfl_sync(0xFFFFFFFFu, si, 31);
    while (cand) {
      const int j = __ffs(cand) - 1;
      cand &= cand - 1;
      s_cand[w][pos++] = ((unsigned)co << 16) | (unsigned)(ck0 + j);
    }
    __syncwarp();
    if (qn >= 32) {
      int done = 0;
      for (; qn - done >= 32; done += 32) survivor(s_cand[w][done + lane]);
      const int rem = qn - done;
      const unsigned e = lane < rem ? s_cand[w][done + lane] : 0u;
      __syncwarp();
      if (lane < rem) s_cand[w][lane] = e;
      qn = rem;
    }
    __syncwarp();
  }
  if (lane < qn) survivor(s_cand[w][lane]);
  __syncwarp();
  if (!isq) return;
  const unsigned b1 = s_b1[w][lane], b2 = s_b2[w][lane];
  const int d1 = b1 == ~0u ? 256 : (int)(b1 >> 16), d2 = b2 == ~0u ? 256 : (int)(b2 >> 16);
  const int k1 = b1 == ~0u ? -1 : (int)(b1 & 0xFFFFu), k2 = b2 == ~0u ? -1 : (int)(b2 & 0xFFFFu);
  bool accept = false;
  if (k1 >= 0 && d1 <= cfg.th) {
    const int lev1 = kps[(int64_t)f * cap + k1].level;
    const int lev2 = k2 >= 0 ? (int)kps[(int64_t)f * cap + k2].level : -1;
    accept = (lev1 != lev2) || (cfg.ratio_den * d1 <= cfg.ratio_num * d2);
  }
  ss_match m;
  m.idx = accept ? k1 : -1;
  m.dist = d1;
  m.dist2 = d2;
  out[qi] = m;
  if (accept && cfg.dedup)
    atomicMin(claim + (int64_t)f * cap + k1, ((unsigned long long)d1 << 32) | (unsigned)qi);
}

__global__ void __launch_bounds__(256) match_window_resolve(int nq, const ss_mp_query* __restrict__ q, int cap,
                                                            const unsigned long long* __restrict__ claim,
                                                            ss_match* __restrict__ out) {
  pdl_wait();
  pdl_trigger();
  const int qi = blockIdx.x * blockDim.x + threadIdx.x;
  if (qi >= nq) return;
  const ss_match m = out[qi];
  if (m.idx < 0) return;
  const unsigned long long mine = ((unsigned long long)m.dist << 32) | (unsigned)qi;
  if (claim[(int64_t)q[qi].frame * cap + m.idx] != mine) out[qi].idx = -1;
}

__global__ void __launch_bounds__(256) match_brute_merge(Geom g, int F, const int32_t* __restrict__ counts,
                                                         int splits, const unsigned long long* __restrict__ partial,
                                                         ss_match_cfg cfg, ss_match* __restrict__ out) {
  pdl_wait();
  pdl_trigger();
  const int gq = blockIdx.x * blockDim.x + threadIdx.x;
  const int cap = g.kp_capacity, L = g.L;
  if (gq >= F * cap) return;
  const int f = gq / cap, k = gq - f * cap;
  ss_match m;
  m.idx = -1;
  m.dist = 256;
  m.dist2 = 256;
  if (k < counts[f * (L + 1) + L]) {
    unsigned long long b1 = ~0ull, b2 = ~0ull;
    for (int s = 0; s < splits * 2; s++) {
      const unsigned long long key = partial[(int64_t)gq * splits * 2 + s];
      if (key < b1) {
        b2 = b1;
        b1 = key;
      } else if (key < b2) {
        b2 = key;
      }
    }
    const int d1 = b1 == ~0ull ? 256 : (int)(b1 >> 32);
    const int d2 = b2 == ~0ull ? 256 : (int)(b2 >> 32);
    m.dist = d1;
    m.dist2 = d2;
    if (b1 != ~0ull && d1 <= cfg.th && cfg.ratio_den * d1 < cfg.ratio_num * d2) m.idx = (int)(b1 & 0xFFFFFFFFu);
  }
  out[gq] = m;
}

// Map-sharded brute force (F4): per slot, the per-split partial top-2 of one map shard reduced
// to its two smallest (distance << 32 | (map_offset + m)); slots >= the frame's count get
// (~0, ~0).  Global indices keep the (distance, index) order of the unsharded matcher.
__global__ void __launch_bounds__(256) brute_shard_top2(Geom g, int F, const int32_t* __restrict__ counts, int splits,
                                                        const unsigned long long* __restrict__ partial, int map_offset,
                                                        unsigned long long* __restrict__ top2) {
  pdl_wait();
  pdl_trigger();
  const int gq = blockIdx.x * blockDim.x + threadIdx.x;
  const int cap = g.kp_capacity, L = g.L;
  if (gq >= F * cap) return;
  const int f = gq / cap, k = gq - f * cap;
  unsigned long long b1 = ~0ull, b2 = ~0ull;
  if (k < counts[f * (L + 1) + L]) {
    for (int s = 0; s < splits * 2; s++) {
      const unsigned long long key = partial[(int64_t)gq * splits * 2 + s];
      if (key < b1) {
        b2 = b1;
        b1 = key;
      } else if (key < b2) {
        b2 = key;
      }
    }
    if (b1 != ~0ull) b1 += (unsigned)map_offset;  // index field: m < 2^31 - offset (checked on the host)
    if (b2 != ~0ull) b2 += (unsigned)map_offset;
  }
  top2[(int64_t)gq * 2] = b1;
  top2[(int64_t)gq * 2 + 1] = b2;
}

// Merge of n_parts shard top-2 lists [part][slot][2] + the O10 accept rule.
__global__ void __launch_bounds__(256) brute_parts_merge(Geom g, int F, const int32_t* __restrict__ counts,
                                                         int n_parts, const unsigned long long* __restrict__ parts,
                                                         ss_match_cfg cfg, ss_match* __restrict__ out) {
  pdl_wait();
  pdl_trigger();
  const int gq = blockIdx.x * blockDim.x + threadIdx.x;
  const int cap = g.kp_capacity, L = g.L;
  const int64_t nslots = (int64_t)F * cap;
  if (gq >= nslots) return;
  const int f = gq / cap, k = gq - f * cap;
  ss_match m;
  m.idx = -1;
  m.dist = 256;
  m.dist2 = 256;
  if (k < counts[f * (L + 1) + L]) {
    unsigned long long b1 = ~0ull, b2 = ~0ull;
    for (int r = 0; r < n_parts; r++) {
      const unsigned long long* pr = parts + ((int64_t)r * nslots + gq) * 2;
      merge_top2(b1, b2, pr[0], pr[1]);
    }
    const int d1 = b1 == ~0ull ? 256 : (int)(b1 >> 32);
    const int d2 = b2 == ~0ull ? 256 : (int)(b2 >> 32);
    m.dist = d1;
    m.dist2 = d2;
    if (b1 != ~0ull && d1 <= cfg.th && cfg.ratio_den * d1 < cfg.ratio_num * d2) m.idx = (int)(b1 & 0xFFFFFFFFu);
  }
  out[gq] = m;
}

}  // namespace

cudaError_t launch_brute_shard_top2(const Geom& g, int n_frames, const int32_t* counts, int splits,
                                    const unsigned long long* partial, int map_offset, unsigned long long* top2,
                                    cudaStream_t s) {
  const int nslots = n_frames * g.kp_capacity;
  if (nslots <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(brute_shard_top2, dim3((nslots + 255) / 256), dim3(256), 0, s, g, n_frames, counts, splits,
                             partial, map_offset, top2);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_brute_parts_merge(const Geom& g, int n_frames, const int32_t* counts, int n_parts,
                                     const unsigned long long* parts, ss_match_cfg cfg, ss_match* out, cudaStream_t s) {
  const int nslots = n_frames * g.kp_capacity;
  if (nslots <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(brute_parts_merge, dim3((nslots + 255) / 256), dim3(256), 0, s, g, n_frames, counts,
                             n_parts, parts, cfg, out);
  return e != cudaSuccess ? e : cudaGetLastError();
}

int match_rows_per_frame(const Geom& g) { return row_off(g, g.L); }
int match_index_stride(const Geom& g) { return lx_off(g) + ((g.kp_capacity + 7) & ~7); }

cudaError_t launch_match_prepare(const Geom& g, int n_frames, const ss_keypoint* kps, const int32_t* counts,
                                 uint16_t* rowidx, unsigned long long* claim, int dedup, cudaStream_t s) {
  const int n = n_frames * g.kp_capacity;
  if (n <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(match_prepare, dim3((n + 255) / 256), dim3(256), 0, s, g, n_frames, kps, counts, rowidx,
                             match_index_stride(g), claim, dedup);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_match_window(const Geom& g, int n_frames, const ss_keypoint* kps, const uint8_t* desc,
                                const int32_t* counts, const uint8_t* taken, int n_queries, const ss_mp_query* q,
                                const uint8_t* qdesc, ss_match_cfg cfg, unsigned long long* claim, ss_match* out,
                                const uint16_t* rowidx, int lanes, cudaStream_t s) {
  if (n_queries <= 0) return cudaSuccess;
  // lanes per query: the fewest that still give 1/16 of a wave of the GPU (148 SMs x 2048
  // threads).  A query's window holds a handful of candidates (0.13 on c2), so extra lanes
  // mostly repeat the per-query work: with several ticks in flight (throughput) fewer lanes
  // win even where the kernel alone gets slower.  Measured (scripts/sweep_lanes.sh): c2 (20 k
  // queries) 1 lane 78.9k vs 8 lanes 76.0k frames/s (steady state), c1 (5 k) 2 lanes 22.9k vs
  // 8 lanes 22.1k; c3 (800 k) 8 lanes 130 us, 4: 97, 2: 83, 1: 64 per launch.
  int wg = 8;
  const int64_t want = 148LL * 2048 / 16;
  while (wg > 1 && (int64_t)n_queries * (wg / 2) >= want) wg /= 2;
  if (lanes == 1 || lanes == 2 || lanes == 4 || lanes == 8) wg = lanes;  // test hook override
  // wg lanes per query on average: 32 / wg queries per warp
  auto kern = wg == 1 ? match_window_kernel<32> : wg == 2 ? match_window_kernel<16> : wg == 4 ? match_window_kernel<8>
                                                                                          : match_window_kernel<4>;
  const int per_block = 8 * (32 / wg);
  cudaError_t e = launch_pdl(kern, dim3((unsigned)((n_queries + per_block - 1) / per_block)), dim3(256), 0, s, g,
                             n_frames, kps, desc, counts, taken, n_queries, q, qdesc, cfg, claim, out, rowidx,
                             match_index_stride(g));
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_match_resolve(const Geom& g, int n_queries, const ss_mp_query* q, const unsigned long long* claim,
                                 ss_match* out, cudaStream_t s) {
  if (n_queries <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(match_window_resolve, dim3((n_queries + 255) / 256), dim3(256), 0, s, n_queries, q,
                             g.kp_capacity, (const unsigned long long*)claim, out);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_brute_merge(const Geom& g, int n_frames, const int32_t* counts, int splits,
                               const unsigned long long* partial, ss_match_cfg cfg, ss_match* out, cudaStream_t s) {
  const int nslots = n_frames * g.kp_capacity;
  match_brute_merge<<<(nslots + 255) / 256, 256, 0, s>>>(g, n_frames, counts, splits, partial, cfg, out);
  return cudaGetLastError();
}

}  // namespace ss
