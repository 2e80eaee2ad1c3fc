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
// from the canonical (level, ly, lx) order; plus the dedup claim table reset.
__global__ void __launch_bounds__(256) match_prepare(Geom g, int F, const ss_keypoint* __restrict__ kps,
                                                     const int32_t* __restrict__ counts, uint16_t* __restrict__ rowidx,
                                                     int rows_per_frame, unsigned long long* __restrict__ claim,
                                                     int dedup) {
  pdl_wait();
  pdl_trigger();
  const int cap = g.kp_capacity, L = g.L;
  const int gt = blockIdx.x * blockDim.x + threadIdx.x;
  if (gt >= F * cap) return;
  if (dedup) claim[gt] = ~0ull;
  const int f = gt / cap, k = gt - f * cap;
  rowidx_fill(g, kps + (int64_t)f * cap, counts + f * (L + 1), rowidx + (int64_t)f * rows_per_frame, k);
}

template <int WG>  // lanes cooperating on one query
__global__ void __launch_bounds__(256) match_window_kernel(Geom g, int F, const ss_keypoint* __restrict__ kps,
                                                           const uint8_t* __restrict__ desc,
                                                           const int32_t* __restrict__ counts,
                                                           const uint8_t* __restrict__ taken, int nq,
                                                           const ss_mp_query* __restrict__ q,
                                                           const uint8_t* __restrict__ qdesc, ss_match_cfg cfg,
                                                           unsigned long long* __restrict__ claim,
                                                           ss_match* __restrict__ out,
                                                           const uint16_t* __restrict__ rowidx, int rows_per_frame) {
  pdl_wait();
  pdl_trigger();
  const int gt = blockIdx.x * blockDim.x + threadIdx.x;
  const int qi = gt / WG, sub = gt % WG;
  const unsigned gmask = ((1u << WG) - 1u) << ((threadIdx.x & 31) & ~(WG - 1));
  if (qi >= nq) return;  // whole groups exit together (WG divides 32)
  const ss_mp_query Q = q[qi];
  const int L = g.L, cap = g.kp_capacity;
  unsigned long long b1 = ~0ull, b2 = ~0ull;  // (distance << 32 | keypoint index)
  const int f = Q.frame;
  if (f >= 0 && f < F) {
    const uint4* qd = reinterpret_cast<const uint4*>(qdesc + (int64_t)qi * SS_DESC_BYTES);
    const uint4 qa = qd[0], qb = qd[1];
    const ss_keypoint* fk = kps + (int64_t)f * cap;
    const uint4* fd = reinterpret_cast<const uint4*>(desc + (int64_t)f * cap * SS_DESC_BYTES);
    const uint8_t* ft = taken ? taken + (int64_t)f * cap : nullptr;
    const float r = Q.radius, nr = -Q.radius;
    const int l0 = max(Q.pred_level - 1, 0), l1 = min(Q.pred_level, L - 1);
    (void)nr;
    const uint16_t* fri = rowidx + (int64_t)f * rows_per_frame;
    for (int l = l0; l <= l1; l++) {
      // rows that can hold |y - v| < r, widened by one row each side (f32 rounding); the exact
      // test below decides, so the superset only costs a few extra candidates
      int rlo, rhi;
      window_rows(g, l, Q.v, r, &rlo, &rhi);
      const uint16_t* ri = fri + row_off(g, l);
      const int kb = ri[rlo], ke = ri[rhi];
      for (int k = kb + sub; k < ke; k += WG) {
        const float dx = __fsub_rn(fk[k].x, Q.u), dy = __fsub_rn(fk[k].y, Q.v);
        if (!(fabsf(dx) < r && fabsf(dy) < r)) continue;
        if (ft && ft[k]) continue;
        const int d = hamming256(qa, qb, fd[2 * k], fd[2 * k + 1]);
        const unsigned long long key = ((unsigned long long)d << 32) | (unsigned)k;
        if (key < b1) {
          b2 = b1;
          b1 = key;
        } else if (key < b2) {
          b2 = key;
        }
      }
    }
  }
#pragma unroll
  for (int o = WG / 2; o > 0; o >>= 1) {
    const unsigned long long o1 = __shfl_xor_sync(gmask, b1, o), o2 = __shfl_xor_sync(gmask, b2, o);
    merge_top2(b1, b2, o1, o2);
  }
  if (sub != 0) return;
  const int d1 = b1 == ~0ull ? 256 : (int)(b1 >> 32), d2 = b2 == ~0ull ? 256 : (int)(b2 >> 32);
  const int k1 = b1 == ~0ull ? -1 : (int)(b1 & 0xFFFFFFFFu), k2 = b2 == ~0ull ? -1 : (int)(b2 & 0xFFFFFFFFu);
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

cudaError_t launch_match_prepare(const Geom& g, int n_frames, const ss_keypoint* kps, const int32_t* counts,
                                 uint16_t* rowidx, unsigned long long* claim, int dedup, cudaStream_t s) {
  const int n = n_frames * g.kp_capacity;
  if (n <= 0) return cudaSuccess;
  cudaError_t e = launch_pdl(match_prepare, dim3((n + 255) / 256), dim3(256), 0, s, g, n_frames, kps, counts, rowidx,
                             match_rows_per_frame(g), claim, dedup);
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
  auto kern = wg == 1 ? match_window_kernel<1> : wg == 2 ? match_window_kernel<2> : wg == 4 ? match_window_kernel<4>
                                                                                            : match_window_kernel<8>;
  const int64_t threads = (int64_t)n_queries * wg;
  cudaError_t e = launch_pdl(kern, dim3((unsigned)((threads + 255) / 256)), dim3(256), 0, s, g, n_frames, kps, desc,
                             counts, taken, n_queries, q, qdesc, cfg, claim, out, rowidx, match_rows_per_frame(g));
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
