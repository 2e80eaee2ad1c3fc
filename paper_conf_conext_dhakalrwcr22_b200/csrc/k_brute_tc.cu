// k_brute_tc.cu -- S10 brute-force Hamming matcher on the 5th-generation tensor cores
// (DESIGN.md §3 O10, §5 "brute_tc").
//
// The brute-force matcher is a dense binary contraction: for keypoint descriptor a and map
// descriptor b (256 bits each), with bits mapped to s8 values e = 1 - 2*bit in {+1, -1},
//     dot(a, b) = sum_i e_a[i] * e_b[i] = 256 - 2 * popcount(a ^ b),
// so Hamming(a, b) = (256 - dot) / 2 exactly (|dot| <= 256, int32 accumulation is exact).
// The dot products of 256 keypoints x 128 map descriptors are two tcgen05.mma kind::i8
// M=128 N=128 tiles (K = 256 in 8 steps of 32) accumulated in TMEM; the epilogue reads
// them back with tcgen05.ld and keeps a per-keypoint top-2 by (distance, map index) on
// packed 16-bit keys (two columns per 32-bit register, VIMNMX.U16x2), merged into a
// 64-bit (distance << 32 | index) top-2 per tile.  Output: the same per-split partial
// top-2 the merge kernel (k_match.cu) reduces, so the accept rule is unchanged.
//
// Operands are pre-expanded per call by brute_expand_kernel from the packed descriptors to
// s8 {+1,-1} in the UMMA K-major no-swizzle canonical layout (8-row x 16-byte core matrices,
// K-adjacent cores 128 B apart (LBO), 8-row groups 2048 B apart (SBO)), so one 32 KB block
// of 128 rows is one contiguous bulk copy (cp.async.bulk) into shared memory.
//
// CTA roles (384 threads, one CTA per SM: 192 KB shared, 512 TMEM columns):
//   warp 0  producer: the CTA's 256 keypoint rows once, then map tiles through a 4-stage ring
//   warp 1  MMA issuer (one thread): 2 accumulators x 8 k-steps per map tile, commit to the
//           stage's empty barrier and the TMEM buffer's full barrier
//   warp 2  TMEM allocator (512 columns = 2 buffers x 2 accumulators x 128 columns)
//   warps 4..11 epilogue: warp w reads TMEM lanes 32*(w%4).. of accumulator (w-4)/4.
#include <algorithm>
#include <cstdlib>

#include "ss_internal.h"

namespace ss {

namespace {

constexpr int TC_M = 128;                    // keypoint rows per CTA (TMEM lanes)
constexpr int TC_N = 128;                    // map rows per CTA per tile; columns per epilogue warp
constexpr int TC_NT = 256;                   // map rows per tile = MMA N (cta_group::2 pair)
constexpr int TC_K = 256;                    // descriptor bits
constexpr int TC_ROWS = 2 * TC_M;            // keypoint rows per CTA pair (MMA M = 256)
constexpr int BLK_BYTES = TC_M * TC_K;       // one expanded 128-row block: 32 KB
constexpr int STAGES = 4;
constexpr int TC_THREADS = 384;
constexpr int SMEM_A = BLK_BYTES;
constexpr int SMEM_B = STAGES * BLK_BYTES;
constexpr int SMEM_BAR = 256;
constexpr int TC_SMEM = SMEM_A + SMEM_B + SMEM_BAR;
constexpr uint32_t TMEM_COLS = 512;

// instruction descriptor: D s32 (bits 4-5 = 2), A/B signed 8-bit (bits 7-9, 10-12 = 1),
// both K-major, N >> 3 at bits 17-22, M >> 4 at bits 24-28
constexpr uint32_t IDESC = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(TC_NT >> 3) << 17) |
                           ((uint32_t)(TC_ROWS >> 4) << 24);  // M = 256, N = 256 (cta_group::2)

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// shared-memory matrix descriptor, K-major, no swizzle: start >> 4 (bits 0-13), LBO >> 4
// (16-29), SBO >> 4 (32-45), version 1 (bit 46), layout type 0 (bits 61-63)
__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr) {
  const uint64_t lo = ((saddr >> 4) & 0x3FFFu) | ((uint64_t)(128 >> 4) << 16);
  const uint64_t hi = (uint64_t)((2048 >> 4) & 0x3FFF) | (1ull << 14);
  return lo | (hi << 32);
}

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_mma2_i8(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %3, p;\n}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(IDESC), "r"(accumulate)
      : "memory");
}
// completion of the leader's MMAs, signalled on the barrier at this offset in BOTH CTAs
__device__ __forceinline__ void tc_commit2_mc(uint32_t bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(bar),
      "h"((uint16_t)3)
      : "memory");
}
__device__ __forceinline__ uint32_t mapa_shared(uint32_t addr, uint32_t cta) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(cta));
  return r;
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// arrival without a memory fence: the epilogue only reports that its TMEM reads are done
// (ordered by tcgen05.fence::before_thread_sync), no data it wrote needs publishing
__device__ __forceinline__ void mbar_arrive_remote_relaxed(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAITC_%=;\n}" ::"r"(bar),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// 32 accumulator columns of this warp's 32 lanes, the low 16 bits of adjacent columns (2i,
// 2i+1) packed into register i (tcgen05.ld .pack::16b): half the TMEM-to-register traffic
#define TC_LD16P(addr, r)                                                                                         \
  asm volatile(                                                                                                   \
      "tcgen05.ld.sync.aligned.32x32b.x16.pack::16b.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15},"  \
      " [%16];"                                                                                                   \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),           \
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])      \
      : "r"(addr))
// wait for this thread's outstanding tcgen05.ld, then pin the 16 registers after the wait (an
// empty asm that "rewrites" them, so no use of them can be scheduled above the wait)
#define TC_WAIT16(r)                                                                                               \
  do {                                                                                                             \
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");                                                \
    asm volatile("" : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]),         \
                 "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]),          \
                 "+r"(r[14]), "+r"(r[15]));                                                                        \
  } while (0)


// Expand packed descriptors (32 B per row) into s8 {+1 (bit 0), -1 (bit 1)} in the canonical
// layout above.  Output byte 16*i.. of a segment is chunk c = (i >> 3) & 15 (descriptor bits
// 16c .. 16c+15) of row 8*(i >> 7) + (i & 7), so every thread writes 16 consecutive bytes and
// eight consecutive threads one whole 128-byte core matrix.  Rows >= n_valid are zero.
__global__ void __launch_bounds__(256) brute_expand_kernel(const uint8_t* __restrict__ q, int q_valid, int64_t q_units,
                                                           int8_t* __restrict__ q_out, const uint8_t* __restrict__ m,
                                                           int m_valid, int64_t m_units, int8_t* __restrict__ m_out) {
  pdl_wait();
  pdl_trigger();
  const int64_t total = q_units + m_units;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const bool isq = i < q_units;
    const int64_t u = isq ? i : i - q_units;
    const int64_t row = ((u >> 7) << 3) | (u & 7);
    const int c = (int)((u >> 3) & 15);
    const uint8_t* src = isq ? q : m;
    const int valid = isq ? q_valid : m_valid;
    uint4 o = make_uint4(0, 0, 0, 0);
    if (row < valid) {
      const uint32_t v = *reinterpret_cast<const uint16_t*>(src + row * SS_DESC_BYTES + 2 * c);
      uint32_t w[4];
#pragma unroll
      for (int j = 0; j < 4; j++) {
        const uint32_t nib = (v >> (4 * j)) & 0xFu;
        const uint32_t t = (nib * 0x00204081u) & 0x01010101u;  // bit i of nib -> bit 8i
        // keypoints: bit 0 -> +1 (0x01), 1 -> -1 (0xFF); map rows: bit 0 -> -64 (0xC0), 1 -> +64
        // (0x40), so the accumulator is -64 * (256 - 2 * Hamming), a 16-bit value
        w[j] = isq ? t * 0xFEu + 0x01010101u : 0xC0C0C0C0u ^ (t << 7);
      }
      o = make_uint4(w[0], w[1], w[2], w[3]);
    }
    reinterpret_cast<uint4*>(isq ? q_out : m_out)[u] = o;
  }
}

// Packed keys of 32 columns (j0 + 2i, j0 + 2i + 1 in the low / high half of v[i]): the
// accumulator half is -64 * dot = 64 * (2d - 256) (16-bit two's complement), so
// 16384 + j + acc = 128 * d + j (<= 32895) comes from ONE lane-wise add (VIADD.16x2).
// Two registers at a time, the running sorted (b1, b2) of {b1, b2, ka, kb} (distinct keys) in
// five VIMNMX: m, M = min / max(ka, kb); b1' = min3(b1, ka, kb); b2' = min3(b2, max(b1, m), M).
template <bool kMasked>
__device__ __forceinline__ void top2_packed(const uint32_t* v, int j0, int valid, uint32_t& b1, uint32_t& b2) {
  uint32_t k[16];
#pragma unroll
  for (int i = 0; i < 16; i++) {
    const int j = j0 + 2 * i;
    const uint32_t c = (uint32_t)(16384 + j) | ((uint32_t)(16384 + j + 1) << 16);
    k[i] = __vadd2(c, v[i]);
    if (kMasked) {
      if (j >= valid) k[i] |= 0xFFFFu;
      if (j + 1 >= valid) k[i] |= 0xFFFF0000u;
    }
  }
#pragma unroll
  for (int i = 0; i < 16; i += 2) {
    const uint32_t m = __vminu2(k[i], k[i + 1]), M = __vmaxu2(k[i], k[i + 1]);
    const uint32_t x = __vmaxu2(b1, m);
    b1 = __vimin3_u16x2(b1, k[i], k[i + 1]);
    b2 = __vimin3_u16x2(b2, x, M);
  }
}

// grid: (2 * pairs, splits), clusters of 2 CTAs = one SM pair per (256-keypoint pair-block,
// map split).  CTA rank r holds keypoint rows [256 pair + 128 r, +128) in its shared memory
// and, per map tile of 256 rows, the 128 rows [256 t + 128 r, +128): the leader (rank 0) issues
// tcgen05.mma.cta_group::2 M=256 N=256 K=32, which reads A and B halves from both SMs and
// writes each CTA's 128 x 256 s32 block into its own TMEM (two buffers of 256 columns).  Each
// SM thus reads 8 KB of operands per 128-cycle MMA (half the shared-memory traffic per MAC of
// the 1-SM M=128 N=128 form).  Split s covers tiles [s*T/S, (s+1)*T/S) of T = ceil(n_map/256).
// Cross-CTA protocol: the peer's relay thread (warp 1) forwards the completion of its own
// operand copies to the leader's full / afull barriers; the leader's commits multicast to both
// CTAs' empty / tfull barriers; the peer's epilogue warps arrive remotely on the leader's tempty.
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(TC_THREADS, 1)
    brute_tc_kernel(const int8_t* __restrict__ qexp, const int8_t* __restrict__ mexp, int n_slots, int n_map,
                    int n_tiles, int splits, unsigned long long* __restrict__ partial) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const int pair = blockIdx.x >> 1, split = blockIdx.y;
  const int t0 = (int)((int64_t)split * n_tiles / splits), t1 = (int)((int64_t)(split + 1) * n_tiles / splits);
  const int nt = t1 - t0;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SMEM_A + SMEM_B);
  const uint32_t sa = smem_u32(smem), sb = sa + SMEM_A;
  const uint32_t bar0 = smem_u32(bars);
  // barrier k at bar0 + 8k: full[0..S), empty[S..2S), tfull[2S, 2S+1], tempty[2S+2, 2S+3], afull
  auto full = [&](int s) { return bar0 + 8u * s; };
  auto empty = [&](int s) { return bar0 + 8u * (STAGES + s); };
  auto tfull = [&](int b) { return bar0 + 8u * (2 * STAGES + b); };
  auto tempty = [&](int b) { return bar0 + 8u * (2 * STAGES + 2 + b); };
  const uint32_t afull = bar0 + 8u * (2 * STAGES + 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * STAGES + 5);
  const bool leader = rank == 0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(full(s), leader ? 2 : 1);  // leader: own copy + the peer's relayed copy
      mbar_init(empty(s), 1);
    }
    for (int b = 0; b < 2; b++) {
      mbar_init(tfull(b), 1);
      mbar_init(tempty(b), 16);  // leader's: 8 local + 8 peer epilogue warps
    }
    mbar_init(afull, leader ? 2 : 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  // the pair's cta_group::2 allocation is collective: warp 2 of BOTH CTAs issues it (the
  // leader alone hangs); both receive the same column base in their own slot
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync();  // barriers of both CTAs initialised, TMEM of both allocated
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();  // the expanded operands come from the previous kernel

  if (warp == 0) {
    if (lane == 0) {  // producer (both CTAs): own A block once, own half of every map tile
      mbar_expect_tx(afull, BLK_BYTES);
      bulk_g2s(sa, qexp + ((int64_t)pair * 2 + rank) * BLK_BYTES, BLK_BYTES, afull);
      for (int t = 0; t < nt; t++) {
        const int s = t % STAGES;
        const uint32_t ph = (uint32_t)(t / STAGES) & 1u;
        mbar_wait(empty(s), ph ^ 1u);
        mbar_expect_tx(full(s), BLK_BYTES);
        bulk_g2s(sb + s * BLK_BYTES, mexp + ((int64_t)(t0 + t) * 2 + rank) * BLK_BYTES, BLK_BYTES, full(s));
      }
      // drain: the leader's multicast commits of the last STAGES tiles arrive on this CTA's
      // empty barriers asynchronously; wait for them so no arrival can land in this shared
      // memory after the CTA has exited (where the next CTA on the SM keeps its barriers)
      for (int t = nt > STAGES ? nt - STAGES : 0; t < nt; t++) mbar_wait(empty(t % STAGES), (uint32_t)(t / STAGES) & 1u);
    }
  } else if (warp == 1) {
    if (lane == 0 && leader) {  // MMA issuer
      mbar_wait_cluster(afull, 0);
      tc_fence_after();
      for (int t = 0; t < nt; t++) {
        const int s = t % STAGES;
        const uint32_t ph = (uint32_t)(t / STAGES) & 1u;
        const int b = t & 1;
        const uint32_t bph = (uint32_t)(t >> 1) & 1u;
        mbar_wait_cluster(tempty(b), bph ^ 1u);
        mbar_wait_cluster(full(s), ph);
        tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(b * TC_NT);
#pragma unroll
        for (int k = 0; k < TC_K / 32; k++)
          tc_mma2_i8(d, umma_desc(sa + k * 256), umma_desc(sb + s * BLK_BYTES + k * 256), k > 0);
        tc_commit2_mc(empty(s));
        tc_commit2_mc(tfull(b));
      }
    } else if (lane == 0) {  // peer relay: own copies landed -> the leader's barriers
      mbar_wait(afull, 0);
      mbar_arrive_remote(mapa_shared(afull, 0));
      for (int t = 0; t < nt; t++) {
        const int s = t % STAGES;
        mbar_wait(full(s), (uint32_t)(t / STAGES) & 1u);
        mbar_arrive_remote(mapa_shared(full(s), 0));
      }
    }
  } else if (warp >= 4) {
    const int hc = (warp - 4) >> 2, quarter = warp & 3;  // column half, TMEM lane quarter
    const int row = quarter * 32 + lane;
    // running top-2 as 32-bit keys (distance << 23 | map index): map indices < 2^23 (ss_create)
    uint32_t g1 = 0xFFFFFFFFu, g2 = 0xFFFFFFFFu;
    const uint32_t tempty_leader0 = mapa_shared(tempty(0), 0), tempty_leader1 = mapa_shared(tempty(1), 0);
    for (int t = 0; t < nt; t++) {
      const int b = t & 1;
      const uint32_t bph = (uint32_t)(t >> 1) & 1u;
      mbar_wait(tfull(b), bph);
      tc_fence_after();
      const uint32_t taddr = tmem + ((uint32_t)(quarter * 32) << 16) + (uint32_t)(b * TC_NT + hc * TC_N);
      const int base = (t0 + t) * TC_NT + hc * TC_N;
      const int valid = min(TC_N, n_map - base);
      uint32_t b1 = 0xFFFFFFFFu, b2 = 0xFFFFFFFFu;
      {
        // four 32-column chunks, software-pipelined: chunk c + 1 is read out of TMEM while the
        // ALU reduces chunk c; the buffer is released as soon as its last chunk has landed
        uint32_t va[16], vb[16];
        TC_LD16P(taddr, va);
        TC_WAIT16(va);
        TC_LD16P(taddr + 32, vb);
        if (valid == TC_N) top2_packed<false>(va, 0, valid, b1, b2); else top2_packed<true>(va, 0, valid, b1, b2);
        TC_WAIT16(vb);
        TC_LD16P(taddr + 64, va);
        if (valid == TC_N) top2_packed<false>(vb, 32, valid, b1, b2); else top2_packed<true>(vb, 32, valid, b1, b2);
        TC_WAIT16(va);
        TC_LD16P(taddr + 96, vb);
        if (valid == TC_N) top2_packed<false>(va, 64, valid, b1, b2); else top2_packed<true>(va, 64, valid, b1, b2);
        TC_WAIT16(vb);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if (leader)
            mbar_arrive(tempty(b));
          else
            mbar_arrive_remote_relaxed(b ? tempty_leader1 : tempty_leader0);
        }
        if (valid == TC_N) top2_packed<false>(vb, 96, valid, b1, b2); else top2_packed<true>(vb, 96, valid, b1, b2);
      }
      // per-lane-half top-2 (16-bit 128 d + j) -> the running 32-bit top-2, branch-free
      // (keys of different columns are distinct; "none" maps to 0xFFFFFFFF)
      auto to32 = [base](uint32_t k) {
        return k == 0xFFFFu ? 0xFFFFFFFFu : (((k & 0xFF80u) << 16) | (k & 127u)) + (uint32_t)base;
      };
      const uint32_t c[4] = {to32(b1 & 0xFFFFu), to32(b2 & 0xFFFFu), to32(b1 >> 16), to32(b2 >> 16)};
#pragma unroll
      for (int i = 0; i < 4; i++) {
        const uint32_t tt = max(g1, c[i]);
        g1 = min(g1, c[i]);
        g2 = min(g2, tt);
      }
    }
    const int gq = pair * TC_ROWS + (int)rank * TC_M + row;
    if (gq < n_slots) {  // one partial per (split, column half): the merges see 2 * splits parts
      auto to64 = [](uint32_t g) {
        return g == 0xFFFFFFFFu ? ~0ull : ((unsigned long long)(g >> 23) << 32) | (g & 0x7FFFFFu);
      };
      unsigned long long* o = partial + ((int64_t)gq * 2 * splits + 2 * split + hc) * 2;
      o[0] = to64(g1);
      o[1] = to64(g2);
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();  // the peer's last MMA and remote arrivals are done before either CTA leaves
  pdl_trigger();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
  }
}

}  // namespace

int64_t brute_tc_query_bytes(int64_t n_slots) { return (n_slots + TC_ROWS - 1) / TC_ROWS * 2LL * BLK_BYTES; }
int64_t brute_tc_map_bytes(int64_t n_map) { return (n_map + TC_NT - 1) / TC_NT * 2LL * BLK_BYTES; }

int brute_tc_splits(int n_slots, int n_map, int max_splits, int n_sm) {
  const int pairs = (n_slots + TC_ROWS - 1) / TC_ROWS;
  const int tiles = (n_map + TC_NT - 1) / TC_NT;
  if (pairs <= 0 || tiles <= 0) return 1;
  // fill whole waves of one CTA per SM (two per pair-block); the first >= 90 % fill wins
  int best = 1;
  double best_eff = -1.0;
  for (int w = 1; w <= 8; w++) {
    const int s = std::max(1, std::min(std::min(w * n_sm / (2 * pairs), tiles), max_splits));
    const int ctas = 2 * pairs * s;
    const double eff = (double)ctas / ((double)n_sm * ((ctas + n_sm - 1) / n_sm));
    if (eff > best_eff + 1e-9) {
      best_eff = eff;
      best = s;
    }
    if (eff >= 0.9) break;
  }
  return best;
}

cudaError_t launch_brute_expand(int n_slots, const uint8_t* desc, int n_map, const uint8_t* map_desc, int8_t* qexp,
                                int8_t* mexp, cudaStream_t s) {
  // either part may be skipped: desc == NULL (map only: ss_brute_map_prepare) or map_desc ==
  // NULL (keypoints only: the map was prepared once)
  const bool doq = desc != nullptr && n_slots > 0, dom = map_desc != nullptr && n_map > 0;
  if (!doq && !dom) return cudaSuccess;
  const int pairs = doq ? (n_slots + TC_ROWS - 1) / TC_ROWS : 0;
  const int tiles = dom ? (n_map + TC_NT - 1) / TC_NT : 0;
  const int64_t q_units = (int64_t)pairs * TC_ROWS * 16, m_units = (int64_t)tiles * TC_NT * 16;
  const int64_t units = q_units + m_units;
  const int blocks = (int)std::min<int64_t>((units + 255) / 256, 148 * 16);
  cudaError_t e = launch_pdl(brute_expand_kernel, dim3(blocks), dim3(256), 0, s, desc, n_slots, q_units, qexp,
                             map_desc, n_map, m_units, mexp);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t brute_tc_init() {  // ss_create, per device
  return cudaFuncSetAttribute(brute_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM);
}

cudaError_t launch_brute_tc(int n_slots, int n_map, const int8_t* qexp, const int8_t* mexp, int splits,
                            unsigned long long* partial, cudaStream_t s) {
  if (n_slots <= 0 || n_map <= 0) return cudaSuccess;
  const int pairs = (n_slots + TC_ROWS - 1) / TC_ROWS;
  const int tiles = (n_map + TC_NT - 1) / TC_NT;
  cudaError_t e = launch_pdl(brute_tc_kernel, dim3(2 * pairs, splits), dim3(TC_THREADS), TC_SMEM, s, qexp, mexp, n_slots, n_map,
                 tiles, splits, partial);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
