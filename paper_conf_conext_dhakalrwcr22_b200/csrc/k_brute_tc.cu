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

constexpr int TC_M = 128;                    // keypoint rows per accumulator (TMEM lanes)
constexpr int TC_N = 128;                    // map rows per tile (TMEM columns per accumulator)
constexpr int TC_K = 256;                    // descriptor bits
constexpr int TC_ROWS = 2 * TC_M;            // keypoint rows per CTA (two accumulators)
constexpr int BLK_BYTES = TC_M * TC_K;       // one expanded 128-row block: 32 KB
constexpr int STAGES = 4;
constexpr int TC_THREADS = 384;
constexpr int SMEM_A = 2 * BLK_BYTES;
constexpr int SMEM_B = STAGES * BLK_BYTES;
constexpr int SMEM_BAR = 256;
constexpr int TC_SMEM = SMEM_A + SMEM_B + SMEM_BAR;
constexpr uint32_t TMEM_COLS = 512;

// instruction descriptor: D s32 (bits 4-5 = 2), A/B signed 8-bit (bits 7-9, 10-12 = 1),
// both K-major, N >> 3 at bits 17-22, M >> 4 at bits 24-28
constexpr uint32_t IDESC = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(TC_N >> 3) << 17) |
                           ((uint32_t)(TC_M >> 4) << 24);

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
__device__ __forceinline__ void tc_mma_i8(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(IDESC), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tc_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

#define TC_LD32(addr, r)                                                                                          \
  asm volatile(                                                                                                   \
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18," \
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"                                              \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),           \
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),     \
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),   \
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])    \
      : "r"(addr))

__device__ __forceinline__ void top2_insert(unsigned long long k, unsigned long long& b1, unsigned long long& b2) {
  if (k < b1) {
    b2 = b1;
    b1 = k;
  } else if (k < b2) {
    b2 = k;
  }
}

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
        w[j] = t * 0xFEu + 0x01010101u;                          // byte 0 -> 0x01 (+1), 1 -> 0xFF (-1)
      }
      o = make_uint4(w[0], w[1], w[2], w[3]);
    }
    reinterpret_cast<uint4*>(isq ? q_out : m_out)[u] = o;
  }
}

// Packed 16-bit key of one column: 128 * distance + column-within-half (distance <= 256,
// column < 64 => key <= 32831; 0xFFFF = "none").  From the s32 dot: 128*d + j =
// 16384 + j - 64*dot.  Two columns (j, j + 64) share one register (low / high halves);
// the low half never borrows from the high one (16384 + j - 64*dot >= 0).
template <bool kMasked>
__device__ __forceinline__ void top2_columns(const uint32_t* lo, const uint32_t* hi, int j0, int valid, uint32_t& b1,
                                             uint32_t& b2) {
#pragma unroll
  for (int i = 0; i < 32; i++) {
    const int j = j0 + i;
    const uint32_t c = (uint32_t)(16384 + j) * 0x10001u;
    uint32_t k = c - (lo[i] << 6) - (hi[i] << 22);
    if (kMasked) {
      if (j >= valid) k |= 0xFFFFu;
      if (j + 64 >= valid) k |= 0xFFFF0000u;
    }
    const uint32_t t = __vmaxu2(b1, k);
    b1 = __vminu2(b1, k);
    b2 = __vminu2(b2, t);
  }
}

// grid: (pairs = ceil(n_slots / 256), splits).  Split s covers map tiles
// [s*T/S, (s+1)*T/S) of T = ceil(n_map / 128); CTAs of one split run side by side, so its
// map tiles are read from L2 by every pair.
__global__ void __launch_bounds__(TC_THREADS, 1) brute_tc_kernel(const int8_t* __restrict__ qexp,
                                                                  const int8_t* __restrict__ mexp, int n_slots,
                                                                  int n_map, int n_tiles, int splits,
                                                                  unsigned long long* __restrict__ partial) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int pair = blockIdx.x, split = blockIdx.y;
  const int t0 = (int)((int64_t)split * n_tiles / splits), t1 = (int)((int64_t)(split + 1) * n_tiles / splits);
  const int nt = t1 - t0;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SMEM_A + SMEM_B);
  const uint32_t sa = smem_u32(smem), sb = sa + SMEM_A;
  const uint32_t bar0 = smem_u32(bars);
  // barrier k at bar0 + 8k: full[0..3], empty[4..7], tfull[8..9], tempty[10..11], a_full[12]
  auto full = [&](int s) { return bar0 + 8u * s; };
  auto empty = [&](int s) { return bar0 + 8u * (STAGES + s); };
  auto tfull = [&](int b) { return bar0 + 8u * (2 * STAGES + b); };
  auto tempty = [&](int b) { return bar0 + 8u * (2 * STAGES + 2 + b); };
  const uint32_t afull = bar0 + 8u * (2 * STAGES + 4);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * STAGES + 5);

  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; s++) {
      mbar_init(full(s), 1);
      mbar_init(empty(s), 1);
    }
    for (int b = 0; b < 2; b++) {
      mbar_init(tfull(b), 1);
      mbar_init(tempty(b), 8);  // one arrive per epilogue warp
    }
    mbar_init(afull, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();  // the expanded operands come from the previous kernel

  if (warp == 0) {
    if (lane == 0) {
      mbar_expect_tx(afull, SMEM_A);
      const int8_t* a = qexp + (int64_t)pair * SMEM_A;
      bulk_g2s(sa, a, BLK_BYTES, afull);
      bulk_g2s(sa + BLK_BYTES, a + BLK_BYTES, BLK_BYTES, afull);
      for (int t = 0; t < nt; t++) {
        const int s = t % STAGES;
        const uint32_t ph = (uint32_t)(t / STAGES) & 1u;
        mbar_wait(empty(s), ph ^ 1u);
        mbar_expect_tx(full(s), BLK_BYTES);
        bulk_g2s(sb + s * BLK_BYTES, mexp + (int64_t)(t0 + t) * BLK_BYTES, BLK_BYTES, full(s));
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      mbar_wait(afull, 0);
      tc_fence_after();
      for (int t = 0; t < nt; t++) {
        const int s = t % STAGES;
        const uint32_t ph = (uint32_t)(t / STAGES) & 1u;
        const int b = t & 1;
        const uint32_t bph = (uint32_t)(t >> 1) & 1u;
        mbar_wait(tempty(b), bph ^ 1u);
        mbar_wait(full(s), ph);
        tc_fence_after();
#pragma unroll
        for (int acc = 0; acc < 2; acc++) {
          const uint32_t d = tmem + (uint32_t)(b * 2 * TC_N + acc * TC_N);
#pragma unroll
          for (int k = 0; k < TC_K / 32; k++)
            tc_mma_i8(d, umma_desc(sa + acc * BLK_BYTES + k * 256), umma_desc(sb + s * BLK_BYTES + k * 256), k > 0);
        }
        tc_commit(empty(s));
        tc_commit(tfull(b));
      }
    }
  } else if (warp >= 4) {
    const int acc = (warp - 4) >> 2, quarter = warp & 3;
    const int row = acc * TC_M + quarter * 32 + lane;
    unsigned long long g1 = ~0ull, g2 = ~0ull;
    for (int t = 0; t < nt; t++) {
      const int b = t & 1;
      const uint32_t bph = (uint32_t)(t >> 1) & 1u;
      mbar_wait(tfull(b), bph);
      tc_fence_after();
      const uint32_t taddr = tmem + ((uint32_t)(quarter * 32) << 16) + (uint32_t)(b * 2 * TC_N + acc * TC_N);
      const int base = (t0 + t) * TC_N;
      const int valid = min(TC_N, n_map - base);
      uint32_t b1 = 0xFFFFFFFFu, b2 = 0xFFFFFFFFu;
#pragma unroll
      for (int h = 0; h < 2; h++) {
        uint32_t lo[32], hi[32];
        TC_LD32(taddr + 32 * h, lo);
        TC_LD32(taddr + 64 + 32 * h, hi);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (valid == TC_N)
          top2_columns<false>(lo, hi, 32 * h, valid, b1, b2);
        else
          top2_columns<true>(lo, hi, 32 * h, valid, b1, b2);
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty(b));
      // per-half top-2 -> the running 64-bit top-2 (distance << 32 | map index)
#pragma unroll
      for (int half = 0; half < 2; half++) {
        const uint32_t k1 = (b1 >> (16 * half)) & 0xFFFFu, k2 = (b2 >> (16 * half)) & 0xFFFFu;
        if (k1 != 0xFFFFu)
          top2_insert(((unsigned long long)(k1 >> 7) << 32) | (unsigned)(base + 64 * half + (k1 & 127)), g1, g2);
        if (k2 != 0xFFFFu)
          top2_insert(((unsigned long long)(k2 >> 7) << 32) | (unsigned)(base + 64 * half + (k2 & 127)), g1, g2);
      }
    }
    const int gq = pair * TC_ROWS + row;
    if (gq < n_slots) {
      partial[((int64_t)gq * splits + split) * 2] = g1;
      partial[((int64_t)gq * splits + split) * 2 + 1] = g2;
    }
  }
  tc_fence_before();
  __syncthreads();
  pdl_trigger();
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
  }
}

}  // namespace

int64_t brute_tc_query_bytes(int64_t n_slots) { return (n_slots + TC_ROWS - 1) / TC_ROWS * (int64_t)SMEM_A; }
int64_t brute_tc_map_bytes(int64_t n_map) { return (n_map + TC_N - 1) / TC_N * (int64_t)BLK_BYTES; }

int brute_tc_splits(int n_slots, int n_map, int max_splits, int n_sm) {
  const int pairs = (n_slots + TC_ROWS - 1) / TC_ROWS;
  const int tiles = (n_map + TC_N - 1) / TC_N;
  if (pairs <= 0 || tiles <= 0) return 1;
  // fill whole waves of one CTA per SM; the first wave count whose fill is >= 90 % wins
  int best = 1;
  double best_eff = -1.0;
  for (int w = 1; w <= 8; w++) {
    const int s = std::max(1, std::min(std::min(w * n_sm / pairs, tiles), max_splits));
    const int ctas = pairs * s;
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
  if (n_slots <= 0 || n_map <= 0) return cudaSuccess;
  const int pairs = (n_slots + TC_ROWS - 1) / TC_ROWS;
  const int tiles = (n_map + TC_N - 1) / TC_N;
  const int64_t q_units = (int64_t)pairs * TC_ROWS * 16, m_units = (int64_t)tiles * TC_N * 16;
  const int64_t units = q_units + m_units;
  const int blocks = (int)std::min<int64_t>((units + 255) / 256, 148 * 16);
  cudaError_t e = launch_pdl(brute_expand_kernel, dim3(blocks), dim3(256), 0, s, desc, n_slots, q_units, qexp,
                             map_desc, n_map, m_units, mexp);
  return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_brute_tc(int n_slots, int n_map, const int8_t* qexp, const int8_t* mexp, int splits,
                            unsigned long long* partial, cudaStream_t s) {
  if (n_slots <= 0 || n_map <= 0) return cudaSuccess;
  const int pairs = (n_slots + TC_ROWS - 1) / TC_ROWS;
  const int tiles = (n_map + TC_N - 1) / TC_N;
  cudaError_t e = cudaFuncSetAttribute(brute_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, TC_SMEM);
  if (e != cudaSuccess) return e;
  e = launch_pdl(brute_tc_kernel, dim3(pairs, splits), dim3(TC_THREADS), TC_SMEM, s, qexp, mexp, n_slots, n_map,
                 tiles, splits, partial);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace ss
