// int_peaks.cu -- measured integer-pipe peaks of one B200 (SURVEY.md §8(d) "N16"; §9 risk 1):
// warp-instruction throughput per SM per clock of the instructions the extraction and matcher
// kernels are made of, so every ALU / DPX / POPC roofline fraction divides by a MEASURED
// number instead of a table value.
//
// Method: one kernel per instruction; every thread runs NCH independent dependency chains of
// the instruction (inline PTX, so the compiler cannot fold or substitute it) for ITERS steps.
// Grid = n_sm * BPS blocks of 512 threads (one full wave, 64 warps per SM).  Each block
// records clock64() before/after its loop; the SM's busy cycles are max(end) - min(start) over
// the blocks resident on it (%smid).  ops/clk/SM = thread-ops issued on that SM / busy cycles
// (median over SMs), which does not depend on the clock the GPU runs at.  The wall-clock
// figure (CUDA events, ops / s) is printed beside it with the SM clock it implies.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o int_peaks int_peaks.cu
// Verify the instruction in SASS: cuobjdump -sass int_peaks | grep -E 'IADD3|LOP3|PRMT|VIMNMX|IDP|POPC|IMAD'
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <vector>

#ifndef ITERS
#define ITERS 4096
#endif
#define NCH 8
#define THREADS 512
#define BPS 4

__device__ __forceinline__ unsigned smid() {
  unsigned r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
  return r;
}

// one step of each chain; `k` is a runtime value the compiler cannot see through (add / min
// read the neighbouring chain, otherwise ptxas folds consecutive steps into one IMAD / min3)
#define OP_IADD3 asm volatile("add.u32 %0, %0, %1;" : "+r"(x[c]) : "r"(x[(c + 1) % NCH]));
#define OP_LOP3 asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(x[c]) : "r"(k), "r"(k2));
#define OP_PRMT asm volatile("prmt.b32 %0, %0, %1, %2;" : "+r"(x[c]) : "r"(k), "r"(k2));
#define OP_POPC asm volatile("popc.b32 %0, %0;" : "+r"(x[c]));
#define OP_DP4A asm volatile("dp4a.u32.u32 %0, %1, %2, %0;" : "+r"(x[c]) : "r"(k), "r"(k2));
#define OP_IMAD asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(x[c]) : "r"(k), "r"(k2));
#define OP_VMIN3 x[c] = __vimin3_u16x2(x[c], k, k2);
#define OP_VMAX3 x[c] = __vimax3_u16x2(x[c], k, k2);
#define OP_VMIN2 asm volatile("min.u16x2 %0, %0, %1;" : "+r"(x[c]) : "r"(x[(c + 1) % NCH]));
#define OP_HMIN2 asm volatile("min.f16x2 %0, %0, %1;" : "+r"(x[c]) : "r"(x[(c + 1) % NCH]));
#define OP_FMIN asm volatile("min.f32 %0, %0, %1;" : "+f"(fx[c]) : "f"(fx[(c + 1) % NCH]));
#define OP_FMIN3 fx[c] = fminf(fminf(fx[c], fx[(c + 1) % NCH]), fx[(c + 2) % NCH]);
#define OP_IMIN asm volatile("min.s32 %0, %0, %1;" : "+r"(x[c]) : "r"(x[(c + 1) % NCH]));
#define OP_VADDMIN x[c] = __viaddmin_u16x2(x[c], k, x[(c + 1) % NCH]);
#define OP_SHF asm volatile("shf.r.wrap.b32 %0, %0, %1, %2;" : "+r"(x[c]) : "r"(k), "r"(k2));

#define KERNEL(NAME, OPSTMT)                                                                   \
  __global__ void __launch_bounds__(THREADS) k_##NAME(uint32_t k, uint32_t k2, uint32_t* sink, \
                                                       unsigned long long* t0, unsigned long long* t1, \
                                                       unsigned* sm) {                          \
    uint32_t x[NCH];                                                                           \
    float fx[NCH];                                                                             \
    _Pragma("unroll") for (int c = 0; c < NCH; c++) x[c] = threadIdx.x * 7 + c;                 \
    _Pragma("unroll") for (int c = 0; c < NCH; c++) fx[c] = (float)(threadIdx.x * 7 + c);       \
    __syncthreads();                                                                           \
    unsigned long long a = clock64();                                                          \
    for (int it = 0; it < ITERS; it++) {                                                       \
      _Pragma("unroll") for (int c = 0; c < NCH; c++) { OPSTMT }                               \
    }                                                                                          \
    __syncthreads();                                                                           \
    unsigned long long b = clock64();                                                          \
    uint32_t s = 0;                                                                            \
    _Pragma("unroll") for (int c = 0; c < NCH; c++) s ^= x[c] ^ __float_as_uint(fx[c]);        \
    if (s == 0xDEADBEEFu) sink[0] = s;                                                         \
    if (threadIdx.x == 0) {                                                                    \
      t0[blockIdx.x] = a;                                                                      \
      t1[blockIdx.x] = b;                                                                      \
      sm[blockIdx.x] = smid();                                                                 \
    }                                                                                          \
  }

KERNEL(iadd3, OP_IADD3)
KERNEL(lop3, OP_LOP3)
KERNEL(prmt, OP_PRMT)
KERNEL(shf, OP_SHF)
KERNEL(popc, OP_POPC)
KERNEL(dp4a, OP_DP4A)
KERNEL(imad, OP_IMAD)
KERNEL(vimin3_u16x2, OP_VMIN3)
KERNEL(vimax3_u16x2, OP_VMAX3)
KERNEL(vminu2, OP_VMIN2)
KERNEL(hmin2, OP_HMIN2)
KERNEL(fmin, OP_FMIN)
KERNEL(fmin3, OP_FMIN3)
KERNEL(imin, OP_IMIN)
KERNEL(viaddmin_u16x2, OP_VADDMIN)

typedef void (*kfn)(uint32_t, uint32_t, uint32_t*, unsigned long long*, unsigned long long*, unsigned*);

int main() {
  int n_sm = 0, clk_khz = 0;
  cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, 0);
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  cudaDeviceProp prop;
  cudaGetDeviceProperties(&prop, 0);
  const int blocks = n_sm * BPS;
  uint32_t* sink;
  unsigned long long *t0, *t1;
  unsigned* sm;
  cudaMalloc(&sink, 4);
  cudaMalloc(&t0, 8 * blocks);
  cudaMalloc(&t1, 8 * blocks);
  cudaMalloc(&sm, 4 * blocks);
  struct {
    const char* name;
    const char* sass;
    kfn f;
  } ks[] = {{"iadd3", "IADD3+IMAD.IADD", k_iadd3},          {"lop3", "LOP3", k_lop3},
            {"prmt", "PRMT", k_prmt},             {"shf", "SHF", k_shf},
            {"popc", "POPC", k_popc},             {"dp4a", "IDP.4A", k_dp4a},
            {"imad", "IMAD", k_imad},             {"vimin3_u16x2", "VIMNMX3.U16x2", k_vimin3_u16x2},
            {"vimax3_u16x2", "VIMNMX3.U16x2", k_vimax3_u16x2}, {"vminu2", "VIMNMX.U16x2", k_vminu2},
            {"hmin2", "HMNMX2", k_hmin2},         {"fmin", "FMNMX", k_fmin},
            {"fmin3", "FMNMX3", k_fmin3},         {"imin", "IMNMX", k_imin},
            {"viaddmin_u16x2", "VIADDMNMX.U16x2", k_viaddmin_u16x2}};
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  printf("{\"gpu\": \"%s\", \"n_sm\": %d, \"clock_rate_khz\": %d, \"threads_per_block\": %d, \"blocks_per_sm\": %d, "
         "\"chains\": %d, \"iters\": %d, \"results\": [\n",
         prop.name, n_sm, clk_khz, THREADS, BPS, NCH, ITERS);
  const int nk = sizeof(ks) / sizeof(ks[0]);
  for (int i = 0; i < nk; i++) {
    for (int rep = 0; rep < 2; rep++) ks[i].f<<<blocks, THREADS>>>(3u, 0x01020304u, sink, t0, t1, sm);  // warm
    cudaEventRecord(e0);
    ks[i].f<<<blocks, THREADS>>>(3u, 0x01020304u, sink, t0, t1, sm);
    cudaEventRecord(e1);
    cudaError_t err = cudaEventSynchronize(e1);
    if (err != cudaSuccess) {
      fprintf(stderr, "%s: %s\n", ks[i].name, cudaGetErrorString(err));
      return 1;
    }
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    std::vector<unsigned long long> a(blocks), b(blocks);
    std::vector<unsigned> s(blocks);
    cudaMemcpy(a.data(), t0, 8 * blocks, cudaMemcpyDeviceToHost);
    cudaMemcpy(b.data(), t1, 8 * blocks, cudaMemcpyDeviceToHost);
    cudaMemcpy(s.data(), sm, 4 * blocks, cudaMemcpyDeviceToHost);
    // per SM: blocks it ran and its busy cycles
    std::vector<unsigned long long> lo(1024, ~0ull), hi(1024, 0);
    std::vector<int> nb(1024, 0);
    for (int j = 0; j < blocks; j++) {
      lo[s[j]] = std::min(lo[s[j]], a[j]);
      hi[s[j]] = std::max(hi[s[j]], b[j]);
      nb[s[j]]++;
    }
    std::vector<double> per;
    for (int q = 0; q < 1024; q++)
      if (nb[q] > 0) per.push_back((double)nb[q] * THREADS * NCH * ITERS / (double)(hi[q] - lo[q]));
    std::sort(per.begin(), per.end());
    const double med = per[per.size() / 2];
    const double total_ops = (double)blocks * THREADS * NCH * ITERS;
    const double tops = total_ops / (ms * 1e-3) / 1e12;
    // the SM clock implied by the two: ops/s / (ops/clk/SM * n_sm)
    const double implied_mhz = total_ops / (ms * 1e-3) / (med * n_sm) / 1e6;
    printf("  {\"op\": \"%s\", \"sass\": \"%s\", \"thread_ops_per_clk_per_sm\": %.2f, \"warp_inst_per_clk_per_sm\": %.3f, "
           "\"tops_wall\": %.3f, \"ms\": %.4f, \"implied_sm_mhz\": %.0f, \"sms_seen\": %zu}%s\n",
           ks[i].name, ks[i].sass, med, med / 32.0, tops, ms, implied_mhz, per.size(), i + 1 < nk ? "," : "");
  }
  printf("]}\n");
  return 0;
}
