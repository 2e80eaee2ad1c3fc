// tma_probe2.cu -- which TMA tensor-map shapes load on this B200: 2-D / 3-D u8 maps with
// various box sizes, one warp, descriptor as a __grid_constant__ kernel parameter.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_probe2 tma_probe2.cu ; ./tma_probe2 CASE
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int RANK>
__global__ void probe(const __grid_constant__ CUtensorMap m, int x, int y, int f, int bytes, uint8_t* out) {
  __shared__ __align__(1024) uint8_t buf[64 * 64];
  __shared__ __align__(8) uint64_t bar;
  const int lane = threadIdx.x;
  const uint32_t b = saddr(&bar);
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
    if (RANK == 2)
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
              saddr(buf)),
          "l"(reinterpret_cast<uint64_t>(&m)), "r"(x), "r"(y), "r"(b)
          : "memory");
    else
      asm volatile(
          "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
              saddr(buf)),
          "l"(reinterpret_cast<uint64_t>(&m)), "r"(x), "r"(y), "r"(f), "r"(b)
          : "memory");
  }
  __syncwarp();
  uint32_t done = 0;
  for (int it = 0; it < 1000000 && !done; it++)
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P1;\n}"
        : "=r"(done)
        : "r"(b), "r"(0u)
        : "memory");
  for (int i = lane; i < bytes; i += 32) out[i] = buf[i];
  if (lane == 0 && !done) out[4095] = 0xEE;
}

int main(int argc, char** argv) {
  const int cs = argc > 1 ? atoi(argv[1]) : 0;
  const int W = 752, H = 480, F = 3, P = 768;
  std::vector<uint8_t> h((size_t)F * H * P);
  for (size_t i = 0; i < h.size(); i++) h[i] = (uint8_t)(i * 7 + (i >> 9));
  uint8_t *d, *o;
  cudaMalloc(&d, h.size());
  cudaMalloc(&o, 4096);
  cudaMemcpy(d, h.data(), h.size(), cudaMemcpyHostToDevice);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  // cases: 0: 2-D box 64x32 x=96 ; 1: 2-D box 64x43 x=100 ; 2: 3-D box 64x43x1 ; 3: 2-D box 16x16 ;
  //        4: 2-D box 64x32 with SWIZZLE_NONE + L2 NONE ; 5: 3-D box 64x32x1
  //        6: 2-D box 64x43 x=96 ; 7: 2-D box 64x32 x=100 ; 8: 2-D box 64x44 x=96 ; 9: 3-D 64x43x1 x=96
  int rank = (cs == 2 || cs == 5 || cs == 9) ? 3 : 2;
  cuuint32_t bw = cs == 3 ? 16 : 64;
  cuuint32_t bh = (cs == 1 || cs == 2 || cs == 6 || cs == 9) ? 43 : (cs == 3 ? 16 : (cs == 8 ? 44 : 32));
  const int x = (cs == 1 || cs == 2 || cs == 7) ? 100 : 96, y = 50, f = 2;
  CUtensorMap m;
  const cuuint64_t dims3[3] = {(cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)F};
  const cuuint64_t str3[2] = {(cuuint64_t)P, (cuuint64_t)P * H};
  const cuuint64_t dims2[2] = {(cuuint64_t)W, (cuuint64_t)H * F};
  const cuuint64_t str2[1] = {(cuuint64_t)P};
  const cuuint32_t box[3] = {bw, bh, 1}, es[3] = {1, 1, 1};
  CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, rank, d, rank == 3 ? dims3 : dims2, rank == 3 ? str3 : str2, box,
                   es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   cs == 4 ? CU_TENSOR_MAP_L2_PROMOTION_NONE : CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  const int bytes = (int)(bw * bh);
  const int yy = rank == 3 ? y : y + f * H;
  cudaMemset(o, 0, 4096);
  if (rank == 3) probe<3><<<1, 32>>>(m, x, y, f, bytes, o);
  else probe<2><<<1, 32>>>(m, x, yy, 0, bytes, o);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<uint8_t> res(4096);
  cudaMemcpy(res.data(), o, 4096, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < (int)bh; i++)
    for (int j = 0; j < (int)bw; j++) bad += res[i * bw + j] != h[((size_t)f * H + y + i) * P + x + j];
  printf("case %d: encode %d, %s, mismatches %d / %d, timeout %d\n", cs, (int)r, cudaGetErrorString(e), bad, bytes,
         res[4095] == 0xEE);
  fflush(stdout);
  return 0;
}
