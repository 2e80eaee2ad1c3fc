// tma_probe.cu -- one-warp TMA tensor-copy probe for the describe kernel's patch loads: a 3-D
// u8 map [frames][h][w] (pitch, frame stride), box 64 x 43 x 1, passed as a __grid_constant__
// struct of 8 maps; variants isolate which PTX form the hardware accepts.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tma_probe tma_probe.cu
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

struct Maps {
  CUtensorMap level[8];
  uint32_t valid;
};

__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int V>
__global__ void probe(const __grid_constant__ Maps maps, int l, int x, int y, int f, uint8_t* out) {
  __shared__ __align__(128) uint8_t buf[64 * 43];
  __shared__ __align__(8) uint64_t bar;
  const int lane = threadIdx.x;
  const uint32_t b = saddr(&bar);
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    if (V != 1) asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(64 * 43) : "memory");
    const CUtensorMap* m = V == 3 ? &maps.level[0] : &maps.level[l];
    if (V == 2)
      asm volatile(
          "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::"r"(
              saddr(buf)),
          "l"(reinterpret_cast<uint64_t>(m)), "r"(x), "r"(y), "r"(f), "r"(b)
          : "memory");
    else
      asm volatile(
          "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
          "[%5];" ::"r"(saddr(buf)),
          "l"(reinterpret_cast<uint64_t>(m)), "r"(x), "r"(y), "r"(f), "r"(b)
          : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t"
      "@!P1 bra W_%=;\n}" ::"r"(b)
      : "memory");
  for (int i = lane; i < 64 * 43; i += 32) out[i] = buf[i];
}

// variant 5: the descriptor in GLOBAL memory (copied there by the host before the launch)
__global__ void probe_gmem(const CUtensorMap* gm, int x, int y, int f, uint8_t* out) {
  __shared__ __align__(128) uint8_t buf[64 * 43];
  __shared__ __align__(8) uint64_t bar;
  const int lane = threadIdx.x;
  const uint32_t b = saddr(&bar);
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(64 * 43) : "memory");
    asm volatile(
        "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], "
        "[%5];" ::"r"(saddr(buf)),
        "l"(reinterpret_cast<uint64_t>(gm)), "r"(x), "r"(y), "r"(f), "r"(b)
        : "memory");
  }
  __syncwarp();
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "W_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n\t"
      "@!P1 bra W_%=;\n}" ::"r"(b)
      : "memory");
  for (int i = lane; i < 64 * 43; i += 32) out[i] = buf[i];
}

int main(int argc, char** argv) {
  const int only = argc > 1 ? atoi(argv[1]) : -1;
  const int W = 752, H = 480, F = 3, P = 768;
  std::vector<uint8_t> h((size_t)F * H * P);
  for (int f = 0; f < F; f++)
    for (int y = 0; y < H; y++)
      for (int x = 0; x < P; x++) h[((size_t)f * H + y) * P + x] = (uint8_t)(x * 7 + y * 13 + f * 31);
  uint8_t *d, *o;
  cudaMalloc(&d, h.size());
  cudaMalloc(&o, 64 * 43);
  cudaMemcpy(d, h.data(), h.size(), cudaMemcpyHostToDevice);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  Maps maps{};
  const cuuint64_t dims[3] = {(cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)F};
  const cuuint64_t strides[2] = {(cuuint64_t)P, (cuuint64_t)P * H};
  const cuuint32_t box[3] = {64, 43, 1}, es[3] = {1, 1, 1};
  for (int l = 0; l < 8; l++) {
    CUresult r = enc(&maps.level[l], CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, d, dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (l == 0) printf("encode rc=%d fn=%p q=%d sizeof(Maps)=%zu\n", (int)r, fn, (int)q, sizeof(Maps));
    fflush(stdout);
  }
  const int x = 100, y = 50, f = 2, l = 3;
  void (*ks[4])(const Maps, int, int, int, int, uint8_t*) = {probe<0>, probe<1>, probe<2>, probe<3>};
  for (int v = 0; v < 4; v++) {
    if (only >= 0 && v != only) continue;
    cudaMemset(o, 0, 64 * 43);
    ks[v]<<<1, 32>>>(maps, l, x, y, f, o);
    cudaError_t e = cudaDeviceSynchronize();
    printf("variant %d launched\n", v);
    fflush(stdout);
    std::vector<uint8_t> r(64 * 43);
    cudaMemcpy(r.data(), o, r.size(), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < 43; i++)
      for (int j = 0; j < 64; j++) bad += r[i * 64 + j] != h[((size_t)f * H + y + i) * P + x + j];
    printf("variant %d: %s, mismatches %d\n", v, cudaGetErrorString(e), bad);
    fflush(stdout);
    if (e != cudaSuccess) return 1;
  }
  if (only == 4 || only == 5) {
    cudaMemset(o, 0, 64 * 43);
    if (only == 4) {  // cluster launch of (1, 1, 1)
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(1);
      cfg.blockDim = dim3(32);
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = 1;
      at[0].val.clusterDim.y = 1;
      at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      cudaLaunchKernelEx(&cfg, probe<0>, maps, l, x, y, f, o);
    } else {
      CUtensorMap* gm;
      cudaMalloc(&gm, sizeof(CUtensorMap));
      cudaMemcpy(gm, &maps.level[l], sizeof(CUtensorMap), cudaMemcpyHostToDevice);
      probe_gmem<<<1, 32>>>(gm, x, y, f, o);
    }
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<uint8_t> r(64 * 43);
    cudaMemcpy(r.data(), o, r.size(), cudaMemcpyDeviceToHost);
    int bad = 0;
    for (int i = 0; i < 43; i++)
      for (int j = 0; j < 64; j++) bad += r[i * 64 + j] != h[((size_t)f * H + y + i) * P + x + j];
    printf("variant %d: %s, mismatches %d\n", only, cudaGetErrorString(e), bad);
    fflush(stdout);
  }
  return 0;
}
