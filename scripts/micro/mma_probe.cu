// Throughput probe: legacy mma.sync u8 m16n8k32 and b1 xor.popc m16n8k256 on sm_100a
// (is a tensor-core Hamming matcher worth it?).  nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cstdio>
#include <cstdint>
__global__ void k(const uint32_t* a, const uint32_t* b, int* out, int iters) {
  uint32_t A[4], B[2];
  for (int i = 0; i < 4; i++) A[i] = a[threadIdx.x * 4 + i];
  for (int i = 0; i < 2; i++) B[i] = b[threadIdx.x * 2 + i];
  int c[4][4] = {};
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int j = 0; j < 4; j++)
      asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.u8.u8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+r"(c[j][0]), "+r"(c[j][1]), "+r"(c[j][2]), "+r"(c[j][3]) : "r"(A[j&3]), "r"(A[(j+1)&3]), "r"(A[2]), "r"(A[3]), "r"(B[0]), "r"(B[1]));
  }
  int s = 0;
  for (int j = 0; j < 4; j++) s += c[j][0] + c[j][1] + c[j][2] + c[j][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void kb(const uint32_t* a, const uint32_t* b, int* out, int iters) {
  uint32_t A[4], B[2];
  for (int i = 0; i < 4; i++) A[i] = a[threadIdx.x * 4 + i];
  for (int i = 0; i < 2; i++) B[i] = b[threadIdx.x * 2 + i];
  int c[4][4] = {};
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int j = 0; j < 4; j++)
    asm volatile("mma.sync.aligned.m16n8k256.row.col.s32.b1.b1.s32.xor.popc {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                 : "+r"(c[j][0]), "+r"(c[j][1]), "+r"(c[j][2]), "+r"(c[j][3]) : "r"(A[j&3]), "r"(A[(j+1)&3]), "r"(A[2]), "r"(A[3]), "r"(B[0]), "r"(B[1]));
  }
  int s = 0;
  for (int j = 0; j < 4; j++) s += c[j][0] + c[j][1] + c[j][2] + c[j][3];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
  uint32_t *a, *b; int* o;
  cudaMalloc(&a, 4096); cudaMalloc(&b, 4096); cudaMalloc(&o, 1 << 22);
  cudaMemset(a, 0x5a, 4096); cudaMemset(b, 0x33, 4096);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int which = 0; which < 2; which++) {
    int iters = which ? 256 : 4096;
    for (int rep = 0; rep < 2; rep++) {
      cudaEventRecord(e0);
      if (which == 0) k<<<148 * 4, 256>>>(a, b, o, iters); else kb<<<148 * 4, 256>>>(a, b, o, iters);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
    }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double mmas = 148.0 * 4 * 8 * iters * 4;
    double macs = mmas * (which ? 16 * 8 * 256 : 16 * 8 * 32);
    printf("%s: %.3f ms, %.2f mma/clk/SM, %.1f TOPS (bit-ops for b1), err=%s\n", which ? "b1 xor.popc m16n8k256" : "u8 m16n8k32",
           ms, mmas / (ms * 1e-3) / 148 / 1.965e9, 2 * macs / (ms * 1e-3) * 1e-12, cudaGetErrorString(cudaGetLastError()));
  }
}
