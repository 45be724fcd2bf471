// Microbenchmark: A-operand delivery through a TMA ring, as in the BERT GEMM stages.  Every CTA streams
// NCH chunks of 128 rows x 64 bf16 (16 KB, SWIZZLE_128B) through a ring of R slots (a slot is refilled as
// soon as its chunk landed).  src 0: every CTA reads the same [128, 768] tile (L2-resident broadcast);
// src 1: every CTA reads its own tile.  Reports the median / max per-CTA time (globaltimer).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_asplos_xiazswwyfc24_b200/csrc -o tools/bench_ring tools/bench_ring.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <algorithm>
#include <cstdio>
#include <vector>

#include "kernels/ptx.cuh"

using namespace souffle;

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__global__ void __launch_bounds__(128, 1) k(const __grid_constant__ CUtensorMap tm, int nch, int R, int src,
                                           int active, unsigned long long* out, unsigned* sync) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[16];
  if (blockIdx.x >= active) return;
  if (threadIdx.x == 0) {
    for (int i = 0; i < R; ++i) ptx::mbar_init(&bar[i], 1);
    ptx::fence_mbar_init();
    atomicAdd(sync, 1u);
    for (long long n = 0; ptx::ld_acquire(sync) < (unsigned)active && n < 20000000; ++n) {}
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  const int row0 = src ? 128 * blockIdx.x : 0;
  unsigned long long t0 = gtime();
  for (int c = 0; c < nch && c < R; ++c) {
    ptx::mbar_arrive_expect_tx(&bar[c], 16384);
    ptx::tma_load_2d(smem + c * 16384, &tm, &bar[c], (c % 12) * 64, row0);
  }
  for (int c = 0; c < nch; ++c) {
    const int s = c % R;
    while (!ptx::mbar_try_wait(&bar[s], (c / R) & 1)) {}
    const int nx = c + R;
    if (nx < nch) {
      ptx::mbar_arrive_expect_tx(&bar[s], 16384);
      ptx::tma_load_2d(smem + s * 16384, &tm, &bar[s], (nx % 12) * 64, row0);
    }
  }
  out[blockIdx.x] = gtime() - t0;
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  void* p = nullptr;
  cudaDriverEntryPointQueryResult qr;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &qr);
  Enc enc = (Enc)p;
  uint16_t* A;
  unsigned long long* out;
  unsigned* sync;
  const int rows = 128 * 148;
  cudaMalloc(&A, (size_t)rows * 768 * 2);
  cudaMalloc(&out, 4096 * 8);
  cudaMalloc(&sync, 64);
  cudaMemset(A, 0, (size_t)rows * 768 * 2);
  CUtensorMap tm;
  cuuint64_t dims[2] = {768, (cuuint64_t)rows};
  cuuint64_t strides[1] = {768 * 2};
  cuuint32_t box[2] = {64, 128};
  cuuint32_t es[2] = {1, 1};
  enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, A, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  std::vector<unsigned long long> h(148);
  for (int src : {0, 1})
    for (int active : {148, 72, 36})
      for (int R : {2, 4, 8, 12}) {
        double med = 0, mx = 0;
        for (int rep = 0; rep < 4; ++rep) {
          cudaMemset(sync, 0, 4);
          k<<<148, 128, 200 * 1024>>>(tm, 12, R, src, active, out, sync);
          cudaError_t e = cudaDeviceSynchronize();
          if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return 1; }
          cudaMemcpy(h.data(), out, active * 8, cudaMemcpyDeviceToHost);
          std::sort(h.begin(), h.begin() + active);
          med = h[active / 2];
          mx = h[active - 1];
        }
        printf("src %d active %3d ring %2d: 192 KB per CTA median %6.0f ns max %6.0f ns -> %5.0f GB/s per CTA, %5.2f TB/s total\n",
               src, active, R, med, mx, 196608.0 / med, 196608.0 * active / mx / 1e3);
      }
  return 0;
}
