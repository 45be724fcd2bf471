// Microbenchmark: how fast can every SM pull an L2-resident activation tile into shared memory?
// (the A operand of a batch-1 GEMM stage is the same 128 x K bf16 tile for every CTA)
//   mode 0: TMA, each CTA loads nchunks x (128 x 64 bf16) = nchunks x 16 KB, one mbarrier
//   mode 1: TMA multicast inside a cluster of CL CTAs (each CTA issues nchunks/CL chunks, multicast)
//   mode 2: ld.global.cg float4 by 256 threads (fp32 tile of the same byte count)
// Reports the median per-CTA latency (globaltimer, ns) from issue to data-in-smem.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_asplos_xiazswwyfc24_b200/csrc -o tools/bench_tma tools/bench_tma.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cooperative_groups.h>
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

template <int MODE, int CL>
__global__ void __launch_bounds__(256, 1) k(const __grid_constant__ CUtensorMap tm, const float* src, int nchunks,
                                           unsigned long long* out, unsigned* sync) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    ptx::fence_mbar_init();
  }
  if (CL > 1) cooperative_groups::this_cluster().sync();
  __syncthreads();
  // crude start alignment: all CTAs spin until everyone arrived
  if (threadIdx.x == 0) {
    atomicAdd(sync, 1u);
    for (long long n = 0; ptx::ld_acquire(sync) < gridDim.x && n < 20000000; ++n) {}
  }
  __syncthreads();
  unsigned long long t0 = gtime();
  if (MODE == 0) {
    if (threadIdx.x == 0) {
      ptx::mbar_arrive_expect_tx(&bar, nchunks * 16384);
      for (int c = 0; c < nchunks; ++c) ptx::tma_load_2d(smem + c * 16384, &tm, &bar, c * 64, 0);
    }
    for (long long n = 0; !ptx::mbar_try_wait(&bar, 0) && n < 20000000; ++n) {}
  } else if (MODE == 1) {
    const unsigned rank = cooperative_groups::this_cluster().block_rank();
    if (threadIdx.x == 0) {
      ptx::mbar_arrive_expect_tx(&bar, nchunks * 16384);
    }
    if (CL > 1) cooperative_groups::this_cluster().sync();   // every CTA armed before any multicast lands
    if (threadIdx.x == 0) {
      for (int c = rank; c < nchunks; c += CL) {
        const uint16_t mask = (uint16_t)((1u << CL) - 1);
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster"
            " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(ptx::smem_u32(smem + c * 16384)),
            "l"(&tm), "r"(ptx::smem_u32(&bar)), "r"(c * 64), "r"(0), "h"(mask)
            : "memory");
      }
    }
    for (long long n = 0; !ptx::mbar_try_wait(&bar, 0) && n < 20000000; ++n) {}
  } else {
    const int n4 = nchunks * 16384 / 16;
    float4* d = reinterpret_cast<float4*>(smem);
    const float4* s = reinterpret_cast<const float4*>(src);
    constexpr int U = 8;
    for (int i = threadIdx.x; i < n4; i += 256 * U) {
      float4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (i + u * 256 < n4) v[u] = __ldcg(s + i + u * 256);
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (i + u * 256 < n4) d[i + u * 256] = v[u];
    }
    __syncthreads();
  }
  unsigned long long t1 = gtime();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  if (CL > 1) cooperative_groups::this_cluster().sync();
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

template <int MODE, int CL>
void run(const CUtensorMap& tm, const float* src, int nchunks, int grid, unsigned long long* out, unsigned* sync) {
  auto fn = k<MODE, CL>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  std::vector<unsigned long long> h(grid);
  std::vector<double> med;
  for (int rep = 0; rep < 5; ++rep) {
    cudaMemset(sync, 0, 4);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(256);
    cfg.dynamicSmemBytes = 200 * 1024;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = CL;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, fn, tm, src, nchunks, out, sync);
    cudaError_t e = cudaDeviceSynchronize();
    printf(".");
    if (e != cudaSuccess) { printf("error %s\n", cudaGetErrorString(e)); return; }
    cudaMemcpy(h.data(), out, grid * 8, cudaMemcpyDeviceToHost);
    std::sort(h.begin(), h.end());
    med.push_back(h[grid / 2]);
    if (rep == 4)
      printf("mode %d cluster %d grid %3d chunks %2d (%3d KB/CTA): median %6.0f ns  max %6llu ns  -> %.0f GB/s per CTA, %.2f TB/s total\n",
             MODE, CL, grid, nchunks, nchunks * 16, (double)h[grid / 2], h[grid - 1],
             nchunks * 16384.0 / h[grid / 2], nchunks * 16384.0 * grid / h[grid - 1] / 1e3);
  }
}

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  void* p = nullptr;
  cudaDriverEntryPointQueryResult qr;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &qr);
  Enc enc = (Enc)p;
  uint16_t* A;
  float* F;
  unsigned long long* out;
  unsigned* sync;
  cudaMalloc(&A, 128 * 3072 * 2);
  cudaMalloc(&F, 128 * 3072 * 4);
  cudaMalloc(&out, 4096 * 8);
  cudaMalloc(&sync, 64);
  cudaMemset(A, 0, 128 * 3072 * 2);
  cudaMemset(F, 0, 128 * 3072 * 4);
  CUtensorMap tm;
  cuuint64_t dims[2] = {3072, 128};
  cuuint64_t strides[1] = {3072 * 2};
  cuuint32_t box[2] = {64, 128};
  cuuint32_t es[2] = {1, 1};
  enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, A, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  for (int grid : {1, 36, 144, 148}) {
    for (int nch : {1, 3, 4, 12}) run<0, 1>(tm, F, nch, grid, out, sync);
  }
  for (int grid : {144}) {
    for (int nch : {4, 12}) {
      run<1, 2>(tm, F, nch, grid, out, sync);
      run<1, 4>(tm, F, nch, grid, out, sync);
    }
  }
  for (int grid : {1, 12, 48, 148})
    for (int nch : {2, 6, 12}) run<2, 1>(tm, F, nch, grid, out, sync);
  return 0;
}
