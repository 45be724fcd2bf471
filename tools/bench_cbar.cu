// Grid barrier microbenchmark: flat single-counter barrier vs hierarchical barrier that first syncs the
// thread-block cluster in hardware (barrier.cluster) and lets one CTA per cluster arrive on the global
// counter.  Per-barrier cycles on CTA 0, 1 CTA per SM.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bench_cbar tools/bench_cbar.cu
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned ld_acq(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_rel(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned cluster_rank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ unsigned cluster_n() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_nctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cbar() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int KIND>
__global__ void __launch_bounds__(256, 1) k(unsigned* ctr, long long* out, int rounds) {
  extern __shared__ char big[];
  long long t0 = clock64();
  const unsigned ncl = gridDim.x / cluster_n();
  for (int r = 1; r <= rounds; ++r) {
    if (KIND == 0) {   // flat
      __syncthreads();
      if (threadIdx.x == 0) {
        red_rel(ctr, 1u);
        while (ld_acq(ctr) < (unsigned)(r * gridDim.x)) {}
      }
      __syncthreads();
    } else {           // hierarchical through the cluster barrier
      cbar();
      if (cluster_rank() == 0 && threadIdx.x == 0) {
        red_rel(ctr, 1u);
        while (ld_acq(ctr) < (unsigned)(r * ncl)) {}
      }
      __syncwarp();
      cbar();
    }
  }
  long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = (t1 - t0) / rounds;
  big[0] = 0;
}

template <int KIND>
void run(int grid, int cl, unsigned* ctr, long long* out) {
  auto f = k<KIND>;
  int smem = 150 * 1024;   // force 1 CTA per SM
  cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (cl > 8) cudaFuncSetAttribute(f, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[2];
  int na = 0;
  at[na].id = cudaLaunchAttributeClusterDimension;
  at[na].val.clusterDim.x = cl; at[na].val.clusterDim.y = 1; at[na].val.clusterDim.z = 1;
  ++na;
  cfg.attrs = at;
  cfg.numAttrs = na;
  int maxc = 0;
  cudaOccupancyMaxActiveClusters(&maxc, f, &cfg);
  if (maxc * cl < grid) {
    printf("kind %d grid %3d cluster %2d: only %d clusters co-resident, skipped\n", KIND, grid, cl, maxc);
    fflush(stdout);
    return;
  }
  for (int rep = 0; rep < 3; ++rep) {
    cudaMemset(ctr, 0, 4096);
    cudaError_t e = cudaLaunchKernelEx(&cfg, f, ctr, out, 2000);
    cudaError_t e2 = cudaDeviceSynchronize();
    long long o = -1;
    cudaMemcpy(&o, out, 8, cudaMemcpyDeviceToHost);
    if (rep == 2)
      printf("kind %d grid %3d cluster %2d (max active clusters %3d): %6lld cycles/barrier %s %s\n", KIND, grid, cl, maxc, o,
             cudaGetErrorString(e), cudaGetErrorString(e2));
    fflush(stdout);
  }
}

int main() {
  unsigned* ctr;
  long long* out;
  cudaMalloc(&ctr, 4096);
  cudaMalloc(&out, 64);
  run<0>(148, 1, ctr, out);
  run<0>(144, 1, ctr, out);
  run<1>(148, 2, ctr, out);
  run<1>(148, 4, ctr, out);
  run<1>(144, 4, ctr, out);
  run<1>(144, 8, ctr, out);
  run<1>(144, 16, ctr, out);
  run<1>(128, 16, ctr, out);
  return 0;
}
