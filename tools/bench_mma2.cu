// Microbenchmark: per-MMA cost of the tcgen05 issue loop with per-chunk (4 MMA) extras:
// V bit0: tcgen05.commit per chunk, bit1: mbarrier try_wait (already complete) per chunk,
// bit2: tcgen05.fence::after_thread_sync per chunk.  48 MMAs (12 chunks), N = 64, single thread.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_asplos_xiazswwyfc24_b200/csrc -o tools/bench_mma2 tools/bench_mma2.cu
#include <cuda_runtime.h>
#include <cstdio>
#include "kernels/ptx.cuh"
using namespace souffle;

template <int V>
__global__ void __launch_bounds__(128, 1) k(long long* out) {
  extern __shared__ __align__(1024) char smem_raw[];
  char* smem = (char*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar, bars[4];
  __shared__ uint32_t tbase;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
  if (threadIdx.x == 0) {
    ptx::mbar_init(&bar, 1);
    for (int i = 0; i < 4; ++i) ptx::mbar_init(&bars[i], 1);
    ptx::fence_mbar_init();
  }
  if (threadIdx.x < 32) ptx::tmem_alloc(&tbase, 256);
  ptx::fence_proxy_async();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x == 0) {
    ptx::mbar_arrive(&bars[3]);
    const uint32_t idesc = ptx::idesc_bf16(128, 64);
    const uint32_t tb = tbase;
    const uint64_t da0 = ptx::sdesc_sw128(ptx::smem_u32(smem)), db0 = ptx::sdesc_sw128(ptx::smem_u32(smem + 65536));
    uint32_t ph = 0;
    for (int rep = 0; rep < 4; ++rep) {
      long long t0 = clock64();
      for (int c = 0; c < 12; ++c) {
        if (V & 2) ptx::mbar_wait(&bars[3], 0);
        if (V & 4) ptx::tc_fence_after();
        const uint64_t da = da0 + (uint64_t)((c & 3) * 1024), db = db0;
        if (V & 8) {
          ptx::mma_bf16_k64(tb, da, db, idesc, c > 0);
        } else {
          ptx::mma_bf16(tb, da, db, idesc, c > 0);
#pragma unroll
          for (int kk = 1; kk < 4; ++kk) ptx::mma_bf16(tb, da + 2 * kk, db + 2 * kk, idesc, 1u);
        }
        if (V & 1) ptx::mma_commit(&bars[c % 3]);
      }
      long long t1 = clock64();
      ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, ph);
      ph ^= 1;
      long long t2 = clock64();
      out[2 * V] = t1 - t0;
      out[2 * V + 1] = t2 - t0;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) ptx::tmem_dealloc(tbase, 256);
}

template <int V>
void run(long long* out) {
  cudaFuncSetAttribute(k<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  k<V><<<1, 128, 100 * 1024>>>(out);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[32];
  cudaMemcpy(h, out, 256, cudaMemcpyDeviceToHost);
  printf("variant %d (commit %d wait %d fence %d): 48 MMAs issue %lld cyc, done %lld cyc (%s)\n", V, V & 1, (V >> 1) & 1,
         (V >> 2) & 1, h[2 * V], h[2 * V + 1], cudaGetErrorString(e));
}

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  long long* out;
  cudaMalloc(&out, 512);
  run<0>(out); run<7>(out); run<8>(out); run<15>(out);
  return 0;
}
