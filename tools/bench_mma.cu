// Microbenchmark: tcgen05.mma (kind::f16, M=128, cta_group::1, SS operands, SW128 K-major) latency
// from issue to tcgen05.commit -> mbarrier completion, for n MMAs of K=16 and several N.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_asplos_xiazswwyfc24_b200/csrc -o tools/bench_mma tools/bench_mma.cu
#include <cuda_runtime.h>
#include <cstdio>

#include "kernels/ptx.cuh"

using namespace souffle;

__global__ void __launch_bounds__(128, 1) k(int N, int nmma, int nw, long long* out) {
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
  if (threadIdx.x < 32) ptx::tmem_alloc(&tbase, 512);
  ptx::fence_proxy_async();
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const int w = threadIdx.x >> 5;
  if (nw == -3) {
    if (threadIdx.x < 32) {   // whole warp runs the loop; one elected lane issues
      const uint32_t idesc = ptx::idesc_bf16(128, N);
      const uint32_t sa = ptx::smem_u32(smem), sb = ptx::smem_u32(smem + 65536);
      const uint32_t tb = tbase;
      const uint64_t da = ptx::sdesc_sw128(sa), db = ptx::sdesc_sw128(sb);
      uint32_t ph = 0;
      if (ptx::elect_one()) ptx::mbar_arrive(&bars[3]);
      __syncwarp();
      for (int rep = 0; rep < 4; ++rep) {
        long long t0 = clock64();
        for (int i = 0; i < nmma; ++i) {
          if ((i & 3) == 0) {
            ptx::mbar_wait(&bars[3], 0);
            ptx::tc_fence_after();
          }
          if (ptx::elect_one())
            ptx::mma_bf16(tb, da + (uint64_t)((i & 3) * 2 + ((i >> 2) & 3) * 1024), db + (uint64_t)((i & 3) * 2), idesc,
                          i > 0);
          if ((i & 3) == 3 && ptx::elect_one()) ptx::mma_commit(&bars[(i >> 2) % 3]);
          __syncwarp();
        }
        long long t1 = clock64();
        if (ptx::elect_one()) ptx::mma_commit(&bar);
        __syncwarp();
        ptx::mbar_wait(&bar, ph);
        ph ^= 1;
        long long t2 = clock64();
        if (threadIdx.x == 0) {
          out[rep * 2] = t1 - t0;
          out[rep * 2 + 1] = t2 - t0;
        }
      }
    }
  } else if (nw <= 0) {
    if (threadIdx.x == 0) {
      const uint32_t idesc = ptx::idesc_bf16(128, N);
      const uint32_t sa = ptx::smem_u32(smem), sb = ptx::smem_u32(smem + 65536);
      const uint32_t tb = tbase;
      const uint64_t da = ptx::sdesc_sw128(sa), db = ptx::sdesc_sw128(sb);
      uint32_t ph = 0;
      // pre-complete bars[3] once so waits on parity 0 return immediately
      ptx::mbar_arrive(&bars[3]);
      for (int rep = 0; rep < 4; ++rep) {
        long long t0 = clock64();
        for (int i = 0; i < nmma; ++i) {
          if (nw == -1 && (i & 3) == 0) ptx::mbar_wait(&bars[3], 0);
          if (nw == -2 && (i & 3) == 0) ptx::tc_fence_after();
          ptx::mma_bf16(tb, da + (uint64_t)((i & 3) * 2 + ((i >> 2) & 3) * 1024), db + (uint64_t)((i & 3) * 2), idesc,
                        i > 0);
          if (nw == 0 && (i & 3) == 3) ptx::mma_commit(&bars[(i >> 2) % 3]);
        }
        long long t1 = clock64();
        ptx::mma_commit(&bar);
        ptx::mbar_wait(&bar, ph);
        ph ^= 1;
        long long t2 = clock64();
        out[rep * 2] = t1 - t0;
        out[rep * 2 + 1] = t2 - t0;
      }
    }
  } else if (nw > 1) {
    if ((threadIdx.x & 31) == 0 && w < nw) {
      const uint32_t idesc = ptx::idesc_bf16(128, N);
      const uint32_t sa = ptx::smem_u32(smem), sb = ptx::smem_u32(smem + 65536);
      const uint32_t tb = tbase + w * N;
      const uint64_t da = ptx::sdesc_sw128(sa), db = ptx::sdesc_sw128(sb);
      uint32_t ph = 0;
      for (int rep = 0; rep < 4; ++rep) {
        long long t0 = clock64();
        for (int i = 0; i < nmma / nw; ++i)
          ptx::mma_bf16(tb, da + (uint64_t)((i & 3) * 2 + ((i >> 2) & 3) * 1024), db + (uint64_t)((i & 3) * 2), idesc,
                        i > 0);
        long long t1 = clock64();
        ptx::mma_commit(&bars[w]);
        ptx::mbar_wait(&bars[w], ph);
        ph ^= 1;
        long long t2 = clock64();
        if (w == 0) {
          out[rep * 2] = t1 - t0;
          out[rep * 2 + 1] = t2 - t0;
        }
      }
    }
  } else if (threadIdx.x == 0) {
    const uint32_t idesc = ptx::idesc_bf16(128, N);
    const uint32_t sa = ptx::smem_u32(smem), sb = ptx::smem_u32(smem + 65536);
    const uint32_t tb = tbase;
    const uint64_t da = ptx::sdesc_sw128(sa), db = ptx::sdesc_sw128(sb);
    uint32_t ph = 0;
    for (int rep = 0; rep < 4; ++rep) {
      long long t0 = clock64();
      for (int i = 0; i < nmma; ++i)
        ptx::mma_bf16(tb, da + (uint64_t)((i & 3) * 2 + ((i >> 2) & 3) * 1024), db + (uint64_t)((i & 3) * 2), idesc,
                      i > 0);
      long long t1 = clock64();
      ptx::mma_commit(&bar);
      ptx::mbar_wait(&bar, ph);
      ph ^= 1;
      long long t2 = clock64();
      out[rep * 2] = t1 - t0;
      out[rep * 2 + 1] = t2 - t0;
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) ptx::tmem_dealloc(tbase, 512);
}

int main() {
  setvbuf(stdout, nullptr, _IONBF, 0);
  long long* out;
  cudaMalloc(&out, 64 * 8);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  for (int nw : {1, 0, -3})
  for (int N : {16, 64})
    for (int n : {16, 48}) {
      k<<<1, 128, 100 * 1024>>>(N, n, nw, out);
      cudaError_t e = cudaDeviceSynchronize();
      long long h[8];
      cudaMemcpy(h, out, 64, cudaMemcpyDeviceToHost);
      printf("mode %d N %3d mmas %2d: issue %5lld cyc, issue->commit done %6lld cyc (%s)\n", nw, N, n, h[6], h[7],
             cudaGetErrorString(e));
    }
  return 0;
}
