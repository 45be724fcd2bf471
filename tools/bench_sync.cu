// Microbenchmark of synchronisation primitives on sm_100a (cycles via clock64, per op):
//   fence.acq_rel.gpu, fence.sc.gpu (__threadfence), fence.proxy.async, red.release + ld.acquire,
//   dependent L2 load latency, and grid barriers (148 CTAs) with several implementations.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bench_sync tools/bench_sync.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <cooperative_groups.h>

__device__ __forceinline__ unsigned ld_acq(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ unsigned ld_relaxed(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_rel(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_relaxed(unsigned* p, unsigned v) {
  asm volatile("red.relaxed.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__global__ void k_primitives(unsigned* buf, long long* out, int iters) {
  if (threadIdx.x != 0) return;
  long long t0, t1;
  // 1. fence.acq_rel.gpu
  t0 = clock64();
  for (int i = 0; i < iters; ++i) { buf[64] = i; asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
  t1 = clock64(); out[0] = (t1 - t0) / iters;
  // 2. __threadfence
  t0 = clock64();
  for (int i = 0; i < iters; ++i) { buf[64] = i; __threadfence(); }
  t1 = clock64(); out[1] = (t1 - t0) / iters;
  // 3. fence.proxy.async
  t0 = clock64();
  for (int i = 0; i < iters; ++i) { buf[64] = i; asm volatile("fence.proxy.async;" ::: "memory"); }
  t1 = clock64(); out[2] = (t1 - t0) / iters;
  // 4. red.release + ld.acquire (round trip on own counter)
  t0 = clock64();
  for (int i = 0; i < iters; ++i) { red_rel(buf, 1); while (ld_acq(buf) < (unsigned)(i + 1)) {} }
  t1 = clock64(); out[3] = (t1 - t0) / iters;
  // 5. dependent L2 load chain (pointer chase in a 64 KB ring, resident in L2; .cg bypasses L1)
  unsigned idx = 0;
  t0 = clock64();
  for (int i = 0; i < iters; ++i) idx = __ldcg(&buf[1024 + idx]);
  t1 = clock64(); out[4] = (t1 - t0) / iters + (idx == 0xFFFFFFFF);
  // 6. ld.acquire alone
  t0 = clock64();
  unsigned s = 0;
  for (int i = 0; i < iters; ++i) s += ld_acq(buf + 128 + (s & 1));
  t1 = clock64(); out[5] = (t1 - t0) / iters + (s == 0xFFFFFFFF);
  // 7. ld.relaxed.gpu alone
  t0 = clock64();
  for (int i = 0; i < iters; ++i) s += ld_relaxed(buf + 128 + (s & 1));
  t1 = clock64(); out[6] = (t1 - t0) / iters + (s == 0xFFFFFFFF);
}

// grid barrier variants; each CTA does `rounds` barriers; report total cycles on CTA 0
template <int KIND>
__global__ void k_grid(unsigned* ctr, long long* out, int rounds) {
  __shared__ int dummy;
  long long t0 = clock64();
  for (int r = 1; r <= rounds; ++r) {
    if (KIND == 0) {  // fence + atomicAdd + volatile spin (classic)
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(ctr, 1u);
        while (*(volatile unsigned*)ctr < (unsigned)(r * gridDim.x)) {}
        __threadfence();
      }
      __syncthreads();
    } else if (KIND == 1) {  // red.release + ld.acquire spin
      __syncthreads();
      if (threadIdx.x == 0) {
        red_rel(ctr, 1u);
        while (ld_acq(ctr) < (unsigned)(r * gridDim.x)) {}
      }
      __syncthreads();
    } else if (KIND == 2) {  // red.release + relaxed spin + acquire fence once
      __syncthreads();
      if (threadIdx.x == 0) {
        red_rel(ctr, 1u);
        while (ld_relaxed(ctr) < (unsigned)(r * gridDim.x)) {}
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncthreads();
    } else if (KIND == 4) {  // hierarchical: group-of-16 counters, last arriver forwards to the root
      __syncthreads();
      if (threadIdx.x == 0) {
        __threadfence();
        const unsigned grp = blockIdx.x / 16, gsz = min(16u, gridDim.x - grp * 16);
        unsigned old = atomicAdd(ctr + 64 + 32 * grp, 1u);
        if (old + 1 == r * gsz) red_rel(ctr, 1u);
        const unsigned ngrp = (gridDim.x + 15) / 16;
        while (ld_acq(ctr) < (unsigned)(r * ngrp)) {}
      }
      __syncthreads();
    } else if (KIND == 5) {  // flag array: each CTA stores its round number; warp 0 polls all flags
      __syncthreads();
      unsigned* flags = ctr + 4096;
      if (threadIdx.x == 0) {
        __threadfence();
        asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(flags + blockIdx.x), "r"((unsigned)r) : "memory");
      }
      if (threadIdx.x < 32) {
        while (true) {
          bool ok = true;
          for (unsigned c = threadIdx.x; c < gridDim.x; c += 32) ok &= ld_relaxed(flags + c) >= (unsigned)r;
          if (__all_sync(0xffffffffu, ok)) break;
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncthreads();
    } else if (KIND == 6) {  // counter + single poller (CTA 0) + per-CTA release flags
      __syncthreads();
      unsigned* flags = ctr + 8192;   // one 128-B line per CTA
      if (threadIdx.x == 0) {
        __threadfence();
        red_rel(ctr, 1u);
      }
      if (blockIdx.x == 0) {
        if (threadIdx.x == 0)
          while (ld_acq(ctr) < (unsigned)(r * gridDim.x)) {}
        __syncwarp();
        if (threadIdx.x < 32)
          for (unsigned c = threadIdx.x; c < gridDim.x; c += 32)
            asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flags + 32 * c), "r"((unsigned)r) : "memory");
      } else if (threadIdx.x == 0) {
        while (ld_acq(flags + 32 * blockIdx.x) < (unsigned)r) {}
      }
      __syncthreads();
    } else if (KIND == 7) {  // K1 with back-off polling
      __syncthreads();
      if (threadIdx.x == 0) {
        red_rel(ctr, 1u);
        while (ld_acq(ctr) < (unsigned)(r * gridDim.x)) __nanosleep(100);
      }
      __syncthreads();
    } else if (KIND == 8) {  // 8 counters on separate lines; lanes 0-7 poll all of them
      __syncthreads();
      if (threadIdx.x == 0) red_rel(ctr + 32 * (blockIdx.x & 7), 1u);
      if (threadIdx.x < 32) {
        const unsigned g = threadIdx.x & 7;
        const unsigned cnt = gridDim.x / 8 + (g < gridDim.x % 8 ? 1u : 0u);
        while (true) {
          bool ok = threadIdx.x >= 8 || ld_relaxed(ctr + 32 * g) >= r * cnt;
          if (__all_sync(0xffffffffu, ok)) break;
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncthreads();
    } else if (KIND == 9) {  // 16 counters on separate lines; lanes 0-15 poll
      __syncthreads();
      if (threadIdx.x == 0) red_rel(ctr + 32 * (blockIdx.x & 15), 1u);
      if (threadIdx.x < 32) {
        const unsigned g = threadIdx.x & 15;
        const unsigned cnt = gridDim.x / 16 + (g < gridDim.x % 16 ? 1u : 0u);
        while (true) {
          bool ok = threadIdx.x >= 16 || ld_relaxed(ctr + 32 * g) >= r * cnt;
          if (__all_sync(0xffffffffu, ok)) break;
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
      __syncthreads();
    } else {  // cooperative groups grid.sync()
      cooperative_groups::this_grid().sync();
    }
  }
  long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = (t1 - t0) / rounds;
  (void)dummy;
}

int main() {
  unsigned* buf;
  long long* out;
  cudaMalloc(&buf, 1 << 22);
  cudaMalloc(&out, 64 * sizeof(long long));
  // pointer-chase ring (stride 67 words) in buf[1024..]
  unsigned h[16384];
  for (int i = 0; i < 16384; ++i) h[i] = (i * 67 + 67) % 16384;
  cudaMemset(buf, 0, 1 << 22);
  cudaMemcpy(buf + 1024, h, sizeof(h), cudaMemcpyHostToDevice);
  k_primitives<<<1, 32>>>(buf, out, 1000);
  long long o[8];
  cudaMemcpy(o, out, sizeof(o), cudaMemcpyDeviceToHost);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("clock %d MHz (nominal)\n", clk / 1000);
  const char* names[] = {"store+fence.acq_rel.gpu", "store+__threadfence", "store+fence.proxy.async",
                         "red.release+ld.acquire roundtrip", "dependent L2 load (ldcg)", "ld.acquire.gpu",
                         "ld.relaxed.gpu"};
  for (int i = 0; i < 7; ++i) printf("%-36s %6lld cycles\n", names[i], o[i]);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (int kind = 0; kind < 10; ++kind) {
    for (int grid : {1, 148}) {
      cudaMemset(buf, 0, 1 << 20);
      void* args[] = {&buf, &out, nullptr};
      int rounds = 200;
      args[2] = &rounds;
      void* fn = kind == 0 ? (void*)k_grid<0> : kind == 1 ? (void*)k_grid<1> : kind == 2 ? (void*)k_grid<2> : kind == 3 ? (void*)k_grid<3> : kind == 4 ? (void*)k_grid<4> : kind == 5 ? (void*)k_grid<5> : kind == 6 ? (void*)k_grid<6> : kind == 7 ? (void*)k_grid<7> : kind == 8 ? (void*)k_grid<8> : (void*)k_grid<9>;
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      cudaLaunchCooperativeKernel(fn, grid, 256, args, 0, 0);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      cudaMemcpy(o, out, 8, cudaMemcpyDeviceToHost);
      printf("grid barrier kind %d grid %3d: %6lld cycles/barrier, %.2f us/barrier (event)  %s\n", kind, grid, o[0],
             ms * 1e3 / rounds, cudaGetErrorString(cudaGetLastError()));
    }
  }
  return 0;
}
