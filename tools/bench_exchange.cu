// t_exchange_min: the one-way latency of the LSTM kernel's dependency exchange (kernels/lstm.cu)
// between two CTAs on different SMs -- a producer stores a 64-bit (value, tag) word with
// st.relaxed.gpu, the consumer spins on ld.relaxed.gpu until the tag matches (no fence: the tag and
// the value are one single-copy-atomic word).  Ping-pong between CTA 0 and CTA `peer`: one-way =
// round trip / 2.  The LSTM's dependency chain is L + T - 1 = 109 wavefront steps, so
// 109 x t_exchange_min is the chain bound of the whole LSTM.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bench_exchange tools/bench_exchange.cu
// run:   tools/bench_exchange [out.json]
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__global__ void pingpong(unsigned long long* words, long long* out, int iters, int peer) {
  if (threadIdx.x != 0) return;
  const int me = blockIdx.x;
  if (me != 0 && me != peer) return;
  unsigned long long* mine = words + (me == 0 ? 0 : 32);     // 256 B apart: different lines
  unsigned long long* other = words + (me == 0 ? 32 : 0);
  long long t0 = 0;
  unsigned long long g0 = 0;
  for (int i = 0; i < iters; ++i) {
    if (me == 0) {
      if (i == 8) {   // warm-up rounds excluded
        t0 = clock64();
        g0 = gtime();
      }
      const unsigned long long w = ((unsigned long long)(2 * i + 1) << 32) | 0x3f800000u;
      asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(mine), "l"(w) : "memory");
      unsigned long long r;
      do {
        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(r) : "l"(other) : "memory");
      } while ((unsigned)(r >> 32) != (unsigned)(2 * i + 2));
    } else {
      unsigned long long r;
      do {
        asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(r) : "l"(other) : "memory");
      } while ((unsigned)(r >> 32) != (unsigned)(2 * i + 1));
      const unsigned long long w = ((unsigned long long)(2 * i + 2) << 32) | (r & 0xffffffffu);
      asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(mine), "l"(w) : "memory");
    }
  }
  if (me == 0) {
    out[0] = (clock64() - t0) / (iters - 8);
    out[1] = (long long)((gtime() - g0) / (iters - 8));   // ns per round trip
  }
}

int main(int argc, char** argv) {
  const char* path = argc > 1 ? argv[1] : nullptr;
  unsigned long long* words;
  long long* out;
  cudaMalloc(&words, 4096);
  cudaMalloc(&out, 64);
  int clk_khz = 0;
  cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  const int iters = 2000;
  long long best = 1LL << 60, worst = 0;
  double sum = 0;
  int n = 0;
  // 200 KB of shared memory per CTA: one CTA per SM, so the two players are on different SMs
  cudaFuncSetAttribute(pingpong, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  long long best_ns = 1LL << 60;
  double sum_ns = 0;
  for (int peer = 1; peer < 148; peer += 7) {   // peers at various SM distances (same / other die)
    cudaMemset(words, 0, 4096);
    pingpong<<<148, 32, 200 * 1024>>>(words, out, iters, peer);
    long long rt[2] = {0, 0};
    cudaMemcpy(rt, out, 16, cudaMemcpyDeviceToHost);
    best = rt[0] < best ? rt[0] : best;
    worst = rt[0] > worst ? rt[0] : worst;
    sum += rt[0];
    best_ns = rt[1] < best_ns ? rt[1] : best_ns;
    sum_ns += rt[1];
    ++n;
  }
  const double ghz = clk_khz / 1e6;
  const double one_way_min_ns = best_ns / 2.0, one_way_mean_ns = sum_ns / n / 2.0;
  char buf[512];
  snprintf(buf, sizeof buf,
           "{\"round_trip_cycles_min\": %lld, \"round_trip_cycles_max\": %lld, \"round_trip_cycles_mean\": %.1f, "
           "\"clock_ghz_nominal\": %.3f, \"t_exchange_min_ns\": %.1f, \"t_exchange_mean_ns\": %.1f, "
           "\"lstm_wavefront_steps\": 109, \"lstm_chain_bound_us\": %.2f, \"lstm_chain_bound_mean_us\": %.2f}\n",
           best, worst, sum / n, ghz, one_way_min_ns, one_way_mean_ns, 109 * one_way_min_ns / 1e3,
           109 * one_way_mean_ns / 1e3);
  printf("%s", buf);
  if (path) {
    FILE* f = fopen(path, "w");
    if (f) {
      fputs(buf, f);
      fclose(f);
    }
  }
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
