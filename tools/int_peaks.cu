// int_peaks.cu — integer-pipe peak microbenchmark for the roofline.
//
// Throughput of independent chains of LOP3 (ALU pipe), IMAD (FMA pipe), an
// alternating LOP3/IMAD stream (both pipes; bounded by issue), SHF (ALU),
// POPC (XU), at full occupancy on every SM; CUDA-event timed.
// Prints one JSON object (thread-ops/s per kind) -> profiles/int_peaks.json.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/int_peaks tools/int_peaks.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

typedef unsigned int u32;

template <int MODE>
__device__ __forceinline__ u32 op(u32 a, u32 b, u32 c) {
  u32 r;
  if constexpr (MODE == 0) asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  else if constexpr (MODE == 1) asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  else if constexpr (MODE == 3) asm volatile("shf.l.wrap.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  else { asm volatile("popc.b32 %0, %1;" : "=r"(r) : "r"(a)); }
  return r;
}

template <int MODE>
__global__ void __launch_bounds__(256) bench(u32* out, u32 iters, u32 b, u32 c) {
  u32 x[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) x[k] = threadIdx.x * 8 + k + blockIdx.x;
  for (u32 i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if constexpr (MODE == 2) x[k] = (j & 1) ? op<1>(x[k], b, c) : op<0>(x[k], b, c);
        else x[k] = op<MODE>(x[k], b, c);
      }
    }
  }
  u32 s = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s ^= x[k];
  if (s == 0x12345678u) out[0] = s;  // keep the chains alive
}

template <int MODE>
double run(const char* name, int sms, u32 iters) {
  u32* out;
  cudaMalloc(&out, 4);
  const int blocks = sms * 8, threads = 256;
  bench<MODE><<<blocks, threads>>>(out, 16, 3u, 5u);  // warm-up
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int rep = 0; rep < 5; ++rep) {
    cudaEventRecord(e0);
    bench<MODE><<<blocks, threads>>>(out, iters, 3u, 5u);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  const double ops = (double)blocks * threads * iters * 16 * 8;
  const double rate = ops / (best / 1e3);
  cudaFree(out);
  fprintf(stderr, "%-10s %.3e thread-ops/s (%.3f ms)\n", name, rate, best);
  return rate;
}

int main() {
  int dev = 0, sms = 0, clk = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);  // kHz
  const u32 iters = 4096;
  double lop3 = run<0>("lop3", sms, iters);
  double imad = run<1>("imad", sms, iters);
  double mixed = run<2>("lop3+imad", sms, iters);
  double shf = run<3>("shf", sms, iters);
  double popc = run<4>("popc", sms, iters / 4);
  printf("{\"sms\": %d, \"clock_khz_attr\": %d, \"unit\": \"thread-ops/s\", \"lop3_alu\": %.6e, "
         "\"imad_fma\": %.6e, \"lop3_imad_mixed\": %.6e, \"shf_alu\": %.6e, \"popc_xu\": %.6e, "
         "\"how\": \"8 independent chains x 16 unrolled ops per thread, %d blocks x 256 "
         "threads, best of 5, CUDA events\"}\n",
         sms, clk, lop3, imad, mixed, shf, popc, sms * 8);
  return 0;
}
