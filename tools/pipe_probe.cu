// pipe_probe.cu — throughput of the ALU-pipe opcodes the ply loop issues
// (DESIGN.md §6): is every LOP3 / SEL / ISETP / IADD3.X / funnel SHF / LOP3->P a
// full-rate (16 lanes/SMSP/clk) instruction, and what does a mix shaped like
// the loop's (ALU : IMAD about 3 : 2) sustain? 8 independent chains per
// thread, 148 x 8 CTAs of 256 threads, best of 5, CUDA events. Tooling.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/pipe_probe tools/pipe_probe.cu
#include <cuda_runtime.h>
#include <cstdio>

typedef unsigned int u32;

template <int M>
__device__ __forceinline__ u32 op(u32 a, u32 b, u32 c, u32& aux) {
  u32 r;
  if constexpr (M == 0) {  // LOP3
    asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  } else if constexpr (M == 1) {  // SEL on a loop-invariant predicate
    asm volatile("{.reg .pred p; setp.ne.u32 p, %2, 0; selp.b32 %0, %1, %3, p;}" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  } else if constexpr (M == 2) {  // ISETP + SEL (predicate from the chain value)
    asm volatile("{.reg .pred p; setp.lt.u32 p, %1, %2; selp.b32 %0, %1, %3, p;}" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  } else if constexpr (M == 3) {  // 64-bit add of chain values: IADD3 + IADD3.X / IMAD.X
    asm volatile("{add.cc.u32 %0, %1, %2; addc.u32 %3, %3, %1;}" : "=r"(r), "+r"(aux) : "r"(a), "r"(b));
  } else if constexpr (M == 4) {  // funnel shift (SHF.R.U64-style)
    asm volatile("shf.r.clamp.b32 %0, %1, %2, 23;" : "=r"(r) : "r"(a), "r"(b));
  } else if constexpr (M == 5) {  // LOP3 with a predicate result + predicated LOP3
    asm volatile("{.reg .pred p; .reg .b32 t; lop3.b32 t, %1, %2, %3, 0x80; setp.ne.u32 p, t, 0;"
                 " mov.b32 %0, %1; @p lop3.b32 %0, %1, %2, %3, 0xF2;}" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  } else if constexpr (M == 6) {  // IMAD
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
  } else if constexpr (M == 7) {  // 3:2 ALU:IMAD mix (LOP3, LOP3, SEL | IMAD, IMAD)
    u32 t0, t1;
    asm volatile("lop3.b32 %0, %1, %2, %3, 0x96;" : "=r"(t0) : "r"(a), "r"(b), "r"(c));
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t1) : "r"(t0), "r"(b), "r"(c));
    asm volatile("lop3.b32 %0, %1, %2, %3, 0xF8;" : "=r"(t0) : "r"(t1), "r"(b), "r"(a));
    asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(t1) : "r"(t0), "r"(c), "r"(b));
    asm volatile("{.reg .pred p; setp.ne.u32 p, %2, 0; selp.b32 %0, %1, %3, p;}" : "=r"(r) : "r"(t1), "r"(b), "r"(c));
  } else {  // BREV
    asm volatile("brev.b32 %0, %1;" : "=r"(r) : "r"(a));
  }
  return r;
}

template <int M>
__global__ void __launch_bounds__(256) bench(u32* out, u32 iters, u32 b, u32 c) {
  u32 x[8], aux[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) { x[k] = threadIdx.x * 8 + k + blockIdx.x; aux[k] = k; }
  for (u32 i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < 16; ++j) {
#pragma unroll
      for (int k = 0; k < 8; ++k) x[k] = op<M>(x[k], b, c, aux[k]);
    }
  }
  u32 s = 0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s ^= x[k] ^ aux[k];
  if (s == 0x12345678u) out[0] = s;
}

template <int M>
void run(const char* name, int sms, u32 iters, int ops_per) {
  u32* out;
  cudaMalloc(&out, 4);
  const int blocks = sms * 8, threads = 256;
  bench<M><<<blocks, threads>>>(out, 16, 3u, 5u);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  float best = 1e30f;
  for (int rep = 0; rep < 5; ++rep) {
    cudaEventRecord(e0);
    bench<M><<<blocks, threads>>>(out, iters, 3u, 5u);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    if (ms < best) best = ms;
  }
  const double calls = (double)blocks * threads * iters * 16 * 8;
  printf("%-34s %.3e calls/s  %.3e SASS-level ops/s (x%d)  %.3f ms\n", name, calls / (best / 1e3),
         calls * ops_per / (best / 1e3), ops_per, best);
  cudaFree(out);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const u32 it = 2048;
  run<0>("lop3", sms, it, 1);
  run<1>("sel (invariant predicate)", sms, it, 1);
  run<2>("isetp+sel", sms, it, 2);

  run<4>("funnel shf", sms, it, 1);
  run<5>("lop3->p + predicated lop3", sms, it, 2);
  run<6>("imad", sms, it, 1);
  run<7>("mix 3 alu : 2 imad", sms, it, 5);
  run<8>("brev", sms, it / 4, 1);
  return 0;
}
