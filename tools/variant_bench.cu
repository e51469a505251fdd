// variant_bench.cu — time the configs[1] playout batch through the C ABI of one
// or more libmcts.so builds (dlopen'ed side by side), CUDA events on a stream.
// Tooling for kernel tuning; not part of the product.
//   nvcc -O2 -o tools/variant_bench tools/variant_bench.cu -ldl
//   tools/variant_bench lib1.so [lib2.so ...]
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include "../include/mcts.h"

typedef mcts_status (*create_t)(const mcts_position*, const mcts_params*, mcts_handle**);
typedef mcts_status (*gen_t)(mcts_handle*, uint64_t, uint32_t, uint32_t, uint32_t, mcts_position*, void*);
typedef mcts_status (*play_t)(mcts_handle*, const mcts_position*, uint32_t, uint32_t, uint64_t, uint32_t,
                              mcts_wdl*, uint64_t*, void*);
typedef void (*destroy_t)(mcts_handle*);

int main(int argc, char** argv) {
  const uint32_t n = 4096, per = 256;
  mcts_position* d_leaves;
  mcts_wdl* d_out;
  uint64_t* d_plies;
  cudaMalloc(&d_leaves, n * sizeof(mcts_position));
  cudaMalloc(&d_out, n * sizeof(mcts_wdl));
  cudaMalloc(&d_plies, 8);
  void* flush;
  cudaMalloc(&flush, 256u << 20);
  cudaStream_t s;
  cudaStreamCreate(&s);
  for (int a = 1; a < argc; ++a) {
    void* lib = dlopen(argv[a], RTLD_NOW | RTLD_LOCAL);
    if (!lib) { printf("%s: dlopen failed: %s\n", argv[a], dlerror()); continue; }
    create_t create = (create_t)dlsym(lib, "mcts_create");
    gen_t gen = (gen_t)dlsym(lib, "mcts_gen_positions_async");
    play_t play = (play_t)dlsym(lib, "mcts_playouts_async");
    destroy_t destroy = (destroy_t)dlsym(lib, "mcts_destroy");
    mcts_params p = {1.0, MCTS_BLOCK, 0, 0, 0};
    mcts_handle* h = nullptr;
    if (create(nullptr, &p, &h)) { printf("%s: create failed\n", argv[a]); continue; }
    gen(h, 2, n, 20, 40, d_leaves, s);
    for (int i = 0; i < 5; ++i) play(h, d_leaves, n, per, 2, 0, d_out, d_plies, s);
    cudaStreamSynchronize(s);
    std::vector<float> ms;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int i = 0; i < 20; ++i) {
      cudaMemsetAsync(flush, i, 256u << 20, s);
      cudaEventRecord(e0, s);
      play(h, d_leaves, n, per, 2, 0, d_out, d_plies, s);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
      float t;
      cudaEventElapsedTime(&t, e0, e1);
      ms.push_back(t);
    }
    float sum = 0, best = 1e9;
    for (float t : ms) { sum += t; if (t < best) best = t; }
    // Checksum of every leaf's W/D/L (FNV-1a): variants must agree bit-exactly.
    std::vector<mcts_wdl> w(n);
    cudaMemcpy(w.data(), d_out, n * sizeof(mcts_wdl), cudaMemcpyDeviceToHost);
    uint64_t hsh = 1469598103934665603ULL;
    for (const mcts_wdl& x : w)
      for (uint32_t v : {x.wins, x.draws, x.losses}) { hsh ^= v; hsh *= 1099511628211ULL; }
    printf("%-60s mean %.4f ms  best %.4f ms  %.3e playouts/s  wdl-hash %016llx  leaf0 %u/%u/%u\n", argv[a],
           sum / ms.size(), best, n * (double)per / (sum / ms.size() / 1e3), (unsigned long long)hsh, w[0].wins,
           w[0].draws, w[0].losses);
    destroy(h);
  }
  return 0;
}
