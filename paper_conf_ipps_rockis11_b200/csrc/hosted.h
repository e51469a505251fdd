// hosted.h — block parallelism with CPU-managed trees and the hybrid CPU-GPU
// processing of PAPER.md §III-A (L312-L339, Fig. 4), the paper's own design:
// "The trees are still controlled by the CPU threads, GPU simulates only"
// (L302-L303). DESIGN.md reading R18.
//
// Per step s, for every tree t (host threads own disjoint sets of trees):
//   1. the host selects and expands the tree's leaf (UCT, R1; a child with
//      n = 0 — a leaf whose GPU result is pending — is an unvisited arm);
//   2. ONE kernel simulates threads_per_tree playouts from every tree's leaf
//      (the playouts kernel, streams c0 = tree id, c1 = s, c2 = thread: the
//      device block search's iteration-s streams);
//   3. while it runs ("CPU can work here!", Fig. 4) the host threads run UCT
//      iterations with one host playout each on the SAME trees (streams c0 =
//      tree id, c1 = 0x80000000 + the tree's CPU iteration count, c2 = 0):
//      exactly cpu_iters per tree per step in iteration mode, as many as fit
//      while the kernel runs in time mode (cpu_iters > 0; there thread 0 only
//      drives the GPU and threads 1..T-1 iterate, so the host work never
//      delays the next step);
//   4. the host backpropagates the kernel's W/D/L along each tree's path.
// Iteration mode is deterministic and bit-exact to the oracle's
// orc_hybrid_search; with cpu_iters = 0 it is the block search bit for bit.
#pragma once
#include <cstdint>

namespace mcts_hosted {

struct LeafRec {  // layout of mcts_position
  uint64_t black, white;
  uint32_t to_move, reserved;
};
struct WdlRec {  // layout of mcts_wdl
  uint32_t wins, draws, losses;
};

// The GPU side, provided by mcts_api.cu: submit() copies the leaves of trees
// [first, first + n) (pinned host) to the device, launches the playouts kernel
// for them at step `step` (streams c0 = tree id) and copies their W/D/L back
// into the pinned `wdl` buffer, all asynchronously, completion tracked in
// `slot` (0 or 1: the two pipelined halves, run in submission order); done()
// polls a slot (1 = finished, 0 = running, < 0 = CUDA error); wait() blocks.
struct Gpu {
  void* ctx;
  int (*submit)(void* ctx, uint32_t first, uint32_t n, uint32_t step, int slot);
  int (*done)(void* ctx, int slot);
  int (*wait)(void* ctx, int slot);
  LeafRec* leaves;    // pinned, n_trees
  const WdlRec* wdl;  // pinned, n_trees
};

struct Args {
  uint64_t own, opp;      // root, side to move first
  uint64_t seed;
  double C;
  uint32_t n_trees, tree_id_base, unit;
  uint64_t steps;         // iteration mode: GPU steps; time mode: cap
  uint32_t cpu_iters;     // iteration mode: CPU iterations per tree per step; time mode: 0 = none, else on
  int64_t deadline_ns;    // steady_clock ns since epoch; 0 = iteration mode
  uint32_t threads;       // host worker threads
  const double* lnT;      // lnT[N] = RN(ln N), N < lnT_size
  uint64_t lnT_size;
};

struct Info {
  uint64_t steps, cpu_iterations, cpu_plies, cpu_depth_sum, cpu_nodes, gpu_nodes;
  double select_ms, gpu_ms, backprop_ms;
};

// Runs the search; writes MCTS_STATS_LEN int64 sums to stats (GPU plies are
// added by the caller: the kernel counts them on the device). Returns 0, or a
// negative value if the GPU side failed.
int run(const Args& a, const Gpu& gpu, int64_t* stats, Info* info);

}  // namespace mcts_hosted
