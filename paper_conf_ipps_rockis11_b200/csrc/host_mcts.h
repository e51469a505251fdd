// host_mcts.h — the CPU side of the hybrid CPU/GPU search (§III-A,
// L312-L339: "the GPU kernel is called asynchronously and the control is given
// back to CPU. Then CPU operates on the same tree ... or trees ... to increase
// their depth"). With device-resident GPU trees the host cannot cheaply walk
// the GPU's trees, so the host threads grow their own trees from the same root
// at one simulation per iteration (the paper's CPU MCTS, L185-L186) while the
// GPU kernel runs, and the root statistics of all trees are summed (L199-L202).
// Semantics per tree are exactly the device UCT's with unit = 1 (R1-R10).
#pragma once
#include <cstdint>
#include <vector>

namespace mcts_host {

struct HostSearchArgs {
  uint64_t own, opp;           // root, side to move first
  uint64_t seed;
  double C;
  uint32_t n_trees;            // host trees (one per thread when time-limited)
  uint32_t tree_id_base;       // Philox c0 of tree t = tree_id_base + t
  uint64_t iterations;         // per tree (iteration mode), or the cap (time mode)
  int64_t deadline_ns;         // steady_clock deadline in ns since epoch, 0 = iteration mode
  uint32_t threads;            // worker threads
  const double* lnT;           // lnT[k] = RN(ln k), k <= iterations (from the device ln table)
};

// Runs the host trees; writes MCTS_STATS_LEN (202) int64 sums into stats.
void search(const HostSearchArgs& a, int64_t* stats);

}  // namespace mcts_host
