// hosted_emul.cpp — TEST HARNESS (tests/test_hosted_host.py): drives the
// product's host half of mcts_search_hosted (csrc/hosted.cpp, the CPU-managed
// trees of PAPER.md L302-L303 / Fig. 4) with the GPU step replaced by the same
// playouts computed on the host (the library's host playout, streams c0 = tree,
// c1 = step, c2 = thread), so the tree logic can be checked against the oracle
// without a GPU. The ln table comes from the caller (the oracle's, in the test).
#include "../../paper_conf_ipps_rockis11_b200/csrc/hosted.h"
#include "../../paper_conf_ipps_rockis11_b200/csrc/host_rules.h"
#include "../../include/mcts.h"
#include <vector>

using namespace mcts_hosted;

namespace {
struct Ctx { LeafRec* leaves; WdlRec* wdl; uint64_t seed; uint32_t unit; uint64_t plies; };

int submit(void* c, uint32_t first, uint32_t n, uint32_t step, int) {
  Ctx* x = (Ctx*)c;
  for (uint32_t t = first; t < first + n; ++t) {
    uint32_t w = 0, d = 0, l = 0;
    for (uint32_t j = 0; j < x->unit; ++j) {
      const int r = host_rules::playout(x->leaves[t].black, x->leaves[t].white, x->seed, t, step, j, &x->plies);
      if (r > 0) ++w; else if (r == 0) ++d; else ++l;
    }
    x->wdl[t] = {w, d, l};
  }
  return 0;
}
int done(void*, int) { return 1; }
int wait(void*, int) { return 0; }
}  // namespace

extern "C" int hosted_emul(uint64_t own, uint64_t opp, uint32_t n_trees, uint32_t unit, uint64_t steps,
                           uint32_t cpu_iters, uint64_t seed, double C, uint32_t threads, const double* lnT,
                           uint64_t lnT_size, int64_t* stats, uint64_t* info6) {
  std::vector<LeafRec> leaves(n_trees);
  std::vector<WdlRec> wdl(n_trees);
  Ctx ctx{leaves.data(), wdl.data(), seed, unit, 0};
  Gpu g{&ctx, submit, done, wait, leaves.data(), wdl.data()};
  Args a{own, opp, seed, C, n_trees, 0, unit, steps, cpu_iters, 0, threads, lnT, lnT_size};
  Info info;
  const int r = run(a, g, stats, &info);
  stats[197] += (int64_t)ctx.plies;  // the "kernel's" plies, as mcts_search_hosted adds them
  info6[0] = info.steps; info6[1] = info.cpu_iterations; info6[2] = info.cpu_plies;
  info6[3] = info.cpu_depth_sum; info6[4] = info.cpu_nodes; info6[5] = info.gpu_nodes;
  return r;
}
