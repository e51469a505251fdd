// hosted.cpp — CPU-managed block-parallel trees with GPU simulation and the
// hybrid CPU-GPU processing of PAPER.md §III-A (see hosted.h).
//
// Host threads own disjoint sets of trees (thread 0 is the caller, which also
// drives the GPU). The trees run in two halves pipelined on the GPU; per half
// and step: select (its GPU leaves into the pinned leaf buffer) -> GPU
// playouts || CPU iterations on the same trees -> backpropagation, phases
// separated by spin barriers, and one half's host phases overlap the other
// half's kernel (see run()). The UCB arithmetic is R1's five IEEE
// round-to-nearest operations (the library is built with -ffp-contract=off).
#include "hosted.h"
#include "host_rules.h"
#include "../../include/mcts.h"

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <thread>
#include <vector>

namespace mcts_hosted {
namespace {

using namespace host_rules;

int64_t now_ns() { return std::chrono::steady_clock::now().time_since_epoch().count(); }

struct Tree {
  std::vector<u64> own, opp, lg, n, w, d;
  std::vector<u32> first;
  std::vector<uint8_t> nchild, limit, move, term;
  std::vector<u32> gpath, cpath;  // the pending GPU leaf's path; scratch for CPU iterations
  u64 cpu_count = 0, cpu_plies = 0, cpu_depth = 0, cpu_nodes = 0, gpu_nodes = 0;
  u64 depth_sum = 0, iterations = 0;

  u32 add(u64 o, u64 p, u32 mv) {
    const u64 l = legal(o, p);
    const bool t = l == 0 && legal(p, o) == 0;
    own.push_back(o); opp.push_back(p); lg.push_back(l);
    n.push_back(0); w.push_back(0); d.push_back(0);
    first.push_back(0xFFFFFFFFu); nchild.push_back(0);
    limit.push_back(t ? 0 : (l ? (uint8_t)popc(l) : 1));
    move.push_back((uint8_t)mv); term.push_back(t ? 1 : 0);
    return (u32)(own.size() - 1);
  }
};

// u = w/n + C*sqrt(ln N / n), R1's order, each operation rounded to nearest.
inline double ucb(u64 w, u64 n, double lnN, double C) {
  const double exploit = (double)w / (double)n;
  const double ratio = lnN / (double)n;
  const double root = std::sqrt(ratio);
  const double explore = C * root;
  return exploit + explore;
}

// Selection (L157-L178; a pending child, n = 0, is unvisited: taken first)
// and expansion (L179-L182: the lowest-index untried move or the pass child)
// of one iteration; the path root..leaf goes to `path`. Returns the leaf.
u32 select_expand(Tree& T, const Args& a, std::vector<u32>& path, bool* expanded) {
  path.clear();
  u32 v = 0;
  path.push_back(v);
  while (!T.term[v] && T.nchild[v] >= T.limit[v]) {
    const u32 f = T.first[v];
    const double lnN = a.lnT[T.n[v]];
    u32 best = f;
    double bu = -INFINITY;
    for (u32 i = 0; i < T.nchild[v]; ++i) {
      const u32 c = f + i;
      if (T.n[c] == 0) { best = c; break; }
      const double u = ucb(T.w[c], T.n[c], lnN, a.C);
      if (u > bu) { bu = u; best = c; }
    }
    v = best;
    path.push_back(v);
  }
  *expanded = false;
  if (!T.term[v]) {
    if (T.nchild[v] == 0) {  // reserve the children's contiguous block
      const u32 lim = T.limit[v];
      const u32 f = (u32)T.own.size();
      for (u32 i = 0; i < lim; ++i) T.add(0, 0, 0);
      T.first[v] = f;
    }
    const u32 c = T.first[v] + T.nchild[v];
    const u64 o = T.own[v], p = T.opp[v], l = T.lg[v];
    u64 co, cp;
    u32 mv;
    if (l == 0) { co = p; cp = o; mv = 64; }
    else {
      const int sq = kth_bit(l, T.nchild[v]);
      const u64 fl = flips(sq, o, p);
      co = p & ~fl; cp = o | fl | (1ULL << sq); mv = (u32)sq;
    }
    const u64 cl = legal(co, cp);
    const bool ct = cl == 0 && legal(cp, co) == 0;
    T.own[c] = co; T.opp[c] = cp; T.lg[c] = cl; T.move[c] = (uint8_t)mv; T.term[c] = ct ? 1 : 0;
    T.limit[c] = ct ? 0 : (cl ? (uint8_t)popc(cl) : 1);
    T.nchild[v] += 1;
    path.push_back(c);
    v = c;
    *expanded = true;
  }
  return v;
}

// Backpropagation (L196-L199): W/D/Lo for the leaf's side to move; the leaf's
// mover collects Lo, its parent W, alternating to the root.
void backprop(Tree& T, const std::vector<u32>& path, u64 count, u64 W, u64 D, u64 Lo) {
  u64 mover = Lo, other = W;
  for (size_t i = path.size(); i-- > 0;) {
    const u32 x = path[i];
    T.n[x] += count; T.w[x] += mover; T.d[x] += D;
    std::swap(mover, other);
  }
}

// One CPU iteration on tree t (one host playout).
void cpu_iteration(Tree& T, const Args& a, u32 t) {
  bool e = false;
  const u32 v = select_expand(T, a, T.cpath, &e);
  T.cpu_nodes += e ? 1 : 0;
  int r;
  if (T.term[v]) {
    const int x = popc(T.own[v]), y = popc(T.opp[v]);
    r = (x > y) - (x < y);
  } else {
    r = playout(T.own[v], T.opp[v], a.seed, a.tree_id_base + t, 0x80000000u + (u32)T.cpu_count, 0u,
                &T.cpu_plies);
  }
  backprop(T, T.cpath, 1, r > 0, r == 0, r < 0);
  T.cpu_count += 1;
  T.cpu_depth += T.cpath.size() - 1;
  T.depth_sum += T.cpath.size() - 1;
  T.iterations += 1;
}

enum Cmd : int { kSelect = 1, kCpu = 2, kBackprop = 3, kExit = 4 };

struct Pool {
  std::atomic<int> gen{0};
  std::atomic<int> cmd{0};
  std::atomic<int> arrived{0};
  std::atomic<int> gpu_done{0};
  std::atomic<int> slot{0};       // the half whose kernel the CPU phase overlaps
  std::atomic<u32> lo{0}, hi{0};  // the phase's tree range
  std::atomic<u64> max_root_n{0};
};

}  // namespace

int run(const Args& a, const Gpu& gpu, int64_t* stats, Info* info) {
  for (int i = 0; i < MCTS_STATS_LEN; ++i) stats[i] = 0;
  *info = Info{};
  std::vector<Tree> trees(a.n_trees);
  for (Tree& T : trees) T.add(a.own, a.opp, 0xFF);
  if (a.n_trees == 0 || trees[0].term[0]) return 0;
  const u32 nthreads = std::max<u32>(1, std::min<u32>(a.threads, a.n_trees));
  const bool timed = a.deadline_ns != 0;
  Pool P;
  int gpu_err = 0;

  // The trees are processed in two halves that alternate on the GPU (one
  // stream, so the device runs them back to back): while half A's kernel
  // runs, the host selects half B's leaves and submits them, then runs the
  // CPU iterations of half A, waits for A and backpropagates it, selects and
  // submits A's next step, and so on. Every tree still sees select -> its
  // kernel || its CPU iterations -> backprop, in that order and with the same
  // streams, so results are unchanged; the host's sequential part
  // now overlaps the other half's kernel instead of idling the GPU.
  const u32 nh = a.n_trees >= 2 ? 2u : 1u;
  const u32 split = nh == 2 ? (a.n_trees + 1) / 2 : a.n_trees;
  const u32 lo_of[2] = {0u, split}, hi_of[2] = {split, a.n_trees};

  // the work of phase `c` on trees [P.lo, P.hi) for thread `w` (trees lo + w,
  // lo + w + T, ...; CPU iterations in time mode: threads 1..T-1)
  auto work = [&](int c, u32 w) {
    const u32 lo = P.lo.load(std::memory_order_relaxed), hi = P.hi.load(std::memory_order_relaxed);
    if (c == kSelect) {
      for (u32 t = lo + w; t < hi; t += nthreads) {
        Tree& T = trees[t];
        bool e = false;
        const u32 v = select_expand(T, a, T.gpath, &e);
        T.gpu_nodes += e ? 1 : 0;
        gpu.leaves[t] = LeafRec{T.own[v], T.opp[v], 0u, 0u};  // black = side to move: to_move 0
      }
    } else if (c == kCpu) {
      if (a.cpu_iters == 0) return;
      if (!timed) {
        for (u32 t = lo + w; t < hi; t += nthreads)
          for (u32 j = 0; j < a.cpu_iters; ++j) cpu_iteration(trees[t], a, t);
        return;
      }
      // time mode: the driving thread only polls the GPU, so the half ends as
      // soon as its kernel does (a host iteration in progress on thread 0
      // would hold the pipeline back); threads 1..T-1 iterate round-robin
      // over the half's trees while the kernel runs
      if (w == 0) {
        const int slot = P.slot.load(std::memory_order_relaxed);
        for (;;) {
          const int dn = gpu.done(gpu.ctx, slot);
          if (dn != 0) {
            if (dn < 0) gpu_err = dn;
            P.gpu_done.store(1, std::memory_order_release);
            return;
          }
        }
      }
      const u32 nw = nthreads - 1;
      if (lo + w - 1 >= hi) return;
      for (u32 t = lo + w - 1;; t += nw) {
        if (t >= hi) t = lo + w - 1;
        if (P.gpu_done.load(std::memory_order_acquire)) break;
        cpu_iteration(trees[t], a, t);
      }
    } else if (c == kBackprop) {
      u64 mx = 0;
      for (u32 t = lo + w; t < hi; t += nthreads) {
        Tree& T = trees[t];
        const WdlRec r = gpu.wdl[t];
        backprop(T, T.gpath, a.unit, r.wins, r.draws, r.losses);
        T.depth_sum += T.gpath.size() - 1;
        T.iterations += 1;
        mx = std::max<u64>(mx, T.n[0]);
      }
      u64 cur = P.max_root_n.load();
      while (mx > cur && !P.max_root_n.compare_exchange_weak(cur, mx)) {}
    }
  };

  std::vector<std::thread> helpers;
  for (u32 w = 1; w < nthreads; ++w) {
    helpers.emplace_back([&, w]() {
      int seen = 0;
      for (;;) {
        int g;
        while ((g = P.gen.load(std::memory_order_acquire)) == seen) std::this_thread::yield();
        seen = g;
        const int c = P.cmd.load(std::memory_order_relaxed);
        if (c == kExit) return;
        work(c, w);
        P.arrived.fetch_add(1, std::memory_order_acq_rel);
      }
    });
  }
  auto phase = [&](int c, u32 half) {  // run phase c on half `half` on every thread (the caller is thread 0)
    P.lo.store(lo_of[half], std::memory_order_relaxed);
    P.hi.store(hi_of[half], std::memory_order_relaxed);
    P.arrived.store(0, std::memory_order_relaxed);
    P.cmd.store(c, std::memory_order_relaxed);
    P.gen.fetch_add(1, std::memory_order_acq_rel);
    work(c, 0);
    while (P.arrived.load(std::memory_order_acquire) < (int)nthreads - 1) std::this_thread::yield();
  };
  // another step may start: budget, deadline, and the ln table covers every
  // parent count its selections can read (the root's count plus the step's
  // CPU iterations)
  auto may_start = [&](u64 step) {
    if (step >= a.steps) return false;
    if (timed && now_ns() >= a.deadline_ns) return false;
    return P.max_root_n.load() + (timed ? 1000000ull : (u64)a.cpu_iters) < a.lnT_size;
  };
  auto launch = [&](u32 half, u64 step) {  // select the half's leaves and submit its kernel
    const int64_t t0 = now_ns();
    phase(kSelect, half);
    info->select_ms += (now_ns() - t0) * 1e-6;
    if (gpu.submit(gpu.ctx, lo_of[half], hi_of[half] - lo_of[half], (u32)step, (int)half) < 0) gpu_err = -1;
    return gpu_err == 0;
  };
  auto finish = [&](u32 half) {  // CPU iterations while its kernel runs, then its backprop
    const int64_t t0 = now_ns();
    P.slot.store((int)half, std::memory_order_relaxed);
    P.gpu_done.store(0, std::memory_order_release);
    phase(kCpu, half);
    if (!gpu_err && !P.gpu_done.load(std::memory_order_acquire)) {
      const int r = gpu.wait(gpu.ctx, (int)half);
      if (r < 0) gpu_err = r;
    }
    if (gpu_err) return false;
    const int64_t t1 = now_ns();
    phase(kBackprop, half);
    info->gpu_ms += (t1 - t0) * 1e-6;
    info->backprop_ms += (now_ns() - t1) * 1e-6;
    return true;
  };

  u64 s = 0;
  if (may_start(0) && launch(0, 0)) {
    for (;;) {  // step s: half 0 is in flight
      if (nh == 2 && !launch(1, s)) break;
      if (!finish(0)) break;
      if (nh == 2) {
        const bool more = may_start(s + 1);
        if (more && !launch(0, s + 1)) break;
        if (!finish(1)) break;
        ++s;
        if (!more) break;
      } else {
        ++s;
        if (!may_start(s) || !launch(0, s)) break;
      }
    }
  }
  P.cmd.store(kExit, std::memory_order_relaxed);
  P.gen.fetch_add(1, std::memory_order_acq_rel);
  for (auto& th : helpers) th.join();
  if (gpu_err) return gpu_err;

  info->steps = s;
  for (const Tree& T : trees) {
    const u32 f = T.first[0];
    for (u32 i = 0; i < T.nchild[0]; ++i) {
      const u32 c = f + i;
      stats[T.move[c]] += (int64_t)T.n[c];
      stats[65 + T.move[c]] += (int64_t)T.w[c];
      stats[130 + T.move[c]] += (int64_t)T.d[c];
    }
    stats[195] += (int64_t)T.n[0];
    stats[196] += (int64_t)T.iterations;
    stats[197] += (int64_t)T.cpu_plies;  // + the kernel's plies (counted on the device)
    stats[198] += (int64_t)T.depth_sum;
    // nodes created (reserved child blocks are not counted)
    stats[200] += (int64_t)(1 + T.cpu_nodes + T.gpu_nodes);
    info->cpu_iterations += T.cpu_count;
    info->cpu_plies += T.cpu_plies;
    info->cpu_depth_sum += T.cpu_depth;
    info->cpu_nodes += T.cpu_nodes;
    info->gpu_nodes += T.gpu_nodes;
  }
  return 0;
}

}  // namespace mcts_hosted
