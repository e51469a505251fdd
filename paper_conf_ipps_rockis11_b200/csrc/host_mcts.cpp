// host_mcts.cpp — host-thread UCT trees for the hybrid CPU/GPU search (see
// host_mcts.h). Same rules, RNG streams and UCT arithmetic as the device path
// (R1-R10) with one simulation per iteration; used only by
// mcts_search_hybrid, never as a substitute for the GPU.
#include "host_mcts.h"
#include "host_rules.h"
#include "../../include/mcts.h"

#include <atomic>
#include <chrono>
#include <cmath>
#include <thread>

namespace mcts_host {
namespace {

using namespace host_rules;

struct Tree {
  std::vector<u64> own, opp, lg;
  std::vector<u32> k, w, d, first, nchild, limit, move;
  std::vector<uint8_t> term;
  void add(u64 o, u64 p, u32 mv) {
    const u64 l = legal(o, p);
    const bool t = l == 0 && legal(p, o) == 0;
    own.push_back(o); opp.push_back(p); lg.push_back(l);
    k.push_back(0); w.push_back(0); d.push_back(0);
    first.push_back(0xFFFFFFFFu); nchild.push_back(0);
    limit.push_back(t ? 0u : (l ? (u32)popc(l) : 1u));
    move.push_back(mv); term.push_back(t ? 1 : 0);
  }
};

void run_tree(const HostSearchArgs& a, u32 t, int64_t* st) {
  Tree T;
  T.add(a.own, a.opp, 0xFFu);
  if (T.term[0]) return;
  u64 plies = 0, depth_sum = 0;
  u64 it = 0;
  std::vector<u32> path;
  for (; it < a.iterations; ++it) {
    if (a.deadline_ns && (it & 15u) == 0 &&
        std::chrono::steady_clock::now().time_since_epoch().count() >= a.deadline_ns)
      break;
    path.clear();
    u32 v = 0;
    path.push_back(v);
    while (!T.term[v] && T.nchild[v] >= T.limit[v]) {  // selection
      const double lnp = a.lnT[T.k[v]];
      u32 best = 0;
      double bu = -INFINITY;
      for (u32 i = 0; i < T.nchild[v]; ++i) {
        const u32 c = T.first[v] + i;
        const double n = (double)T.k[c];  // unit = 1: n = k
        const double u = (double)T.w[c] / n + a.C * std::sqrt(lnp / n);
        if (u > bu) { bu = u; best = c; }
      }
      v = best;
      path.push_back(v);
    }
    if (!T.term[v]) {  // expansion: children stored in a reserved contiguous block
      if (T.nchild[v] == 0) {
        T.first[v] = (u32)T.own.size();
        for (u32 i = 0; i < T.limit[v]; ++i) T.add(0, 0, 0);  // placeholders
      }
      const u32 c = T.first[v] + T.nchild[v];
      const u64 o = T.own[v], p = T.opp[v], l = T.lg[v];
      u64 co, cp;
      u32 mv;
      if (l == 0) { co = p; cp = o; mv = 64; }
      else {
        const int sq = kth_bit(l, T.nchild[v]);
        const u64 f = flips(sq, o, p);
        co = p & ~f; cp = o | f | (1ULL << sq); mv = (u32)sq;
      }
      const u64 cl = legal(co, cp);
      const bool ct = cl == 0 && legal(cp, co) == 0;
      T.own[c] = co; T.opp[c] = cp; T.lg[c] = cl; T.move[c] = mv; T.term[c] = ct ? 1 : 0;
      T.limit[c] = ct ? 0u : (cl ? (u32)popc(cl) : 1u);
      T.nchild[v] += 1;
      v = c;
      path.push_back(v);
    }
    depth_sum += path.size() - 1;
    int r;  // simulation (one per iteration)
    if (T.term[v]) {
      const int x = popc(T.own[v]), y = popc(T.opp[v]);
      r = (x > y) - (x < y);
    } else {
      r = playout(T.own[v], T.opp[v], a.seed, a.tree_id_base + t, (u32)it, 0u, &plies);
    }
    u32 mover_wins = r < 0, other_wins = r > 0;  // backpropagation
    const u32 draw = r == 0;
    for (size_t i = path.size(); i-- > 0;) {
      const u32 x = path[i];
      T.k[x] += 1; T.w[x] += mover_wins; T.d[x] += draw;
      std::swap(mover_wins, other_wins);
    }
  }
  // root children -> stats (int64 sums, layout of include/mcts.h MCTS_STATS_LEN)
  for (u32 i = 0; i < T.nchild[0]; ++i) {
    const u32 c = T.first[0] + i;
    st[T.move[c]] += T.k[c];
    st[65 + T.move[c]] += T.w[c];
    st[130 + T.move[c]] += T.d[c];
  }
  st[195] += T.k[0];
  st[196] += (int64_t)it;
  st[197] += (int64_t)plies;
  st[198] += (int64_t)depth_sum;
}

}  // namespace

void search(const HostSearchArgs& a, int64_t* stats) {
  for (int i = 0; i < MCTS_STATS_LEN; ++i) stats[i] = 0;
  const u32 T = a.threads ? a.threads : 1;
  std::vector<std::vector<int64_t>> part(T, std::vector<int64_t>(MCTS_STATS_LEN, 0));
  std::atomic<u32> next{0};
  auto worker = [&](u32 tid) {
    for (;;) {
      const u32 t = next.fetch_add(1);
      if (t >= a.n_trees) break;
      run_tree(a, t, part[tid].data());
    }
  };
  std::vector<std::thread> pool;
  for (u32 i = 1; i < T; ++i) pool.emplace_back(worker, i);
  worker(0);
  for (auto& th : pool) th.join();
  for (u32 i = 0; i < T; ++i)
    for (int j = 0; j < MCTS_STATS_LEN; ++j) stats[j] += part[i][j];
}

}  // namespace mcts_host
