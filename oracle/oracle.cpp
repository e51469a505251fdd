// oracle/oracle.cpp — CPU ORACLE. TEST INFRASTRUCTURE ONLY.
//
// Plain, slow, obviously-correct CPU implementation of what the hot path of
// Rocki & Suda, "Large-Scale Parallel Monte Carlo Tree Search on GPU"
// (IPDPSW 2011) computes: random 8x8 Reversi playouts (PAPER.md L149-L153,
// §II "A simulation is defined as a series of random moves which are performed
// until the end of a game is reached (until neither of the players can move)")
// and the UCT iteration Selection/Expansion/Simulation/Backpropagation
// (§II-A, Fig. 1) run independently per tree and summed at
// the root (L199-L202) — the block-parallel scheme (L294-L311, §III-6) and the
// leaf-parallel scheme (L231-L237, §III-5) are both "n_trees trees, `unit`
// simulations per iteration" in this formulation.
//
// Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference
// legs may load this library. It shares no code, header or table with the CUDA
// path under paper_conf_ipps_rockis11_b200/ (nothing is included from there and
// nothing there includes this).
//
// Readings of the paper where it is silent or garbled are listed in DESIGN.md
// §3 ("Readings"); each function below names the reading it follows.
//
// Parity pins (tests/test_oracle_*.py): perft from the opening (north_star),
// an independent Python mailbox/ray-walk cross-check, the 8 board symmetries,
// Random123 Philox known-answer vectors, closed-form pick-bucket counts, the
// exact random-play outcome distribution of small endgames, a 45-digit decimal
// ln reference, high-precision UCB values, a hand trace of the first UCT
// iterations (incl. the depth sum of the paper's Fig. 8 "Depth", L490-L511),
// tree invariants, depth sum = sum of non-root visits / unit, the
// multi-tree merge identity, the UCB operation order (R1) against five
// re-orderings, and the CPU opponent (orc_mcts_timed, iteration-capped) equal
// to the iteration-mode search bit for bit.
//
// Deliberately NOT tuned: move generation walks every empty square in every
// direction with (row, col) coordinates; every RNG word recomputes Philox.

#include <cstdint>
#include <cstring>
#include <cmath>
#include <vector>
#include <thread>
#include <algorithm>
#include <chrono>
#include <atomic>
#include <quadmath.h>

extern "C" {
typedef struct {
  uint64_t black, white;
  uint32_t to_move;   // 0 = black to move, 1 = white to move
  uint32_t reserved;
} orc_position;
}

namespace {

// ---------------------------------------------------------------------------
// Board rules (standard Othello; the paper only fixes the end condition,
// PAPER.md L150-L151).  Square s = 8*row + col, bit s of a uint64 mask.
// DESIGN.md reading R7 (board, colours, first player).
// ---------------------------------------------------------------------------
const int DR[8] = {-1, -1, -1, 0, 0, 1, 1, 1};
const int DC[8] = {-1, 0, 1, -1, 1, -1, 0, 1};

inline uint64_t sqbit(int r, int c) { return 1ULL << (8 * r + c); }
inline bool inside(int r, int c) { return r >= 0 && r < 8 && c >= 0 && c < 8; }
inline bool has(uint64_t b, int r, int c) { return (b & sqbit(r, c)) != 0; }

// Discs of `opp` flipped when the side owning `own` plays on square sq:
// in each direction, a run of >= 1 opponent discs ended by an own disc.
uint64_t flips(uint64_t own, uint64_t opp, int sq) {
  int r0 = sq / 8, c0 = sq % 8;
  if (has(own | opp, r0, c0)) return 0;
  uint64_t all = 0;
  for (int d = 0; d < 8; ++d) {
    uint64_t run = 0;
    int r = r0 + DR[d], c = c0 + DC[d];
    while (inside(r, c) && has(opp, r, c)) {
      run |= sqbit(r, c);
      r += DR[d];
      c += DC[d];
    }
    if (run != 0 && inside(r, c) && has(own, r, c)) all |= run;
  }
  return all;
}

// Legal squares: empty squares whose placement flips at least one disc.
uint64_t legal(uint64_t own, uint64_t opp) {
  uint64_t m = 0;
  for (int s = 0; s < 64; ++s)
    if (flips(own, opp, s) != 0) m |= 1ULL << s;
  return m;
}

int popcount64(uint64_t x) {
  int c = 0;
  for (int s = 0; s < 64; ++s) c += (int)((x >> s) & 1);
  return c;
}

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., SC'11; the cuRAND/Random123 round).
// DESIGN.md reading R5 (RNG).
// ---------------------------------------------------------------------------
void philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c[4] = {ctr_in[0], ctr_in[1], ctr_in[2], ctr_in[3]};
  uint32_t k[2] = {key_in[0], key_in[1]};
  for (int round = 0; round < 10; ++round) {
    uint64_t p0 = (uint64_t)0xD2511F53u * c[0];
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c[2];
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c[1] ^ k[0];
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c[3] ^ k[1];
    uint32_t n3 = lo0;
    c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
    k[0] += 0x9E3779B9u;
    k[1] += 0xBB67AE85u;
  }
  out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

// Word w of the stream with counter prefix (c0, c1, c2) and key = seed:
// counter = (c0, c1, c2, w / 4), word = output[w % 4]  (reading R5).
uint32_t rng_word(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t w) {
  uint32_t ctr[4] = {c0, c1, c2, w / 4};
  uint32_t key[2] = {(uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)};
  uint32_t out[4];
  philox4x32_10(ctr, key, out);
  return out[w % 4];
}

// Uniform pick among c legal moves (reading R4): k = floor(r * c / 2^32),
// then the k-th legal square in ascending index order (k = 0 is the lowest).
int pick(uint64_t moves, uint32_t r) {
  uint32_t c = (uint32_t)popcount64(moves);
  uint32_t k = (uint32_t)(((uint64_t)r * c) >> 32);
  uint32_t seen = 0;
  for (int s = 0; s < 64; ++s) {
    if ((moves >> s) & 1) {
      if (seen == k) return s;
      ++seen;
    }
  }
  return -1;  // moves == 0: caller never asks
}

// Random playout from (own to move, opp). PAPER.md L149-L153: random moves
// until neither player can move; the result is judged for the player to move
// at the start (reading R3: +1 win, 0 draw, -1 loss by disc count).
// Passes consume no RNG word; every decision with >= 1 legal move consumes
// exactly one (reading R5).
int playout(uint64_t own, uint64_t opp, uint64_t seed, uint32_t c0, uint32_t c1,
            uint32_t c2, uint32_t* plies_out) {
  uint64_t me = own, op = opp;
  bool start_to_move = true;  // is `me` the player who moved first?
  uint32_t w = 0, plies = 0;
  for (;;) {
    uint64_t moves = legal(me, op);
    if (moves == 0) {
      if (legal(op, me) == 0) break;  // neither player can move: game over
      std::swap(me, op);              // pass
      start_to_move = !start_to_move;
      continue;
    }
    uint32_t r = rng_word(seed, c0, c1, c2, w);
    ++w;
    int sq = pick(moves, r);
    uint64_t f = flips(me, op, sq);
    me |= f | (1ULL << sq);
    op &= ~f;
    std::swap(me, op);
    start_to_move = !start_to_move;
    ++plies;
  }
  uint64_t a = start_to_move ? me : op;
  uint64_t b = start_to_move ? op : me;
  if (plies_out) *plies_out += plies;
  int da = popcount64(a), db = popcount64(b);
  return da > db ? 1 : (da == db ? 0 : -1);
}

void to_own_opp(const orc_position& p, uint64_t* own, uint64_t* opp) {
  if (p.to_move == 0) { *own = p.black; *opp = p.white; }
  else { *own = p.white; *opp = p.black; }
}

// ---------------------------------------------------------------------------
// ln table (reading R9): lnT[k] = RN(ln(k * unit)), correctly rounded.
// Oracle form: the binary128 library logarithm rounded once to double.
// ---------------------------------------------------------------------------
double ln_rn(uint64_t x) {
  __float128 q = logq((__float128)x);
  return (double)q;
}

// ---------------------------------------------------------------------------
// UCT. Reading R1 (UCB1 formula), R2 (draws), R6
// (expansion order, pass child), R8 (final move), R10 (unit per iteration).
// ---------------------------------------------------------------------------
struct Node {
  uint64_t own, opp;   // side to move's discs, the other side's discs
  int move;            // move into this node: 0..63, 64 = pass, -1 = root
  int parent;
  uint64_t n, w, d;    // simulations through node, wins of mover(node), draws
  uint64_t legal_moves;
  bool terminal;
  std::vector<int> children;  // expansion order == ascending move index
};

Node make_node(uint64_t own, uint64_t opp, int move, int parent) {
  Node v;
  v.own = own; v.opp = opp; v.move = move; v.parent = parent;
  v.n = v.w = v.d = 0;
  v.legal_moves = legal(own, opp);
  v.terminal = (v.legal_moves == 0) && (legal(opp, own) == 0);
  return v;
}

// Number of children the node can ever have: its legal moves, or one pass child.
int child_limit(const Node& v) {
  if (v.terminal) return 0;
  return v.legal_moves ? popcount64(v.legal_moves) : 1;
}

bool fully_expanded(const Node& v) { return (int)v.children.size() >= child_limit(v); }

// u = w/n + C * sqrt(lnT[N] / n), each operation rounded to nearest, in this
// order, no fused multiply-add (reading R1).
double ucb(uint64_t w, uint64_t n, double ln_parent, double C) {
  double exploit = (double)w / (double)n;
  double ratio = ln_parent / (double)n;
  double root = std::sqrt(ratio);
  double explore = C * root;
  return exploit + explore;
}

struct TreeResult {
  std::vector<Node> nodes;
  uint64_t iterations = 0;
  uint64_t depth_sum = 0;  // sum over iterations of the simulated node's depth (edges from the root)
  uint64_t refused = 0;    // iterations whose expansion the full node pool refused (R12)
};

// One UCT iteration (number `it`) on a tree whose root is nodes[0], with `unit`
// playouts per iteration, playout streams keyed (c0 = tree_id, c1 = it,
// c2 = thread), ln table lnT[k] = RN(ln(k * unit)) indexed by k = parent n / unit.
// Both the iteration-mode search (search_tree) and the CPU opponent
// (orc_mcts_timed) grow their trees with this one function.
void uct_iteration(TreeResult* out, uint64_t it, uint32_t unit, uint64_t seed, uint32_t tree_id,
                   double C, uint64_t capacity, const std::vector<double>& lnT, uint64_t* plies) {
  std::vector<Node>& nodes = out->nodes;
  // 1) Selection (L157-L178): descend through fully expanded nodes.
  std::vector<int> path;
  int v = 0;
  path.push_back(v);
  while (!nodes[v].terminal && fully_expanded(nodes[v])) {
    const Node& p = nodes[v];
    double ln_parent = lnT[p.n / unit];
    int best = -1;
    double best_u = -INFINITY;
    for (int c : p.children) {
      double u = ucb(nodes[c].w, nodes[c].n, ln_parent, C);
      if (u > best_u) { best_u = u; best = c; }
    }
    v = best;
    path.push_back(v);
  }
  // 2) Expansion (L179-L182): one node per iteration, lowest untried move.
  if (!nodes[v].terminal && nodes.size() < capacity) {
    const Node& p = nodes[v];
    int mv;
    uint64_t cown, copp;
    if (p.legal_moves == 0) {
      mv = 64;  // pass child
      cown = p.opp; copp = p.own;
    } else {
      int idx = (int)p.children.size(), seen = 0;
      mv = -1;
      for (int s = 0; s < 64; ++s) {
        if ((p.legal_moves >> s) & 1) {
          if (seen == idx) { mv = s; break; }
          ++seen;
        }
      }
      uint64_t f = flips(p.own, p.opp, mv);
      uint64_t mover = p.own | f | (1ULL << mv);
      uint64_t other = p.opp & ~f;
      cown = other; copp = mover;
    }
    nodes.push_back(make_node(cown, copp, mv, v));
    int c = (int)nodes.size() - 1;
    nodes[v].children.push_back(c);
    v = c;
    path.push_back(v);
  } else if (!nodes[v].terminal) {
    out->refused += 1;  // pool full: simulate from the selected node itself (R12)
  }
  // 3) Simulation (L183-L195): `unit` playouts from the leaf.
  uint64_t wins = 0, draws = 0, losses = 0;  // for the leaf's side to move
  const Node& leaf = nodes[v];
  if (leaf.terminal) {
    int a = popcount64(leaf.own), b = popcount64(leaf.opp);
    if (a > b) wins = unit; else if (a == b) draws = unit; else losses = unit;
  } else {
    for (uint32_t t = 0; t < unit; ++t) {
      uint32_t pl = 0;
      int r = playout(leaf.own, leaf.opp, seed, tree_id, (uint32_t)it, t, &pl);
      *plies += pl;
      if (r > 0) ++wins; else if (r == 0) ++draws; else ++losses;
    }
  }
  out->depth_sum += path.size() - 1;  // the paper's tree depth (Fig. 8)
  // 4) Backpropagation (L196-L199): the leaf's mover is the opponent of the
  // leaf's side to move, so it collects `losses`; roles alternate upwards.
  uint64_t mover_wins = losses, other_wins = wins;
  for (int i = (int)path.size() - 1; i >= 0; --i) {
    Node& x = nodes[path[i]];
    x.n += unit;
    x.w += mover_wins;
    x.d += draws;
    std::swap(mover_wins, other_wins);
  }
  out->iterations = it + 1;
}

// One tree of the search: `iterations` UCT iterations (uct_iteration) from a
// fresh root.
void search_tree(uint64_t root_own, uint64_t root_opp, uint32_t unit, uint64_t iterations,
                 uint64_t seed, uint32_t tree_id, double C, uint64_t capacity,
                 const std::vector<double>& lnT, TreeResult* out, uint64_t* plies_total) {
  std::vector<Node>& nodes = out->nodes;
  nodes.clear();
  nodes.push_back(make_node(root_own, root_opp, -1, -1));
  out->iterations = 0;
  if (nodes[0].terminal) return;
  uint64_t plies = 0;
  for (uint64_t it = 0; it < iterations; ++it)
    uct_iteration(out, it, unit, seed, tree_id, C, capacity, lnT, &plies);
  if (plies_total) *plies_total += plies;
}

// ---------------------------------------------------------------------------
// Hybrid CPU-GPU processing on CPU-managed trees (§III-A,
// Fig. 4), on the block-parallel trees as the paper built them: "The trees are
// still controlled by the CPU threads, GPU simulates only" (L302-L303). DESIGN.md
// reading R18. Per tree, per step s:
//   1. select + expand one leaf (the GPU's leaf of this step);
//   2. GPU: `unit` playouts from it, streams (c0 = tree_id, c1 = s, c2 = 0..unit-1)
//      — the block search's iteration-s streams;
//   3. "CPU can work here!" (Fig. 4): cpu_iters UCT iterations on the SAME tree,
//      one playout each, streams (c0 = tree_id, c1 = 0x80000000 + s*cpu_iters + j, c2 = 0);
//   4. backpropagate step 2's result along step 1's path.
// Selection is R1 with the parent's simulation count N (GPU steps add `unit`,
// CPU iterations 1, so ln is RN(ln N) of any N) and one more rule: a child
// with n = 0 — a leaf whose GPU simulations are still pending — is unvisited,
// scored +inf as in UCB1 (ref [2]), lowest index first.
// ---------------------------------------------------------------------------
struct HybridCounts {
  uint64_t cpu_iterations = 0, cpu_plies = 0, cpu_depth_sum = 0, cpu_nodes = 0, gpu_nodes = 0;
};

double ln_of(std::vector<double>& lnT, uint64_t N) {
  if (N >= lnT.size()) {
    size_t old = lnT.size();
    lnT.resize(std::max<size_t>(N + 1, old * 2));
    for (size_t k = old; k < lnT.size(); ++k) lnT[k] = ln_rn(k);
  }
  return lnT[N];
}

// Steps 1 (and the CPU iterations' selection + expansion): returns the path
// root..leaf; *expanded = 1 if a node was added.
std::vector<int> select_expand_pending(std::vector<Node>& nodes, double C, std::vector<double>& lnT,
                                       int* expanded) {
  std::vector<int> path;
  int v = 0;
  path.push_back(v);
  while (!nodes[v].terminal && fully_expanded(nodes[v])) {
    const Node& p = nodes[v];
    int best = -1;
    double best_u = -INFINITY;
    for (int c : p.children) {
      if (nodes[c].n == 0) { best = c; break; }  // pending: unvisited, +inf (first in index order)
      double u = ucb(nodes[c].w, nodes[c].n, ln_of(lnT, p.n), C);
      if (u > best_u) { best_u = u; best = c; }
    }
    v = best;
    path.push_back(v);
  }
  *expanded = 0;
  if (!nodes[v].terminal) {
    const Node& p = nodes[v];
    int mv;
    uint64_t cown, copp;
    if (p.legal_moves == 0) {
      mv = 64;
      cown = p.opp; copp = p.own;
    } else {
      int idx = (int)p.children.size(), seen = 0;
      mv = -1;
      for (int sq = 0; sq < 64; ++sq)
        if ((p.legal_moves >> sq) & 1) { if (seen == idx) { mv = sq; break; } ++seen; }
      uint64_t f = flips(p.own, p.opp, mv);
      cown = p.opp & ~f; copp = p.own | f | (1ULL << mv);
    }
    nodes.push_back(make_node(cown, copp, mv, v));
    int c = (int)nodes.size() - 1;
    nodes[v].children.push_back(c);
    path.push_back(c);
    *expanded = 1;
  }
  return path;
}

// Results (wins, draws, losses for the leaf's side to move) of `count`
// playouts from the leaf with streams (c0, c1, c2 = 0..count-1).
void simulate(const Node& leaf, uint32_t count, uint64_t seed, uint32_t c0, uint32_t c1, uint64_t* wdl,
              uint64_t* plies) {
  wdl[0] = wdl[1] = wdl[2] = 0;
  if (leaf.terminal) {
    int a = popcount64(leaf.own), b = popcount64(leaf.opp);
    wdl[a > b ? 0 : (a == b ? 1 : 2)] = count;
    return;
  }
  for (uint32_t t = 0; t < count; ++t) {
    uint32_t pl = 0;
    int r = playout(leaf.own, leaf.opp, seed, c0, c1, t, &pl);
    *plies += pl;
    ++wdl[r > 0 ? 0 : (r == 0 ? 1 : 2)];
  }
}

// Step 4 / the CPU iterations' backpropagation (L196-L199): n += count along
// the path, w += wins of each node's mover, d += draws.
void backprop_path(std::vector<Node>& nodes, const std::vector<int>& path, uint32_t count, const uint64_t* wdl) {
  uint64_t mover_wins = wdl[2], other_wins = wdl[0];
  for (int i = (int)path.size() - 1; i >= 0; --i) {
    Node& x = nodes[path[i]];
    x.n += count;
    x.w += mover_wins;
    x.d += wdl[1];
    std::swap(mover_wins, other_wins);
  }
}

void hybrid_tree(uint64_t root_own, uint64_t root_opp, uint32_t unit, uint64_t steps, uint32_t cpu_iters,
                 uint64_t seed, uint32_t tree_id, double C, TreeResult* out, uint64_t* plies,
                 HybridCounts* hc) {
  std::vector<Node>& nodes = out->nodes;
  nodes.clear();
  nodes.push_back(make_node(root_own, root_opp, -1, -1));
  out->iterations = 0;
  if (nodes[0].terminal) return;
  std::vector<double> lnT(1, 0.0);
  for (uint64_t s = 0; s < steps; ++s) {
    int e = 0;
    std::vector<int> gpath = select_expand_pending(nodes, C, lnT, &e);  // 1
    hc->gpu_nodes += e;
    uint64_t g[3];
    simulate(nodes[gpath.back()], unit, seed, tree_id, (uint32_t)s, g, plies);  // 2
    out->depth_sum += gpath.size() - 1;
    for (uint32_t j = 0; j < cpu_iters; ++j) {  // 3: on the same tree while the GPU works
      std::vector<int> cpath = select_expand_pending(nodes, C, lnT, &e);
      hc->cpu_nodes += e;
      uint64_t c[3], cp = 0;
      simulate(nodes[cpath.back()], 1, seed, tree_id, 0x80000000u + (uint32_t)(s * cpu_iters + j), c, &cp);
      backprop_path(nodes, cpath, 1, c);
      *plies += cp;
      hc->cpu_plies += cp;
      hc->cpu_iterations += 1;
      hc->cpu_depth_sum += cpath.size() - 1;
      out->depth_sum += cpath.size() - 1;
    }
    backprop_path(nodes, gpath, unit, g);  // 4
    out->iterations += 1 + cpu_iters;
  }
}

uint64_t perft_rec(uint64_t own, uint64_t opp, int depth, bool pass_is_ply) {
  if (depth == 0) return 1;
  uint64_t m = legal(own, opp);
  if (m == 0) {
    if (legal(opp, own) == 0) return 1;  // game over: a leaf
    return perft_rec(opp, own, pass_is_ply ? depth - 1 : depth, pass_is_ply);
  }
  uint64_t total = 0;
  for (int s = 0; s < 64; ++s) {
    if (!((m >> s) & 1)) continue;
    uint64_t f = flips(own, opp, s);
    total += perft_rec(opp & ~f, own | f | (1ULL << s), depth - 1, pass_is_ply);
  }
  return total;
}

int resolve_threads(int nthreads) {
  if (nthreads > 0) return nthreads;
  unsigned h = std::thread::hardware_concurrency();
  return h ? (int)h : 1;
}

}  // namespace

// ===========================================================================
// C ABI of the oracle (loaded with ctypes by tests/ and bench.py's CPU legs).
// ===========================================================================
extern "C" {

uint64_t orc_legal(uint64_t own, uint64_t opp) { return legal(own, opp); }
uint64_t orc_flips(uint64_t own, uint64_t opp, int sq) { return flips(own, opp, sq); }
int orc_pick(uint64_t moves, uint32_t r) { return pick(moves, r); }

uint64_t orc_perft(uint64_t black, uint64_t white, uint32_t to_move, int depth, int pass_is_ply) {
  uint64_t own = to_move ? white : black, opp = to_move ? black : white;
  return perft_rec(own, opp, depth, pass_is_ply != 0);
}

void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  philox4x32_10(ctr, key, out);
}

uint32_t orc_rng_word(uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2, uint32_t w) {
  return rng_word(seed, c0, c1, c2, w);
}

// One playout; returns +1/0/-1 for the side to move in `pos`, adds plies.
int orc_playout(const orc_position* pos, uint64_t seed, uint32_t c0, uint32_t c1, uint32_t c2,
                uint32_t* plies) {
  uint64_t own, opp;
  to_own_opp(*pos, &own, &opp);
  return playout(own, opp, seed, c0, c1, c2, plies);
}

// Batched playouts (the mcts_playouts contract): leaf i gets n_per_leaf
// playouts with streams (c0 = leaf_id_base + i, c1 = 0, c2 = j). Output
// wdl[3*i + {0,1,2}] = wins, draws, losses for leaf i's side to move.
// Returns the total number of plies (non-pass moves) played.
uint64_t orc_playouts(const orc_position* leaves, uint32_t n_leaves, uint32_t n_per_leaf,
                      uint64_t seed, uint32_t leaf_id_base, uint32_t* wdl, int nthreads) {
  int T = resolve_threads(nthreads);
  std::vector<uint64_t> plies(T, 0);
  std::atomic<uint32_t> next{0};
  auto worker = [&](int tid) {
    for (;;) {
      uint32_t i = next.fetch_add(1);
      if (i >= n_leaves) break;
      uint64_t own, opp;
      to_own_opp(leaves[i], &own, &opp);
      uint32_t w = 0, d = 0, l = 0, pl = 0;
      for (uint32_t j = 0; j < n_per_leaf; ++j) {
        int r = playout(own, opp, seed, leaf_id_base + i, 0u, j, &pl);
        if (r > 0) ++w; else if (r == 0) ++d; else ++l;
      }
      wdl[3 * (size_t)i + 0] = w;
      wdl[3 * (size_t)i + 1] = d;
      wdl[3 * (size_t)i + 2] = l;
      plies[tid] += pl;
    }
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < T; ++t) pool.emplace_back(worker, t);
  worker(0);
  for (auto& th : pool) th.join();
  uint64_t total = 0;
  for (uint64_t p : plies) total += p;
  return total;
}

double orc_ln(uint64_t x) { return ln_rn(x); }

// lnT[k] = RN(ln(k * unit)) for k = 1..K; lnT[0] = 0 (never used).
void orc_ln_table(uint32_t unit, uint32_t K, double* out) {
  out[0] = 0.0;
  for (uint32_t k = 1; k <= K; ++k) out[k] = ln_rn((uint64_t)k * unit);
}

double orc_ucb(uint64_t w, uint64_t n, double ln_parent, double C) { return ucb(w, n, ln_parent, C); }

// Full search (the mcts_search contract, iteration mode). stats layout:
// [0,65) visits, [65,130) wins (for the root's side to move), [130,195) draws,
// [195] root visits, [196] iterations, [197] playout plies, [198] sum over
// iterations of the simulated node's depth, [199] expansions refused by a full
// pool, [200] nodes, [201] node capacity; summed over trees tree_id_base ..
// tree_id_base + n_trees - 1. capacity = max nodes per tree (0 = iterations+1).
// Returns best move (max visits, lowest index on ties) or -1 if the root is
// terminal. plies_out (nullable) receives the playout plies.
int orc_uct_search(const orc_position* root, uint32_t n_trees, uint32_t unit, uint64_t iterations,
                   uint64_t seed, uint32_t tree_id_base, double C, uint64_t capacity,
                   int64_t* stats, uint64_t* plies_out, int nthreads) {
  for (int i = 0; i < 202; ++i) stats[i] = 0;
  uint64_t own, opp;
  to_own_opp(*root, &own, &opp);
  if (capacity == 0) capacity = iterations + 1;
  std::vector<double> lnT(iterations + 2);
  orc_ln_table(unit, (uint32_t)(iterations + 1), lnT.data());
  std::vector<TreeResult> res(n_trees);
  std::vector<uint64_t> plies(n_trees, 0);
  int T = std::min<int>(resolve_threads(nthreads), (int)std::max<uint32_t>(n_trees, 1));
  std::atomic<uint32_t> next{0};
  auto worker = [&]() {
    for (;;) {
      uint32_t t = next.fetch_add(1);
      if (t >= n_trees) break;
      search_tree(own, opp, unit, iterations, seed, tree_id_base + t, C, capacity, lnT, &res[t],
                  &plies[t]);
    }
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < T; ++t) pool.emplace_back(worker);
  worker();
  for (auto& th : pool) th.join();
  uint64_t ptot = 0;
  for (uint32_t t = 0; t < n_trees; ++t) {
    const std::vector<Node>& nodes = res[t].nodes;
    for (int c : nodes[0].children) {
      int mv = nodes[c].move;
      stats[mv] += (int64_t)nodes[c].n;
      stats[65 + mv] += (int64_t)nodes[c].w;
      stats[130 + mv] += (int64_t)nodes[c].d;
    }
    stats[195] += (int64_t)nodes[0].n;
    stats[196] += (int64_t)res[t].iterations;
    stats[198] += (int64_t)res[t].depth_sum;
    stats[199] += (int64_t)res[t].refused;
    if (!nodes[0].terminal) {  // a terminal root is no search: all stats stay 0
      stats[200] += (int64_t)nodes.size();
      stats[201] += (int64_t)capacity;
    }
    ptot += plies[t];
  }
  stats[197] = (int64_t)ptot;
  if (plies_out) *plies_out = ptot;
  if (res.empty() || res[0].nodes[0].terminal) return -1;
  int best = -1;
  int64_t bv = -1;
  for (int mv = 0; mv < 65; ++mv)
    if (stats[mv] > bv) { bv = stats[mv]; best = mv; }
  return best;
}

// One tree, dumped for invariant tests. Arrays of length >= capacity
// (capacity 0 = iterations+1): parent, move, n, w, d, terminal. Returns the
// node count.
int64_t orc_uct_tree(const orc_position* root, uint32_t unit, uint64_t iterations, uint64_t seed,
                     uint32_t tree_id, double C, uint64_t capacity, int32_t* parent, int32_t* move,
                     uint64_t* n, uint64_t* w, uint64_t* d, uint8_t* terminal) {
  uint64_t own, opp;
  to_own_opp(*root, &own, &opp);
  if (capacity == 0) capacity = iterations + 1;
  std::vector<double> lnT(iterations + 2);
  orc_ln_table(unit, (uint32_t)(iterations + 1), lnT.data());
  TreeResult r;
  search_tree(own, opp, unit, iterations, seed, tree_id, C, capacity, lnT, &r, nullptr);
  for (size_t i = 0; i < r.nodes.size(); ++i) {
    parent[i] = r.nodes[i].parent;
    move[i] = r.nodes[i].move;
    n[i] = r.nodes[i].n;
    w[i] = r.nodes[i].w;
    d[i] = r.nodes[i].d;
    terminal[i] = r.nodes[i].terminal ? 1 : 0;
  }
  return (int64_t)r.nodes.size();
}

// Synthetic position generator (DESIGN.md §4 input recipe). Position p:
// key = seed, counter = (p, 0xFFFFFFFF, attempt, j). Word 0 gives
// L = lmin + floor(r * (lmax - lmin + 1) / 2^32) non-pass plies of uniform
// random play from the opening, consuming words 1, 2, ...; passes are taken and
// not counted. A game that ends before L plies, or a terminal result, retries
// with attempt + 1.
void orc_gen_positions(uint64_t seed, uint32_t n, uint32_t lmin, uint32_t lmax, orc_position* out) {
  for (uint32_t p = 0; p < n; ++p) {
    // lmax <= 50 keeps >= 10 empty squares, so a non-terminal result is found
    // after a few attempts; the cap only guards against misuse (result: opening).
    out[p].black = 0x0000000810000000ULL; out[p].white = 0x0000001008000000ULL;
    out[p].to_move = 0; out[p].reserved = 0;
    for (uint32_t attempt = 0; attempt < (1u << 16); ++attempt) {
      uint32_t span = lmax - lmin + 1;
      uint32_t L = lmin + (uint32_t)(((uint64_t)rng_word(seed, p, 0xFFFFFFFFu, attempt, 0) * span) >> 32);
      uint64_t me = 0x0000000810000000ULL, op = 0x0000001008000000ULL;  // black, white
      uint32_t stm = 0, w = 1, plies = 0;
      bool ok = true;
      while (plies < L) {
        uint64_t m = legal(me, op);
        if (m == 0) {
          if (legal(op, me) == 0) { ok = false; break; }
          std::swap(me, op); stm ^= 1u;
          continue;
        }
        int sq = pick(m, rng_word(seed, p, 0xFFFFFFFFu, attempt, w));
        ++w;
        uint64_t f = flips(me, op, sq);
        me |= f | (1ULL << sq);
        op &= ~f;
        std::swap(me, op); stm ^= 1u;
        ++plies;
      }
      if (!ok) continue;
      if (legal(me, op) == 0 && legal(op, me) == 0) continue;
      out[p].black = stm == 0 ? me : op;
      out[p].white = stm == 0 ? op : me;
      out[p].to_move = stm;
      out[p].reserved = 0;
      break;
    }
  }
}

// Hybrid CPU-GPU search on CPU-managed trees (hybrid_tree above; the
// mcts_search_hosted contract): n_trees trees (ids tree_id_base + t), `steps`
// GPU steps of `unit` playouts each with cpu_iters CPU iterations per step.
// stats as orc_uct_search ([196] counts GPU steps and CPU iterations, [197]
// all plies, [198] both depth sums; [199] 0, [200] nodes, [201] 0 = unbounded);
// cpu[0..4] = CPU iterations, CPU plies, CPU depth sum, nodes added by CPU
// iterations, nodes added by GPU steps. cpu_iters = 0 is the block-parallel
// search (uct_search) bit for bit. Returns the best move (R8).
int orc_hybrid_search(const orc_position* root, uint32_t n_trees, uint32_t unit, uint64_t steps,
                      uint32_t cpu_iters, uint64_t seed, uint32_t tree_id_base, double C, int64_t* stats,
                      int64_t* cpu, int nthreads) {
  for (int i = 0; i < 202; ++i) stats[i] = 0;
  for (int i = 0; i < 5; ++i) cpu[i] = 0;
  uint64_t own, opp;
  to_own_opp(*root, &own, &opp);
  std::vector<TreeResult> res(n_trees);
  std::vector<uint64_t> plies(n_trees, 0);
  std::vector<HybridCounts> hc(n_trees);
  int T = std::min<int>(resolve_threads(nthreads), (int)std::max<uint32_t>(n_trees, 1));
  std::atomic<uint32_t> next{0};
  auto worker = [&]() {
    for (;;) {
      uint32_t t = next.fetch_add(1);
      if (t >= n_trees) break;
      hybrid_tree(own, opp, unit, steps, cpu_iters, seed, tree_id_base + t, C, &res[t], &plies[t], &hc[t]);
    }
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < T; ++t) pool.emplace_back(worker);
  worker();
  for (auto& th : pool) th.join();
  for (uint32_t t = 0; t < n_trees; ++t) {
    const std::vector<Node>& nodes = res[t].nodes;
    if (nodes[0].terminal) continue;
    for (int c : nodes[0].children) {
      int mv = nodes[c].move;
      stats[mv] += (int64_t)nodes[c].n;
      stats[65 + mv] += (int64_t)nodes[c].w;
      stats[130 + mv] += (int64_t)nodes[c].d;
    }
    stats[195] += (int64_t)nodes[0].n;
    stats[196] += (int64_t)res[t].iterations;
    stats[197] += (int64_t)plies[t];
    stats[198] += (int64_t)res[t].depth_sum;
    stats[200] += (int64_t)nodes.size();
    cpu[0] += (int64_t)hc[t].cpu_iterations;
    cpu[1] += (int64_t)hc[t].cpu_plies;
    cpu[2] += (int64_t)hc[t].cpu_depth_sum;
    cpu[3] += (int64_t)hc[t].cpu_nodes;
    cpu[4] += (int64_t)hc[t].gpu_nodes;
  }
  if (n_trees == 0 || res[0].nodes[0].terminal) return -1;
  int best = -1;
  int64_t bv = 0;
  for (int mv = 0; mv < 65; ++mv)
    if (stats[mv] > bv) { bv = stats[mv]; best = mv; }
  return best;
}

// Root-parallel CPU MCTS opponent: one tree
// per thread, one playout per iteration (unit = 1), grown with the same
// uct_iteration as the iteration-mode search; roots summed (L199-L202).
// Thread t is tree t: streams (c0 = t, c1 = iteration, c2 = 0), exactly
// uct_search(root, nthreads, unit 1, ..., tree_id_base 0) for the same
// iteration counts. Stops at the wall-clock budget (budget_ms > 0; not
// reproducible) and/or after max_iterations per tree (> 0; then with no
// deadline it is bit-exact to uct_search(root, nthreads, 1, max_iterations)).
// Node pool unbounded. stats as in orc_uct_search. Returns the chosen move
// (max visits, lowest index on ties; -1 terminal).
int orc_mcts_timed(const orc_position* root, int nthreads, double budget_ms, uint64_t seed,
                   double C, int64_t* stats, uint64_t max_iterations) {
  for (int i = 0; i < 202; ++i) stats[i] = 0;
  uint64_t own, opp;
  to_own_opp(*root, &own, &opp);
  Node r0 = make_node(own, opp, -1, -1);
  if (r0.terminal) return -1;
  if (budget_ms <= 0.0 && max_iterations == 0) return -1;
  int T = resolve_threads(nthreads);
  auto t0 = std::chrono::steady_clock::now();
  auto deadline = t0 + std::chrono::duration<double, std::milli>(budget_ms);
  const uint64_t cap = max_iterations ? max_iterations : ~0ULL;
  std::vector<TreeResult> res(T);
  std::vector<uint64_t> plies(T, 0);
  auto worker = [&](int tid) {
    // ln table for unit 1 (lnT[k] = RN(ln k)), extended as the tree grows
    std::vector<double> lnT(1, 0.0);
    TreeResult& tr = res[tid];
    tr.nodes.clear();
    tr.nodes.push_back(make_node(own, opp, -1, -1));
    uint64_t it = 0;
    while (it < cap && (budget_ms <= 0.0 || std::chrono::steady_clock::now() < deadline)) {
      uint64_t chunk = std::min<uint64_t>(64, cap - it);  // deadline checked every 64 iterations
      size_t need = it + chunk + 2;
      if (lnT.size() < need) {
        size_t old = lnT.size();
        lnT.resize(need * 2);
        for (size_t k = old; k < lnT.size(); ++k) lnT[k] = ln_rn(k);
      }
      for (uint64_t j = 0; j < chunk; ++j, ++it)
        uct_iteration(&tr, it, 1u, seed, (uint32_t)tid, C, ~0ULL, lnT, &plies[tid]);
    }
    tr.iterations = it;
  };
  std::vector<std::thread> pool;
  for (int t = 1; t < T; ++t) pool.emplace_back(worker, t);
  worker(0);
  for (auto& th : pool) th.join();
  for (int t = 0; t < T; ++t) {
    const std::vector<Node>& nodes = res[t].nodes;
    for (int c : nodes[0].children) {
      int mv = nodes[c].move;
      stats[mv] += (int64_t)nodes[c].n;
      stats[65 + mv] += (int64_t)nodes[c].w;
      stats[130 + mv] += (int64_t)nodes[c].d;
    }
    stats[195] += (int64_t)nodes[0].n;
    stats[196] += (int64_t)res[t].iterations;
    stats[197] += (int64_t)plies[t];
    stats[198] += (int64_t)res[t].depth_sum;
    stats[200] += (int64_t)nodes.size();
  }
  int best = -1;
  int64_t bv = 0;
  for (int mv = 0; mv < 65; ++mv)
    if (stats[mv] > bv) { bv = stats[mv]; best = mv; }
  return best;
}

}  // extern "C"
