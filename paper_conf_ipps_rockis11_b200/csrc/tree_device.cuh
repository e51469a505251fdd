// tree_device.cuh — device-resident UCT tree (§II-A).
//
// One pool of node slots per tree in HBM, structure-of-arrays so the 32 lanes
// of the selecting warp read 32 sibling statistics with one coalesced load per
// field. A node's children occupy a contiguous block of `limit` slots that is
// reserved the first time the node is expanded; children are created one per
// iteration (L181 "I add one node per iteration") in ascending move order, so
// child i of a node is its i-th legal move (or the pass child, move 64).
//
// Visit counts are stored in iterations (k); n = k * unit. This is exact: every
// visit of a node adds `unit` playouts (L186-L195), and it indexes the ln table
// lnT[k] = RN(ln(k * unit)) directly (R9).
#pragma once
#include <cstdint>
#include "reversi_device.cuh"

namespace mcts_dev {

constexpr u32 kNoChild = 0xFFFFFFFFu;
constexpr int kMaxPath = 160;  // > 60 moves + passes + root

// Debug build (MCTS_DEBUG_BOUNDS=1, tools/build_variants.py "bounds"): every
// tree-slot index and path position is checked and a violation traps with the
// line number printed — the stand-in for compute-sanitizer's memcheck, which
// this GPU pool does not allow. Compiled out of the product build.
#ifndef MCTS_DEBUG_BOUNDS
#define MCTS_DEBUG_BOUNDS 0
#endif
#if MCTS_DEBUG_BOUNDS
#define MCTS_CHECK(cond)                                                          \
  do {                                                                             \
    if (!(cond)) {                                                                 \
      printf("MCTS_CHECK failed: %s (%s:%d)\n", #cond, __FILE__, __LINE__);      \
      __trap();                                                                    \
    }                                                                              \
  } while (0)
#else
#define MCTS_CHECK(cond) do {} while (0)
#endif
constexpr unsigned kFull = 0xFFFFFFFFu;

struct TreePool {
  u64* own;    // discs of the side to move at the node
  u64* opp;    // discs of the other side
  u64* legal;  // legal moves of the side to move
  u32* k;      // iterations through the node (n = k * unit)
  u32* w;      // playouts won by mover(node) = the side that moved into it
  u32* d;      // drawn playouts
  u32* first;  // first child slot (tree-relative) or kNoChild
  u32* meta;   // nchild | limit << 8 | move << 16 | terminal << 24
  u32* vl;     // virtual visits of in-flight workers (MCTS_TREE only, tree_parallel.cuh)
  u32 slot_cap;
};

__device__ __forceinline__ u32 meta_nchild(u32 m) { return m & 0xFFu; }
__device__ __forceinline__ u32 meta_limit(u32 m) { return (m >> 8) & 0xFFu; }
__device__ __forceinline__ u32 meta_move(u32 m) { return (m >> 16) & 0xFFu; }
__device__ __forceinline__ bool meta_term(u32 m) { return (m >> 24) != 0u; }

// Create node s (one thread). With `hot` the hot-loop move generator
// (legal_moves_hot, pinned by the device perft) replaces the plain one.
// Returns the meta word; *lg_out (optional) receives the legal moves.
__device__ __forceinline__ u32 init_node(const TreePool& T, size_t s, u64 own, u64 opp, u32 move,
                                         bool hot = false, u64* lg_out = nullptr) {
  u64 lg;
  bool term;
  if (hot) {
    const u64 ro = __brevll(own), rp = __brevll(opp);
    lg = legal_moves_hot(own, opp, ro, rp);
    term = lg == 0ULL && legal_moves_hot(opp, own, rp, ro) == 0ULL;
  } else {
    lg = legal_moves(own, opp);
    term = is_terminal(own, opp, lg);
  }
  const u32 limit = term ? 0u : (lg ? (u32)__popcll(lg) : 1u);
  const u32 meta = (limit << 8) | (move << 16) | ((term ? 1u : 0u) << 24);
  T.own[s] = own;
  T.opp[s] = opp;
  T.legal[s] = lg;
  T.k[s] = 0;
  T.w[s] = 0;
  T.d[s] = 0;
  T.first[s] = kNoChild;
  T.meta[s] = meta;
  if (lg_out) *lg_out = lg;
  return meta;
}

// The owning warp's view of its current path (shared memory; block and leaf
// schemes, where one warp is the tree's only reader and writer): the node
// slots root..leaf with the (k, w, d) it last read or wrote for each, and the
// root's board and control values. Selection fills it, backpropagation
// writes the updated statistics from it without reading the tree again, and
// the root (position 0) stays current across iterations, so an iteration
// reads the tree only at the levels it descends.
struct PathCache {
  u32 node[kMaxPath];
  u32 k[kMaxPath], w[kMaxPath], d[kMaxPath];
  u64 root_own, root_opp, root_legal;
  u32 root_meta, root_first;
};

// Create the root (one thread) and its cache entry.
__device__ __forceinline__ u32 init_root(const TreePool& T, size_t base, u64 own, u64 opp, PathCache* pc) {
  u64 lg;
  const u32 meta = init_node(T, base, own, opp, 0xFFu, true, &lg);
  pc->node[0] = 0;
  pc->k[0] = 0; pc->w[0] = 0; pc->d[0] = 0;
  pc->root_own = own; pc->root_opp = opp; pc->root_legal = lg;
  pc->root_meta = meta; pc->root_first = kNoChild;
  return meta;
}

// u = w/n + C*sqrt(lnT[k_parent]/n): five IEEE round-to-nearest operations in
// this order, no contraction (R1) — bit-identical to the oracle.
__device__ __forceinline__ double ucb_value(u32 w, u32 k, u32 unit, double ln_parent, double C) {
  const double n = (double)((unsigned long long)k * unit);
  const double exploit = __ddiv_rn((double)w, n);
  const double explore = __dmul_rn(C, __dsqrt_rn(__ddiv_rn(ln_parent, n)));
  return __dadd_rn(exploit, explore);
}

#ifndef MCTS_REDUX_ARGMAX
#define MCTS_REDUX_ARGMAX 1
#endif

// Warp argmax of (u, i): the largest u, the lowest i among equal u; lanes with
// no candidate hold i = kNoChild (u = -inf). Returns the winning i in every
// lane. With MCTS_REDUX_ARGMAX the doubles are mapped to order-preserving
// 64-bit keys and reduced with three warp reductions (max of the high words,
// max of the low words among the lanes that hold it, min index among the
// lanes that hold both) instead of five rounds of shuffles; same result.
__device__ __forceinline__ u32 warp_argmax(double u, u32 i) {
#if MCTS_REDUX_ARGMAX
  const unsigned long long b = (unsigned long long)__double_as_longlong(u);
  const unsigned long long key = i == kNoChild ? 0ULL : ((b >> 63) ? ~b : (b | 0x8000000000000000ULL));
  const u32 hi = (u32)(key >> 32), lo = (u32)key;
  const u32 mhi = __reduce_max_sync(kFull, hi);
  const u32 mlo = __reduce_max_sync(kFull, hi == mhi ? lo : 0u);
  return __reduce_min_sync(kFull, (hi == mhi && lo == mlo) ? i : kNoChild);
#else
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    const double ou = __shfl_xor_sync(kFull, u, off);
    const u32 oi = __shfl_xor_sync(kFull, i, off);
    if (ou > u || (ou == u && oi < i)) { u = ou; i = oi; }
  }
  return i;
#endif
}

struct LeafInfo {
  u64 own, opp;
  u32 term;
  u32 refused;  // lane 0: the node wanted its first child but the pool was full (R12)
  int depth;
};

// Selection + expansion of one iteration, executed by one full warp that
// owns the tree. pc (shared) receives the path root..leaf and its
// statistics; *slot_used (shared) is the tree's slot allocator; rays is the
// CTA's shared ray table (flips_loop). Returns the leaf (same value in every
// lane).
//
// Latency (round 2): the warp walks the tree through L2, so each level costs
// its dependent round trips. A level's lanes load their children's UCB
// statistics (w, k) together with everything the next step needs (d, meta,
// first, board, legal moves), and the winner's values are broadcast from its
// lane: descending one level is ONE round trip (lnT[k] is issued alongside),
// the root comes from the cache, and the expansion needs no read at all —
// instead of the five dependent reads per level, a root read and a board read
// of round 1.
template <bool BOARDS = true>  // false: the chosen node's board is read once after the descent
__device__ __forceinline__ LeafInfo select_expand(const TreePool& T, size_t base, PathCache* pc,
                                                  u32* slot_used, const double* __restrict__ lnT,
                                                  u32 unit, double C, int lane,
                                                  const u64* __restrict__ rays) {
  u32 v = 0;
  int depth = 0;
  // Control values are read by one lane and broadcast, so every lane takes the
  // same path through the loop (a leaf kernel whose leader lanes loaded them
  // individually diverged and deadlocked).
  u32 meta = 0, first = 0, kv = 0;
  if (lane == 0) { meta = pc->root_meta; first = pc->root_first; kv = pc->k[0]; }
  meta = __shfl_sync(kFull, meta, 0);
  first = __shfl_sync(kFull, first, 0);
  kv = __shfl_sync(kFull, kv, 0);
  u64 own = pc->root_own, opp = pc->root_opp, lg = pc->root_legal;  // used by lane 0 only
  // Selection (L157-L178): descend while the node is non-terminal and fully expanded.
  // (depth bound: a game has < 128 plies incl. passes; never reached)
  while (!meta_term(meta) && meta_nchild(meta) >= meta_limit(meta) && depth < kMaxPath - 2) {
    const u32 nch = meta_nchild(meta);
    const double lnp = lnT[kv];
    double best_u = -__longlong_as_double(0x7FF0000000000000LL);  // -inf
    u32 best_i = kNoChild, bm = 0, bf = 0, bk = 0, bw = 0, bd = 0;
    u64 bo = 0, bp = 0, bl = 0;
    for (u32 i = (u32)lane; i < nch; i += 32u) {
      MCTS_CHECK(first != kNoChild && first + i < T.slot_cap);
      const size_t c = base + first + i;
      const u32 wc = T.w[c], kc = T.k[c], dc = T.d[c], mc = T.meta[c], fc = T.first[c];
      u64 oc = 0, pc_ = 0, lc = 0;
      if (BOARDS) { oc = T.own[c]; pc_ = T.opp[c]; lc = T.legal[c]; }
      const double u = ucb_value(wc, kc, unit, lnp, C);
      if (u > best_u) {
        best_u = u; best_i = i;
        bm = mc; bf = fc; bk = kc; bw = wc; bd = dc; bo = oc; bp = pc_; bl = lc;
      }
    }
    best_i = warp_argmax(best_u, best_i);
    // child best_i was scored by lane best_i mod 32, whose own best it is
    const int src = (int)(best_i & 31u);
    v = first + best_i;
    meta = __shfl_sync(kFull, bm, src);
    first = __shfl_sync(kFull, bf, src);
    kv = __shfl_sync(kFull, bk, src);
    const u32 wv = __shfl_sync(kFull, bw, src), dv = __shfl_sync(kFull, bd, src);
    if (BOARDS) {
      own = __shfl_sync(kFull, bo, src);
      opp = __shfl_sync(kFull, bp, src);
      lg = __shfl_sync(kFull, bl, src);
    }
    ++depth;
    MCTS_CHECK(depth < kMaxPath && v < T.slot_cap);
    if (lane == 0) { pc->node[depth] = v; pc->k[depth] = kv; pc->w[depth] = wv; pc->d[depth] = dv; }
  }
  // Expansion (L179-L182), lane 0: the lowest-index untried move, or the pass
  // child. The leaf returned is v or the new child, from registers.
  LeafInfo L;
  L.refused = 0;
  u32 c = kNoChild;
  u32 term = meta_term(meta) ? 1u : 0u;
  if (!BOARDS && depth > 0 && lane == 0) {
    own = T.own[base + v];
    opp = T.opp[base + v];
    lg = T.legal[base + v];
  }
  if (lane == 0 && !term) {
    const u32 nch = meta_nchild(meta), limit = meta_limit(meta);
    u32 f0 = first;
    if (nch == 0u) {
      if (*slot_used + limit <= T.slot_cap) {
        f0 = *slot_used;
        *slot_used += limit;
        T.first[base + v] = f0;
      } else {
        f0 = kNoChild;  // pool full (time mode): simulate from v itself
        L.refused = 1;
      }
    }
    if (f0 != kNoChild) {
      c = f0 + nch;
      u64 cown, copp;
      u32 mv;
      if (lg == 0ULL) {
        cown = opp; copp = own; mv = 64u;  // pass: same discs, turn swaps
      } else {
        const int sq = kth_set_bit(lg, nch);
        const u64 f = flips_loop(sq, own, opp, __brevll(own), __brevll(opp), rays);
        cown = opp & ~f; copp = own | f | (1ULL << sq); mv = (u32)sq;
      }
      MCTS_CHECK(c < T.slot_cap && nch < limit && depth + 1 < kMaxPath);
      term = meta_term(init_node(T, base + c, cown, copp, mv, true)) ? 1u : 0u;
      T.meta[base + v] = meta + 1u;  // ++nchild
      if (depth == 0) { pc->root_meta = meta + 1u; pc->root_first = f0; }
      pc->node[depth + 1] = c;
      pc->k[depth + 1] = 0; pc->w[depth + 1] = 0; pc->d[depth + 1] = 0;
      own = cown; opp = copp;
    }
  }
  c = __shfl_sync(kFull, c, 0);
  __syncwarp();
  if (c != kNoChild) ++depth;
  L.own = __shfl_sync(kFull, own, 0);
  L.opp = __shfl_sync(kFull, opp, 0);
  L.term = __shfl_sync(kFull, term, 0);
  L.depth = depth;
  return L;
}

// Backpropagation (L196-L199) by the owning warp, lanes over path positions
// (distinct nodes), from the cached statistics (stores only). W/D/Lo are the
// leaf batch's wins/draws/losses for the leaf's side to move; the leaf's mover
// collects Lo, its parent W, alternating to the root. The root's cache entry
// is kept current.
__device__ __forceinline__ void backprop(const TreePool& T, size_t base, PathCache* pc, int depth,
                                         u32 W, u32 D, u32 Lo, int lane) {
  for (int p = lane; p <= depth; p += 32) {
    MCTS_CHECK(pc->node[p] < T.slot_cap);
    const size_t s = base + pc->node[p];
    const int lvl = depth - p;
    const u32 k = pc->k[p] + 1u, w = pc->w[p] + ((lvl & 1) ? W : Lo), d = pc->d[p] + D;
    T.k[s] = k;
    T.w[s] = w;
    T.d[s] = d;
    if (p == 0) { pc->k[0] = k; pc->w[0] = w; pc->d[0] = d; }
  }
  __syncwarp();
}

// Fused root merge (a10): add this tree's root-child statistics into the int64
// stats vector (see MCTS_STATS_LEN in include/mcts.h). Integer atomics are
// order-independent, so the sum is deterministic. Also the pool diagnostics:
// [199] refused expansions, [200] slots used, [201] slot capacity.
__device__ __forceinline__ void merge_pool(long long* stats, unsigned long long refused, u32 used,
                                           u32 cap) {
  unsigned long long* st = reinterpret_cast<unsigned long long*>(stats);
  if (refused) atomicAdd(st + 199, refused);
  atomicAdd(st + 200, (unsigned long long)used);
  atomicAdd(st + 201, (unsigned long long)cap);
}

__device__ __forceinline__ void merge_root(const TreePool& T, size_t base, u32 unit, u32 iterations,
                                           long long* stats, int lane) {
  const u32 meta = T.meta[base];
  const u32 nch = meta_nchild(meta);
  const u32 first = T.first[base];
  unsigned long long* st = reinterpret_cast<unsigned long long*>(stats);
  for (u32 i = (u32)lane; i < nch; i += 32u) {
    const size_t c = base + first + i;
    const u32 mv = meta_move(T.meta[c]);
    atomicAdd(st + mv, (unsigned long long)T.k[c] * unit);
    atomicAdd(st + 65 + mv, (unsigned long long)T.w[c]);
    atomicAdd(st + 130 + mv, (unsigned long long)T.d[c]);
  }
  if (lane == 0) {
    atomicAdd(st + 195, (unsigned long long)T.k[base] * unit);
    atomicAdd(st + 196, (unsigned long long)iterations);
  }
}

}  // namespace mcts_dev
