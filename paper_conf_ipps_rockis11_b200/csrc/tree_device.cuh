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

__device__ __forceinline__ u32 init_node(const TreePool& T, size_t s, u64 own, u64 opp, u32 move) {
  const u64 lg = legal_moves(own, opp);
  const bool term = is_terminal(own, opp, lg);
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

struct LeafInfo {
  u64 own, opp;
  u32 term;
  u32 refused;  // lane 0: the node wanted its first child but the pool was full (R12)
  int depth;
};

// Selection + expansion of one iteration, executed by one full warp.
// path (shared) receives the node slots root..leaf; *slot_used (shared) is the
// tree's slot allocator. Returns the leaf (same value in every lane).
//
// Latency (round 2): the warp walks the tree through L2, so each level costs
// its dependent round trips. A level's lanes load their children's (w, k)
// for UCB together with the children's control values (meta, first), and the
// winner's are broadcast from its lane, so descending one level is ONE round
// trip (plus lnT[k], whose address is known as soon as the parent is chosen)
// instead of five (meta, first, k, lnT, children). Only this warp writes the
// tree (block and leaf schemes), so the values read are the current ones.
__device__ __forceinline__ LeafInfo select_expand(const TreePool& T, size_t base, u32* path,
                                                  u32* slot_used, const double* __restrict__ lnT,
                                                  u32 unit, double C, int lane) {
  u32 v = 0;
  int depth = 0;
  if (lane == 0) path[0] = 0;
  // Control values (meta, first child, count) of the current node are read by
  // one lane and broadcast, so every lane takes the same path through the
  // loop whatever the memory system returns to each lane's own load (a leaf
  // kernel whose leader lanes loaded them individually diverged and
  // deadlocked).
  u32 meta = 0, first = 0, kv = 0;
  if (lane == 0) { meta = T.meta[base]; first = T.first[base]; kv = T.k[base]; }
  meta = __shfl_sync(kFull, meta, 0);
  first = __shfl_sync(kFull, first, 0);
  kv = __shfl_sync(kFull, kv, 0);
  // Selection (L157-L178): descend while the node is non-terminal and fully expanded.
  // (depth bound: a game has < 128 plies incl. passes; never reached)
  while (!meta_term(meta) && meta_nchild(meta) >= meta_limit(meta) && depth < kMaxPath - 2) {
    const u32 nch = meta_nchild(meta);
    const double lnp = lnT[kv];
    double best_u = -__longlong_as_double(0x7FF0000000000000LL);  // -inf
    u32 best_i = kNoChild, best_meta = 0, best_first = 0, best_k = 0;
    for (u32 i = (u32)lane; i < nch; i += 32u) {
      const size_t c = base + first + i;
      const u32 wc = T.w[c], kc = T.k[c], mc = T.meta[c], fc = T.first[c];
      const double u = ucb_value(wc, kc, unit, lnp, C);
      if (u > best_u) { best_u = u; best_i = i; best_meta = mc; best_first = fc; best_k = kc; }
    }
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      const double ou = __shfl_xor_sync(kFull, best_u, off);
      const u32 oi = __shfl_xor_sync(kFull, best_i, off);
      if (ou > best_u || (ou == best_u && oi < best_i)) { best_u = ou; best_i = oi; }
    }
    // child best_i was scored by lane best_i mod 32, whose own best it is
    const int src = (int)(best_i & 31u);
    v = first + best_i;
    meta = __shfl_sync(kFull, best_meta, src);
    first = __shfl_sync(kFull, best_first, src);
    kv = __shfl_sync(kFull, best_k, src);
    ++depth;
    if (lane == 0) path[depth] = v;
  }
  // Expansion (L179-L182): the lowest-index untried move, or the pass child.
  // Lane 0 reads v's board once; the leaf it returns is v or the new child,
  // from registers.
  LeafInfo L;
  L.refused = 0;
  u32 c = kNoChild;
  u64 own = 0, opp = 0;
  u32 term = meta_term(meta) ? 1u : 0u;
  if (lane == 0) {
    own = T.own[base + v];
    opp = T.opp[base + v];
    const u64 lg = T.legal[base + v];
    if (!term) {
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
          const u64 f = flips(sq, own, opp);
          cown = opp & ~f; copp = own | f | (1ULL << sq); mv = (u32)sq;
        }
        term = meta_term(init_node(T, base + c, cown, copp, mv)) ? 1u : 0u;
        T.meta[base + v] = meta + 1u;  // ++nchild
        path[depth + 1] = c;
        own = cown; opp = copp;
      }
    }
  }
  c = __shfl_sync(kFull, c, 0);
  __syncwarp();
  if (c != kNoChild) {
    v = c;
    ++depth;
  }
  L.own = __shfl_sync(kFull, own, 0);
  L.opp = __shfl_sync(kFull, opp, 0);
  L.term = __shfl_sync(kFull, term, 0);
  L.depth = depth;
  return L;
}

// Backpropagation (L196-L199) by one warp, lanes over path positions (distinct
// nodes). W/D/Lo are the leaf batch's wins/draws/losses for the leaf's side to
// move; the leaf's mover collects Lo, its parent W, alternating to the root.
__device__ __forceinline__ void backprop(const TreePool& T, size_t base, const u32* path, int depth,
                                         u32 W, u32 D, u32 Lo, int lane) {
  for (int p = lane; p <= depth; p += 32) {
    const size_t s = base + path[p];
    const int lvl = depth - p;
    T.k[s] += 1u;
    T.w[s] += (lvl & 1) ? W : Lo;
    T.d[s] += D;
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
