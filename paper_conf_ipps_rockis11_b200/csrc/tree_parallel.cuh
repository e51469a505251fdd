// tree_parallel.cuh — tree parallelism on one shared device tree (MCTS_TREE;
// SURVEY.md §8(f) NEXT-4).
//
// The paper compares leaf, root and its own block parallelism (PAPER.md
// L211-L244, Fig. 2) and names Chaslot et al.'s third scheme, tree
// parallelism, through its reference list: "To be effective tree
// parallelization requires two techniques: adequately handling of (1) local
// mutexes and (2) virtual loss". Its block-parallel trees are
// shallow (L313-L319); a single tree grown by every CTA of the GPU is the
// opposite trade. Here the W workers are CTAs of `unit` threads (one UCT
// iteration = `unit` playouts from one leaf, as in block parallelism) sharing
// ONE tree in HBM:
//   * selection (warp 0): UCB on counts that include the virtual visits of the
//     other workers currently below a node (k + vl; the parent's count
//     excludes the selecting worker's own virtual visit), so concurrent
//     workers spread over the tree; the chosen child gets vl += 1;
//   * expansion: the lowest-index untried move is claimed with one CAS on the
//     node's child counter (the "local mutex" is that CAS); the claimer
//     initialises the child and reserves the child's own child block
//     (eagerly, one atomicAdd on the pool allocator), then publishes it with a
//     release store of its meta word; readers skip unpublished children;
//   * simulation: the CTA plays `unit` playouts from the leaf (the hot loop of
//     reversi_device.cuh), RNG streams (c0 = tree id, c1 = iteration ticket
//     from a global counter, c2 = thread);
//   * backpropagation: atomic adds of (k, w, d) along the path, then vl -= 1.
// With W = 1 nothing races, the virtual-loss terms are zero at every read and
// the search is the sequential UCT of the oracle with one tree, bit for bit
// (tests/test_gpu_tree.py). With W > 1 the result depends on timing (as on
// any parallel machine): tests check the tree invariants (tree_check_kernel).
//
// All tree fields are read with L1-bypassing loads (ld.relaxed/acquire.gpu):
// a slot published by another SM may share an L1 line with a slot this SM
// already read.
#pragma once
#include <cstdint>
#include "reversi_device.cuh"
#include "tree_device.cuh"

namespace mcts_dev {

struct TreeSync {
  u32 ticket;              // next iteration ticket (Philox c1)
  u32 used;                // slot allocator
  unsigned long long ends; // invariant check: sum over nodes of k - sum(children k)
};

__device__ __forceinline__ u32 ld_acq(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ u32 ld_rlx(const u32* p) {
  u32 v;
  asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(u32* p, u32 v) {
  asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Create node s (one thread): board, counters, the creator's virtual visit,
// its child block (limit slots, or kNoChild when the pool is full: the node
// is then never expanded, R12), and publish.
__device__ __forceinline__ void tree_init_node(const TreePool& T, TreeSync* S, u32 s, u64 own, u64 opp,
                                               u32 move, u32 vl0) {
  const u64 lg = legal_moves(own, opp);
  const bool term = is_terminal(own, opp, lg);
  const u32 limit = term ? 0u : (lg ? (u32)__popcll(lg) : 1u);
  u32 first = kNoChild;
  if (limit) {
    const u32 f = atomicAdd(&S->used, limit);
    if ((unsigned long long)f + limit <= T.slot_cap) first = f;
  }
  T.own[s] = own;
  T.opp[s] = opp;
  T.legal[s] = lg;
  T.k[s] = 0;
  T.w[s] = 0;
  T.d[s] = 0;
  T.vl[s] = vl0;
  T.first[s] = first;
  st_rel(&T.meta[s], (limit << 8) | (move << 16) | ((term ? 1u : 0u) << 24));  // != 0: published
}

__global__ void tree_root_kernel(TreePool T, TreeSync* S, DevPosition root) {
  S->ticket = 0;
  S->used = 1;
  S->ends = 0;
  const u64 own = root.to_move ? root.white : root.black;
  const u64 opp = root.to_move ? root.black : root.white;
  tree_init_node(T, S, 0, own, opp, 0xFFu, 0u);
}

// Selection + expansion on the shared tree by one warp (see the header). The
// path (shared) gets root..leaf; every node on it carries this worker's
// virtual visit on return.
//
// One load round trip per level: the lanes read every child's (meta, k, vl, w,
// first) together with relaxed loads, and the winner's values become the next
// level's node state (its meta, first, and k + vl for the parent term) without
// re-reading. A child read that races its creation sees either meta == 0
// (skipped) or the cleared pool values (k = vl = w = 0, first = kNoChild:
// the node is then simulated instead of descended; both harmless, W = 1 never
// races). Boards are read after an acquire fence.
__device__ __forceinline__ LeafInfo tree_select_expand(const TreePool& T, TreeSync* S, u32* path,
                                                       const double* __restrict__ lnT, u32 unit,
                                                       double C, int lane) {
  u32 v = 0;
  int depth = 0;
  // lane 0's reads, broadcast: other workers change the root concurrently, so
  // lanes reading it themselves could disagree and split the warp
  u32 meta = 0, first = 0, kp = 0;
  if (lane == 0) {
    meta = ld_acq(&T.meta[0]);
    first = ld_rlx(&T.first[0]);
    kp = ld_rlx(&T.k[0]) + ld_rlx(&T.vl[0]);  // read before our own virtual visit
  }
  meta = __shfl_sync(kFull, meta, 0);
  first = __shfl_sync(kFull, first, 0);
  kp = __shfl_sync(kFull, kp, 0);
  if (lane == 0) {
    path[0] = 0;
    atomicAdd(&T.vl[0], 1u);
  }
  u32 refused = 0;
  for (;;) {
    if (meta_term(meta) || depth >= kMaxPath - 2) break;
    if (first == kNoChild) {
      // Either v's child block was refused when v was created (pool full, R12)
      // or the batch read of v's fields raced its publication (meta seen,
      // first still the cleared value). Lane 0 re-reads first after a fence,
      // so only a real refusal is counted; either way v is simulated in place.
      if (lane == 0) {
        __threadfence();
        first = ld_acq(&T.first[v]);
      }
      first = __shfl_sync(kFull, first, 0);
      if (first == kNoChild) {
        refused = 1;
        break;
      }
    }
    // Expansion: claim the lowest-index untried move (one CAS on the counter).
    if (meta_nchild(meta) < meta_limit(meta)) {
      u32 claimed = kNoChild, mnow = meta;
      if (lane == 0) {
        u32 m = meta;
        while (meta_nchild(m) < meta_limit(m)) {
          const u32 old = atomicCAS(&T.meta[v], m, m + 1u);
          if (old == m) { claimed = meta_nchild(m); break; }
          m = old;
        }
        mnow = m;
        if (claimed != kNoChild) {
          __threadfence();  // acquire: v's board was published before its meta
          const u64 own = __ldcg(&T.own[v]), opp = __ldcg(&T.opp[v]), lg = __ldcg(&T.legal[v]);
          const u32 c = first + claimed;
          MCTS_CHECK(c < T.slot_cap && depth + 1 < kMaxPath);
          if (lg == 0ULL) {
            tree_init_node(T, S, c, opp, own, 64u, 1u);  // pass: same discs, turn swaps
          } else {
            const int sq = kth_set_bit(lg, claimed);
            const u64 f = flips(sq, own, opp);
            tree_init_node(T, S, c, opp & ~f, own | f | (1ULL << sq), (u32)sq, 1u);
          }
          path[depth + 1] = c;
        }
      }
      claimed = __shfl_sync(kFull, claimed, 0);
      if (claimed != kNoChild) {
        v = first + claimed;
        ++depth;
        break;
      }
      meta = __shfl_sync(kFull, mnow, 0);  // fully claimed meanwhile: select among the children
    }
    // Selection: UCB over the published children with virtual visits.
    const u32 nch = meta_nchild(meta);
    const double lnp = lnT[kp];  // parent count k + vl without our own virtual visit
    double best_u = -__longlong_as_double(0x7FF0000000000000LL);
    u32 best_i = kNoChild, best_meta = 0, best_first = kNoChild, best_k = 0;
    for (u32 i = (u32)lane; i < nch; i += 32u) {
      const u32 c = first + i;
      MCTS_CHECK(c < T.slot_cap);
      const u32 mc = ld_rlx(&T.meta[c]);
      const u32 kc = ld_rlx(&T.k[c]), vc = ld_rlx(&T.vl[c]), wc = ld_rlx(&T.w[c]);
      const u32 fc = ld_rlx(&T.first[c]);
      if (mc == 0u) continue;  // claimed, not yet published
      const u32 kk = kc + vc;
      const double u = ucb_value(wc, kk ? kk : 1u, unit, lnp, C);
      if (u > best_u || best_i == kNoChild) {
        best_u = u; best_i = i; best_meta = mc; best_first = fc; best_k = kk;
      }
    }
    best_i = warp_argmax(best_u, best_i);  // lanes without a published child hold kNoChild
    if (best_i == kNoChild) break;  // no child published yet: simulate from v
    const int src = (int)(best_i & 31u);
    v = first + best_i;
    meta = __shfl_sync(kFull, best_meta, src);
    first = __shfl_sync(kFull, best_first, src);
    kp = __shfl_sync(kFull, best_k, src);  // v's k + vl, read before our own virtual visit
    ++depth;
    if (lane == 0) {
      MCTS_CHECK(depth < kMaxPath && v < T.slot_cap);
      path[depth] = v;
      atomicAdd(&T.vl[v], 1u);
    }
  }
  __syncwarp();
  __threadfence();  // acquire: the leaf's board was published before its meta
  LeafInfo L;
  L.own = __ldcg(&T.own[v]);
  L.opp = __ldcg(&T.opp[v]);
  L.term = meta_term(ld_acq(&T.meta[v])) ? 1u : 0u;
  L.refused = refused;
  L.depth = depth;
  return L;
}

// Backpropagation with atomics (lanes over the path), then the virtual
// visits are withdrawn (after the counts, so k + vl never drops to 0).
__device__ __forceinline__ void tree_backprop(const TreePool& T, const u32* path, int depth, u32 W, u32 D,
                                              u32 Lo, int lane) {
  for (int p = lane; p <= depth; p += 32) {
    const u32 s = path[p];
    const int lvl = depth - p;
    atomicAdd(&T.k[s], 1u);
    const u32 x = (lvl & 1) ? W : Lo;
    if (x) atomicAdd(&T.w[s], x);
    if (D) atomicAdd(&T.d[s], D);
  }
  __threadfence();
  for (int p = lane; p <= depth; p += 32) atomicSub(&T.vl[path[p]], 1u);
  __syncwarp();
}

template <int MAX_THREADS, int MIN_BLOCKS>
__global__ void __launch_bounds__(MAX_THREADS, MIN_BLOCKS)
tree_search_kernel(TreePool T, SearchArgs a, TreeSync* S) {
  __shared__ u32 path[kMaxPath];
  __shared__ u64 s_own, s_opp;
  __shared__ u32 s_term, s_stop, s_it;
  __shared__ u32 s_w[32], s_d[32];
  __shared__ int s_depth;
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, a.rays);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nwarps = blockDim.x >> 5;
  const u32 unit = blockDim.x;
  const u64 deadline = a.budget_ns ? (*a.t0 + a.budget_ns) : 0ULL;
  __syncthreads();

  u32 plies = 0;
  u32 done = 0;
  unsigned long long depth_sum = 0;  // lane 0 of warp 0
  unsigned long long refused = 0;    // lane 0 of warp 0
  if (!meta_term(ld_acq(&T.meta[0]))) {
    for (;;) {
      if (warp == 0) {
        u32 stop = 0, it = 0;
        if (lane == 0) {
          if (a.budget_ns && globaltimer_ns() >= deadline) {
            stop = 1;
          } else {
            it = atomicAdd(&S->ticket, 1u);
            stop = it >= a.max_iterations;
          }
        }
        stop = __shfl_sync(kFull, stop, 0);
        if (!stop) {
          const LeafInfo L = tree_select_expand(T, S, path, a.lnT, unit, a.C, lane);
          if (lane == 0) {
            s_own = L.own; s_opp = L.opp; s_term = L.term; s_depth = L.depth; s_it = it;
            depth_sum += (unsigned)L.depth;
            refused += L.refused;
          }
        }
        if (lane == 0) s_stop = stop;
      }
      __syncthreads();
      if (s_stop) break;
      int r;
      if (s_term) {
        const int x = __popcll(s_own), y = __popcll(s_opp);
        r = (x > y) - (x < y);
      } else {
        r = playout(s_own, s_opp, a.key, a.tree_id_base, s_it, (u32)tid, s_rays, &plies);
      }
      const u32 bw = __popc(__ballot_sync(kFull, r == 1));
      const u32 bd = __popc(__ballot_sync(kFull, r == 0));
      if (lane == 0) { s_w[warp] = bw; s_d[warp] = bd; }
      __syncthreads();
      if (warp == 0) {
        u32 W = lane < nwarps ? s_w[lane] : 0u;
        u32 D = lane < nwarps ? s_d[lane] : 0u;
        W = __reduce_add_sync(kFull, W);
        D = __reduce_add_sync(kFull, D);
        tree_backprop(T, path, s_depth, W, D, unit - W - D, lane);
      }
      ++done;
    }
  }
  const u32 bp = __reduce_add_sync(kFull, plies);
  if (lane == 0) s_w[warp] = bp;
  __syncthreads();
  if (warp == 0) {
    unsigned long long P = lane < nwarps ? s_w[lane] : 0u;
    for (int off = 16; off > 0; off >>= 1) P += __shfl_xor_sync(kFull, P, off);
    unsigned long long* st = reinterpret_cast<unsigned long long*>(a.stats);
    if (lane == 0 && P) atomicAdd(st + 197, P);
    if (lane == 0 && done) atomicAdd(st + 196, (unsigned long long)done);
    if (lane == 0 && depth_sum) atomicAdd(st + 198, depth_sum);
    if (lane == 0 && refused) atomicAdd(st + 199, refused);
  }
}

// Root merge (a10) of the shared tree, after the search kernel (stream order),
// plus the pool diagnostics [200] slots used, [201] capacity (see merge_pool).
__global__ void tree_merge_kernel(TreePool T, const TreeSync* S, u32 unit, long long* stats) {
  merge_root(T, 0, unit, 0u, stats, threadIdx.x & 31);
  if (threadIdx.x == 0 && !meta_term(T.meta[0]))
    merge_pool(stats, 0ULL, S->used < T.slot_cap ? S->used : T.slot_cap, T.slot_cap);
}

// Before a search: clear the fields a racing reader may see (meta = 0:
// unpublished; k = w = vl = 0; first = kNoChild) over the slots the previous
// search of this pool carving used (S->used, clamped to the capacity); the
// rest of the pool is still clean from the last full clear.
__global__ void tree_clear_kernel(TreePool T, const TreeSync* S) {
  const u32 n = S->used < T.slot_cap ? S->used : T.slot_cap;
  for (u32 s = blockIdx.x * blockDim.x + threadIdx.x; s < n; s += gridDim.x * blockDim.x) {
    T.meta[s] = 0u;
    T.k[s] = 0u;
    T.w[s] = 0u;
    T.vl[s] = 0u;
    T.first[s] = kNoChild;
  }
}

// Invariants of the finished tree (MCTS_FLAG_CHECK_TREE): every published node
// has vl = 0, w + d <= k * unit, and k >= sum of its children's k (+1 for a
// non-root node: the iteration that created it ended there); summed over all
// nodes, k - sum(children k) = the iterations run. Violations set *error = 2.
__global__ void tree_check_kernel(TreePool T, TreeSync* S, u32 unit, u32 n_slots, int* error) {
  unsigned long long ends = 0;
  for (u32 s = blockIdx.x * blockDim.x + threadIdx.x; s < n_slots; s += gridDim.x * blockDim.x) {
    const u32 meta = T.meta[s];
    if (meta == 0u) continue;
    bool bad = T.vl[s] != 0u || (unsigned long long)T.w[s] + T.d[s] > (unsigned long long)T.k[s] * unit;
    unsigned long long ch = 0;
    const u32 first = T.first[s];
    if (first != kNoChild)
      for (u32 i = 0; i < meta_nchild(meta); ++i) {
        if (T.meta[first + i] == 0u) bad = true;  // claimed but never published
        ch += T.k[first + i];
      }
    if (ch + (s ? 1u : 0u) > T.k[s]) bad = true;
    ends += T.k[s] - ch;
    if (bad) atomicExch(error, 2);
  }
  for (int off = 16; off > 0; off >>= 1) ends += __shfl_xor_sync(kFull, ends, off);
  if ((threadIdx.x & 31) == 0 && ends) atomicAdd(&S->ends, ends);
}

__global__ void tree_check_total_kernel(const TreeSync* S, const long long* stats, int* error) {
  if (S->ends != (unsigned long long)stats[196]) atomicExch(error, 2);
}

}  // namespace mcts_dev
