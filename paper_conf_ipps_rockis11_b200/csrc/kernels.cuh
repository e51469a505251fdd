// kernels.cuh — the sm_100a kernels of the hot path.
//
//   playouts_kernel      a1-a6: batched random playouts, warp ballot W/D/L
//   block_search_kernel  a1-a10: block-parallel UCT, one tree per CTA
//                        (PAPER.md L294-L311), root merge fused at the end
//   leaf_search_kernel   a12: leaf-parallel UCT, one tree, the whole grid
//                        simulates from the same leaf
//   tree_search_kernel   NEXT-4: tree parallelism, every CTA on one shared tree
//                        with virtual loss (tree_parallel.cuh)
//   ln_table_kernel      lnT[k] = RN(ln(k*unit)) for the UCB term (R9)
//   gen_positions_kernel synthetic input recipe
#pragma once
#include <cstdint>
#include <cooperative_groups.h>
#include "reversi_device.cuh"
#include "ln_device.cuh"
#include "tree_device.cuh"
#include "playouts.cuh"

namespace mcts_dev {

__device__ __forceinline__ u64 globaltimer_ns() {
  u64 t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// ---------------------------------------------------------------------------
// Block-parallel UCT: CTA t owns tree t. Per iteration
// warp 0 selects + expands (warp-cooperative UCB argmax), every thread plays
// one playout from the new leaf (c0 = tree id, c1 = iteration, c2 = thread),
// warps reduce outcomes with ballot/popc, warp 0 backpropagates. No host
// round trip and no inter-CTA communication until the fused root merge.
// ---------------------------------------------------------------------------
struct SearchArgs {
  DevPosition root;
  uint2 key;
  double C;
  const double* lnT;
  long long* stats;      // MCTS_STATS_LEN int64 (accumulated)
  const u64* t0;         // device timestamp written before the launch (time mode)
  u64 budget_ns;         // 0 = iteration mode
  u32 max_iterations;    // iteration budget, or the time-mode cap
  u32 tree_id_base;
  u32 unit;              // playouts per iteration per tree
  int* error;            // reserved error flag (0 = ok)
  const u64* rays;       // global ray table (kRayTable u64)
};


#ifndef MCTS_BLOCK_BOARDS
#define MCTS_BLOCK_BOARDS false  // block kernel: read the chosen leaf's board after the descent (fewer registers)
#endif

template <int MAX_THREADS, int MIN_BLOCKS>
__global__ void __launch_bounds__(MAX_THREADS, MIN_BLOCKS)
block_search_kernel(TreePool T, SearchArgs a) {
  __shared__ PathCache pc;
  __shared__ u64 s_own, s_opp;
  __shared__ u32 s_term, s_stop, s_slot_used;
  __shared__ u32 s_w[32], s_d[32];
  __shared__ int s_depth;
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, a.rays);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nwarps = blockDim.x >> 5;
  const u32 tree = blockIdx.x;
  const size_t base = (size_t)tree * T.slot_cap;
  const u32 c0 = a.tree_id_base + tree;
  const u32 unit = blockDim.x;
  const u64 deadline = a.budget_ns ? (*a.t0 + a.budget_ns) : 0ULL;

  if (tid == 0) {
    const u64 own = a.root.to_move ? a.root.white : a.root.black;
    const u64 opp = a.root.to_move ? a.root.black : a.root.white;
    init_root(T, base, own, opp, &pc);
    s_slot_used = 1;
  }
  __syncthreads();

  u32 plies = 0;
  u32 it = 0;
  unsigned long long depth_sum = 0;  // lane 0 of warp 0: sum of leaf depths (Fig. 8 "Depth")
  unsigned long long refused = 0;    // lane 0 of warp 0: expansions refused by a full pool
  if (!meta_term(pc.root_meta)) {
    for (;; ++it) {
      if (warp == 0) {
        u32 stop = 0;
        if (lane == 0) {
          stop = it >= a.max_iterations;
          if (!stop && a.budget_ns) stop = globaltimer_ns() >= deadline;
        }
        stop = __shfl_sync(kFull, stop, 0);
        if (!stop) {
          const LeafInfo L = select_expand<MCTS_BLOCK_BOARDS>(T, base, &pc, &s_slot_used, a.lnT, unit, a.C, lane, s_rays);
          if (lane == 0) {
            s_own = L.own; s_opp = L.opp; s_term = L.term; s_depth = L.depth;
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
        r = playout(s_own, s_opp, a.key, c0, it, (u32)tid, s_rays, &plies);
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
        backprop(T, base, &pc, s_depth, W, D, unit - W - D, lane);
      }
    }
  }
  // fused per-GPU root merge (a10) + ply count
  const u32 bp = __reduce_add_sync(kFull, plies);
  if (lane == 0) s_w[warp] = bp;
  __syncthreads();
  if (warp == 0) {
    unsigned long long P = lane < nwarps ? s_w[lane] : 0u;
    for (int off = 16; off > 0; off >>= 1) P += __shfl_xor_sync(kFull, P, off);
    if (lane == 0 && P) atomicAdd(reinterpret_cast<unsigned long long*>(a.stats) + 197, P);
    if (lane == 0 && depth_sum) atomicAdd(reinterpret_cast<unsigned long long*>(a.stats) + 198, depth_sum);
    if (lane == 0 && !meta_term(pc.root_meta)) merge_pool(a.stats, refused, s_slot_used, T.slot_cap);
    merge_root(T, base, unit, it, a.stats, lane);
  }
}

// ---------------------------------------------------------------------------
// Leaf-parallel UCT: one tree; every thread of the grid
// plays out from the same leaf each iteration. CTA 0's warp 0 owns the tree
// (select/expand/backprop). Per iteration: the leader publishes the leaf in a
// small global struct and releases it with an iteration-stamped flag (thread
// 0 of every other CTA spins on it with acquire loads, then a CTA barrier) ->
// every thread simulates, CTAs ballot-reduce and add their wins/draws with
// atomics -> one cooperative-groups grid barrier -> the leader backpropagates
// and selects. All CTAs are co-resident (cooperative launch). Round 1 used a
// grid barrier for the leaf hand-off too; after cg's grid.sync the CTAs' warp
// 0 ran its playouts split in two (24.6 instead of 30.4 threads per
// instruction, ncu r2z3), which doubled the batch latency: 53 -> 31 us per
// iteration with the flag. MCTS_LEAF_POST (CTAs post packed
// sums, the leader polls: no grid barrier at all) measured 4% slower.
// ---------------------------------------------------------------------------
// Tooling only (tools/leaf_compare.py variants): 1 = the leaf kernel skips the
// playouts (every result a draw), so its iteration time is the serial part
// alone (barriers, backprop, selection, expansion). Never set in a product build.
#ifndef MCTS_LEAF_PROBE
#define MCTS_LEAF_PROBE 0
#endif

#ifndef MCTS_LEAF_FLAG
#define MCTS_LEAF_FLAG 1  // the leader publishes the leaf with a release flag instead of a grid barrier
#endif
#ifndef MCTS_LEAF_POST
#define MCTS_LEAF_POST 0  // CTAs post (count, wins, draws) in one packed atomic; the leader polls it
#endif


struct LeafSync {
  u64 own, opp;
  u32 term, stop;
  u32 wd[2][2];     // per-iteration-parity wins, draws (grid-barrier variant)
  u32 flag;         // MCTS_LEAF_FLAG: iteration + 1 of the published leaf
  u32 pad;
  unsigned long long post[2];  // MCTS_LEAF_POST, per iteration parity: CTAs << 48 | wins << 24 | draws
};

__device__ __forceinline__ unsigned long long leaf_ld_relaxed64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ u32 leaf_ld_acquire(const u32* p) {
  u32 v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__global__ void __launch_bounds__(128)
leaf_search_kernel(TreePool T, SearchArgs a, LeafSync* S) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  __shared__ PathCache pc;
  __shared__ u32 s_slot_used;
  __shared__ int s_depth;
  __shared__ u32 s_w[4], s_d[4];
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, a.rays);

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const bool leader = blockIdx.x == 0 && warp == 0;
  const u32 unit = a.unit;
  const u64 deadline = a.budget_ns ? (*a.t0 + a.budget_ns) : 0ULL;
  if (blockIdx.x == 0 && tid == 0) {
    const u64 own = a.root.to_move ? a.root.white : a.root.black;
    const u64 opp = a.root.to_move ? a.root.black : a.root.white;
    init_root(T, 0, own, opp, &pc);
    s_slot_used = 1;
  }
  __syncthreads();
  u32 plies = 0;
  u32 it = 0;
  unsigned long long depth_sum = 0;  // leader lane 0
  unsigned long long refused = 0;    // leader lane 0
  for (;; ++it) {
    if (leader) {
      if (it > 0) {
        const u32 par = (it - 1) & 1u;
#if MCTS_LEAF_POST
        // every CTA's (count, wins, draws) arrives in one packed word; lane 0
        // polls it with relaxed loads (no acquire: that would drop the tree's
        // lines from this SM's L1 on every poll) and clears the slot for
        // iteration it + 1 before the next leaf is published
        u32 W = 0, D = 0;
        if (lane == 0) {
          unsigned long long v;
          while (((v = leaf_ld_relaxed64(&S->post[par])) >> 48) != gridDim.x) {}
          W = (u32)(v >> 24) & 0xFFFFFFu;
          D = (u32)v & 0xFFFFFFu;
          S->post[par] = 0ULL;
        }
        W = __shfl_sync(kFull, W, 0);
        D = __shfl_sync(kFull, D, 0);
#else
        const u32 W = S->wd[par][0], D = S->wd[par][1];
        __syncwarp();
        if (lane == 0) { S->wd[par][0] = 0; S->wd[par][1] = 0; }
#endif
        backprop(T, 0, &pc, s_depth, W, D, unit - W - D, lane);
      }
      u32 stop = 0;
      if (lane == 0) {
        stop = meta_term(pc.root_meta) || it >= a.max_iterations;
        if (!stop && a.budget_ns) stop = globaltimer_ns() >= deadline;
      }
      stop = __shfl_sync(kFull, stop, 0);
      if (!stop) {
        const LeafInfo L = select_expand(T, 0, &pc, &s_slot_used, a.lnT, unit, a.C, lane, s_rays);
        if (lane == 0) {
          s_depth = L.depth; S->own = L.own; S->opp = L.opp; S->term = L.term;
          depth_sum += (unsigned)L.depth;
          refused += L.refused;
        }
      }
      if (lane == 0) S->stop = stop;
#if MCTS_LEAF_FLAG
      if (lane == 0) {
        __threadfence();
        asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(&S->flag), "r"(it + 1u) : "memory");
      }
#endif
    }
#if MCTS_LEAF_FLAG
    // one-to-all hand-off: the other CTAs wait for the leader's flag (their
    // acquire also drops stale lines of S from their SM's L1); CTA 0 reads
    // the leaf its own warp 0 wrote after the CTA barrier. The results still
    // come back through the grid barrier below.
    if (blockIdx.x != 0 && tid == 0) {
      while (leaf_ld_acquire(&S->flag) != it + 1u) {}
    }
    __syncthreads();
    __syncwarp();  // every warp enters the playouts converged (see the note above the kernel)
#else
    grid.sync();
#endif
    const u32 stop = __ldcg(&S->stop);
    const u64 own = __ldcg(&S->own), opp = __ldcg(&S->opp);
    const u32 term = __ldcg(&S->term);
    if (stop) break;
    int r;
    if (term) {
      const int x = __popcll(own), y = __popcll(opp);
      r = (x > y) - (x < y);
    } else {
#if MCTS_LEAF_PROBE
      r = 0;
#else
      r = playout(own, opp, a.key, a.tree_id_base, it, blockIdx.x * blockDim.x + tid, s_rays, &plies);
#endif
    }
    const u32 bw = __popc(__ballot_sync(kFull, r == 1));
    const u32 bd = __popc(__ballot_sync(kFull, r == 0));
    if (lane == 0) { s_w[warp] = bw; s_d[warp] = bd; }
    __syncthreads();
    if (tid == 0) {
      const u32 par = it & 1u;
#if MCTS_LEAF_POST
      const unsigned long long w = s_w[0] + s_w[1] + s_w[2] + s_w[3], d = s_d[0] + s_d[1] + s_d[2] + s_d[3];
      atomicAdd(&S->post[par], (1ULL << 48) | (w << 24) | d);
#else
      atomicAdd(&S->wd[par][0], s_w[0] + s_w[1] + s_w[2] + s_w[3]);
      atomicAdd(&S->wd[par][1], s_d[0] + s_d[1] + s_d[2] + s_d[3]);
#endif
    }
#if !MCTS_LEAF_POST
    grid.sync();
#endif
  }
  const u32 bp = __reduce_add_sync(kFull, plies);
  if (lane == 0 && bp) atomicAdd(reinterpret_cast<unsigned long long*>(a.stats) + 197, (unsigned long long)bp);
  if (leader && lane == 0 && depth_sum)
    atomicAdd(reinterpret_cast<unsigned long long*>(a.stats) + 198, depth_sum);
  if (leader && lane == 0 && !meta_term(pc.root_meta)) merge_pool(a.stats, refused, s_slot_used, T.slot_cap);
  if (leader) merge_root(T, 0, unit, it, a.stats, lane);
}

}  // namespace mcts_dev

#include "tree_parallel.cuh"

namespace mcts_dev {

// ---------------------------------------------------------------------------
__global__ void ln_table_kernel(double* __restrict__ out, u32 unit, u32 K) {
  const u32 k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k > K) return;
  out[k] = k == 0 ? 0.0 : ln_rn((unsigned long long)k * unit);
}

__global__ void stamp_kernel(u64* t0) { *t0 = globaltimer_ns(); }

// ---------------------------------------------------------------------------
// Perft (leaf count of the move tree to a given depth) with the hot-loop move
// generator and flips (legal_moves_hot / flips_loop), to pin them directly to
// the north_star perft counts. Stage 1 (one thread) lists the frontier at
// depth `split`; stage 2 runs one depth-first search per frontier node with an
// explicit stack. A game-over node before the depth counts 1; a pass consumes
// a ply iff pass_is_ply (R11).
// ---------------------------------------------------------------------------
struct PerftNode {
  u64 own, opp;
  u32 depth;  // remaining depth
  u32 pad;
};

__device__ __forceinline__ u64 perft_moves(u64 P, u64 O) {
  return legal_moves_hot(P, O, __brevll(P), __brevll(O));
}

// Depth-first leaf count from (own, opp) with `depth` plies to go. Nodes whose
// remaining depth reaches `stop_at` (stage 1) are written to `frontier`
// instead of expanded. Stack frames hold a node and its untried moves, so the
// stack depth is at most 2 * depth + 1 (pass frames included).
__device__ unsigned long long perft_dfs(u64 own, u64 opp, u32 depth, u32 pass_is_ply, u32 stop_at,
                                        const u64* rays, PerftNode* frontier, u32 cap, u32* count) {
  struct F { u64 own, opp, moves; u32 depth, pass; };
  F st[2 * 16 + 2];
  int sp = 0;
  unsigned long long cnt = 0;
  auto push = [&](u64 o, u64 p, u32 d) {
    if (d == 0) { ++cnt; return; }
    if (d == stop_at) {
      const u32 k = atomicAdd(count, 1u);
      if (k < cap) frontier[k] = {o, p, d, 0};
      return;
    }
    const u64 m = perft_moves(o, p);
    if (m == 0ULL) {
      if (perft_moves(p, o) == 0ULL) { ++cnt; return; }  // game over: a leaf
      st[sp++] = {o, p, 0ULL, d, 1u};                     // pass
      return;
    }
    if (d == 1) { cnt += (u32)__popcll(m); return; }
    st[sp++] = {o, p, m, d, 0u};
  };
  push(own, opp, depth);
  while (sp > 0) {
    F& f = st[sp - 1];
    if (f.pass) {
      const F c = f;
      --sp;
      push(c.opp, c.own, pass_is_ply ? c.depth - 1 : c.depth);
      continue;
    }
    if (f.moves == 0ULL) { --sp; continue; }
    const int sq = __ffsll((long long)f.moves) - 1;
    f.moves &= f.moves - 1;
    const u64 fl = flips_loop(sq, f.own, f.opp, __brevll(f.own), __brevll(f.opp), rays);
    const u64 o = f.opp & ~fl, p = f.own | fl | (1ULL << sq);
    push(o, p, f.depth - 1);
  }
  return cnt;
}

__global__ void perft_frontier_kernel(u64 own, u64 opp, u32 depth, u32 stop_at, u32 pass_is_ply,
                                      const u64* __restrict__ g_rays, PerftNode* out, u32 cap,
                                      u32* count, unsigned long long* leaves) {
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, g_rays);
  __syncthreads();
  if (threadIdx.x != 0) return;
  const unsigned long long c = perft_dfs(own, opp, depth, pass_is_ply, stop_at, s_rays, out, cap, count);
  atomicAdd(leaves, c);
}

__global__ void perft_dfs_kernel(const PerftNode* __restrict__ nodes, u32 n, u32 pass_is_ply,
                                 const u64* __restrict__ g_rays, unsigned long long* leaves) {
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, g_rays);
  __syncthreads();
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const PerftNode v = nodes[i];
  const unsigned long long c = perft_dfs(v.own, v.opp, v.depth, pass_is_ply, 0xFFFFFFFFu, s_rays,
                                         nullptr, 0, nullptr);
  if (c) atomicAdd(leaves, c);
}

// Synthetic positions, one thread per position.
__global__ void gen_positions_kernel(uint2 key, u32 n, u32 lmin, u32 lmax, DevPosition* out) {
  const u32 p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  const u32 span = lmax - lmin + 1u;
  DevPosition q0;  // attempts are capped (never reached for lmax <= 50): opening
  q0.black = 0x0000000810000000ULL; q0.white = 0x0000001008000000ULL; q0.to_move = 0; q0.reserved = 0;
  out[p] = q0;
  for (u32 attempt = 0; attempt < (1u << 16); ++attempt) {
    PlayoutRng rng;
    rng.key = key; rng.c0 = p; rng.c1 = 0xFFFFFFFFu; rng.c2 = attempt; rng.w = 0;
    rng.buf = make_uint4(0, 0, 0, 0);
    const u32 L = lmin + __umulhi(rng.next(), span);
    u64 me = 0x0000000810000000ULL, op = 0x0000001008000000ULL;
    u32 stm = 0, plies = 0;
    bool ok = true, passed = false;
    while (plies < L) {
      const u64 m = legal_moves(me, op);
      if (m == 0ULL) {
        if (passed) { ok = false; break; }
        passed = true;
      } else {
        passed = false;
        const int sq = pick_square(m, rng.next());
        const u64 f = flips(sq, me, op);
        me |= f | (1ULL << sq);
        op &= ~f;
        ++plies;
      }
      const u64 t = me; me = op; op = t;
      stm ^= 1u;
    }
    if (!ok) continue;
    if (is_terminal(me, op, legal_moves(me, op))) continue;
    DevPosition q;
    q.black = stm == 0u ? me : op;
    q.white = stm == 0u ? op : me;
    q.to_move = stm;
    q.reserved = 0;
    out[p] = q;
    return;
  }
}

}  // namespace mcts_dev
