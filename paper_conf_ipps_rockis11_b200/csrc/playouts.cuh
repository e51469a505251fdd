// playouts.cuh — the headline kernel (a1-a6): batched random playouts with a
// warp-ballot W/D/L reduction. Kept in its own file so the
// committed ncu capture of this kernel can be tied to its sources
// (bench.py kernel_source_hash: reversi_device.cuh + this file + nvcc flags).
#pragma once
#include <cstdint>
#include "reversi_device.cuh"

namespace mcts_dev {

constexpr unsigned kFullMask = 0xFFFFFFFFu;

struct DevPosition {  // layout of mcts_position
  u64 black, white;
  u32 to_move, reserved;
};

struct WdlOut {  // layout of mcts_wdl
  u32 wins, draws, losses;
};

// ---------------------------------------------------------------------------
// Batched playouts, persistent: the grid is sized to the resident capacity and
// each warp repeatedly takes the next chunk of 32 playouts from a work counter
// (dynamic balancing; the per-CTA ray table is loaded once). Playout g of a
// launch is playout j = g mod n_per_leaf of leaf g / n_per_leaf (leaf-major, so
// a warp's 32 lanes usually share a leaf and finish within a ply or two of each
// other); its RNG stream is (c0 = leaf_id_base + leaf, c1, c2 = j) — c1 = 0
// for mcts_playouts, the step for the CPU-managed trees of mcts_search_hosted.
// Outcomes are reduced per (warp, leaf) with match_any + ballot + popc
// and added with one atomic per counter; plies with one atomic per warp.
// ---------------------------------------------------------------------------
#ifndef MCTS_PLAYOUT_THREADS
#define MCTS_PLAYOUT_THREADS 256
#endif
#ifndef MCTS_PLAYOUT_MINB
#define MCTS_PLAYOUT_MINB 1
#endif
constexpr int kPlayoutThreads = MCTS_PLAYOUT_THREADS;

__global__ void rays_init_kernel(u64* g_rays) {
  fill_rays(g_rays);
}

__device__ __forceinline__ void load_rays(u64* s_rays, const u64* __restrict__ g_rays) {
  for (int i = threadIdx.x; i < kRayTable; i += blockDim.x) s_rays[i] = g_rays[i];
}

#ifndef MCTS_LANE_STREAM
#define MCTS_LANE_STREAM 0  // > 0: R playouts per lane per chunk, each lane restarts on its own
#endif

#if MCTS_LANE_STREAM
// Variant: a warp takes a chunk of 32*R playouts; lane l plays playouts
// l, l + 32, ..., l + 32 (R - 1) of the chunk back to back, starting the next
// as soon as its current one ends (ply pairs as in playout()), so a lane
// idles only at the end of the chunk instead of at the end of every playout.
// Results accumulate per lane while the leaf stays the same and are flushed
// with atomics (warp-aggregated by leaf at the chunk end). Same RNG streams,
// same W/D/L as playouts_kernel.
__device__ __forceinline__ void flush_wdl(WdlOut* out, u32 leaf, u32 w, u32 d, u32 l) {
  if (w) atomicAdd(&out[leaf].wins, w);
  if (d) atomicAdd(&out[leaf].draws, d);
  if (l) atomicAdd(&out[leaf].losses, l);
}

__global__ void __launch_bounds__(kPlayoutThreads, MCTS_PLAYOUT_MINB)
playouts_kernel(const DevPosition* __restrict__ leaves, u32 n_leaves, u32 n_per_leaf, uint2 key,
                u32 leaf_id_base, u32 c1, WdlOut* __restrict__ out, unsigned long long* plies_out,
                const u64* __restrict__ g_rays, u32* __restrict__ work) {
  constexpr u32 R = MCTS_LANE_STREAM;
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, g_rays);
  __syncthreads();
  const u64 total = (u64)n_leaves * n_per_leaf;
  const u32 n_chunks = (u32)((total + 32 * R - 1) / (32 * R));
  const int lane = threadIdx.x & 31;
  u32 plies = 0;
  PlayoutRng rng;
  rng.key = key; rng.c1 = c1; rng.c0 = 0; rng.c2 = 0; rng.w = 0;
  rng.buf = make_uint4(0, 0, 0, 0);
  for (;;) {
    u32 chunk = 0;
    if (lane == 0) chunk = atomicAdd(work, 1u);
    chunk = __shfl_sync(kFullMask, chunk, 0);
    if (chunk >= n_chunks) break;
    const u64 base = (u64)chunk * (32u * R) + (u32)lane;
    u32 r = 0, n = 0, empties = 0;
    bool busy = false, passed = false;
    u64 me = 0, op = 0;
    u32 acc = 0xFFFFFFFFu, aw = 0, ad = 0, al = 0;
    for (;;) {
      if (!busy && r < R) {
        const u64 g = base + 32ull * r;
        ++r;
        if (g < total) {
          const u32 leaf = (u32)(g / n_per_leaf);
          if (leaf != acc) {
            if (acc != 0xFFFFFFFFu) flush_wdl(out, acc, aw, ad, al);
            acc = leaf; aw = ad = al = 0;
          }
          const DevPosition p = leaves[leaf];
          me = p.to_move ? p.white : p.black;
          op = p.to_move ? p.black : p.white;
          rng.c0 = leaf_id_base + leaf;
          rng.c2 = (u32)(g - (u64)leaf * n_per_leaf);
          n = 0;
          passed = false;
          empties = 64u - (u32)__popcll(me | op);
          busy = true;
        }
      }
      if (!__any_sync(kFullMask, busy)) break;
      if (busy) {  // one ply pair of playout()
        bool end = n == empties;
        if (!end) {
          if (ply(me, op, rng, n, s_rays)) { passed = false; ++n; }
          else if (passed) end = true;
          else passed = true;
        }
        if (!end) {
          end = n == empties;
          if (!end) {
            if (ply(op, me, rng, n, s_rays)) { passed = false; ++n; }
            else if (passed) end = true;
            else passed = true;
          }
        }
        if (end) {
          plies += n;
          const int a = __popcll(me), b = __popcll(op);
          aw += a > b; ad += a == b; al += a < b;
          busy = false;
        }
      }
    }
    // chunk end: one atomic per counter per (warp, leaf)
    const u32 grp = __match_any_sync(kFullMask, acc);
    const u32 sw = __reduce_add_sync(grp, aw), sd = __reduce_add_sync(grp, ad), sl = __reduce_add_sync(grp, al);
    if (acc != 0xFFFFFFFFu && lane == __ffs(grp) - 1) flush_wdl(out, acc, sw, sd, sl);
  }
  if (plies_out) {
    const u32 s = __reduce_add_sync(kFullMask, plies);
    if (lane == 0 && s) atomicAdd(plies_out, (unsigned long long)s);
  }
}
#else
__global__ void __launch_bounds__(kPlayoutThreads, MCTS_PLAYOUT_MINB)
playouts_kernel(const DevPosition* __restrict__ leaves, u32 n_leaves, u32 n_per_leaf, uint2 key,
                u32 leaf_id_base, u32 c1, WdlOut* __restrict__ out, unsigned long long* plies_out,
                const u64* __restrict__ g_rays, u32* __restrict__ work) {
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, g_rays);
  __syncthreads();
  const u64 total = (u64)n_leaves * n_per_leaf;
  const u32 n_chunks = (u32)((total + 31) / 32);
  const int lane = threadIdx.x & 31;
  u32 plies = 0;
  for (;;) {
    u32 chunk = 0;
    if (lane == 0) chunk = atomicAdd(work, 1u);
    chunk = __shfl_sync(kFullMask, chunk, 0);
    if (chunk >= n_chunks) break;
    const u64 g = (u64)chunk * 32u + (u32)lane;
    const bool active = g < total;
    u32 leaf = 0xFFFFFFFFu;
    int r = 2;
    if (active) {
      leaf = (u32)(g / n_per_leaf);
      const u32 j = (u32)(g - (u64)leaf * n_per_leaf);
      const DevPosition p = leaves[leaf];
      const u64 own = p.to_move ? p.white : p.black;
      const u64 opp = p.to_move ? p.black : p.white;
      r = playout(own, opp, key, leaf_id_base + leaf, c1, j, s_rays, &plies);
    }
    const u32 grp = __match_any_sync(kFullMask, leaf);
    const u32 wins = __popc(__ballot_sync(kFullMask, r == 1) & grp);
    const u32 draws = __popc(__ballot_sync(kFullMask, r == 0) & grp);
    const u32 losses = __popc(__ballot_sync(kFullMask, r == -1) & grp);
    if (active && lane == __ffs(grp) - 1) {
      if (wins) atomicAdd(&out[leaf].wins, wins);
      if (draws) atomicAdd(&out[leaf].draws, draws);
      if (losses) atomicAdd(&out[leaf].losses, losses);
    }
  }
  if (plies_out) {
    const u32 s = __reduce_add_sync(kFullMask, plies);
    if (lane == 0 && s) atomicAdd(plies_out, (unsigned long long)s);
  }
}
#endif

}  // namespace mcts_dev
