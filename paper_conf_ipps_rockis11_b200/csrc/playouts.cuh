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

#ifndef MCTS_PAIR
#define MCTS_PAIR 0  // tuning variant: two lock-step playouts per thread (playout_pair)
#endif

#if MCTS_PAIR
__device__ __forceinline__ void reduce_wdl(u32 leaf, int r, bool active, int lane, WdlOut* __restrict__ out) {
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

__global__ void __launch_bounds__(kPlayoutThreads, MCTS_PLAYOUT_MINB)
playouts_kernel(const DevPosition* __restrict__ leaves, u32 n_leaves, u32 n_per_leaf, uint2 key,
                u32 leaf_id_base, u32 c1, WdlOut* __restrict__ out, unsigned long long* plies_out,
                const u64* __restrict__ g_rays, u32* __restrict__ work) {
  __shared__ u64 s_rays[kRayTable];
  load_rays(s_rays, g_rays);
  __syncthreads();
  const u64 total = (u64)n_leaves * n_per_leaf;
  const u32 n_chunks = (u32)((total + 63) / 64);  // 64 playouts per warp chunk: lanes x 2
  const int lane = threadIdx.x & 31;
  u32 plies = 0;
  for (;;) {
    u32 chunk = 0;
    if (lane == 0) chunk = atomicAdd(work, 1u);
    chunk = __shfl_sync(kFullMask, chunk, 0);
    if (chunk >= n_chunks) break;
    const u64 gx = (u64)chunk * 64u + (u32)lane, gy = gx + 32u;
    const bool ax = gx < total, ay = gy < total;
    u32 lx = 0xFFFFFFFFu, ly = 0xFFFFFFFFu, jx = 0, jy = 0;
    u64 mx = 0, ox = 0, my = 0, oy = 0;
    if (ax) {
      lx = (u32)(gx / n_per_leaf);
      jx = (u32)(gx - (u64)lx * n_per_leaf);
      const DevPosition p = leaves[lx];
      mx = p.to_move ? p.white : p.black;
      ox = p.to_move ? p.black : p.white;
    }
    if (ay) {
      ly = (u32)(gy / n_per_leaf);
      jy = (u32)(gy - (u64)ly * n_per_leaf);
      const DevPosition p = leaves[ly];
      my = p.to_move ? p.white : p.black;
      oy = p.to_move ? p.black : p.white;
    }
    int rx = 2, ry = 2;
    playout_pair(mx, ox, leaf_id_base + lx, jx, ax, my, oy, leaf_id_base + ly, jy, ay, key, c1, s_rays,
                 &plies, rx, ry);
    if (!ax) rx = 2;
    if (!ay) ry = 2;
    reduce_wdl(lx, rx, ax, lane, out);
    reduce_wdl(ly, ry, ay, lane, out);
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
