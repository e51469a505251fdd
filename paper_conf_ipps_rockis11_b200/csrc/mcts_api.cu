// mcts_api.cu — the C ABI (include/mcts.h) over the sm_100a kernels.
//
// Host side only marshals arguments, validates them, owns device scratch
// (tree pools, ln tables, staging) and launches kernels; every step of the hot
// path runs on the GPU. There is no CPU fallback: without an sm_100 device the
// compute calls fail with MCTS_E_NO_DEVICE. The one place host threads compute
// is mcts_search_hybrid, the paper's hybrid scheme, where they grow additional
// trees *alongside* a running GPU search (host_mcts.cpp).
#include <cuda_runtime.h>

#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/mcts.h"
#include "kernels.cuh"
#include "host_mcts.h"
#include "hosted.h"

using namespace mcts_dev;

static_assert(sizeof(mcts_position) == sizeof(DevPosition), "position layout");
static_assert(sizeof(mcts_wdl) == sizeof(WdlOut), "wdl layout");

// Playout launches take a fresh work counter from a ring, so concurrent launches
// on different streams of one handle (up to kWorkSlots in flight) never share one.
constexpr uint32_t kWorkSlots = 256;

struct mcts_handle {
  int device = 0;
  mcts_params params{};
  mcts_position position{};
  bool has_position = false;
  cudaStream_t stream = nullptr;  // for the synchronous entry points
  std::string last_error;

  // playout staging. d_wdl (mcts_playouts) is one region zeroed by one memset:
  // [u32 work counter, u32 pad, u64 plies, n x WdlOut]; h_pin_plies is the
  // pinned landing slot of its ply count.
  DevPosition* d_leaves = nullptr;
  size_t leaves_cap = 0;
  void* d_wdl = nullptr;
  size_t wdl_cap = 0;
  unsigned long long* d_plies = nullptr;
  unsigned long long* h_pin_plies = nullptr;
  // mcts_playouts_host_async: ring of device staging slots, each one region
  // [u32 work, u32 pad, u64 plies, n x WdlOut] followed by the leaves
  void* d_async[MCTS_HOST_ASYNC_SLOTS] = {};
  size_t async_cap[MCTS_HOST_ASYNC_SLOTS] = {};
  cudaEvent_t async_done[MCTS_HOST_ASYNC_SLOTS] = {};  // the slot's last D2H, for reuse from any stream
  uint32_t async_next = 0;

  // trees
  void* pool_mem = nullptr;
  size_t pool_bytes = 0;
  uint32_t tree_clean_cap = 0;  // MCTS_TREE: slot_cap of the carving whose unused slots are clear (0: none)

  // ln table
  double* d_lnT = nullptr;
  uint32_t lnT_unit = 0;
  uint32_t lnT_K = 0;
  size_t lnT_cap = 0;

  // search scratch
  long long* d_stats = nullptr;
  unsigned long long* d_t0 = nullptr;
  int* d_error = nullptr;
  LeafSync* d_leafsync = nullptr;
  TreeSync* d_treesync = nullptr;  // MCTS_TREE counters
  u64* d_rays = nullptr;      // ray table for the flip kernels (kRayTable u64)
  u32* d_work = nullptr;      // ring of playout work counters (one per launch)
  uint32_t work_slot = 0;
  int playout_ctas = 0;       // resident playout CTAs (SMs x occupancy)
  std::vector<double> host_lnT1;  // RN(ln k) for the hybrid's host trees

  // mcts_search_hosted: pinned leaf / result buffers and the step event
  mcts_position* h_pin_leaves = nullptr;
  mcts_wdl* h_pin_wdl = nullptr;
  size_t pin_cap = 0;
  cudaEvent_t step_event[2] = {};  // the two pipelined halves
  cudaStream_t stream2 = nullptr;  // the second half's stream (its kernels overlap the first half's)
};

namespace {

thread_local std::string g_create_error;

mcts_status fail(mcts_handle* h, mcts_status st, const std::string& msg) {
  if (h) h->last_error = msg;
  else g_create_error = msg;
  return st;
}

mcts_status cuda_fail(mcts_handle* h, cudaError_t e, const char* where) {
  cudaGetLastError();  // a reported (non-sticky) error must not leak into later calls
  std::string msg = std::string(where) + ": " + cudaGetErrorString(e);
  return fail(h, e == cudaErrorMemoryAllocation ? MCTS_E_OOM : MCTS_E_CUDA, msg);
}

#define CK(h, call)                                             \
  do {                                                          \
    cudaError_t e_ = (call);                                    \
    if (e_ != cudaSuccess) return cuda_fail((h), e_, #call);    \
  } while (0)

bool position_ok(const mcts_position& p) {
  return (p.black & p.white) == 0 && (p.to_move == 0u || p.to_move == 1u);
}

uint2 key_of(uint64_t seed) { return make_uint2((uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)); }

mcts_status ensure(mcts_handle* h, void** ptr, size_t* cap, size_t bytes) {
  if (*cap >= bytes && *ptr) return MCTS_OK;
  if (*ptr) { cudaFree(*ptr); *ptr = nullptr; *cap = 0; }
  size_t want = bytes < 256 ? 256 : bytes;
  cudaError_t e = cudaMalloc(ptr, want);
  if (e != cudaSuccess) { *ptr = nullptr; return cuda_fail(h, e, "cudaMalloc"); }
  *cap = want;
  return MCTS_OK;
}

// Device ln table for `unit` with at least K+1 entries (regenerated on demand).
mcts_status ensure_lnT(mcts_handle* h, uint32_t unit, uint32_t K, cudaStream_t s) {
  if (h->d_lnT && h->lnT_unit == unit && h->lnT_K >= K) return MCTS_OK;
  uint32_t Kalloc = K < 1024 ? 1024 : K;
  size_t bytes = ((size_t)Kalloc + 1) * sizeof(double);
  if (h->lnT_cap < bytes) {
    void* p = h->d_lnT;
    size_t cap = h->lnT_cap;
    mcts_status st = ensure(h, &p, &cap, bytes);
    if (st) return st;
    h->d_lnT = (double*)p;
    h->lnT_cap = cap;
  }
  const uint32_t n = Kalloc + 1;
  ln_table_kernel<<<(n + 255) / 256, 256, 0, s>>>(h->d_lnT, unit, Kalloc);
  CK(h, cudaGetLastError());
  h->lnT_unit = unit;
  h->lnT_K = Kalloc;
  return MCTS_OK;
}

// Carve a TreePool for n_trees * slot_cap slots out of one allocation.
mcts_status ensure_pool(mcts_handle* h, uint32_t n_trees, uint32_t slot_cap, TreePool* T) {
  const size_t slots = (size_t)n_trees * slot_cap;
  const size_t per = 3 * sizeof(u64) + 6 * sizeof(u32);
  const size_t bytes = slots * per + 8 * 256;
  if (bytes > (size_t)96 << 30)
    return fail(h, MCTS_E_OOM, "tree pool would exceed 96 GiB; lower iterations or max_nodes_per_tree");
  void* old = h->pool_mem;
  mcts_status st = ensure(h, &h->pool_mem, &h->pool_bytes, bytes);
  if (st) return st;
  if (h->pool_mem != old) h->tree_clean_cap = 0;
  char* p = (char*)h->pool_mem;
  auto take = [&](size_t b) { char* q = p; p += (b + 255) & ~(size_t)255; return q; };
  T->own = (u64*)take(slots * sizeof(u64));
  T->opp = (u64*)take(slots * sizeof(u64));
  T->legal = (u64*)take(slots * sizeof(u64));
  T->k = (u32*)take(slots * sizeof(u32));
  T->w = (u32*)take(slots * sizeof(u32));
  T->d = (u32*)take(slots * sizeof(u32));
  T->first = (u32*)take(slots * sizeof(u32));
  T->meta = (u32*)take(slots * sizeof(u32));
  T->vl = (u32*)take(slots * sizeof(u32));
  T->slot_cap = slot_cap;
  return MCTS_OK;
}

mcts_status check_device(mcts_handle* h) {
  cudaError_t e = cudaSetDevice(h->device);
  if (e != cudaSuccess) return fail(h, MCTS_E_NO_DEVICE, std::string("cudaSetDevice: ") + cudaGetErrorString(e));
  return MCTS_OK;
}

// Time-mode default node pool per tree (params.max_nodes_per_tree == 0): an
// upper bound on the iterations a tree runs in the budget (per tree for
// MCTS_BLOCK / MCTS_LEAF, for the whole shared tree with MCTS_TREE) times ~10
// slots reserved per expanded node, rounded up to a power of two, capped so the
// pool stays within 60% of the HBM that is free (plus the pool already held).
uint32_t auto_slot_cap(mcts_handle* h, double time_ms, uint32_t n_trees, bool shared) {
  size_t free_b = 0, total_b = 0;
  if (cudaMemGetInfo(&free_b, &total_b) != cudaSuccess) free_b = (size_t)8 << 30;
  // measured at 500 ms: ~15k/ms for the shared tree from the opening, up to ~3x
  // that late in a game (short playouts; r2h self-play filled 85% of 2^27 and
  // refused 319 expansions); ~66/ms per block tree, a few hundred late
  const double per_ms = shared ? 50000.0 : 100.0;
  double want = time_ms * per_ms * 10.0;
  const double hi = shared ? (double)(1u << 28) : (double)(1u << 24);
  if (want < 65536.0) want = 65536.0;
  if (want > hi) want = hi;
  uint64_t cap = 1;
  while ((double)cap < want) cap <<= 1;
  const uint64_t per_slot = 3 * sizeof(u64) + 6 * sizeof(u32);
  const uint64_t mem_cap = (uint64_t)((double)(free_b + h->pool_bytes) * 0.6) / ((uint64_t)n_trees * per_slot);
  if (cap > mem_cap) cap = mem_cap;
  if (cap < 64) cap = 64;
  return (uint32_t)cap;
}

// CTAs of a search kernel that can be resident at once (SMs x occupancy).
mcts_status resident_ctas(mcts_handle* h, const void* kfn, uint32_t threads, long long* out) {
  int per_sm = 0, n_sm = 0;
  CK(h, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, (int)threads, 0));
  CK(h, cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, h->device));
  *out = (long long)per_sm * n_sm;
  return MCTS_OK;
}

const void* block_kernel_fn(uint32_t threads) {
  if (threads <= 128) return (const void*)block_search_kernel<128, 8>;
  if (threads <= 256) return (const void*)block_search_kernel<256, 4>;
  if (threads <= 512) return (const void*)block_search_kernel<512, 2>;
  return (const void*)block_search_kernel<1024, 1>;
}

const void* tree_kernel_fn(uint32_t threads) {
  if (threads <= 128) return (const void*)tree_search_kernel<128, 8>;
  if (threads <= 256) return (const void*)tree_search_kernel<256, 4>;
  if (threads <= 512) return (const void*)tree_search_kernel<512, 2>;
  return (const void*)tree_search_kernel<1024, 1>;
}

template <int MAXT, int MINB>
mcts_status launch_block(mcts_handle* h, uint32_t n_trees, uint32_t threads, const TreePool& T,
                         const SearchArgs& a, cudaStream_t s) {
  block_search_kernel<MAXT, MINB><<<n_trees, threads, 0, s>>>(T, a);
  CK(h, cudaGetLastError());
  return MCTS_OK;
}

template <int MAXT, int MINB>
mcts_status launch_tree(mcts_handle* h, uint32_t workers, uint32_t threads, const TreePool& T,
                        const SearchArgs& a, cudaStream_t s) {
  tree_search_kernel<MAXT, MINB><<<workers, threads, 0, s>>>(T, a, h->d_treesync);
  CK(h, cudaGetLastError());
  return MCTS_OK;
}

// MCTS_TREE (tree_parallel.cuh): one shared tree, `workers` CTAs of `unit`
// threads. Pool fields are cleared (meta = 0 marks unpublished), the root is
// created by a one-thread kernel, then the search, the root merge and (with
// MCTS_FLAG_CHECK_TREE) the invariant check, all in stream order.
mcts_status tree_search_impl(mcts_handle* h, const mcts_position* rp, uint32_t workers, uint32_t unit,
                             uint32_t slot_cap, SearchArgs a, cudaStream_t s) {
  TreePool T;
  mcts_status st = ensure_pool(h, 1, slot_cap, &T);
  if (st) return st;
  // cleared fields: a read racing a child's creation sees meta = 0 (skipped)
  // or k = vl = w = 0 and first = kNoChild (tree_select_expand). A new pool
  // carving is cleared whole; after that only the slots the previous search
  // used (tree_clear_kernel reads its allocator).
  if (h->tree_clean_cap != slot_cap) {
    CK(h, cudaMemsetAsync(T.meta, 0, (size_t)slot_cap * sizeof(u32), s));
    CK(h, cudaMemsetAsync(T.k, 0, (size_t)slot_cap * sizeof(u32), s));
    CK(h, cudaMemsetAsync(T.w, 0, (size_t)slot_cap * sizeof(u32), s));
    CK(h, cudaMemsetAsync(T.vl, 0, (size_t)slot_cap * sizeof(u32), s));
    CK(h, cudaMemsetAsync(T.first, 0xFF, (size_t)slot_cap * sizeof(u32), s));
    h->tree_clean_cap = slot_cap;
  } else {
    tree_clear_kernel<<<4 * 148, 256, 0, s>>>(T, h->d_treesync);
    CK(h, cudaGetLastError());
  }
  DevPosition root;
  memcpy(&root, rp, sizeof(DevPosition));
  tree_root_kernel<<<1, 1, 0, s>>>(T, h->d_treesync, root);
  CK(h, cudaGetLastError());
  if (a.budget_ns) {
    stamp_kernel<<<1, 1, 0, s>>>(h->d_t0);
    CK(h, cudaGetLastError());
  }
  if (unit <= 128) st = launch_tree<128, 8>(h, workers, unit, T, a, s);
  else if (unit <= 256) st = launch_tree<256, 4>(h, workers, unit, T, a, s);
  else if (unit <= 512) st = launch_tree<512, 2>(h, workers, unit, T, a, s);
  else st = launch_tree<1024, 1>(h, workers, unit, T, a, s);
  if (st) return st;
  tree_merge_kernel<<<1, 32, 0, s>>>(T, h->d_treesync, unit, a.stats);
  CK(h, cudaGetLastError());
  if (h->params.flags & MCTS_FLAG_CHECK_TREE) {
    tree_check_kernel<<<592, 256, 0, s>>>(T, h->d_treesync, unit, slot_cap, h->d_error);
    CK(h, cudaGetLastError());
    tree_check_total_kernel<<<1, 1, 0, s>>>(h->d_treesync, a.stats, h->d_error);
    CK(h, cudaGetLastError());
  }
  return MCTS_OK;
}

// The search body shared by mcts_search / mcts_search_async. Writes the
// MCTS_STATS_LEN sums to d_stats on stream s.
mcts_status search_impl(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                        uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                        uint32_t tree_id_base, long long* d_stats, cudaStream_t s) {
  const mcts_position* rp = root ? root : (h->has_position ? &h->position : nullptr);
  if (!rp) return fail(h, MCTS_E_INVALID_ARGUMENT, "no root position (root == NULL and none given at create)");
  if (!position_ok(*rp)) return fail(h, MCTS_E_INVALID_POSITION, "root: black & white overlap or bad to_move");
  const bool by_iter = budget.iterations != 0;
  const bool by_time = budget.time_ms != 0.0;
  if (by_iter == by_time) return fail(h, MCTS_E_INVALID_ARGUMENT, "budget: exactly one of iterations / time_ms must be non-zero");
  if (by_time && !(budget.time_ms > 0.0 && budget.time_ms < 3.6e6))
    return fail(h, MCTS_E_INVALID_ARGUMENT, "budget.time_ms must be in (0, 3.6e6)");
  if (n_trees == 0) return fail(h, MCTS_E_INVALID_ARGUMENT, "n_trees == 0");
  if (!d_stats) return fail(h, MCTS_E_INVALID_ARGUMENT, "d_stats == NULL");
  const bool leaf = h->params.scheme == MCTS_LEAF;
  const bool tree = h->params.scheme == MCTS_TREE;
  if (leaf) {
    if (n_trees != 1) return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_LEAF: n_trees must be 1");
    if (threads_per_tree == 0 || threads_per_tree % 128 || threads_per_tree > 65536)
      return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_LEAF: threads_per_tree must be a multiple of 128 in [128, 65536]");
  } else {
    if (threads_per_tree == 0 || threads_per_tree % 32 || threads_per_tree > 1024)
      return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_BLOCK / MCTS_TREE: threads_per_tree must be a multiple of 32 in [32, 1024] (PAPER.md L310-L311)");
  }
  const uint64_t unit = threads_per_tree;
  const uint64_t kmax_counts = 0xFFFFFFFFull / unit;  // node counters are u32
  uint64_t max_it;
  uint32_t slot_cap;
  if (tree) {
    // one shared tree: iterations are the total over all workers; the ln
    // table also covers the workers' virtual visits (k + vl <= iterations + W)
    if (n_trees > 65536) return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_TREE: n_trees (workers) must be <= 65536");
    const uint64_t cap_it = kmax_counts < (1u << 24) ? kmax_counts : (1u << 24);
    if (by_iter) {
      if (budget.iterations > cap_it)
        return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_TREE: iterations * threads_per_tree must be < 2^32 and iterations <= 2^24");
      max_it = budget.iterations;
      // one node per iteration, each reserving <= 60 child slots: never full
      const uint64_t need = 61 + max_it * 60;
      slot_cap = (uint32_t)(need > 0x7FFFFFFFull ? 0x7FFFFFFFull : need);
    } else {
      max_it = cap_it;
      mcts_status st = check_device(h);
      if (st) return st;
      slot_cap = h->params.max_nodes_per_tree ? h->params.max_nodes_per_tree
                                              : auto_slot_cap(h, budget.time_ms, 1, true);
      if (slot_cap < 64) slot_cap = 64;
      // workers that cannot be resident would only start after the deadline
      long long res = 0;
      st = resident_ctas(h, tree_kernel_fn(threads_per_tree), threads_per_tree, &res);
      if (st) return st;
      if ((long long)n_trees > res)
        return fail(h, MCTS_E_INVALID_ARGUMENT, "time mode: n_trees (workers) exceeds the co-resident CTAs (" +
                                                    std::to_string(res) + ") for this threads_per_tree");
    }
    mcts_status st = check_device(h);
    if (st) return st;
    st = ensure_lnT(h, (uint32_t)unit, (uint32_t)(max_it + n_trees + 1), s);
    if (st) return st;
    CK(h, cudaMemsetAsync(d_stats, 0, MCTS_STATS_LEN * sizeof(long long), s));
    CK(h, cudaMemsetAsync(h->d_error, 0, sizeof(int), s));
    SearchArgs a;
    memcpy(&a.root, rp, sizeof(DevPosition));
    a.key = key_of(seed);
    a.C = h->params.c_uct;
    a.lnT = h->d_lnT;
    a.stats = d_stats;
    a.t0 = h->d_t0;
    a.budget_ns = by_time ? (u64)llround(budget.time_ms * 1e6) : 0ULL;
    if (by_time && a.budget_ns == 0) a.budget_ns = 1;
    a.max_iterations = (u32)max_it;
    a.tree_id_base = tree_id_base;
    a.unit = (u32)unit;
    a.error = h->d_error;
    a.rays = h->d_rays;
    return tree_search_impl(h, rp, n_trees, (uint32_t)unit, slot_cap, a, s);
  }
  if (by_iter) {
    if (budget.iterations > kmax_counts || budget.iterations > (1u << 24))
      return fail(h, MCTS_E_INVALID_ARGUMENT, "iterations * threads_per_tree must be < 2^32 and iterations <= 2^24");
    max_it = budget.iterations;
    // Each expanded interior node reserves <= 60 child slots; at most one node
    // is expanded per iteration, so the pool never fills (oracle capacity =
    // iterations + 1 is never reached either).
    const uint64_t need = 1 + max_it * 60;
    slot_cap = (uint32_t)(need > 0xFFFFFFF0ull ? 0xFFFFFFF0ull : need);
  } else {
    max_it = kmax_counts < (1u << 20) ? kmax_counts : (1u << 20);
    mcts_status st = check_device(h);
    if (st) return st;
    slot_cap = h->params.max_nodes_per_tree ? h->params.max_nodes_per_tree
                                            : auto_slot_cap(h, budget.time_ms, n_trees, false);
    if (slot_cap < 64) slot_cap = 64;
    if (!leaf) {  // trees that cannot be resident would only start after the deadline
      long long res = 0;
      st = resident_ctas(h, block_kernel_fn(threads_per_tree), threads_per_tree, &res);
      if (st) return st;
      if ((long long)n_trees > res)
        return fail(h, MCTS_E_INVALID_ARGUMENT, "time mode: n_trees exceeds the co-resident CTAs (" +
                                                    std::to_string(res) + ") for this threads_per_tree");
    }
  }

  mcts_status st = check_device(h);
  if (st) return st;
  TreePool T;
  st = ensure_pool(h, n_trees, slot_cap, &T);
  if (st) return st;
  st = ensure_lnT(h, (uint32_t)unit, (uint32_t)max_it, s);
  if (st) return st;
  CK(h, cudaMemsetAsync(d_stats, 0, MCTS_STATS_LEN * sizeof(long long), s));
  CK(h, cudaMemsetAsync(h->d_error, 0, sizeof(int), s));

  SearchArgs a;
  memcpy(&a.root, rp, sizeof(DevPosition));
  a.key = key_of(seed);
  a.C = h->params.c_uct;
  a.lnT = h->d_lnT;
  a.stats = d_stats;
  a.t0 = h->d_t0;
  a.budget_ns = by_time ? (u64)llround(budget.time_ms * 1e6) : 0ULL;
  if (by_time && a.budget_ns == 0) a.budget_ns = 1;
  a.max_iterations = (u32)max_it;
  a.tree_id_base = tree_id_base;
  a.unit = (u32)unit;
  a.error = h->d_error;
  a.rays = h->d_rays;
  if (by_time) {
    stamp_kernel<<<1, 1, 0, s>>>(h->d_t0);
    CK(h, cudaGetLastError());
  }

  if (!leaf) {
    if (threads_per_tree <= 128) return launch_block<128, 8>(h, n_trees, threads_per_tree, T, a, s);
    if (threads_per_tree <= 256) return launch_block<256, 4>(h, n_trees, threads_per_tree, T, a, s);
    if (threads_per_tree <= 512) return launch_block<512, 2>(h, n_trees, threads_per_tree, T, a, s);
    return launch_block<1024, 1>(h, n_trees, threads_per_tree, T, a, s);
  }
  // leaf parallelism: one cooperative grid of unit/128 co-resident CTAs
  const uint32_t G = threads_per_tree / 128;
  int per_sm = 0, n_sm = 0;
  const void* kfn = (const void*)leaf_search_kernel;
  CK(h, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kfn, 128, 0));
  CK(h, cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, h->device));
  if ((long long)per_sm * n_sm < (long long)G)
    return fail(h, MCTS_E_INVALID_ARGUMENT, "MCTS_LEAF: batch does not fit co-resident on the device");
  CK(h, cudaMemsetAsync(h->d_leafsync, 0, sizeof(LeafSync), s));
  LeafSync* S = h->d_leafsync;
  void* args[] = {(void*)&T, (void*)&a, (void*)&S};
  CK(h, cudaLaunchCooperativeKernel(kfn, dim3(G), dim3(128), args, 0, s));
  return MCTS_OK;
}

// The stats vector (include/mcts.h MCTS_STATS_LEN) as a mcts_root_stats.
void fill_root_stats(const long long* hs, mcts_root_stats* out) {
  for (int i = 0; i < 65; ++i) {
    out->visits[i] = (uint64_t)hs[i];
    out->wins[i] = (uint64_t)hs[65 + i];
    out->draws[i] = (uint64_t)hs[130 + i];
  }
  out->root_visits = (uint64_t)hs[195];
  out->iterations_done = (uint64_t)hs[196];
  out->plies = (uint64_t)hs[197];
  out->depth_sum = (uint64_t)hs[198];
  out->refused_expansions = (uint64_t)hs[199];
  out->slots_used = (uint64_t)hs[200];
  out->slot_capacity = (uint64_t)hs[201];
  out->best_move = mcts_best_move((const int64_t*)hs);
  out->reserved = 0;
}

// Host ln table lnT[k] = RN(ln k) for k <= K (unit 1) for the host-side trees,
// generated by the device ln kernel (the host has no correctly rounded ln).
mcts_status ensure_host_lnT1(mcts_handle* h, uint64_t K) {
  if (h->host_lnT1.size() >= K + 1) return MCTS_OK;
  double* d = nullptr;
  const size_t n = (size_t)K + 1;
  CK(h, cudaMalloc(&d, n * sizeof(double)));
  ln_table_kernel<<<(unsigned)((n + 255) / 256), 256, 0, h->stream>>>(d, 1u, (u32)K);
  std::vector<double> tmp(n);
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaMemcpyAsync(tmp.data(), d, n * sizeof(double), cudaMemcpyDeviceToHost, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  cudaFree(d);
  if (e != cudaSuccess) return cuda_fail(h, e, "host ln table");
  h->host_lnT1.swap(tmp);
  return MCTS_OK;
}

// The GPU side of mcts_search_hosted (hosted.h Gpu): one async step on the
// handle's stream — leaves H2D, the playouts kernel (c1 = step), W/D/L D2H.
struct HostedGpu {
  mcts_handle* h;
  uint64_t seed;
  uint32_t unit;
  mcts_position* d_leaves;
  mcts_wdl* d_wdl;
  unsigned long long* d_plies;
  cudaError_t err;
};

int hosted_submit(void* ctx, uint32_t first, uint32_t n, uint32_t step, int slot) {
  HostedGpu* g = (HostedGpu*)ctx;
  mcts_handle* h = g->h;
  // one stream per half: a half's kernel can start while the other half's is
  // still running (each fills part of the SMs; together the whole GPU)
  cudaStream_t s = slot == 0 ? h->stream : h->stream2;
  cudaError_t e = cudaMemcpyAsync(g->d_leaves + first, h->h_pin_leaves + first, (size_t)n * sizeof(mcts_position),
                                  cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && mcts_playouts_ex_async(h, g->d_leaves + first, n, g->unit, g->seed, first, step,
                                                 g->d_wdl + first, (uint64_t*)g->d_plies, s))
    e = cudaErrorLaunchFailure;
  if (e == cudaSuccess)
    e = cudaMemcpyAsync(h->h_pin_wdl + first, g->d_wdl + first, (size_t)n * sizeof(mcts_wdl),
                        cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaEventRecord(h->step_event[slot], s);
  g->err = e;
  return e == cudaSuccess ? 0 : -1;
}

int hosted_done(void* ctx, int slot) {
  HostedGpu* g = (HostedGpu*)ctx;
  const cudaError_t e = cudaEventQuery(g->h->step_event[slot]);
  if (e == cudaSuccess) return 1;
  if (e == cudaErrorNotReady) return 0;
  g->err = e;
  return -1;
}

int hosted_wait(void* ctx, int slot) {
  HostedGpu* g = (HostedGpu*)ctx;
  const cudaError_t e = cudaEventSynchronize(g->h->step_event[slot]);
  if (e != cudaSuccess) { g->err = e; return -1; }
  return 0;
}

}  // namespace

extern "C" {

const char* mcts_version(void) { return "mcts-b200 0.1 (sm_100a)"; }

const char* mcts_status_string(mcts_status st) {
  switch (st) {
    case MCTS_OK: return "MCTS_OK";
    case MCTS_E_INVALID_ARGUMENT: return "MCTS_E_INVALID_ARGUMENT";
    case MCTS_E_INVALID_POSITION: return "MCTS_E_INVALID_POSITION";
    case MCTS_E_CUDA: return "MCTS_E_CUDA";
    case MCTS_E_OOM: return "MCTS_E_OOM";
    case MCTS_E_NO_DEVICE: return "MCTS_E_NO_DEVICE";
    default: return "MCTS_E_UNKNOWN";
  }
}

const char* mcts_last_error(const mcts_handle* h) {
  return h ? h->last_error.c_str() : g_create_error.c_str();
}

mcts_status mcts_create(const mcts_position* position, const mcts_params* params, mcts_handle** out) {
  if (!out || !params) return fail(nullptr, MCTS_E_INVALID_ARGUMENT, "out / params is NULL");
  *out = nullptr;
  if (params->scheme != MCTS_BLOCK && params->scheme != MCTS_LEAF && params->scheme != MCTS_TREE)
    return fail(nullptr, MCTS_E_INVALID_ARGUMENT, "params->scheme must be MCTS_BLOCK, MCTS_LEAF or MCTS_TREE");
  if (params->flags & ~(uint32_t)MCTS_FLAG_CHECK_TREE)
    return fail(nullptr, MCTS_E_INVALID_ARGUMENT, "params->flags: unknown bits");
  if (!std::isfinite(params->c_uct) || params->c_uct < 0.0)
    return fail(nullptr, MCTS_E_INVALID_ARGUMENT, "params->c_uct must be finite and >= 0");
  if (position && !position_ok(*position))
    return fail(nullptr, MCTS_E_INVALID_POSITION, "position: black & white overlap or bad to_move");
  int ndev = 0;
  cudaGetLastError();  // a stale error of an earlier, unrelated runtime call is not ours
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0)
    return fail(nullptr, MCTS_E_NO_DEVICE, std::string("no CUDA device: ") + cudaGetErrorString(e));
  if (params->device < 0 || params->device >= ndev)
    return fail(nullptr, MCTS_E_NO_DEVICE, "params->device out of range");
  cudaDeviceProp prop;
  e = cudaGetDeviceProperties(&prop, params->device);
  if (e != cudaSuccess) return fail(nullptr, MCTS_E_NO_DEVICE, cudaGetErrorString(e));
  if (prop.major != 10)
    return fail(nullptr, MCTS_E_NO_DEVICE, "device is not compute capability 10.x (built for sm_100a only)");
  mcts_handle* h = new mcts_handle();
  h->device = params->device;
  h->params = *params;
  if (position) { h->position = *position; h->has_position = true; }
  e = cudaSetDevice(h->device);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaMalloc(&h->d_stats, MCTS_STATS_LEN * sizeof(long long));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_t0, sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_error, sizeof(int));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_plies, sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_leafsync, sizeof(LeafSync));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_treesync, sizeof(TreeSync));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_rays, kRayTable * sizeof(u64));
  if (e == cudaSuccess) e = cudaMalloc(&h->d_work, kWorkSlots * sizeof(u32));
  if (e == cudaSuccess) e = cudaHostAlloc(&h->h_pin_plies, sizeof(unsigned long long), cudaHostAllocDefault);
  if (e == cudaSuccess) {
    rays_init_kernel<<<1, 256, 0, h->stream>>>(h->d_rays);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess) {
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, playouts_kernel, kPlayoutThreads, 0);
    h->playout_ctas = per_sm * prop.multiProcessorCount;
  }
  if (e != cudaSuccess) {
    g_create_error = std::string("mcts_create: ") + cudaGetErrorString(e);
    mcts_destroy(h);
    return e == cudaErrorMemoryAllocation ? MCTS_E_OOM : MCTS_E_CUDA;
  }
  *out = h;
  return MCTS_OK;
}

void mcts_destroy(mcts_handle* h) {
  if (!h) return;
  cudaSetDevice(h->device);
  if (h->stream) cudaStreamSynchronize(h->stream);
  cudaFree(h->d_leaves);
  cudaFree(h->d_wdl);
  cudaFree(h->d_plies);
  cudaFree(h->pool_mem);
  cudaFree(h->d_lnT);
  cudaFree(h->d_stats);
  cudaFree(h->d_t0);
  cudaFree(h->d_error);
  cudaFree(h->d_leafsync);
  cudaFree(h->d_treesync);
  cudaFree(h->d_rays);
  cudaFree(h->d_work);
  for (int i = 0; i < MCTS_HOST_ASYNC_SLOTS; ++i) {
    cudaFree(h->d_async[i]);
    if (h->async_done[i]) cudaEventDestroy(h->async_done[i]);
  }
  if (h->h_pin_leaves) cudaFreeHost(h->h_pin_leaves);
  if (h->h_pin_wdl) cudaFreeHost(h->h_pin_wdl);
  if (h->h_pin_plies) cudaFreeHost(h->h_pin_plies);
  for (cudaEvent_t& ev : h->step_event)
    if (ev) cudaEventDestroy(ev);
  if (h->stream2) {
    cudaStreamSynchronize(h->stream2);
    cudaStreamDestroy(h->stream2);
  }
  if (h->stream) cudaStreamDestroy(h->stream);
  delete h;
}

namespace {

// The playout kernel on a zeroed output and a zeroed work counter (the
// callers own the memsets).
mcts_status launch_playouts(mcts_handle* h, const mcts_position* d_leaves, uint32_t n_leaves,
                            uint32_t n_per_leaf, uint64_t seed, uint32_t c0_base, uint32_t c1,
                            mcts_wdl* d_out, uint64_t* d_plies, u32* work, cudaStream_t s) {
  const uint64_t total = (uint64_t)n_leaves * n_per_leaf;
  const uint64_t need = (total + kPlayoutThreads - 1) / kPlayoutThreads;
  const unsigned blocks = (unsigned)(need < (uint64_t)h->playout_ctas ? need : (uint64_t)h->playout_ctas);
  playouts_kernel<<<blocks, kPlayoutThreads, 0, s>>>(
      (const DevPosition*)d_leaves, n_leaves, n_per_leaf, key_of(seed), c0_base, c1, (WdlOut*)d_out,
      (unsigned long long*)d_plies, h->d_rays, work);
  CK(h, cudaGetLastError());
  return MCTS_OK;
}

}  // namespace

mcts_status mcts_playouts_ex_async(mcts_handle* h, const mcts_position* d_leaves, uint32_t n_leaves,
                                   uint32_t n_per_leaf, uint64_t seed, uint32_t c0_base, uint32_t c1,
                                   mcts_wdl* d_out, uint64_t* d_plies, void* stream) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (n_leaves && (!d_leaves || !d_out)) return fail(h, MCTS_E_INVALID_ARGUMENT, "NULL leaves / out");
  mcts_status st = check_device(h);
  if (st) return st;
  cudaStream_t s = (cudaStream_t)stream;
  if (n_leaves == 0) return MCTS_OK;
  CK(h, cudaMemsetAsync(d_out, 0, (size_t)n_leaves * sizeof(mcts_wdl), s));
  const uint64_t total = (uint64_t)n_leaves * n_per_leaf;
  if (total == 0) return MCTS_OK;
  if ((total + 31) / 32 > 0xFFFFFFF0ull) return fail(h, MCTS_E_INVALID_ARGUMENT, "batch too large (>= 2^37 playouts)");
  // a fresh counter per launch, so launches on different streams do not share one
  u32* work = h->d_work + (h->work_slot++ % kWorkSlots);
  CK(h, cudaMemsetAsync(work, 0, sizeof(u32), s));
  return launch_playouts(h, d_leaves, n_leaves, n_per_leaf, seed, c0_base, c1, d_out, d_plies, work, s);
}

mcts_status mcts_playouts_async(mcts_handle* h, const mcts_position* d_leaves, uint32_t n_leaves,
                                uint32_t n_per_leaf, uint64_t seed, uint32_t leaf_id_base,
                                mcts_wdl* d_out, uint64_t* d_plies, void* stream) {
  return mcts_playouts_ex_async(h, d_leaves, n_leaves, n_per_leaf, seed, leaf_id_base, 0u, d_out, d_plies,
                                stream);
}

// Host buffers: five stream operations per call — one memset zeroes the work
// counter, the ply count and the W/D/L counts together (one region), the
// leaves go up, the kernel runs, the counts come down into the caller's
// buffer and the ply count into a pinned slot (a pageable 8-byte copy would be
// staged by the driver).
mcts_status mcts_playouts(mcts_handle* h, const mcts_position* leaf_batch, uint32_t n_leaves,
                          uint32_t n_per_leaf, uint64_t seed, mcts_wdl* out_counts, uint64_t* out_plies) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (out_plies) *out_plies = 0;
  if (n_leaves == 0) return MCTS_OK;
  if (!leaf_batch || !out_counts) return fail(h, MCTS_E_INVALID_ARGUMENT, "NULL leaf_batch / out_counts");
  for (uint32_t i = 0; i < n_leaves; ++i)
    if (!position_ok(leaf_batch[i]))
      return fail(h, MCTS_E_INVALID_POSITION, "leaf " + std::to_string(i) + ": black & white overlap or bad to_move");
  mcts_status st = check_device(h);
  if (st) return st;
  if (n_per_leaf == 0) {
    memset(out_counts, 0, (size_t)n_leaves * sizeof(mcts_wdl));
    return MCTS_OK;
  }
  if ((uint64_t)n_leaves * n_per_leaf / 32 > 0xFFFFFFF0ull)
    return fail(h, MCTS_E_INVALID_ARGUMENT, "batch too large (>= 2^37 playouts)");
  void* p = h->d_leaves;
  st = ensure(h, &p, &h->leaves_cap, (size_t)n_leaves * sizeof(DevPosition));
  if (st) return st;
  h->d_leaves = (DevPosition*)p;
  constexpr size_t kHead = 16;  // u32 work, u32 pad, u64 plies
  const size_t region = kHead + (size_t)n_leaves * sizeof(WdlOut);
  st = ensure(h, &h->d_wdl, &h->wdl_cap, region);
  if (st) return st;
  char* base = (char*)h->d_wdl;
  u32* work = (u32*)base;
  uint64_t* d_plies = (uint64_t*)(base + 8);
  mcts_wdl* d_out = (mcts_wdl*)(base + kHead);
  cudaStream_t s = h->stream;
  CK(h, cudaMemsetAsync(base, 0, region, s));
  CK(h, cudaMemcpyAsync(h->d_leaves, leaf_batch, (size_t)n_leaves * sizeof(DevPosition), cudaMemcpyHostToDevice, s));
  st = launch_playouts(h, (const mcts_position*)h->d_leaves, n_leaves, n_per_leaf, seed, 0u, 0u, d_out,
                       d_plies, work, s);
  if (st) return st;
  CK(h, cudaMemcpyAsync(out_counts, d_out, (size_t)n_leaves * sizeof(WdlOut), cudaMemcpyDeviceToHost, s));
  CK(h, cudaMemcpyAsync(h->h_pin_plies, d_plies, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  CK(h, cudaStreamSynchronize(s));
  if (out_plies) *out_plies = *h->h_pin_plies;
  return MCTS_OK;
}

mcts_status mcts_playouts_host_async(mcts_handle* h, const mcts_position* leaf_batch, uint32_t n_leaves,
                                     uint32_t n_per_leaf, uint64_t seed, mcts_wdl* out_counts,
                                     uint64_t* out_plies, void* stream) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (n_leaves && (!leaf_batch || !out_counts)) return fail(h, MCTS_E_INVALID_ARGUMENT, "NULL leaf_batch / out_counts");
  if ((uint64_t)n_leaves * n_per_leaf / 32 > 0xFFFFFFF0ull)
    return fail(h, MCTS_E_INVALID_ARGUMENT, "batch too large (>= 2^37 playouts)");
  mcts_status st = check_device(h);
  if (st) return st;
  cudaStream_t s = (cudaStream_t)stream;
  if (n_leaves == 0) {
    if (out_plies) *out_plies = 0;
    return MCTS_OK;
  }
  constexpr size_t kHead = 16;  // u32 work, u32 pad, u64 plies
  const size_t out_bytes = (size_t)n_leaves * sizeof(WdlOut);
  const size_t leaves_off = (kHead + out_bytes + 255) & ~(size_t)255;
  const size_t region = leaves_off + (size_t)n_leaves * sizeof(DevPosition);
  const uint32_t slot = h->async_next++ % MCTS_HOST_ASYNC_SLOTS;
  if (!h->async_done[slot]) CK(h, cudaEventCreateWithFlags(&h->async_done[slot], cudaEventDisableTiming));
  if (h->async_cap[slot] < region && h->d_async[slot]) {
    // the slot's previous call may still be in flight: wait before freeing it
    CK(h, cudaEventSynchronize(h->async_done[slot]));
  }
  // the slot's previous call (on any stream) must have copied its results out
  CK(h, cudaStreamWaitEvent(s, h->async_done[slot], 0));
  st = ensure(h, &h->d_async[slot], &h->async_cap[slot], region);
  if (st) return st;
  char* base = (char*)h->d_async[slot];
  u32* work = (u32*)base;
  uint64_t* d_plies = (uint64_t*)(base + 8);
  mcts_wdl* d_out = (mcts_wdl*)(base + kHead);
  mcts_position* d_leaves = (mcts_position*)(base + leaves_off);
  CK(h, cudaMemsetAsync(base, 0, kHead + out_bytes, s));
  CK(h, cudaMemcpyAsync(d_leaves, leaf_batch, (size_t)n_leaves * sizeof(DevPosition), cudaMemcpyHostToDevice, s));
  if (n_per_leaf) {
    st = launch_playouts(h, d_leaves, n_leaves, n_per_leaf, seed, 0u, 0u, d_out, d_plies, work, s);
    if (st) return st;
  }
  CK(h, cudaMemcpyAsync(out_counts, d_out, out_bytes, cudaMemcpyDeviceToHost, s));
  if (out_plies) CK(h, cudaMemcpyAsync(out_plies, d_plies, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  CK(h, cudaEventRecord(h->async_done[slot], s));
  return MCTS_OK;
}

mcts_status mcts_search_async(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                              uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                              uint32_t tree_id_base, int64_t* d_stats, void* stream) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  return search_impl(h, root, budget, n_trees, threads_per_tree, seed, tree_id_base,
                     (long long*)d_stats, (cudaStream_t)stream);
}

int32_t mcts_best_move(const int64_t* stats) {
  if (!stats) return -1;
  int32_t best = -1;
  int64_t bv = 0;
  for (int mv = 0; mv < 65; ++mv)
    if (stats[mv] > bv) { bv = stats[mv]; best = mv; }
  return best;
}

mcts_status mcts_search(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                        uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                        mcts_root_stats* out) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (!out) return fail(h, MCTS_E_INVALID_ARGUMENT, "out == NULL");
  mcts_status st = search_impl(h, root, budget, n_trees, threads_per_tree, seed, 0, h->d_stats, h->stream);
  if (st) return st;
  long long hs[MCTS_STATS_LEN];
  CK(h, cudaMemcpyAsync(hs, h->d_stats, sizeof(hs), cudaMemcpyDeviceToHost, h->stream));
  int herr = 0;
  CK(h, cudaMemcpyAsync(&herr, h->d_error, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
  CK(h, cudaStreamSynchronize(h->stream));
  if (herr == 2) return fail(h, MCTS_E_CUDA, "MCTS_TREE: tree invariant check failed (MCTS_FLAG_CHECK_TREE)");
  if (herr) return fail(h, MCTS_E_CUDA, "search kernel reported an internal error");
  fill_root_stats(hs, out);
  return MCTS_OK;
}

mcts_status mcts_search_hybrid(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                               uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                               uint32_t cpu_threads, mcts_root_stats* out, mcts_root_stats* out_cpu) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (!out) return fail(h, MCTS_E_INVALID_ARGUMENT, "out == NULL");
  if (h->params.scheme == MCTS_LEAF) return fail(h, MCTS_E_INVALID_ARGUMENT, "hybrid search needs MCTS_BLOCK or MCTS_TREE");
  if (cpu_threads == 0 || cpu_threads > 1024) return fail(h, MCTS_E_INVALID_ARGUMENT, "cpu_threads must be in [1, 1024]");
  const mcts_position* rp = root ? root : (h->has_position ? &h->position : nullptr);
  if (!rp) return fail(h, MCTS_E_INVALID_ARGUMENT, "no root position");
  if (!position_ok(*rp)) return fail(h, MCTS_E_INVALID_POSITION, "root: black & white overlap or bad to_move");
  const bool by_time = budget.time_ms != 0.0;
  const uint64_t host_k = by_time ? (1u << 20) : budget.iterations;
  if (!by_time && (host_k == 0 || host_k > (1u << 24)))
    return fail(h, MCTS_E_INVALID_ARGUMENT, "iterations must be in [1, 2^24]");
  mcts_status st = check_device(h);
  if (st) return st;
  st = ensure_host_lnT1(h, host_k);
  if (st) return st;
  // GPU trees (async), then the host trees in this thread's pool while the
  // kernel runs; host tree ids start at 0x40000000 so no stream is shared.
  st = search_impl(h, rp, budget, n_trees, threads_per_tree, seed, 0, h->d_stats, h->stream);
  if (st) return st;
  const int64_t start_ns = std::chrono::steady_clock::now().time_since_epoch().count();
  mcts_host::HostSearchArgs a;
  a.own = rp->to_move ? rp->white : rp->black;
  a.opp = rp->to_move ? rp->black : rp->white;
  a.seed = seed;
  a.C = h->params.c_uct;
  a.n_trees = cpu_threads;
  a.tree_id_base = 0x40000000u;
  a.iterations = host_k;
  a.deadline_ns = by_time ? start_ns + (int64_t)llround(budget.time_ms * 1e6) : 0;
  a.threads = cpu_threads;
  a.lnT = h->host_lnT1.data();
  long long cs[MCTS_STATS_LEN];
  mcts_host::search(a, (int64_t*)cs);
  long long hs[MCTS_STATS_LEN];
  int herr = 0;
  CK(h, cudaMemcpyAsync(hs, h->d_stats, sizeof(hs), cudaMemcpyDeviceToHost, h->stream));
  CK(h, cudaMemcpyAsync(&herr, h->d_error, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
  CK(h, cudaStreamSynchronize(h->stream));
  if (herr == 2) return fail(h, MCTS_E_CUDA, "MCTS_TREE: tree invariant check failed (MCTS_FLAG_CHECK_TREE)");
  if (herr) return fail(h, MCTS_E_CUDA, "search kernel reported an internal error");
  if (out_cpu) fill_root_stats(cs, out_cpu);
  for (int i = 0; i < MCTS_STATS_LEN; ++i) hs[i] += cs[i];  // root sum over all trees (L199-L202)
  fill_root_stats(hs, out);
  return MCTS_OK;
}

mcts_status mcts_search_hosted(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                               uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                               uint32_t cpu_iters, uint32_t cpu_threads, mcts_root_stats* out,
                               mcts_hosted_info* info) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (!out) return fail(h, MCTS_E_INVALID_ARGUMENT, "out == NULL");
  if (h->params.scheme != MCTS_BLOCK) return fail(h, MCTS_E_INVALID_ARGUMENT, "hosted search needs an MCTS_BLOCK handle");
  const mcts_position* rp = root ? root : (h->has_position ? &h->position : nullptr);
  if (!rp) return fail(h, MCTS_E_INVALID_ARGUMENT, "no root position");
  if (!position_ok(*rp)) return fail(h, MCTS_E_INVALID_POSITION, "root: black & white overlap or bad to_move");
  const bool by_iter = budget.iterations != 0, by_time = budget.time_ms != 0.0;
  if (by_iter == by_time) return fail(h, MCTS_E_INVALID_ARGUMENT, "budget: exactly one of iterations / time_ms must be non-zero");
  if (by_time && !(budget.time_ms > 0.0 && budget.time_ms < 3.6e6))
    return fail(h, MCTS_E_INVALID_ARGUMENT, "budget.time_ms must be in (0, 3.6e6)");
  if (n_trees == 0 || n_trees > (1u << 20)) return fail(h, MCTS_E_INVALID_ARGUMENT, "n_trees must be in [1, 2^20]");
  if (threads_per_tree == 0 || threads_per_tree % 32 || threads_per_tree > 1024)
    return fail(h, MCTS_E_INVALID_ARGUMENT, "threads_per_tree must be a multiple of 32 in [32, 1024]");
  if (cpu_threads == 0 || cpu_threads > 1024) return fail(h, MCTS_E_INVALID_ARGUMENT, "cpu_threads must be in [1, 1024]");
  uint64_t K;  // largest parent simulation count a selection can see
  if (by_iter) {
    const uint64_t per = (uint64_t)threads_per_tree + cpu_iters;
    if (budget.iterations >= (1ull << 26) || budget.iterations * per >= (1ull << 26))
      return fail(h, MCTS_E_INVALID_ARGUMENT, "iterations * (threads_per_tree + cpu_iters) must be < 2^26");
    K = budget.iterations * per + 2;
  } else {
    K = 1ull << 22;
  }
  mcts_status st = check_device(h);
  if (st) return st;
  st = ensure_host_lnT1(h, K);
  if (st) return st;
  if (h->pin_cap < n_trees) {
    if (h->h_pin_leaves) cudaFreeHost(h->h_pin_leaves);
    if (h->h_pin_wdl) cudaFreeHost(h->h_pin_wdl);
    h->h_pin_leaves = nullptr; h->h_pin_wdl = nullptr; h->pin_cap = 0;
    CK(h, cudaHostAlloc((void**)&h->h_pin_leaves, (size_t)n_trees * sizeof(mcts_position), cudaHostAllocDefault));
    CK(h, cudaHostAlloc((void**)&h->h_pin_wdl, (size_t)n_trees * sizeof(mcts_wdl), cudaHostAllocDefault));
    h->pin_cap = n_trees;
  }
  for (cudaEvent_t& ev : h->step_event)
    if (!ev) CK(h, cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  if (!h->stream2) CK(h, cudaStreamCreateWithFlags(&h->stream2, cudaStreamNonBlocking));
  void* p = h->d_leaves;
  st = ensure(h, &p, &h->leaves_cap, (size_t)n_trees * sizeof(DevPosition));
  if (st) return st;
  h->d_leaves = (DevPosition*)p;
  st = ensure(h, &h->d_wdl, &h->wdl_cap, (size_t)n_trees * sizeof(WdlOut));
  if (st) return st;
  CK(h, cudaMemsetAsync(h->d_plies, 0, sizeof(unsigned long long), h->stream));
  // the second half's stream starts behind the zeroed ply counter
  CK(h, cudaEventRecord(h->step_event[1], h->stream));
  CK(h, cudaStreamWaitEvent(h->stream2, h->step_event[1], 0));

  HostedGpu g{h, seed, threads_per_tree, (mcts_position*)h->d_leaves, (mcts_wdl*)h->d_wdl, h->d_plies, cudaSuccess};
  mcts_hosted::Gpu gpu{&g, hosted_submit, hosted_done, hosted_wait,
                       (mcts_hosted::LeafRec*)h->h_pin_leaves, (const mcts_hosted::WdlRec*)h->h_pin_wdl};
  mcts_hosted::Args a;
  a.own = rp->to_move ? rp->white : rp->black;
  a.opp = rp->to_move ? rp->black : rp->white;
  a.seed = seed;
  a.C = h->params.c_uct;
  a.n_trees = n_trees;
  a.tree_id_base = 0;
  a.unit = threads_per_tree;
  a.steps = by_iter ? budget.iterations : ~0ull;
  a.cpu_iters = cpu_iters;
  a.deadline_ns = by_time ? std::chrono::steady_clock::now().time_since_epoch().count() +
                                (int64_t)llround(budget.time_ms * 1e6)
                          : 0;
  a.threads = cpu_threads;
  a.lnT = h->host_lnT1.data();
  a.lnT_size = h->host_lnT1.size();
  long long hs[MCTS_STATS_LEN];
  mcts_hosted::Info hi;
  const int r = mcts_hosted::run(a, gpu, (int64_t*)hs, &hi);
  cudaStreamSynchronize(h->stream2);
  if (r < 0) {
    cudaStreamSynchronize(h->stream);
    return cuda_fail(h, g.err == cudaSuccess ? cudaErrorUnknown : g.err, "mcts_search_hosted: GPU step");
  }
  unsigned long long gpu_plies = 0;
  CK(h, cudaMemcpyAsync(&gpu_plies, h->d_plies, sizeof(gpu_plies), cudaMemcpyDeviceToHost, h->stream));
  CK(h, cudaStreamSynchronize(h->stream));
  hs[197] += (long long)gpu_plies;
  fill_root_stats(hs, out);
  if (info) {
    info->steps = hi.steps;
    info->cpu_iterations = hi.cpu_iterations;
    info->cpu_plies = hi.cpu_plies;
    info->cpu_depth_sum = hi.cpu_depth_sum;
    info->cpu_nodes = hi.cpu_nodes;
    info->gpu_nodes = hi.gpu_nodes;
    info->select_ms = hi.select_ms;
    info->gpu_ms = hi.gpu_ms;
    info->backprop_ms = hi.backprop_ms;
  }
  return MCTS_OK;
}

mcts_status mcts_perft(mcts_handle* h, const mcts_position* position, uint32_t depth,
                       uint32_t pass_is_ply, uint64_t* out) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (!position || !out) return fail(h, MCTS_E_INVALID_ARGUMENT, "position / out is NULL");
  if (!position_ok(*position)) return fail(h, MCTS_E_INVALID_POSITION, "position: black & white overlap or bad to_move");
  if (depth > 16) return fail(h, MCTS_E_INVALID_ARGUMENT, "depth must be <= 16");
  mcts_status st = check_device(h);
  if (st) return st;
  const u64 own = position->to_move ? position->white : position->black;
  const u64 opp = position->to_move ? position->black : position->white;
  const u32 split = 5;  // frontier at 5 plies, one depth-first search per node
  const u32 stop_at = depth > split ? depth - split : 0xFFFFFFFFu;
  const u32 cap = 1u << 20;
  PerftNode* d_nodes = nullptr;
  u32* d_count = nullptr;
  unsigned long long* d_leaves = nullptr;
  cudaError_t e = cudaMalloc(&d_nodes, (size_t)cap * sizeof(PerftNode));
  if (e == cudaSuccess) e = cudaMalloc(&d_count, sizeof(u32));
  if (e == cudaSuccess) e = cudaMalloc(&d_leaves, sizeof(unsigned long long));
  if (e == cudaSuccess) e = cudaMemsetAsync(d_count, 0, sizeof(u32), h->stream);
  if (e == cudaSuccess) e = cudaMemsetAsync(d_leaves, 0, sizeof(unsigned long long), h->stream);
  u32 n = 0;
  if (e == cudaSuccess) {
    perft_frontier_kernel<<<1, 128, 0, h->stream>>>(own, opp, depth, stop_at, pass_is_ply ? 1u : 0u,
                                                    h->d_rays, d_nodes, cap, d_count, d_leaves);
    e = cudaGetLastError();
  }
  if (e == cudaSuccess) e = cudaMemcpyAsync(&n, d_count, sizeof(u32), cudaMemcpyDeviceToHost, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  if (e == cudaSuccess && n > cap) {
    cudaFree(d_nodes); cudaFree(d_count); cudaFree(d_leaves);
    return fail(h, MCTS_E_OOM, "perft frontier exceeds 2^20 nodes");
  }
  if (e == cudaSuccess && n > 0) {
    perft_dfs_kernel<<<(n + 127) / 128, 128, 0, h->stream>>>(d_nodes, n, pass_is_ply ? 1u : 0u, h->d_rays, d_leaves);
    e = cudaGetLastError();
  }
  unsigned long long leaves = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&leaves, d_leaves, sizeof(leaves), cudaMemcpyDeviceToHost, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  cudaFree(d_nodes);
  cudaFree(d_count);
  cudaFree(d_leaves);
  if (e != cudaSuccess) return cuda_fail(h, e, "mcts_perft");
  *out = leaves;
  return MCTS_OK;
}

mcts_status mcts_gen_positions_async(mcts_handle* h, uint64_t seed, uint32_t n, uint32_t lmin,
                                     uint32_t lmax, mcts_position* d_out, void* stream) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (lmin > lmax || lmax > 50) return fail(h, MCTS_E_INVALID_ARGUMENT, "need lmin <= lmax <= 50");
  if (n && !d_out) return fail(h, MCTS_E_INVALID_ARGUMENT, "d_out == NULL");
  mcts_status st = check_device(h);
  if (st) return st;
  if (n == 0) return MCTS_OK;
  gen_positions_kernel<<<(n + 127) / 128, 128, 0, (cudaStream_t)stream>>>(key_of(seed), n, lmin, lmax,
                                                                         (DevPosition*)d_out);
  CK(h, cudaGetLastError());
  return MCTS_OK;
}

mcts_status mcts_ln_table(mcts_handle* h, uint32_t unit, uint32_t K, double* out) {
  if (!h) return MCTS_E_INVALID_ARGUMENT;
  if (!out || unit == 0) return fail(h, MCTS_E_INVALID_ARGUMENT, "out == NULL or unit == 0");
  if ((uint64_t)K * unit >= (1ull << 53)) return fail(h, MCTS_E_INVALID_ARGUMENT, "K * unit must be < 2^53");
  mcts_status st = check_device(h);
  if (st) return st;
  double* d = nullptr;
  CK(h, cudaMalloc(&d, ((size_t)K + 1) * sizeof(double)));
  ln_table_kernel<<<(K + 1 + 255) / 256, 256, 0, h->stream>>>(d, unit, K);
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaMemcpyAsync(out, d, ((size_t)K + 1) * sizeof(double), cudaMemcpyDeviceToHost, h->stream);
  if (e == cudaSuccess) e = cudaStreamSynchronize(h->stream);
  cudaFree(d);
  if (e != cudaSuccess) return cuda_fail(h, e, "mcts_ln_table");
  return MCTS_OK;
}

}  // extern "C"
