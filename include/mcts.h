/*
 * mcts.h — C ABI of the B200 block-parallel Monte Carlo Tree Search library
 * (libmcts.so, sm_100a).
 *
 * Method: Rocki & Suda, "Large-Scale Parallel Monte Carlo Tree Search on GPU",
 * IPDPSW 2011. Citations below are PAPER.md line ranges.
 *   - random playouts: L149-L153 (§II) — random moves until neither player can
 *     move; success = a win at the end;
 *   - UCT iteration Selection / Expansion / Simulation / Backpropagation:
 *     L155-L202 (§II-A, Fig. 1), UCB formula L163-L169;
 *   - leaf parallelism: L231-L237 (§III-5, Fig. 2a);
 *   - block parallelism (one tree per thread block, threads = simulations per
 *     iteration): L294-L311 (§III-6, Fig. 2c, Fig. 3);
 *   - root statistics summed over trees: L199-L202; over GPUs: L474-L475.
 * Readings where the paper is silent or garbled (UCB1 form, draws, pick rule,
 * RNG streams, expansion order, pass child, ln table, move choice) are
 * DESIGN.md §3 R1..R10; results are bit-exact to the CPU oracle under them.
 *
 * Conventions
 *   - Square s = 8*row + col (row 0 = rank 1, col 0 = file a) is bit s.
 *   - Ownership: the caller owns every input/output buffer (host or device as
 *     each argument states). The handle owns its device scratch (tree pools,
 *     ln table, staging) and frees it in mcts_destroy.
 *   - A handle is not thread-safe; use one per host thread / rank. Playout
 *     launches on one handle may overlap on different streams (each launch
 *     takes its own scratch, up to 256 in flight); searches may not overlap
 *     another search of the same handle (they share its tree pool).
 *   - Errors: no exception crosses the ABI; every function returns an
 *     mcts_status (< 0 on error) and mcts_last_error() gives the text.
 *   - Streams are passed as `void*` holding a cudaStream_t (NULL = the legacy
 *     default stream). *_async calls enqueue work and return without a host
 *     synchronisation; their device outputs are valid once the stream is.
 *   - Compute never falls back to the CPU: without an sm_100 device every
 *     compute entry point returns MCTS_E_NO_DEVICE.
 */
#ifndef MCTS_B200_MCTS_H
#define MCTS_B200_MCTS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t mcts_status;
#define MCTS_OK 0
#define MCTS_E_INVALID_ARGUMENT (-1)
#define MCTS_E_INVALID_POSITION (-2)
#define MCTS_E_CUDA (-3)
#define MCTS_E_OOM (-4)
#define MCTS_E_NO_DEVICE (-5)

/* A Reversi position: disc masks and the side to move (0 black, 1 white).
 * Valid iff (black & white) == 0 and to_move in {0, 1}. 24 bytes. */
typedef struct {
  uint64_t black;
  uint64_t white;
  uint32_t to_move;
  uint32_t reserved; /* must be 0 */
} mcts_position;

/* Playout outcome counts for one leaf, from the perspective of the leaf's side
 * to move (success = win; draws counted separately, R2). */
typedef struct {
  uint32_t wins;
  uint32_t draws;
  uint32_t losses;
} mcts_wdl;

#define MCTS_BLOCK 0u /* block parallelism: one tree per CTA (L294-L311) */
#define MCTS_LEAF 1u  /* leaf parallelism: one tree, the whole batch per leaf (L231-L237) */
#define MCTS_TREE 2u  /* tree parallelism: every CTA on one shared tree with virtual loss
                         (Chaslot et al.) */

/* mcts_params.flags */
#define MCTS_FLAG_CHECK_TREE 1u /* MCTS_TREE: after each search, check the tree invariants on the
                                   device (vl = 0, k >= sum of children k (+1 below the root),
                                   sum of k - children k = iterations); a violation makes
                                   mcts_search return MCTS_E_CUDA */

typedef struct {
  double c_uct;                /* UCB exploration constant C (L169); finite, >= 0; R1 default 1.0 */
  uint32_t scheme;             /* MCTS_BLOCK, MCTS_LEAF or MCTS_TREE */
  uint32_t max_nodes_per_tree; /* time mode: node-slot pool per tree; 0 = sized from the
                                  time budget and free HBM (stats [199]-[201]
                                  report refusals and use) */
  int32_t device;              /* CUDA device ordinal */
  uint32_t flags;              /* 0 or MCTS_FLAG_CHECK_TREE; other bits: INVALID_ARGUMENT */
} mcts_params;

/* Exactly one of iterations / time_ms is non-zero. Iteration mode is
 * deterministic and bit-exact to the oracle; time mode (a %globaltimer
 * deadline per search) is not reproducible. */
typedef struct {
  uint64_t iterations; /* UCT iterations per tree (MCTS_TREE: in total over the workers) */
  double time_ms;      /* wall-clock budget of the search kernel */
} mcts_budget;

/* Device statistics vector written by mcts_search_async (int64, summed over
 * trees; sums again across GPUs with one allreduce, L199-L202, L474-L475):
 *   [0,65)    root-child visits n by move (0..63 squares, 64 = pass)
 *   [65,130)  root-child wins for the root's side to move
 *   [130,195) root-child draws
 *   [195]     root visits (= playouts simulated)
 *   [196]     UCT iterations (summed over trees)
 *   [197]     playout plies (non-pass moves simulated)
 *   [198]     sum over iterations of the simulated node's depth (edges
 *             from the root; mean tree depth = [198] / [196], the paper's
 *             "Depth" of Fig. 8)
 *   [199]     iterations whose expansion was refused because the tree's node
 *             pool was full (time mode only; "I add one node per iteration",
 *             L179-L182, cannot hold then: the selected node is simulated
 *             again, R12). 0 in iteration mode.
 *   [200]     node-pool slots used (summed over trees; a node reserves its
 *             whole child block at its first expansion)
 *   [201]     node-pool slot capacity (summed over trees)
 * [0,200) are bit-exact to the oracle in iteration mode; [200] and [201]
 * describe this library's pools (the oracle counts nodes, not slots). */
#define MCTS_STATS_LEN 202

typedef struct {
  uint64_t visits[65];
  uint64_t wins[65];
  uint64_t draws[65];
  uint64_t root_visits;
  uint64_t iterations_done;
  uint64_t plies;
  uint64_t depth_sum; /* [198]: sum over iterations of the simulated node's depth */
  uint64_t refused_expansions; /* [199]: expansions refused by a full node pool */
  uint64_t slots_used;         /* [200] */
  uint64_t slot_capacity;      /* [201] */
  int32_t best_move; /* argmax visits, lowest index on ties (R8); -1 if the root is terminal */
  int32_t reserved;
} mcts_root_stats;

typedef struct mcts_handle mcts_handle;

/* Create a handle bound to params->device. `position` (host, nullable) is the
 * default root for mcts_search. Errors: INVALID_ARGUMENT (null out/params,
 * bad scheme or c_uct), INVALID_POSITION, NO_DEVICE (not compute capability
 * 10.x), CUDA. */
mcts_status mcts_create(const mcts_position* position, const mcts_params* params,
                        mcts_handle** out);

/* Free the handle and its device memory. NULL is a no-op. */
void mcts_destroy(mcts_handle* h);

/* Batched random playouts: leaf i gets
 * n_per_leaf playouts with RNG streams (c0 = i, c1 = 0, c2 = j) and
 * out_counts[i] their W/D/L. Host buffers in and out (the call does the H2D
 * copy, one kernel, the D2H copy, and synchronises). n_leaves == 0 or
 * n_per_leaf == 0 is valid (all-zero output). Terminal leaves return their
 * result n_per_leaf times; a leaf whose side must pass starts with the pass.
 * Errors: INVALID_ARGUMENT (null pointers with n_leaves > 0), INVALID_POSITION
 * (any leaf), OOM, CUDA. out_plies (host, nullable) receives the plies played. */
mcts_status mcts_playouts(mcts_handle* h, const mcts_position* leaf_batch, uint32_t n_leaves,
                          uint32_t n_per_leaf, uint64_t seed, mcts_wdl* out_counts,
                          uint64_t* out_plies);

/* mcts_playouts with host buffers, asynchronous (a serving pipeline: step
 * i + 1's copies and launch are enqueued while step i runs). Enqueues on
 * `stream` the H2D copy of leaf_batch, the playouts, the D2H copy of the counts
 * into out_counts and of the ply count into *out_plies, and returns without
 * waiting; the results are valid once the stream has reached this point
 * (cudaStreamSynchronize / an event). leaf_batch, out_counts and out_plies
 * must be pinned host memory (cudaHostAlloc / torch pin_memory) and stay
 * untouched until then; out_plies may be NULL. Same results as mcts_playouts.
 * Device staging: a ring of MCTS_HOST_ASYNC_SLOTS slots per handle; a slot's
 * reuse waits (cudaStreamWaitEvent) for its previous call's copies, so calls
 * may use different streams. Leaves are not validated (as
 * mcts_playouts_async). Errors: INVALID_ARGUMENT, OOM, CUDA. */
#define MCTS_HOST_ASYNC_SLOTS 8
mcts_status mcts_playouts_host_async(mcts_handle* h, const mcts_position* leaf_batch, uint32_t n_leaves,
                                     uint32_t n_per_leaf, uint64_t seed, mcts_wdl* out_counts,
                                     uint64_t* out_plies, void* stream);

/* Device-pointer / stream variant. d_leaves (device, n_leaves), d_out (device,
 * n_leaves, overwritten), d_plies (device uint64, nullable, ACCUMULATED into).
 * Streams use c0 = leaf_id_base + i so a batch split across GPUs by leaf range
 * reproduces the single-GPU result. Leaves are not validated (garbage in,
 * garbage out; no memory hazard). */
mcts_status mcts_playouts_async(mcts_handle* h, const mcts_position* d_leaves, uint32_t n_leaves,
                                uint32_t n_per_leaf, uint64_t seed, uint32_t leaf_id_base,
                                mcts_wdl* d_out, uint64_t* d_plies, void* stream);

/* The same kernel with the full stream key: leaf i's playouts use (c0 =
 * c0_base + i, c1, c2 = j). mcts_playouts_async is c1 = 0. This is the
 * "GPU simulates only" half of the paper's CPU-managed trees (L302-L303):
 * c1 = the step, so a step's batch reproduces the block search's iteration. */
mcts_status mcts_playouts_ex_async(mcts_handle* h, const mcts_position* d_leaves, uint32_t n_leaves,
                                   uint32_t n_per_leaf, uint64_t seed, uint32_t c0_base, uint32_t c1,
                                   mcts_wdl* d_out, uint64_t* d_plies, void* stream);

/* UCT search with the handle's scheme:
 *   MCTS_BLOCK: n_trees independent trees, one per CTA of threads_per_tree
 *               threads (multiple of 32, 32..1024); threads_per_tree playouts
 *               per iteration per tree (L186-L195, L294-L311).
 *   MCTS_LEAF:  n_trees must be 1; threads_per_tree (multiple of 128, <= 65536)
 *               playouts from the same leaf per iteration (L231-L237).
 *   MCTS_TREE:  ONE tree shared by n_trees workers (CTAs of threads_per_tree
 *               threads, multiple of 32, <= 1024; n_trees <= 65536), virtual
 *               loss in selection, a CAS per expansion. The
 *               iteration budget is the total over the workers (<= 2^24);
 *               c1 = a global iteration ticket. With n_trees == 1 the result
 *               equals MCTS_BLOCK with one tree bit for bit; with more workers
 *               it depends on timing (tree invariants: MCTS_FLAG_CHECK_TREE).
 * Playout streams: c0 = tree id, c1 = iteration, c2 = thread. root (host,
 * nullable = the create-time position). out (host) receives the root stats
 * summed over trees and the best move. Synchronous.
 * Errors: INVALID_ARGUMENT (budget not exactly one of iterations/time_ms,
 * n_trees == 0, bad threads_per_tree, iterations*threads_per_tree >= 2^32),
 * INVALID_POSITION, OOM, CUDA. */
mcts_status mcts_search(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                        uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                        mcts_root_stats* out);

/* Stream variant for multi-GPU use: trees get ids tree_id_base + t (rank r
 * passes r * n_trees), and the MCTS_STATS_LEN int64 sums are written (not
 * accumulated) to d_stats (device) on `stream`, ready for one in-place
 * allreduce(sum). root is a host pointer (read before return). */
mcts_status mcts_search_async(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                              uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                              uint32_t tree_id_base, int64_t* d_stats, void* stream);

/* Hybrid CPU/GPU search (§III-A):
 * the block-parallel GPU search of mcts_search_async runs while cpu_threads
 * host threads grow one tree each from the same root with one simulation per
 * iteration (the paper's CPU MCTS, L185-L186; Philox streams c0 = 0x40000000 +
 * thread, c1 = iteration, c2 = 0); the root statistics of all GPU and host
 * trees are summed (L199-L202) into out, the host trees' share alone into
 * out_cpu (nullable). Iteration mode: every GPU tree and every host tree runs
 * budget.iterations iterations (deterministic; host trees = the oracle's UCT
 * with unit 1). Time mode: both sides stop at time_ms. MCTS_BLOCK or
 * MCTS_TREE handles (with MCTS_TREE the GPU part is the one shared tree of
 * n_trees workers); errors as mcts_search plus INVALID_ARGUMENT for a
 * MCTS_LEAF handle or cpu_threads outside [1, 1024]. Synchronous. */
mcts_status mcts_search_hybrid(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                               uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                               uint32_t cpu_threads, mcts_root_stats* out, mcts_root_stats* out_cpu);

/* mcts_search_hosted diagnostics: how the work split between CPU and GPU. */
typedef struct {
  uint64_t steps;          /* GPU steps (one playout kernel over every tree's leaf) */
  uint64_t cpu_iterations; /* UCT iterations the host threads ran on the same trees */
  uint64_t cpu_plies;      /* plies of their playouts */
  uint64_t cpu_depth_sum;  /* sum of their simulated nodes' depths */
  uint64_t cpu_nodes;      /* nodes added by CPU iterations */
  uint64_t gpu_nodes;      /* nodes added by the GPU steps' selections */
  double select_ms;        /* host time selecting the GPU leaves (the sequential part, L303-L310) */
  double gpu_ms;           /* host time while the kernel was in flight (CPU iterating) */
  double backprop_ms;      /* host time backpropagating the kernel's results */
} mcts_hosted_info;

/* Block parallelism with CPU-managed trees, the paper's own design ("The trees
 * are still controlled by the CPU threads, GPU simulates only", L302-L303),
 * and its hybrid CPU-GPU processing (§III-A, Fig. 4): per step the
 * host threads select one leaf per tree, ONE playout kernel simulates
 * threads_per_tree playouts from each (streams c0 = tree, c1 = step, c2 =
 * thread), and while it runs the host threads run UCT iterations with one host
 * playout each on the SAME trees (streams c0 = tree, c1 = 0x80000000 + the
 * tree's CPU iteration count, c2 = 0); then the kernel's results are
 * backpropagated. Selection is R1 with the parent's simulation count (GPU
 * steps add threads_per_tree, CPU iterations 1); a child whose GPU result is
 * pending (n = 0) is an unvisited arm, taken first (R18).
 *   iteration mode: budget.iterations GPU steps, exactly cpu_iters CPU
 *     iterations per tree per step: deterministic, bit-exact to the oracle;
 *     cpu_iters = 0 is the MCTS_BLOCK search bit for bit;
 *   time mode: steps until time_ms; cpu_iters > 0 lets the host iterate while
 *     each kernel runs (as many as fit; the caller's thread only drives the
 *     GPU, the other cpu_threads - 1 iterate), 0 = no CPU iterations.
 * MCTS_BLOCK handle; n_trees in [1, 2^20]; threads_per_tree a multiple of 32
 * in [32, 1024]; cpu_threads in [1, 1024] host threads (the caller's thread
 * included); iteration mode: iterations * (threads_per_tree + cpu_iters)
 * < 2^26. out (host): root stats summed over trees ([196] counts GPU steps
 * and CPU iterations; [200] nodes; [201] 0, the host pools are unbounded);
 * info (host, nullable). Synchronous; single GPU (tree ids 0..n_trees-1). */
mcts_status mcts_search_hosted(mcts_handle* h, const mcts_position* root, mcts_budget budget,
                               uint32_t n_trees, uint32_t threads_per_tree, uint64_t seed,
                               uint32_t cpu_iters, uint32_t cpu_threads, mcts_root_stats* out,
                               mcts_hosted_info* info);

/* Best move from a (merged) stats vector on the host: argmax of visits[0..64],
 * lowest index on ties, -1 if all zero (R8). */
int32_t mcts_best_move(const int64_t* stats);

/* Synthetic inputs: position p is the result of
 * L = lmin + floor(r0 * (lmax - lmin + 1) / 2^32) non-pass uniform random
 * plies from the opening, RNG stream (c0 = p, c1 = 0xFFFFFFFF, c2 = attempt);
 * games that end early or terminal results retry with attempt + 1.
 * d_out (device, n). Requires lmin <= lmax <= 50 (>= 10 empties, so the
 * retry loop ends quickly; attempts are capped at 2^16, result = opening). */
mcts_status mcts_gen_positions_async(mcts_handle* h, uint64_t seed, uint32_t n, uint32_t lmin,
                                     uint32_t lmax, mcts_position* d_out, void* stream);

/* Perft: number of leaves of the move tree of `position` at `depth` plies
 * (a game-over node before that counts 1; a pass counts as a ply iff
 * pass_is_ply), computed on the device with the playout kernels' move
 * generator and flips — pins them to the known counts (north_star: 4, 12, 56,
 * 244, 1396, 8200, 55092, 390216 from the opening). depth <= 16; *out (host).
 * Errors: INVALID_ARGUMENT, INVALID_POSITION, OOM (frontier > 2^20), CUDA. */
mcts_status mcts_perft(mcts_handle* h, const mcts_position* position, uint32_t depth,
                       uint32_t pass_is_ply, uint64_t* out);

/* The device ln table used by UCT selection (R9): out[k] = RN(ln(k * unit))
 * for k = 1..K, out[0] = 0. out is a host array of K + 1 doubles. */
mcts_status mcts_ln_table(mcts_handle* h, uint32_t unit, uint32_t K, double* out);

const char* mcts_status_string(mcts_status st);
const char* mcts_last_error(const mcts_handle* h);
const char* mcts_version(void);

#ifdef __cplusplus
}
#endif

#endif /* MCTS_B200_MCTS_H */
