"""Multi-GPU partitioning.

Trees are independent: rank r owns global trees [r*n, (r+1)*n) (their Philox
c0 ids), so the merged result does not depend on the number of GPUs. The only
collective is one in-place allreduce(sum) of the MCTS_STATS_LEN int64 root
statistics per move decision. The playout-batch path shards by leaf range with
no collective at all (each rank owns its output slice).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from ._native import STATS_LEN, best_move


def tree_id_base(rank: int, n_trees_per_rank: int) -> int:
    return rank * n_trees_per_rank


def leaf_range(rank: int, world: int, n_leaves: int) -> tuple:
    """Contiguous leaf slice of rank r (sizes differ by at most one)."""
    q, r = divmod(n_leaves, world)
    start = rank * q + min(rank, r)
    return start, start + q + (1 if rank < r else 0)


def merge_root_stats(stats: torch.Tensor, group=None, force: bool = False) -> torch.Tensor:
    """The single cross-GPU exchange: in-place allreduce(sum) of root stats
    (skipped at world size 1 unless `force`, which tests use to run the
    collective's code path on one GPU)."""
    if dist.is_available() and dist.is_initialized() and (force or dist.get_world_size(group) > 1):
        dist.all_reduce(stats, op=dist.ReduceOp.SUM, group=group)
    return stats


def best_move_from(stats) -> int:
    """R8 through the library (mcts_best_move): argmax visits over moves 0..64,
    lowest index on ties, -1 if none."""
    s = stats.cpu().numpy() if isinstance(stats, torch.Tensor) else np.asarray(stats)
    return best_move(s)


def search(mcts, root, n_trees: int, threads_per_tree: int, seed: int, iterations: int = 0,
           time_ms: float = 0.0, group=None, stream=None, force_collective: bool = False) -> dict:
    """This rank's search (the handle's scheme) + the root-stats allreduce. For
    MCTS_TREE each rank grows one shared tree with Philox c0 = rank * n_trees
    (root parallelism across GPUs, tree parallelism inside one). Everything
    runs on `stream` (default: the current stream); the host waits for that
    stream before reading the merged stats."""
    rank = dist.get_rank(group) if dist.is_available() and dist.is_initialized() else 0
    s = stream if stream is not None else torch.cuda.current_stream()
    with torch.cuda.stream(s):
        stats = torch.zeros(STATS_LEN, dtype=torch.int64, device=f"cuda:{mcts.device}")
        mcts.search_async(root, iterations, time_ms, n_trees, threads_per_tree, seed,
                          tree_id_base(rank, n_trees), stats.data_ptr(), s)
        merge_root_stats(stats, group, force=force_collective)
    s.synchronize()
    host = stats.cpu().numpy()
    return dict(stats=host, best_move=best_move(host))
