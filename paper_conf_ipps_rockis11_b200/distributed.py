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

from ._native import STATS_LEN


def tree_id_base(rank: int, n_trees_per_rank: int) -> int:
    return rank * n_trees_per_rank


def leaf_range(rank: int, world: int, n_leaves: int) -> tuple:
    """Contiguous leaf slice of rank r (sizes differ by at most one)."""
    q, r = divmod(n_leaves, world)
    start = rank * q + min(rank, r)
    return start, start + q + (1 if rank < r else 0)


def merge_root_stats(stats: torch.Tensor, group=None) -> torch.Tensor:
    """The single cross-GPU exchange: in-place allreduce(sum) of root stats."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(stats, op=dist.ReduceOp.SUM, group=group)
    return stats


def best_move_from(stats) -> int:
    """argmax visits over moves 0..64, lowest index on ties, -1 if none (R8)."""
    s = np.asarray(stats if not isinstance(stats, torch.Tensor) else stats.cpu().numpy())
    v = s[:65]
    if v.max() <= 0:
        return -1
    return int(np.argmax(v))


def search(mcts, root, n_trees: int, threads_per_tree: int, seed: int, iterations: int = 0,
           time_ms: float = 0.0, group=None, stream=None) -> dict:
    """This rank's search (the handle's scheme) + the root-stats allreduce. For
    MCTS_TREE each rank grows one shared tree with Philox c0 = rank * n_trees
    (root parallelism across GPUs, tree parallelism inside one)."""
    rank = dist.get_rank(group) if dist.is_available() and dist.is_initialized() else 0
    stats = torch.zeros(STATS_LEN, dtype=torch.int64, device=f"cuda:{mcts.device}")
    s = stream if stream is not None else torch.cuda.current_stream()
    mcts.search_async(root, iterations, time_ms, n_trees, threads_per_tree, seed,
                      tree_id_base(rank, n_trees), stats.data_ptr(), s)
    with torch.cuda.stream(s):
        merge_root_stats(stats, group)
    host = stats.cpu().numpy()
    return dict(stats=host, best_move=best_move_from(host))
