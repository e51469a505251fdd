"""B200-native block-parallel Monte Carlo Tree Search for 8x8 Reversi.

Rocki & Suda, "Large-Scale Parallel Monte Carlo Tree Search on GPU" (IPDPSW
2011). The hot path (random playouts, device-resident block-parallel UCT,
leaf-parallel comparison, per-GPU root merge) runs in hand-written sm_100a
kernels behind the C ABI of include/mcts.h (libmcts.so, built in-tree); this
package is a thin ctypes binding plus torch plumbing (device memory, streams,
torch.distributed for the one cross-GPU allreduce).
"""
from ._native import (  # noqa: F401
    EXPORTS, MCTS_BLOCK, MCTS_FLAG_CHECK_TREE, MCTS_LEAF, MCTS_TREE, POSITION_DTYPE, STATS_LEN, Mcts, MctsError, best_move, load,
    version,
)
from .positions import OPENING, opening, position, own_opp  # noqa: F401
