"""GPU parity at the BASELINE sizes, in the launch shapes bench.py times, run
long enough to reach the method's decision logic:

* every search here runs more iterations than its root has legal moves, so
  after the root is fully expanded every further iteration SELECTS by UCB
   — asserted as depth_sum > iterations (stats[198] >
  stats[196]): an iteration that only expands a root child has depth 1;
* configs[1] (4096 x 256, the bench's exact batch) and the opening-phase batch
  are compared on ALL 4096 leaves;
* a constructed root with 34 legal moves exercises the second lane pass of the
  warp-cooperative UCB argmax (children 32.. of a node) in the block, leaf and
  one-worker shared-tree kernels.

Oracle: the CPU reference on all host cores (seconds per case).
"""
import numpy as np
import pytest
import torch

import paper_conf_ipps_rockis11_b200 as pkg
from paper_conf_ipps_rockis11_b200 import device as dev

pytestmark = pytest.mark.gpu

# a position (own = side to move = black) with 34 legal moves, found by a hill
# climb on oracle.legal; not reachable from the opening, which does not matter
# to UCT (the root is an input)
WIDE_OWN, WIDE_OPP = 0x6024350012F48100, 0x520202A4025A00


def _root_with_few_moves(orc, seed0, lmin, lmax, max_moves):
    for seed in range(seed0, seed0 + 500):
        r = orc.gen_positions(seed, 1, lmin, lmax)
        own, opp = pkg.own_opp(r)
        c = bin(orc.legal(own, opp)).count("1")
        if 2 <= c <= max_moves:
            return r, c
    raise AssertionError("no root found")


def _cmp(res, ostats, obest):
    assert res["stats"][:200].tolist() == ostats[:200].tolist()
    assert res["best_move"] == obest


def _selected(stats):
    """UCB selections happened: the mean simulated depth exceeds 1."""
    assert stats[198] > stats[196] > 0


@pytest.fixture(scope="module")
def block():
    m = pkg.Mcts(c_uct=1.0, scheme="block", device=0)
    yield m
    m.close()


@pytest.fixture(scope="module")
def leaf():
    m = pkg.Mcts(c_uct=1.0, scheme="leaf", device=0)
    yield m
    m.close()


# ---------------------------------------------------------------- playouts, every leaf
@pytest.mark.parametrize("lmin,lmax", [(20, 40), (0, 8)])
def test_playouts_config1_all_leaves(block, orc, lmin, lmax):
    """configs[1] (4096 mid-game positions x 256, seed 2) and the opening-phase
    batch, async with device buffers as bench.py launches it: every leaf."""
    n, per, seed = 4096, 256, 2
    d_leaves = dev.gen_positions(block, seed, n, lmin, lmax)
    d_out = dev.empty_wdl(n)
    d_plies = torch.zeros(1, dtype=torch.int64, device="cuda")
    block.playouts_async(d_leaves.data_ptr(), n, per, seed, 0, d_out.data_ptr(), d_plies.data_ptr(),
                         torch.cuda.current_stream())
    torch.cuda.synchronize()
    leaves = orc.gen_positions(seed, n, lmin, lmax)
    assert (dev.tensor_to_positions(d_leaves) == leaves).all()
    owdl, oplies = orc.playouts(leaves, per, seed=seed)
    assert (d_out.cpu().numpy() == owdl).all()
    assert int(d_plies.item()) == oplies


# ---------------------------------------------------------------- block parallelism
def test_search_config2_reaches_selection(block, orc):
    """configs[2]'s launch shape (1184 trees x 128 threads) for 24 iterations
    on a root with <= 12 moves: half the iterations select by UCB."""
    root, c = _root_with_few_moves(orc, 12, 20, 30, 12)
    res = block.search(root, iterations=24, n_trees=1184, threads_per_tree=128, seed=1000)
    ostats, obest, _ = orc.uct_search(root, 1184, 128, 24, 1000)
    _cmp(res, ostats, obest)
    _selected(res["stats"])
    assert res["iterations"] == 1184 * 24 and res["stats"][199] == 0


def test_search_4736_trees_of_32_reaches_selection(block, orc):
    """Fig. 5's largest block-32 shape (4736 trees x 32) for 20 iterations."""
    root, c = _root_with_few_moves(orc, 31, 30, 40, 10)
    res = block.search(root, iterations=20, n_trees=4736, threads_per_tree=32, seed=8)
    ostats, obest, _ = orc.uct_search(root, 4736, 32, 20, 8)
    _cmp(res, ostats, obest)
    _selected(res["stats"])


# ---------------------------------------------------------------- leaf parallelism
@pytest.mark.parametrize("threads,iters,seed", [(16384, 40, 4), (65536, 20, 9)])
def test_search_leaf_full_batch_reaches_selection(leaf, orc, threads, iters, seed):
    """configs[3] (1 tree x 16384 threads per leaf batch, 128 co-resident CTAs
    with a flag hand-off and a grid barrier) and the largest batch (65536) long enough that the
    multi-CTA select -> simulate -> backprop loop runs UCB selections."""
    root, c = _root_with_few_moves(orc, 15, 30, 40, 10)
    res = leaf.search(root, iterations=iters, n_trees=1, threads_per_tree=threads, seed=seed)
    ostats, obest, oplies = orc.uct_search(root, 1, threads, iters, seed)
    _cmp(res, ostats, obest)
    assert res["plies"] == oplies
    _selected(res["stats"])


# ---------------------------------------------------------------- > 32 children
def test_wide_root_has_more_than_32_moves(orc):
    assert bin(orc.legal(WIDE_OWN, WIDE_OPP)).count("1") == 34


@pytest.mark.parametrize("scheme,n_trees,threads,iters", [
    ("block", 3, 32, 120), ("block", 2, 256, 70), ("leaf", 1, 256, 80), ("tree", 1, 64, 120)])
def test_wide_root_second_lane_pass(orc, scheme, n_trees, threads, iters):
    """34 root children: lanes 0 and 1 of the selecting warp score children
    i and i + 32; the lowest-index tie rule must hold across the two passes."""
    root = orc.position(WIDE_OWN, WIDE_OPP, 0)
    m = pkg.Mcts(c_uct=1.0, scheme=scheme, device=0)
    res = m.search(root, iterations=iters, n_trees=n_trees, threads_per_tree=threads, seed=5)
    ostats, obest, _ = orc.uct_search(root, n_trees, threads, iters, 5)
    _cmp(res, ostats, obest)
    _selected(res["stats"])
    # children 32 and 33 (the highest-index legal squares) were visited after expansion
    legal = [s for s in range(64) if (orc.legal(WIDE_OWN, WIDE_OPP) >> s) & 1]
    assert res["stats"][legal[32]] > 0 and res["stats"][legal[33]] > 0
    m.close()
