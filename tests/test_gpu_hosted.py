"""mcts_search_hosted: the paper's block parallelism with CPU-managed trees and
its hybrid CPU-GPU processing (§III-A, Fig. 4;
DESIGN.md R18), through the C ABI, against the oracle (orc_hybrid_search).

* cpu_iters = 0: the host-managed trees with one playout kernel per step are
  the device block search bit for bit (same selections, same streams);
* cpu_iters > 0, iteration mode: bit-exact to the oracle's hybrid search
  (host threads add UCT iterations to the same trees while the kernel runs);
* time mode: the CPU's share of iterations and nodes is reported and the root
  identities hold.
"""
import numpy as np
import pytest
import torch

import paper_conf_ipps_rockis11_b200 as pkg
from paper_conf_ipps_rockis11_b200 import device as dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def block():
    m = pkg.Mcts(c_uct=1.0, scheme="block", device=0)
    yield m
    m.close()


def test_playouts_ex_stream_key(block, orc):
    """c1 reaches the playouts: leaf i, playout j uses (c0_base + i, c1, j)."""
    leaves = orc.gen_positions(3, 40, 20, 40)
    d = dev.positions_to_tensor(leaves)
    out = dev.empty_wdl(40)
    block.playouts_ex_async(d.data_ptr(), 40, 33, 9, 100, 7, out.data_ptr(), 0, None)
    torch.cuda.synchronize()
    got = out.cpu().numpy()
    for i in (0, 17, 39):
        w = dr = l = 0
        for j in range(33):
            r, _ = orc.playout(leaves[i:i + 1], 9, 100 + i, 7, j)
            w += r > 0; dr += r == 0; l += r < 0
        assert got[i].tolist() == [w, dr, l]


@pytest.mark.parametrize("n_trees,threads,steps,seed,C,lmin,lmax,cpu_threads", [
    (1, 64, 100, 1, 1.0, 0, 0, 1),       # configs[0] as CPU-managed trees
    (37, 32, 60, 4, 0.25, 20, 40, 5),
    (300, 128, 12, 6, 1.0, 10, 30, 16),
])
def test_hosted_without_cpu_equals_block_search(block, orc, n_trees, threads, steps, seed, C, lmin, lmax,
                                                cpu_threads):
    m = pkg.Mcts(c_uct=C, scheme="block", device=0)
    root = orc.gen_positions(seed, 1, lmin, lmax) if lmax else orc.opening()
    res = m.search_hosted(root, iterations=steps, n_trees=n_trees, threads_per_tree=threads, seed=seed,
                          cpu_iters=0, cpu_threads=cpu_threads)
    want, wbest, wplies = orc.uct_search(root, n_trees, threads, steps, seed, C=C)
    assert res["stats"][:199].tolist() == want[:199].tolist()
    assert res["best_move"] == wbest and res["plies"] == wplies
    assert res["info"]["steps"] == steps and res["info"]["cpu_iterations"] == 0
    m.close()


@pytest.mark.parametrize("n_trees,threads,steps,cpu_iters,seed,C,lmin,lmax,cpu_threads", [
    (1, 64, 40, 4, 3, 1.0, 0, 0, 1),
    (24, 32, 30, 3, 5, 0.25, 20, 40, 7),
    (64, 128, 10, 16, 8, 1.0, 30, 45, 16),
])
def test_hosted_hybrid_iteration_mode_bit_exact(orc, n_trees, threads, steps, cpu_iters, seed, C, lmin, lmax,
                                                cpu_threads):
    m = pkg.Mcts(c_uct=C, scheme="block", device=0)
    root = orc.gen_positions(seed, 1, lmin, lmax) if lmax else orc.opening()
    res = m.search_hosted(root, iterations=steps, n_trees=n_trees, threads_per_tree=threads, seed=seed,
                          cpu_iters=cpu_iters, cpu_threads=cpu_threads)
    want, wbest, cpu = orc.hybrid_search(root, n_trees, threads, steps, cpu_iters, seed, C=C)
    assert res["stats"][:201].tolist() == want[:201].tolist()
    assert res["best_move"] == wbest
    info = res["info"]
    assert info["cpu_iterations"] == cpu["iterations"] == n_trees * steps * cpu_iters
    assert info["cpu_plies"] == cpu["plies"] and info["cpu_depth_sum"] == cpu["depth_sum"]
    assert info["cpu_nodes"] == cpu["cpu_nodes"] and info["gpu_nodes"] == cpu["gpu_nodes"]
    m.close()


def test_hosted_time_mode(block, orc):
    root = orc.gen_positions(21, 1, 10, 20)
    res = block.search_hosted(root, time_ms=100.0, n_trees=296, threads_per_tree=128, seed=2, cpu_iters=1,
                              cpu_threads=8)
    s, info = res["stats"], res["info"]
    assert info["steps"] > 5 and info["cpu_iterations"] > 0
    assert s[195] == info["steps"] * 296 * 128 + info["cpu_iterations"] == s[:65].sum()
    assert s[196] == info["steps"] * 296 + info["cpu_iterations"]
    own, opp = pkg.own_opp(root)
    assert (orc.legal(own, opp) >> res["best_move"]) & 1


def test_hosted_terminal_root_and_errors(block, orc):
    full_black = (1 << 40) - 1
    res = block.search_hosted(orc.position(full_black, ((1 << 64) - 1) & ~full_black, 0), iterations=3,
                              n_trees=4, threads_per_tree=32, seed=1)
    assert res["best_move"] == -1 and (res["stats"] == 0).all()
    with pytest.raises(pkg.MctsError):
        block.search_hosted(orc.opening(), iterations=3, n_trees=4, threads_per_tree=48, seed=1)
    leaf = pkg.Mcts(scheme="leaf", device=0)
    with pytest.raises(pkg.MctsError):
        leaf.search_hosted(orc.opening(), iterations=3, n_trees=1, threads_per_tree=128, seed=1)
    leaf.close()
