"""MCTS_TREE (tree parallelism on one shared device tree).

One worker: nothing races and the virtual-loss terms vanish, so the search is
the oracle's sequential UCT with one tree — compared bit for bit. Many workers:
the result depends on timing (as for any parallel tree search), so the tests
check what holds regardless: the device-side tree invariants
(MCTS_FLAG_CHECK_TREE: no virtual visit left, k(v) >= sum of children k (+1
below the root), sum over nodes of k - children k = iterations run) and the
root statistics identities.
"""
import numpy as np
import pytest
import torch

import paper_conf_ipps_rockis11_b200 as pkg

pytestmark = pytest.mark.gpu


def _tree(C=1.0, check=True, max_nodes=0):
    return pkg.Mcts(c_uct=C, scheme="tree", device=0, max_nodes_per_tree=max_nodes,
                    flags=pkg.MCTS_FLAG_CHECK_TREE if check else 0)


def test_tree_single_worker_config0_bit_exact(orc):
    """BASELINE configs[0] (opening, 64 threads, 100 iterations, seed 1) as one worker."""
    m = _tree()
    res = m.search(pkg.opening(), iterations=100, n_trees=1, threads_per_tree=64, seed=1)
    ostats, obest, oplies = orc.uct_search(orc.opening(), 1, 64, 100, 1)
    assert res["stats"][:200].tolist() == ostats[:200].tolist()
    assert res["best_move"] == obest and res["plies"] == oplies
    m.close()


@pytest.mark.parametrize("threads,iters,seed,C,lmin,lmax", [
    (32, 400, 4, 1.0, 20, 40),
    (128, 150, 5, 0.25, 10, 30),
    (96, 120, 6, 2.0, 30, 50),
    (1024, 10, 7, 1.0, 0, 8),
    (64, 300, 8, 0.0, 20, 40),
])
def test_tree_single_worker_bit_exact(orc, threads, iters, seed, C, lmin, lmax):
    m = _tree(C)
    root = orc.gen_positions(seed, 1, lmin, lmax)
    res = m.search(root, iterations=iters, n_trees=1, threads_per_tree=threads, seed=seed)
    ostats, obest, oplies = orc.uct_search(root, 1, threads, iters, seed, C=C)
    assert res["stats"][:200].tolist() == ostats[:200].tolist()
    assert res["best_move"] == obest and res["plies"] == oplies
    m.close()


def test_tree_single_worker_tree_id_base(orc):
    """c0 = tree_id_base through the async entry point (the multi-GPU layout)."""
    m = _tree()
    root = orc.gen_positions(9, 1, 20, 40)
    st = torch.zeros(pkg.STATS_LEN, dtype=torch.int64, device="cuda")
    m.search_async(root, 40, 0.0, 1, 64, 3, 5, st.data_ptr(), torch.cuda.current_stream())
    torch.cuda.synchronize()
    ostats, _, _ = orc.uct_search(root, 1, 64, 40, 3, tree_id_base=5)
    assert st.cpu().numpy()[:200].tolist() == ostats[:200].tolist()
    m.close()


def test_tree_terminal_and_pass_roots(orc):
    m = _tree()
    full_black = (1 << 40) - 1
    full_white = ((1 << 64) - 1) & ~full_black
    res = m.search(orc.position(full_black, full_white, 0), iterations=5, n_trees=64, threads_per_tree=32, seed=1)
    assert res["best_move"] == -1 and (res["stats"] == 0).all()
    root = orc.position(0b11, 0b100, 1)
    res = m.search(root, iterations=6, n_trees=1, threads_per_tree=32, seed=2)
    ostats, obest, _ = orc.uct_search(root, 1, 32, 6, 2)
    assert res["stats"][:200].tolist() == ostats[:200].tolist() and res["best_move"] == 64
    m.close()


def _root_identities(res, root, orc, unit, iterations=None):
    s = res["stats"]
    it = res["iterations"]
    if iterations is not None:
        assert it == iterations
    assert s[195] == it * unit                      # every iteration passes the root
    assert s[:65].sum() <= s[195]                   # the rest ended at the root itself
    assert (s[65:130] + s[130:195] <= s[:65]).all()
    own, opp = pkg.own_opp(root)
    legal = orc.legal(own, opp)
    visited = np.nonzero(s[:64])[0]
    assert all((legal >> int(mv)) & 1 for mv in visited)
    assert (legal >> res["best_move"]) & 1


@pytest.mark.parametrize("workers,threads,iters", [(2, 64, 500), (148, 128, 3000), (1184, 128, 20000),
                                                   (4736, 32, 20000)])
def test_tree_many_workers_invariants(orc, workers, threads, iters):
    m = _tree()
    root = orc.gen_positions(31, 1, 10, 30)
    res = m.search(root, iterations=iters, n_trees=workers, threads_per_tree=threads, seed=11)
    _root_identities(res, root, orc, threads, iterations=iters)
    m.close()


def test_tree_time_mode_invariants(orc):
    """configs[2] launch shape as workers of one tree, 100 ms, invariants checked on the device."""
    m = _tree(C=0.25)
    root = orc.opening()
    res = m.search(root, time_ms=100.0, n_trees=1184, threads_per_tree=128, seed=12)
    assert res["iterations"] > 1184
    _root_identities(res, root, orc, 128)
    m.close()


def test_tree_time_mode_pool_full(orc):
    """A small pool fills up: nodes created without a child block are simulated, never expanded."""
    m = _tree(max_nodes=4096)
    root = orc.gen_positions(32, 1, 20, 30)
    res = m.search(root, time_ms=30.0, n_trees=296, threads_per_tree=64, seed=13)
    _root_identities(res, root, orc, 64)
    m.close()


def test_tree_argument_errors(orc):
    m = _tree()
    with pytest.raises(pkg.MctsError):
        m.search(pkg.opening(), iterations=10, n_trees=4, threads_per_tree=48, seed=1)
    with pytest.raises(pkg.MctsError):
        m.search(pkg.opening(), iterations=(1 << 24) + 1, n_trees=4, threads_per_tree=32, seed=1)
    with pytest.raises(pkg.MctsError):
        m.search(pkg.opening(), iterations=10, n_trees=65537, threads_per_tree=32, seed=1)
    m.close()
    with pytest.raises(pkg.MctsError):
        pkg.Mcts(scheme="tree", device=0, flags=4)


def test_tree_hybrid_iteration_mode(orc):
    """NEXT-1 on top of NEXT-4: the shared tree (one worker: deterministic) plus
    host trees, root sums merged — the oracle's two searches added up."""
    m = _tree()
    root = orc.gen_positions(42, 1, 20, 30)
    res = m.search_hybrid(root, iterations=60, n_trees=1, threads_per_tree=64, seed=14, cpu_threads=3)
    g, _, gp = orc.uct_search(root, 1, 64, 60, 14)
    c, _, cp = orc.uct_search(root, 3, 1, 60, 14, tree_id_base=0x40000000)
    merged = g + c
    assert res["stats"][:200].tolist() == merged[:200].tolist()
    assert res["plies"] == gp + cp
    m.close()


def test_tree_hybrid_time_mode(orc):
    m = _tree()
    root = orc.opening()
    res = m.search_hybrid(root, time_ms=50.0, n_trees=592, threads_per_tree=128, seed=15, cpu_threads=4)
    assert res["cpu"]["iterations"] > 0 and res["iterations"] > res["cpu"]["iterations"]
    assert res["stats"][195] == (res["iterations"] - res["cpu"]["iterations"]) * 128 + res["cpu"]["iterations"]
    m.close()
