"""Pins for the oracle's UCT search (R1, R2, R6, R8, R10).

* hand trace from the opening: the first four iterations expand the root's
  legal moves in ascending order and each child's (n, w, d) equals the
  (losses, draws) of the playout batch keyed (tree, iteration, 0..unit-1);
* the fifth selection is the UCB argmax computed here at 50 digits;
* tree invariants (n(v) = unit + sum of children for expanded interior nodes,
  root n = iterations * unit, perspective identity for w, multiples of unit);
* the multi-tree merge identity (root sums);
* pool-full behaviour, terminal root, best move = max visits.
"""
from decimal import Decimal, getcontext

import numpy as np
import pytest

import reversi_ref as ref

getcontext().prec = 50


def own_opp(p):
    p = p[0] if p.shape else p
    if int(p["to_move"]) == 0:
        return int(p["black"]), int(p["white"])
    return int(p["white"]), int(p["black"])


def child_position(orc, parent_pos, move):
    own, opp = own_opp(parent_pos)
    stm = int(parent_pos[0]["to_move"])
    if move == 64:
        no, nm = opp, own
    else:
        no, nm = ref.apply(own, opp, move)
    # no = new side to move's discs, nm = mover's discs
    new_stm = 1 - stm
    return orc.position(no if new_stm == 0 else nm, nm if new_stm == 0 else no, new_stm)


def test_hand_trace_first_iterations(orc):
    unit, seed, tree = 64, 1, 0
    root = orc.opening()
    t = orc.uct_tree(root, unit, 5, seed, tree_id=tree, C=1.0)
    assert t["move"][:5].tolist() == [-1, 19, 26, 37, 44]
    assert t["parent"][1:5].tolist() == [0, 0, 0, 0]
    children = []
    for it, mv in enumerate([19, 26, 37, 44]):
        cp = child_position(orc, root, mv)
        w = d = l = 0
        for j in range(unit):
            r, _ = orc.playout(cp, seed, tree, it, j)
            w += r > 0; d += r == 0; l += r < 0
        node = it + 1
        if node != int(t["parent"][5]):
            assert int(t["n"][node]) == unit
            assert int(t["w"][node]) == l  # mover(child) = root's side to move
            assert int(t["d"][node]) == d
        children.append((node, l, d))
    # the fifth iteration descends by UCB from the root (T = 4*unit)
    lnT = float(Decimal(4 * unit).ln())
    best, best_u = None, None
    for node, w, d in children:
        u = Decimal(w) / Decimal(unit) + (Decimal(lnT) / Decimal(unit)).sqrt()
        if best_u is None or u > best_u:
            best, best_u = node, u
    assert int(t["parent"][5]) == best
    sel_pos = child_position(orc, root, int(t["move"][best]))
    lm = orc.legal(*own_opp(sel_pos))
    assert int(t["move"][5]) == ref.squares(lm)[0]


def _check_invariants(t, unit, iterations, capacity_hit=False):
    parent, n, w, d, term = t["parent"], t["n"], t["w"], t["d"], t["terminal"]
    cnt = len(parent)
    kids = [[] for _ in range(cnt)]
    for v in range(1, cnt):
        assert parent[v] < v
        kids[parent[v]].append(v)
    assert int(n[0]) == iterations * unit
    assert sum(int(n[c]) for c in kids[0]) == int(n[0])
    for v in range(cnt):
        assert int(n[v]) % unit == 0 and int(n[v]) > 0
        assert int(w[v]) + int(d[v]) <= int(n[v])
        if v == 0:
            continue
        if term[v]:
            assert not kids[v]
            continue
        sn = sum(int(n[c]) for c in kids[v])
        # leaf-simulation contribution of v itself (wins for mover(v)):
        # children's w are wins for the *other* side, so v gains their losses.
        own_n = int(n[v]) - sn
        own_w = int(w[v]) - sum(int(n[c]) - int(w[c]) - int(d[c]) for c in kids[v])
        own_d = int(d[v]) - sum(int(d[c]) for c in kids[v])
        if capacity_hit:
            assert own_n >= unit and own_n % unit == 0
        else:
            assert own_n == unit
        assert 0 <= own_w and 0 <= own_d and own_w + own_d <= own_n


@pytest.mark.parametrize("seed,unit,iters", [(1, 32, 300), (2, 1, 2000), (3, 64, 150)])
def test_tree_invariants(orc, seed, unit, iters):
    for p in orc.gen_positions(seed, 3, 10, 40):
        t = orc.uct_tree(np.array([p]), unit, iters, seed, tree_id=seed, C=1.0)
        assert len(t["parent"]) == iters + 1 or t["terminal"].any()
        _check_invariants(t, unit, iters)


def test_pool_full(orc):
    p = orc.gen_positions(5, 1, 20, 30)
    t = orc.uct_tree(p, 32, 200, 5, tree_id=0, C=1.0, capacity=40)
    assert len(t["parent"]) == 40
    _check_invariants(t, 32, 200, capacity_hit=True)


def test_merge_identity(orc):
    root = orc.gen_positions(8, 1, 20, 30)
    full, best_full, plies_full = orc.uct_search(root, 8, 32, 20, seed=3, tree_id_base=0)
    parts = np.zeros_like(full)
    plies = 0
    for r in range(4):
        s, _, pl = orc.uct_search(root, 2, 32, 20, seed=3, tree_id_base=2 * r)
        parts += s
        plies += pl
    assert (parts == full).all() and plies == plies_full
    assert full[195] == 8 * 20 * 32 and full[196] == 8 * 20
    assert full[:65].sum() == full[195]
    assert best_full == int(np.argmax(full[:65]))


def test_single_tree_equals_tree_dump(orc):
    root = orc.opening()
    s, best, _ = orc.uct_search(root, 1, 64, 100, seed=1)
    t = orc.uct_tree(root, 64, 100, 1)
    for v in range(1, len(t["parent"])):
        if t["parent"][v] == 0:
            mv = int(t["move"][v])
            assert s[mv] == t["n"][v] and s[65 + mv] == t["w"][v] and s[130 + mv] == t["d"][v]
    assert best == int(np.argmax(s[:65]))


def test_terminal_root(orc):
    black = (1 << 40) - 1
    white = ((1 << 64) - 1) & ~black
    s, best, plies = orc.uct_search(orc.position(black, white, 0), 4, 32, 10, seed=1)
    assert best == -1 and (s == 0).all() and plies == 0


def test_pass_root(orc):
    # white to move must pass: the only child is the pass child (index 64)
    black, white = 0b11, 0b100
    s, best, _ = orc.uct_search(orc.position(black, white, 1), 2, 32, 3, seed=1)
    assert best == 64 and s[64] == 2 * 3 * 32 and s[:64].sum() == 0


def test_depth_sum_hand_trace(orc):
    """stats[198] = sum over iterations of the simulated node's depth (the
    paper's tree depth, Fig. 8). From the opening the first four iterations
    expand the four root children (depth 1 each) and the fifth expands a child
    of the selected one (depth 2): 1 + 1 + 1 + 1 + 2 = 6."""
    s4, _, _ = orc.uct_search(orc.opening(), 1, 64, 4, seed=1)
    s5, _, p5 = orc.uct_search(orc.opening(), 1, 64, 5, seed=1)
    assert s4[198] == 4 and s5[198] == 6
    assert s5[197] == p5  # [197] = playout plies, also returned separately


@pytest.mark.parametrize("seed,unit,iters,cap", [(1, 32, 300, 0), (2, 1, 2000, 0), (5, 32, 200, 40)])
def test_depth_sum_equals_tree_visits(orc, seed, unit, iters, cap):
    """Every iteration adds `unit` to n of each node on its path below the root,
    so the depth sum equals sum over non-root nodes of n / unit (the tree dump
    against the search's own depth bookkeeping, incl. a full pool)."""
    for p in orc.gen_positions(seed, 2, 10, 40):
        root = np.array([p])
        s, _, _ = orc.uct_search(root, 1, unit, iters, seed, tree_id_base=seed, capacity=cap)
        t = orc.uct_tree(root, unit, iters, seed, tree_id=seed, C=1.0, capacity=cap)
        assert int(s[198]) == sum(int(x) for x in t["n"][1:]) // unit


# ---------------------------------------------------------------- the CPU opponent
@pytest.mark.parametrize("threads,iters,seed,C,lmin,lmax", [
    (1, 300, 3, 1.0, 0, 0),      # the opening
    (4, 200, 5, 0.25, 20, 40),   # the C the self-play runs use
    (3, 150, 7, 2.0, 40, 50),    # late game: passes and terminal nodes in the tree
    (16, 64, 9, 0.0, 10, 30),    # pure exploitation
])
def test_mcts_timed_capped_equals_uct_search(orc, threads, iters, seed, C, lmin, lmax):
    """The root-parallel CPU opponent, capped at `iters`
    iterations per thread with no deadline, is T independent unit-1 trees keyed
    (c0 = thread, c1 = iteration, c2 = 0) summed at the root: bit for bit
    uct_search(root, T, 1, iters, seed) — the root stats, counters and the move."""
    root = orc.gen_positions(seed, 1, lmin, lmax) if lmax else orc.opening()
    got, best = orc.mcts_timed(root, threads, 0.0, seed, C=C, max_iterations=iters)
    want, wbest, plies = orc.uct_search(root, threads, 1, iters, seed, C=C)
    assert got[:201].tolist() == want[:201].tolist()  # [201]: the opponent's pool is unbounded
    assert best == wbest
    assert got[196] == threads * iters and got[195] == threads * iters and got[197] == plies


def test_mcts_timed_cap_with_generous_deadline(orc):
    """A deadline that does not bind changes nothing."""
    root = orc.gen_positions(11, 1, 20, 30)
    got, best = orc.mcts_timed(root, 2, 60000.0, 4, C=0.5, max_iterations=100)
    want, wbest, _ = orc.uct_search(root, 2, 1, 100, 4, C=0.5)
    assert got[:201].tolist() == want[:201].tolist() and best == wbest


def test_mcts_timed_time_mode_invariants(orc):
    """Time mode (the self-play opponent): one playout per iteration, root
    visits = iterations = sum of root-child visits, legal best move = argmax."""
    root = orc.gen_positions(12, 1, 10, 30)
    s, best = orc.mcts_timed(root, 4, 60.0, 5, C=0.25)
    assert s[196] >= 4 and s[195] == s[196] == s[:65].sum()
    assert (s[65:130] + s[130:195] <= s[:65]).all()
    own, opp = own_opp(root)
    assert (orc.legal(own, opp) >> best) & 1
    assert best == int(np.argmax(s[:65]))


def test_mcts_timed_terminal_root(orc):
    full_black = (1 << 40) - 1
    s, best = orc.mcts_timed(orc.position(full_black, ((1 << 64) - 1) & ~full_black, 0), 2, 0.0, 1,
                             max_iterations=10)
    assert best == -1 and (s == 0).all()


@pytest.mark.parametrize("seed,cap,lmin,lmax", [(5, 40, 20, 30), (6, 12, 40, 50), (7, 300, 0, 10)])
def test_refused_expansions_counter(orc, seed, cap, lmin, lmax):
    """stats[199] (expansions refused by a full pool, R12) from the tree dump:
    every iteration either expands one node, ends at a terminal node, or is
    refused, so refused = iterations - (nodes - 1) - sum over terminal nodes
    of (visits / unit - 1) (the iteration that created a terminal node ended
    there as its expansion). [200] = nodes, [201] = capacity."""
    unit, iters = 32, 400
    root = orc.gen_positions(seed, 1, lmin, lmax)
    s, _, _ = orc.uct_search(root, 1, unit, iters, seed, capacity=cap)
    t = orc.uct_tree(root, unit, iters, seed, tree_id=0, C=1.0, capacity=cap)
    nodes = len(t["parent"])
    term_ends = sum(int(n) // unit - 1 for n, term, par in zip(t["n"], t["terminal"], t["parent"])
                    if term and par >= 0)
    assert s[199] == iters - (nodes - 1) - term_ends
    assert s[200] == nodes and s[201] == cap
    if nodes == cap:
        assert s[199] > 0
    s0, _, _ = orc.uct_search(root, 1, unit, iters, seed)  # iteration-mode pool: never refuses
    assert s0[199] == 0 and s0[:199].tolist() != [] and s0[201] == iters + 1
