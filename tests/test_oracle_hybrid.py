"""Pins for the oracle's hybrid CPU-GPU search on CPU-managed trees
(§III-A, Fig. 4; reading R18).

* with no CPU iterations it is the block-parallel search (uct_search) bit for
  bit: each step selects, expands, simulates `unit` playouts with the
  iteration-s streams and backpropagates before the next selection;
* a hand trace of the first two steps from the opening with two CPU
  iterations per step, built from single oracle playouts and the independent
  Python rules: the CPU iterations expand the root's next untried moves while
  the GPU leaf is pending, a pending leaf (n = 0) is taken first (UCB1's
  unvisited arm), and the rest is the R1 argmax;
* accounting identities: root visits = steps*unit + CPU iterations per tree,
  nodes = 1 + nodes added by GPU steps + by CPU iterations.
"""
import math

import numpy as np
import pytest

import reversi_ref as ref


@pytest.mark.parametrize("n_trees,unit,steps,seed,C,lmin,lmax", [
    (3, 32, 60, 5, 1.0, 0, 0), (2, 64, 40, 6, 0.25, 20, 40), (4, 1, 300, 7, 2.0, 40, 50)])
def test_hybrid_without_cpu_iterations_is_block_search(orc, n_trees, unit, steps, seed, C, lmin, lmax):
    root = orc.gen_positions(seed, 1, lmin, lmax) if lmax else orc.opening()
    s, b, cpu = orc.hybrid_search(root, n_trees, unit, steps, 0, seed, tree_id_base=9, C=C)
    u, ub, _ = orc.uct_search(root, n_trees, unit, steps, seed, tree_id_base=9, C=C)
    assert s[:199].tolist() == u[:199].tolist() and b == ub
    assert cpu["iterations"] == 0 and cpu["cpu_nodes"] == 0


def _pos(orc, own, opp, stm):
    return orc.position(own if stm == 0 else opp, opp if stm == 0 else own, stm)


def _batch(orc, own, opp, stm, seed, c0, c1, count):
    """(wins, draws, losses) for the side to move, one oracle playout per stream."""
    w = d = l = 0
    for j in range(count):
        r, _ = orc.playout(_pos(orc, own, opp, stm), seed, c0, c1, j)
        w += r > 0; d += r == 0; l += r < 0
    return w, d, l


def test_hybrid_hand_trace_two_steps(orc):
    unit, seed, C = 32, 3, 1.0
    B, W = orc.OPENING_BLACK, orc.OPENING_WHITE
    root_moves = ref.squares(ref.legal(B, W))  # [19, 26, 37, 44]
    child = {}
    for mv in root_moves:  # ref.apply -> (discs of the new side to move = white, of the mover = black)
        child[mv] = ref.apply(B, W, mv)
    stats = {mv: [0, 0, 0] for mv in root_moves}  # n, w (for black = root side), d

    def add(mv, wdl, count):  # wdl for the child's side to move (white): black's wins = white's losses
        stats[mv][0] += count; stats[mv][1] += wdl[2]; stats[mv][2] += wdl[1]

    # step 0: GPU leaf = 19 (pending); CPU iterations expand 26 then 37
    g0 = _batch(orc, *child[19], 1, seed, 0, 0, unit)
    add(26, _batch(orc, *child[26], 1, seed, 0, 0x80000000, 1), 1)
    add(37, _batch(orc, *child[37], 1, seed, 0, 0x80000001, 1), 1)
    add(19, g0, unit)
    # step 1: GPU leaf = 44 (pending); CPU iteration 0 takes the pending 44
    # (n = 0: unvisited) and expands 44's lowest legal move
    own44, opp44 = child[44]
    first = ref.squares(ref.legal(own44, opp44))[0]
    nb, nw = ref.apply(own44, opp44, first)  # white moved: black (stm 0) to move
    r = _batch(orc, nb, nw, 0, seed, 0, 0x80000002, 1)  # for black = the root side
    stats[44][0] += 1; stats[44][1] += r[0]; stats[44][2] += r[1]  # 44's w counts black's wins
    # CPU iteration 1: every root child visited; R1 argmax with N = root visits
    N = sum(v[0] for v in stats.values())
    lnN = orc.ln(N)
    best, bu = None, None
    for mv in root_moves:  # ascending index, strict > keeps the first maximum
        n, w, _ = stats[mv]
        u = w / n + C * math.sqrt(lnN / n)
        if bu is None or u > bu:
            best, bu = mv, u
    assert best != 44 or stats[44][0] > 0
    got, _, cpu = orc.hybrid_search(orc.opening(), 1, unit, 2, 2, seed, C=C)
    for mv in root_moves:
        if mv in (best, 44):
            continue
        assert got[mv] == stats[mv][0] and got[65 + mv] == stats[mv][1] and got[130 + mv] == stats[mv][2], mv
    # the step-1 GPU result lands on 44; the second CPU iteration added one visit under `best`
    assert got[44] == stats[44][0] + unit + (1 if best == 44 else 0)
    assert got[best] == stats[best][0] + (1 if best != 44 else unit + 1)
    assert got[195] == 2 * unit + 4 and cpu["iterations"] == 4 and cpu["cpu_nodes"] == 4
    assert cpu["gpu_nodes"] == 2


@pytest.mark.parametrize("steps,cpu_iters,unit", [(50, 3, 32), (20, 16, 128), (200, 1, 1)])
def test_hybrid_accounting(orc, steps, cpu_iters, unit):
    root = orc.gen_positions(4, 1, 10, 30)
    s, b, cpu = orc.hybrid_search(root, 3, unit, steps, cpu_iters, 11)
    assert s[195] == 3 * steps * (unit + cpu_iters) == s[:65].sum()
    assert s[196] == 3 * steps * (1 + cpu_iters)
    assert cpu["iterations"] == 3 * steps * cpu_iters
    assert s[200] == 3 + cpu["cpu_nodes"] + cpu["gpu_nodes"]
    assert cpu["depth_sum"] <= s[198] and s[197] >= cpu["plies"]
    own, opp = (int(root[0]["black"]), int(root[0]["white"])) if root[0]["to_move"] == 0 else \
        (int(root[0]["white"]), int(root[0]["black"]))
    assert (orc.legal(own, opp) >> b) & 1 and b == int(np.argmax(s[:65]))
