"""Pins for the oracle's random playouts and batch driver.

* a step-by-step pure-Python re-derivation of a playout (independent rules in
  reversi_ref, RNG words pinned by the Philox KATs) must agree exactly;
* the empirical outcome rates of many playouts from small endgames must match
  the exact uniform-random-play distribution obtained by exhaustive
  enumeration (brute force), within 4.5 sigma;
* terminal and pass-only leaves, and the batch stream-id layout.
"""
import math
import random

import numpy as np
import pytest

import reversi_ref as ref


def py_playout(orc, own, opp, seed, c0, c1, c2):
    me, op, start, w, plies = own, opp, True, 0, 0
    while True:
        m = ref.legal(me, op)
        if m == 0:
            if ref.legal(op, me) == 0:
                break
            me, op, start = op, me, not start
            continue
        r = orc.rng_word(seed, c0, c1, c2, w)
        w += 1
        sq = ref.squares(m)
        s = sq[(r * len(sq)) >> 32]
        me, op = ref.apply(me, op, s)
        start = not start
        plies += 1
    a, b = (me, op) if start else (op, me)
    pa, pb = ref.popcount(a), ref.popcount(b)
    return (1 if pa > pb else 0 if pa == pb else -1), plies


def _pos(orc, own, opp, to_move=0):
    if to_move == 0:
        return orc.position(own, opp, 0)
    return orc.position(opp, own, 1)


def test_playout_matches_python_rederivation(orc):
    rng = random.Random(2)
    gen = orc.gen_positions(9, 24, 0, 50)
    for i, p in enumerate(gen):
        own, opp = (int(p["black"]), int(p["white"])) if p["to_move"] == 0 else (int(p["white"]), int(p["black"]))
        for j in range(3):
            seed = rng.getrandbits(64)
            c = (rng.getrandbits(32), rng.getrandbits(32), rng.getrandbits(32))
            got = orc.playout(np.array([p]), seed, *c)
            assert got == py_playout(orc, own, opp, seed, *c)


def _endgame_positions(n_empty, count, seed):
    rng = random.Random(seed)
    out = []
    while len(out) < count:
        own, opp = 0x0000000810000000, 0x0000001008000000
        while True:
            empties = 64 - ref.popcount(own | opp)
            m = ref.legal(own, opp)
            if m == 0:
                if ref.legal(opp, own) == 0:
                    break
                own, opp = opp, own
                continue
            if empties == n_empty:
                out.append((own, opp))
                break
            own, opp = ref.apply(own, opp, rng.choice(ref.squares(m)))
    return out


@pytest.mark.parametrize("n_empty,seed", [(6, 1), (7, 2), (8, 3)])
def test_outcome_distribution_matches_exhaustive_enumeration(orc, n_empty, seed):
    N = 6000
    asym = 0.0
    for own, opp in _endgame_positions(n_empty, 3, seed):
        pw, pd, pl = (float(x) for x in ref.exact_outcome_probs(own, opp))
        wdl, _ = orc.playouts(_pos(orc, own, opp), N, seed=1234 + n_empty)
        emp = wdl[0] / N
        for p, e in zip((pw, pd, pl), emp):
            sigma = math.sqrt(max(p * (1 - p), 1e-12) / N)
            assert abs(e - p) <= 4.5 * sigma + 1e-12, (own, opp, (pw, pd, pl), emp)
        asym = max(asym, abs(pw - pl) / math.sqrt(1.0 / N))
    # the positions must be able to tell a win from a loss (catches a sign slip)
    assert asym > 8


def test_terminal_leaf(orc):
    # Full board, black 40 white 24, black "to move": game over, black wins.
    black = (1 << 40) - 1
    white = ((1 << 64) - 1) & ~black
    wdl, plies = orc.playouts(orc.position(black, white, 0), 50, seed=5)
    assert wdl.tolist() == [[50, 0, 0]] and plies == 0
    wdl, plies = orc.playouts(orc.position(black, white, 1), 50, seed=5)
    assert wdl.tolist() == [[0, 0, 50]] and plies == 0
    # a drawn terminal
    black = (1 << 32) - 1
    white = ((1 << 64) - 1) & ~black
    wdl, _ = orc.playouts(orc.position(black, white, 0), 7, seed=5)
    assert wdl.tolist() == [[0, 7, 0]]


def test_pass_leaf(orc):
    # Black a1,b1 and white c1 with white to move: white brackets nothing and
    # passes; black's only move d1 takes the last white disc; game over, white loses.
    black, white = 0b11, 0b100
    assert ref.legal(white, black) == 0 and ref.legal(black, white) != 0
    wdl, plies = orc.playouts(orc.position(black, white, 1), 20, seed=3)
    assert wdl.tolist() == [[0, 0, 20]] and plies == 20  # one move each, white loses


def test_batch_stream_layout(orc):
    leaves = orc.gen_positions(2, 12, 20, 40)
    wdl, plies = orc.playouts(leaves, 16, seed=77, leaf_id_base=1000, nthreads=3)
    tot = 0
    for i in range(len(leaves)):
        w = d = l = 0
        for j in range(16):
            r, pl = orc.playout(leaves[i:i + 1], 77, 1000 + i, 0, j)
            tot += pl
            w += r > 0; d += r == 0; l += r < 0
        assert wdl[i].tolist() == [w, d, l]
    assert plies == tot
    assert (wdl.sum(axis=1) == 16).all()


def test_zero_playouts(orc):
    wdl, plies = orc.playouts(orc.opening(), 0, seed=1)
    assert wdl.tolist() == [[0, 0, 0]] and plies == 0
