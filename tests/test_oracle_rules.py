"""Pins for the oracle's Reversi rules (oracle.cpp legal/flips/perft).

Pinned against: the perft counts in BASELINE.json north_star (golden file),
an independent shift/mask bitboard (tests/reversi_ref.py), the 8 board
symmetries and the disc-count invariants of a move.
"""
import os
import random

import pytest

import reversi_ref as ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _golden_perft():
    rows = []
    with open(os.path.join(GOLDEN, "perft_opening.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                d, a, b = (int(x) for x in line.split())
                rows.append((d, a, b))
    return rows


@pytest.mark.parametrize("depth,with_pass,without_pass", _golden_perft())
def test_perft_opening(orc, depth, with_pass, without_pass):
    assert orc.perft(orc.OPENING_BLACK, orc.OPENING_WHITE, 0, depth, True) == with_pass
    if depth <= 8 or without_pass != with_pass:
        assert orc.perft(orc.OPENING_BLACK, orc.OPENING_WHITE, 0, depth, False) == without_pass


def test_opening_moves(orc):
    # black's opening moves are d3, c4, f5, e6 = 19, 26, 37, 44.
    m = orc.legal(orc.OPENING_BLACK, orc.OPENING_WHITE)
    assert ref.squares(m) == [19, 26, 37, 44]


def _random_positions(n, seed):
    rng = random.Random(seed)
    out = []
    while len(out) < n:
        own, opp = orc_open = (0x0000000810000000, 0x0000001008000000)
        while True:
            out.append((own, opp))
            m = ref.legal(own, opp)
            if m == 0:
                if ref.legal(opp, own) == 0:
                    break
                own, opp = opp, own
                continue
            sq = rng.choice(ref.squares(m))
            own, opp = ref.apply(own, opp, sq)
    return out[:n]


def test_legal_and_flips_match_independent_bitboard(orc):
    for own, opp in _random_positions(3000, 7):
        m = orc.legal(own, opp)
        assert m == ref.legal(own, opp)
        for sq in range(64):
            assert orc.flips(own, opp, sq) == ref.flips(own, opp, sq)


def test_legal_on_random_masks(orc):
    # Arbitrary (not necessarily reachable) disjoint masks stress the edges.
    rng = random.Random(11)
    for _ in range(3000):
        a = rng.getrandbits(64)
        b = rng.getrandbits(64) & ~a
        if rng.random() < 0.5:
            b &= rng.getrandbits(64)
        assert orc.legal(a, b) == ref.legal(a, b)
        sq = rng.randrange(64)
        assert orc.flips(a, b, sq) == ref.flips(a, b, sq)


def test_symmetry_invariance(orc):
    for own, opp in _random_positions(400, 3):
        m = orc.legal(own, opp)
        for f in ref.SYMMETRIES:
            assert orc.legal(ref.transform(own, f), ref.transform(opp, f)) == ref.transform(m, f)


def test_apply_invariants(orc):
    for own, opp in _random_positions(1500, 5):
        m = orc.legal(own, opp)
        for sq in ref.squares(m):
            f = orc.flips(own, opp, sq)
            assert f != 0 and (f & ~opp) == 0
            k = ref.popcount(f)
            new_mover = own | f | (1 << sq)
            new_other = opp & ~f
            assert new_mover & new_other == 0
            assert ref.popcount(new_mover) == ref.popcount(own) + 1 + k
            assert ref.popcount(new_other) == ref.popcount(opp) - k
        # a non-legal empty square flips nothing
        empty = ~(own | opp) & ref.FULL
        for sq in ref.squares(empty & ~m):
            assert orc.flips(own, opp, sq) == 0
