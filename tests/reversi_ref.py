"""Independent pure-Python Reversi rules used only to cross-check the oracle.

A shift/mask bitboard (the oracle walks (row, col) rays instead), so a wrap or
direction slip in either implementation shows up as a disagreement. Pure
Python: small cases only.
"""
from __future__ import annotations

FULL = (1 << 64) - 1
NOT_A = 0xFEFEFEFEFEFEFEFE  # clears file a (col 0) after an eastward shift
NOT_H = 0x7F7F7F7F7F7F7F7F  # clears file h (col 7) after a westward shift

# (shift amount, post-shift mask); positive = towards higher square index.
DIRS = [
    (1, NOT_A), (-1, NOT_H),
    (8, FULL), (-8, FULL),
    (9, NOT_A), (-9, NOT_H),
    (7, NOT_H), (-7, NOT_A),
]


def shift(b: int, s: int, mask: int) -> int:
    if s > 0:
        return ((b << s) & FULL) & mask
    return (b >> (-s)) & mask


def popcount(x: int) -> int:
    return bin(x).count("1")


def legal(own: int, opp: int) -> int:
    empty = ~(own | opp) & FULL
    moves = 0
    for s, m in DIRS:
        t = shift(own, s, m) & opp
        for _ in range(5):
            t |= shift(t, s, m) & opp
        moves |= shift(t, s, m) & empty
    return moves


def flips(own: int, opp: int, sq: int) -> int:
    if ((own | opp) >> sq) & 1:
        return 0
    out = 0
    for s, m in DIRS:
        run = 0
        x = shift(1 << sq, s, m)
        while x & opp:
            run |= x
            x = shift(x, s, m)
        if run and (x & own):
            out |= run
    return out


def apply(own: int, opp: int, sq: int):
    f = flips(own, opp, sq)
    return opp & ~f, own | f | (1 << sq)  # (new own = old opponent, new opp = mover)


def squares(mask: int):
    return [s for s in range(64) if (mask >> s) & 1]


# The 8 dihedral symmetries of the board as square maps.
def _sym(k: int):
    def f(sq: int) -> int:
        r, c = divmod(sq, 8)
        for _ in range(k % 4):
            r, c = c, 7 - r
        if k >= 4:
            c = 7 - c
        return 8 * r + c
    return f


SYMMETRIES = [_sym(k) for k in range(8)]


def transform(mask: int, f) -> int:
    out = 0
    for s in squares(mask):
        out |= 1 << f(s)
    return out


def exact_outcome_probs(own: int, opp: int):
    """Exact (P(win), P(draw), P(loss)) for the side to move under uniform random
    play (each legal move with probability 1/c, passes forced) — brute force."""
    from fractions import Fraction
    memo = {}

    def rec(me: int, op: int, start: bool):
        key = (me, op, start)
        if key in memo:
            return memo[key]
        m = legal(me, op)
        if m == 0:
            if legal(op, me) == 0:
                a, b = (me, op) if start else (op, me)
                pa, pb = popcount(a), popcount(b)
                r = (Fraction(1), Fraction(0), Fraction(0)) if pa > pb else (
                    (Fraction(0), Fraction(1), Fraction(0)) if pa == pb else
                    (Fraction(0), Fraction(0), Fraction(1)))
            else:
                r = rec(op, me, not start)
        else:
            sq = squares(m)
            acc = [Fraction(0)] * 3
            for s in sq:
                no, nm = apply(me, op, s)
                sub = rec(no, nm, not start)
                for i in range(3):
                    acc[i] += sub[i]
            r = tuple(x / len(sq) for x in acc)
        memo[key] = r
        return r

    return rec(own, opp, True)
