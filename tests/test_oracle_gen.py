"""Pins for the synthetic position generator (DESIGN.md §4 input recipe).

Re-derived step by step in Python with the independent rules of reversi_ref
and the KAT-pinned RNG words; plus reachability invariants.
"""
import reversi_ref as ref


def py_gen(orc, seed, p, lmin, lmax):
    attempt = 0
    while True:
        span = lmax - lmin + 1
        L = lmin + ((orc.rng_word(seed, p, 0xFFFFFFFF, attempt, 0) * span) >> 32)
        me, op, stm, w, plies, ok = 0x0000000810000000, 0x0000001008000000, 0, 1, 0, True
        while plies < L:
            m = ref.legal(me, op)
            if m == 0:
                if ref.legal(op, me) == 0:
                    ok = False
                    break
                me, op, stm = op, me, stm ^ 1
                continue
            sq = ref.squares(m)
            s = sq[(orc.rng_word(seed, p, 0xFFFFFFFF, attempt, w) * len(sq)) >> 32]
            w += 1
            me, op = ref.apply(me, op, s)
            stm ^= 1
            plies += 1
        if ok and not (ref.legal(me, op) == 0 and ref.legal(op, me) == 0):
            return (me, op, stm) if stm == 0 else (op, me, stm), L
        attempt += 1


def test_generator_matches_python(orc):
    for seed, lmin, lmax in [(2, 20, 40), (3, 0, 8), (4, 40, 50)]:
        g = orc.gen_positions(seed, 40, lmin, lmax)
        for p in range(40):
            (b, w, stm), L = py_gen(orc, seed, p, lmin, lmax)
            assert (int(g[p]["black"]), int(g[p]["white"]), int(g[p]["to_move"])) == (b, w, stm)
            assert ref.popcount(b | w) == 4 + L
            assert lmin <= L <= lmax


def test_generator_invariants(orc):
    g = orc.gen_positions(2, 4096, 20, 40)
    for p in g:
        b, w = int(p["black"]), int(p["white"])
        assert b & w == 0
        assert 24 <= ref.popcount(b | w) <= 44
        assert not (ref.legal(b, w) == 0 and ref.legal(w, b) == 0)
    # deterministic
    g2 = orc.gen_positions(2, 4096, 20, 40)
    assert (g == g2).all()
    op = orc.gen_positions(1, 3, 0, 0)
    assert all(int(x["black"]) == orc.OPENING_BLACK and int(x["white"]) == orc.OPENING_WHITE
               and int(x["to_move"]) == 0 for x in op)
