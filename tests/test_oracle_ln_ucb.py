"""Pins for the ln table (reading R9) and the UCB value (reading R1).

ln: every entry must equal the double nearest to ln(k*unit) computed with
50-digit decimal arithmetic (Python's decimal module, then a correctly rounded
decimal->double conversion), including the glibc-misrounded regression values
in tests/golden/ln_regression.txt.

UCB: u = w/n + C*sqrt(ln(T)/n) (UCB1) compared with a
50-digit evaluation; five correctly rounded operations keep the double within a
few ulp of the exact value.
"""
import math
import os
import random
from decimal import Decimal, getcontext

import pytest

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
getcontext().prec = 50


def rn_ln(x: int) -> float:
    return float(Decimal(x).ln())


def test_ln_regression(orc):
    with open(os.path.join(GOLDEN, "ln_regression.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                x, h = line.split()
                assert orc.ln(int(x)) == float.fromhex(h) == rn_ln(int(x))


@pytest.mark.parametrize("unit,K", [(1, 12000), (64, 3000), (128, 3000), (16384, 2000), (1, 0)])
def test_ln_table_correctly_rounded(orc, unit, K):
    t = orc.ln_table(unit, K)
    assert t[0] == 0.0
    for k in range(1, K + 1):
        assert t[k] == rn_ln(k * unit), (k, unit)


def test_ln_near_midpoint_cases(orc):
    # the values n <= 2^16 whose ln lies within 1e-3 ulp of a rounding midpoint
    hard = []
    for n in range(2, 1 << 16):
        exact = Decimal(n).ln()
        d = float(exact)
        ulp = math.ulp(d)
        frac = (exact - Decimal(d)) / Decimal(ulp)
        if abs(abs(frac) - Decimal("0.5")) < Decimal("0.001"):
            hard.append(n)
    assert 9170 in hard
    for n in hard:
        assert orc.ln(n) == rn_ln(n)
    rng = random.Random(4)
    for _ in range(3000):
        n = rng.randrange(1 << 16, 1 << 40)
        assert orc.ln(n) == rn_ln(n)


def test_ucb_against_high_precision(orc):
    rng = random.Random(9)
    for _ in range(4000):
        unit = rng.choice([1, 32, 64, 128, 16384])
        n = unit * rng.randrange(1, 5000)
        w = rng.randrange(0, n + 1)
        T = n + unit * rng.randrange(1, 50000)
        C = rng.choice([0.0, 0.5, 1.0, math.sqrt(2), 2.0])
        lnT = rn_ln(T)
        got = orc.ucb(w, n, lnT, C)
        exact = Decimal(w) / Decimal(n) + Decimal(C) * (Decimal(lnT) / Decimal(n)).sqrt()
        assert abs(Decimal(got) - exact) <= 4 * Decimal(math.ulp(float(exact))), (w, n, T, C)


def test_ucb_terms_are_distinguishable(orc):
    # exploitation only (C = 0) and exploration only (w = 0)
    assert orc.ucb(3, 4, 10.0, 0.0) == 0.75
    assert orc.ucb(0, 4, 16.0, 1.0) == 2.0
    assert orc.ucb(0, 4, 16.0, 0.5) == 1.0
    assert orc.ucb(2, 4, 16.0, 1.0) == 2.5


def _ucb_r1(w, n, lnT, C):
    """Reading R1's operation order, each step an IEEE double RN operation
    (Python floats): exploit = w/n; ratio = lnT/n; root = sqrt(ratio);
    explore = C*root; u = exploit + explore."""
    exploit = float(w) / float(n)
    root = math.sqrt(lnT / float(n))
    return exploit + C * root


def _alternatives(w, n, lnT, C):
    """Plausible mis-orderings of the same formula, each correctly rounded per step."""
    from fractions import Fraction
    exploit = float(w) / float(n)
    root = math.sqrt(lnT / float(n))
    return {
        "sqrt(lnT)/sqrt(n)": exploit + C * (math.sqrt(lnT) / math.sqrt(float(n))),
        "C*sqrt(lnT)/sqrt(n)": exploit + (C * math.sqrt(lnT)) / math.sqrt(float(n)),
        "fma(C, root, exploit)": float(Fraction(C) * Fraction(root) + Fraction(exploit)),
        "sqrt(C*C*lnT/n)": exploit + math.sqrt(C * C * lnT / float(n)),
        "(w + C*sqrt(lnT*n))/n": (float(w) + C * math.sqrt(lnT * float(n))) / float(n),
    }


def test_ucb_operation_order_pinned(orc):
    """The oracle's UCB is R1's five RN operations in R1's order, bit for bit,
    and each plausible re-ordering differs from it on some of these inputs (so
    the test would catch the slip, which the 4-ulp bound above cannot)."""
    rng = random.Random(17)
    differs = {}
    for _ in range(20000):
        unit = rng.choice([1, 32, 64, 128, 16384])
        n = unit * rng.randrange(1, 5000)
        w = rng.randrange(0, n + 1)
        T = n + unit * rng.randrange(1, 50000)
        C = rng.choice([0.25, 0.5, 1.0 / 3.0, math.sqrt(2), 0.7, 1.5])
        lnT = rn_ln(T)
        got = orc.ucb(w, n, lnT, C)
        want = _ucb_r1(w, n, lnT, C)
        assert got == want, (w, n, T, C)
        for name, alt in _alternatives(w, n, lnT, C).items():
            if alt != want:
                differs[name] = differs.get(name, 0) + 1
    for name in _alternatives(1, 2, 1.0, 1.0):
        assert differs.get(name, 0) >= 20, (name, differs)
