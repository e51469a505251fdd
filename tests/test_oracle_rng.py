"""Pins for the oracle's RNG and move pick (readings R4, R5)."""
import os
import random

import pytest

import reversi_ref as ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _kats():
    rows = []
    with open(os.path.join(GOLDEN, "philox_kat.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                v = [int(x, 16) for x in line.split()]
                rows.append((v[0:4], v[4:6], v[6:10]))
    return rows


@pytest.mark.parametrize("ctr,key,out", _kats())
def test_philox_known_answers(orc, ctr, key, out):
    assert orc.philox(ctr, key) == out


def test_word_layout(orc):
    # word w of stream (c0,c1,c2) with key = seed is output[w % 4] of
    # Philox(counter = (c0, c1, c2, w // 4), key = (seed lo, seed hi)).
    seed = 0x0123456789ABCDEF
    for w in range(16):
        blk = orc.philox([5, 6, 7, w // 4], [seed & 0xFFFFFFFF, seed >> 32])
        assert orc.rng_word(seed, 5, 6, 7, w) == blk[w % 4]


@pytest.mark.parametrize("c", list(range(1, 65)))
def test_pick_bucket_boundaries(orc, c):
    # k = floor(r*c/2^32): bucket k is [ceil(k*2^32/c), ceil((k+1)*2^32/c)),
    # so each bucket holds floor(2^32/c) or ceil(2^32/c) values of r.
    rng = random.Random(c)
    bits = sorted(rng.sample(range(64), c))
    mask = sum(1 << b for b in bits)
    starts = [-(-k * 2**32 // c) for k in range(c + 1)]
    for k in range(c):
        size = starts[k + 1] - starts[k]
        assert size in (2**32 // c, -(-(2**32) // c))
        assert orc.pick(mask, starts[k]) == bits[k]
        assert orc.pick(mask, starts[k + 1] - 1) == bits[k]


def test_pick_kth_bit_random_masks(orc):
    rng = random.Random(1)
    for _ in range(5000):
        mask = rng.getrandbits(64) & rng.getrandbits(64)
        if mask == 0:
            continue
        r = rng.getrandbits(32)
        sq = ref.squares(mask)
        assert orc.pick(mask, r) == sq[(r * len(sq)) >> 32]
