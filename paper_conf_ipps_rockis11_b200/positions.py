"""Host-side position records (layout of mcts_position; no game logic here)."""
from __future__ import annotations

import numpy as np

from ._native import POSITION_DTYPE

OPENING_BLACK = 0x0000000810000000
OPENING_WHITE = 0x0000001008000000
OPENING = (OPENING_BLACK, OPENING_WHITE, 0)


def position(black: int, white: int, to_move: int) -> np.ndarray:
    p = np.zeros(1, dtype=POSITION_DTYPE)
    p["black"], p["white"], p["to_move"] = black, white, to_move
    return p


def opening() -> np.ndarray:
    return position(*OPENING)


def own_opp(p) -> tuple:
    p = p.reshape(-1)[0] if isinstance(p, np.ndarray) and p.shape else p
    if int(p["to_move"]) == 0:
        return int(p["black"]), int(p["white"])
    return int(p["white"]), int(p["black"])
