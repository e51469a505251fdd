"""torch plumbing: device buffers in the layouts the C ABI expects.

positions: int64 tensor [n, 3] (black, white, to_move | reserved << 32) = 24 B
wdl:       int32 tensor [n, 3] (wins, draws, losses)
stats:     int64 tensor [202]  (include/mcts.h MCTS_STATS_LEN)
"""
from __future__ import annotations

import numpy as np
import torch

from ._native import POSITION_DTYPE, STATS_LEN


def positions_to_tensor(p: np.ndarray, device="cuda", pin: bool = False) -> torch.Tensor:
    raw = np.ascontiguousarray(p, dtype=POSITION_DTYPE).view(np.int64).reshape(-1, 3)
    t = torch.from_numpy(raw.copy())
    if device == "cpu":
        return t.pin_memory() if pin else t
    return t.to(device)


def tensor_to_positions(t: torch.Tensor) -> np.ndarray:
    raw = t.detach().to("cpu").contiguous().numpy().astype(np.int64, copy=False)
    return raw.reshape(-1).view(POSITION_DTYPE).copy()


def empty_positions(n: int, device="cuda") -> torch.Tensor:
    return torch.empty((n, 3), dtype=torch.int64, device=device)


def empty_wdl(n: int, device="cuda") -> torch.Tensor:
    return torch.empty((n, 3), dtype=torch.int32, device=device)


def empty_stats(device="cuda") -> torch.Tensor:
    return torch.zeros(STATS_LEN, dtype=torch.int64, device=device)


def gen_positions(mcts, seed: int, n: int, lmin: int, lmax: int, device="cuda") -> torch.Tensor:
    """Synthetic positions generated on the device (mcts_gen_positions_async)."""
    out = empty_positions(n, device)
    mcts.gen_positions_async(seed, n, lmin, lmax, out.data_ptr(), torch.cuda.current_stream())
    return out
