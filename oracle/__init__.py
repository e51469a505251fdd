"""CPU oracle — TEST INFRASTRUCTURE ONLY.

ctypes binding of ``oracle/oracle.cpp`` (plain C++, fp64, no shared code with
the CUDA path). Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package. The
product path (``paper_conf_ipps_rockis11_b200``) never does.

Each wrapper cites the PAPER.md passage the C++ function follows; see the
header of oracle.cpp for the pins and DESIGN.md §3 for the readings.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.cpp")
LIB = os.path.join(HERE, "liboracle.so")

POSITION_DTYPE = np.dtype(
    [("black", "<u8"), ("white", "<u8"), ("to_move", "<u4"), ("reserved", "<u4")]
)
N_STATS = 202


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain -O2, no FP contraction, IEEE double)."""
    if not force and os.path.exists(LIB) and os.path.getmtime(LIB) >= os.path.getmtime(SRC):
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [
        "g++", "-std=c++17", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
        "-shared", "-pthread", SRC, "-o", tmp, "-lquadmath",
    ]
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    return LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB)
        u64, u32, i32, dbl = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_double
        vp = ctypes.c_void_p
        L.orc_legal.argtypes = [u64, u64]; L.orc_legal.restype = u64
        L.orc_flips.argtypes = [u64, u64, i32]; L.orc_flips.restype = u64
        L.orc_pick.argtypes = [u64, u32]; L.orc_pick.restype = i32
        L.orc_perft.argtypes = [u64, u64, u32, i32, i32]; L.orc_perft.restype = u64
        L.orc_philox4x32_10.argtypes = [vp, vp, vp]; L.orc_philox4x32_10.restype = None
        L.orc_rng_word.argtypes = [u64, u32, u32, u32, u32]; L.orc_rng_word.restype = u32
        L.orc_playout.argtypes = [vp, u64, u32, u32, u32, vp]; L.orc_playout.restype = i32
        L.orc_playouts.argtypes = [vp, u32, u32, u64, u32, vp, i32]; L.orc_playouts.restype = u64
        L.orc_ln.argtypes = [u64]; L.orc_ln.restype = dbl
        L.orc_ln_table.argtypes = [u32, u32, vp]; L.orc_ln_table.restype = None
        L.orc_ucb.argtypes = [u64, u64, dbl, dbl]; L.orc_ucb.restype = dbl
        L.orc_uct_search.argtypes = [vp, u32, u32, u64, u64, u32, dbl, u64, vp, vp, i32]
        L.orc_uct_search.restype = i32
        L.orc_uct_tree.argtypes = [vp, u32, u64, u64, u32, dbl, u64, vp, vp, vp, vp, vp, vp]
        L.orc_uct_tree.restype = ctypes.c_int64
        L.orc_gen_positions.argtypes = [u64, u32, u32, u32, vp]; L.orc_gen_positions.restype = None
        L.orc_mcts_timed.argtypes = [vp, i32, dbl, u64, dbl, vp, u64]; L.orc_mcts_timed.restype = i32
        L.orc_hybrid_search.argtypes = [vp, u32, u32, u64, u32, u64, u32, dbl, vp, vp, i32]
        L.orc_hybrid_search.restype = i32
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


OPENING_BLACK = 0x0000000810000000
OPENING_WHITE = 0x0000001008000000


def position(black: int, white: int, to_move: int) -> np.ndarray:
    p = np.zeros(1, dtype=POSITION_DTYPE)
    p["black"], p["white"], p["to_move"] = black, white, to_move
    return p


def opening() -> np.ndarray:
    return position(OPENING_BLACK, OPENING_WHITE, 0)


def legal(own: int, opp: int) -> int:
    """Legal-move mask for the side owning `own` (standard Othello, DESIGN R7)."""
    return int(lib().orc_legal(own, opp))


def flips(own: int, opp: int, sq: int) -> int:
    return int(lib().orc_flips(own, opp, sq))


def pick(moves: int, r: int) -> int:
    """k = floor(r*c/2^32), k-th legal square ascending (DESIGN R4)."""
    return int(lib().orc_pick(moves, r))


def perft(black: int, white: int, to_move: int, depth: int, pass_is_ply: bool = True) -> int:
    return int(lib().orc_perft(black, white, to_move, depth, int(pass_is_ply)))


def philox(ctr, key) -> list:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    lib().orc_philox4x32_10(_ptr(c), _ptr(k), _ptr(out))
    return [int(x) for x in out]


def rng_word(seed: int, c0: int, c1: int, c2: int, w: int) -> int:
    return int(lib().orc_rng_word(seed, c0, c1, c2, w))


def playout(pos: np.ndarray, seed: int, c0: int, c1: int, c2: int):
    """One random playout. Returns (+1/0/-1, plies)."""
    plies = ctypes.c_uint32(0)
    r = lib().orc_playout(_ptr(pos), seed, c0, c1, c2, ctypes.addressof(plies))
    return int(r), int(plies.value)


def playouts(leaves: np.ndarray, n_per_leaf: int, seed: int, leaf_id_base: int = 0,
             nthreads: int = 0):
    """Batched playouts: returns (wdl[n,3] uint32, total plies)."""
    leaves = np.ascontiguousarray(leaves, dtype=POSITION_DTYPE)
    n = leaves.shape[0]
    out = np.zeros((n, 3), dtype=np.uint32)
    plies = lib().orc_playouts(_ptr(leaves), n, n_per_leaf, seed, leaf_id_base, _ptr(out), nthreads)
    return out, int(plies)


def ln(x: int) -> float:
    return float(lib().orc_ln(x))


def ln_table(unit: int, K: int) -> np.ndarray:
    out = np.zeros(K + 1, dtype=np.float64)
    lib().orc_ln_table(unit, K, _ptr(out))
    return out


def ucb(w: int, n: int, ln_parent: float, C: float) -> float:
    return float(lib().orc_ucb(w, n, ln_parent, C))


def uct_search(root: np.ndarray, n_trees: int, unit: int, iterations: int, seed: int,
               tree_id_base: int = 0, C: float = 1.0, capacity: int = 0, nthreads: int = 0):
    """UCT search, iteration mode. Returns (stats[202], best, plies);
    stats[197] = plies, stats[198] = sum over iterations of the simulated node's depth,
    [199] expansions refused by a full pool, [200] nodes, [201] node capacity (summed)."""
    stats = np.zeros(N_STATS, dtype=np.int64)
    plies = ctypes.c_uint64(0)
    best = lib().orc_uct_search(_ptr(root), n_trees, unit, iterations, seed, tree_id_base, C,
                                capacity, _ptr(stats), ctypes.addressof(plies), nthreads)
    return stats, int(best), int(plies.value)


def uct_tree(root: np.ndarray, unit: int, iterations: int, seed: int, tree_id: int = 0,
             C: float = 1.0, capacity: int = 0) -> dict:
    cap = capacity if capacity else iterations + 1
    parent = np.zeros(cap, np.int32); move = np.zeros(cap, np.int32)
    n = np.zeros(cap, np.uint64); w = np.zeros(cap, np.uint64); d = np.zeros(cap, np.uint64)
    term = np.zeros(cap, np.uint8)
    cnt = lib().orc_uct_tree(_ptr(root), unit, iterations, seed, tree_id, C, capacity,
                             _ptr(parent), _ptr(move), _ptr(n), _ptr(w), _ptr(d), _ptr(term))
    return dict(parent=parent[:cnt], move=move[:cnt], n=n[:cnt], w=w[:cnt], d=d[:cnt],
                terminal=term[:cnt])


def gen_positions(seed: int, n: int, lmin: int, lmax: int) -> np.ndarray:
    """Synthetic mid-game generator."""
    out = np.zeros(n, dtype=POSITION_DTYPE)
    lib().orc_gen_positions(seed, n, lmin, lmax, _ptr(out))
    return out


def mcts_timed(root: np.ndarray, nthreads: int, budget_ms: float, seed: int, C: float = 1.0,
               max_iterations: int = 0):
    """Root-parallel CPU MCTS opponent, one tree per thread,
    unit 1, grown by the same UCT iteration as uct_search. Stops at budget_ms
    (> 0) and/or max_iterations per tree (> 0); with only the cap it equals
    uct_search(root, nthreads, 1, max_iterations, seed) bit for bit."""
    stats = np.zeros(N_STATS, dtype=np.int64)
    best = lib().orc_mcts_timed(_ptr(root), nthreads, budget_ms, seed, C, _ptr(stats), max_iterations)
    return stats, int(best)


def hybrid_search(root: np.ndarray, n_trees: int, unit: int, steps: int, cpu_iters: int, seed: int,
                  tree_id_base: int = 0, C: float = 1.0, nthreads: int = 0):
    """Hybrid CPU-GPU processing on CPU-managed trees (Fig. 4;
    DESIGN.md R18): per step a GPU leaf of `unit` playouts, cpu_iters one-playout
    CPU iterations on the same tree meanwhile, then the GPU backprop. Returns
    (stats[202], best, cpu) with cpu = dict(iterations, plies, depth_sum, cpu_nodes, gpu_nodes)."""
    stats = np.zeros(N_STATS, dtype=np.int64)
    cpu = np.zeros(5, dtype=np.int64)
    best = lib().orc_hybrid_search(_ptr(root), n_trees, unit, steps, cpu_iters, seed, tree_id_base, C,
                                   _ptr(stats), _ptr(cpu), nthreads)
    return stats, int(best), dict(iterations=int(cpu[0]), plies=int(cpu[1]), depth_sum=int(cpu[2]),
                                  cpu_nodes=int(cpu[3]), gpu_nodes=int(cpu[4]))
