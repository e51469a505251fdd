"""ctypes binding of libmcts.so (include/mcts.h). Argument marshalling only.

Every compute step runs in the CUDA library; if libmcts.so is missing or no
sm_100 device is present the calls raise — there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

POSITION_DTYPE = np.dtype(
    [("black", "<u8"), ("white", "<u8"), ("to_move", "<u4"), ("reserved", "<u4")]
)
WDL_DTYPE = np.dtype([("wins", "<u4"), ("draws", "<u4"), ("losses", "<u4")])
STATS_LEN = 202
MCTS_BLOCK, MCTS_LEAF, MCTS_TREE = 0, 1, 2
MCTS_FLAG_CHECK_TREE = 1

# every symbol include/mcts.h declares
EXPORTS = (
    "mcts_create", "mcts_destroy", "mcts_playouts", "mcts_playouts_async", "mcts_search",
    "mcts_search_async", "mcts_search_hybrid", "mcts_search_hosted", "mcts_playouts_ex_async", "mcts_playouts_host_async", "mcts_best_move", "mcts_perft", "mcts_gen_positions_async", "mcts_ln_table",
    "mcts_status_string", "mcts_last_error", "mcts_version",
)


class MctsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{msg} (status {status})")
        self.status = status


class Position(ctypes.Structure):
    _fields_ = [("black", ctypes.c_uint64), ("white", ctypes.c_uint64),
                ("to_move", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


class Params(ctypes.Structure):
    _fields_ = [("c_uct", ctypes.c_double), ("scheme", ctypes.c_uint32),
                ("max_nodes_per_tree", ctypes.c_uint32), ("device", ctypes.c_int32),
                ("flags", ctypes.c_uint32)]


class Budget(ctypes.Structure):
    _fields_ = [("iterations", ctypes.c_uint64), ("time_ms", ctypes.c_double)]


class RootStats(ctypes.Structure):
    _fields_ = [("visits", ctypes.c_uint64 * 65), ("wins", ctypes.c_uint64 * 65),
                ("draws", ctypes.c_uint64 * 65), ("root_visits", ctypes.c_uint64),
                ("iterations_done", ctypes.c_uint64), ("plies", ctypes.c_uint64),
                ("depth_sum", ctypes.c_uint64), ("refused_expansions", ctypes.c_uint64),
                ("slots_used", ctypes.c_uint64), ("slot_capacity", ctypes.c_uint64),
                ("best_move", ctypes.c_int32), ("reserved", ctypes.c_int32)]


class HostedInfo(ctypes.Structure):
    _fields_ = [("steps", ctypes.c_uint64), ("cpu_iterations", ctypes.c_uint64), ("cpu_plies", ctypes.c_uint64),
                ("cpu_depth_sum", ctypes.c_uint64), ("cpu_nodes", ctypes.c_uint64), ("gpu_nodes", ctypes.c_uint64),
                ("select_ms", ctypes.c_double), ("gpu_ms", ctypes.c_double), ("backprop_ms", ctypes.c_double)]


_lib = None


def load(build_if_missing: bool = True) -> ctypes.CDLL:
    """Load the in-tree libmcts.so (building it with nvcc if it is missing)."""
    global _lib
    if _lib is not None:
        return _lib
    lib_path = os.environ.get("MCTS_LIB", _build.LIB)  # tooling: a tuning variant (tools/build_variants.py)
    if not os.path.exists(lib_path):
        if not build_if_missing or lib_path != _build.LIB:
            raise FileNotFoundError(f"{lib_path} is missing: run __graft_entry__.build()")
        _build.build()
    L = ctypes.CDLL(lib_path)
    vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32
    P = ctypes.POINTER
    L.mcts_create.argtypes = [P(Position), P(Params), P(vp)]
    L.mcts_create.restype = i32
    L.mcts_destroy.argtypes = [vp]
    L.mcts_destroy.restype = None
    L.mcts_playouts.argtypes = [vp, vp, u32, u32, u64, vp, P(u64)]
    L.mcts_playouts.restype = i32
    L.mcts_playouts_async.argtypes = [vp, vp, u32, u32, u64, u32, vp, vp, vp]
    L.mcts_playouts_async.restype = i32
    L.mcts_playouts_ex_async.argtypes = [vp, vp, u32, u32, u64, u32, u32, vp, vp, vp]
    L.mcts_playouts_ex_async.restype = i32
    L.mcts_playouts_host_async.argtypes = [vp, vp, u32, u32, u64, vp, vp, vp]
    L.mcts_playouts_host_async.restype = i32
    L.mcts_search_hosted.argtypes = [vp, P(Position), Budget, u32, u32, u64, u32, u32, P(RootStats), P(HostedInfo)]
    L.mcts_search_hosted.restype = i32
    L.mcts_search.argtypes = [vp, P(Position), Budget, u32, u32, u64, P(RootStats)]
    L.mcts_search.restype = i32
    L.mcts_search_async.argtypes = [vp, P(Position), Budget, u32, u32, u64, u32, vp, vp]
    L.mcts_search_async.restype = i32
    L.mcts_search_hybrid.argtypes = [vp, P(Position), Budget, u32, u32, u64, u32, P(RootStats), P(RootStats)]
    L.mcts_search_hybrid.restype = i32
    L.mcts_perft.argtypes = [vp, P(Position), u32, u32, P(u64)]
    L.mcts_perft.restype = i32
    L.mcts_best_move.argtypes = [vp]
    L.mcts_best_move.restype = i32
    L.mcts_gen_positions_async.argtypes = [vp, u64, u32, u32, u32, vp, vp]
    L.mcts_gen_positions_async.restype = i32
    L.mcts_ln_table.argtypes = [vp, u32, u32, vp]
    L.mcts_ln_table.restype = i32
    L.mcts_status_string.argtypes = [i32]
    L.mcts_status_string.restype = ctypes.c_char_p
    L.mcts_last_error.argtypes = [vp]
    L.mcts_last_error.restype = ctypes.c_char_p
    L.mcts_version.argtypes = []
    L.mcts_version.restype = ctypes.c_char_p
    _lib = L
    return L


def _pos(p) -> Position:
    if isinstance(p, Position):
        return p
    if isinstance(p, np.ndarray):
        p = p.reshape(-1)[0]
        return Position(int(p["black"]), int(p["white"]), int(p["to_move"]), 0)
    black, white, to_move = p
    return Position(black, white, to_move, 0)


def _stream_ptr(stream) -> int:
    if stream is None:
        return 0
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)  # torch.cuda.Stream


class Mcts:
    """One library handle (mcts_create/mcts_destroy) bound to a device."""

    def __init__(self, position=None, c_uct: float = 1.0, scheme: str = "block",
                 max_nodes_per_tree: int = 0, device: int = 0, flags: int = 0):
        self.L = load()
        sch = {"block": MCTS_BLOCK, "leaf": MCTS_LEAF, "tree": MCTS_TREE}[scheme]
        params = Params(c_uct, sch, max_nodes_per_tree, device, flags)
        h = ctypes.c_void_p()
        pp = ctypes.byref(_pos(position)) if position is not None else None
        st = self.L.mcts_create(pp, ctypes.byref(params), ctypes.byref(h))
        if st != 0:
            raise MctsError(st, self.L.mcts_last_error(None).decode())
        self.h = h
        self.scheme = scheme
        self.device = device

    def close(self):
        if getattr(self, "h", None):
            self.L.mcts_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def _check(self, st: int):
        if st != 0:
            raise MctsError(st, self.L.mcts_last_error(self.h).decode())

    # --- mcts_playouts (host buffers) ------------------------------------
    def playouts(self, leaves: np.ndarray, n_per_leaf: int, seed: int):
        """Host-buffer batched playouts. Returns (wdl uint32[n,3], plies)."""
        leaves = np.ascontiguousarray(leaves, dtype=POSITION_DTYPE)
        n = leaves.shape[0]
        out = np.zeros((n, 3), dtype=np.uint32)
        plies = ctypes.c_uint64(0)
        self._check(self.L.mcts_playouts(self.h, leaves.ctypes.data if n else None, n, n_per_leaf,
                                         seed, out.ctypes.data if n else None, ctypes.byref(plies)))
        return out, int(plies.value)

    def playouts_host_ptr(self, leaves_ptr: int, n: int, n_per_leaf: int, seed: int, out_ptr: int):
        """Same call on raw host pointers (e.g. pinned torch tensors)."""
        plies = ctypes.c_uint64(0)
        self._check(self.L.mcts_playouts(self.h, leaves_ptr, n, n_per_leaf, seed, out_ptr,
                                         ctypes.byref(plies)))
        return int(plies.value)

    def playouts_host_async(self, leaves_ptr: int, n: int, n_per_leaf: int, seed: int, out_ptr: int,
                            plies_ptr: int = 0, stream=None):
        """mcts_playouts_host_async on raw pinned host pointers: enqueued on
        `stream`, valid after the stream is synchronised."""
        self._check(self.L.mcts_playouts_host_async(self.h, leaves_ptr, n, n_per_leaf, seed, out_ptr,
                                                    plies_ptr or None, _stream_ptr(stream)))

    # --- mcts_playouts_async (device pointers) ---------------------------
    def playouts_async(self, d_leaves_ptr: int, n_leaves: int, n_per_leaf: int, seed: int,
                       leaf_id_base: int, d_out_ptr: int, d_plies_ptr: int = 0, stream=None):
        self._check(self.L.mcts_playouts_async(self.h, d_leaves_ptr, n_leaves, n_per_leaf, seed,
                                               leaf_id_base, d_out_ptr, d_plies_ptr or None,
                                               _stream_ptr(stream)))

    # --- mcts_search -------------------------------------------------------
    def search(self, root=None, iterations: int = 0, time_ms: float = 0.0, n_trees: int = 1,
               threads_per_tree: int = 64, seed: int = 1) -> dict:
        out = RootStats()
        rp = ctypes.byref(_pos(root)) if root is not None else None
        self._check(self.L.mcts_search(self.h, rp, Budget(iterations, time_ms), n_trees,
                                       threads_per_tree, seed, ctypes.byref(out)))
        return self._stats_dict(out)

    @staticmethod
    def _stats_dict(out: "RootStats") -> dict:
        stats = np.zeros(STATS_LEN, dtype=np.int64)
        stats[0:65] = np.ctypeslib.as_array(out.visits)
        stats[65:130] = np.ctypeslib.as_array(out.wins)
        stats[130:195] = np.ctypeslib.as_array(out.draws)
        stats[195], stats[196], stats[197] = out.root_visits, out.iterations_done, out.plies
        stats[198], stats[199] = out.depth_sum, out.refused_expansions
        stats[200], stats[201] = out.slots_used, out.slot_capacity
        return dict(stats=stats, best_move=int(out.best_move), root_visits=int(out.root_visits),
                    iterations=int(out.iterations_done), plies=int(out.plies),
                    depth_sum=int(out.depth_sum), refused_expansions=int(out.refused_expansions),
                    slots_used=int(out.slots_used), slot_capacity=int(out.slot_capacity))

    def search_hybrid(self, root=None, iterations: int = 0, time_ms: float = 0.0, n_trees: int = 1,
                      threads_per_tree: int = 64, seed: int = 1, cpu_threads: int = 1) -> dict:
        """mcts_search_hybrid: GPU block-parallel trees + host trees, root sums merged."""
        out, cpu = RootStats(), RootStats()
        rp = ctypes.byref(_pos(root)) if root is not None else None
        self._check(self.L.mcts_search_hybrid(self.h, rp, Budget(iterations, time_ms), n_trees,
                                              threads_per_tree, seed, cpu_threads, ctypes.byref(out),
                                              ctypes.byref(cpu)))
        d = self._stats_dict(out)
        d["cpu"] = self._stats_dict(cpu)
        return d

    def search_hosted(self, root=None, iterations: int = 0, time_ms: float = 0.0, n_trees: int = 1,
                      threads_per_tree: int = 64, seed: int = 1, cpu_iters: int = 0, cpu_threads: int = 1) -> dict:
        """mcts_search_hosted: CPU-managed trees, GPU playouts per step, and cpu_iters
        host iterations per tree per step on the same trees (Fig. 4)."""
        out, info = RootStats(), HostedInfo()
        rp = ctypes.byref(_pos(root)) if root is not None else None
        self._check(self.L.mcts_search_hosted(self.h, rp, Budget(iterations, time_ms), n_trees, threads_per_tree,
                                              seed, cpu_iters, cpu_threads, ctypes.byref(out), ctypes.byref(info)))
        d = self._stats_dict(out)
        d["info"] = {k: getattr(info, k) for k, _ in HostedInfo._fields_}
        return d

    def playouts_ex_async(self, d_leaves_ptr: int, n_leaves: int, n_per_leaf: int, seed: int, c0_base: int,
                          c1: int, d_out_ptr: int, d_plies_ptr: int = 0, stream=None):
        self._check(self.L.mcts_playouts_ex_async(self.h, d_leaves_ptr, n_leaves, n_per_leaf, seed, c0_base, c1,
                                                  d_out_ptr, d_plies_ptr or None, _stream_ptr(stream)))

    def search_async(self, root, iterations: int, time_ms: float, n_trees: int,
                     threads_per_tree: int, seed: int, tree_id_base: int, d_stats_ptr: int,
                     stream=None):
        self._check(self.L.mcts_search_async(self.h, ctypes.byref(_pos(root)),
                                             Budget(iterations, time_ms), n_trees,
                                             threads_per_tree, seed, tree_id_base, d_stats_ptr,
                                             _stream_ptr(stream)))

    # --- inputs / tables ---------------------------------------------------
    def gen_positions_async(self, seed: int, n: int, lmin: int, lmax: int, d_out_ptr: int,
                            stream=None):
        self._check(self.L.mcts_gen_positions_async(self.h, seed, n, lmin, lmax, d_out_ptr,
                                                    _stream_ptr(stream)))

    def perft(self, position, depth: int, pass_is_ply: bool = True) -> int:
        out = ctypes.c_uint64(0)
        self._check(self.L.mcts_perft(self.h, ctypes.byref(_pos(position)), depth, int(pass_is_ply),
                                      ctypes.byref(out)))
        return int(out.value)

    def ln_table(self, unit: int, K: int) -> np.ndarray:
        out = np.zeros(K + 1, dtype=np.float64)
        self._check(self.L.mcts_ln_table(self.h, unit, K, out.ctypes.data))
        return out


def best_move(stats: np.ndarray) -> int:
    s = np.ascontiguousarray(stats, dtype=np.int64)
    return int(load().mcts_best_move(s.ctypes.data))


def version() -> str:
    return load().mcts_version().decode()
