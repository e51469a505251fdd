"""Build libmcts.so tuning variants into build/variants/ (see tools/variant_bench.cu).
Knobs: MCTS_PICK_LUT, MCTS_UPD_F, MCTS_EAST_F (reversi_device.cuh),
MCTS_PLAYOUT_THREADS, MCTS_PLAYOUT_MINB (kernels.cuh)."""
import os, sys, concurrent.futures as cf
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis11_b200 import _build

VARIANTS = {
    "base": [],
    "no_lut": ["MCTS_PICK_LUT=0"],
    "no_upd_f": ["MCTS_UPD_F=0"],
    "no_east_f": ["MCTS_EAST_F=0"],
    "t128": ["MCTS_PLAYOUT_THREADS=128"],
    "flip_k0": ["MCTS_FLIP_K=0"],
    "split0": ["MCTS_SPLIT=0"],
    "minb4": ["MCTS_PLAYOUT_MINB=4"],
    "bitlut0": ["MCTS_BIT_LUT=0"],
    "xy0": ["MCTS_FLIP_XY=0"],
    "pred0": ["MCTS_PRED_FLIP=0"],
    "pred2": ["MCTS_PRED_FLIP=2"],
    "pshl": ["MCTS_PICK_SHL=1"],
    "map3": ["MCTS_MAPBACK3=1"],
    "rmb": ["MCTS_RM_BREV=1"],
    "nw0": ["MCTS_NW=0"],
    "zt0": ["MCTS_ZT=0"],
    "hxp0": ["MCTS_HXP=0"],
    "old3": ["MCTS_NW=0", "MCTS_ZT=0", "MCTS_HXP=0"],
    "minb5": ["MCTS_PLAYOUT_MINB=5"],
    "t128m9": ["MCTS_PLAYOUT_THREADS=128", "MCTS_PLAYOUT_MINB=9"],
    "t128m10": ["MCTS_PLAYOUT_THREADS=128", "MCTS_PLAYOUT_MINB=10"],
    "t128m11": ["MCTS_PLAYOUT_THREADS=128", "MCTS_PLAYOUT_MINB=11"],
    "t64m20": ["MCTS_PLAYOUT_THREADS=64", "MCTS_PLAYOUT_MINB=20"],
    "leafprobe": ["MCTS_LEAF_PROBE=1"],
    "bounds": ["MCTS_DEBUG_BOUNDS=1"],
    "pair": ["MCTS_PAIR=1"],
    "pair_m3": ["MCTS_PAIR=1", "MCTS_PLAYOUT_MINB=3"],
    "pair_t128m5": ["MCTS_PAIR=1", "MCTS_PLAYOUT_THREADS=128", "MCTS_PLAYOUT_MINB=5"],
}

if __name__ == "__main__":
    names = sys.argv[1:] or list(VARIANTS)
    d = os.path.join(_build.ROOT, "build", "variants")
    os.makedirs(d, exist_ok=True)
    for f in os.listdir(d):
        os.remove(os.path.join(d, f))
    def one(n):
        out = os.path.join(d, f"libmcts_{n}.so")
        _build.build(out=out, defines=VARIANTS[n])
        return out
    with cf.ThreadPoolExecutor(4) as ex:
        for p in ex.map(one, names):
            print(p)
