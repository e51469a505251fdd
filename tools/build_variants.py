"""Build libmcts.so tuning variants into build/variants/ (see tools/variant_bench.cu)."""
import os, sys, concurrent.futures as cf
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis11_b200 import _build

VARIANTS = {
    "base": [],
    "east_plain": ["MCTS_EAST_PLAIN=1"],
    "no_east": ["MCTS_MG_EAST_CARRY=0"],
    "rng_select": ["MCTS_RNG_SELECT=1"],
    "minb10": ["MCTS_PLAYOUT_MINB=10"],
    "minb12": ["MCTS_PLAYOUT_MINB=12"],
    "minb8": ["MCTS_PLAYOUT_MINB=8"],
    "t256": ["MCTS_PLAYOUT_THREADS=256"],
    "t64_minb16": ["MCTS_PLAYOUT_THREADS=64", "MCTS_PLAYOUT_MINB=16"],
    "right_mix": ["MCTS_MG_RIGHT=kMix"],
    "left_fma": ["MCTS_MG_LEFT=kFma"],
    "upd_f": ["MCTS_UPD_F=1"],
}

if __name__ == "__main__":
    names = sys.argv[1:] or list(VARIANTS)
    os.makedirs(os.path.join(_build.ROOT, "build", "variants"), exist_ok=True)
    for f in os.listdir(os.path.join(_build.ROOT, "build", "variants")):
        os.remove(os.path.join(_build.ROOT, "build", "variants", f))
    def one(n):
        out = os.path.join(_build.ROOT, "build", "variants", f"libmcts_{n}.so")
        _build.build(out=out, defines=VARIANTS[n])
        return out
    with cf.ThreadPoolExecutor(4) as ex:
        for p in ex.map(one, names):
            print(p)
