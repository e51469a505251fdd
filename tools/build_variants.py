"""Build libmcts.so tuning variants into build/variants/ (see tools/variant_bench.cu)."""
import os, sys, concurrent.futures as cf
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_rockis11_b200 import _build

F = "kFma"
VARIANTS = {
    "base": [],
    "up_all_fma": [f"MCTS_UP_M2={F}", f"MCTS_UP_S1={F}", f"MCTS_UP_S2={F}", f"MCTS_UP_D1={F}", f"MCTS_UP_D2={F}", f"MCTS_UP_FIN={F}"],
    "up_m2_fin": [f"MCTS_UP_M2={F}", f"MCTS_UP_FIN={F}"],
    "up_s1_s2": [f"MCTS_UP_S1={F}", f"MCTS_UP_S2={F}"],
    "up_d1_d2": [f"MCTS_UP_D1={F}", f"MCTS_UP_D2={F}"],
    "up_m2_s1_d1": [f"MCTS_UP_M2={F}", f"MCTS_UP_S1={F}", f"MCTS_UP_D1={F}"],
    "up_s1_d1_fin": [f"MCTS_UP_S1={F}", f"MCTS_UP_D1={F}", f"MCTS_UP_FIN={F}"],
    "up_m2": [f"MCTS_UP_M2={F}"],
    "up_fin": [f"MCTS_UP_FIN={F}"],
    "upd_f": ["MCTS_UPD_F=1"],
    "pick_lut": ["MCTS_PICK_LUT=1"],
    "pick_lut_up_d1_d2": ["MCTS_PICK_LUT=1", f"MCTS_UP_D1={F}", f"MCTS_UP_D2={F}"],
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
