import sys, time
sys.path.insert(0, '.')
import paper_conf_ipps_rockis11_b200 as pkg
from paper_conf_ipps_rockis11_b200 import _native
scheme, it, thr, trees = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
flags = int(sys.argv[5]) if len(sys.argv) > 5 else 0
m = pkg.Mcts(scheme=scheme)
if flags:
    m.L.mcts_destroy(m.h)
    import ctypes
    h = ctypes.c_void_p()
    p = _native.Params(1.0, 1 if scheme == "leaf" else 0, 0, 0, flags)
    assert m.L.mcts_create(None, ctypes.byref(p), ctypes.byref(h)) == 0
    m.h = h
t = time.time()
r = m.search(pkg.opening(), iterations=it, n_trees=trees, threads_per_tree=thr, seed=1000)
print(sys.argv[1:], "ok", round(time.time() - t, 3), r["iterations"], r["best_move"], r["stats"][:65].sum(), flush=True)
