"""Debug helper: leaf-parallel search in a subprocess per case (GPU box only)."""
import sys, time
sys.path.insert(0, '.')
import numpy as np
import paper_conf_ipps_rockis11_b200 as pkg
case = sys.argv[1]
m = pkg.Mcts(scheme="leaf")
root = pkg.opening()
t = time.time()
if case.startswith("it"):
    it, thr = map(int, case[2:].split("x"))
    r = m.search(root, iterations=it, n_trees=1, threads_per_tree=thr, seed=1000)
else:
    ms, thr = case[2:].split("x")
    r = m.search(root, time_ms=float(ms), n_trees=1, threads_per_tree=int(thr), seed=1000)
print(case, "ok", time.time() - t, r["iterations"], r["root_visits"], r["best_move"], flush=True)
