"""Leaf-parallel kernel shakedown (tooling, run under gpurun): one search per
process (so a hang costs one timeout), growing grids, iteration and time mode.
usage: python tools/leaf_debug.py THREADS ITERS [TIME_MS]"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_rockis11_b200 as pkg
import oracle

threads, iters = int(sys.argv[1]), int(sys.argv[2])
ms = float(sys.argv[3]) if len(sys.argv) > 3 else 0.0
m = pkg.Mcts(c_uct=1.0, scheme="leaf", device=0)
root = oracle.gen_positions(15, 1, 30, 40)
t0 = time.time()
try:
    r = m.search(root, iterations=0 if ms else iters, time_ms=ms, n_trees=1, threads_per_tree=threads, seed=4)
    print(f"threads {threads} iters {iters} ms {ms}: ok {time.time() - t0:.2f}s iterations {r['iterations']} "
          f"best {r['best_move']}", flush=True)
    if not ms and threads * iters <= 16384 * 8:
        s, b, _ = oracle.uct_search(root, 1, threads, iters, 4)
        print("  parity", (s[:200] == r["stats"][:200]).all(), flush=True)
except pkg.MctsError as e:
    print(f"threads {threads} iters {iters} ms {ms}: ERROR {e} {time.time() - t0:.2f}s", flush=True)
