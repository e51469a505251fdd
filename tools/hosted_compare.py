"""Hosted-search (CPU-managed trees) speed of several library
builds side by side (tooling, run under gpurun): python tools/hosted_compare.py
LIB [LIB ...] — each in its own process (MCTS_LIB): configs[2] shape from the
opening, 500 ms, 16 host threads, GPU-only and with CPU iterations."""
import os, subprocess, sys

CHILD = r'''
import os, sys
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_rockis11_b200 as pkg
m = pkg.Mcts(c_uct=1.0, scheme="block", device=0)
root = pkg.opening()
m.search_hosted(root, time_ms=100.0, n_trees=1184, threads_per_tree=128, seed=1, cpu_iters=0, cpu_threads=16)
out = []
for cpu in (0, 1):
    r = m.search_hosted(root, time_ms=500.0, n_trees=1184, threads_per_tree=128, seed=1, cpu_iters=cpu, cpu_threads=16)
    i = r["info"]
    out.append("cpu_iters=%d steps %d select_ms %.1f gpu_ms %.1f" % (cpu, i["steps"], i["select_ms"], i["gpu_ms"]))
print(os.path.basename(os.environ["MCTS_LIB"]), " | ".join(out))
'''
for lib in sys.argv[1:]:
    env = dict(os.environ, MCTS_LIB=os.path.abspath(lib))
    out = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=300)
    print(out.stdout.strip() or out.stderr[-800:], flush=True)
