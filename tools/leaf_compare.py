"""Leaf-parallel kernel variants side by side (tooling, run under gpurun):
python tools/leaf_compare.py LIB [LIB ...] — each in its own process (MCTS_LIB),
configs[3] (1 tree x 16384 threads) from the opening, 500 ms time mode x 3 and
200 iterations in iteration mode (CUDA events); then configs[2] block search
(1184 x 128) the same way (iterations per tree)."""
import os, subprocess, sys

CHILD = r'''
import os, sys, time
sys.path.insert(0, os.getcwd())
import torch, paper_conf_ipps_rockis11_b200 as pkg
m = pkg.Mcts(c_uct=1.0, scheme="leaf", device=0)
root = pkg.opening()
its = []
for _ in range(3):
    r = m.search(root, time_ms=500.0, n_trees=1, threads_per_tree=16384, seed=7)
    its.append(r["iterations"])
st = torch.zeros(pkg.STATS_LEN, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
m.search_async(root, 200, 0.0, 1, 16384, 7, 0, st.data_ptr(), s); torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(s); m.search_async(root, 200, 0.0, 1, 16384, 7, 0, st.data_ptr(), s); e1.record(s); torch.cuda.synchronize()
print(os.environ["MCTS_LIB"], "leaf time-mode iterations/500ms", its, "iteration mode us/iter %.1f" % (e0.elapsed_time(e1) * 1e3 / 200), flush=True)
b = pkg.Mcts(c_uct=1.0, scheme="block", device=0)
its = []
for _ in range(3):
    r = b.search(root, time_ms=500.0, n_trees=1184, threads_per_tree=128, seed=7)
    its.append(round(r["iterations"] / 1184, 1))
b.search_async(root, 200, 0.0, 1184, 128, 7, 0, st.data_ptr(), s); torch.cuda.synchronize()
e0.record(s); b.search_async(root, 200, 0.0, 1184, 128, 7, 0, st.data_ptr(), s); e1.record(s); torch.cuda.synchronize()
print(os.environ["MCTS_LIB"], "block time-mode iterations/tree/500ms", its, "iteration mode us/iter %.1f" % (e0.elapsed_time(e1) * 1e3 / 200), flush=True)
'''
for lib in sys.argv[1:]:
    env = dict(os.environ, MCTS_LIB=os.path.abspath(lib))
    out = subprocess.run([sys.executable, "-c", CHILD], env=env, capture_output=True, text=True, timeout=120)
    print(out.stdout.strip() or out.stderr[-500:], flush=True)
