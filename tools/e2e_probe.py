"""Where the end-to-end call's time goes (tooling, run under gpurun): wall time
per mcts_playouts call (pinned host buffers, synchronous) for a tiny batch
(the fixed per-call cost), a full-width batch of single playouts and the
configs[1] batch, against the same batch's device-timed kernel."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_rockis11_b200 as pkg
from paper_conf_ipps_rockis11_b200 import device as dev

m = pkg.Mcts(c_uct=1.0, scheme="block")
d_leaves = dev.gen_positions(m, 2, 4096, 20, 40)
h_leaves = torch.empty((4096, 3), dtype=torch.int64).pin_memory()
h_leaves.copy_(d_leaves.cpu())
h_out = torch.empty((4096, 3), dtype=torch.int32).pin_memory()

def wall(n, per, reps=50):
    for _ in range(3):
        m.playouts_host_ptr(h_leaves.data_ptr(), n, per, 2, h_out.data_ptr())
    t0 = time.perf_counter()
    for _ in range(reps):
        m.playouts_host_ptr(h_leaves.data_ptr(), n, per, 2, h_out.data_ptr())
    return (time.perf_counter() - t0) / reps * 1e6

for n, per in [(1, 32), (4096, 1), (4096, 256)]:
    print(f"mcts_playouts {n} x {per}: {wall(n, per):.1f} us per call", flush=True)
out = torch.zeros((4096, 3), dtype=torch.int32, device="cuda")
plies = torch.zeros(1, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
m.playouts_async(d_leaves.data_ptr(), 4096, 256, 2, 0, out.data_ptr(), plies.data_ptr(), s)
torch.cuda.synchronize()
e0.record(s)
for _ in range(20):
    m.playouts_async(d_leaves.data_ptr(), 4096, 256, 2, 0, out.data_ptr(), plies.data_ptr(), s)
e1.record(s)
torch.cuda.synchronize()
print(f"mcts_playouts_async 4096 x 256 back to back: {e0.elapsed_time(e1) / 20 * 1e3:.1f} us per launch (device)")
