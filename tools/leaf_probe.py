"""Where the leaf-parallel iteration's time goes (tooling, run under gpurun).
Times (CUDA events): one 16384-playout batch from the opening through the playout
kernel, and the leaf/block search in iteration mode, per iteration."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_rockis11_b200 as pkg

def ev_time(fn, reps=10):
    s = torch.cuda.current_stream()
    fn(); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    for _ in range(reps):
        fn()
    e1.record(s); torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps

m = pkg.Mcts(c_uct=1.0, scheme="block")
op = np.zeros(1, dtype=pkg.POSITION_DTYPE); op[0] = pkg.opening()
for nl, per in [(1, 16384), (64, 256), (512, 32), (4096, 256)]:
    leaves = torch.from_numpy(np.repeat(op, nl).view(np.uint8)).cuda()
    out = torch.zeros(nl * 3, dtype=torch.int32, device="cuda")
    plies = torch.zeros(1, dtype=torch.int64, device="cuda")
    s = torch.cuda.current_stream()
    t = ev_time(lambda: m.playouts_async(leaves.data_ptr(), nl, per, 7, 0, out.data_ptr(), plies.data_ptr(), s))
    print(f"playouts opening {nl}x{per}: {t*1e3:.1f} us/launch, {nl*per/t/1e3:.3e} playouts/s", flush=True)
for scheme, trees, thr in [("leaf", 1, 16384), ("block", 1184, 128)]:
    mm = pkg.Mcts(c_uct=1.0, scheme=scheme)
    for iters in (50, 200):
        st = torch.zeros(pkg.STATS_LEN, dtype=torch.int64, device="cuda")
        s = torch.cuda.current_stream()
        t = ev_time(lambda: mm.search_async(pkg.opening(), iters, 0.0, trees, thr, 1, 0, st.data_ptr(), s), reps=3)
        print(f"{scheme} search {trees}x{thr} {iters} iterations: {t:.2f} ms, {t/iters*1e3:.1f} us/iteration", flush=True)
    mm.close()
