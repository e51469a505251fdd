"""Multi-rank search on one GPU (gloo stands in for NCCL; every rank uses cuda:0):
rank r searches trees [r*n, (r+1)*n) through distributed.search and the one
allreduce must reproduce a single search over all k*n trees bit for bit, which
is the oracle's result."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, q, scheme, n_trees):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_rockis11_b200 as pkg
        from paper_conf_ipps_rockis11_b200 import distributed
        torch.cuda.set_device(0)
        m = pkg.Mcts(c_uct=1.0, scheme=scheme, device=0)
        root = np.zeros(1, dtype=pkg.POSITION_DTYPE)
        root["black"], root["white"], root["to_move"] = 0x0000000810000000, 0x0000001008000000, 0
        r = distributed.search(m, root, n_trees=n_trees, threads_per_tree=64, seed=11, iterations=12)
        q.put((rank, r["stats"].tolist(), r["best_move"]))
        m.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("scheme,n_trees", [("block", 24), ("tree", 1)])
def test_two_rank_allreduce_matches_single_search(orc, scheme, n_trees):
    """block: 24 trees per rank; tree: one one-worker shared tree per rank
    (c0 = rank), i.e. root parallelism across ranks over tree-parallel GPUs."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_rank, args=(r, world, port, q, scheme, n_trees)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    ostats, obest, _ = orc.uct_search(orc.opening(), n_trees * world, 64, 12, 11)
    for rank, stats, best in res:
        assert stats[:200] == ostats[:200].tolist()
        assert best == obest


def _nccl_world1(port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda:0"))
    try:
        import paper_conf_ipps_rockis11_b200 as pkg
        from paper_conf_ipps_rockis11_b200 import distributed
        m = pkg.Mcts(c_uct=1.0, scheme="block", device=0)
        root = np.zeros(1, dtype=pkg.POSITION_DTYPE)
        root["black"], root["white"], root["to_move"] = 0x0000000810000000, 0x0000001008000000, 0
        s = torch.cuda.Stream()
        r = distributed.search(m, root, n_trees=16, threads_per_tree=64, seed=11, iterations=30, stream=s,
                               force_collective=True)
        q.put((dist.get_backend(), r["stats"].tolist(), r["best_move"]))
        m.close()
    finally:
        dist.destroy_process_group()


def test_nccl_allreduce_path_world1(orc):
    """The NCCL branch of the one collective (merge_root_stats) executed on a
    B200: a world-1 NCCL group with the allreduce forced, on a side stream;
    the sum over one rank is the rank's own search = the oracle's."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_world1, args=(_free_port(), q))
    p.start()
    backend, stats, best = q.get(timeout=600)
    p.join(timeout=120)
    assert p.exitcode == 0 and backend == "nccl"
    ostats, obest, _ = orc.uct_search(orc.opening(), 16, 64, 30, 11)
    assert stats[:200] == ostats[:200].tolist() and best == obest


def test_bench_gpus2_self_launch():
    """`python bench.py --gpus 2` without torchrun launches two ranks itself
    (gloo on one GPU here: BENCH_SAME_DEVICE / BENCH_BACKEND are the
    single-GPU test hooks) and reports n_gpus 2 with a merged search root."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, BENCH_SAME_DEVICE="1", BENCH_BACKEND="gloo")
    env.pop("WORLD_SIZE", None)
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "3",
                          "--warmup", "3", "--no-cpu", "--search-ms", "50"],
                         capture_output=True, text=True, timeout=900, cwd=root, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["search"]["allreduce"] is True
    assert d["search"]["iterations_per_tree"] > 0
    assert out.stderr.count("process group: backend=gloo") == 2
