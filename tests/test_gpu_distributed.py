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
        assert stats[:199] == ostats[:199].tolist()
        assert best == obest
