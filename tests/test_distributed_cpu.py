"""World-size-2 gloo tests of the multi-GPU host logic (CPU, no GPU needed).

Each rank computes its trees' root statistics (the oracle stands in for the
per-rank GPU search here), the package's merge_root_stats does the one
allreduce, and the merged vector must equal a single search over all trees
(exact integer identity).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ipps_rockis11_b200.distributed import (
            best_move_from, leaf_range, merge_root_stats, tree_id_base)
        root = oracle.gen_positions(21, 1, 20, 30)
        n = 5
        local, _, _ = oracle.uct_search(root, n, 32, 12, seed=4, tree_id_base=tree_id_base(rank, n))
        st = torch.from_numpy(local.astype(np.int64))  # MCTS_STATS_LEN layout (202)
        merge_root_stats(st)
        # leaf-range sharding of a playout batch (no collective on the data path)
        leaves = oracle.gen_positions(2, 11, 20, 40)
        a, b = leaf_range(rank, world, len(leaves))
        wdl, _ = oracle.playouts(leaves[a:b], 8, seed=5, leaf_id_base=a)
        q.put((rank, st.numpy().copy(), best_move_from(st), a, b, wdl))
    finally:
        dist.destroy_process_group()


def test_two_rank_root_merge_identity():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle
    root = oracle.gen_positions(21, 1, 20, 30)
    full, best, _ = oracle.uct_search(root, 5 * world, 32, 12, seed=4)
    for rank, st, bm, a, b, wdl in res:
        assert st.tolist() == full.tolist()
        assert bm == best
    # the shards tile the batch and reproduce one call
    leaves = oracle.gen_positions(2, 11, 20, 40)
    whole, _ = oracle.playouts(leaves, 8, seed=5)
    got = np.zeros_like(whole)
    for rank, st, bm, a, b, wdl in res:
        got[a:b] = wdl
    assert (got == whole).all()


def test_leaf_range_partition():
    from paper_conf_ipps_rockis11_b200.distributed import leaf_range
    for n in [0, 1, 7, 4096, 4097]:
        for world in [1, 2, 3, 8]:
            spans = [leaf_range(r, world, n) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (a0, b0), (a1, b1) in zip(spans, spans[1:]):
                assert b0 == a1
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1


def test_merge_is_noop_single_process():
    from paper_conf_ipps_rockis11_b200.distributed import merge_root_stats, best_move_from
    t = torch.arange(202, dtype=torch.int64)
    assert torch.equal(merge_root_stats(t.clone()), t)
    s = np.zeros(202, dtype=np.int64)
    assert best_move_from(s) == -1
