"""The host half of mcts_search_hosted (csrc/hosted.cpp: the paper's CPU-managed
trees, and the hybrid CPU iterations of Fig. 4) on CPU: a
test harness (tests/native/hosted_emul.cpp) runs it with the GPU step replaced
by the library's host playouts on the same streams, and the result must equal
the oracle's hybrid search (and, with no CPU iterations, uct_search) bit for
bit — multi-threaded, with the same phase barriers as on the GPU box."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = [os.path.join(HERE, "native", "hosted_emul.cpp"),
       os.path.join(HERE, "..", "paper_conf_ipps_rockis11_b200", "csrc", "hosted.cpp")]


@pytest.fixture(scope="module")
def emul(tmp_path_factory):
    so = str(tmp_path_factory.mktemp("hosted") / "libhosted_emul.so")
    subprocess.check_call(["g++", "-std=c++17", "-O2", "-ffp-contract=off", "-fPIC", "-shared", "-pthread",
                           *SRC, "-o", so])
    L = ctypes.CDLL(so)
    u64, u32 = ctypes.c_uint64, ctypes.c_uint32
    L.hosted_emul.argtypes = [u64, u64, u32, u32, u64, u32, u64, ctypes.c_double, u32, ctypes.c_void_p, u64,
                              ctypes.c_void_p, ctypes.c_void_p]
    L.hosted_emul.restype = ctypes.c_int
    return L


def _own_opp(r):
    r = r[0]
    return (int(r["black"]), int(r["white"])) if r["to_move"] == 0 else (int(r["white"]), int(r["black"]))


@pytest.mark.parametrize("n_trees,unit,steps,cpu_iters,seed,C,lmin,lmax,threads", [
    (1, 64, 100, 0, 1, 1.0, 0, 0, 1),
    (37, 32, 60, 0, 4, 0.25, 20, 40, 5),
    (1, 64, 40, 4, 3, 1.0, 0, 0, 1),
    (24, 32, 30, 3, 5, 0.25, 20, 40, 7),
    (64, 128, 10, 16, 8, 1.0, 30, 45, 16),
    (5, 1, 300, 2, 9, 2.0, 40, 50, 3),
])
def test_hosted_host_half_matches_oracle(orc, emul, n_trees, unit, steps, cpu_iters, seed, C, lmin, lmax, threads):
    root = orc.gen_positions(seed, 1, lmin, lmax) if lmax else orc.opening()
    K = steps * (unit + cpu_iters) + 2
    lnT = orc.ln_table(1, K)
    stats = np.zeros(202, np.int64)
    info = np.zeros(6, np.uint64)
    own, opp = _own_opp(root)
    assert emul.hosted_emul(own, opp, n_trees, unit, steps, cpu_iters, seed, C, threads, lnT.ctypes.data,
                            len(lnT), stats.ctypes.data, info.ctypes.data) == 0
    want, wbest, cpu = orc.hybrid_search(root, n_trees, unit, steps, cpu_iters, seed, C=C)
    assert stats[:201].tolist() == want[:201].tolist()
    assert int(info[0]) == steps and int(info[1]) == cpu["iterations"] and int(info[2]) == cpu["plies"]
    assert int(info[3]) == cpu["depth_sum"] and int(info[4]) == cpu["cpu_nodes"] and int(info[5]) == cpu["gpu_nodes"]
    if cpu_iters == 0:
        u, _, _ = orc.uct_search(root, n_trees, unit, steps, seed, C=C)
        assert stats[:199].tolist() == u[:199].tolist()
