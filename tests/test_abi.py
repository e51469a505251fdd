"""CPU-side checks of the C ABI: libmcts.so builds, loads, exports every symbol
include/mcts.h declares, and fails loudly (no CPU fallback) without a GPU."""
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    src = open(os.path.join(ROOT, "include", "mcts.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(mcts_[a-z_]+)\s*\(", src)
    return sorted(set(names))


def test_header_exports_match_binding():
    import paper_conf_ipps_rockis11_b200 as pkg
    assert sorted(pkg.EXPORTS) == header_functions()


def test_library_loads_and_exports_every_symbol():
    import ctypes
    import paper_conf_ipps_rockis11_b200 as pkg
    lib = pkg.load()
    for name in header_functions():
        assert hasattr(lib, name), name
    assert b"sm_100a" in lib.mcts_version()
    assert lib.mcts_status_string(-5) == b"MCTS_E_NO_DEVICE"
    assert lib.mcts_best_move(None) == -1


def test_sass_is_sm100a():
    import subprocess
    import paper_conf_ipps_rockis11_b200 as pkg
    from paper_conf_ipps_rockis11_b200 import _build
    pkg.load()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _build.LIB],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_best_move_host_helper():
    import numpy as np
    import paper_conf_ipps_rockis11_b200 as pkg
    s = np.zeros(pkg.STATS_LEN, dtype=np.int64)
    assert pkg.best_move(s) == -1
    s[[19, 26, 37]] = [5, 9, 9]
    assert pkg.best_move(s) == 26
    s[64] = 10
    assert pkg.best_move(s) == 64


def test_no_cpu_fallback_without_gpu():
    import torch
    import paper_conf_ipps_rockis11_b200 as pkg
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(pkg.MctsError) as ei:
        pkg.Mcts()
    assert ei.value.status == -5  # MCTS_E_NO_DEVICE


def test_missing_library_fails_loudly(tmp_path):
    """No CPU fallback: with the CUDA library missing the binding raises."""
    import subprocess, sys
    code = ("import paper_conf_ipps_rockis11_b200 as pkg\n"
            "try:\n    pkg.Mcts()\nexcept FileNotFoundError as e:\n    print('raised', e)\n")
    env = dict(os.environ, MCTS_LIB=str(tmp_path / "missing.so"))
    out = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=120,
                         cwd=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    assert out.stdout.startswith("raised"), out.stdout + out.stderr
