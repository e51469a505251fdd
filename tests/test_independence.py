"""The oracle and the CUDA path share no code (task contract ③): nothing under
oracle/ includes or imports the package or the C ABI header, and nothing in the
package (kernels, host code, binding) includes or imports the oracle. Only
tests/, bench.py's CPU legs and __graft_entry__.smoke() may use the oracle."""
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ipps_rockis11_b200")
ORACLE = os.path.join(ROOT, "oracle")
SRC_EXT = (".py", ".cu", ".cuh", ".cpp", ".h", ".c")


def _sources(d):
    for base, _, files in os.walk(d):
        for f in files:
            if f.endswith(SRC_EXT):
                yield os.path.join(base, f)


def _code_lines(path):
    for line in open(path, encoding="utf-8", errors="replace"):
        s = line.strip()
        if s.startswith(("#include", "import ", "from ")):
            yield s


def test_oracle_uses_nothing_from_the_cuda_path():
    bad = []
    for p in _sources(ORACLE):
        for s in _code_lines(p):
            if re.search(r"paper_conf_ipps_rockis11_b200|csrc|include/mcts\.h|\"mcts\.h\"", s):
                bad.append((os.path.relpath(p, ROOT), s))
    assert not bad, bad


def test_cuda_path_uses_nothing_from_the_oracle():
    bad = []
    for p in _sources(PKG):
        for s in _code_lines(p):
            if re.search(r"\boracle\b", s):
                bad.append((os.path.relpath(p, ROOT), s))
    assert not bad, bad
