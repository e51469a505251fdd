"""Host-side helpers of bench.py (no GPU): clock-record parsing and the integer
roofline denominator."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_clocks_summary(tmp_path):
    p = tmp_path / "clk.csv"
    p.write_text(
        "0, 1965, 1965, 700.1, 0x0, Not Active, Not Active, Not Active, Not Active\n"
        "1, 1000, 1965, 300.0, 0x0, Not Active, Not Active, Not Active, Not Active\n"
        "0, 1950, 1965, 720.4, 0x4, Not Active, Not Active, Not Active, Active\n"
        "0, 1965, 1965, 710.0, 0x0, Not Active, Not Active, Not Active, Not Active\n")
    s = bench.clocks_summary(str(p), 0)
    assert s["samples"] == 3 and s["sm_mhz"] == 1965.0 and s["sm_max_mhz"] == 1965.0
    assert s["reasons"] == ["sw_power_cap"]
    assert bench.clocks_summary(str(tmp_path / "missing.csv"), 0)["samples"] == 0


def test_integer_peak_uses_measured_file():
    peak, basis, alu = bench.integer_peak()
    ip = json.load(open(os.path.join(ROOT, "profiles", "int_peaks.json")))
    assert peak == ip["lop3_imad_mixed"] and alu == ip["lop3_alu"]
    assert "measured" in basis
    # the measured mixed rate cannot exceed the issue-slot count at the max clock
    assert peak <= 148 * 4 * 32 * 1965e6 * 1.001
